#!/bin/bash
TAG=${1:-r02z}
mkdir -p gpurun_out/sanitizer
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests/test_gpu_inbound.py tests/test_gpu_ring.py -m gpu -q -x > gpurun_out/${TAG}_pytest_in.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_in.log
timeout 600 python tools/inbound_ab.py > gpurun_out/${TAG}_inbound_ab.txt 2>&1; cat gpurun_out/${TAG}_inbound_ab.txt
NBA_IPSEC_LIB=build/variants/nolane.so timeout 600 python tools/inbound_ab.py > gpurun_out/${TAG}_inbound_ab_nolane.txt 2>&1; cat gpurun_out/${TAG}_inbound_ab_nolane.txt
for tool in racecheck synccheck memcheck; do
  timeout 420 compute-sanitizer --tool $tool python tools/sanitize_cases.py inbound > gpurun_out/sanitizer/${TAG}_${tool}_inbound.txt 2>&1
  echo "$tool inbound rc=$? $(grep -E 'SUMMARY|result ==' gpurun_out/sanitizer/${TAG}_${tool}_inbound.txt | tr '\n' ' ')"
done
