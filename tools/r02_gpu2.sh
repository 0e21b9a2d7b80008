#!/bin/bash
# r02 GPU session 2: tests, smoke, ring A/B (TMA staging), ring phase trace, sanitizers.
TAG=${1:-r02b}
mkdir -p gpurun_out/sanitizer
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log
timeout 600 python tools/ring_ab.py run > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
timeout 300 python tools/ring_ab.py trace > gpurun_out/${TAG}_ring_trace.txt 2>&1; cat gpurun_out/${TAG}_ring_trace.txt
for tool in memcheck racecheck synccheck initcheck; do
  for c in c1 ring_small inbound c4 ring64; do
    timeout 420 compute-sanitizer --tool $tool python tools/sanitize_cases.py $c > gpurun_out/sanitizer/${TAG}_${tool}_${c}.txt 2>&1
    echo "$tool $c rc=$? $(grep -E 'SUMMARY|result ==' gpurun_out/sanitizer/${TAG}_${tool}_${c}.txt | tr '\n' ' ')"
  done
done
