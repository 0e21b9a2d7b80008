#!/bin/bash
TAG=${1:-r02v}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests/test_gpu_ring.py tests/test_gpu_inbound.py -m gpu -q -x > gpurun_out/${TAG}_pytest_in.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_in.log
timeout 600 python tools/inbound_ab.py > gpurun_out/${TAG}_inbound_ab.txt 2>&1; cat gpurun_out/${TAG}_inbound_ab.txt
for M in bench out128 out128in128; do
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_fused_ring --csv python tools/traffic_probe.py $M > gpurun_out/${TAG}_traffic_$M.csv 2>&1
  grep -E "dram__bytes|duration" gpurun_out/${TAG}_traffic_$M.csv | tr '\n' ' '; echo " <- $M"
done
