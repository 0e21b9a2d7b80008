#!/bin/bash
TAG=${1:-r02x}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests/test_gpu_ring_bench.py tests/test_gpu_ring.py -m gpu -q -x > gpurun_out/${TAG}_pytest_ring.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_ring.log
AB_PASSES=2 timeout 900 python tools/ring_ab.py run 64 128 1514 imix > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
