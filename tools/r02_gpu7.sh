#!/bin/bash
TAG=${1:-r02e}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python tools/ring_ab.py run > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
timeout 300 python tools/ring_ab.py trace > gpurun_out/${TAG}_ring_trace.txt 2>&1; cat gpurun_out/${TAG}_ring_trace.txt
