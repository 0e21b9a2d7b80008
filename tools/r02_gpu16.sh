#!/bin/bash
TAG=${1:-r02s}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
timeout 300 python tools/inbound_ab.py trace > gpurun_out/${TAG}_inbound_trace.txt 2>&1; cat gpurun_out/${TAG}_inbound_trace.txt
timeout 300 python tools/ring_ab.py trace > gpurun_out/${TAG}_ring_trace.txt 2>&1; cat gpurun_out/${TAG}_ring_trace.txt
