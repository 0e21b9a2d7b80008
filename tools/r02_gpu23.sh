#!/bin/bash
TAG=${1:-r02ab}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
timeout 600 python tools/inbound_ab.py 64 1514 > gpurun_out/${TAG}_inbound.txt 2>&1; cat gpurun_out/${TAG}_inbound.txt
AB_PASSES=2 timeout 900 python tools/ring_ab.py run 64 1514 imix > gpurun_out/${TAG}_ab.txt 2>&1; cat gpurun_out/${TAG}_ab.txt
