#!/bin/bash
TAG=${1:-r02y}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
AB_PASSES=3 timeout 900 python tools/ring_ab.py run > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
