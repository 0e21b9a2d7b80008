#!/bin/bash
TAG=${1:-r02z}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
mkdir -p build/v2 && mv build/variants/nolane.so build/v2/
AB_PASSES=2 timeout 900 python tools/ring_ab.py run > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
mv build/v2/nolane.so build/variants/
bash tools/r02_gpu20.sh $TAG
