#!/bin/bash
# inbound: GPU tests, ring forms side by side, phase trace of the pipelined ring
TAG=${1:-inb}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "inbound or replay" > gpurun_out/${TAG}_pytest_in.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_in.log
timeout 600 python tools/inbound_ab.py 64 1514 imix > gpurun_out/${TAG}_inbound.txt 2>&1; cat gpurun_out/${TAG}_inbound.txt
timeout 300 python tools/inbound_ab.py trace 64 imix > gpurun_out/${TAG}_in_trace.txt 2>&1; cat gpurun_out/${TAG}_in_trace.txt
for V in $VARIANTS; do  # (NBA_IPSEC_LIB variants, pipelined form forced)
  NBA_IPSEC_LIB=build/variants/$V.so NBA_IPSEC_RING_IN_PIPE=1 timeout 600 python tools/inbound_ab.py 64 1514 imix 2>&1 | grep pipelined | sed "s/^/$V /" | tee gpurun_out/${TAG}_inbound_$V.txt
done
