#!/bin/bash
# ncu --set full of the pipelined inbound ring (forced) and the outbound ring at IMIX (profiles/r02be_imix_balance.md)
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
NBA_IPSEC_RING_IN_PIPE=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_in_fused_ring_pipe' -c 1 -o gpurun_out/prof_r02be_inpipe_c4 -f python tools/run_inbound.py --config 4 --batches 4 --ring > gpurun_out/r02be_prof.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_fused_ring_pipe' -c 1 -o gpurun_out/prof_r02be_ring_c4 -f python tools/run_batches.py --config 4 --batches 4 --ring 4 >> gpurun_out/r02be_prof.log 2>&1
tail -3 gpurun_out/r02be_prof.log
