#!/bin/bash
# One gpurun session: build, tests, bench, launch list, ncu full captures, microbench.
# usage: tools/gpu_round.sh TAG [full]
TAG=${1:-r01}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_eurosys_kimjlmsm15_b200/csrc -I include \
     -o build/microbench tools/microbench.cu 2>/dev/null && build/microbench > gpurun_out/microbench_$TAG.json
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi_$TAG.txt
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 22 --warmup 3 --no-sweep --no-cpu --no-inbound --no-alb > /dev/null 2>&1
if [ "$2" == "full" ]; then
  for C in 2 3 4; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_(fused|prologue)' \
      -s 3 -c 1 -o gpurun_out/prof_${TAG}_c$C -f python tools/run_batches.py --config $C --batches 5 > gpurun_out/ncu_${TAG}_c$C.log 2>&1
  done
  for C in 2 3 4; do   # the persistent ring kernel: one run of 4 batch slots (4 batches)
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_fused_ring' \
      -c 1 -o gpurun_out/prof_${TAG}_ring_c$C -f python tools/run_batches.py --config $C --batches 1 --ring 4 > gpurun_out/ncu_${TAG}_ring_c$C.log 2>&1
  done
  for C in 2 3 4; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_in_' \
      -s 2 -c 1 -o gpurun_out/prof_${TAG}_in_c$C -f python tools/run_inbound.py --config $C --batches 3 > gpurun_out/ncu_${TAG}_in_c$C.log 2>&1
  done
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_(aes|hmac|gather|scatter)' \
      -s 4 -c 4 -o gpurun_out/prof_${TAG}_unfused_c3 -f python tools/run_batches.py --config 3 --batches 3 --pipeline 1 > /dev/null 2>&1
fi
ls -la gpurun_out | tail -20
