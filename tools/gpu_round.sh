#!/bin/bash
# One gpurun session: tests, bench, launch list, ncu full captures.
# usage: tools/gpu_round.sh TAG [full]
TAG=${1:-r01}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi_$TAG.txt
timeout 900 python bench.py --steps 50 --warmup 10 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-sweep --no-cpu > /dev/null 2>&1
if [ "$2" == "full" ]; then
  for C in 2 3 4; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_(aes|hmac|gather|scatter|prologue|fused)' \
      -s 5 -c 6 -o gpurun_out/prof_${TAG}_c$C -f python tools/run_batches.py --config $C --batches 3 > gpurun_out/ncu_${TAG}_c$C.log 2>&1
  done
fi
ls -la gpurun_out
