#!/bin/bash
# r02 final-state session: tests, smoke, bench (default run as the driver does), launch list,
# ncu captures of the ring (64 B / 1514 B / IMIX) and the inbound kernel, microbench, sanitizers.
TAG=${1:-r02j}
mkdir -p gpurun_out/sanitizer
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_eurosys_kimjlmsm15_b200/csrc -I include \
     -o build/microbench tools/microbench.cu 2>/dev/null && timeout 120 build/microbench > gpurun_out/microbench_$TAG.json
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/${TAG}_clocks.csv &
SMI=$!
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_${TAG}_s20.json 2> gpurun_out/bench_${TAG}_s20.err
timeout 900 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
kill $SMI
tail -c 700 gpurun_out/bench_${TAG}.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 22 --warmup 3 --no-sweep --no-cpu --no-inbound --no-alb > /dev/null 2>&1
for C in 2 3 4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_fused_ring' \
      -c 1 -o gpurun_out/prof_${TAG}_ring_c$C -f python tools/run_batches.py --config $C --batches 1 --ring 6 > /dev/null 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_in_' \
      -s 2 -c 1 -o gpurun_out/prof_${TAG}_in_c$C -f python tools/run_inbound.py --config $C --batches 3 > /dev/null 2>&1
done
ls gpurun_out/ | grep $TAG | head -40
# compute-sanitizer is closed on this GPU pool (runs under it left GPUs needing a reset);
# the cases stay in tools/sanitize_cases.py for a pool where it is open
