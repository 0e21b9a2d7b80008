#!/bin/bash
# r02 GPU session 3: ring A/B variants, phase traces, ncu of the ring (base + bulk-prefetch variant).
TAG=${1:-r02c}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
timeout 300 python -m pytest tests/test_gpu_ring_bench.py tests/test_gpu_ring.py -m gpu -q -x > gpurun_out/${TAG}_pytest_ring.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_ring.log
timeout 900 python tools/ring_ab.py run > gpurun_out/${TAG}_ring_ab.txt 2>&1; cat gpurun_out/${TAG}_ring_ab.txt
timeout 300 python tools/ring_ab.py trace > gpurun_out/${TAG}_ring_trace.txt 2>&1; cat gpurun_out/${TAG}_ring_trace.txt
for V in base bulkpf; do
  LIBENV=""; [ "$V" != base ] && LIBENV="NBA_IPSEC_LIB=build/variants/$V.so"
  env $LIBENV timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_fused_ring' \
      -c 1 -o gpurun_out/prof_${TAG}_ring_c2_$V -f python tools/run_batches.py --config 2 --batches 1 --ring 4 > gpurun_out/ncu_${TAG}_$V.log 2>&1
  echo "ncu $V rc=$?"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 22 --warmup 3 --no-sweep --no-cpu --no-inbound --no-alb > /dev/null 2>&1
echo "launches rc=$?"
