#!/bin/bash
mkdir -p gpurun_out/sanitizer
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
python -c "import oracle; oracle.build()"
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/s9_pytest_gpu.log 2>&1; tail -3 gpurun_out/s9_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s9_smoke.log 2>&1; echo smoke rc=$?
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/s9_bench_s20.json 2> gpurun_out/s9_bench_s20.err; echo bench rc=$?
