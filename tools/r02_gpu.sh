#!/bin/bash
# r02 GPU session: build, new parity tests first, full -m gpu suite, microbench, bench.
TAG=${1:-r02a}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
python -c "import oracle; oracle.build()"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_eurosys_kimjlmsm15_b200/csrc -I include \
     -o build/microbench tools/microbench.cu 2>/dev/null && timeout 120 build/microbench > gpurun_out/microbench_$TAG.json
timeout 900 python -m pytest tests/test_gpu_ring_bench.py tests/test_gpu_dispatch.py tests/test_gpu_ring.py -m gpu -x -q > gpurun_out/${TAG}_pytest_new.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_new.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${TAG}_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -c 1500 gpurun_out/bench_$TAG.json; tail -5 gpurun_out/bench_$TAG.err
