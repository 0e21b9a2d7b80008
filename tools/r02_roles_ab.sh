#!/bin/bash
# role-split ring: parity tests, per-size timing against the pipelined form (K = 200 and 20), phase trace
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests/test_gpu_ring_roles.py tests/test_gpu_ring_bench.py -q -x > gpurun_out/rab_pytest.log 2>&1; tail -1 gpurun_out/rab_pytest.log
for K in 200 20; do echo "K=$K $(RING_K=$K timeout 300 python tools/ring_forms.py 64 128 256 512 2>&1 | tail -1)"; done
NBA_IPSEC_LIB=build/variants/rtrace.so timeout 300 python tools/roles_trace.py 64 2>&1 | tail -1
