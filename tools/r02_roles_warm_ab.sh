#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
python -c "import oracle; oracle.build()"
timeout 900 python -m pytest tests/test_gpu_ring_roles.py -q -x > gpurun_out/s10_pytest_roles.log 2>&1; tail -1 gpurun_out/s10_pytest_roles.log
for rep in 1 2; do
for K in 20 200; do
  echo "warm K=$K $(RING_K=$K FORMS=roles timeout 300 python tools/ring_forms.py 64 128 512 2>&1 | tail -1)"
  echo "nowarm K=$K $(NBA_IPSEC_LIB=build/variants/nowarm.so RING_K=$K FORMS=roles timeout 300 python tools/ring_forms.py 64 128 512 2>&1 | tail -1)"
done; done
NBA_IPSEC_LIB=build/variants/rtrace.so timeout 300 python tools/roles_trace.py 64 512 2>&1 | tail -1
