set -x
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null
timeout 700 python -m pytest tests -m gpu -q > gpurun_out/${1:-r01x}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${1:-r01x}_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${1:-r01x}_smoke.log 2>&1; tail -1 gpurun_out/${1:-r01x}_smoke.log
bash tools/gpu_round.sh ${1:-r01x} full > gpurun_out/${1:-r01x}_round.log 2>&1
timeout 300 python tools/trace_phases.py 2 3 4 --flush > gpurun_out/${1:-r01x}_trace_phases.txt 2>&1
tail -c 300 gpurun_out/bench_${1:-r01x}.json
