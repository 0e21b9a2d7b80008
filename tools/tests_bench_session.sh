#!/bin/bash
# GPU tests + the default bench line
TAG=${1:-tb}
mkdir -p gpurun_out
python -m paper_conf_eurosys_kimjlmsm15_b200.build >/dev/null || exit 1
python -c "import oracle; oracle.build()"
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; tail -3 gpurun_out/bench_${TAG}.err
python - <<PY
import json
d = json.loads(open("gpurun_out/bench_${TAG}.json").read().strip().splitlines()[-1])
print({k: d.get(k) for k in ("value", "ms_per_step", "roofline", "e2e")})
print("by_size", d.get("by_size"))
print("inbound", {k: (round(v["gbps"], 1), round(v["us_per_step"], 2), v["ring_form"]) for k, v in (d.get("inbound") or {}).items()})
PY
