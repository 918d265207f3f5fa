#!/bin/bash
# FEM configs: C5 (setup + 100 applies, LU and inverse variants), C4 extraction b = 8/16/24/32, SV
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python bench.py --config C5 --steps 5 --warmup 2 > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
for b in 8 16 24 32; do
  timeout 200 python bench.py --config C4 --block $b --steps 20 --warmup 3 > gpurun_out/bench_C4_b$b.json 2> gpurun_out/bench_C4_b$b.err
done
python - <<'PY'
import json
for f in ["bench_C5"] + [f"bench_C4_b{b}" for b in (8, 16, 24, 32)]:
    try:
        d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
        print(f, "ms %.4f" % d["ms_per_step"], d.get("breakdown_ms"), "frac %.3f" % d["roofline"]["frac"],
              "inverse", d.get("inverse_variant", {}) and {k: d["inverse_variant"][k] for k in ("ms_per_step", "breakdown_ms", "apply_roofline")})
    except Exception as e:
        print(f, "FAILED", e, open(f"gpurun_out/{f}.err").read()[-1500:])
PY
