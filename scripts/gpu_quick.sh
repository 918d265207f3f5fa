#!/bin/bash
# quick GPU iteration: parity tests + bench lines of the batched configs
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 420 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > gpurun_out/pytest.txt
for c in C3 C2 C3f32; do
  timeout 240 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
cat gpurun_out/pytest.txt
for c in C3 C2 C3f32; do python - "$c" <<'PY'
import json,sys
c=sys.argv[1]
try:
    d=json.loads(open(f"gpurun_out/bench_{c}.json").read().strip().splitlines()[-1])
    print(c, "ms/step %.3f" % d["ms_per_step"], "value %.3g" % d["value"], "breakdown", {k: round(v,3) for k,v in d["breakdown_ms"].items()}, "frac %.3f" % d["roofline"]["frac"], "fused", round(d["fused_gesv"]["ms_per_step"],3) if d.get("fused_gesv") else None, "clk", d["clocks"].get("sm_mhz"))
except Exception as e:
    print(c, "FAILED", e, open(f"gpurun_out/bench_{c}.err").read()[-2000:])
PY
done
