#!/bin/bash
# C4 (all b) and C5 setup timings for an extraction variant
cd "$(dirname "$0")/../.."
timeout 600 python -m pytest tests/test_gpu_extract.py -x -q 2>&1 | tail -1
for b in 8 16 24 32; do
  timeout 200 python bench.py --config C4 --block $b --steps 20 --warmup 3 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C4 b=$b', round(d['ms_per_step'],4), round(d['roofline']['frac'],3))"
done
timeout 300 python bench.py --config C5 --steps 5 --warmup 2 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C5', round(d['ms_per_step'],3), d['breakdown_ms'])"
