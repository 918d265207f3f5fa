#!/bin/bash
# A/B: C5 setup and C3 with the current library and the ba8f404 library, same box
cd "$(dirname "$0")/../.."
for i in 1 2; do
for tree in . oldtree; do
  (cd $tree && timeout 300 python bench.py --config C5 --steps 5 --warmup 2 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$tree C5', round(d['ms_per_step'],3), d['breakdown_ms'])")
  (cd $tree && timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu --no-e2e --no-fused 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$tree C3', round(d['ms_per_step'],3), d['breakdown_ms'])")
done
done
