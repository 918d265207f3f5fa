#!/bin/bash
# e2e (bj_gesv_host) time vs the number of pipeline chunks, same box
cd "$(dirname "$0")/../.."
for k in 1 2 4 8 16; do
  BJ_GESV_HOST_CHUNKS=$k timeout 300 python bench.py --no-cpu --no-fused --steps 3 --warmup 3 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('chunks $k e2e ms', round(d['e2e']['ms_per_step'],2), 'step', round(d['ms_per_step'],3))"
done
