#!/bin/bash
# per-rank step time of C3 shards (1M / N blocks) on one GPU: the fixed
# per-step overhead that decides strong scaling at N = 8
cd "$(dirname "$0")/../.."
for nb in 1000000 500000 250000 125000; do
  timeout 300 python bench.py --nblocks $nb --steps 20 --warmup 5 --no-cpu --no-e2e --no-fused 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('nb', $nb, 'ms', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['breakdown_ms'].items()}, 'launches', d['gpu_launches'])"
done
