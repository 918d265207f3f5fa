#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for k in uniform int; do
  timeout 240 python bench.py --config C3 --kind $k --steps 10 --warmup 3 --no-e2e --no-cpu --no-fused > gpurun_out/bench_C3_$k.json 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/bench_C3_$k.json').read().strip().splitlines()[-1])
print('$k', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, 'nonzero info', d['nonzero_info_blocks'])"
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C3int.csv \
    python bench.py --config C3 --kind int --steps 1 --warmup 1 --no-e2e --no-cpu --no-fused > /dev/null 2>&1
