#!/bin/bash
# per-launch device times (ncu, cold-cache, serialised) of one bench step
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
CFG=$1; shift
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$CFG.csv \
    python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu --no-fused "$@" > gpurun_out/launches_$CFG.out 2>&1
tail -2 gpurun_out/launches_$CFG.out
