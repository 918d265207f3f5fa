#!/bin/bash
# ncu capture of the GETRF 17-32 kernel on C2 (40k x 32 fp64) -- one launch
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
CFG=${1:-C2}
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_getrf_fast<.*17" -s 1 -c 1 \
    -o gpurun_out/getrf_$CFG python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu > gpurun_out/ncu_$CFG.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$CFG.csv \
    python bench.py --config $CFG --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
tail -3 gpurun_out/ncu_$CFG.log
