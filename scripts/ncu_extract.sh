#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
B=${1:-24}
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C4_b$B.csv \
    python bench.py --config C4 --block $B --steps 2 --warmup 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_extract" -s 2 -c 2 \
    -o gpurun_out/extract_b$B python bench.py --config C4 --block $B --steps 1 --warmup 1 > gpurun_out/ncu_extract.log 2>&1
tail -2 gpurun_out/ncu_extract.log
