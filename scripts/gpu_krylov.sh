#!/bin/bash
# NEXT(4) GPU job: C5K bench line, launch list, one ncu --set full capture of k_spmv
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python bench.py --config C5K --steps 5 --warmup 3 > gpurun_out/bench_C5K.json 2> gpurun_out/bench_C5K.err
tail -c 3000 gpurun_out/bench_C5K.json; tail -5 gpurun_out/bench_C5K.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5K.csv \
    python bench.py --config C5K --steps 1 --warmup 0 --no-cpu > gpurun_out/launches_C5K.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k k_spmv -s 3 -c 1 \
    -o gpurun_out/spmv_C5K python bench.py --config C5K --steps 1 --warmup 0 --no-cpu > gpurun_out/ncu_spmv.log 2>&1
tail -3 gpurun_out/ncu_spmv.log
