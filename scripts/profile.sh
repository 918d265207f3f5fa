#!/bin/bash
# Profile capture on the GPU box (run under gpurun).  Usage:
#   scripts/profile.sh <tag> <kernel-regex> [bench args...]
# Writes compact exports to gpurun_out/<tag>_{raw,details}.csv and a gzipped
# SASS source page; the .ncu-rep itself stays in /tmp (too large to ship).
set -u
tag=$1; shift
kre=$1; shift
mkdir -p gpurun_out /tmp/prof
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:${kre}" -c 1 \
    -o /tmp/prof/${tag} -f python bench.py --no-e2e --no-cpu "$@" > gpurun_out/${tag}_ncu.log 2>&1
ncu -i /tmp/prof/${tag}.ncu-rep --page raw --csv > gpurun_out/${tag}_raw.csv 2>&1
ncu -i /tmp/prof/${tag}.ncu-rep --page details --csv > gpurun_out/${tag}_details.csv 2>&1
ncu -i /tmp/prof/${tag}.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip -6 > gpurun_out/${tag}_sass.csv.gz
