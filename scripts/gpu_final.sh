#!/bin/bash
# the driver's bench invocations + the other configs, and the ncu launch list of the headline
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/final
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 500 > gpurun_out/final/clocks.csv &
SMI=$!
timeout 600 python bench.py > gpurun_out/final/bench_default.json 2> gpurun_out/final/bench_default.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/final/bench_reference.json 2> gpurun_out/final/bench_reference.err
for c in C3f32 C2 C1; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu > gpurun_out/final/bench_$c.json 2> gpurun_out/final/bench_$c.err
done
timeout 300 python bench.py --config C5 --steps 5 --warmup 2 > gpurun_out/final/bench_C5.json 2> gpurun_out/final/bench_C5.err
timeout 300 python bench.py --config SV --steps 10 --warmup 3 > gpurun_out/final/bench_SV.json 2> gpurun_out/final/bench_SV.err
for b in 8 16 24 32; do
  timeout 200 python bench.py --config C4 --block $b --steps 20 --warmup 3 > gpurun_out/final/bench_C4_b$b.json 2> gpurun_out/final/bench_C4_b$b.err
done
kill $SMI
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_C3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-fused > /dev/null 2>&1
for f in gpurun_out/final/bench_*.json; do echo "$f: $(tail -c 400 $f)"; done
