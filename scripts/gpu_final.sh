#!/bin/bash
# Round-end evidence run (under gpurun): GPU tests, smoke, the driver's bench
# invocations, every config's bench line, launch lists and the ncu summary of
# the headline step.  Output: gpurun_out/final/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/final
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/final/pytest_gpu.txt 2>&1
tail -3 gpurun_out/final/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/final/smoke.txt
timeout 600 python bench.py > gpurun_out/final/bench_default.json 2> gpurun_out/final/bench_default.err
timeout 600 python bench.py --impl reference > gpurun_out/final/bench_reference.json 2> gpurun_out/final/bench_reference.err
for c in C3f32 C2 C1; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu > gpurun_out/final/bench_$c.json 2> gpurun_out/final/bench_$c.err
done
timeout 300 python bench.py --config C3 --kind int --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/final/bench_C3_int.json 2> gpurun_out/final/bench_C3_int.err
timeout 300 python bench.py --config C5 --steps 5 --warmup 2 > gpurun_out/final/bench_C5.json 2> gpurun_out/final/bench_C5.err
timeout 300 python bench.py --config C5K --steps 5 --warmup 3 > gpurun_out/final/bench_C5K.json 2> gpurun_out/final/bench_C5K.err
timeout 300 python bench.py --config SV --steps 10 --warmup 3 > gpurun_out/final/bench_SV.json 2> gpurun_out/final/bench_SV.err
for b in 8 16 24 32; do
  timeout 200 python bench.py --config C4 --block $b --steps 20 --warmup 3 > gpurun_out/final/bench_C4_b$b.json 2> gpurun_out/final/bench_C4_b$b.err
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_C3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-fused > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_C5K.csv \
    python bench.py --config C5K --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
bash scripts/profile_round.sh C3 --no-fused > /dev/null 2>&1
cp gpurun_out/ncu_C3_summary.json gpurun_out/final/ 2>/dev/null
for f in gpurun_out/final/bench_*.json; do echo "$f: $(tail -c 300 $f)"; done
