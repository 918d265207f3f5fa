mkdir -p gpurun_out
python scripts/c4probe.py > gpurun_out/c4probe.txt 2>&1
for b in 24 8 16 32; do python bench.py --config C4 --block $b --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c4_$b.json 2>/dev/null; done
python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu > gpurun_out/c3.json 2>gpurun_out/c3.err
