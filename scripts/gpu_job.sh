mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
for b in 24 8 16 32; do python bench.py --config C4 --block $b --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c4_$b.json 2>/dev/null; done
python bench.py --config C5 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/c5.json 2>gpurun_out/c5.err
