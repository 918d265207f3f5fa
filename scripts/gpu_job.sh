mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c4.json 2>/dev/null
