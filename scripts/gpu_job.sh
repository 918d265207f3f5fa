# scratch GPU job (edited per call)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu > gpurun_out/c3.json 2>gpurun_out/c3.err
python bench.py --config C2 --steps 20 --warmup 3 --no-e2e --no-cpu > gpurun_out/c2.json 2>gpurun_out/c2.err
python bench.py --config C3f32 --steps 20 --warmup 3 --no-e2e --no-cpu > gpurun_out/c3f32.json 2>gpurun_out/c3f32.err
python bench.py --config C5 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/c5.json 2>gpurun_out/c5.err
python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c4.json 2>gpurun_out/c4.err
