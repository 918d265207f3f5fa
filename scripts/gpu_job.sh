mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python bench.py > gpurun_out/bench_C3.json 2>gpurun_out/bench_C3.err
python bench.py --config C2 --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_C2.json 2>gpurun_out/bench_C2.err
python bench.py --config C3f32 --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_C3f32.json 2>gpurun_out/bench_C3f32.err
python bench.py --config C5 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_C5.json 2>gpurun_out/bench_C5.err
bash scripts/profile_round.sh C3 > gpurun_out/prof.log 2>&1
