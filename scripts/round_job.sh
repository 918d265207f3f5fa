set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
bash scripts/gpu_job.sh
python bench.py --config C4 --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_C4.json 2>gpurun_out/bench_C4.err
python bench.py --impl reference > gpurun_out/bench_ref.json 2>gpurun_out/bench_ref.err
bash scripts/sv_job.sh
