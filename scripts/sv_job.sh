# Supervariable blocking (NEXT 2) on the GPU box: parity tests, bench line, launch list.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_supervariable.py tests/test_gpu_extract.py -q > gpurun_out/pytest_sv.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_sv.txt
timeout 300 python bench.py --config SV --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_SV.json 2>gpurun_out/bench_SV.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_SV.csv python bench.py --config SV --steps 1 --warmup 1 --no-cpu > gpurun_out/launches_SV.log 2>&1
