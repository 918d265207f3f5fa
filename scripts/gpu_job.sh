mkdir -p gpurun_out
timeout 300 scripts/micro/bin/grbx > gpurun_out/grbx.txt 2>&1
