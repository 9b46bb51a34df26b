mkdir -p gpurun_out
GPA_TRACE=1 timeout 600 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/trace.log 2>&1
