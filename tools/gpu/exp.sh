set -x
mkdir -p gpurun_out
GPA_AUTO_SIBLINGS=1000 timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/bench_alltrie.log 2>&1
GPA_TRACE=1 timeout 600 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_trace.log 2>&1
