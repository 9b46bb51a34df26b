# tensor-core pair kernel: parity tests + a short bench (1 GPU)
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "pairs or fig2 or random_candidates" > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tc.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_tc.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --kernel pairs > gpurun_out/bench_cc.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_cc.log
