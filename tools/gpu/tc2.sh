set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "pairs or fig2 or random_candidates or mine_configs" > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tc.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_tc.log
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_pairs_tc -c 1 -o gpurun_out/prof_pairs_tc $B > gpurun_out/ncu_pairs_tc.log 2>&1
