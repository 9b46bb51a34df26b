set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "random_candidates or many_rows or fig2 or mine_configs or t40i10d10m" > gpurun_out/pytest_tm.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tm.log
timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/bench_tm.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_tm.log
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_trie_tm -s 3 -c 1 -o gpurun_out/prof_trie_tm $B > gpurun_out/ncu_trie_tm.log 2>&1
