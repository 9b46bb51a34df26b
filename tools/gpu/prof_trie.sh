mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_trie -s 2 -c 1 -o gpurun_out/prof_trie6 $B > gpurun_out/ncu_trie6.log 2>&1
