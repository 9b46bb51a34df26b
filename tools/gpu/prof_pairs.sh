mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_pairs -c 1 -o gpurun_out/prof_pairs3 $B > gpurun_out/ncu_pairs3.log 2>&1
