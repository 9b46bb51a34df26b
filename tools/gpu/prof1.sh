set -x
mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_pairs -c 1 -o gpurun_out/prof_pairs $B > gpurun_out/ncu_pairs.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_prefix -s 4 -c 1 -o gpurun_out/prof_prefix $B > gpurun_out/ncu_prefix.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bitset_build -c 1 -o gpurun_out/prof_bitset $B > gpurun_out/ncu_bitset.log 2>&1
ls -la gpurun_out
