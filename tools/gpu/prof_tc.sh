# bench + ncu --set full of the tensor-core pair kernel on T40I10D10M
set -x
mkdir -p gpurun_out
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tc.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_tc.log
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_pairs_tc -c 1 -o gpurun_out/prof_pairs_tc $B > gpurun_out/ncu_pairs_tc.log 2>&1
