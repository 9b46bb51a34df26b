# Full round check: smoke, every GPU test, the default bench line, the reference arm, the NCCL
# path at N=1, the ncu launch list and full captures of the counting kernels.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/nvsmi.txt
lscpu | head -20 > gpurun_out/lscpu.txt; nproc >> gpurun_out/lscpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/bench_ref.log
timeout 900 python bench.py --dist --steps 3 --warmup 1 --no-cpu-baseline > gpurun_out/bench_dist1.log 2>&1; echo "dist rc=$?" >> gpurun_out/bench_dist1.log
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_pairs_tc -c 1 -o gpurun_out/prof_pairs_tc $B > gpurun_out/ncu_pairs_tc.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"count_pairs_kernel" -c 1 -o gpurun_out/prof_pairs $B --kernel pairs > gpurun_out/ncu_pairs.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"count_trie_kernel<7" -c 1 -o gpurun_out/prof_trie $B > gpurun_out/ncu_trie.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:count_prefix -c 1 -o gpurun_out/prof_prefix $B --kernel prefix > gpurun_out/ncu_prefix.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"bitset_build|hist_validate" -c 2 -o gpurun_out/prof_build $B > gpurun_out/ncu_build.log 2>&1
