# Round evidence: bench line (+ oracle reference arm), ncu launch list of one step, ncu --set full of
# the top kernels (pext k=3, count_pairs_tc, count_proj k=3)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > gpurun_out/smi.txt
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.jsonl 2> gpurun_out/bench_ref.err
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"pext3_kernel|count_pairs_tc_kernel|count_proj_kernel" -c 3 -o gpurun_out/prof_top $B > gpurun_out/ncu_top.log 2>&1
echo done
