# one optimisation iteration: projected-list parity subset, the bench line, pext3 capture
mkdir -p gpurun_out
make -q || make -j16 > gpurun_out/make.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "proj or mine or fig2 or rules" > gpurun_out/t_iter.log 2>&1; echo "rc=$?" >> gpurun_out/t_iter.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pext3_kernel" -c 1 -o gpurun_out/prof_pext3 $B > gpurun_out/ncu_pext3.log 2>&1
