# quick: bitset / mine parity subset, per-step times, launch list of one step
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "bitset or mine_random or mine_configs or dense_long or overlapped or fig2 or max_k or nccl or count_random" > gpurun_out/t_quick.log 2>&1
tail -2 gpurun_out/t_quick.log
timeout 300 python tools/gpu/steps.py t40i10d10m auto 6 > gpurun_out/steps.log 2>&1
tail -1 gpurun_out/steps.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_q.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_q.log 2>&1
