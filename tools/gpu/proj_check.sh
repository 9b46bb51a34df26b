# projected-list path: parity subset, per-step times, launch list of one step
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "mine_random or mine_configs or dense_long or overlapped or fig2 or max_k or nccl" > gpurun_out/t_proj.log 2>&1
tail -2 gpurun_out/t_proj.log
timeout 300 python tools/gpu/steps.py t40i10d10m auto 6 > gpurun_out/steps.log 2>&1
cat gpurun_out/steps.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_proj.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b.log 2>&1
