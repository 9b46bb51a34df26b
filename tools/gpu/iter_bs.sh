mkdir -p gpurun_out
make -q || make -j16 > gpurun_out/make.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "bitset or mine or fig2 or overlapped or t40" > gpurun_out/t_iter.log 2>&1; echo "rc=$?" >> gpurun_out/t_iter.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules > gpurun_out/ncu_launch.log 2>&1
