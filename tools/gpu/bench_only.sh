mkdir -p gpurun_out
make -q || make -j16 > gpurun_out/make.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
