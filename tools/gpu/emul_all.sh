mkdir -p gpurun_out
for S in 1 2 4 8; do
timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --emulate-shard $S > gpurun_out/emul_$S.log 2>&1
done
