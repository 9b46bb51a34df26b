mkdir -p gpurun_out
for S in 2 4 8; do
GPA_TRACE=1 timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --emulate-shard $S > gpurun_out/emul_$S.log 2>&1
done
