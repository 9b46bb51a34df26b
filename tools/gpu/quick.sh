# usage: bash tools/gpu/quick.sh "<pytest -k expr>" "<bench extra args>"
set -x
mkdir -p gpurun_out
K="${1:-not t40i10d10m}"
timeout 1200 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e $2 > gpurun_out/bench_q.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_q.log
nproc > gpurun_out/nproc.txt
