#!/bin/bash
# One gpurun call: build check, a pytest selection (-m gpu), a bench line and the launch list.
#   tools/gpu/check.sh "<pytest -k expr or ''>" [bench args]
set -u
mkdir -p gpurun_out
K="${1:-}"
shift || true
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -k "$K" > gpurun_out/pytest_gpu.log 2>&1
else
  timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1
fi
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -30 gpurun_out/pytest_gpu.log
timeout 600 python bench.py "$@" > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
echo "bench rc=$?"; tail -3 gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci > gpurun_out/ncu_bench.log 2>&1
echo "ncu rc=$?"
python tools/launch_summary.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1; head -40 gpurun_out/launches.txt
