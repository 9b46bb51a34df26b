#!/bin/bash
# Quick iteration: a pytest -k selection, a short bench line (no CI / rules / CPU legs) and the
# launch list of one step.   tools/gpu/quick.sh "<pytest -k expr>"
set -u
mkdir -p gpurun_out
if [ -n "${1:-}" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x -k "$1" > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
fi
timeout 600 python bench.py --steps 10 --warmup 3 --no-ci --no-rules --no-cpu-baseline > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
echo "bench rc=$?"; tail -3 gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.jsonl').readline())
print('ms/step', d['ms_per_step'], 'e2e', d['e2e']['ms_per_step'], 'launches', d['gpu_launches'])
print('phases', {k: round(v, 2) for k, v in d['phase_ms_last_step'].items()})
print('kernel ms by k', {k: round(v, 2) for k, v in d['kernel_time_ms'].items()})
for k, r in d['roofline_by_kernel'].items(): print(k, round(r['kernel_ms'], 3), r['bound'], round(r['frac'], 3))
"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci > gpurun_out/ncu_bench.log 2>&1
echo "ncu rc=$?"
python tools/launch_summary.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1; head -30 gpurun_out/launches.txt
