#!/bin/bash
# Per-generation device timeline (GPA_TRACE) of one mining pass at S = 1 and at the S = 8 shard,
# and the launch list of the S = 8 shard.
set -u
mkdir -p gpurun_out
A="--steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-rules --no-ci"
GPA_TRACE=1 timeout 300 python bench.py $A > gpurun_out/trace_s1.json 2> gpurun_out/trace_s1.txt; echo "s1 rc=$?"
GPA_TRACE=1 timeout 300 python bench.py $A --emulate-shard 8 > gpurun_out/trace_s8.json 2> gpurun_out/trace_s8.txt; echo "s8 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_s8.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci --emulate-shard 8 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_s8.csv > gpurun_out/launches_s8.txt 2>&1; head -40 gpurun_out/launches_s8.txt
