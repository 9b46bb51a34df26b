#!/bin/bash
# Round evidence in one call: GPU suite, smoke(), default bench line, reference arm, launch list,
# ncu --set full of the top kernels, all-configs table vs the full-size oracle, scaling emulation,
# 20-step bench.
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.jsonl 2> gpurun_out/bench_reference.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci > gpurun_out/ncu_bench.log 2>&1
python tools/launch_summary.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1; head -12 gpurun_out/launches.txt
timeout 900 ncu --set full --clock-control none --import-source on \
  -k "regex:scan_build|count_pairs_tc|pext3|count_proj_kernel|pext_kernel|join_kernel" -c 8 \
  -o gpurun_out/top -f python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci > gpurun_out/top.log 2>&1
echo "ncu top rc=$?"
bash tools/gpu/tables.sh
