#!/bin/bash
# Evidence tables: every BASELINE.json config vs the oracle, the one-GPU scaling emulation, a 20-step bench line.
set -u
mkdir -p gpurun_out
timeout 1500 python bench.py --all-configs > gpurun_out/all_configs.jsonl 2> gpurun_out/all_configs.err; echo "all rc=$?"
for S in 1 2 4 8; do
  timeout 600 python bench.py --emulate-shard $S --steps 10 --warmup 3 --no-e2e --no-ci --no-rules --no-cpu-baseline \
    > gpurun_out/emul_$S.jsonl 2>> gpurun_out/emul.err; echo "emul $S rc=$?"
done
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench20.jsonl 2> gpurun_out/bench20.err; echo "bench rc=$?"
