#!/bin/bash
# ncu --set full of selected kernels of one bench step.   tools/gpu/prof.sh <regex> <skip> <count> <name> [bench args]
set -u
mkdir -p gpurun_out
RE="$1"; SKIP="$2"; CNT="$3"; NAME="$4"; shift 4
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$RE" -s "$SKIP" -c "$CNT" \
  -o "gpurun_out/$NAME" -f python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-rules --no-ci "$@" \
  > "gpurun_out/$NAME.log" 2>&1
echo "ncu rc=$?"; tail -3 "gpurun_out/$NAME.log"
