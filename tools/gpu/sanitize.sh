#!/bin/bash
# compute-sanitizer over every kernel path (tools/gpu/san_run.py); summaries into gpurun_out/san_*.txt
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/gpu/san_run.py > gpurun_out/san_$tool.txt 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/san_$tool.txt
done
