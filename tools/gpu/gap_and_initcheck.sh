cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
./tools/microbench/launch_gap > gpurun_out/launch_gap.txt 2>&1; cat gpurun_out/launch_gap.txt
timeout 1500 compute-sanitizer --tool initcheck --print-limit 20 python tools/gpu/san_run.py > gpurun_out/san_initcheck.txt 2>&1; echo "initcheck rc=$?"; tail -3 gpurun_out/san_initcheck.txt
timeout 900 python -m pytest tests -m gpu -q -x -k "mine_configs or t40i10d10m_every or fused" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
