cd $GRAFT_REPO_ROOT
GPA_TRACE=1 python tools/gpu/one_mine.py t40i10d10m 3 > gpurun_out/trace.log 2>&1
tail -60 gpurun_out/trace.log
