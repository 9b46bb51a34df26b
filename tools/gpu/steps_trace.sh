GPA_TRACE=1 timeout 300 python tools/gpu/steps.py t40i10d10m auto 8 > gpurun_out/steps.log 2> gpurun_out/steps.err
