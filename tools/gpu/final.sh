# Round-end evidence: smoke, every GPU test, then evidence.sh (bench, reference arm, launch list, top-kernel captures)
mkdir -p gpurun_out
make -q || make -j16 > gpurun_out/make.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
bash tools/gpu/evidence.sh
