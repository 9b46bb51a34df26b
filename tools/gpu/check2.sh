# new parity test (set-bit-walk generation 3) + compute-sanitizer over the current kernels (pext3 included)
mkdir -p gpurun_out
make -q || make -j16 > gpurun_out/make.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "k3_set_bit_walk or proj or mine_configs" > gpurun_out/t_new.log 2>&1; echo "rc=$?" >> gpurun_out/t_new.log
bash tools/gpu/sanitize.sh
