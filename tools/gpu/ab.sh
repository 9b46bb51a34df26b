# GPU parity subset + a short bench (optionally several env settings: ab.sh "<-k>" "ENV=a" "ENV=b" ...)
mkdir -p gpurun_out
K="${1:-trie or mine or count}"; shift
timeout 1200 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
i=0
for e in "${@:-X=0}"; do
  env $e timeout 600 python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_ab$i.log 2>&1
  i=$((i+1))
done
