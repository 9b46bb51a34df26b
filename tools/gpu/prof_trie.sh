# ncu --set full of count_trie launches (generations k=6 and k=7 by default) on T40I10D10M
mkdir -p gpurun_out
TAG="${1:-trie}"; SKIP="${2:-2}"; CNT="${3:-2}"
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"count_(trie|class)" -s $SKIP -c $CNT -o gpurun_out/prof_$TAG $B > gpurun_out/ncu_$TAG.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_$TAG.log
