# compute-sanitizer memcheck / racecheck / synccheck on small mining runs (every kernel)
mkdir -p gpurun_out
cat > /tmp/san.py <<'PY'
import sys, numpy as np
sys.path.insert(0, ".")
import gen, paper_conf_cluster_zhangzb11a_b200 as gpa
for name in ["chess", "mushroom"]:
    ds = gen.make(name)
    th = gpa.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    for kern in (gpa.KERNEL_AUTO, gpa.KERNEL_V0, gpa.KERNEL_PREFIX, gpa.KERNEL_TRIE, gpa.KERNEL_PROJ):
        r = gpa.mine(ds, min_count=th, options=gpa.Options(count_kernel=kern, max_k=6))
        print(name, kern, len(r.frequent()))
# overlapped ingest (host input >= 262,144 transactions) and the device level transition
ds = gen.random_db(5, 270000, 40, max_len=12)
r = gpa.mine(ds, min_count=5000, keep_candidates=True)
print("overlap", len(r.frequent()))
r = gpa.mine(ds, min_count=5000, options=gpa.Options(host_candgen=True, overlap_ingest=False))
print("host", len(r.frequent()))
ds = gen.random_db(3, 20000, 300, max_len=40, duplicates=True, unsorted=True)
with gpa.Bitset(ds) as bs:
    rows = bs.rows()
    rng = np.random.default_rng(0)
    for k in (2, 3, 5):
        c = np.array(sorted({tuple(sorted(rng.choice(rows, k, replace=False))) for _ in range(500)}), np.uint32)
        for kern in (gpa.KERNEL_PAIRS, gpa.KERNEL_TRIE, gpa.KERNEL_PREFIX):
            print(k, kern, int(bs.count(c, kernel=kern).sum()))
PY
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san.py > gpurun_out/san_$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/san_$tool.log
done
