"""Small runs of every kernel path for compute-sanitizer (tools/gpu/sanitize.sh)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("mushroom")
th = gpa.min_count(ds.n_tx, "0.20")
a = gpa.mine(ds, min_count=th, keep_candidates=True)                                    # fused loop (+ one-pass build)
b = gpa.mine(ds, min_count=th, options=gpa.Options(multi_kernel=True))                  # projected lists
c = gpa.mine(ds, min_count=th, options=gpa.Options(count_kernel=gpa.KERNEL_PAIRS, complete_intersection=True))
assert a.frequent() == b.frequent() == c.frequent()
with gpa.Bitset(ds, row_min_count=th) as bs:                                           # compaction
    assert len(bs.count(a.levels[2].cand)) == a.levels[2].n_cand
t = gen.make("t40i10d100k")
d = gpa.mine(t, min_count=gpa.min_count(t.n_tx, "0.01"))                                # fused with the tc pair Gram
e = gpa.mine(t, min_count=gpa.min_count(t.n_tx, "0.01"), options=gpa.Options(multi_kernel=True))  # pext3, pext, joins
assert d.frequent() == e.frequent()
print("san_run ok", len(a.frequent()), len(d.frequent()))
