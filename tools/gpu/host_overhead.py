"""Per-call host overhead of gpa.mine() on T40I10D10M (device CSR): Python wall clock of the call,
the library's own wall clock (timing['total']), and the teardown of the previous result."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("t40i10d10m")
th = gpa.min_count(ds.n_tx, gen.CONFIGS["t40i10d10m"].minsup)
o = torch.from_numpy(ds.offsets.view(np.int64)).cuda(); it = torch.from_numpy(ds.items.view(np.int32)).cuda()
res = None
for i in range(8):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    res = None
    t1 = time.perf_counter()
    res = gpa.mine(o, it, ds.n_items, min_count=th)
    t2 = time.perf_counter()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    print(f"teardown {1e3*(t1-t0):.3f} ms, mine() {1e3*(t2-t1):.3f} ms (library total {res.timing_ms['total']:.3f}), "
          f"sync after {1e3*(t3-t2):.3f} ms")
