"""Per-call end-to-end time of gpa_mine on pinned host input (T40I10D10M), to see outliers."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("t40i10d10m")
th = gpa.min_count(ds.n_tx, "0.005")
h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
h_items = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
for r in sys.argv[1:] or ["0", "3"]:
    os.environ["GPA_PACK_RAW_EVERY"] = r
    ts = []
    res = None
    for i in range(12):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        res = gpa.mine(h_off, h_items, ds.n_items, min_count=th)
        torch.cuda.synchronize()
        ts.append((time.perf_counter() - t0) * 1e3)
    print("raw_every", r, " ".join(f"{t:.1f}" for t in ts))
