"""End-to-end gpa_mine from pinned host memory: per-step wall time and phase split."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import gen
import paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("t40i10d10m")
theta = gpa.min_count(ds.n_tx, "0.005")
h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
h_it = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
for i in range(4):
    torch.cuda.synchronize(); t = time.perf_counter()
    r = gpa.mine(h_off, h_it, ds.n_items, min_count=theta)
    torch.cuda.synchronize()
    print(f"e2e step {i}: {(time.perf_counter() - t) * 1e3:.1f} ms", {k: round(v, 1) for k, v in r.timing_ms.items()}, flush=True)
