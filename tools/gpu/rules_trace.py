"""Association rules on T40I10D10M's F: wall time of MineResult.rules (GPA_TRACE=1 for the split)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import gen
import paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("t40i10d10m")
off = torch.from_numpy(ds.offsets.view(np.int64)).cuda(); it = torch.from_numpy(ds.items.view(np.int32)).cuda()
r = gpa.mine(off, it, ds.n_items, min_count=gpa.min_count(ds.n_tx, "0.005"))
for i in range(3):
    t = time.perf_counter(); rl = r.rules("0.9"); print(f"rules {len(rl)} in {(time.perf_counter() - t) * 1e3:.1f} ms", flush=True)
