"""One gpa_mine of a BASELINE.json config with the CSR on the device (profiling helper)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
name = sys.argv[1] if len(sys.argv) > 1 else "accidents"
ds = gen.make(name)
th = gpa.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
o = torch.from_numpy(ds.offsets.view(np.int64)).cuda(); it = torch.from_numpy(ds.items.view(np.int32)).cuda()
for _ in range(int(sys.argv[2]) if len(sys.argv) > 2 else 2):
    r = gpa.mine(o, it, ds.n_items, min_count=th)
print(name, len(r.levels), len(r.frequent()))
