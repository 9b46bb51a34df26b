"""Host timeline (GPA_HOST_TRACE) of the complete-intersection pass (count_pairs + trie walk) on T40I10D10M."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
ds = gen.make("t40i10d10m")
th = gpa.min_count(ds.n_tx, "0.005")
o = torch.from_numpy(ds.offsets.view(np.int64)).cuda(); it = torch.from_numpy(ds.items.view(np.int32)).cuda()
opts = gpa.Options(count_kernel=gpa.KERNEL_PAIRS, complete_intersection=True)
for i in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    if i == 2: os.environ["GPA_HOST_TRACE"] = "1"
    r = gpa.mine(o, it, ds.n_items, min_count=th, options=opts)
    torch.cuda.synchronize(); print("wall ms", (time.perf_counter() - t0) * 1e3, file=sys.stderr)
