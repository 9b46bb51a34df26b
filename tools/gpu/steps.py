"""Per-step wall times of gpa_mine on a config (device-resident CSR), with the phase split."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import gen
import paper_conf_cluster_zhangzb11a_b200 as gpa
name = sys.argv[1] if len(sys.argv) > 1 else "t40i10d10m"
kern = {"auto": gpa.KERNEL_AUTO, "trie": gpa.KERNEL_TRIE, "proj": gpa.KERNEL_PROJ}[sys.argv[2] if len(sys.argv) > 2 else "auto"]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 8
ds = gen.make(name)
theta = gpa.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
off = torch.from_numpy(ds.offsets.view(np.int64)).cuda(); it = torch.from_numpy(ds.items.view(np.int32)).cuda()
for i in range(n):
    torch.cuda.synchronize(); t = time.perf_counter()
    r = gpa.mine(off, it, ds.n_items, min_count=theta, options=gpa.Options(count_kernel=kern))
    torch.cuda.synchronize(); dt = (time.perf_counter() - t) * 1e3
    print(f"step {i}: {dt:.1f} ms (C total {r.timing_ms['total']:.1f}, phases " +
          " ".join(f"{k}:{v:.1f}" for k, v in r.timing_ms.items()) + f")  |F|={sum(lv.n_freq for lv in r.levels)}  levels " +
          " ".join(f"k{lv.k}:{lv.stats['count_ms']:.1f}" for lv in r.levels[1:]), flush=True)
