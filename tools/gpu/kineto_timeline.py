"""Device timeline of one gpa_mine pass from CUPTI (torch.profiler sees every kernel of the process,
including libgpapriori's): kernel start/end, the idle gaps between them, per generation.
   python tools/gpu/kineto_timeline.py [config] [shard S] > timeline.txt"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
from torch.profiler import profile, ProfilerActivity
import gen, paper_conf_cluster_zhangzb11a_b200 as gpa

name = sys.argv[1] if len(sys.argv) > 1 else "t40i10d10m"
S = int(sys.argv[2]) if len(sys.argv) > 2 else 1
ds = gen.make(name)
n = ds.n_tx
if S > 1:
    n = (ds.n_tx // S + 102399) // 102400 * 102400
off = ds.offsets[: n + 1].copy()
items = ds.items[: off[-1]]
th = gpa.min_count(n, gen.CONFIGS[name].minsup)
o = torch.from_numpy(off.view(np.int64)).cuda()
it = torch.from_numpy(items.view(np.int32)).cuda()
for _ in range(3):
    gpa.mine(o, it, ds.n_items, min_count=th)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    r = gpa.mine(o, it, ds.n_items, min_count=th)
    torch.cuda.synchronize()
path = f"/tmp/kineto_{os.getpid()}.json"
prof.export_chrome_trace(path)
ev = [e for e in json.load(open(path))["traceEvents"] if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset")]
ev.sort(key=lambda e: e["ts"])
t0 = ev[0]["ts"]
busy = sum(e["dur"] for e in ev)
end = max(e["ts"] + e["dur"] for e in ev)
print(f"# {name} S={S} n_tx={n}: span {(end - t0) / 1e3:.3f} ms, busy {busy / 1e3:.3f} ms, {len(ev)} ops")
last_end = t0
agg = {}
for e in ev:
    gap = e["ts"] - last_end
    nm = e["name"].replace("(anonymous namespace)::", "").replace("void ", "").replace("gpa::", "").split("(")[0][:40]
    print(f"{(e['ts'] - t0) / 1e3:9.3f} gap {gap:8.1f} us  dur {e['dur']:8.1f} us  {e.get('cat')[:6]} {nm}")
    a = agg.setdefault(nm, [0, 0.0, 0.0])
    a[0] += 1
    a[1] += e["dur"]
    a[2] += max(gap, 0)
    last_end = max(last_end, e["ts"] + e["dur"])
print("# per op: count, busy us, idle-before us")
for nm, (c, d, g) in sorted(agg.items(), key=lambda kv: -kv[1][2]):
    print(f"#  {nm:40s} {c:4d} {d:10.1f} {g:10.1f}")
