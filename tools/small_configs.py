#!/usr/bin/env python
"""GPU mining time of the four small BASELINE.json configurations (device-resident CSR and
pinned host input), median of 20, with the launch count per call -- the latency-bound regime."""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
import paper_conf_cluster_zhangzb11a_b200 as gpa  # noqa: E402

for name in ["chess", "mushroom", "t40i10d100k", "accidents"]:
    ds = gen.make(name)
    theta = gpa.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    d_off = torch.from_numpy(ds.offsets.view(np.int64)).cuda()
    d_items = torch.from_numpy(ds.items.view(np.int32)).cuda()
    h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
    h_items = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
    for _ in range(3):
        r = gpa.mine(d_off, d_items, ds.n_items, min_count=theta)
    ts, te, la = [], [], []
    for _ in range(20):
        torch.cuda.synchronize()
        l0 = gpa.kernel_launches()
        t = time.perf_counter()
        r = gpa.mine(d_off, d_items, ds.n_items, min_count=theta)
        ts.append(time.perf_counter() - t)
        la.append(gpa.kernel_launches() - l0)
        t = time.perf_counter()
        gpa.mine(h_off, h_items, ds.n_items, min_count=theta)
        te.append(time.perf_counter() - t)
    print(json.dumps({"config": name, "generations": len(r.levels), "frequent": len(r.frequent()),
                      "gpu_ms": 1e3 * float(np.median(ts)), "gpu_e2e_ms": 1e3 * float(np.median(te)),
                      "launches": int(np.median(la)), "phases": {k: round(v, 3) for k, v in r.timing_ms.items()}}))
