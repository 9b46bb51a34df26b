#!/usr/bin/env python
"""Benchmark of the GPApriori support-counting hot path on B200.

One STEP = one full pass of the hot path over the workload:
validation + generation-1 histogram, static-bitset build, and every generation's candidate
generation, GPU support counting, (all-reduce), threshold -- i.e. one gpa_mine() call.

  value  = sum_{k>=2} |C_k| * N  /  step time     (candidate x transaction / s, whole job)
           inputs (CSR) already resident in HBM when the timed region starts;
  e2e    = the same metric through gpa_mine() with pinned HOST buffers: the upload of the CSR (the
           library packs the item ids to ceil(log2 n_items) bits on the host before the H2D) and
           the D2H of every generation's frequent itemsets are inside the timed region.

Workload: BASELINE.json configs[4], T40I10D10M (10M transactions, 1,000 items, minsup 0.005) --
the configuration the north star grades (HBM-bound bitset, 1.25 GB > 126 MB L2, so no L2 flush
is needed between steps).  Multi-GPU (torchrun): the transaction axis is sharded across ranks
(contiguous, 102,400-transaction chunks), counts are summed with NCCL all-reduce inside the
library; the total work is fixed ("strong" scaling), time = max over ranks.

--impl reference times the CPU oracle (oracle/, the parity reference) as it stands on the
host cores, on a bounded prefix sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--config", default="t40i10d10m", choices=list(gen.CONFIGS))
    p.add_argument("--kernel", default="auto", choices=["auto", "v0", "prefix", "pairs", "trie", "pairs_tc", "proj"])
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-rules", action="store_true", help="skip the association-rules measurement")
    p.add_argument("--dist", action="store_true", help="use the NCCL path even with one rank")
    p.add_argument("--all-configs", action="store_true",
                   help="table of every BASELINE.json config (GPU mine time vs the oracle); not a bench line")
    p.add_argument("--emulate-shard", type=int, default=0,
                   help="scaling study on one GPU: mine the first 1/S of the transactions with min_count/S "
                        "(about one rank's share of the work at S GPUs); not a bench line")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-ci", action="store_true", help="skip the complete-intersection (north-star kernel) leg")
    p.add_argument("--cpu-sample-tx", type=int, default=0, help="oracle sample size (0 = auto)")
    return p.parse_args()


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = "clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown," \
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown," \
             "clocks_event_reasons.sw_power_cap"

    def __init__(self, device: int):
        self.device = device
        self.samples = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5)
                vals = [v.strip() for v in out.stdout.strip().split(",")]
                if len(vals) == 7:
                    self.samples.append(vals)
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for s in self.samples for n, v in zip(names, s[3:]) if v.lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def shard_range(n_tx: int, rank: int, world: int, quest: bool = True):
    """Contiguous rank ranges: Quest data on generator-chunk boundaries (102,400 transactions,
    so each rank generates only its own chunks), other data on 512-transaction boundaries."""
    ch = gen.chunk_size() if quest else 512
    n_chunks = (n_tx + ch - 1) // ch
    c0 = n_chunks * rank // world
    c1 = n_chunks * (rank + 1) // world
    return min(n_tx, c0 * ch), min(n_tx, c1 * ch)


def cpu_sample_size(cfg, requested):
    if requested:
        return requested
    return {"t40i10d10m": 819_200, "t40i10d100k": 25_000, "accidents": 100_000}.get(cfg.name, cfg.n_tx)


def run_oracle_sample(cfg, n_sample):
    """The oracle (as it stands) on the first n_sample transactions of the workload, threshold
    ratio unchanged.  Returns (cand_tx, seconds, threads, description)."""
    import oracle
    ds = gen.make(cfg.name, tx_begin=0, tx_end=min(n_sample, cfg.n_tx))
    theta = oracle.min_count(ds.n_tx, cfg.minsup)
    threads = max(1, len(os.sched_getaffinity(0)))
    t0 = time.perf_counter()
    r = oracle.mine_ds(ds, theta, threads=threads)
    dt = time.perf_counter() - t0
    cand_tx = sum(len(lv.cand) for lv in r.levels[1:]) * ds.n_tx
    desc = (f"oracle.mine on the first {ds.n_tx} transactions of {cfg.name} (minsup {cfg.minsup}, "
            f"min_count {theta}); {len(r.levels)} generations")
    return cand_tx, dt, threads, desc


def reference_arm(args, cfg, rank, world):
    """--impl reference: the CPU oracle timed on the host cores (rank 0 only)."""
    if rank != 0:
        return
    n_sample = cpu_sample_size(cfg, args.cpu_sample_tx)
    for _ in range(args.warmup):
        run_oracle_sample(cfg, min(n_sample, 20_000))
    vals, secs = [], []
    desc, threads, cand_tx = "", 1, 0
    for _ in range(args.steps):
        cand_tx, dt, threads, desc = run_oracle_sample(cfg, n_sample)
        vals.append(cand_tx / dt)
        secs.append(dt)
    v = float(np.median(vals))
    line = {
        "impl": "reference", "metric": "support-count cand*tx/s (whole mining pass)", "value": v,
        "unit": "cand*tx/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": float(np.median(secs)) * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfg.name, "n_tx": cfg.n_tx, "n_items": cfg.n_items, "minsup": cfg.minsup,
                   "sample_tx": n_sample},
        "cpu_baseline": {"value": v, "unit": "cand*tx/s", "cores": threads, "kind": "oracle", "sample": desc},
        "e2e": {"value": v, "unit": "cand*tx/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def all_configs_table(args):
    """Every BASELINE.json configuration: GPU mining time (device-resident and end to end) against
    the CPU oracle on all host cores; checks the frequent itemsets are identical."""
    import torch
    import oracle
    import paper_conf_cluster_zhangzb11a_b200 as gpa
    threads = max(1, len(os.sched_getaffinity(0)))
    rows = []
    for name, cfg in gen.CONFIGS.items():
        ds = gen.make(name)
        theta = gpa.min_count(ds.n_tx, cfg.minsup)
        d_off = torch.from_numpy(ds.offsets.view(np.int64)).cuda()
        d_items = torch.from_numpy(ds.items.view(np.int32)).cuda()
        h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
        h_items = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
        for _ in range(2):
            res = gpa.mine(d_off, d_items, ds.n_items, min_count=theta)
        ts, te = [], []
        for _ in range(5):
            torch.cuda.synchronize()
            t = time.perf_counter()
            res = gpa.mine(d_off, d_items, ds.n_items, min_count=theta)
            ts.append(time.perf_counter() - t)
            t = time.perf_counter()
            gpa.mine(h_off, h_items, ds.n_items, min_count=theta)
            te.append(time.perf_counter() - t)
        t = time.perf_counter()
        ref = oracle.mine_ds(ds, theta, threads=threads)
        to = time.perf_counter() - t
        same = res.frequent() == ref.frequent()
        ms, me = 1e3 * float(np.median(ts)), 1e3 * float(np.median(te))
        rows.append({"config": name, "n_tx": ds.n_tx, "min_count": theta, "generations": len(res.levels),
                     "frequent": len(res.frequent()), "cand_tx": res.cand_tx, "gpu_ms": ms, "gpu_e2e_ms": me,
                     "oracle_ms": to * 1e3, "oracle_threads": threads, "speedup_e2e": to * 1e3 / me,
                     "identical_F": same})
        print(json.dumps(rows[-1]), flush=True)


def wire_bytes(offsets: np.ndarray, n_items: int, raw_every: int = 4) -> int:
    """Host-to-device bytes of gpa_mine on host input: the library's overlapped ingest (>= 262,144
    transactions, <= 16,384 item ids; runtime/ingest.cpp) sends the offsets and, per chunk (8 chunks
    of whole 8,192-transaction stripes), the item ids as ceil(log2 n_items)-bit fields in blocks of 32
    ids -- every raw_every-th chunk from chunk 0 raw (u32); otherwise everything goes raw."""
    n_tx = len(offsets) - 1
    o = offsets.astype(np.int64)
    raw = int(offsets.nbytes) + 4 * int(o[-1])
    b = max(1, int(n_items - 1).bit_length())
    if not (n_tx >= 8 * 4 * 8192 and 2 <= n_items <= 16384 and b <= 16):
        return raw
    ct = -(-n_tx // 8)
    ct = -(-ct // 8192) * 8192
    cuts = list(range(0, n_tx, ct)) + [n_tx]
    total = int(offsets.nbytes)
    for c in range(len(cuts) - 1):
        n = int(o[cuts[c + 1]] - o[cuts[c]])
        total += 4 * n if raw_every and c % raw_every == 0 else -(-n // 32) * b * 4
    return total


def load_peaks() -> dict:
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def average_stats(level_stats: dict) -> dict:
    out = {}
    for k, sts in level_stats.items():
        a = dict(sts[-1])
        for f in ("count_ms", "build_ms", "setup_ms", "allreduce_ms"):
            a[f] = float(np.mean([st[f] for st in sts]))
        out[k] = a
    return out


def pitch_bytes(n_tx: int) -> int:
    """Row pitch of the static bitset (csrc/common.h pitch_words_for: 4 KB multiples)."""
    w = (n_tx + 31) // 32
    w = (w + 1023) // 1024 * 1024
    return 4 * max(w, 1024)


TRAFFIC_KEYS = {"pairs_tc": "count_pairs_tc_kernel", "pairs": "count_pairs_kernel", "prefix": "count_prefix_kernel"}


def traffic_entry(kernel: str, k: int):
    """The committed ncu --set full figures of a launch (profiles/traffic.json): DRAM bytes per
    launch and, where captured, the issue-active fraction."""
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
    except Exception:
        return None
    for key in (f"{kernel} (k={k})", TRAFFIC_KEYS.get(kernel, ""), f"count_trie_kernel<{k}, 2>"):
        if key in tr and (kernel == "trie" or not key.startswith("count_trie")):
            return tr[key]
    return None


def roofline_records(res, stats_avg: dict, n_tx: int, peaks: dict, sm_max: float) -> list:
    """Per generation and launch kind: {kernel, k, kernel_ms, bound, achieved, peak, unit, frac,
    traffic, ...}.  achieved = ALGORITHMIC work / the launch's CUDA-event time:
      pairs_tc        tensor: 2 |C_2| N int8 ops against the int8 dense peak = 2 x the measured bf16
                      burst peak (MEASURED_PEAKS.json; nominal int8 : bf16 = 4.5 : 2.25)
      lists           hbm: the projected-list build (pext3 / pext): every source list read once + the
                      new lists written once (build_bytes)
      count_proj      hbm: the lists of L_{k-1} read once + the counts written (count_bytes)
      pairs / trie / prefix / v0   alu: |C_k| N cand*tx against the POPC (XU) pipe: 148 SM x 16 /clk
                      (measured, profiles/r01_microbench_popc.txt) / POPC-per-word x 32 tx x f_SM
    Every number is reproducible from the line's own fields: frac = achieved / peak."""
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    bf16 = float(peaks.get("bf16_tflops", 1590.0))
    basis = "of measured" if peaks else "of fallback"
    recs = []
    n_rows = res.levels[0].n_freq
    for lv in res.levels[1:]:
        st = stats_avg.get(lv.k)
        if st is None:
            continue
        name = st["kernel_name"]
        work = lv.n_cand * n_tx
        if name == "proj":
            bms, sms = st["build_ms"], st["setup_ms"]
            cms = st["count_ms"] - bms - sms
            for kern, ms, by in (("lists", bms, st["build_bytes"]), ("count_proj", cms, st["count_bytes"])):
                ach = by / (ms * 1e-3) / 1e9
                recs.append({"kernel": kern, "k": lv.k, "kernel_ms": ms, "bound": "hbm", "achieved": ach,
                             "peak": hbm, "unit": "GB/s", "frac": ach / hbm, "algorithmic_bytes": by,
                             "peak_basis": f"HBM copy bandwidth ({basis})"})
            continue
        ms = st["count_ms"]
        if name == "pairs_tc":
            peak = 2.0 * bf16
            ach = 2.0 * work / (ms * 1e-3) / 1e12
            by = n_rows * pitch_bytes(n_tx)
            recs.append({"kernel": "pairs_tc", "k": lv.k, "kernel_ms": ms, "bound": "tensor", "achieved": ach,
                         "peak": peak, "unit": "TOPS (int8)", "frac": ach / peak, "work_cand_tx": work,
                         "algorithmic_bytes": by, "peak_basis": f"int8 dense = 2 x bf16 burst {bf16:.1f} TFLOP/s "
                                                                f"({basis})",
                         "hbm_view": {"achieved": by / (ms * 1e-3) / 1e9, "peak": hbm, "unit": "GB/s",
                                      "frac": by / (ms * 1e-3) / 1e9 / hbm}})
            continue
        ppw = 0.75 if name == "pairs" else 1.0
        peak = 148 * 16 / ppw * 32 * sm_max * 1e6 / 1e12
        ach = work / (ms * 1e-3) / 1e12
        recs.append({"kernel": name, "k": lv.k, "kernel_ms": ms, "bound": "alu", "achieved": ach, "peak": peak,
                     "unit": "Tcand*tx/s", "frac": ach / peak, "work_cand_tx": work,
                     "peak_basis": f"POPC (XU) pipe: 148 SM x 16 /clk / {ppw} POPC per 32-tx word x 32 x "
                                   f"{sm_max:.0f} MHz"})
    for r in recs:
        kern = {"lists": "pext3_kernel" if r["k"] == 3 else "pext_kernel",
                "count_proj": "count_proj_kernel<0>" if r["k"] == 3 else "count_proj_kernel<1>"}.get(r["kernel"],
                                                                                                   r["kernel"])
        t = traffic_entry(kern, r["k"])
        r["traffic"] = t.get("dram_bytes") if t else None
        for key in ("issue_active", "tensor_pipe_active", "alu_pipe_active"):
            if t and key in t:
                r[key] = t[key]
    return recs


def rescale(r: dict) -> None:
    """Recompute achieved / frac from kernel_ms (after the max over ranks)."""
    ms = r["kernel_ms"]
    if r["bound"] == "hbm":
        r["achieved"] = r["algorithmic_bytes"] / (ms * 1e-3) / 1e9
    elif r["bound"] == "tensor":
        r["achieved"] = 2.0 * r["work_cand_tx"] / (ms * 1e-3) / 1e12
    else:
        r["achieved"] = r["work_cand_tx"] / (ms * 1e-3) / 1e12
    r["frac"] = r["achieved"] / r["peak"]


def aggregate_by_kernel(recs: list) -> dict:
    out = {}
    for r in recs:
        a = out.setdefault(r["kernel"], {"bound": r["bound"], "peak": r["peak"], "unit": r["unit"], "kernel_ms": 0.0,
                                         "launches": 0, "_num": 0.0})
        a["kernel_ms"] += r["kernel_ms"]
        a["launches"] += 1
        a["_num"] += r["achieved"] * r["kernel_ms"]
    for a in out.values():
        a["achieved"] = a.pop("_num") / a["kernel_ms"] if a["kernel_ms"] > 0 else 0.0
        a["frac"] = a["achieved"] / a["peak"]
    return out


def complete_intersection_leg(args, gpa, torch, ds, theta, dist, stream, local, barrier, max_over_ranks, res_main,
                              peaks, sm_max, n_tx):
    """gpa_mine with count_kernel PAIRS + GPA_COMPLETE_INTERSECTION: popcount(AND of the candidate's
    rows) for every generation -- the paper's complete intersection (P18@394) and the north star's
    kernel, CUDA cores only.  Same inputs (resident in HBM), same K steps, CUDA events."""
    opts = gpa.Options(count_kernel=gpa.KERNEL_PAIRS, complete_intersection=True, stream=stream.cuda_stream,
                       device=local)
    d_off = torch.from_numpy(ds.offsets.view(np.int64)).cuda()
    d_items = torch.from_numpy(ds.items.view(np.int32)).cuda()
    for _ in range(max(2, min(args.warmup, 3))):   # the leg's own warm-up (its scans and plans grow buffers)
        r = gpa.mine(d_off, d_items, ds.n_items, min_count=theta, dist=dist, options=opts)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    level_stats = {}
    steps = max(1, min(args.steps, 5))
    e0.record(stream)
    for _ in range(steps):
        r = gpa.mine(d_off, d_items, ds.n_items, min_count=theta, dist=dist, options=opts)
        for lv in r.levels[1:]:
            level_stats.setdefault(lv.k, []).append(dict(lv.stats))
    e1.record(stream)
    barrier()
    ms = max_over_ranks(e0.elapsed_time(e1) / steps)
    recs = roofline_records(r, average_stats(level_stats), n_tx, peaks, sm_max)
    for x in recs:
        x["kernel_ms"] = max_over_ranks(x["kernel_ms"])
        rescale(x)
        x.pop("peak_basis", None)
    dom = dict(max(recs, key=lambda x: x["kernel_ms"]))
    dom["kernel"] = f"{dom['kernel']} (generation {dom.pop('k')}, the longest launch)"
    by = aggregate_by_kernel(recs)
    count_ms = sum(x["kernel_ms"] for x in recs)
    return {"what": "k = 2: CUDA-core AND-popcount pair Gram (count_pairs); k >= 3: trie walk / prefix streaming "
                    "over the static bitset (count_trie / count_prefix); no tensor cores, no projected lists",
            "ms_per_step": ms, "value": r.cand_tx / (ms * 1e-3), "unit": "cand*tx/s", "steps": steps,
            "count_ms": count_ms, "count_throughput": r.cand_tx / (count_ms * 1e-3),
            "identical_F": r.frequent() == res_main.frequent(), "roofline": dom, "roofline_by_kernel": by}


def main():
    args = parse()
    if args.all_configs:
        all_configs_table(args)
        return
    cfg = gen.CONFIGS[args.config]
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and rank == 0:
        print(f"# note: WORLD_SIZE={world} but --gpus={args.gpus}; using WORLD_SIZE", file=sys.stderr)
    if args.impl == "reference":
        reference_arm(args, cfg, rank, world)
        return

    import torch
    import torch.distributed as tdist
    import paper_conf_cluster_zhangzb11a_b200 as gpa

    torch.cuda.set_device(local)
    dist = None
    if world > 1 or args.dist:
        if not tdist.is_initialized():
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", "29531")
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local), rank=rank, world_size=world)
        dist = gpa.Dist.from_torch(local)

    # ---- this rank's shard of the workload (synthetic, seeded)
    b0, b1 = shard_range(cfg.n_tx, rank, world, cfg.kind == "quest")
    theta = gpa.min_count(cfg.n_tx, cfg.minsup)
    if args.emulate_shard > 1:
        b0, b1 = shard_range(cfg.n_tx, 0, args.emulate_shard, cfg.kind == "quest")
        theta = max(1, theta * (b1 - b0) // cfg.n_tx)
    ds = gen.make(cfg.name, tx_begin=b0, tx_end=b1)
    # SHA-256 of this rank's CSR bytes (offsets then items): the identity of the synthetic input
    import hashlib
    sha = hashlib.sha256()
    sha.update(np.ascontiguousarray(ds.offsets, dtype=np.uint64).data)
    sha.update(np.ascontiguousarray(ds.items, dtype=np.uint32).data)
    dataset_sha256 = sha.hexdigest()
    kern = {"auto": gpa.KERNEL_AUTO, "v0": gpa.KERNEL_V0, "prefix": gpa.KERNEL_PREFIX,
            "pairs": gpa.KERNEL_PAIRS, "trie": gpa.KERNEL_TRIE, "pairs_tc": gpa.KERNEL_PAIRS_TC,
            "proj": gpa.KERNEL_PROJ}[args.kernel]
    stream = torch.cuda.current_stream()
    opts = gpa.Options(count_kernel=kern, stream=stream.cuda_stream, device=local)
    d_off = torch.from_numpy(ds.offsets.view(np.int64)).cuda()
    d_items = torch.from_numpy(ds.items.view(np.int32)).cuda()
    torch.cuda.synchronize()

    def barrier():
        if dist is not None:
            tdist.barrier(device_ids=[local])
        torch.cuda.synchronize()

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        return float(t.item())

    # ---- warm-up
    res = None
    for _ in range(max(args.warmup, 0)):
        res = gpa.mine(d_off, d_items, ds.n_items, min_count=theta, dist=dist, options=opts)
    # ---- timed: K steps, inputs resident in HBM
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    level_stats = {}
    barrier()
    launches0 = gpa.kernel_launches()
    with ClockSampler(local) as clocks:
        ev0.record(stream)
        for _ in range(args.steps):
            res = gpa.mine(d_off, d_items, ds.n_items, min_count=theta, dist=dist, options=opts)
            for lv in res.levels[1:]:
                level_stats.setdefault(lv.k, []).append(dict(lv.stats))
        ev1.record(stream)
        barrier()
    launches = gpa.kernel_launches() - launches0   # every kernel the library launched in the region
    stats_avg = average_stats(level_stats)
    step_ms = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
    n_tx = res.n_tx
    cand_tx = res.cand_tx
    value = cand_tx / (step_ms * 1e-3)

    # ---- rooflines (roofline_records): one record per launch kind and generation, its CUDA-event
    # time measured inside the timed region on the launching stream (the library records its events
    # on the stream the caller passes), its algorithmic work / bytes from the level statistics
    peaks = load_peaks()
    clk = clocks.summary()
    sm_max = clk.get("sm_max_mhz") or peaks.get("sm_max_mhz", 1965.0)
    recs = roofline_records(res, stats_avg, n_tx, peaks, sm_max)
    for r in recs:
        r["kernel_ms"] = max_over_ranks(r["kernel_ms"])
        rescale(r)
    roof = dict(max(recs, key=lambda r: r["kernel_ms"]))   # the single longest launch
    roof["kernel"] = f"{roof['kernel']} (generation {roof.pop('k')}, the longest launch)"
    roof_all = aggregate_by_kernel(recs)

    # ---- end to end: pinned host CSR, H2D + every D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
        h_items = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
        opts_h = gpa.Options(count_kernel=kern, stream=stream.cuda_stream, device=local)
        # the host path's own warm-up (page-locked staging, result blocks): results are held as in the
        # timed loop (the previous one alive while the next is built), so both sets of the result's
        # page-locked blocks exist before timing
        r2 = None
        for _ in range(max(3, args.warmup)):
            r2 = gpa.mine(h_off, h_items, ds.n_items, min_count=theta, dist=dist, options=opts_h)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        step_times = os.environ.get("GPA_BENCH_STEP_TIMES") == "1"
        e0.record(stream)
        for _ in range(args.steps):
            t_s = time.perf_counter()
            r2 = gpa.mine(h_off, h_items, ds.n_items, min_count=theta, dist=dist, options=opts_h)
            if step_times:
                print(f"# e2e step {(time.perf_counter() - t_s) * 1e3:.1f} ms (host wall)", file=sys.stderr)
        e1.record(stream)
        barrier()
        e2e_ms = max_over_ranks(e0.elapsed_time(e1) / args.steps)
        assert r2.frequent() == res.frequent()
        h2d = int(ds.offsets.nbytes + ds.items.nbytes)
        wire = wire_bytes(ds.offsets, ds.n_items, int(os.environ.get("GPA_PACK_RAW_EVERY", "4")))
        # the histogram, and every generation's frequent itemsets (k item ids + support each)
        d2h = 4 * ds.n_items + 4 * sum(lv.n_freq * (lv.k + 1) for lv in r2.levels[1:])
        e2e = {"value": cand_tx / (e2e_ms * 1e-3), "unit": "cand*tx/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": h2d * world, "h2d_wire_bytes_per_step": wire * world,
               "d2h_bytes_per_step": d2h}

    # ---- association rules from this pass's F (outside the timed mining region): wall time
    # of gpa_rules_create (F to the device, enumeration, rules back to the host)
    rules = None
    if rank == 0 and not args.no_rules:
        minconf = "0.9"
        res.rules(minconf)   # warm-up
        torch.cuda.synchronize()
        tr0 = time.perf_counter()
        rl = res.rules(minconf)
        tr = (time.perf_counter() - tr0) * 1e3
        tested = sum(lv.n_freq * (2 ** lv.k - 2) for lv in res.levels[1:])
        rules = {"minconf": minconf, "n_rules": len(rl), "antecedents_tested": tested, "ms": tr,
                 "antecedents_per_s": tested / (tr * 1e-3)}

    # ---- the north star's own path, timed in the same run: complete intersection for every k
    # (k = 2: the CUDA-core AND-popcount pair Gram, no tensor cores; k >= 3: the trie walk / prefix
    # kernels over the static bitset, P18@394), inputs resident in HBM, same K steps
    ci = None
    if not args.no_ci:
        ci = complete_intersection_leg(args, gpa, torch, ds, theta, dist, stream, local, barrier, max_over_ranks,
                                       res, peaks, sm_max, n_tx)

    # ---- CPU baseline: the oracle on a bounded sample (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        ct, dt, threads, desc = run_oracle_sample(cfg, cpu_sample_size(cfg, args.cpu_sample_tx))
        cpu = {"value": ct / dt, "unit": "cand*tx/s", "cores": threads, "kind": "oracle", "sample": desc,
               "seconds": dt}

    if rank == 0:
        line = {
            "metric": "support-count cand*tx/s (whole mining pass)",
            "value": value,
            "unit": "cand*tx/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": step_ms,
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": cfg.name, "n_tx": n_tx, "n_items": cfg.n_items, "minsup": cfg.minsup,
                       "min_count": theta, "generations": len(res.levels), "cand_tx_per_step": cand_tx,
                       "frequent_itemsets": sum(lv.n_freq for lv in res.levels),
                       "l2_flush": "not needed: bitset 1.25 GB and CSR 1.6 GB exceed the 126 MB L2"
                       if cfg.name == "t40i10d10m" else "none (small config)",
                       "parallelism": f"tx-shard x{world}", "kernel": args.kernel,
                       "dataset_sha256": dataset_sha256},
            "roofline": roof,
            "roofline_by_kernel": roof_all,
            "cpu_baseline": cpu,
            "rules": rules,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
            "kernel_time_ms": {f"k{k}": st["count_ms"] for k, st in sorted(stats_avg.items())},
            "count_throughput": cand_tx / (sum(st["count_ms"] for st in stats_avg.values()) * 1e-3),
            "complete_intersection": ci,
            "phase_ms_last_step": res.timing_ms,
        }
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.close()
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
