#!/usr/bin/env python
"""Benchmark of the GPApriori support-counting hot path on B200.

One STEP = one full pass of the hot path over the workload:
validation + generation-1 histogram, static-bitset build, and every generation's candidate
generation, GPU support counting, (all-reduce), threshold -- i.e. one gpa_mine() call.

  value  = sum_{k>=2} |C_k| * N  /  step time     (candidate x transaction / s, whole job)
           inputs (CSR) already resident in HBM when the timed region starts;
  e2e    = the same metric through gpa_mine() with pinned HOST buffers: the H2D copy of the CSR
           and the D2H of every generation's counts are inside the timed region.

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
    level_ms, build_ms, setup_ms = {}, {}, {}
    barrier()
    launches0 = gpa.kernel_launches()
    with ClockSampler(local) as clocks:
        ev0.record(stream)
        for _ in range(args.steps):
            res = gpa.mine(d_off, d_items, ds.n_items, min_count=theta, dist=dist, options=opts)
            for lv in res.levels[1:]:
                level_ms.setdefault(lv.k, []).append(lv.stats["count_ms"])
                build_ms.setdefault(lv.k, []).append(lv.stats["build_ms"])
                setup_ms.setdefault(lv.k, []).append(lv.stats["setup_ms"])
        ev1.record(stream)
        barrier()
    launches = gpa.kernel_launches() - launches0   # every kernel the library launched in the region
    step_ms = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
    n_tx = res.n_tx
    cand_tx = res.cand_tx
    value = cand_tx / (step_ms * 1e-3)

    # ---- rooflines.  The CUDA-core counting kernels are bound by the XU pipe that executes POPC
    # (16 / clk / SM on sm_100a, profiles/r01_microbench_popc.txt), not by HBM (the bitset is
    # re-read from L2 / shared memory).  Peak in cand*tx/s = 148 SM x 16 POPC/clk / (POPC per
    # word) x 32 tx/word x f_SM:  the pair kernel counts 4 words with 3 POPC (carry-save adder)
    # -> 0.75 POPC / word; the trie / prefix / v0 kernels use 1 POPC / word.  The tensor-core pair
    # kernel (pairs_tc) is a u8 GEMM: "tensor" bound, achieved = 2 x |C_2| x N integer ops (the
    # algorithmic MACs; tile padding below the diagonal not counted) / time against the int8
    # dense peak = 2 x the measured bf16 peak (MEASURED_PEAKS.json; int8 : bf16 = 4.5 : 2.25
    # PFLOP/s nominal).  "achieved" uses the algorithmic work |C_k| x N of the launch and its
    # CUDA-event time inside the timed region.
    sm_max = None
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    clk = clocks.summary()
    sm_max = clk.get("sm_max_mhz") or peaks.get("sm_max_mhz", 1965.0)
    popc_per_word = {"pairs": 0.75}
    # ALU and FMA pipes: 64 lanes / clk / SM each (rt_SMSP = 2 cycles per warp instruction on both,
    # /opt/skills/guides/B300_MICROARCH.md "Pipe rates"), 148 SMs on B200
    int_peak = 148 * 128 * sm_max * 1e6 / 1e12
    PEXT_OPS = 17   # per member-word: HD compress 5 x (AND, shift, merge) + append (shift, OR)

    # one record per launch kind and generation: (name, k, ms per step, algorithmic work)
    recs = []
    for lv in res.levels[1:]:
        ms = float(np.mean(level_ms[lv.k]))
        if lv.stats["kernel_name"] == "proj":
            bms = float(np.mean(build_ms[lv.k]))
            sms = float(np.mean(setup_ms[lv.k]))
            recs.append(("pext", lv.k, bms, lv.stats["build_words"], lv))
            recs.append(("count_proj", lv.k, ms - bms - sms, lv.n_cand * n_tx, lv))
        else:
            recs.append((lv.stats["kernel_name"], lv.k, ms, lv.n_cand * n_tx, lv))

    def roof_for(rs):
        name = rs[0][0]
        ms = max_over_ranks(sum(r[2] for r in rs))
        work = sum(r[3] for r in rs)
        if name == "pairs_tc":
            bf16 = float(peaks.get("bf16_tflops", 2250.0 * 1965 / 1965))
            peak = 2.0 * bf16
            ach = 2.0 * work / (ms * 1e-3) / 1e12
            return {"bound": "tensor", "achieved": ach, "peak": peak, "unit": "TOPS (int8, 2 ops per cand*tx)",
                    "frac": ach / peak,
                    "peak_basis": f"int8 dense = 2 x measured bf16 {bf16:.1f} TFLOP/s (MEASURED_PEAKS.json)"
                                  if "bf16_tflops" in peaks else "int8 dense = 2 x 2250 TFLOP/s nominal bf16 (no "
                                  "MEASURED_PEAKS.json)",
                    "kernel_ms": ms, "work": work, "cand_tx_per_s": work / (ms * 1e-3)}
        if name == "pext":
            ach = work * PEXT_OPS / (ms * 1e-3) / 1e12
            return {"bound": "alu", "achieved": ach, "peak": int_peak, "unit": "T int ops/s", "frac": ach / int_peak,
                    "peak_basis": f"ALU + FMA pipes, 2 x 64 lanes/clk/SM x 148 SM x {sm_max:.0f} MHz; "
                                  f"{PEXT_OPS} algorithmic ops per compressed 32-bit mask word and member (the HD "
                                  f"compress formulation as a work-normalised rate; generation 3 runs a warp bit gather on the same work unit)",
                    "kernel_ms": ms, "work": work, "work_unit": "mask words x members"}
        if name == "count_proj":
            return {"bound": None, "achieved": work / (ms * 1e-3) / 1e12, "peak": None, "unit": "Tcand*tx/s "
                    "(effective: supports of |C_k| x N cand*tx from the projected lists)", "frac": None,
                    "kernel_ms": ms, "work": work}
        ppw = popc_per_word.get(name, 1.0)
        peak = 148 * 16 / ppw * 32 * sm_max * 1e6 / 1e12
        ach = work / (ms * 1e-3) / 1e12
        return {"bound": "alu", "achieved": ach, "peak": peak, "unit": "Tcand*tx/s", "frac": ach / peak,
                "peak_basis": f"XU pipe: 148 SM x 16 POPC/clk / {ppw} POPC per 32-tx word x 32 x {sm_max:.0f} MHz "
                              f"(POPC rate measured, profiles/r01_microbench_popc.txt)",
                "kernel_ms": ms, "work": work}

    by_kernel = {}
    for r in recs:
        by_kernel.setdefault(r[0], []).append(r)
    roof_all = {name: roof_for(rs) for name, rs in by_kernel.items()}
    dom = max(recs, key=lambda r: r[2])   # single longest launch
    roof = roof_for([dom])
    roof["kernel"] = f"{dom[0] if dom[0] == 'pext' else 'count_' + dom[0]} (generation {dom[1]}, the longest launch)"
    # DRAM traffic per launch of this kernel from the committed ncu --set full capture
    # (profiles/traffic.json, written from profiles/r*_ncu_*.txt); null if not captured
    roof["traffic"] = None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        key = {"pairs": "count_pairs_kernel", "prefix": "count_prefix_kernel", "pext": "pext3_kernel (k=3)" if dom[1] == 3 else f"pext_kernel (k={dom[1]})",
               "pairs_tc": "count_pairs_tc_kernel"}.get(dom[0], f"count_trie_kernel<{dom[1]}, 2>")
        if key in tr:
            roof["traffic"] = tr[key]["dram_bytes"]
            roof["traffic_unit"] = "bytes per launch (ncu dram__bytes_read.sum + dram__bytes_write.sum)"
            if dom[0] == "pext" and "algorithmic_bytes" in tr[key]:
                roof["algorithmic_bytes"] = tr[key]["algorithmic_bytes"]
                # the same launch against HBM: algorithmic bytes / its event time vs the measured copy bandwidth
                # (far below 1: the build is issue-bound, not memory-bound)
                if "hbm_gbs" in peaks:
                    gbs = roof["algorithmic_bytes"] / (roof["kernel_ms"] * 1e-3) / 1e9
                    roof["hbm_view"] = {"achieved": gbs, "peak": float(peaks["hbm_gbs"]), "unit": "GB/s",
                                        "frac": gbs / float(peaks["hbm_gbs"])}
            elif dom[1] == 2:   # each of the n rows read once (streaming design)
                roof["algorithmic_bytes"] = (dom[4].stats["n_groups"] + 1) * (n_tx / 8)
    except Exception:
        pass
    for r in roof_all.values():
        r.pop("peak_basis", None)

    # ---- end to end: pinned host CSR, H2D + every D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        h_off = torch.from_numpy(ds.offsets.view(np.int64)).pin_memory()
        h_items = torch.from_numpy(ds.items.view(np.int32)).pin_memory()
        opts_h = gpa.Options(count_kernel=kern, stream=stream.cuda_stream, device=local)
        gpa.mine(h_off, h_items, ds.n_items, min_count=theta, dist=dist, options=opts_h)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            r2 = gpa.mine(h_off, h_items, ds.n_items, min_count=theta, dist=dist, options=opts_h)
        e1.record(stream)
        barrier()
        e2e_ms = max_over_ranks(e0.elapsed_time(e1) / args.steps)
        assert r2.frequent() == res.frequent()
        h2d = int(ds.offsets.nbytes + ds.items.nbytes)
        # the histogram, and every generation's frequent itemsets (k item ids + support each)
        d2h = 4 * ds.n_items + 4 * sum(lv.n_freq * (lv.k + 1) for lv in r2.levels[1:])
        e2e = {"value": cand_tx / (e2e_ms * 1e-3), "unit": "cand*tx/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h}

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
                       "parallelism": f"tx-shard x{world}", "kernel": args.kernel},
            "roofline": roof,
            "roofline_by_kernel": roof_all,
            "cpu_baseline": cpu,
            "rules": rules,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
            "kernel_time_ms": {f"k{k}": float(np.mean(v)) for k, v in sorted(level_ms.items())},
            "count_throughput": cand_tx / (sum(float(np.mean(v)) for v in level_ms.values()) * 1e-3),
            "phase_ms_last_step": res.timing_ms,
        }
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.close()
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
