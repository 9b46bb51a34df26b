"""Cached full-size oracle runs (test infrastructure; calls only ``oracle/`` and ``gen/``).

A full oracle pass over T40I10D10M takes ~2 minutes on 16 host cores, so its result -- every
generation's (C_k, counts) -- is cached under the git-ignored ``data/`` directory, keyed by the
SHA-256 of the CSR bytes (offsets then items) and the threshold.  Nothing here reads the CUDA
path: a cache file is written only from ``oracle.mine_ds`` output (``tools/oracle_cache.py`` or the
first test run that misses it) and is re-validated on load against the dataset's SHA-256.
"""
from __future__ import annotations

import hashlib
import json
import os
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
DATA = os.path.join(ROOT, "data")


def dataset_sha256(ds) -> str:
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(ds.offsets, dtype=np.uint64).tobytes())
    h.update(np.ascontiguousarray(ds.items, dtype=np.uint32).tobytes())
    return h.hexdigest()


def cache_path(sha: str, theta: int) -> str:
    return os.path.join(DATA, f"oracle_{sha[:24]}_{theta}.npz")


def load_or_run(ds, theta: int, threads: int | None = None, log=print):
    """(levels, sha, seconds): levels = [(cand (n, k) uint32, count (n,) uint32), ...] of the
    oracle on ds at theta, from the cache or from a fresh oracle run (then cached)."""
    import oracle
    sha = dataset_sha256(ds)
    path = cache_path(sha, theta)
    if os.path.exists(path):
        with np.load(path) as z:
            meta = json.loads(str(z["meta"]))
            if meta.get("sha256") == sha and meta.get("theta") == theta:
                levels = [(z[f"cand{k}"], z[f"count{k}"]) for k in range(1, meta["n_levels"] + 1)]
                log(f"oracle cache hit: {os.path.relpath(path, ROOT)} (sha256 {sha})")
                return levels, sha, 0.0
    t0 = time.perf_counter()
    ref = oracle.mine_ds(ds, theta, threads=threads)
    dt = time.perf_counter() - t0
    levels = [(lv.cand, lv.count) for lv in ref.levels]
    os.makedirs(DATA, exist_ok=True)
    arrays = {}
    for k, (c, n) in enumerate(levels, start=1):
        arrays[f"cand{k}"] = c
        arrays[f"count{k}"] = n
    meta = {"sha256": sha, "theta": theta, "n_levels": len(levels), "n_tx": ds.n_tx, "oracle_seconds": dt,
            "threads": threads or len(os.sched_getaffinity(0))}
    tmp = path + ".tmp.npz"
    np.savez(tmp, meta=json.dumps(meta), **arrays)
    os.replace(tmp, path)
    log(f"oracle run: {dt:.1f} s, cached as {os.path.relpath(path, ROOT)} (sha256 {sha})")
    return levels, sha, dt
