#!/usr/bin/env python
"""Write the cached full-size oracle results (data/oracle_<sha>_<theta>.npz) for BASELINE.json's
configurations.  Calls only oracle/ and gen/ (tests/oracle_cache.py); prints each dataset's SHA-256.

    python tools/oracle_cache.py [config ...]      (default: t40i10d10m)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import gen  # noqa: E402
import oracle  # noqa: E402
import oracle_cache  # noqa: E402

for name in sys.argv[1:] or ["t40i10d10m"]:
    cfg = gen.CONFIGS[name]
    ds = gen.make(name)
    theta = oracle.min_count(ds.n_tx, cfg.minsup)
    levels, sha, dt = oracle_cache.load_or_run(ds, theta)
    print(f"{name}: sha256 {sha} theta {theta} generations {len(levels)} "
          f"candidates {sum(len(c) for c, _ in levels[1:])} oracle {dt:.1f} s")
