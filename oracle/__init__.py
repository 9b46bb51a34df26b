"""CPU oracle for GPApriori support counting -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_cluster_zhangzb11a_b200``); neither imports the other.  The arithmetic lives in
``apriori_oracle.c`` (plain C, gcc); this file is ctypes marshalling only.  See the C file's
header for the paper passages each function follows and DESIGN.md for the readings taken.

Parity status: every function here is pinned (tests/test_oracle_*.py); none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from fractions import Fraction

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "apriori_oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_LIB = None


def build() -> None:
    """Compile apriori_oracle.c -> liboracle.so (building the checker is not using it)."""
    if os.path.exists(_SO) and os.path.getmtime(_SO) >= os.path.getmtime(_SRC):
        return
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-Wall", "-o", _SO, _SRC, "-lpthread"])


class _Level(ctypes.Structure):
    _fields_ = [("k", ctypes.c_uint32), ("n_cand", ctypes.c_uint64),
                ("cand", ctypes.POINTER(ctypes.c_uint32)), ("count", ctypes.POINTER(ctypes.c_uint32))]


class _Result(ctypes.Structure):
    _fields_ = [("n_tx", ctypes.c_uint64), ("min_count", ctypes.c_uint64), ("n_items", ctypes.c_uint32),
                ("n_levels", ctypes.c_uint32), ("levels", ctypes.POINTER(_Level))]


def _lib():
    global _LIB
    if _LIB is None:
        build()
        lib = ctypes.CDLL(_SO)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        lib.oracle_min_count.restype = ctypes.c_uint64
        lib.oracle_min_count.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        lib.oracle_support.restype = ctypes.c_int
        lib.oracle_support.argtypes = [u64p, u32p, ctypes.c_uint64, ctypes.c_uint32, u32p, ctypes.c_uint32,
                                       ctypes.c_int, u64p]
        lib.oracle_support_batch.restype = ctypes.c_int
        lib.oracle_support_batch.argtypes = [u64p, u32p, ctypes.c_uint64, ctypes.c_uint32, u32p,
                                             ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, u64p]
        lib.oracle_candgen.restype = ctypes.c_int
        lib.oracle_candgen.argtypes = [u32p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                                       ctypes.POINTER(u32p), u64p]
        lib.oracle_mine.restype = ctypes.c_int
        lib.oracle_mine.argtypes = [u64p, u32p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int,
                                    ctypes.POINTER(ctypes.POINTER(_Result))]
        lib.oracle_result_free.argtypes = [ctypes.POINTER(_Result)]
        _LIB = lib
    return _LIB


def _threads(n):
    return max(1, len(os.sched_getaffinity(0))) if n is None else int(n)


def _u64(a):
    a = np.ascontiguousarray(a, dtype=np.uint64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


def _u32(a):
    a = np.ascontiguousarray(a, dtype=np.uint32)
    if a.size == 0:
        a = np.zeros(1, dtype=np.uint32)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


def min_count(n_tx: int, minsup: str | Fraction) -> int:
    """max(1, ceil(minsup * n_tx)), minsup an exact decimal fraction (Q2)."""
    f = Fraction(minsup)
    return int(_lib().oracle_min_count(n_tx, f.numerator, f.denominator))


@dataclass
class Level:
    k: int
    cand: np.ndarray     # (n_cand, k) uint32 original item ids, lexicographic
    count: np.ndarray    # (n_cand,) uint32


@dataclass
class MineResult:
    n_tx: int
    min_count: int
    n_items: int
    levels: list = field(default_factory=list)   # levels[0] is k = 1

    def frequent(self) -> dict:
        """F as {tuple(itemset): support}."""
        out = {}
        for lv in self.levels:
            keep = lv.count >= self.min_count
            for row, c in zip(lv.cand[keep], lv.count[keep]):
                out[tuple(int(x) for x in row)] = int(c)
        return out

    def level_map(self, k: int) -> dict:
        lv = self.levels[k - 1]
        return {tuple(int(x) for x in row): int(c) for row, c in zip(lv.cand, lv.count)}


def mine(offsets, items, n_items: int, min_count_: int, threads: int | None = None) -> MineResult:
    """Level-wise Apriori over the horizontal layout; every generation's (C_k, counts) kept."""
    lib = _lib()
    o, op = _u64(offsets)
    it, ip = _u32(items)
    n_tx = len(o) - 1
    res = ctypes.POINTER(_Result)()
    rc = lib.oracle_mine(op, ip, n_tx, n_items, min_count_, _threads(threads), ctypes.byref(res))
    if rc != 0:
        raise ValueError(f"oracle_mine: invalid database (code {rc})")
    try:
        R = res.contents
        out = MineResult(int(R.n_tx), int(R.min_count), int(R.n_items))
        for i in range(R.n_levels):
            L = R.levels[i]
            n, k = int(L.n_cand), int(L.k)
            cand = np.ctypeslib.as_array(L.cand, (max(n * k, 1),))[: n * k].copy().reshape(n, k)
            cnt = np.ctypeslib.as_array(L.count, (max(n, 1),))[:n].copy()
            out.levels.append(Level(k, cand, cnt))
    finally:
        lib.oracle_result_free(res)
    return out


def mine_ds(ds, min_count_: int, threads: int | None = None) -> MineResult:
    return mine(ds.offsets, ds.items, ds.n_items, min_count_, threads)


def support(offsets, items, n_items: int, itemset, threads: int | None = None) -> int:
    """supp(X) by the literal definition: one subset test per transaction."""
    lib = _lib()
    o, op = _u64(offsets)
    it, ip = _u32(items)
    x, xp = _u32(list(itemset))
    s = ctypes.c_uint64()
    rc = lib.oracle_support(op, ip, len(o) - 1, n_items, xp, len(list(itemset)), _threads(threads), ctypes.byref(s))
    if rc != 0:
        raise ValueError("oracle_support: invalid database")
    return int(s.value)


def support_batch(offsets, items, n_items: int, itemsets: np.ndarray, threads: int | None = None) -> np.ndarray:
    """Literal supports of M sorted k-itemsets ((M, k) array)."""
    lib = _lib()
    X = np.ascontiguousarray(itemsets, dtype=np.uint32)
    M, k = X.shape
    o, op = _u64(offsets)
    it, ip = _u32(items)
    xs, xp = _u32(X.reshape(-1))
    out = np.zeros(max(M, 1), dtype=np.uint64)
    rc = lib.oracle_support_batch(op, ip, len(o) - 1, n_items, xp, k, M, _threads(threads),
                                  out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
    if rc != 0:
        raise ValueError(f"oracle_support_batch: invalid input (code {rc})")
    return out[:M]


def candgen(L: np.ndarray, prune: bool = True) -> np.ndarray:
    """C_k from L_{k-1} ((n, k-1) lexicographically sorted array): join (+ prune)."""
    lib = _lib()
    L = np.ascontiguousarray(L, dtype=np.uint32)
    n, km1 = L.shape
    Lb, lp = _u32(L.reshape(-1))
    cp = ctypes.POINTER(ctypes.c_uint32)()
    nc = ctypes.c_uint64()
    lib.oracle_candgen(lp, n, km1, 1 if prune else 0, ctypes.byref(cp), ctypes.byref(nc))
    k = km1 + 1
    m = int(nc.value)
    out = np.ctypeslib.as_array(cp, (max(m * k, 1),))[: m * k].copy().reshape(m, k) if m else np.zeros((0, k), np.uint32)
    ctypes.CDLL(None).free(ctypes.cast(cp, ctypes.c_void_p))
    return out


def rules(F: dict, minconf, itemsets=None) -> dict:
    """Association rules from F ({itemset tuple: support}) by their definition (Q19,
    Agrawal & Srikant ref [2]): for every X in F with |X| >= 2 and every non-empty proper subset A
    of X, A => X \\ A when supp(X) / supp(A) >= minconf, compared exactly (Fraction).  Plain Python,
    for small F (or a few ``itemsets`` X of a large F).  Returns {(A, X \\ A): (supp(X), supp(A))}."""
    from itertools import combinations
    mc = Fraction(str(minconf)) if not isinstance(minconf, Fraction) else minconf
    out = {}
    for X in (F if itemsets is None else itemsets):
        sx = F[X]
        if len(X) < 2:
            continue
        for r in range(1, len(X)):
            for A in combinations(X, r):
                sa = F[A]
                if Fraction(sx, sa) >= mc:
                    out[(A, tuple(v for v in X if v not in A))] = (sx, sa)
    return out
