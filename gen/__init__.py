"""Seeded synthetic transaction databases (test / bench input only).

This module holds none of the mined method's arithmetic: it draws transactions and
returns them as a canonical CSR (each transaction sorted, duplicate-free).  It is the
only code shared by the oracle side (``oracle/``) and the CUDA side
(``paper_conf_cluster_zhangzb11a_b200``), as the build rules allow.

The five configurations are the ones BASELINE.json names; their shapes follow the
paper's Table 2 (PAPER.md P23@242-420: T40I10D100K 942 items / avg 40 / 92,113 tx,
chess 75 / 37 / 3,196, accidents 468 / 34 / 340,183) and SURVEY.md §8(d).  The FIMI
originals are not available offline; the generator families are ours (DESIGN.md
"Input recipe").
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from fractions import Fraction

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgen.so")
        if not os.path.exists(path):
            build()
        lib = ctypes.CDLL(path)
        lib.gen_quest.restype = ctypes.c_int
        lib.gen_quest.argtypes = [
            ctypes.c_uint64, ctypes.c_uint64, ctypes.c_double, ctypes.c_double, ctypes.c_uint32,
            ctypes.c_uint32, ctypes.c_double, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
            ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_uint64)]
        lib.gen_free.argtypes = [ctypes.c_void_p]
        lib.gen_chunk_size.restype = ctypes.c_uint32
        _LIB = lib
    return _LIB


def build() -> None:
    """Compile gen/quest.c into gen/libgen.so (plain C, gcc)."""
    import subprocess
    src = os.path.join(_HERE, "quest.c")
    out = os.path.join(_HERE, "libgen.so")
    if os.path.exists(out) and os.path.getmtime(out) >= os.path.getmtime(src):
        return
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", out, src, "-lm", "-lpthread"])


@dataclass
class Dataset:
    """Canonical CSR transaction database.

    offsets: uint64[n_tx+1], offsets[0] = 0;  items: uint32[offsets[-1]];  n_items: id universe.
    ``tx_begin`` is the global index of the first transaction (non-zero for a rank shard).
    """
    name: str
    offsets: np.ndarray
    items: np.ndarray
    n_items: int
    n_tx_total: int
    tx_begin: int = 0

    @property
    def n_tx(self) -> int:
        return len(self.offsets) - 1

    @property
    def nnz(self) -> int:
        return int(self.offsets[-1])

    def transactions(self):
        o = self.offsets
        return [self.items[o[i]:o[i + 1]] for i in range(self.n_tx)]


@dataclass(frozen=True)
class Config:
    name: str
    kind: str          # "quest" | "chess" | "mushroom" | "accidents"
    n_tx: int
    n_items: int
    minsup: str        # decimal string; min_count = max(1, ceil(minsup * N)) exactly (Q2)
    seed: int
    avg_tx: float = 0.0
    avg_pat: float = 0.0
    n_pat: int = 0

    @property
    def minsup_fraction(self) -> Fraction:
        return Fraction(self.minsup)


CONFIGS = {
    "chess": Config("chess", "chess", 3196, 75, "0.90", 1),
    "mushroom": Config("mushroom", "mushroom", 8124, 119, "0.20", 2),
    "t40i10d100k": Config("t40i10d100k", "quest", 100_000, 1000, "0.01", 3, 40.0, 10.0, 2000),
    "accidents": Config("accidents", "accidents", 340_183, 468, "0.30", 4),
    "t40i10d10m": Config("t40i10d10m", "quest", 10_000_000, 1000, "0.005", 5, 40.0, 10.0, 2000),
}


def chunk_size() -> int:
    """Quest transactions are generated in independent chunks of this many (a multiple of 512)."""
    return int(_lib().gen_chunk_size())


def quest(seed: int, n_tx: int, n_items: int, avg_tx: float, avg_pat: float, n_pat: int,
          tx_begin: int = 0, tx_end: int | None = None, corr: float = 0.5, threads: int | None = None,
          name: str = "quest") -> Dataset:
    """IBM-Quest-style transactions [tx_begin, tx_end) of an n_tx database (C generator)."""
    lib = _lib()
    if tx_end is None:
        tx_end = n_tx
    if threads is None:
        threads = max(1, min(32, len(os.sched_getaffinity(0))))
    po, pi, nnz = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_uint64()
    rc = lib.gen_quest(seed, n_tx, avg_tx, avg_pat, n_items, n_pat, corr, tx_begin, tx_end, threads,
                       ctypes.byref(po), ctypes.byref(pi), ctypes.byref(nnz))
    if rc != 0:
        raise ValueError("gen_quest: bad arguments (tx_begin must be a multiple of chunk_size())")
    n = tx_end - tx_begin
    try:
        offsets = np.ctypeslib.as_array(ctypes.cast(po, ctypes.POINTER(ctypes.c_uint64)), (n + 1,)).copy()
        items = (np.ctypeslib.as_array(ctypes.cast(pi, ctypes.POINTER(ctypes.c_uint32)), (max(nnz.value, 1),))
                 [: nnz.value].copy())
    finally:
        lib.gen_free(po)
        lib.gen_free(pi)
    return Dataset(name, offsets, items, n_items, n_tx, tx_begin)


def _attribute_db(name: str, rng: np.random.Generator, n_tx: int, cards: list[int], value_probs,
                  cls: np.ndarray, present: np.ndarray) -> Dataset:
    """Attribute-value transactions: attribute a contributes item offset[a] + value when present.

    value_probs[a] is a (n_classes, cards[a]) matrix of per-class value probabilities; cls is the
    latent class of each transaction; present is a bool (n_tx, n_attr) mask.  Items come out sorted
    because attribute offsets are increasing and each attribute contributes at most one item.
    """
    offs = np.concatenate([[0], np.cumsum(cards)]).astype(np.int64)
    cols = []
    for a, card in enumerate(cards):
        cdf = np.cumsum(value_probs[a], axis=1)
        cdf[:, -1] = 1.0
        u = rng.random(n_tx)
        v = (u[:, None] >= cdf[cls]).sum(axis=1)
        v = np.minimum(v, card - 1)
        cols.append(offs[a] + v)
    mat = np.stack(cols, axis=1).astype(np.uint32)
    lens = present.sum(axis=1).astype(np.uint64)
    offsets = np.zeros(n_tx + 1, dtype=np.uint64)
    np.cumsum(lens, out=offsets[1:])
    items = mat[present]  # row-major: per transaction, attributes in increasing order
    return Dataset(name, offsets, items.astype(np.uint32), int(offs[-1]), n_tx)


def chess(seed: int = 1, n_tx: int = 3196) -> Dataset:
    """chess-shaped: 36 binary + 1 ternary attribute = 75 items, exactly 37 items per transaction.

    Dominant-value probability d_a = 0.999 - 0.5 (a/36)^2.
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    cards = [2] * 36 + [3]
    probs = []
    for a, c in enumerate(cards):
        d = 0.999 - 0.5 * (a / 36.0) ** 2
        p = np.full(c, (1.0 - d) / (c - 1))
        p[rng.integers(c)] = d
        probs.append(p[None, :])
    cls = np.zeros(n_tx, dtype=np.int64)
    present = np.ones((n_tx, len(cards)), dtype=bool)
    return _attribute_db("chess", rng, n_tx, cards, probs, cls, present)


MUSHROOM_CARDS = [2, 6, 4, 10, 2, 9, 2, 2, 2, 12, 2, 5, 4, 4, 9, 9, 1, 4, 3, 5, 9, 6, 7]


def mushroom(seed: int = 2, n_tx: int = 8124) -> Dataset:
    """mushroom-shaped: 23 attributes (UCI cardinalities, 119 items), exactly 23 items per transaction.

    A 2-value latent class (P = 0.518 / 0.482) is attribute 0 itself; every other attribute's
    per-class value distribution is Dirichlet(0.3).
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    cls = (rng.random(n_tx) >= 0.518).astype(np.int64)
    probs = []
    for a, c in enumerate(MUSHROOM_CARDS):
        if a == 0:
            probs.append(np.eye(2))
        else:
            probs.append(rng.dirichlet(np.full(c, 0.3), size=2))
    present = np.ones((n_tx, len(MUSHROOM_CARDS)), dtype=bool)
    return _attribute_db("mushroom", rng, n_tx, MUSHROOM_CARDS, probs, cls, present)


def accidents(seed: int = 4, n_tx: int = 340_183) -> Dataset:
    """accidents-shaped: 29 always-present + 11 optional (p = 0.45) attributes, 468 items.

    Four latent classes (P = .4/.3/.2/.1).  Each attribute has a dominant value whose
    probability is drawn from U(0.35, 0.95) and perturbed per class by N(0, 0.05); the other
    values share the rest by a Zipf(1.2) law over a seeded permutation.  Calibrated so that at
    minsup 0.30 about 36 items are frequent and mining runs 8 levels deep.
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    n_attr_fixed, n_attr_opt = 29, 11
    n_attr = n_attr_fixed + n_attr_opt
    # cardinalities >= 2 summing to 468
    raw = rng.dirichlet(np.full(n_attr, 1.2)) * (468 - 2 * n_attr)
    cards = (np.floor(raw).astype(int) + 2).tolist()
    for i in range(468 - sum(cards)):
        cards[i % n_attr] += 1
    n_cls = 4
    cls = rng.choice(n_cls, size=n_tx, p=[0.4, 0.3, 0.2, 0.1])
    probs = []
    for c in cards:
        d = 0.35 + 0.6 * rng.random()
        rest = 1.0 / np.arange(1, c) ** 1.2
        rest /= rest.sum()
        dom = int(rng.integers(c))
        others = np.array([v for v in range(c) if v != dom])
        m = np.zeros((n_cls, c))
        for k in range(n_cls):
            dk = float(np.clip(d + 0.05 * rng.normal(), 0.01, 0.995))
            m[k, dom] = dk
            m[k, others[rng.permutation(c - 1)]] = (1.0 - dk) * rest
        probs.append(m)
    present = np.ones((n_tx, n_attr), dtype=bool)
    present[:, n_attr_fixed:] = rng.random((n_tx, n_attr_opt)) < 0.45
    return _attribute_db("accidents", rng, n_tx, cards, probs, cls, present)


def make(name: str, tx_begin: int = 0, tx_end: int | None = None, n_tx: int | None = None) -> Dataset:
    """Generate configuration ``name`` (or its transactions [tx_begin, tx_end)).

    ``n_tx`` overrides the database size (used for bounded samples); Quest shards must start on
    a multiple of chunk_size().
    """
    cfg = CONFIGS[name]
    total = cfg.n_tx if n_tx is None else n_tx
    if tx_end is None:
        tx_end = total
    if cfg.kind == "quest":
        return quest(cfg.seed, total, cfg.n_items, cfg.avg_tx, cfg.avg_pat, cfg.n_pat, tx_begin, tx_end, name=name)
    full = {"chess": chess, "mushroom": mushroom, "accidents": accidents}[cfg.kind](cfg.seed, total)
    return subset(full, tx_begin, tx_end)


def subset(ds: Dataset, tx_begin: int, tx_end: int) -> Dataset:
    """Contiguous transaction range of a dataset (a rank shard or a bounded sample)."""
    o = ds.offsets
    offsets = (o[tx_begin:tx_end + 1] - o[tx_begin]).astype(np.uint64)
    items = ds.items[o[tx_begin]:o[tx_end]].copy()
    return Dataset(ds.name, offsets, items, ds.n_items, ds.n_tx_total, ds.tx_begin + tx_begin)


def random_db(seed: int, n_tx: int, n_items: int, max_len: int, p_empty: float = 0.1,
              duplicates: bool = False, unsorted: bool = False) -> Dataset:
    """Small random database for parity tests: lengths uniform in [0, max_len], optional
    duplicate / unsorted items inside a transaction (non-canonical input), empty transactions."""
    rng = np.random.Generator(np.random.PCG64(seed))
    rows = []
    # skewed item popularity so that deep itemsets are frequent
    pop = rng.dirichlet(np.full(n_items, 0.5))
    for _ in range(n_tx):
        if rng.random() < p_empty:
            rows.append(np.zeros(0, dtype=np.uint32))
            continue
        ln = int(rng.integers(1, max_len + 1))
        ln = min(ln, n_items)
        t = rng.choice(n_items, size=ln, replace=False, p=pop).astype(np.uint32)
        if duplicates and ln > 0 and rng.random() < 0.5:
            t = np.concatenate([t, t[: max(1, ln // 3)]])
        if not unsorted:
            t = np.unique(t)
        else:
            rng.shuffle(t)
        rows.append(t)
    lens = np.array([len(r) for r in rows], dtype=np.uint64)
    offsets = np.zeros(n_tx + 1, dtype=np.uint64)
    np.cumsum(lens, out=offsets[1:])
    items = np.concatenate(rows).astype(np.uint32) if rows and offsets[-1] > 0 else np.zeros(0, np.uint32)
    return Dataset("random", offsets, items, n_items, n_tx)


def from_lists(txs, n_items: int, name: str = "lists") -> Dataset:
    """CSR from a list of item lists (kept as given: no sorting / dedup)."""
    lens = np.array([len(t) for t in txs], dtype=np.uint64)
    offsets = np.zeros(len(txs) + 1, dtype=np.uint64)
    np.cumsum(lens, out=offsets[1:])
    items = (np.concatenate([np.asarray(t, dtype=np.uint32) for t in txs]) if offsets[-1] > 0
             else np.zeros(0, np.uint32))
    return Dataset(name, offsets, items.astype(np.uint32), n_items, len(txs))

