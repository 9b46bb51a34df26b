"""Host-side logic of the GPU path, tested on CPU: the library's own join + prune candidate
generation (runtime/candgen.cpp, compiled here into a test shim) against the oracle's
independent implementation and against the definition; and the grouping invariants the counting
kernels rely on (lexicographic order, groups = (k-1)-prefix runs)."""
import ctypes
import os
import subprocess
from itertools import combinations

import numpy as np
import pytest

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_cluster_zhangzb11a_b200", "csrc")


@pytest.fixture(scope="module")
def shim(tmp_path_factory):
    import nvidia.nccl
    nccl = list(nvidia.nccl.__path__)[0]
    out = tmp_path_factory.mktemp("shim") / "libcandgen_shim.so"
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-I", CSRC, "-I",
                           os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include", "-I",
                           os.path.join(nccl, "include"), os.path.join(ROOT, "tests", "cpp", "candgen_shim.cpp"),
                           os.path.join(CSRC, "runtime", "candgen.cpp"), os.path.join(CSRC, "runtime", "pool.cpp"), "-o", str(out)])
    lib = ctypes.CDLL(str(out))
    lib.shim_candgen.restype = ctypes.c_int
    lib.shim_plan_trie.restype = ctypes.c_int
    return lib


def run_shim(lib, L):
    L = np.ascontiguousarray(L, dtype=np.uint32)
    n, km1 = L.shape
    cap = max(16, n * n)
    pre = np.zeros(cap * km1 + 1, np.uint32)
    off = np.zeros(cap + 2, np.uint64)
    ext = np.zeros(cap + 1, np.uint32)
    ng, nc = ctypes.c_uint64(), ctypes.c_uint64()
    rc = lib.shim_candgen(L.ctypes.data_as(ctypes.c_void_p), ctypes.c_uint64(n), ctypes.c_uint32(km1),
                          pre.ctypes.data_as(ctypes.c_void_p), off.ctypes.data_as(ctypes.c_void_p),
                          ext.ctypes.data_as(ctypes.c_void_p), ctypes.c_uint64(cap), ctypes.byref(ng), ctypes.byref(nc))
    assert rc == 0
    G, M = ng.value, nc.value
    pre = pre[: G * km1].reshape(G, km1)
    off = off[: G + 1]
    ext = ext[:M]
    cands = []
    for g in range(G):
        assert off[g + 1] > off[g]  # groups are non-empty
        for j in range(int(off[g]), int(off[g + 1])):
            cands.append(tuple(int(x) for x in pre[g]) + (int(ext[j]),))
    return cands, pre, off


@pytest.mark.parametrize("seed", range(10))
def test_candgen_matches_oracle_and_definition(shim, seed):
    rng = np.random.default_rng(seed)
    n, km1 = 10, int(rng.integers(1, 5))
    allsets = list(combinations(range(n), km1))
    L = sorted(s for s in allsets if rng.random() < 0.6)
    if not L:
        return
    got, pre, off = run_shim(shim, np.array(L, dtype=np.uint32).reshape(-1, km1))
    ref = [tuple(map(int, r)) for r in oracle.candgen(np.array(L, dtype=np.uint32).reshape(-1, km1))]
    Ls = set(L)
    defn = [X for X in combinations(range(n), km1 + 1) if all(S in Ls for S in combinations(X, km1))]
    assert got == ref == defn
    # groups are distinct (k-1)-prefixes in increasing order
    assert [tuple(p) for p in pre.tolist()] == sorted(set(tuple(p) for p in pre.tolist()))


@pytest.mark.parametrize("name", ["mushroom", "chess"])
def test_candgen_real_levels(shim, name):
    """Every generation of a real mining run, incl. the threaded path (large L)."""
    ds = gen.make(name)
    theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    r = oracle.mine_ds(ds, theta)
    for lv, nxt in zip(r.levels[1:], r.levels[2:]):
        L = lv.cand[lv.count >= theta]
        got, _, _ = run_shim(shim, L)
        assert got == [tuple(map(int, x)) for x in nxt.cand]


def test_candgen_threaded_large(shim):
    """A large L_2 (~20k pairs) forces the multi-threaded split; result must equal the oracle's."""
    rng = np.random.default_rng(3)
    pairs = sorted({tuple(sorted(rng.choice(400, 2, replace=False))) for _ in range(20000)})
    L = np.array(pairs, dtype=np.uint32)
    got, _, _ = run_shim(shim, L)
    assert got == [tuple(map(int, x)) for x in oracle.candgen(L)]


def run_plan(lib, L, n_rows):
    L = np.ascontiguousarray(L, dtype=np.uint32)
    n, km1 = L.shape
    k = km1 + 1
    cap = max(64, n * n)
    blocks = np.zeros(cap * 4, np.uint32)
    rows = np.zeros(cap, np.uint32)
    lrows = np.zeros(cap * 16, np.uint8)
    lcp = np.zeros(cap, np.uint8)
    cand = np.zeros(cap * k, np.uint32)
    nb, nr, nc = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
    P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
    rc = lib.shim_plan_trie(P(L), ctypes.c_uint64(n), ctypes.c_uint32(km1), ctypes.c_uint32(n_rows), P(blocks),
                            ctypes.byref(nb), P(rows), ctypes.byref(nr), P(lrows), P(lcp), P(cand),
                            ctypes.c_uint64(cap), ctypes.byref(nc))
    assert rc == 0
    M = nc.value
    return (blocks[: nb.value * 4].reshape(-1, 4), rows[: nr.value], lrows[: M * 16].reshape(M, 16), lcp[:M],
            cand[: M * k].reshape(M, k))


@pytest.mark.parametrize("name,k", [("mushroom", 3), ("mushroom", 5), ("chess", 4), ("random", 3), ("random", 9),
                                    ("dense", 3)])
def test_trie_plan_invariants(shim, name, k):
    """Blocks tile the candidates in order with <= 256 candidates and <= trie_max_rows(k) rows;
    local row bytes map back to each candidate's rows; lcp is the shared prefix with the previous
    candidate, reset to 0 at every warp chunk (ceil(n/8)) start -- what count_trie assumes."""
    if name == "dense":  # all pairs of 80 rows: 82,160 candidates -> the parallel (multi-range) plan
        L = np.array(list(combinations(range(80), 2)), np.uint32)
        n_rows = 80
    elif name == "random":
        rng = np.random.default_rng(k)
        L = np.array(sorted({tuple(sorted(rng.choice(300, k - 1, replace=False))) for _ in range(6000)}), np.uint32)
        L = np.array(sorted({tuple(x) for x in L.tolist()} |
                            {tuple([0, 1, 2, 3, 4, 5, 6, 7][: k - 2]) + (q,) for q in range(8, 200)}), np.uint32)
        n_rows = 300
    else:
        ds = gen.make(name)
        theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
        r = oracle.mine_ds(ds, theta)
        lv = r.levels[k - 2]
        L = lv.cand[lv.count >= theta]
        n_rows = ds.n_items
    blocks, rows, lrows, lcp, cand = run_plan(shim, L, n_rows)
    M = len(cand)
    if M == 0:
        return
    rmax = 32 if k >= 3 else 64
    pos = 0
    for cb, nc, rb, nr in blocks.tolist():
        assert cb == pos and 0 < nc <= 256 and nr <= rmax
        chunk = (nc + 7) // 8
        for i in range(nc):
            c = cb + i
            assert [int(rows[rb + int(lrows[c, d])]) for d in range(k)] == cand[c].tolist()
            assert all(lrows[c, d] < nr for d in range(k))
            if i % chunk == 0:
                assert lcp[c] == 0
            else:
                l = 0
                while l < k - 1 and cand[c, l] == cand[c - 1, l]:
                    l += 1
                assert lcp[c] == l
        pos += nc
    assert pos == M


# ---------------------------------------------------------------- projected lists (proj.cu)

SEG_W = 2048   # proj.cu kSegW: mask segment of 2,048 words (u16 positions)


def _segment_positions(mask):
    """proj.cu pos_kernel: per segment, the segment-relative positions (word << 5 | bit) of the
    mask's set bits, in increasing order, as u16."""
    out = []
    for s0 in range(0, len(mask), SEG_W):
        seg = mask[s0:s0 + SEG_W]
        bits = np.unpackbits(seg.view(np.uint8), bitorder="little")
        out.append(np.nonzero(bits)[0].astype(np.uint16))
    return out


def _gather_list(mask, src):
    """proj.cu gather_item: per segment, rounds of 32 positions; round r's word = ballot over lanes
    l of bit (pos[32r + l] & 31) of src word (segment base + pos >> 5); words padded per segment,
    the list padded to a multiple of 4 words with zeros."""
    words = []
    for s, pos in enumerate(_segment_positions(mask)):
        for r in range(0, len(pos), 32):
            w = 0
            for lane, v in enumerate(pos[r:r + 32].tolist()):
                x = int(src[s * SEG_W + (v >> 5)])
                if x >> (v & 31) & 1:
                    w |= 1 << lane
            words.append(w)
    words += [0] * (-len(words) % 4)
    return np.array(words, dtype=np.uint32)


def _bits(words):
    return np.unpackbits(np.asarray(words, dtype=np.uint32).view(np.uint8), bitorder="little")


def test_gather_lists_match_definition():
    """The projected-list layout of proj.cu (segment positions + ballot gather, per-segment word
    padding): dropping each segment's padding bits gives exactly the definition -- the bits of the
    source at the set positions of the mask, in order (V_X[i] = B[x][t_i]); and the
    padded lists of one class give the same popcount-of-AND supports as the unpadded definition."""
    rng = np.random.default_rng(11)
    for trial, (n_words, dens) in enumerate([(100, 0.05), (SEG_W, 0.3), (SEG_W + 37, 0.02), (2 * SEG_W + 4, 0.6),
                                             (5000, 0.0), (64, 1.0)]):
        mask = (rng.random(n_words * 32) < dens)
        mk = np.packbits(mask, bitorder="little").view(np.uint32)
        srcs = [np.packbits(rng.random(n_words * 32) < 0.4, bitorder="little").view(np.uint32) for _ in range(3)]
        lists = [_gather_list(mk, s) for s in srcs]
        segs = _segment_positions(mk)
        for s, L in zip(srcs, lists):
            assert len(L) % 4 == 0
            b = _bits(L)
            got, at = [], 0
            for pos in segs:          # drop the per-segment padding bits
                got.append(b[at:at + len(pos)])
                at += (len(pos) + 31) // 32 * 32
            assert not b[at:].any()
            got = np.concatenate(got) if got else np.zeros(0, np.uint8)
            want = _bits(s)[np.nonzero(mask)[0]]
            assert np.array_equal(got, want), trial
        # supports of {a, b} within the class = popc(AND) of the padded lists
        for i in range(3):
            for j in range(i + 1, 3):
                want = int((_bits(srcs[i]) & _bits(srcs[j]) & mask).sum())
                assert int((_bits(lists[i]) & _bits(lists[j])).sum()) == want
