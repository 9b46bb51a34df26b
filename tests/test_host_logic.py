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

def _hd_compress(x, m):
    """The operation sequence of proj.cu's hd_prep / hd_apply (Hacker's Delight 7-4 compress,
    right shifts as umulhi by 2^(32-s), left shifts as multiplies), vectorised over uint32."""
    M32 = np.uint64(0xFFFFFFFF)
    x = x.astype(np.uint64)
    m = m.astype(np.uint64)

    def shl(v, s):
        return (v * np.uint64(1 << s)) & M32

    def shr(v, s):
        return (v * np.uint64(1 << (32 - s))) >> np.uint64(32)

    mk = shl(~m & M32, 1)
    mv = []
    mm = m.copy()
    for i in range(5):
        mp = mk ^ shl(mk, 1)
        for sh in (2, 4, 8, 16):
            mp ^= shl(mp, sh)
        v = mp & mm
        mv.append(v)
        mm = (mm ^ v) | shr(v, 1 << i)
        mk &= ~mp & M32
    t = x & mv[0]
    y = (x & m & (~mv[0] & M32)) | shr(t, 1)
    for i in range(1, 5):
        t = y & mv[i]
        y = (y & (~mv[i] & M32)) | shr(t, 1 << i)
    return y.astype(np.uint32)


def _pext_ref(x, m):
    out = np.zeros_like(x)
    k = np.zeros_like(x)
    for i in range(32):
        sel = (m >> np.uint32(i)) & np.uint32(1)
        bit = (x >> np.uint32(i)) & np.uint32(1)
        out |= (bit & sel) << k
        k += sel
    return out


def test_compress_matches_pext():
    """proj.cu's parallel bit extract equals the bit-by-bit definition (random, sparse, dense,
    empty and full masks)."""
    rng = np.random.default_rng(11)
    n = 200_000
    x = rng.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    m = rng.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    m[::3] &= rng.integers(0, 2 ** 32, len(m[::3]), dtype=np.uint64).astype(np.uint32)   # sparse
    m[1::7] = 0xFFFFFFFF
    m[2::11] = 0
    m[3::13] = 0x80000001
    assert np.array_equal(_hd_compress(x, m), _pext_ref(x, m))


def _sparse_compress(x, m):
    """The sparse-mask sequence of proj.cu's pext_item<G, true> (generation 3): the mask's trailing
    ones stay, every further set bit p of rank i comes from bit i of (x >> (p - i)), the shift as
    umulhi(x, 2^(32 - (p - i)))."""
    c = bin(m).count("1")
    i0 = 32 if m == 0xFFFFFFFF else ((~m & 0xFFFFFFFF) & -(~m & 0xFFFFFFFF)).bit_length() - 1
    idm = 0xFFFFFFFF if i0 >= 32 else (1 << i0) - 1
    y, mm, i = x & idm, m & ~idm & 0xFFFFFFFF, i0
    for _ in range(c - min(i0, c)):
        p = (mm & -mm).bit_length() - 1
        mm &= mm - 1
        y |= ((x * (1 << (32 - (p - i)))) >> 32) & (1 << i)
        i += 1
    return y


def test_sparse_compress_matches_pext():
    rng = np.random.default_rng(12)
    xs = rng.integers(0, 2 ** 32, 20000, dtype=np.uint64).tolist()
    ms = rng.integers(0, 2 ** 32, 20000, dtype=np.uint64)
    ms[::2] &= rng.integers(0, 2 ** 32, 10000, dtype=np.uint64) & rng.integers(0, 2 ** 32, 10000, dtype=np.uint64)
    ms[1::9] = 0xFFFFFFFF
    ms[2::11] = 0
    ms[3::13] = 0x0000FFFF | 0x80000000
    ms = ms.tolist()
    ref = _pext_ref(np.array(xs, dtype=np.uint32), np.array(ms, dtype=np.uint32)).tolist()
    assert [_sparse_compress(x, m) for x, m in zip(xs, ms)] == ref


def _seg3_words(counts):
    """proj_dev.cuh seg3_warp: words of one (segment, class) -- its set bits packed densely."""
    return (sum(counts) + 31) // 32


def _pext3_pack(mask_chunks, member_chunks):
    """pext3_kernel's packing of one (segment, class) written out step by step: per 64-word chunk
    (lane l holds words 2l, 2l + 1) the set bits are ranked in word order; ballot t takes rank
    32 t + r - pend at lane r (nothing outside [0, C)); every ballot ORs into the open slot (slots
    zeroed after each flush of 32 words); a ballot that fills its word moves to the next slot, the
    last partial one stays open (pend bits) for the next chunk.  Returns per-member word lists."""
    n_mem = len(member_chunks)
    keep = [[0] * 32 for _ in range(n_mem)]
    out = [[] for _ in range(n_mem)]
    wc = pend = 0
    for j, mw in enumerate(mask_chunks):
        pos = [(wi << 5) | b for wi in range(64) for b in range(32) if (int(mw[wi]) >> b) & 1]
        C = len(pos)
        if C == 0:
            continue
        tot = pend + C
        full, nb = tot >> 5, (tot >> 5) + (1 if tot & 31 else 0)
        for t in range(nb):
            for q in range(n_mem):
                b = 0
                for r in range(32):
                    rank = 32 * t + r - pend
                    if 0 <= rank < C:
                        code = pos[rank]
                        b |= ((int(member_chunks[q][j][code >> 5]) >> (code & 31)) & 1) << r
                keep[q][wc & 31] |= b
            if t < full:
                wc += 1
                if wc % 32 == 0:
                    for q in range(n_mem):
                        out[q] += keep[q]
                        keep[q] = [0] * 32
        pend = tot & 31
    left = (wc & 31) + (1 if pend else 0)
    for q in range(n_mem):
        out[q] += keep[q][:left]
    return out


@pytest.mark.parametrize("density", [0.002, 0.02, 0.05, 0.3, 0.9])
def test_pext3_carry_packing(density):
    """Generation 3's carried packing: every member's words hold exactly pext(member, mask) over the
    segment, packed densely (the last word zero above its bits), and the word count equals the
    size pass (seg3_warp) -- sparse masks through dense, with empty chunks between."""
    rng = np.random.default_rng(int(density * 1000))
    n_chunks, n_mem = 40, 3
    mask = rng.random((n_chunks, 64, 32)) < density
    mask[5] = False
    mask[6] = False
    mask[7] = False
    mask[7, 0, :3] = True
    pw = (mask * (1 << np.arange(32, dtype=np.uint64))).sum(axis=2).astype(np.uint32)
    mem = rng.integers(0, 2 ** 32, (n_mem, n_chunks, 64), dtype=np.uint64).astype(np.uint32)
    out = _pext3_pack(pw, mem)
    counts = [int(mask[j].sum()) for j in range(n_chunks)]
    total = sum(counts)
    assert len(out[0]) == _seg3_words(counts)
    for q in range(n_mem):
        want = [int((mem[q][j][w] >> b) & 1) for j in range(n_chunks) for w in range(64) for b in range(32)
                if mask[j, w, b]]
        got = [(out[q][i >> 5] >> (i & 31)) & 1 for i in range(32 * len(out[q]))]
        assert got[:total] == want and not any(got[total:])
    assert _seg3_words([0] * 5) == 0 and _seg3_words([32]) == 1 and _seg3_words([33]) == 2
    assert _seg3_words([20, 0, 0]) == 1 and _seg3_words([20, 5, 0, 13]) == 2
