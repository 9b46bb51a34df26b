"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar: bit-exact -- supports are integers.  Inputs are the seeded
generators of gen/; expected values come only from oracle/ (or, for the bit layout, from a
numpy bit-packing written here).  Sizes span several tiles / stripes plus ragged tails.
"""
import os
from fractions import Fraction
from itertools import combinations

import numpy as np
import pytest

import gen
import oracle
import paper_conf_cluster_zhangzb11a_b200 as gpa

pytestmark = pytest.mark.gpu

KERNELS = [gpa.KERNEL_V0, gpa.KERNEL_PREFIX, gpa.KERNEL_PAIRS, gpa.KERNEL_TRIE, gpa.KERNEL_PAIRS_TC]


def expected_bits(ds, item_of_row, pitch_words):
    """Row r, transaction t -> word t//32, bit t%32 (LSB first), built with numpy."""
    out = np.zeros((len(item_of_row), pitch_words), dtype=np.uint32)
    pos = {int(it): r for r, it in enumerate(item_of_row)}
    for t, tx in enumerate(ds.transactions()):
        for it in set(int(x) for x in tx):
            if it in pos:
                out[pos[it], t // 32] |= np.uint32(1 << (t % 32))
    return out


def assert_mine_equal(res, ref):
    assert len(res.levels) == len(ref.levels), ([lv.n_cand for lv in res.levels], [len(l.cand) for l in ref.levels])
    for lv, rl in zip(res.levels, ref.levels):
        assert lv.k == rl.k
        assert np.array_equal(lv.cand, rl.cand), f"C_{lv.k} differs"
        assert np.array_equal(lv.counts, rl.count), f"counts of C_{lv.k} differ"
    assert res.frequent() == ref.frequent()


# ---------------------------------------------------------------- Fig. 2 (P13@2637)

def test_fig2_bitset_and_supports(fig2):
    txs, vert = fig2
    ds = gen.from_lists(txs, 8)
    with gpa.Bitset(ds) as bs:
        assert bs.n_tx == 4 and bs.n_rows == 7
        assert list(bs.rows()) == [1, 2, 3, 4, 5, 6, 7]
        words = bs.export()
        for cand, tids, bits in vert:
            if len(cand) == 1:
                w = int(words[cand[0] - 1, 0])
                assert "".join("1" if (w >> t) & 1 else "0" for t in range(4)) == bits  # T1 = bit 0
            for kern in KERNELS:
                assert bs.count(np.array([cand]), kernel=kern)[0] == bits.count("1")
    for theta in (1, 2, 3, 4):
        for kern in (gpa.KERNEL_AUTO, gpa.KERNEL_V0, gpa.KERNEL_PREFIX, gpa.KERNEL_TRIE):
            res = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=kern), keep_candidates=True)
            assert_mine_equal(res, oracle.mine_ds(ds, theta))


# ---------------------------------------------------------------- bitset layout

@pytest.mark.parametrize("n_tx", [1, 31, 32, 33, 511, 512, 513, 1023, 1024, 1025, 4097])
def test_bitset_layout_ragged_sizes(n_tx):
    ds = gen.random_db(n_tx, n_tx, 40, max_len=12, duplicates=True, unsorted=True)
    with gpa.Bitset(ds) as bs:
        assert bs.row_pitch_bytes % 128 == 0 and bs.row_pitch_bytes * 8 >= n_tx
        rows = bs.rows()
        ref = oracle.mine_ds(ds, 1).levels[0].count
        assert np.array_equal(bs.item_counts(), ref)
        assert np.array_equal(rows, np.nonzero(ref)[0])
        assert np.array_equal(bs.export(), expected_bits(ds, rows, bs.row_pitch_bytes // 4))


def test_bitset_row_min_count_and_absent_items():
    ds = gen.random_db(5, 3000, 64, max_len=10)
    ref = oracle.mine_ds(ds, 1).levels[0].count
    with gpa.Bitset(ds, row_min_count=60) as bs:
        assert np.array_equal(bs.rows(), np.nonzero(ref >= 60)[0])
        absent = [i for i in range(64) if ref[i] < 60]
        if absent:
            with pytest.raises(gpa.GpaError) as e:
                bs.count(np.array([[absent[0]]]))
            assert e.value.status == 2  # GPA_ERR_RANGE


# ---------------------------------------------------------------- gpa_count vs the literal definition

@pytest.mark.parametrize("kern", KERNELS)
@pytest.mark.parametrize("k", [1, 2, 3, 5, 8, 12, 16, 20])
def test_count_random_candidates(kern, k):
    rng = np.random.default_rng(k * 7 + kern)
    ds = gen.random_db(100 + k, 20_000 + 37 * k, 24, max_len=16)
    with gpa.Bitset(ds) as bs:
        rows = bs.rows()
        cands = np.array(sorted({tuple(sorted(rng.choice(rows, size=k, replace=False))) for _ in range(300)}),
                         dtype=np.uint32)
        cands = cands[rng.permutation(len(cands))]  # any order
        got = bs.count(cands, kernel=kern)
        ref = oracle.support_batch(ds.offsets, ds.items, ds.n_items, cands)
        assert np.array_equal(got, ref.astype(np.uint32))


@pytest.mark.parametrize("kern", [gpa.KERNEL_TRIE, gpa.KERNEL_PREFIX])
@pytest.mark.parametrize("k", [3, 4, 7])
def test_count_many_rows_per_block(kern, k):
    """Random candidates over 300 items: trie blocks are cut at 64 distinct rows / 256 candidates,
    warps at 32 candidates; counts over a ragged 70,001-transaction axis (stripe tail)."""
    rng = np.random.default_rng(k)
    ds = gen.random_db(77 + k, 70_001, 300, max_len=60, p_empty=0.05)
    with gpa.Bitset(ds) as bs:
        rows = bs.rows()
        cands = np.array(sorted({tuple(sorted(rng.choice(rows[:120] if i % 2 else rows, size=k, replace=False)))
                                 for i in range(1500)}), dtype=np.uint32)
        got = bs.count(cands, kernel=kern)
        ref = oracle.support_batch(ds.offsets, ds.items, ds.n_items, cands)
        assert np.array_equal(got, ref.astype(np.uint32))


@pytest.mark.parametrize("kern", [gpa.KERNEL_PAIRS, gpa.KERNEL_PAIRS_TC])
@pytest.mark.parametrize("n_items", [2, 3, 127, 128, 129, 200, 255, 256, 257, 385, 513])
def test_pairs_kernel_tile_boundaries(kern, n_items):
    """All pairs of n rows through the tiled kernels, n around the 128-row (CUDA-core kernel,
    tensor-core A side) and 256-row (tensor-core B side) tile edges."""
    ds = gen.random_db(n_items, 3000, n_items, max_len=min(n_items, 40), p_empty=0.0)
    with gpa.Bitset(ds) as bs:
        rows = bs.rows()
        pairs = np.array(list(combinations(rows.tolist(), 2)), dtype=np.uint32).reshape(-1, 2)
        if len(pairs) == 0:
            return
        got = bs.count(pairs, kernel=kern)
        ref = oracle.support_batch(ds.offsets, ds.items, ds.n_items, pairs)
        assert np.array_equal(got, ref.astype(np.uint32))


@pytest.mark.parametrize("n_tx", [1, 127, 129, 8191, 8193, 100_003, 1_000_001])
def test_pairs_tc_transaction_axis(n_tx):
    """The tensor-core pair Gram over transaction counts that cut its 128-transaction stages and
    its K-split anywhere (dense rows: counts far above one stage), equal to the CUDA-core kernel
    and, on sampled pairs, to the literal definition."""
    ds = gen.random_db(n_tx % 97 + 5, n_tx, 150, max_len=60, p_empty=0.02)
    with gpa.Bitset(ds) as bs:
        rows = bs.rows()
        pairs = np.array(list(combinations(rows.tolist(), 2)), dtype=np.uint32).reshape(-1, 2)
        if len(pairs) == 0:
            return
        tc = bs.count(pairs, kernel=gpa.KERNEL_PAIRS_TC)
        cc = bs.count(pairs, kernel=gpa.KERNEL_PAIRS)
        assert np.array_equal(tc, cc)
        rng = np.random.default_rng(n_tx)
        pick = rng.choice(len(pairs), size=min(len(pairs), 200), replace=False)
        ref = oracle.support_batch(ds.offsets, ds.items, ds.n_items, pairs[pick])
        assert np.array_equal(tc[pick], ref.astype(np.uint32))


def test_count_errors():
    ds = gen.random_db(9, 500, 10, max_len=5, p_empty=0.0)
    with gpa.Bitset(ds) as bs:
        with pytest.raises(gpa.GpaError) as e:
            bs.count(np.array([[3, 2]]))
        assert e.value.status == 1
        with pytest.raises(gpa.GpaError) as e:
            bs.count(np.array([[1, 10]]))
        assert e.value.status == 1
        assert len(bs.count(np.zeros((0, 3), np.uint32))) == 0


def test_invalid_csr_rejected():
    with pytest.raises(gpa.GpaError) as e:
        gpa.mine(np.array([0, 2, 1], np.uint64), np.array([1, 2], np.uint32), 4, min_count=1)
    assert e.value.status == 1
    with pytest.raises(gpa.GpaError) as e:
        gpa.mine(np.array([0, 2], np.uint64), np.array([1, 9], np.uint32), 4, min_count=1)
    assert e.value.status == 1
    with pytest.raises(gpa.GpaError) as e:
        gpa.mine(np.array([1, 2], np.uint64), np.array([1, 2], np.uint32), 4, min_count=1)
    assert e.value.status == 1


# ---------------------------------------------------------------- gpa_mine vs the oracle (every level)

@pytest.mark.parametrize("seed", range(8))
def test_mine_random(seed):
    rng = np.random.default_rng(seed)
    ds = gen.random_db(seed, int(rng.integers(1, 3000)), int(rng.integers(2, 30)), max_len=12,
                       duplicates=seed % 2 == 1, unsorted=seed % 3 == 0)
    theta = int(rng.integers(1, max(2, ds.n_tx // 8)))
    ref = oracle.mine_ds(ds, theta)
    for kern in (gpa.KERNEL_AUTO, gpa.KERNEL_V0, gpa.KERNEL_PREFIX, gpa.KERNEL_TRIE, gpa.KERNEL_PROJ):
        for host in (False, True):
            res = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=kern, host_candgen=host),
                           keep_candidates=True)
            assert res.n_tx == ds.n_tx
            assert_mine_equal(res, ref)


@pytest.mark.parametrize("name", ["chess", "mushroom", "t40i10d100k", "accidents"])
def test_mine_configs(name):
    ds = gen.make(name)
    theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    assert gpa.min_count(ds.n_tx, gen.CONFIGS[name].minsup) == theta
    ref = oracle.mine_ds(ds, theta)
    kernels = [gpa.KERNEL_AUTO, gpa.KERNEL_PAIRS, gpa.KERNEL_PREFIX, gpa.KERNEL_TRIE, gpa.KERNEL_PROJ] + (
        [gpa.KERNEL_V0] if name in ("chess", "mushroom") else [])
    # AUTO = pairs (k = 2) + projected lists (k >= 3); device-side candidate generation by default,
    # the host thread-pool join + prune as the reference path
    for kern in kernels:
        res = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=kern), keep_candidates=True)
        assert_mine_equal(res, ref)
    res = gpa.mine(ds, min_count=theta, options=gpa.Options(host_candgen=True), keep_candidates=True)
    assert_mine_equal(res, ref)


def test_mine_device_input_equals_host_input():
    import torch
    ds = gen.make("mushroom")
    theta = oracle.min_count(ds.n_tx, "0.20")
    off = torch.from_numpy(ds.offsets.view(np.int64)).cuda()
    it = torch.from_numpy(ds.items.view(np.int32)).cuda()
    a = gpa.mine(off, it, ds.n_items, min_count=theta, keep_candidates=True)
    b = gpa.mine(ds, min_count=theta, keep_candidates=True)
    for la, lb in zip(a.levels, b.levels):
        assert np.array_equal(la.cand, lb.cand) and np.array_equal(la.counts, lb.counts)
    # and on a caller-provided torch stream
    s = torch.cuda.Stream()
    c = gpa.mine(off, it, ds.n_items, min_count=theta, options=gpa.Options(stream=s.cuda_stream))
    assert c.frequent() == b.frequent()


def test_mine_max_k_and_degenerate():
    ds = gen.make("chess")
    theta = oracle.min_count(ds.n_tx, "0.90")
    res = gpa.mine(ds, min_count=theta, options=gpa.Options(max_k=3))
    assert len(res.levels) == 3
    ref = oracle.mine_ds(ds, theta)
    for k in (1, 2, 3):
        fi, fs = res.frequent(k)
        keep = ref.levels[k - 1].count >= theta
        assert np.array_equal(fi, ref.levels[k - 1].cand[keep]) and np.array_equal(fs, ref.levels[k - 1].count[keep])
    # theta above every count: only generation 1, nothing frequent
    res = gpa.mine(ds, min_count=ds.n_tx + 1)
    assert len(res.levels) == 1 and res.frequent() == {}
    # empty database
    res = gpa.mine(np.zeros(1, np.uint64), np.zeros(0, np.uint32), 5, min_count=1)
    assert res.frequent() == {} and res.n_tx == 0
    # replicated transaction: all 2^L - 1 subsets, support N
    T = [1, 4, 6, 9, 12, 13]
    rep = gen.from_lists([T] * 700, 16)
    F = gpa.mine(rep, min_count=700).frequent()
    assert len(F) == 2 ** len(T) - 1 and set(F.values()) == {700}


# ---------------------------------------------------------------- full-size bench configuration

@pytest.fixture(scope="module")
def t40_full():
    """T40I10D10M (BASELINE.json configs[4]) at full size, mined once in the bench's launch
    configuration (default kernels, host input through the overlapped ingest), and the oracle's
    every (C_k, count) -- cached under data/ by the CSR's SHA-256 and theta (tests/oracle_cache.py;
    written only from oracle output), computed on the host cores on a cache miss."""
    import oracle_cache
    name = "t40i10d10m"
    ds = gen.make(name)
    theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    res = gpa.mine(ds, min_count=theta, keep_candidates=True)
    levels, sha, _ = oracle_cache.load_or_run(ds, theta)
    return ds, theta, res, levels, sha


def test_t40i10d10m_every_candidate(t40_full):
    """North-star parity at full size: EVERY candidate's count of every generation (1.16 M
    candidates over 16 generations: the 77-segment projected lists at 10 M transactions with their
    32-bit offsets) and F, bit-exact against the oracle."""
    ds, theta, res, levels, sha = t40_full
    assert len(res.levels) == len(levels), (len(res.levels), len(levels))
    for lv, (cand, count) in zip(res.levels, levels):
        assert np.array_equal(lv.cand, cand), f"C_{lv.k} differs"
        assert np.array_equal(lv.counts, count), f"counts of C_{lv.k} differ"
        keep = count >= theta
        assert np.array_equal(lv.freq_items, cand[keep]) and np.array_equal(lv.freq_support, count[keep]), lv.k
    assert sum(len(c) for c, _ in levels[1:]) > 1_000_000


@pytest.mark.parametrize("name", ["chess", "mushroom", "t40i10d100k", "accidents", "t40i10d10m"])
def test_shard_sum_equals_oracle(name, request):
    """Shard invariance on the GPU (SURVEY.md §4 "shard emulator"): the database split at a
    512-aligned interior boundary (a 102,400-transaction generator chunk for the Quest configs), one
    static bitset per shard (row_min_count 0: every item owns a row), and the SUM over the shards of
    gpa_count(C_k) equals the oracle's count of every candidate of every generation."""
    ds = gen.make(name)
    theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    if name == "t40i10d10m":
        levels = request.getfixturevalue("t40_full")[3]
    else:
        levels = [(lv.cand, lv.count) for lv in oracle.mine_ds(ds, theta).levels]
    ch = gen.chunk_size() if gen.CONFIGS[name].kind == "quest" and ds.n_tx > 2 * gen.chunk_size() else 512
    cut = (ds.n_tx // 2 + ch - 1) // ch * ch
    assert 0 < cut < ds.n_tx
    acc = [np.zeros(len(c), np.uint64) for c, _ in levels]
    for b0, b1 in ((0, cut), (cut, ds.n_tx)):
        with gpa.Bitset(gen.subset(ds, b0, b1), row_min_count=0) as bs:
            assert bs.n_rows == ds.n_items
            acc[0] += bs.item_counts()
            for k, (cand, _) in enumerate(levels[1:], start=2):
                if len(cand):
                    acc[k - 1] += bs.count(cand)
    for k, ((cand, count), got) in enumerate(zip(levels, acc), start=1):
        assert np.array_equal(got, count.astype(np.uint64)), f"{name}: shard sums of C_{k}"


def test_t40i10d10m_full_size_sampled(t40_full):
    """BASELINE.json's largest config at full size in the bench's launch configuration: every
    level's counts on sampled candidates against the LITERAL definition (one subset test per
    transaction, independent of the oracle's trie walk), level 1 against numpy.bincount, and
    invariants (|C_2| = C(|L_1|, 2), downward closure of F)."""
    ds, theta, res, _, _ = t40_full
    c1 = np.bincount(ds.items, minlength=ds.n_items)
    assert np.array_equal(res.levels[0].counts, c1)
    n1 = int((c1 >= theta).sum())
    assert res.levels[1].n_cand == n1 * (n1 - 1) // 2
    F = res.frequent()
    for X, s in F.items():
        if len(X) > 1:
            for Y in combinations(X, len(X) - 1):
                assert F[Y] >= s
    rng = np.random.default_rng(5)
    sample, expect = [], []
    for lv in res.levels[1:]:
        # frequent and infrequent candidates alike, plus the extremes of the level
        idx = set(rng.choice(lv.n_cand, size=min(6, lv.n_cand), replace=False).tolist())
        idx |= {int(np.argmax(lv.counts)), int(np.argmin(lv.counts))}
        for i in sorted(idx):
            sample.append(lv.cand[i])
            expect.append(lv.counts[i])
    for k in sorted({len(c) for c in sample}):
        cs = np.array([c for c in sample if len(c) == k], dtype=np.uint32)
        ex = np.array([e for c, e in zip(sample, expect) if len(c) == k], dtype=np.uint64)
        lit = oracle.support_batch(ds.offsets, ds.items, ds.n_items, cs)
        assert np.array_equal(lit, ex), k
    # association rules at full size (150 M antecedents), a property check (the supports are this
    # run's, already checked on samples above): for sampled itemsets X, the reported antecedent masks
    # are exactly those with supp(X) / supp(A) >= 0.9 over F, with supp(A) as in F
    rules = res.rules("0.9")
    flat = [tuple(r) for lv in res.levels for r in lv.freq_items.tolist()]
    first2 = res.levels[0].n_freq
    pick = np.sort(rng.choice(np.arange(first2, len(flat)), size=300, replace=False))
    sel = np.isin(rules.itemset, pick)
    got = {}
    for x, m, sa in zip(rules.itemset[sel].tolist(), rules.antecedent_mask[sel].tolist(),
                        rules.antecedent_support[sel].tolist()):
        got.setdefault(x, {})[m] = sa
    n_rules = 0
    for x in pick.tolist():
        X = flat[x]
        want = {}
        for m in range(1, 2 ** len(X) - 1):
            A = tuple(v for q, v in enumerate(X) if m >> q & 1)
            if Fraction(F[X], F[A]) >= Fraction(9, 10):
                want[m] = F[A]
        assert got.get(x, {}) == want, X
        n_rules += len(want)
    assert n_rules > 0


def test_nccl_single_rank_dist_matches_local():
    """The NCCL path end to end on one GPU: unique id broadcast through torch.distributed, a
    1-rank communicator, and every all-reduce of gpa_mine (flags, N, histogram, counts)."""
    import torch
    import torch.distributed as tdist
    if not tdist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        tdist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    d = gpa.Dist.from_torch(0)
    try:
        ds = gen.make("mushroom")
        theta = oracle.min_count(ds.n_tx, "0.20")
        a = gpa.mine(ds, min_count=theta, dist=d, options=gpa.Options(device=0), keep_candidates=True)
        assert_mine_equal(a, oracle.mine_ds(ds, theta))
        with gpa.Bitset(ds, dist=d, options=gpa.Options(device=0)) as bs:
            c = oracle.mine_ds(ds, theta).levels[2].cand
            assert np.array_equal(bs.count(c), oracle.support_batch(ds.offsets, ds.items, ds.n_items, c).astype(np.uint32))
    finally:
        d.close()
        tdist.destroy_process_group()


@pytest.mark.parametrize("host", [False, True])
def test_mine_dense_long_runs(host):
    """Dense DB: L_2 is (nearly) all pairs, so the join runs are long (device hash-set prune under
    load, groups of up to ~40 siblings) and generations go deep."""
    ds = gen.random_db(42, 6000, 44, max_len=24, p_empty=0.02)   # 10 generations, |C_6| = 24,036
    theta = 500
    ref = oracle.mine_ds(ds, theta)
    res = gpa.mine(ds, min_count=theta, options=gpa.Options(host_candgen=host), keep_candidates=True)
    assert_mine_equal(res, ref)
    assert max(len(lv.cand) for lv in ref.levels[1:]) > 20000


def test_overlapped_ingest_equals_sequential():
    """Host input >= 262,144 transactions takes the chunked upload overlapped with histogram,
    bitset build and generation-2 counting; results equal the sequential path and the oracle."""
    ds = gen.make("accidents")
    theta = oracle.min_count(ds.n_tx, "0.30")
    ref = oracle.mine_ds(ds, theta)
    a = gpa.mine(ds, min_count=theta, keep_candidates=True)
    b = gpa.mine(ds, min_count=theta, options=gpa.Options(overlap_ingest=False), keep_candidates=True)
    assert_mine_equal(a, ref)
    assert_mine_equal(b, ref)


def test_overlapped_ingest_row_estimate_miss():
    """An item absent from the first chunk but frequent overall is missing from the chunk-0 row
    estimate R0: the ingest must fall back to rebuilding the bitset (exact result either way)."""
    rng = np.random.default_rng(9)
    n = 300_000
    base = rng.random((n, 12)) < 0.3
    late = np.zeros(n, dtype=bool)
    late[n // 2:] = rng.random(n - n // 2) < 0.6   # item 12: only in the second half, 30 % overall
    mat = np.concatenate([base, late[:, None]], axis=1)
    lens = mat.sum(axis=1).astype(np.uint64)
    offsets = np.zeros(n + 1, np.uint64)
    np.cumsum(lens, out=offsets[1:])
    items = np.nonzero(mat)[1].astype(np.uint32)
    ds = gen.Dataset("late", offsets, items, 13, n)
    theta = n // 10
    ref = oracle.mine_ds(ds, theta)
    res = gpa.mine(ds, min_count=theta, keep_candidates=True)
    assert (12,) in res.frequent()
    assert_mine_equal(res, ref)


def test_packed_upload_invalid_and_unpacked_paths(monkeypatch):
    """Host input on the overlapped path uploads the item ids bit-packed (b = ceil(log2 n_items)
    bits): results equal the oracle with packing and with GPA_NO_PACKED_UPLOAD (read per call); an id
    >= n_items that still fits in b bits, and one that does not (the chunk then goes raw), are both
    rejected by the validation -- in a late chunk, not only chunk 0."""
    ds = gen.make("accidents")          # 468 item ids -> 9-bit fields
    theta = oracle.min_count(ds.n_tx, "0.30")
    ref = oracle.mine_ds(ds, theta)
    assert_mine_equal(gpa.mine(ds, min_count=theta, keep_candidates=True), ref)
    monkeypatch.setenv("GPA_NO_PACKED_UPLOAD", "1")
    assert_mine_equal(gpa.mine(ds, min_count=theta, keep_candidates=True), ref)
    monkeypatch.delenv("GPA_NO_PACKED_UPLOAD")
    for every in ("0", "1", "2"):        # every chunk packed / every chunk raw / alternating
        monkeypatch.setenv("GPA_PACK_RAW_EVERY", every)
        assert_mine_equal(gpa.mine(ds, min_count=theta, keep_candidates=True), ref)
    monkeypatch.delenv("GPA_PACK_RAW_EVERY")
    for bad in (ds.n_items, 1 << 12):   # in range of 9 bits (>= n_items) / out of 9 bits
        items = ds.items.copy()
        items[len(items) - 5] = bad
        with pytest.raises(gpa.GpaError) as e:
            gpa.mine(ds.offsets, items, ds.n_items, min_count=theta)
        assert e.value.status == 1


def test_c_example_fimi_roundtrip(tmp_path, fig2):
    """The C example (C ABI only) on the Fig. 2 database written as a FIMI file: every frequent
    itemset and support as the oracle computes them."""
    import subprocess
    txs, _ = fig2
    dat = tmp_path / "fig2.dat"
    dat.write_text("\n".join(" ".join(map(str, t)) for t in txs) + "\n")
    exe = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "examples", "gpa_mine_fimi")
    out = subprocess.run([exe, str(dat), "0.5"], capture_output=True, text=True, check=True).stdout
    got = {}
    for line in out.strip().splitlines():
        items, sup = line.rsplit(" (", 1)
        got[tuple(int(x) for x in items.split())] = int(sup.rstrip(")"))
    ref = oracle.mine_ds(gen.from_lists(txs, 8), 2).frequent()
    assert got == ref


# ---------------------------------------------------------------- projected lists: fallback

@pytest.mark.parametrize("how", ["mb0", "k4", "k6"])
def test_proj_fallback_to_complete_intersection(monkeypatch, how):
    """When a generation's projected lists do not fit (forced with GPA_PROJ_MAX_MB=0 at generation 3,
    or GPA_PROJ_TEST_MAX_K after generation 4 / 6), gpa_mine switches to complete intersection for
    the remaining generations, with every (C_k, count) unchanged."""
    ds = gen.make("mushroom")
    theta = oracle.min_count(ds.n_tx, "0.20")
    ref = oracle.mine_ds(ds, theta)
    if how == "mb0":
        monkeypatch.setenv("GPA_PROJ_MAX_MB", "0")
    else:
        monkeypatch.setenv("GPA_PROJ_TEST_MAX_K", how[1:])
    res = gpa.mine(ds, min_count=theta, keep_candidates=True, options=gpa.Options(multi_kernel=True))
    assert_mine_equal(res, ref)
    kinds = {lv.k: lv.stats["kernel_name"] for lv in res.levels[2:]}
    last = 2 if how == "mb0" else int(how[1:])
    assert all((kinds[k] == "proj") == (k <= last) for k in kinds), kinds


@pytest.mark.parametrize("n_tx,n_items,max_len,theta", [(70_000, 40, 10, 1400), (140_000, 60, 12, 2800),
                                                          (9_000, 40, 12, 90)])
def test_proj_multi_segment_classes(n_tx, n_items, max_len, theta):
    """Projected lists (proj.cu): class masks spanning several 131,072-transaction segments (70,000 /
    140,000 transactions: bitset rows of 2,188 / 4,375 words), classes of more than 16 members
    (several pext items per segment), ragged segment and list tails -- every (C_k, count) of every
    generation equal to the oracle, and the generations k >= 3 really ran on the lists."""
    ds = gen.random_db(n_tx % 1000 + n_items, n_tx, n_items, max_len=max_len, p_empty=0.01)
    ref = oracle.mine_ds(ds, theta)
    res = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=gpa.KERNEL_PROJ), keep_candidates=True)
    assert_mine_equal(res, ref)
    assert len(res.levels) >= 4
    assert all(lv.stats["kernel_name"] == "proj" for lv in res.levels[2:])


@pytest.mark.parametrize("name", ["mushroom", "chess", "random"])
def test_proj_k3_set_bit_walk_pext(name):
    """Generation 3's lists by the set-bit-walk pext (GPA_PROJ_K3_PEXT=1, read once per process, so
    a child process) instead of the default warp bit gather (pext3_kernel): every frequent itemset and
    support equal to the oracle's."""
    import json
    import subprocess
    import sys
    if name == "random":
        ds, theta = gen.random_db(11, 8000, 40, max_len=16), 80
        spec = "gen.random_db(11, 8000, 40, max_len=16), 80"
    else:
        ds = gen.make(name)
        theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
        spec = f"gen.make({name!r}), {theta}"
    code = ("import json, gen, paper_conf_cluster_zhangzb11a_b200 as gpa\n"
            f"ds, th = {spec}\n"
            "r = gpa.mine(ds, min_count=th, options=gpa.Options(multi_kernel=True))\n"
            "print(json.dumps(sorted([list(map(int, s)), int(c)] for s, c in r.frequent().items())))\n")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, GPA_PROJ_K3_PEXT="1")
    out = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True, text=True,
                         check=True, timeout=600).stdout
    got = {tuple(s): c for s, c in json.loads(out.strip().splitlines()[-1])}
    ref = oracle.mine_ds(ds, theta).frequent()
    assert got == {tuple(map(int, s)): int(c) for s, c in ref.items()}
    assert max(len(s) for s in got) >= 4


@pytest.mark.parametrize("name", ["chess", "mushroom", "accidents", "fig2", "dense", "random"])
def test_fused_single_launch_equals_oracle(fig2, name):
    """GPA_KERNEL_FUSED (the whole level loop in one cooperative launch: complete-intersection
    counting, threshold, join + prune as grid-wide phases) against the oracle on every (C_k, count)
    and F, and against the multi-kernel path; exactly one library launch for all generations."""
    if name == "fig2":
        ds, theta = gen.from_lists(fig2[0], 8), 2
    elif name == "dense":
        ds, theta = gen.random_db(42, 6000, 44, max_len=24, p_empty=0.02), 500
    elif name == "random":
        ds, theta = gen.random_db(5, 2500, 28, max_len=12, duplicates=True, unsorted=True), 40
    else:
        ds = gen.make(name)
        theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    ref = oracle.mine_ds(ds, theta)
    l0 = gpa.kernel_launches()
    res = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=gpa.KERNEL_FUSED), keep_candidates=True)
    assert_mine_equal(res, ref)
    assert all(lv.stats["kernel_name"] == "fused" for lv in res.levels[1:])
    multi = gpa.mine(ds, min_count=theta, options=gpa.Options(multi_kernel=True), keep_candidates=True)
    assert_mine_equal(multi, ref)
    assert all(lv.stats["kernel_name"] != "fused" for lv in multi.levels[1:])
    # default options pick the fused path for these small problems
    l1 = gpa.kernel_launches()
    auto = gpa.mine(ds, min_count=theta, options=gpa.Options(overlap_ingest=False))
    assert auto.frequent() == ref.frequent()
    assert all(lv.stats["kernel_name"] == "fused" for lv in auto.levels[1:])
    assert gpa.kernel_launches() - l1 <= 4   # one-pass build (+ row compaction) + the fused loop


def test_fused_capacity_overflow_falls_back(monkeypatch):
    """A generation larger than the fused path's capacity (forced with GPA_FUSED_TEST_CAP) reruns on the
    multi-kernel path: every (C_k, count) unchanged."""
    import json
    import subprocess
    import sys
    code = ("import json, gen, oracle, paper_conf_cluster_zhangzb11a_b200 as gpa\n"
            "ds = gen.make('mushroom'); th = oracle.min_count(ds.n_tx, '0.20')\n"
            "r = gpa.mine(ds, min_count=th, keep_candidates=True)\n"
            "ref = oracle.mine_ds(ds, th)\n"
            "ok = all((lv.cand == rl.cand).all() and (lv.counts == rl.count).all() for lv, rl in zip(r.levels, ref.levels))\n"
            "print(json.dumps([bool(ok and len(r.levels) == len(ref.levels)), sorted({lv.stats['kernel_name'] for lv in r.levels[1:]})]))\n")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", code], cwd=root, env=dict(os.environ, GPA_FUSED_TEST_CAP="100"),
                         capture_output=True, text=True, check=True, timeout=600).stdout
    ok, kinds = json.loads(out.strip().splitlines()[-1])
    assert ok and "fused" not in kinds, kinds


def test_complete_intersection_flag():
    """GPA_COMPLETE_INTERSECTION: k >= 3 by the paper's complete intersection (trie / prefix over the
    static bitset), k = 2 on the CUDA-core pair Gram with count_kernel PAIRS -- the north-star path
    the bench times beside the default: same (C_k, counts) as the oracle."""
    for name in ("mushroom", "t40i10d100k"):
        ds = gen.make(name)
        theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
        res = gpa.mine(ds, min_count=theta, keep_candidates=True,
                       options=gpa.Options(count_kernel=gpa.KERNEL_PAIRS, complete_intersection=True))
        assert_mine_equal(res, oracle.mine_ds(ds, theta))
        kinds = {lv.stats["kernel_name"] for lv in res.levels[2:]}
        assert res.levels[1].stats["kernel_name"] == "pairs" and kinds <= {"trie", "prefix"}, kinds


# ---------------------------------------------------------------- association rules (f4)

@pytest.mark.parametrize("name,minconf", [("fig2", "0.5"), ("fig2", "1"), ("chess", "0.95"), ("mushroom", "0.8"),
                                          ("random", "0.3"), ("replicated", "1")])
def test_rules_vs_oracle(fig2, name, minconf):
    """gpa_rules_create on the device vs the definition (oracle.rules) on the same F: every rule,
    supp(X) and supp(A) identical."""
    if name == "fig2":
        ds, theta = gen.from_lists(fig2[0], 8), 2
    elif name == "random":
        ds = gen.random_db(7, 3000, 24, max_len=12)
        theta = 60
    elif name == "replicated":
        ds, theta = gen.from_lists([[0, 3, 4, 7, 9, 10, 12, 15]] * 40, 16), 40
    else:
        ds = gen.make(name)
        theta = oracle.min_count(ds.n_tx, gen.CONFIGS[name].minsup)
    res = gpa.mine(ds, min_count=theta)
    F = res.frequent()
    assert F == oracle.mine_ds(ds, theta).frequent()
    got = res.rules(minconf).as_dict()
    want = oracle.rules(F, minconf)
    assert got == want
    if name == "replicated":
        assert len(got) == 3 ** 8 - 2 ** 9 + 1


def test_rules_errors_and_empty():
    ds = gen.random_db(8, 500, 12, max_len=5)
    res = gpa.mine(ds, min_count=10 ** 6)   # nothing frequent
    assert len(res.rules("0.5")) == 0
    res = gpa.mine(ds, min_count=20)
    with pytest.raises(gpa.GpaError):
        res.rules(Fraction(1, 2 ** 33))   # conf_den >= 2^32
