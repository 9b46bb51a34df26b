"""Pins for the CPU oracle (oracle/) against things other than itself (CPU only).

Each test names what fixes the expected value: the paper's printed example (Fig. 2, Fig. 4),
the definition evaluated by exhaustive enumeration (tests/bruteforce.py), a closed form, an
invariant, a metamorphic relation, or a library routine (numpy.bincount, fractions).
"""
from fractions import Fraction
from itertools import combinations
from math import comb

import numpy as np
import pytest

import bruteforce
import gen
import oracle


def ds_from(txs, n_items):
    return gen.from_lists(txs, n_items)


def mine_lists(txs, n_items, theta):
    d = ds_from(txs, n_items)
    return oracle.mine_ds(d, theta, threads=2)


# ---------------------------------------------------------------- Fig. 2 (P13@2637-2860)

def test_fig2_printed_vertical_lists(fig2):
    """Every printed tidset / bitset of Fig. 2(B) is reproduced by the oracle's supports:
    supp over the tidset's transactions = |tidset| and supp over the others = 0; the support
    equals the number of 1s of the printed bitset."""
    txs, vert = fig2
    for cand, tids, bits in vert:
        assert len(bits) == len(txs)
        assert [i + 1 for i, b in enumerate(bits) if b == "1"] == tids  # tidset == bitset (T1 left-most)
        full = ds_from(txs, 8)
        assert oracle.support(full.offsets, full.items, 8, cand) == bits.count("1")
        inside = ds_from([txs[t - 1] for t in tids], 8)
        outside = ds_from([txs[t - 1] for t in range(1, 5) if t not in tids], 8)
        assert oracle.support(inside.offsets, inside.items, 8, cand) == len(tids)
        if outside.n_tx:
            assert oracle.support(outside.offsets, outside.items, 8, cand) == 0


def test_fig2_mine_levels_match_printed(fig2):
    """Level-1 counts and the three printed pair supports ({1,2}:1, {1,3}:2, {1,4}:2)."""
    txs, vert = fig2
    r = mine_lists(txs, 8, 1)
    c1 = r.levels[0].count
    for cand, tids, bits in vert:
        if len(cand) == 1:
            assert c1[cand[0]] == bits.count("1")
        else:
            assert r.level_map(2)[cand] == bits.count("1")
    assert c1[0] == 0  # item 0 never occurs (ids are the paper's 1..7)


@pytest.mark.parametrize("theta", [1, 2, 3, 4, 5])
def test_fig2_bruteforce_every_level(fig2, theta):
    txs, _ = fig2
    r = mine_lists(txs, 8, theta)
    bf = bruteforce.levels(txs, 8, theta)
    assert [lv.k for lv in r.levels] == [k for k, _ in bf]
    for lv, (k, m) in zip(r.levels, bf):
        assert r.level_map(k) == m
    assert r.frequent() == bruteforce.frequent(txs, 8, theta)


def test_fig2_closed_form_theta1(fig2):
    """theta = 1: sum over C_k of supports = sum_t C(|t|, k) (every k-subset of a transaction
    is a candidate); for Fig. 2 this is 19, 36, 34, 16, 3 for k = 1..5."""
    txs, _ = fig2
    r = mine_lists(txs, 8, 1)
    sums = [int(lv.count.astype(np.int64).sum()) for lv in r.levels]
    expect = [sum(comb(len(set(t)), k) for t in txs) for k in range(1, len(sums) + 1)]
    assert sums == expect
    assert expect[:5] == [19, 36, 34, 16, 3]


# ---------------------------------------------------------------- join rule (Fig. 4, P18@863)

def test_fig4_join_rule():
    L3 = np.array([(1, 2, 4), (1, 2, 5), (1, 2, 6)], dtype=np.uint32)
    C4 = oracle.candgen(L3, prune=False)
    assert [tuple(map(int, r)) for r in C4] == [(1, 2, 4, 5), (1, 2, 4, 6), (1, 2, 5, 6)]
    # with prune, (1,2,4,5) needs (1,4,5), (2,4,5) etc. in L3: absent -> pruned
    assert len(oracle.candgen(L3, prune=True)) == 0
    full = sorted(set(L3.tolist() and [tuple(x) for x in L3.tolist()]) |
                  {(1, 4, 5), (2, 4, 5), (1, 4, 6), (2, 4, 6)})
    C4p = oracle.candgen(np.array(full, dtype=np.uint32), prune=True)
    assert [tuple(map(int, r)) for r in C4p] == [(1, 2, 4, 5), (1, 2, 4, 6)]


@pytest.mark.parametrize("seed", range(6))
def test_candgen_equals_definition(seed):
    """C_k = {X : |X| = k, every (k-1)-subset in L_{k-1}} for random downward-closed-or-not L."""
    rng = np.random.default_rng(seed)
    n, km1 = 9, int(rng.integers(1, 4))
    allsets = list(combinations(range(n), km1))
    pick = rng.random(len(allsets)) < 0.5
    L = sorted(s for s, p in zip(allsets, pick) if p)
    Lset = set(L)
    expect = [X for X in combinations(range(n), km1 + 1)
              if all(S in Lset for S in combinations(X, km1))]
    got = oracle.candgen(np.array(L, dtype=np.uint32).reshape(-1, km1), prune=True)
    assert [tuple(map(int, r)) for r in got] == expect


# ---------------------------------------------------------------- brute force on random tiny DBs

@pytest.mark.parametrize("seed", range(12))
def test_random_tiny_vs_bruteforce(seed):
    rng = np.random.default_rng(100 + seed)
    n_items = int(rng.integers(3, 11))
    d = gen.random_db(seed, int(rng.integers(0, 64)), n_items, max_len=n_items,
                      duplicates=bool(seed % 2), unsorted=bool(seed % 3 == 0))
    txs = [list(t) for t in d.transactions()]
    theta = int(rng.integers(1, 6))
    r = oracle.mine_ds(d, theta, threads=3)
    bf = bruteforce.levels(txs, n_items, theta)
    assert [lv.k for lv in r.levels] == [k for k, _ in bf]
    for lv, (k, m) in zip(r.levels, bf):
        assert r.level_map(k) == m
    assert r.frequent() == bruteforce.frequent(txs, n_items, theta)


# ---------------------------------------------------------------- closed forms

@pytest.mark.parametrize("L,N", [(1, 5), (4, 3), (7, 2), (10, 1)])
def test_replicated_transaction(L, N):
    """N copies of one transaction T: F = all 2^L - 1 non-empty subsets, each with support N."""
    T = list(range(3, 3 + 2 * L, 2))
    for theta in (1, N):
        r = mine_lists([T] * N, 3 + 2 * L, theta)
        F = r.frequent()
        assert len(F) == 2 ** L - 1
        assert set(F.values()) == {N}


def test_singletons():
    """Each transaction a single item: F = items with count >= theta, and L_2 is empty."""
    txs = [[i % 7] for i in range(40)]
    r = mine_lists(txs, 9, 6)
    F = r.frequent()
    assert F == {(i,): 6 for i in range(7) if 40 // 7 + (1 if i < 40 % 7 else 0) >= 6}
    assert all(c == 0 for c in r.levels[1].count)


def test_empty_database():
    d = gen.from_lists([], 5)
    r = oracle.mine_ds(d, 1)
    assert len(r.levels) == 1 and r.frequent() == {}
    assert oracle.min_count(0, "0.5") == 1


def test_theta1_closed_form_random():
    d = gen.random_db(7, 40, 12, max_len=6)
    r = oracle.mine_ds(d, 1)
    txs = [set(map(int, t)) for t in d.transactions()]
    for lv in r.levels:
        assert int(lv.count.astype(np.int64).sum()) == sum(comb(len(t), lv.k) for t in txs)


# ---------------------------------------------------------------- library routines

@pytest.mark.parametrize("name", ["chess", "mushroom"])
def test_level1_is_bincount(name):
    d = gen.make(name)
    cfg = gen.CONFIGS[name]
    r = oracle.mine_ds(d, oracle.min_count(d.n_tx, cfg.minsup))
    assert np.array_equal(r.levels[0].count, np.bincount(d.items, minlength=d.n_items))


def test_level1_bincount_noncanonical():
    d = gen.random_db(3, 200, 30, max_len=12, duplicates=True, unsorted=True)
    canon = np.concatenate([np.unique(t) for t in d.transactions()] + [np.zeros(0, np.uint32)])
    r = oracle.mine_ds(d, 5)
    assert np.array_equal(r.levels[0].count, np.bincount(canon.astype(np.int64), minlength=30))


def test_min_count_rule():
    """max(1, ceil(minsup * N)) in exact rationals (fractions), incl. the binary-float trap
    0.07 * 100 = 7.000000000000001 (ceil 8 would be wrong)."""
    cases = {(3196, "0.90"): 2877, (8124, "0.20"): 1625, (100_000, "0.01"): 1000,
             (340_183, "0.30"): 102055, (10_000_000, "0.005"): 50000, (100, "0.07"): 7, (5, "0"): 1}
    for (n, s), want in cases.items():
        f = Fraction(s) * n
        assert max(1, -(-f.numerator // f.denominator)) == want
        assert oracle.min_count(n, s) == want


# ---------------------------------------------------------------- invariants and metamorphic relations

@pytest.mark.parametrize("name", ["chess", "mushroom"])
def test_downward_closure_and_literal_counts(name):
    d = gen.make(name)
    theta = oracle.min_count(d.n_tx, gen.CONFIGS[name].minsup)
    r = oracle.mine_ds(d, theta)
    F = r.frequent()
    for X, s in F.items():
        for j in range(1, len(X)):
            for Y in combinations(X, j):
                assert Y in F and F[Y] >= s
    # the transaction-scan counter equals the literal definition (one subset test per tx)
    for lv in r.levels[1:]:
        lit = oracle.support_batch(d.offsets, d.items, d.n_items, lv.cand)
        assert np.array_equal(lit.astype(np.uint32), lv.count)
    assert len(r.levels[1].cand) == comb(int((r.levels[0].count >= theta).sum()), 2)


def test_metamorphic_permute_relabel_double():
    d = gen.random_db(11, 120, 14, max_len=8)
    txs = [list(map(int, t)) for t in d.transactions()]
    theta = 6
    F = mine_lists(txs, 14, theta).frequent()
    rng = np.random.default_rng(0)
    perm_tx = [txs[i] for i in rng.permutation(len(txs))]
    assert mine_lists(perm_tx, 14, theta).frequent() == F
    relabel = rng.permutation(14)
    rel = [[int(relabel[x]) for x in t] for t in txs]
    Fr = mine_lists(rel, 14, theta).frequent()
    assert Fr == {tuple(sorted(int(relabel[x]) for x in X)): s for X, s in F.items()}
    Fd = mine_lists(txs + txs, 14, 2 * theta).frequent()
    assert Fd == {X: 2 * s for X, s in F.items()}


def test_shard_invariance():
    """Any partition of the transactions: summed per-shard counts == unsharded counts."""
    d = gen.make("mushroom")
    theta = oracle.min_count(d.n_tx, "0.20")
    r = oracle.mine_ds(d, theta)
    for lv in r.levels[1:4]:
        parts = [gen.subset(d, a, b) for a, b in ((0, 512), (512, 4096), (4096, d.n_tx))]
        tot = sum(oracle.support_batch(p.offsets, p.items, p.n_items, lv.cand).astype(np.int64) for p in parts)
        assert np.array_equal(tot, lv.count.astype(np.int64))


# ---------------------------------------------------------------- association rules (f4, Q19)

def test_rules_fig2_confidences(fig2):
    """Fig. 2 database at theta = 2: {1} => {3} has confidence supp{1,3} / supp{1} = 2/2, {3} => {1}
    2/4 (supports printed in Fig. 2, P13@2637-2860)."""
    txs, _ = fig2
    ds = gen.from_lists(txs, 8)
    F = oracle.mine_ds(ds, 2).frequent()
    r1 = oracle.rules(F, "1")
    assert r1[((1,), (3,))] == (2, 2)
    assert ((3,), (1,)) not in r1
    r5 = oracle.rules(F, "0.5")
    assert r5[((3,), (1,))] == (2, 4)
    assert all(Fraction(sx, sa) >= Fraction(1, 2) for sx, sa in r5.values())
    # every rule's antecedent and consequent partition a frequent itemset
    for (A, B), (sx, sa) in r5.items():
        X = tuple(sorted(A + B))
        assert F[X] == sx and F[A] == sa and not set(A) & set(B)


def test_rules_closed_forms():
    """Replicated transaction T (|T| = L, N copies): every rule has confidence 1, so at any minconf
    <= 1 there are sum_{k>=2} C(L, k)(2^k - 2) = 3^L - 2^(L+1) + 1 of them; minconf 0 keeps all
    sum_X (2^|X| - 2) candidates on any F; minconf above 1 keeps none."""
    L = 6
    ds = gen.from_lists([list(range(2, 2 + L))] * 50, 12)
    F = oracle.mine_ds(ds, 50).frequent()
    assert len(oracle.rules(F, "1")) == 3 ** L - 2 ** (L + 1) + 1
    ds = gen.random_db(3, 200, 10, max_len=6)
    F = oracle.mine_ds(ds, 5).frequent()
    assert len(oracle.rules(F, "0")) == sum(2 ** len(X) - 2 for X in F if len(X) >= 2)
    assert len(oracle.rules(F, "1.01")) == 0
