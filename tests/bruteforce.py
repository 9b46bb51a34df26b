"""Independent second oracle for TINY inputs: exhaustive enumeration in pure Python.

Pins the C oracle (oracle/apriori_oracle.c) without sharing any of its code:
  * F is computed from the definition supp(X) = #{i : X subset-of t_i} (PAPER.md P3@613-P4@0)
    over ALL non-empty itemsets of the item universe, with set-subset tests;
  * every C_k is built straight from its definition {X : |X| = k, all (k-1)-subsets in
    L_{k-1}} (Q7/Q13) by filtering all k-subsets of the universe -- not by
    a join -- which pins the oracle's join + prune.
Only usable for universes of at most ~16 items.
"""
from itertools import combinations


def canonical(txs):
    return [frozenset(int(x) for x in t) for t in txs]


def supp(txs, X):
    X = frozenset(X)
    return sum(1 for t in txs if X <= t)


def frequent(txs, n_items, theta):
    txs = canonical(txs)
    out = {}
    for k in range(1, n_items + 1):
        for X in combinations(range(n_items), k):
            s = supp(txs, X)
            if s >= theta:
                out[X] = s
    return out


def levels(txs, n_items, theta):
    """[(k, {candidate: count})] for k = 1.. with the stopping rule "L_k empty or C_{k+1} empty"."""
    txs = canonical(txs)
    out = []
    C = [(i,) for i in range(n_items)]
    k = 1
    while C:
        counts = {X: supp(txs, X) for X in C}
        out.append((k, counts))
        L = {X for X, c in counts.items() if c >= theta}
        if not L:
            break
        k += 1
        C = [X for X in combinations(range(n_items), k)
             if all(S in L for S in combinations(X, k - 1))]
    return out
