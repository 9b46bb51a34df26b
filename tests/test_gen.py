"""Seeded input generators (gen/): determinism pins and shard consistency (CPU).

The bench, the parity tests and the cached oracle results (tests/oracle_cache.py) all key on these
inputs, so they must not drift: each configuration's CSR is pinned by its SHA-256
(tests/golden/gen_sha256.txt), and a Quest database generated shard by shard (the multi-GPU
bench's per-rank generation) must be byte-identical to the whole.
"""
import os

import numpy as np
import pytest

import gen
import oracle_cache

HERE = os.path.dirname(os.path.abspath(__file__))


def _pins():
    out = {}
    for line in open(os.path.join(HERE, "golden", "gen_sha256.txt")):
        if line.strip() and not line.startswith("#"):
            name, n_tx, nnz, sha = line.split()
            out[name] = (int(n_tx), int(nnz), sha)
    return out


@pytest.mark.parametrize("name", ["chess", "mushroom", "t40i10d100k", "accidents"])
def test_generator_sha256_pinned(name):
    n_tx, nnz, sha = _pins()[name]
    ds = gen.make(name)
    assert (ds.n_tx, ds.nnz) == (n_tx, nnz)
    assert oracle_cache.dataset_sha256(ds) == sha
    # canonical CSR: sorted, duplicate-free transactions, ids in range
    o = ds.offsets
    assert o[0] == 0 and np.all(np.diff(o.astype(np.int64)) >= 0)
    assert ds.items.max() < ds.n_items
    for t in range(0, ds.n_tx, max(1, ds.n_tx // 500)):
        tx = ds.items[o[t]:o[t + 1]]
        assert np.all(np.diff(tx.astype(np.int64)) > 0)


def test_quest_shards_concatenate_to_whole():
    whole = gen.make("t40i10d100k")
    ch = gen.chunk_size()
    parts = [gen.make("t40i10d100k", tx_begin=a, tx_end=min(a + ch, whole.n_tx)) for a in range(0, whole.n_tx, ch)]
    items = np.concatenate([p.items for p in parts])
    lens = np.concatenate([np.diff(p.offsets.astype(np.int64)) for p in parts])
    assert np.array_equal(items, whole.items)
    assert np.array_equal(lens, np.diff(whole.offsets.astype(np.int64)))


def test_generator_repeatable():
    a = gen.make("mushroom")
    b = gen.make("mushroom")
    assert oracle_cache.dataset_sha256(a) == oracle_cache.dataset_sha256(b)
    r1 = gen.random_db(5, 300, 20, max_len=8)
    r2 = gen.random_db(5, 300, 20, max_len=8)
    assert np.array_equal(r1.items, r2.items) and np.array_equal(r1.offsets, r2.offsets)
