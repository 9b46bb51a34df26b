"""bench.py's roofline arithmetic on a synthetic result (CPU): every reported fraction must be
reproducible from the line's own fields (achieved = algorithmic work or bytes / event time,
frac = achieved / peak), and the longest launch is the one reported."""
import types

import pytest

import bench

PEAKS = {"hbm_gbs": 6551.4, "bf16_tflops": 1641.7, "sm_max_mhz": 1965.0}


def fake_result(n_tx):
    L = lambda k, n_cand, n_freq, kern, **st: types.SimpleNamespace(
        k=k, n_cand=n_cand, n_freq=n_freq, stats=dict(kernel_name=kern, **st))
    levels = [L(1, 1000, 900, "v0"), L(2, 404_550, 5000, "pairs_tc"), L(3, 20_000, 9000, "proj"),
              L(4, 15_000, 8000, "trie")]
    return types.SimpleNamespace(levels=levels, n_tx=n_tx, cand_tx=sum(l.n_cand for l in levels[1:]) * n_tx)


def test_roofline_records_reproducible():
    n_tx = 10_000_000
    res = fake_result(n_tx)
    st = {2: dict(kernel_name="pairs_tc", count_ms=4.0, build_ms=0.0, setup_ms=0.0, allreduce_ms=0.0),
          3: dict(kernel_name="proj", count_ms=6.0, build_ms=4.5, setup_ms=0.5, allreduce_ms=0.0,
                  build_bytes=2_400_000_000, count_bytes=1_200_000_000),
          4: dict(kernel_name="trie", count_ms=1.0, build_ms=0.0, setup_ms=0.0, allreduce_ms=0.0)}
    recs = bench.roofline_records(res, st, n_tx, PEAKS, 1965.0)
    by = {(r["kernel"], r["k"]): r for r in recs}
    tc = by[("pairs_tc", 2)]
    assert tc["bound"] == "tensor" and tc["peak"] == pytest.approx(2 * 1641.7)
    assert tc["achieved"] == pytest.approx(2 * 404_550 * n_tx / 4e-3 / 1e12)
    px = by[("lists", 3)]
    assert px["bound"] == "hbm" and px["achieved"] == pytest.approx(2.4e9 / 4.5e-3 / 1e9)
    cp = by[("count_proj", 3)]
    assert cp["kernel_ms"] == pytest.approx(1.0) and cp["achieved"] == pytest.approx(1.2e9 / 1e-3 / 1e9)
    tr = by[("trie", 4)]
    assert tr["bound"] == "alu" and tr["peak"] == pytest.approx(148 * 16 * 32 * 1965e6 / 1e12)
    for r in recs:
        assert r["frac"] == pytest.approx(r["achieved"] / r["peak"])
        x = dict(r)
        bench.rescale(x)
        assert x["frac"] == pytest.approx(r["frac"])
    agg = bench.aggregate_by_kernel(recs)
    assert agg["pairs_tc"]["kernel_ms"] == pytest.approx(4.0) and agg["lists"]["launches"] == 1


def test_pitch_bytes_matches_library_rule():
    assert bench.pitch_bytes(1) == 4096
    assert bench.pitch_bytes(32768) == 4096
    assert bench.pitch_bytes(32769) == 8192
    assert bench.pitch_bytes(10_000_000) == 1_253_376


def test_wire_bytes_follow_the_packed_upload():
    """The bench's e2e wire bytes: offsets + per chunk either 4 bytes per id (raw) or ceil(n / 32) blocks
    of b words (b = ceil(log2 n_items) = 10 for 1,000 ids); small inputs and > 16,384 ids go raw."""
    import numpy as np
    n_tx = 300_000
    lens = np.full(n_tx, 7, np.uint64)
    offsets = np.zeros(n_tx + 1, np.uint64)
    np.cumsum(lens, out=offsets[1:])
    raw = offsets.nbytes + 4 * 7 * n_tx
    assert bench.wire_bytes(offsets, 20_000) == raw                 # > 16,384 ids
    assert bench.wire_bytes(offsets[:1001], 1000) == offsets[:1001].nbytes + 4 * 7 * 1000   # small input
    # 8 chunks of 40,960 transactions (37,500 rounded up to 8,192), the last one 13,280
    chunks = [40_960] * 7 + [n_tx - 7 * 40_960]
    packed = lambda n: -(-7 * n // 32) * 10 * 4
    assert bench.wire_bytes(offsets, 1000, 0) == offsets.nbytes + sum(packed(n) for n in chunks)
    assert bench.wire_bytes(offsets, 1000, 4) == offsets.nbytes + sum(
        4 * 7 * n if c % 4 == 0 else packed(n) for c, n in enumerate(chunks))
    assert bench.wire_bytes(offsets, 1000, 1) == raw
