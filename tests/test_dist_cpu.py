"""Multi-GPU host logic on CPU (world_size 2, gloo, 127.0.0.1): the transaction sharding plan
used by bench.py / gpa_mine under torchrun, the per-level count all-reduce semantics (partial
counts of the shards sum to the unsharded counts -- computed here with the oracle, the CUDA path
needs GPUs), and the broadcast of the 128-byte NCCL unique id through torch.distributed."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, n_tx, cands, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, ROOT)
    import bench
    b0, b1 = bench.shard_range(n_tx, rank, world, gen.CONFIGS[name].kind == "quest")
    ds = gen.make(name, tx_begin=b0, tx_end=b1, n_tx=n_tx)
    # level-1 histogram and candidate counts of this shard, summed across ranks (the library's
    # ncclAllReduce(u32, sum) per generation)
    h = torch.from_numpy(np.bincount(ds.items, minlength=ds.n_items).astype(np.int64))
    c = torch.from_numpy(oracle.support_batch(ds.offsets, ds.items, ds.n_items, cands, threads=1).astype(np.int64))
    ntx = torch.tensor([ds.n_tx], dtype=torch.int64)
    for t in (h, c, ntx):
        tdist.all_reduce(t)
    # the NCCL unique id travels as 128 bytes from rank 0
    uid = bytes(range(128)) if rank == 0 else bytes(128)
    t = torch.tensor(list(uid), dtype=torch.uint8)
    tdist.broadcast(t, 0)
    out_q.put((rank, b0, b1, h.numpy(), c.numpy(), int(ntx.item()), bytes(t.tolist())))
    tdist.destroy_process_group()


@pytest.mark.parametrize("name,n_tx", [("t40i10d100k", 250_000), ("mushroom", 8124)])
def test_two_rank_sharding_matches_unsharded(name, n_tx):
    full = gen.make(name, n_tx=n_tx)
    theta = oracle.min_count(full.n_tx, gen.CONFIGS[name].minsup)
    ref = oracle.mine_ds(full, theta)
    rng = np.random.default_rng(0)
    picks = []
    for lv in ref.levels[1:4]:
        idx = rng.choice(len(lv.cand), size=min(40, len(lv.cand)), replace=False)
        picks.append(lv.cand[idx])
    k = picks[0].shape[1]
    cands = picks[0]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, n_tx, cands, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, a0, a1, h0, c0, n0, u0), (r1, b0, b1, h1, c1, n1, u1) = res
    # contiguous, ordered, covering, 512-aligned except the end
    assert a0 == 0 and a1 == b0 and b1 == n_tx and a1 % 512 == 0 and 0 < a1 < n_tx
    assert n0 == n1 == n_tx
    # all-reduced generation-1 counts and candidate counts equal the unsharded ones
    assert np.array_equal(h0, ref.levels[0].count.astype(np.int64)) and np.array_equal(h0, h1)
    want = oracle.support_batch(full.offsets, full.items, full.n_items, cands).astype(np.int64)
    assert np.array_equal(c0, want) and np.array_equal(c1, want)
    assert u0 == u1 == bytes(range(128))


def test_shard_ranges_many_worlds():
    import sys
    sys.path.insert(0, ROOT)
    import bench
    for n_tx, quest in ((10_000_000, True), (340_183, False), (8124, False), (3196, False)):
        for world in (1, 2, 4, 8):
            r = [bench.shard_range(n_tx, i, world, quest) for i in range(world)]
            assert r[0][0] == 0 and r[-1][1] == n_tx
            for (a, b), (c, d) in zip(r, r[1:]):
                assert b == c and b % 512 == 0


def _host_allreduce_worker(rank, world, port, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, ROOT)
    import paper_conf_cluster_zhangzb11a_b200 as gpa
    # the values the library sends: counts (u32 sums near / above 2^31), flags and n_items
    # agreement (u32 max incl. complements ~n), N (u64 sums)
    a = np.array([2 ** 31 + rank, 7 * rank, 0xFFFFFFFF - rank, 1], dtype=np.uint32)
    b = np.array([5 + rank, 2 ** 32 - 10 * (rank + 1)], dtype=np.uint32)
    c = np.array([2 ** 40 + rank, 2 ** 63 + rank], dtype=np.uint64)
    d = np.array([2 ** 63 + rank, rank], dtype=np.uint64)
    gpa.torch_host_allreduce(a, "max")
    gpa.torch_host_allreduce(b, "sum")
    gpa.torch_host_allreduce(c, "sum")
    gpa.torch_host_allreduce(d, "max")
    out_q.put((rank, a.tolist(), b.tolist(), c.tolist(), d.tolist()))
    tdist.destroy_process_group()


def test_host_transport_callback_unsigned_semantics():
    """The host-staged transport's callback (gpa_dist_create_host over gloo, used by the world-2
    GPU test): element-wise unsigned max and wrap-around sums of u32 / u64 arrays across 2 ranks."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    ps = [ctx.Process(target=_host_allreduce_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    want_a = [2 ** 31 + 1, 7, 0xFFFFFFFF, 1]
    want_b = [5 + 6, (2 ** 32 - 10 + 2 ** 32 - 20) % 2 ** 32]
    want_c = [2 ** 41 + 1, (2 ** 64 + 1) % 2 ** 64]
    want_d = [2 ** 63 + 1, 1]
    for _, a, b, c, d in res:
        assert a == want_a and b == want_b and c == want_c and d == want_d
