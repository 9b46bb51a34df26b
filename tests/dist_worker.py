"""World-size-2 worker of tests/test_dist_gpu.py: launched by torch.distributed.run, both ranks on
cuda:0, collectives over gloo through the library's host-staged transport
(gpa_dist_create_host) -- NCCL refuses two ranks on one GPU, and the GPU box has one.

Each rank mines its contiguous transaction shard (gpa_mine with dist, the library's sharded path:
rank-local bitset, per-generation all-reduce of the count vector) and must reproduce the
oracle's every (C_k, count) and F of the WHOLE database; gpa_count over dist must return global
supports; every rank must have issued the same collective sequence (gpa_dist_log); a rank-local
input error must fail on every rank instead of stranding the other inside a collective.
Writes one JSON line per check to $GPA_DIST_OUT.<rank>; exits non-zero on any failure.
"""
import json
import os
import sys
import traceback

import numpy as np
import torch
import torch.distributed as tdist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_cluster_zhangzb11a_b200 as gpa  # noqa: E402

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
out = open(os.environ.get("GPA_DIST_OUT", "/tmp/gpa_dist") + f".{rank}", "w")


def report(**kw):
    kw["rank"] = rank
    out.write(json.dumps(kw) + "\n")
    out.flush()


def logs_equal(d: gpa.Dist) -> bool:
    mine = d.log()
    allv = [None] * world
    tdist.all_gather_object(allv, mine)
    return all(v == allv[0] for v in allv) and len(mine) > 0


def shard_bounds(n_tx: int, cut: int):
    return (0, cut) if rank == 0 else (cut, n_tx)


def check_mine(name, ds, theta, cut, dist):
    b0, b1 = shard_bounds(ds.n_tx, cut)
    shard = gen.subset(ds, b0, b1)
    ref = oracle.mine_ds(ds, theta)
    res = gpa.mine(shard, min_count=theta, dist=dist, options=gpa.Options(device=0), keep_candidates=True)
    assert res.n_tx == ds.n_tx, (res.n_tx, ds.n_tx)
    assert len(res.levels) == len(ref.levels), (len(res.levels), len(ref.levels))
    for lv, rl in zip(res.levels, ref.levels):
        assert np.array_equal(lv.cand, rl.cand), f"{name}: C_{lv.k} differs"
        assert np.array_equal(lv.counts, rl.count), f"{name}: counts of C_{lv.k} differ"
    assert res.frequent() == ref.frequent()
    # gpa_count over the same communicator: global supports of C_3 (or the deepest level)
    lv = ref.levels[min(2, len(ref.levels) - 1)]
    if len(lv.cand):
        with gpa.Bitset(shard, row_min_count=theta, dist=dist, options=gpa.Options(device=0)) as bs:
            assert np.array_equal(bs.count(lv.cand), lv.count), f"{name}: gpa_count over dist"
    return len(ref.levels), sum(len(l.cand) for l in ref.levels)


def main():
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    d = gpa.Dist.host_from_torch(0)
    ok = True
    cases = [
        # (name, dataset, threshold, rank-0 shard size: a 512-aligned interior cut)
        ("mushroom", gen.make("mushroom"), oracle.min_count(8124, "0.20"), 4096),
        ("accidents", gen.make("accidents"), oracle.min_count(340_183, "0.30"), 170_496),
        ("t40i10d100k", gen.make("t40i10d100k"), oracle.min_count(100_000, "0.01"), 51_200),
        # shards on both sides of the overlapped-ingest threshold (262,144 transactions): the
        # ingest path must be chosen collectively (rank 0 alone would be eligible)
        ("straddle", gen.make("accidents"), oracle.min_count(340_183, "0.30"), 300_032),
    ]
    for name, ds, theta, cut in cases:
        try:
            n0 = len(d.log())
            gens, ncand = check_mine(name, ds, theta, cut, d)
            same = logs_equal(d)
            report(case=name, ok=same, generations=gens, candidates=ncand, collectives=len(d.log()) - n0)
            ok &= same
        except Exception as e:
            traceback.print_exc()
            report(case=name, ok=False, error=str(e))
            ok = False
            break
    # a rank-local input error: rank 1's CSR is invalid (offsets[0] != 0); both ranks must fail
    # (GPA_ERR_INVALID), neither may hang inside a collective
    try:
        good = gen.random_db(3, 2000, 20, max_len=8)
        off = good.offsets.copy()
        if rank == 1:
            off[0] = 1
        try:
            gpa.mine(off, good.items, good.n_items, min_count=10, dist=d, options=gpa.Options(device=0))
            report(case="local_error", ok=False, error="no error raised")
            ok = False
        except gpa.GpaError as e:
            report(case="local_error", ok=e.status == 1, status=e.status, msg=str(e))
            ok &= e.status == 1
        # an invalid candidate on one rank only: gpa_count fails on both
        with gpa.Bitset(good, dist=d, options=gpa.Options(device=0)) as bs:
            cand = np.array([[1, 2]], np.uint32) if rank == 0 else np.array([[2, 1]], np.uint32)
            try:
                bs.count(cand)
                report(case="local_cand_error", ok=False, error="no error raised")
                ok = False
            except gpa.GpaError as e:
                report(case="local_cand_error", ok=e.status == 1, status=e.status)
                ok &= e.status == 1
        same = logs_equal(d)
        report(case="logs_after_errors", ok=same)
        ok &= same
    except Exception as e:
        traceback.print_exc()
        report(case="errors", ok=False, error=str(e))
        ok = False
    d.close()
    tdist.destroy_process_group()
    out.close()
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
