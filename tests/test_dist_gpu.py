"""The library's sharded path with TWO ranks, executed on the GPU.

The GPU box has one B200 and NCCL refuses two ranks on one device, so the two ranks (one process
each, launched by torch.distributed.run) share cuda:0 and reduce through the library's host-staged
transport over gloo (gpa_dist_create_host): the same library code path as NCCL -- rank-local
static bitsets over contiguous transaction shards, one all-reduce of every generation's count
vector, collective path decisions -- only the transport differs.  Checks (tests/dist_worker.py):
every (C_k, count) and F of the whole database equal to the oracle on mushroom, accidents,
T40I10D100K and shards straddling the overlapped-ingest threshold; gpa_count over dist; identical
collective logs on both ranks; rank-local input errors fail on both ranks without a hang.
"""
import json
import os
import socket
import subprocess
import sys

import pytest

import gen
import oracle
import paper_conf_cluster_zhangzb11a_b200 as gpa

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_world2_host_transport_on_one_gpu(tmp_path):
    outp = str(tmp_path / "dist")
    env = dict(os.environ, GPA_DIST_OUT=outp, PYTHONPATH=ROOT)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.join(ROOT, "tests", "dist_worker.py")]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    lines = []
    for r in range(2):
        if os.path.exists(f"{outp}.{r}"):
            lines += [json.loads(x) for x in open(f"{outp}.{r}") if x.strip()]
    assert p.returncode == 0, (p.stdout[-3000:], p.stderr[-3000:], lines)
    cases = {(x["case"], x["rank"]) for x in lines if x.get("ok")}
    for case in ("mushroom", "accidents", "t40i10d100k", "straddle", "local_error", "local_cand_error",
                 "logs_after_errors"):
        assert (case, 0) in cases and (case, 1) in cases, (case, lines)


def test_dist_log_single_rank_host_transport():
    """One rank, host transport: the collective log records each all-reduce (op, dtype, n) in order;
    the sum over one rank is the identity, so the result equals the oracle."""
    calls = []

    def allreduce(arr, op):
        calls.append((op, arr.dtype.itemsize, len(arr)))

    d = gpa.Dist(0, 1, 0, host_allreduce=allreduce)
    try:
        ds = gen.make("chess")
        theta = oracle.min_count(ds.n_tx, "0.90")
        res = gpa.mine(ds, min_count=theta, dist=d, options=gpa.Options(device=0), keep_candidates=True)
        ref = oracle.mine_ds(ds, theta)
        assert res.frequent() == ref.frequent()
        log = d.log()
        assert len(log) == len(calls) > 0
        # first collective: the input agreement (3 x u32 max); then validation flags, histogram, N
        assert log[0] == (gpa.OP_MAX, gpa.DT_U32, 3)
        assert (gpa.OP_SUM, gpa.DT_U32, ds.n_items) in log
        n1 = int((ref.levels[0].count >= theta).sum())
        assert (gpa.OP_SUM, gpa.DT_U32, n1 * (n1 - 1) // 2) in log     # generation-2 counts
        for op, isz, n in calls:
            assert op in ("sum", "max") and isz in (4, 8) and n > 0
    finally:
        d.close()


def test_host_transport_callback_failure_marks_handle():
    """A failing collective (callback returns non-zero) fails the call with GPA_ERR_NCCL and the
    handle reports GPA_ERR_STATE afterwards."""
    def allreduce(arr, op):
        raise RuntimeError("peer lost")

    d = gpa.Dist(0, 1, 0, host_allreduce=allreduce)
    try:
        ds = gen.make("chess")
        with pytest.raises(gpa.GpaError) as e:
            gpa.mine(ds, min_count=100, dist=d, options=gpa.Options(device=0))
        assert e.value.status == 5
        with pytest.raises(gpa.GpaError) as e:
            gpa.mine(ds, min_count=100, dist=d, options=gpa.Options(device=0))
        assert e.value.status == 6
    finally:
        d.close()
