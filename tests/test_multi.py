"""Multi-GPU host logic on CPU: owner bounds, split sizes and the record exchange with gloo, world size 2.

The exchange is the one data-path collective of the sharded path; here each rank
owns synthetic partition-ordered "records" whose words encode (source rank, partition, index), and
the test checks every rank receives exactly the records of the partitions it owns, from every rank.
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_owner_bounds_and_send_counts():
    sys.path.insert(0, ROOT)
    from paper_conf_icdcs_qiul17_b200.multi import owner_bounds, send_counts

    b = owner_bounds(10, 3)
    assert b.tolist() == [0, 3, 6, 10]
    pr = np.array([1, 0, 2, 5, 0, 0, 1, 1, 1, 4])
    assert send_counts(pr, b).tolist() == [3, 5, 7]
    assert owner_bounds(5, 8)[-1] == 5 and np.all(np.diff(owner_bounds(5, 8)) >= 0)


def _worker(rank, world, port, n_fine, R, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icdcs_qiul17_b200.multi import exchange_records, owner_bounds

    rng = np.random.default_rng(100 + rank)
    part_records = rng.integers(0, 4, size=n_fine)
    rows = []
    for p in range(n_fine):
        for i in range(part_records[p]):
            rows.append([rank, p, i] + [7] * (R - 3))
    recs = torch.tensor(np.array(rows, dtype=np.int32).reshape(-1)) if rows else torch.zeros(0, dtype=torch.int32)
    bounds = owner_bounds(n_fine, world)
    out, n, per_src = exchange_records(recs, part_records, bounds, R)
    got = out[: n * R].view(n, R).numpy()
    # expected: records of owned partitions from every source, in source order, partition order within
    lo, hi = bounds[rank], bounds[rank + 1]
    exp = []
    for src in range(world):
        pr = np.random.default_rng(100 + src).integers(0, 4, size=n_fine)
        for p in range(lo, hi):
            for i in range(pr[p]):
                exp.append([src, p, i] + [7] * (R - 3))
    q.put((rank, got.tolist() == exp, int(n), per_src.tolist()))
    dist.destroy_process_group()


@pytest.mark.parametrize("n_fine,R", [(37, 4), (5, 8)])
def test_exchange_records_gloo_world2(n_fine, R):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_fine, R, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _, _ in res), res


def test_stream_plan_ranges():
    """Row f2 host logic: consecutive ranges covering every fine partition, each within the staging
    budget unless a single partition exceeds it."""
    sys.path.insert(0, ROOT)
    from paper_conf_icdcs_qiul17_b200.stream import plan_ranges

    rng = np.random.default_rng(5)
    for budget in (1, 7, 50, 10 ** 9):
        rec = rng.integers(0, 20, 300)
        rr = plan_ranges(rec, budget)
        assert rr[0][0] == 0 and rr[-1][1] == len(rec)
        assert all(a[1] == b[0] for a, b in zip(rr, rr[1:]))
        for lo, hi in rr:
            assert hi > lo
            assert rec[lo:hi].sum() <= budget or (rec[lo:hi] > 0).sum() == 1
