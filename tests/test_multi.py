"""Multi-GPU host logic on CPU (gloo, world size 2): owner bounds, the histogram collectives, the
peer-buffer handle protocol, and the read shards of strong scaling.

The data path itself (emission into peer buffers through IPC pointers) needs a GPU: it is covered
by tests/test_gpu_multi.py (two processes on one GPU).
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


def test_owner_bounds():
    sys.path.insert(0, ROOT)
    from paper_conf_icdcs_qiul17_b200.multi import owner_bounds

    b = owner_bounds(10, 3)
    assert b.tolist() == [0, 3, 6, 10]
    assert owner_bounds(5, 8)[-1] == 5 and np.all(np.diff(owner_bounds(5, 8)) >= 0)
    for n, w in ((1_579_008, 8), (7, 2), (1, 1)):
        b = owner_bounds(n, w)
        assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0) and np.diff(b).max() - np.diff(b).min() <= 1


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icdcs_qiul17_b200.multi import PeerBuffers, all_reduce_sum, gather_rows

    res = {}
    t = torch.arange(5, dtype=torch.int64) + 10 * rank
    res["gather"] = gather_rows(t).tolist()
    u = torch.full((3,), rank + 1, dtype=torch.int64)
    res["sum"] = all_reduce_sum(u).tolist()
    # handle protocol with fake IPC: a handle names (rank, generation); opening one "maps" it
    opened = []
    pb = PeerBuffers(export=lambda x: ("h", rank, x.numel()),
                     open_=lambda h, n: (None, 1000 * h[1] + h[2]) if not opened.append(h) else None)
    bufs = [torch.zeros(4, dtype=torch.int32), None, torch.zeros(9, dtype=torch.int32)]
    bufs[1] = bufs[0]
    trace = []
    for step in range(3):
        # rank 1 reallocates its buffer at step 2 only; rank 0 never does
        b = bufs[step] if rank == 1 else bufs[0]
        ptrs = pb.update(b)
        trace.append((ptrs[1 - rank], len(opened)))
    res["trace"] = trace
    q.put((rank, res))
    dist.destroy_process_group()


def test_collectives_and_peer_handle_protocol_gloo_world2():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert res[r]["gather"] == [0, 1, 2, 3, 4, 10, 11, 12, 13, 14]
        assert res[r]["sum"] == [3, 3, 3]
    # rank 0 sees rank 1's buffer: opened at step 0 (4 words), unchanged at step 1 (no reopen),
    # reopened at step 2 (9 words)
    assert res[0]["trace"] == [(1004, 1), (1004, 1), (1009, 2)]
    # rank 1 opens rank 0's buffer once
    assert [n for _, n in res[1]["trace"]] == [1, 1, 1] and res[1]["trace"][0][0] == 4


def test_read_shards_concatenate_to_the_configuration():
    """Strong scaling: the ranks' read ranges are exactly the configuration's reads."""
    sys.path.insert(0, ROOT)
    from synth import make_config

    full = make_config("ecoli", scale=0.6)     # 1.66 M reads: two generator chunks
    for w in (2, 3):
        parts = [make_config("ecoli", scale=0.6, shard=(r, w)) for r in range(w)]
        assert sum(p.n_reads for p in parts) == full.n_reads
        assert np.array_equal(np.concatenate([p.seq for p in parts]), full.seq)


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
