"""Row e on one GPU: two processes (ranks) on cuda:0 run multi.ShardedBuilder end to end -- each
its own half of the reads through Step 1, emission of every record into its owner's buffer through
the CUDA IPC peer pointer (the multi-GPU data path; between two processes on one device the IPC
mapping is the same mechanism as over NVLink), Step 2 on the owned partitions.  The union of the
two ranks' vertices must equal the oracle on all reads, bit-exact, on each of two consecutive steps
(the second step must reuse the buffers: no staging overflow, no IPC re-open).

The control plane runs on gloo here (NCCL refuses two ranks on one device); on a multi-GPU box the
histogram gather / K-mer sum use NCCL (multi.gather_rows / all_reduce_sum).
"""
import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import VERTEX_DTYPE  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import build as _build  # noqa: E402
from synth import ReadSet, genome, make_reads  # noqa: E402

from gpu_helpers import compare_vertices  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NT = os.cpu_count() or 1
_build.build()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _reads(n=20_000, seed=9):
    g = genome(120_000, seed=seed)
    seq, offs = make_reads(g, n, 100, 0.01, seed=seed + 1)
    return ReadSet(seq, offs)


def _rank(rank, world, port, k, p, np_, refine, n_reads, q, two_level=False):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icdcs_qiul17_b200 import encode_reads, _lib
    from paper_conf_icdcs_qiul17_b200.multi import ShardedBuilder

    rs = _reads(n_reads)
    total = rs.n_kmers(k)
    mine = rs.subset(n_reads * rank // world, n_reads * (rank + 1) // world)
    sb = ShardedBuilder(k, p, np_, total, "cuda:0", refine=refine)
    if two_level:  # pass 2 through the two-level scatter at this size: buckets locally, then the peers
        sb.src.two_level_min_bytes, sb.src.two_level_words = 0, (4, 8, 16)
        assert sb.src.use_two_level() or sb.src.staging.numel() == 0
    d_bases, d_off = sb.src.upload(encode_reads(mine.seq), mine.offsets)
    stream = torch.cuda.current_stream()
    outs = []
    for step in range(2):
        sb.step(d_bases, d_off, stream, out_cap=total // 2 + 1024)
        st = _lib.dbg_sync_status(sb.dst.d_status, stream)
        outs.append((st, sb.dst.vertices(sort=False).tobytes(), sb.pass1_runs, sb.peers.reopened, sb.n_recv))
    q.put((rank, outs))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("k,p,np_,refine,two_level", [(31, 11, 16, 64, False), (63, 19, 8, 16, False),
                                                      (31, 11, 16, 1024, True), (63, 19, 8, 2048, True)])
def test_sharded_builder_two_ranks_one_gpu_equals_oracle(k, p, np_, refine, two_level):
    import torch.multiprocessing as mp

    world, n_reads = 2, 20_000
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, world, port, k, p, np_, refine, n_reads, q, two_level))
             for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for pr in procs:
        pr.join(timeout=120)
    rs = _reads(n_reads)
    orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT)
    for step in range(2):
        parts = []
        for r in range(world):
            st, raw, pass1_runs, reopened, n_recv = res[r][step]
            assert st == 0 and pass1_runs == 1   # no staging overflow (no repeated pass 1)
            assert reopened == 1          # the peer's buffer was mapped once and reused
            assert n_recv > 0
            parts.append(np.frombuffer(raw, dtype=VERTEX_DTYPE))
        allv = np.concatenate(parts)
        allv = allv[np.lexsort((allv["kmer_lo"], allv["kmer_hi"]))]
        compare_vertices(allv, orc)
