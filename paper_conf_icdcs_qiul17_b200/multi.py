"""Multi-GPU sharding of the hot path (Sec. III-A, Eq. (2)).

One process per GPU (torch.distributed, NCCL):

  1. each rank runs Step 1 (MSP, dbg_msp_partition) on its own reads -- reads are independent
     (the paper splits the input into equal partitions, L396-398);
  2. fine partition p is owned by the rank r with bounds[r] <= p < bounds[r+1]; records are already
     in partition order, so the records for rank r are one contiguous slice -- ONE exchange
     (all_to_all_single over NVLink) routes them to their owner; per-partition sizes are summed with
     an all_reduce (they size the tables);
  3. each rank builds the subgraphs of its own partitions (Step 2, no inter-GPU traffic: identical
     vertices share a partition, L463-467);
  4. the totals are reduced with one all_reduce -- NCCL is used only for the exchange and the reduces.

The host-side logic (owner bounds, split sizes, exchange) runs on any backend; tests drive it with
gloo on CPU tensors (tests/test_multi.py).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def owner_bounds(n_fine: int, world: int) -> np.ndarray:
    """Contiguous fine-partition ranges, one per rank: rank r owns [b[r], b[r+1])."""
    return np.array([r * n_fine // world for r in range(world + 1)], dtype=np.int64)


def send_counts(part_records: np.ndarray, bounds: np.ndarray) -> np.ndarray:
    """Records this rank sends to each owner (its records are in partition order)."""
    c = np.concatenate([[0], np.cumsum(part_records, dtype=np.int64)])
    return c[bounds[1:]] - c[bounds[:-1]]


def exchange_records(records: torch.Tensor, part_records: np.ndarray, bounds: np.ndarray, rec_words: int,
                     group=None) -> tuple[torch.Tensor, int, np.ndarray]:
    """All-to-all of the partition-ordered records (int32 words, rec_words per record): returns the
    records of this rank's partitions from every rank (source-rank order), their count, and the
    per-source counts."""
    world = dist.get_world_size(group)
    dev = records.device
    sc = send_counts(part_records, bounds)
    sc_t = torch.from_numpy(sc).to(dev)
    all_sc = torch.empty(world * world, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(all_sc, sc_t, group=group)
    rank = dist.get_rank(group)
    rc = all_sc.view(world, world)[:, rank].cpu().numpy()
    n_send = int(sc.sum())
    out = torch.empty(max(int(rc.sum()), 1) * rec_words, dtype=torch.int32, device=dev)
    dist.all_to_all_single(out[: int(rc.sum()) * rec_words], records[: n_send * rec_words],
                           [int(x) * rec_words for x in rc], [int(x) * rec_words for x in sc], group=group)
    return out, int(rc.sum()), rc


def global_sizes(part_records: np.ndarray, part_kmers: np.ndarray, device, group=None):
    """Per-partition record and K-mer counts summed over ranks (one all_reduce)."""
    t = torch.from_numpy(np.concatenate([part_records, part_kmers]).astype(np.int64)).to(device)
    dist.all_reduce(t, group=group)
    t = t.cpu().numpy()
    n = len(part_records)
    return t[:n], t[n:]


def distributed_step(builder, d_bases, d_offsets, stream, out_cap: int, group=None):
    """One sharded pass of the hot path on this rank; returns nothing (totals in builder.d_stats)."""
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    builder.owned = (0, builder.np)
    builder.msp(d_bases, d_offsets, stream)                      # Step 1 on local reads
    while not builder.sync_sizes():                               # staging overflow: grown, repeat
        builder.msp(d_bases, d_offsets, stream)
    bounds = owner_bounds(builder.np, world)
    g_rec, g_kmr = global_sizes(builder.part_records, builder.part_kmers, builder.device, group)
    recv, n_recv, _ = exchange_records(builder.records, builder.part_records, bounds, builder.rec_words, group)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    builder.load_exchanged(recv, n_recv, g_rec, g_kmr, (lo, hi), stream)
    builder.plan(stream)
    builder.reset_output(out_cap, stream)
    builder.step2(stream)                                         # Step 2 on owned partitions
