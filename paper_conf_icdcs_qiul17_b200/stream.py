"""Row f2: the overlapped ingest pipeline for inputs larger than HBM (Sec. III-E,
L687-707: "an execution pipeline to overlap the input data transfer, the computation on processors
and the output data transfer ... Step 1 consists of extracting read partitions, superkmer
generation, and superkmer output.  Step 2 consists of superkmer partition loading, hashing, and
subgraph output").

The paper writes the superkmer partitions to disk after Step 1 and loads them one at a time in
Step 2.  On B200 the superkmers of a range of partitions stay in HBM instead, and the reads are
streamed from pinned host memory in batches, once per range:

    sizing pass   for each read batch: H2D (copy stream) || dbg_msp_partition_range(all
                  partitions, staging_cap 0) -- per-partition record counts only
    plan          consecutive fine-partition ranges whose records fit the staging budget
    range r       for each read batch: H2D (copy stream) || dbg_msp_partition_range(range r,
                  append) -- the range's superkmers accumulate in the staging
                  -> pass 2 (scatter) -> Step 2 of the range (on chip + global tier)
                  -> D2H of the range's vertices (copy stream) || the next range's Step 1

Input transfer, computation and output transfer of consecutive batches / ranges overlap through
two CUDA streams and events (the three pipeline stages of Fig. 5); two device buffers per stream
direction make the double buffering.  ``resident=True`` uploads the read batches once and keeps
them in HBM (only the partition ranges are passes).  Every kernel is the single-pass path's
(libdbg.so); this module only sequences calls and copies.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

from . import _lib
from ._lib import VERTEX_DTYPE
from .graph import DbgBuilder, auto_fine_p, auto_refine, encode_reads


@dataclass
class StreamResult:
    vertices: np.ndarray          # VERTEX_DTYPE, sorted by (kmer_hi, kmer_lo) when requested
    stats: dict
    n_kmers: int
    ranges: list = field(default_factory=list)     # fine-partition ranges, one pass each
    batches: int = 0
    h2d_bytes: int = 0


def _batches(seq: np.ndarray, offsets: np.ndarray, batch_reads: int):
    """Host stage 1: ASCII reads -> pinned packed batches (a0 per batch; offsets rebased)."""
    offsets = np.asarray(offsets, dtype=np.int64)
    out = []
    for r0 in range(0, len(offsets) - 1, batch_reads):
        r1 = min(len(offsets) - 1, r0 + batch_reads)
        b0, b1 = int(offsets[r0]), int(offsets[r1])
        packed = encode_reads(seq[b0:b1], pin=True)
        offs = torch.from_numpy((offsets[r0:r1 + 1] - b0).astype(np.int64)).pin_memory()
        out.append((packed, offs, r1 - r0))
    return out


def plan_ranges(part_records: np.ndarray, budget_records: int) -> list[tuple[int, int]]:
    """Consecutive fine-partition ranges whose record counts fit the staging budget (a single
    partition larger than the budget gets a range of its own; the staging grows for it)."""
    ranges, lo, acc = [], 0, 0
    for p, n in enumerate(part_records.tolist()):
        if acc and acc + n > budget_records:
            ranges.append((lo, p))
            lo, acc = p, 0
        acc += n
    ranges.append((lo, len(part_records)))
    return ranges


class StreamingBuilder:
    """Streams read batches through Step 1 once per partition range; Step 2 per range."""

    def __init__(self, builder: DbgBuilder, staging_budget_records: int, resident: bool = False):
        if builder.mode != "smem":
            raise ValueError("the streaming pipeline runs the smem Step 2")
        self.b = builder
        self.budget = max(1, int(staging_budget_records))
        self.resident = resident
        dev = builder.device
        self.compute = torch.cuda.current_stream(dev)
        self.copy = torch.cuda.Stream(dev)   # H2D of the read batches
        self.d2h = torch.cuda.Stream(dev)    # D2H of the ranges' vertices (its own stream, so the next
        self.h2d_bytes = 0                   # range's H2D does not queue behind it)

    # -- input stage: batch i into device slot i % 2 (or its resident copy)
    def _inputs(self, batches):
        """Yields (d_bases, d_offsets, n_reads) per batch, each H2D issued on the copy stream
        ahead of its use, overlapped with the previous batch's MSP on the compute stream."""
        dev = self.b.device
        if self.resident:
            if not hasattr(self, "_resident"):
                with torch.cuda.stream(self.copy):
                    self._resident = [(p.to(dev, non_blocking=True), o.to(dev, non_blocking=True), n)
                                      for p, o, n in batches]
                    self.h2d_bytes += sum(p.numel() * 8 + o.numel() * 8 for p, o, _ in batches)
                self.compute.wait_stream(self.copy)
            yield from self._resident
            return
        cap_w = max(p.numel() for p, _, _ in batches)
        cap_o = max(o.numel() for _, o, _ in batches)
        slots = [(torch.empty(cap_w, dtype=torch.int64, device=dev), torch.empty(cap_o, dtype=torch.int64, device=dev))
                 for _ in range(2)]
        free = [torch.cuda.Event(), torch.cuda.Event()]
        ready = [torch.cuda.Event(), torch.cuda.Event()]
        for ev in free:
            ev.record(self.compute)

        def issue(i):
            p, o, _ = batches[i]
            db, do = slots[i % 2]
            self.copy.wait_event(free[i % 2])  # the MSP that read this slot two batches ago is done
            with torch.cuda.stream(self.copy):
                db[:p.numel()].copy_(p, non_blocking=True)
                do[:o.numel()].copy_(o, non_blocking=True)
            ready[i % 2].record(self.copy)
            self.h2d_bytes += p.numel() * 8 + o.numel() * 8

        issue(0)
        for i in range(len(batches)):
            if i + 1 < len(batches):
                issue(i + 1)  # stage 1 of the next batch overlaps stage 2 of this one
            self.compute.wait_event(ready[i % 2])
            p, o, n = batches[i]
            db, do = slots[i % 2]
            yield db[:p.numel()], do[:o.numel()], n
            free[i % 2].record(self.compute)

    def _pass1(self, batches, lo: int, hi: int, count_only: bool) -> None:
        b = self.b
        if count_only:
            saved, b.staging = b.staging, torch.empty(0, dtype=torch.int32, device=b.device)
        for i, (db, do, n) in enumerate(self._inputs(batches)):
            _lib.dbg_msp_partition_range(b.prm, db, db.numel(), do, n, b.part_set(False), lo, hi, i > 0,
                                         self.compute)
        if count_only:
            b.staging = saved
        if b._h_sizes.numel() != 2 * b.np:
            b._h_sizes = torch.empty(2 * b.np, dtype=torch.int64, pin_memory=True)
        with torch.cuda.stream(self.compute):
            b._h_sizes[:b.np].copy_(b.d_n_records, non_blocking=True)
            b._h_sizes[b.np:].copy_(b.d_n_kmers, non_blocking=True)
        b._sizes_ev.record(self.compute)
        b._sizes_pending = True

    def run(self, batches, sort: bool = True, out_frac: float = 0.5, sink=None) -> StreamResult:
        """sink: None -- every range's vertices go D2H and are returned; else sink(d_records, n) is
        called per range with the range's records on the device (a uint8 view of n dbg_vertex), for
        graphs larger than host memory (the sink copies out what it needs); the result then holds
        no vertices, and stats["checksum"] is the order-independent checksum over all ranges."""
        b = self.b
        # sizing pass: per-partition record counts over every batch (nothing staged)
        self._pass1(batches, 0, b.np, count_only=True)
        b._sizes_ev.synchronize()
        b._sizes_pending = False
        b.part_records = b._h_sizes[:b.np].numpy().copy()
        b.part_kmers = b._h_sizes[b.np:].numpy().copy()
        total_kmers = int(b.part_kmers.sum())
        sizing = b.part_records.copy()  # the range passes overwrite b.part_records
        ranges = plan_ranges(sizing, self.budget)
        parts, stats = [], {"distinct": 0, "sum_count": 0, "sum_edges": 0}
        pending = None  # (host buffer, event, n) of the previous range's output D2H
        for lo, hi in ranges:
            want = int(sizing[lo:hi].sum())
            b.staging = torch.empty(0, dtype=torch.int32, device=b.device) if want == 0 else b.staging
            if b.staging.numel() < want * b.rec_words:
                b.staging = torch.empty(max(want, 1) * b.rec_words, dtype=torch.int32, device=b.device)
            b.records = b.records if b.records.numel() >= b.staging.numel() else torch.empty_like(b.staging)
            self._pass1(batches, lo, hi, count_only=False)
            if not b.sync_sizes():
                raise RuntimeError("staging overflow in a streamed range (sizing pass disagrees)")
            # pass 2 (scatter) and Step 2 of this range
            _lib.dbg_msp_partition(b.prm, 1, 1, b.d_rec_off, 0, b.part_set(True), self.compute)
            b.owned = (lo, hi)
            n_k = int(b.part_kmers[lo:hi].sum())
            if pending is not None:  # the previous range's output buffer is read before reuse
                self.compute.wait_event(pending[1])
            b.reset_output(int(out_frac * n_k) + 1024, self.compute)
            while True:
                b.step2(self.compute)
                st = _lib.dbg_sync_status(b.d_status, self.compute)
                if st == _lib.DBG_ENOSPACE and int(b.d_n_out.item()) > b.out_cap():
                    b.reset_output(int(b.d_n_out.item()), self.compute)
                    continue
                if st != _lib.DBG_OK:
                    raise _lib.DbgError("streamed Step 2", st, _lib.dbg_status_string(st))
                break
            n_out = int(b.d_n_out.item())
            for k, v in zip(("distinct", "sum_count", "sum_edges"), b.d_stats[:3].cpu().numpy().view(np.uint64)):
                stats[k] += int(v)
            if sink is not None:
                with torch.cuda.stream(self.compute):
                    b.d_stats[3].zero_()
                _lib.dbg_checksum_vertices(b.prm, b.out, n_out, b.d_stats, self.compute)
                stats["checksum"] = (stats.get("checksum", 0) + int(b.d_stats[3:].cpu().numpy().view(np.uint64)[0])) \
                    % (1 << 64)
                sink(b.out[:n_out * VERTEX_DTYPE.itemsize], n_out)
                continue
            if pending is not None:
                pending[1].synchronize()
                parts.append(pending[0][:pending[2]].copy())
            # stage 3: D2H of this range's vertices on the copy stream, overlapped with the next
            # range's Step 1
            host = torch.empty(n_out * VERTEX_DTYPE.itemsize, dtype=torch.uint8, pin_memory=True)
            done = torch.cuda.Event()
            self.d2h.wait_stream(self.compute)
            with torch.cuda.stream(self.d2h):
                host.copy_(b.out[:n_out * VERTEX_DTYPE.itemsize], non_blocking=True)
            done.record(self.d2h)
            pending = (host.numpy().view(VERTEX_DTYPE), done, n_out)
        if pending is not None:
            pending[1].synchronize()
            parts.append(pending[0][:pending[2]].copy())
        verts = np.concatenate(parts) if parts else np.zeros(0, dtype=VERTEX_DTYPE)
        if sort:
            verts = verts[np.lexsort((verts["kmer_lo"], verts["kmer_hi"]))]
        b.owned = (0, b.np)
        return StreamResult(verts, stats, total_kmers, ranges, len(batches), self.h2d_bytes)


def build_graph_streamed(seq: np.ndarray, offsets: np.ndarray, k: int, p: int, num_partitions: int,
                         batch_reads: int = 1 << 20, staging_budget_records: int = 1 << 26,
                         resident: bool = False, lam: float = 2.0, alpha: float = 0.5, device="cuda",
                         refine: int | str = "auto", fine_p: int | str = "auto", min_count: int = 0,
                         smem_split: int = 0, sort: bool = True) -> StreamResult:
    """The public call of row f2: reads (ASCII, concatenated) -> graph records, streamed."""
    lens = np.diff(np.asarray(offsets, dtype=np.int64))
    n_kmers = int(np.maximum(lens - k + 1, 0).sum())
    if refine == "auto":
        refine = auto_refine(n_kmers, k, p, num_partitions, lam, alpha)
    if fine_p == "auto":
        fine_p = auto_fine_p(n_kmers, k, p, lam, alpha)
    b = DbgBuilder(k, p, num_partitions, lam, alpha, device, mode="smem", refine=refine, smem_split=smem_split,
                   fine_p=fine_p, min_count=min_count)
    batches = _batches(np.ascontiguousarray(seq, dtype=np.uint8), offsets, batch_reads)
    return StreamingBuilder(b, staging_budget_records, resident).run(batches, sort=sort)
