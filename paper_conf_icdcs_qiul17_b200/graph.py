"""Host orchestration of the hot path over the C ABI (include/dbg.h).

PyTorch provides device memory and the stream; every step of the path runs in
libdbg.so kernels:

    a0     encode_reads          dbg_encode_ascii (host C)
    a1     DbgBuilder.upload     H2D copy of the packed reads
    a2-a4  DbgBuilder.msp        dbg_msp_partition pass 1 (minimizers, superkmers,
                                 staging, sizes) -> size readback -> pass 2 (scatter)
    a5     DbgBuilder.plan       dbg_table_plan[_split] (lambda/(4 alpha) N^i_kmer)
    a5-a7  DbgBuilder.step2      mode "smem" (the default): dbg_build_subgraphs_smem builds
                                 every partition whose table fits on chip (grouped, or split
                                 over several CTAs) in shared memory, then
                                 dbg_hash_build_list + dbg_extract_graph build the remaining
                                 (oversize) partitions in global tables, in batches;
                                 mode "resident": dbg_hash_build + dbg_extract_graph for all
    a7     DbgBuilder.vertices   dbg_sort_vertices + D2H

The paper builds "one partition at a time"; here the
device works on NP*refine fine partitions (dbg.h), many at once.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

from . import _lib
from ._lib import VERTEX_DTYPE, VERTEX_WIDE_DTYPE, STATS_FIELDS

# dbg.h: NP * refine <= 2^24 - 1 (the fine pid field of the record header)
MAX_FINE_PARTITIONS = (1 << 24) - 1


def encode_reads(seq: np.ndarray, pin: bool = False) -> torch.Tensor:
    """Row a0: ASCII reads (concatenated) -> packed 2-bit words (uint64 as int64 tensor)."""
    seq = np.ascontiguousarray(seq, dtype=np.uint8)
    n_words = _lib.dbg_packed_words(len(seq))
    out = torch.empty(n_words, dtype=torch.int64, pin_memory=pin)
    _lib.dbg_encode_ascii(seq, out.data_ptr())
    return out


@dataclass
class GraphResult:
    vertices: np.ndarray | None          # VERTEX_DTYPE records (sorted if requested), or None
    n_vertices: int
    stats: dict
    n_kmers: int
    part_kmers: np.ndarray
    part_records: np.ndarray
    batches: list = field(default_factory=list)


class _null:
    def __enter__(self):
        return None

    def __exit__(self, *a):
        return False


def _grow(t: torch.Tensor, n: int, dtype, device, slack: float = 1.0) -> torch.Tensor:
    if t.numel() >= n and t.numel() > 0:
        return t
    del t
    return torch.empty(max(int(n * slack), 16), dtype=dtype, device=device)


class DbgBuilder:
    """Reusable buffers + the call sequence of the path for one (K, P, NP) setting."""

    def __init__(self, k: int, p: int, num_partitions: int, lam: float = 2.0, alpha: float = 0.5,
                 device: str | torch.device = "cuda", table_budget_bytes: int | None = None,
                 mode: str = "smem", refine: int = 1, smem_split: int = 0,
                 fine_p: int = 0, min_count: int = 0):
        if k % 2 == 0 or not 1 <= k <= 127:
            raise ValueError("K must be odd and 1..127 (DESIGN.md reading C)")
        if k > 63 and mode != "resident":
            raise ValueError("K > 63 (row f3) runs through the resident tables: mode='resident'")
        if not 1 <= p <= min(k, 31):
            raise ValueError("P must be in 1..min(K, 31)")
        if mode not in ("smem", "resident"):
            raise ValueError(mode)
        self.k, self.p, self.mode = k, p, mode
        self.vdtype = VERTEX_WIDE_DTYPE if k > 63 else VERTEX_DTYPE  # dbg_vertex_wide for K > 63
        self.np_out = num_partitions                 # the paper's NP (dbg_vertex.pid)
        self.refine = max(1, int(refine))
        self.np = num_partitions * self.refine       # fine partitions the device works on
        self.owned = (0, self.np)  # fine partitions this builder hashes (multi-GPU: a shard)
        self.smem_split = int(smem_split)  # 0: library default (dbg_params.smem_split)
        self.fine_p = int(fine_p)          # 0: P (dbg_params.fine_p)
        self.min_count = int(min_count)    # row f4: drop vertices with count < min_count (0, 1: none)
        self.prm = _lib.params(k, p, num_partitions, lam, alpha, self.refine, self.smem_split, self.fine_p,
                               self.min_count)
        self.device = torch.device(device)
        _lib.load()
        self.rec_words = _lib.dbg_record_words(self.prm)
        self.slot_bytes = _lib.dbg_slot_bytes(self.prm)
        self.key_bytes = _lib.dbg_key_bytes(self.prm)
        dev = self.device
        NP = self.np
        i64 = dict(dtype=torch.int64, device=dev)
        self.d_n_records = torch.zeros(NP, **i64)
        self.d_n_kmers = torch.zeros(NP, **i64)
        self.d_rec_off = torch.zeros(NP + 1, **i64)
        self.d_fill = torch.zeros(NP, **i64)
        self.d_staged = torch.zeros(1, **i64)
        self.d_tab_off = torch.zeros(NP + 1, **i64)
        self.d_status = torch.zeros(1, dtype=torch.int32, device=dev)
        self.d_n_out = torch.zeros(1, **i64)
        self.d_stats = torch.zeros(4, **i64)
        self.staging = torch.empty(0, dtype=torch.int32, device=dev)
        self.records = torch.empty(0, dtype=torch.int32, device=dev)
        # two-level counting-sort scatter (pass 2) through a third record buffer
        # (dbg_partition_set.d_scratch + d_work; msp.cu ts_level_a/b): above 8192 fine partitions
        # the one-level scatter pays one returning global atomic per record; with a staging
        # beyond L2 two levels win (r02z1: chr14 8.82 vs 14.14 ms, bumblebee 17.61 vs 19.61 ms),
        # on E. coli's 0.35 GB they lose (0.65 vs 0.51 ms)
        self.scratch = torch.empty(0, dtype=torch.int32, device=dev)
        self.scatter_work = torch.zeros(_lib.dbg_scatter_work_words(self.prm), **i64)
        self.two_level = NP > 8192
        self.two_level_min_bytes = 2 << 30
        self.two_level_words = (4, 8, 16)  # record widths that take it
        self.table = torch.empty(0, dtype=torch.uint8, device=dev)
        self.work = torch.empty(0, dtype=torch.uint8, device=dev)
        self.out = torch.empty(0, dtype=torch.uint8, device=dev)
        self.table_budget_bytes = table_budget_bytes
        self.part_kmers = np.zeros(NP, dtype=np.int64)
        self.part_records = np.zeros(NP, dtype=np.int64)
        self.caps = np.zeros(NP, dtype=np.int64)
        self.tab_host = np.zeros(NP + 1, dtype=np.int64)
        self.batches: list[tuple[int, int]] = []
        self._caps_key = None
        self._batch_key = None
        self._big_key = None
        self._batches_cache: list[tuple[int, int]] = []
        self._dirty = False
        self._tab_key = None
        self._any_global = False
        self._h_sizes = torch.empty(0, dtype=torch.int64)
        self._sizes_ev = torch.cuda.Event() if self.device.type == "cuda" else None
        self._sizes_pending = False
        self.overflowed = False
        self.timer: dict | None = None  # name -> list of (start, end) CUDA events, when set

    # ------------------------------------------------------------------ timing helper
    def _mark(self, name: str, stream):
        if self.timer is None:
            return None
        ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
        ev[0].record(stream)
        self.timer.setdefault(name, []).append(ev)
        return ev

    @staticmethod
    def _done(ev, stream):
        if ev is not None:
            ev[1].record(stream)

    # ------------------------------------------------------------------ a1
    def upload(self, packed: torch.Tensor, offsets, stream=None):
        """H2D of the packed reads and base offsets (row a1)."""
        if not isinstance(offsets, torch.Tensor):
            offsets = torch.from_numpy(np.ascontiguousarray(offsets, dtype=np.uint64).view(np.int64))
        with torch.cuda.stream(stream) if stream is not None else _null():
            d_bases = packed.to(self.device, non_blocking=True)
            d_offsets = offsets.to(self.device, non_blocking=True)
        return d_bases, d_offsets

    # ------------------------------------------------------------------ a2-a4
    def part_set(self, with_records: bool) -> _lib.dbg_partition_set:
        scratch = None
        if with_records and self.use_two_level():
            self.scratch = _grow(self.scratch, self.records.numel(), torch.int32, self.device)
            scratch = self.scratch
        cap = self.staging.numel() // self.rec_words
        return _lib.partition_set(self.d_n_records, self.d_n_kmers, self.d_rec_off, self.d_fill, self.d_staged,
                                  self.staging, cap, self.records if with_records else None, scratch,
                                  work=self.scatter_work if scratch is not None else None)

    def use_two_level(self) -> bool:
        return (self.two_level and self.rec_words in self.two_level_words
                and self.staging.numel() * 4 >= self.two_level_min_bytes)

    def _staging_estimate(self, n_kmers_upper: int, n_reads: int) -> int:
        w = self.k - self.p + 1
        return int(min(n_kmers_upper, 2.6 * n_kmers_upper / (w + 1) + 2 * n_reads)) + 4096

    def msp(self, d_bases: torch.Tensor, d_offsets: torch.Tensor, stream=None):
        """Step 1: pass 1 (minimizers, superkmers, sizes, staging), the sizes copied back
        asynchronously, pass 2 (scatter).  Nothing here waits for the device: sync_sizes() reads
        the sizes when the host needs them, after the device work behind them is enqueued."""
        stream = stream or torch.cuda.current_stream(self.device)
        self.msp_pass1(d_bases, d_offsets, stream)
        # room for every staged record: after an overflow pass 2 and Step 2 do nothing (dbg.h)
        self.records = _grow(self.records, self.staging.numel(), torch.int32, self.device)
        ev = self._mark("msp_scatter", stream)
        _lib.dbg_msp_partition(self.prm, d_bases, d_bases.numel(), d_offsets, d_offsets.numel() - 1,
                               self.part_set(True), stream)
        self._done(ev, stream)

    def msp_pass1(self, d_bases: torch.Tensor, d_offsets: torch.Tensor, stream=None):
        """Pass 1 of Step 1 only (minimizers, superkmers into the staging, per-partition sizes),
        and the asynchronous copy of the sizes (sync_sizes)."""
        stream = stream or torch.cuda.current_stream(self.device)
        n_reads = d_offsets.numel() - 1
        n_words = d_bases.numel()
        if self.staging.numel() == 0:
            self.staging = _grow(self.staging, self._staging_estimate(n_words * 32, n_reads) * self.rec_words,
                                 torch.int32, self.device)
        self.overflowed = False
        ev = self._mark("msp_pass1", stream)
        _lib.dbg_msp_partition(self.prm, d_bases, n_words, d_offsets, n_reads, self.part_set(False), stream)
        self._done(ev, stream)
        if self._h_sizes.numel() != 2 * self.np:
            self._h_sizes = torch.empty(2 * self.np, dtype=torch.int64, pin_memory=True)
        with torch.cuda.stream(stream):
            self._h_sizes[:self.np].copy_(self.d_n_records, non_blocking=True)
            self._h_sizes[self.np:].copy_(self.d_n_kmers, non_blocking=True)
        self._sizes_ev.record(stream)
        self._sizes_pending = True

    def msp_overlapped(self, h_packed: torch.Tensor, h_offsets: torch.Tensor, d_bases: torch.Tensor,
                       d_offsets: torch.Tensor, n_batches: int = 8, stream=None, copy_stream=None):
        """Rows a1-a4 with the upload overlapped (Sec. III-E): the pinned host reads go
        H2D in n_batches read ranges on copy_stream, and pass 1 of range b (dbg_msp_partition_range
        over all partitions, appending) runs on `stream` as soon as its words have arrived, while
        range b+1 is still in flight; then the sizes copy and pass 2 as in msp()."""
        stream = stream or torch.cuda.current_stream(self.device)
        copy_stream = copy_stream or torch.cuda.Stream(self.device)
        n_reads = h_offsets.numel() - 1
        n_words = h_packed.numel()
        if self.staging.numel() == 0:
            self.staging = _grow(self.staging, self._staging_estimate(n_words * 32, n_reads) * self.rec_words,
                                 torch.int32, self.device)
        self.overflowed = False
        offs = h_offsets.numpy()
        bounds = [n_reads * i // n_batches for i in range(n_batches + 1)]
        copy_stream.wait_stream(stream)  # d_bases / d_offsets are free (the previous step is done with them)
        w_done = 0
        ev = self._mark("msp_pass1", stream)
        for i in range(n_batches):
            r0, r1 = bounds[i], bounds[i + 1]
            w1 = min(n_words, int(offs[r1]) // 32 + 2)  # the words of reads < r1 (+ the pad word)
            with torch.cuda.stream(copy_stream):
                if w1 > w_done:
                    d_bases[w_done:w1].copy_(h_packed[w_done:w1], non_blocking=True)
                d_offsets[r0:r1 + 1].copy_(h_offsets[r0:r1 + 1], non_blocking=True)
            w_done = max(w_done, w1)
            arrived = torch.cuda.Event()
            arrived.record(copy_stream)
            stream.wait_event(arrived)
            if r1 > r0 or i == 0:
                _lib.dbg_msp_partition_range(self.prm, d_bases, n_words, d_offsets[r0:], r1 - r0,
                                             self.part_set(False), 0, self.np, i > 0, stream)
        self._done(ev, stream)
        if self._h_sizes.numel() != 2 * self.np:
            self._h_sizes = torch.empty(2 * self.np, dtype=torch.int64, pin_memory=True)
        with torch.cuda.stream(stream):
            self._h_sizes[:self.np].copy_(self.d_n_records, non_blocking=True)
            self._h_sizes[self.np:].copy_(self.d_n_kmers, non_blocking=True)
        self._sizes_ev.record(stream)
        self._sizes_pending = True
        self.records = _grow(self.records, self.staging.numel(), torch.int32, self.device)
        ev = self._mark("msp_scatter", stream)
        _lib.dbg_msp_partition(self.prm, d_bases, n_words, d_offsets, n_reads, self.part_set(True), stream)
        self._done(ev, stream)

    def sync_sizes(self) -> bool:
        """Waits for the pass-1 sizes (part_records, part_kmers).  False after a staging overflow:
        the staging has been grown and the step must be repeated (self.overflowed)."""
        if not self._sizes_pending:
            return not self.overflowed
        self._sizes_ev.synchronize()
        sizes = self._h_sizes.numpy()
        self.part_records = sizes[:self.np].copy()
        self.part_kmers = sizes[self.np:].copy()
        self._sizes_pending = False
        total = int(self.part_records.sum())
        if total > self.staging.numel() // self.rec_words:
            self.staging = _grow(self.staging, total * self.rec_words, torch.int32, self.device, 1.05)
            self.overflowed = True
        return not self.overflowed

    # ------------------------------------------------------------------ a5
    def plan(self, stream=None) -> list[tuple[int, int]]:
        """Sizing (row a5).  Mode "smem": the on-chip plan runs on the device inside
        dbg_build_subgraphs_smem, and the global tables of oversize partitions are planned in
        step2 once the sizes are back -- nothing to do here.  Other modes: tables for all."""
        stream = stream or torch.cuda.current_stream(self.device)
        if self.mode == "smem":
            return self.batches
        if not self.sync_sizes():
            self.batches = []
            return self.batches
        return self._plan_tables(stream)

    def _plan_tables(self, stream) -> list[tuple[int, int]]:
        """Global tables: capacities (host copy of the C sizing functions, cached per size
        vector), batches that fit the table budget, and d_table_offset on the device."""
        key = (self.part_kmers.tobytes(), self.prm.lambda_, self.prm.alpha, self.mode, self.owned)
        if self._caps_key != key:
            nz = np.nonzero(self.part_kmers)[0]
            self.caps = np.zeros(self.np, dtype=np.int64)
            uniq, inv = np.unique(self.part_kmers[nz], return_inverse=True)
            cap_u = np.array([_lib.dbg_table_capacity(self.prm, int(n)) for n in uniq], dtype=np.int64)
            if self.mode == "smem":  # on-chip partitions need no global table
                cap_u[np.array([_lib.dbg_smem_onchip(self.prm, int(n)) > 0 for n in uniq], dtype=bool)] = 0
            self.caps[nz] = cap_u[inv]
            lo, hi = self.owned
            self.caps[:lo] = 0
            self.caps[hi:] = 0
            self._caps_key = key
            self._any_global = bool(self.caps.any())
        if self.mode == "smem" and not self._any_global:
            self.batches = []
            return self.batches
        ev = self._mark("plan", stream)
        # d_fill is idle after the scatter: scratch of the multi-CTA scan
        if self.mode == "smem":
            _lib.dbg_table_plan_split(self.prm, self.d_n_kmers, self.d_tab_off, self.d_fill, stream)
        else:
            _lib.dbg_table_plan(self.prm, self.d_n_kmers, self.d_tab_off, self.d_fill, stream)
        self._done(ev, stream)
        if self._tab_key != self._caps_key:
            self.tab_host = np.zeros(self.np + 1, dtype=np.int64)
            self.tab_host[1:] = np.cumsum(self.caps)
            self._tab_key = self._caps_key
        budget = self.table_budget_bytes
        if budget is None:  # once per builder: cudaMemGetInfo costs milliseconds
            free, _ = torch.cuda.mem_get_info(self.device)
            budget = self.table_budget_bytes = max(int(free * 0.6), 1 << 26)
        max_slots = max(budget // self.slot_bytes, int(self.caps.max(initial=0)))
        bkey = (self._caps_key, max_slots)
        if self._batch_key != bkey:  # greedy batches of consecutive partitions (vectorised)
            batches, b, th = [], self.owned[0], self.tab_host
            while b < self.owned[1]:
                e = int(np.searchsorted(th, th[b] + max_slots, side="right")) - 1
                e = min(max(e, b + 1), self.owned[1])
                if th[e] > th[b]:
                    batches.append((b, e))
                b = e
            self._batches_cache = batches
            self._batch_key = bkey
        batches = self._batches_cache
        self.batches = batches
        need = max((self.tab_host[e] - self.tab_host[b] for b, e in batches), default=0) * self.slot_bytes
        self.table = self._clean_buffer(self.table, int(need), stream)
        return batches

    def _clean_buffer(self, t: torch.Tensor, nbytes: int, stream) -> torch.Tensor:
        """Tables must be all-zero before hashing; extraction leaves them clean again
        (clean-on-extract, hash.cu), so a buffer is zeroed only when (re)allocated or
        after an interrupted build."""
        grown = _grow(t, nbytes, torch.uint8, self.device)
        if grown is not t or self._dirty:
            with torch.cuda.stream(stream):
                grown.zero_()
            self._dirty = False
        return grown

    # ------------------------------------------------------------------ a5-a7
    def reset_output(self, cap: int, stream=None) -> None:
        with torch.cuda.stream(stream or torch.cuda.current_stream(self.device)):
            self.d_n_out.zero_()
            self.d_stats.zero_()
            self.d_status.zero_()
        self.out = _grow(self.out, cap * self.vdtype.itemsize, torch.uint8, self.device)

    def out_cap(self) -> int:
        return self.out.numel() // self.vdtype.itemsize

    def step2(self, stream=None) -> None:
        """Hash + extract of every partition (output appended to self.out)."""
        stream = stream or torch.cuda.current_stream(self.device)
        self._dirty = True  # until every hashed table has been extracted
        self._step2(stream)
        self._dirty = False

    def _step2(self, stream) -> None:
        if self.overflowed:  # pass 2 did nothing; the caller repeats the step
            return
        if self.mode == "smem":
            ev = self._mark("step2_smem", stream)
            wsb = _lib.dbg_smem_workspace_bytes(self.prm)
            self.work = _grow(self.work, wsb, torch.uint8, self.device)
            _lib.dbg_build_subgraphs_smem(self.prm, self.part_set(True), self.owned[0], self.owned[1], self.work,
                                          self.work.numel(), self.out, self.out_cap(), self.d_n_out, self.d_stats,
                                          self.d_status, stream)
            self._done(ev, stream)
            # the sizes are read back while the on-chip kernel runs; then the global tier
            if not self.sync_sizes():
                return
            self._plan_tables(stream)
        for (b, e) in self.batches:
            ev = self._mark("hash_build", stream)
            if self.mode == "smem":  # only the oversize partitions have records to hash here
                pids, prefix = self._big_list(b, e)
                _lib.dbg_hash_build_list(self.prm, self.part_set(True), b, e, pids, prefix, pids.numel(),
                                         self.table, self.d_tab_off, self.d_status, stream)
            else:
                _lib.dbg_hash_build(self.prm, self.part_set(True), b, e, self.table, self.d_tab_off,
                                    self.d_status, stream)
            self._done(ev, stream)
            ev = self._mark("extract", stream)
            _lib.dbg_extract_graph(self.prm, self.table, self.d_tab_off, b, e, self.out, self.out_cap(),
                                   self.d_n_out, self.d_stats, self.d_status, stream)
            self._done(ev, stream)

    def _big_list(self, b: int, e: int):
        """Device list of the partitions in [b, e) with a global table (capacity > 0) and the prefix
        of their 32-record chunk counts (cached per plan)."""
        key = (self._caps_key, b, e)
        if self._big_key != key:
            pids = np.nonzero(self.caps[b:e])[0].astype(np.int64) + b
            chunks = (self.part_records[pids] + 31) // 32
            prefix = np.zeros(len(pids) + 1, dtype=np.int64)
            prefix[1:] = np.cumsum(chunks)
            self._big = (torch.from_numpy(pids.astype(np.int32)).to(self.device),
                         torch.from_numpy(prefix).to(self.device))
            self._big_key = key
        return self._big

    def stats(self, checksum: bool = True, stream=None) -> dict:
        """Totals of the last extraction; the checksum is computed here (dbg_checksum_vertices)."""
        stream = stream or torch.cuda.current_stream(self.device)
        if checksum and self.k <= 63:
            n = min(int(self.d_n_out.item()), self.out_cap())
            with torch.cuda.stream(stream):
                self.d_stats[3].zero_()
            _lib.dbg_checksum_vertices(self.prm, self.out, n, self.d_stats, stream)
        s = self.d_stats.cpu().numpy().view(np.uint64)
        return {f: int(v) for f, v in zip(STATS_FIELDS, s)}

    def vertices(self, sort: bool = True, stream=None) -> np.ndarray:
        """D2H of the compacted records (sorted on the device by dbg_sort_vertices)."""
        stream = stream or torch.cuda.current_stream(self.device)
        n = int(self.d_n_out.item())
        nbytes = n * self.vdtype.itemsize
        src = self.out[:nbytes]
        if self.k > 63:  # dbg_vertex_wide: sorted on the host (dbg_sort_vertices takes K <= 63)
            v = src.cpu().numpy().view(self.vdtype)
            if sort and n:
                k = v["kmer"]
                v = v[np.lexsort((k[:, 3], k[:, 2], k[:, 1], k[:, 0]))]
            return v
        if sort and n:
            dst = torch.empty(nbytes, dtype=torch.uint8, device=self.device)
            wsb = _lib.dbg_sort_workspace_bytes(self.prm, n)
            ws = torch.empty(wsb, dtype=torch.uint8, device=self.device)
            _lib.dbg_sort_vertices(self.prm, src, dst, n, ws, wsb, stream)
            src = dst
        return src.cpu().numpy().view(VERTEX_DTYPE)

    # ------------------------------------------------------------------ whole path
    def build(self, d_bases, d_offsets, stream=None, out_cap: int | None = None,
              want_vertices: bool = True, sort: bool = True) -> GraphResult:
        stream = stream or torch.cuda.current_stream(self.device)
        self.msp(d_bases, d_offsets, stream)
        while not self.sync_sizes():  # staging overflow: grown, repeat Step 1
            self.msp(d_bases, d_offsets, stream)
        self.plan(stream)
        n_kmers = int(self.part_kmers.sum())
        cap = out_cap if out_cap is not None else max(self.out_cap(), n_kmers // 2 + 1024)
        while True:
            self.reset_output(cap, stream)
            self.step2(stream)
            st = _lib.dbg_sync_status(self.d_status, stream)
            if st == _lib.DBG_ENOSPACE and int(self.d_n_out.item()) > self.out_cap():
                cap = int(self.d_n_out.item())
                continue
            if st == _lib.DBG_ETABLEFULL:  # reading O: rebuild at capacity N^i_kmer (tables are clean again)
                if self.prm.lambda_ / (4 * self.prm.alpha) >= 1.0:
                    raise _lib.DbgError("dbg_hash_build", st, "table full at capacity >= N^i_kmer")
                self.prm = _lib.params(self.k, self.p, self.np_out, 2.0, 0.5, self.refine, self.smem_split,
                                       self.fine_p, self.min_count)
                self.plan(stream)
                continue
            if st != _lib.DBG_OK:
                raise _lib.DbgError("dbg_sync_status", st, _lib.dbg_status_string(st))
            break
        verts = self.vertices(sort=sort, stream=stream) if want_vertices else None
        return GraphResult(verts, int(self.d_n_out.item()), self.stats(), n_kmers, self.part_kmers.copy(),
                           self.part_records.copy(), list(self.batches))


GRAPH_HEADER_DTYPE = np.dtype([("magic", "S8"), ("k", "<u4"), ("p", "<u4"), ("num_partitions", "<u4"),
                               ("min_count", "<u4"), ("n_vertices", "<u8"), ("reserved", "<u8", (4,))])
assert GRAPH_HEADER_DTYPE.itemsize == 64


def write_graph(path: str, prm: _lib.dbg_params, vertices: np.ndarray, append: bool = False) -> None:
    """Row f4 graph writer (dbg_write_graph): host records -> graph file (64-B header + records)."""
    v = np.ascontiguousarray(vertices, dtype=VERTEX_DTYPE)
    _lib.dbg_write_graph(path, prm, v if len(v) else None, len(v), append)


def read_graph(path: str) -> tuple[dict, np.ndarray]:
    """Reads a file written by dbg_write_graph: (header fields, records)."""
    raw = np.fromfile(path, dtype=np.uint8)
    h = raw[:64].view(GRAPH_HEADER_DTYPE)[0]
    if bytes(h["magic"]).ljust(8, b"\0") != b"PHDBG\0\0\x01":
        raise ValueError(f"{path}: not a graph file")
    n = int(h["n_vertices"])
    recs = raw[64:64 + n * VERTEX_DTYPE.itemsize].view(VERTEX_DTYPE)
    if len(recs) != n:
        raise ValueError(f"{path}: truncated ({len(recs)} of {n} records)")
    return {f: int(h[f]) for f in ("k", "p", "num_partitions", "min_count", "n_vertices")}, recs.copy()


def auto_refine(n_kmers: int, k: int, p: int, num_partitions: int, lam: float = 2.0, alpha: float = 0.5,
                fill: float = 0.25) -> int:
    """Refinement F so that an average fine partition's table (Property-1 capacity) is about
    `fill` of one CTA's shared-memory table (dbg_smem_table_slots): minimizer skew (PAPER.md
    Fig. 6) makes the largest partitions ~20x the mean, and small partitions are
    packed into groups on chip anyway."""
    prm = _lib.params(k, p, num_partitions, lam, alpha)
    slots = _lib.dbg_smem_table_slots(prm)
    per_part = max(1.0, fill * slots / max(lam / (4 * alpha), 1e-9))
    f = max(1, int(np.ceil(n_kmers / (num_partitions * per_part))))
    return max(1, min(f, MAX_FINE_PARTITIONS // num_partitions))


def auto_fine_p(n_kmers: int, k: int, p: int, lam: float = 2.0, alpha: float = 0.5) -> int:
    """Minimizer length of the device's fine partitioning (dbg_params.fine_p): the smallest P' >= P
    with 4^P' >= 4 (K - P' + 1) N / slots.  A P'-mer occurs about 2G / 4^P' times in a genome of G
    bases and a lexicographically small one is the minimizer of about K - P' + 1 K-mers per
    occurrence, so at coverage N / G its partition holds about 2 (K - P' + 1) N / 4^P' K-mers; the
    rule keeps that below half a CTA table even for the most frequent minimizers."""
    slots = _lib.dbg_smem_table_slots(_lib.params(k, p, 1, lam, alpha))
    ratio = max(lam / (4 * alpha), 1e-9)
    for q in range(p, min(k, 31) + 1):
        if 4.0 ** q >= 4.0 * (k - q + 1) * n_kmers * ratio / slots:
            return q
    return min(k, 31)


def launch_builder(k: int, p: int, num_partitions: int, n_kmers: int, lam: float = 2.0, alpha: float = 0.5,
                   device="cuda", min_count: int = 0, **kw) -> DbgBuilder:
    """The builder in the launch configuration bench.py times: on-chip Step 2 with the automatic
    refinement F (auto_refine) and device minimizer length P' (auto_fine_p) for a workload of
    n_kmers K-mers.  The full-size parity tests use the same function."""
    refine = kw.pop("refine", None) or auto_refine(n_kmers, k, p, num_partitions, lam, alpha)
    fine_p = kw.pop("fine_p", None) or auto_fine_p(n_kmers, k, p, lam, alpha)
    return DbgBuilder(k, p, num_partitions, lam, alpha, device, refine=refine, fine_p=fine_p, min_count=min_count,
                      **kw)


def build_graph(seq: np.ndarray, offsets: np.ndarray, k: int, p: int, num_partitions: int,
                lam: float = 2.0, alpha: float = 0.5, device="cuda", sort: bool = True,
                table_budget_bytes: int | None = None, mode: str = "smem",
                refine: int | str = "auto", smem_split: int = 0,
                fine_p: int | str = "auto", min_count: int = 0) -> GraphResult:
    """ASCII reads -> De Bruijn graph records (the public one-call API)."""
    lens = np.diff(np.asarray(offsets, dtype=np.int64))
    n_kmers = int(np.maximum(lens - k + 1, 0).sum())
    if k > 63:  # row f3: resident tables, partitions on P
        mode, refine, fine_p = "resident", 1 if refine == "auto" else refine, 0
    if refine == "auto":
        refine = auto_refine(n_kmers, k, p, num_partitions, lam, alpha) if mode == "smem" else 1
    if fine_p == "auto":
        fine_p = auto_fine_p(n_kmers, k, p, lam, alpha) if mode == "smem" else 0
    builder = DbgBuilder(k, p, num_partitions, lam, alpha, device, table_budget_bytes, mode, refine,
                         smem_split, fine_p, min_count)
    packed = encode_reads(seq)
    d_bases, d_offsets = builder.upload(packed, offsets)
    return builder.build(d_bases, d_offsets, sort=sort)
