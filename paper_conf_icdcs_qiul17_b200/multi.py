"""Multi-GPU sharding of the hot path (Sec. III-A, Eq. (2)).

One process per GPU (torch.distributed; NCCL on GPUs, gloo for the CPU tests):

  1. every rank runs pass 1 of Step 1 (MSP, dbg_msp_partition) on its own contiguous read range --
     reads are independent, and the paper splits the input into equal parts (L396-398);
  2. fine partition f is owned by the rank r with bounds[r] <= f < bounds[r+1] (contiguous ranges);
     the per-partition record counts (the NP-length histogram) are gathered and the K-mer counts
     summed -- the only collectives on the data path besides the final statistics reduce;
  3. dbg_exchange_plan turns the gathered histogram into, for this rank, the record slot where its
     records of each partition start in the owner's buffer, and the partition set of the
     partitions it owns;
  4. pass 2 (the scatter) writes every record straight into its owner's partition buffer through
     IPC-mapped peer pointers (NVLink / NVSwitch on a multi-GPU box) -- emission into peer memory,
     no staging copy and no NCCL all-to-all; one host barrier then publishes the buffers;
  5. every rank builds the subgraphs of its own partitions (Step 2; no inter-GPU traffic: identical
     vertices share a partition, L463-467); the statistics are summed at the end (bench.py).

The owners' buffers are shared once per (re)allocation: PeerBuffers all-gathers a generation
number per rank every step and the IPC handles only when one changed.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import _lib
from .graph import DbgBuilder, _grow, launch_builder


def owner_bounds(n_fine: int, world: int) -> np.ndarray:
    """Contiguous fine-partition ranges, one per rank: rank r owns [b[r], b[r+1])."""
    return np.array([r * n_fine // world for r in range(world + 1)], dtype=np.int64)


def _backend(group=None) -> str:
    return dist.get_backend(group)


def gather_rows(t: torch.Tensor, group=None) -> torch.Tensor:
    """[n] tensor of every rank -> [world * n] (rank q's row at q*n), on t's device."""
    world = dist.get_world_size(group)
    if _backend(group) == "nccl":
        out = torch.empty(world * t.numel(), dtype=t.dtype, device=t.device)
        dist.all_gather_into_tensor(out, t.contiguous(), group=group)
        return out
    parts = [torch.empty(t.numel(), dtype=t.dtype) for _ in range(world)]
    dist.all_gather(parts, t.detach().cpu(), group=group)
    return torch.cat(parts).to(t.device)


def all_reduce_sum(t: torch.Tensor, group=None) -> torch.Tensor:
    """In-place sum over ranks (staged through the host on a gloo group)."""
    if _backend(group) == "nccl":
        dist.all_reduce(t, group=group)
        return t
    c = t.detach().cpu()
    dist.all_reduce(c, group=group)
    t.copy_(c)
    return t


def _ipc_export(t: torch.Tensor):
    """CUDA IPC description of t's storage (torch's own IPC plumbing, as torch.multiprocessing)."""
    return t.untyped_storage()._share_cuda_()


def _ipc_open(handle, nbytes: int, dtype=torch.int32):
    """Maps a peer's exported storage into this process; returns (keep-alive object, device pointer).
    The buffer lives on the peer's GPU (handle[0]); this device's kernels write it over NVLink, so
    peer access to that GPU is enabled first (a no-op for a buffer on this GPU)."""
    dev = int(handle[0])
    if torch.cuda.is_available() and dev != torch.cuda.current_device():
        _lib.dbg_enable_peer_access(dev)
    st = torch.UntypedStorage._new_shared_cuda(*handle)
    return st, st.data_ptr()


class PeerBuffers:
    """Device pointers of every rank's record buffer, valid in this process.

    Each step, update(local) all-gathers one generation number per rank (the local generation
    changes when the local buffer is reallocated); only when some rank's generation changed are the
    IPC handles all-gathered and the changed peers re-opened.  export / open_ are injectable for
    the CPU (gloo) tests of this protocol."""

    def __init__(self, group=None, export=_ipc_export, open_=_ipc_open):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.export, self.open_ = export, open_
        self.gen = 0
        self._key = None
        self.gens = [-1] * self.world
        self.ptrs = [0] * self.world
        self._keep = [None] * self.world
        self.reopened = 0  # handles opened so far (tests)

    def update(self, local: torch.Tensor) -> list[int]:
        key = (local.data_ptr(), local.numel())
        if key != self._key:
            self._key = key
            self.gen += 1
        g = torch.tensor([self.gen], dtype=torch.int64)
        gens = [torch.zeros(1, dtype=torch.int64) for _ in range(self.world)]
        dist.all_gather(gens, g, group=self._cpu_group())
        gens = [int(x) for x in gens]
        if gens != self.gens:
            mine = self.export(local) if local.numel() else None
            handles = [None] * self.world
            dist.all_gather_object(handles, (self.gen, mine), group=self._cpu_group())
            for r, (gr, h) in enumerate(handles):
                if r == self.rank:
                    self.ptrs[r] = local.data_ptr()
                elif gr != self.gens[r]:
                    self._keep[r] = None
                    if h is None:
                        self.ptrs[r] = 0
                    else:
                        self._keep[r], self.ptrs[r] = self.open_(h, 0)
                        self.reopened += 1
            self.gens = gens
        self.ptrs[self.rank] = local.data_ptr()
        return list(self.ptrs)

    def _cpu_group(self):
        """Control-plane collectives (generation numbers, handles) on a gloo group: host objects."""
        if _backend(self.group) == "gloo":
            return self.group
        if not hasattr(self, "_gloo"):
            self._gloo = dist.new_group(backend="gloo")
        return self._gloo


class ShardedBuilder:
    """Row e: one rank's share of the sharded hot path.  `src` runs Step 1 on this rank's reads and
    emits every record into its owner's buffer; `dst` holds the owned partitions (its records buffer
    is the one peers write into) and runs Step 2 on them.  Every rank must use the same workload
    size (n_kmers_total) so that the fine partitioning (refine, fine_p) is the same everywhere."""

    def __init__(self, k: int, p: int, num_partitions: int, n_kmers_total: int, device, group=None,
                 lam: float = 2.0, alpha: float = 0.5, min_count: int = 0, **kw):
        self.group = group
        self.world, self.rank = dist.get_world_size(group), dist.get_rank(group)
        self.device = torch.device(device)
        self.src = launch_builder(k, p, num_partitions, n_kmers_total, lam, alpha, device=self.device,
                                  min_count=min_count, **kw)
        s = self.src
        self.dst = DbgBuilder(k, p, num_partitions, lam, alpha, self.device, refine=s.refine, fine_p=s.fine_p,
                              min_count=min_count, smem_split=s.smem_split)
        NP = s.np
        self.np = NP
        self.bounds = owner_bounds(NP, self.world)
        self.owned = (int(self.bounds[self.rank]), int(self.bounds[self.rank + 1]))
        self.dst.owned = self.owned
        dev = self.device
        self.d_bounds = torch.from_numpy(self.bounds.astype(np.int32)).to(dev)
        self.d_kmers = torch.zeros(NP, dtype=torch.int64, device=dev)
        self.d_dest = torch.zeros(NP + 1, dtype=torch.int64, device=dev)
        self.d_prefix = torch.zeros(NP + 1, dtype=torch.int64, device=dev)
        self.d_ptrs = torch.zeros(self.world, dtype=torch.int64, device=dev)
        lo, hi = self.owned
        self._h_sizes = torch.empty(2 * (hi - lo) + 1, dtype=torch.int64, pin_memory=dev.type == "cuda")
        self._h_ptrs = torch.empty(self.world, dtype=torch.int64, pin_memory=dev.type == "cuda")
        self.peers = PeerBuffers(group)
        self.n_recv = 0
        self.timer = None

    def _barrier(self):
        if _backend(self.group) == "nccl":
            dist.barrier(group=self.group, device_ids=[self.device.index])
        else:
            dist.barrier(group=self.group)

    def step(self, d_bases: torch.Tensor, d_offsets: torch.Tensor, stream, out_cap: int) -> None:
        s, d = self.src, self.dst
        lo, hi = self.owned
        NP = self.np
        # Step 1, pass 1 on the local reads (repeated after a staging overflow)
        s.msp_pass1(d_bases, d_offsets, stream)
        self.pass1_runs = 1
        while not s.sync_sizes():
            s.msp_pass1(d_bases, d_offsets, stream)
            self.pass1_runs += 1
        # the NP-length histogram and the K-mer sums (the only data-path collectives)
        with torch.cuda.stream(stream):
            counts = gather_rows(s.d_n_records, self.group)
            self.d_kmers.copy_(s.d_n_kmers)
            all_reduce_sum(self.d_kmers, self.group)
        # where this rank's records go, and the partition set of the owned partitions (dst's arrays);
        # s.d_fill is idle until pass 2 zeroes it: scratch of the scan
        _lib.dbg_exchange_plan(s.prm, counts, self.d_kmers, self.world, self.rank, self.d_bounds, self.d_dest,
                               d.d_n_records, d.d_n_kmers, d.d_rec_off, self.d_prefix, s.d_fill, stream)
        with torch.cuda.stream(stream):
            m = hi - lo
            self._h_sizes[:m].copy_(d.d_n_records[lo:hi], non_blocking=True)
            self._h_sizes[m:2 * m].copy_(d.d_n_kmers[lo:hi], non_blocking=True)
            self._h_sizes[2 * m:].copy_(d.d_rec_off[NP:], non_blocking=True)
        stream.synchronize()
        hs = self._h_sizes.numpy()
        d.part_records = np.zeros(NP, dtype=np.int64)
        d.part_kmers = np.zeros(NP, dtype=np.int64)
        d.part_records[lo:hi] = hs[:m]
        d.part_kmers[lo:hi] = hs[m:2 * m]
        self.n_recv = int(hs[2 * m])
        R = s.rec_words
        if d.records.numel() < self.n_recv * R:
            d.records = _grow(d.records, self.n_recv * R, torch.int32, self.device, 1.1)
        ptrs = self.peers.update(d.records)
        self._h_ptrs.copy_(torch.tensor(ptrs, dtype=torch.int64))
        with torch.cuda.stream(stream):
            self.d_ptrs.copy_(self._h_ptrs, non_blocking=True)
        # pass 2: every staged record into its owner's buffer (peer memory), partition order
        scratch = None
        if s.use_two_level():  # two-level scatter (msp.cu): level 1 locally, level 2 into the owners' buffers
            s.scratch = _grow(s.scratch, s.staging.numel(), torch.int32, self.device)
            scratch = s.scratch
        part = _lib.partition_set(s.d_n_records, s.d_n_kmers, self.d_dest, s.d_fill, s.d_staged, s.staging,
                                  s.staging.numel() // R, d.records, scratch, self.d_ptrs, self.d_bounds,
                                  self.world, work=s.scatter_work if scratch is not None else None)
        ev = s._mark("msp_scatter", stream)
        _lib.dbg_msp_partition(s.prm, d_bases, d_bases.numel(), d_offsets, d_offsets.numel() - 1, part, stream)
        s._done(ev, stream)
        stream.synchronize()
        self._barrier()          # every peer's records have landed in this rank's buffer
        # Step 2 on the owned partitions
        d._sizes_pending = False
        d.overflowed = False
        with torch.cuda.stream(stream):
            d.d_staged.zero_()
        d.plan(stream)
        d.reset_output(out_cap, stream)
        d.step2(stream)
