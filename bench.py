#!/usr/bin/env python
"""Benchmark of the ParaHash hot path on B200: K-mers hashed per second (graph build, device-timed).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config chr14] [--impl ours|reference]

One step = one pass of the whole hot path over the configuration's
synthetic reads, resident in HBM: MSP pass 1 -> size readback -> MSP pass 2 (scatter into
partition order) -> on-chip Step 2 (table sizing, hashing, extraction of the vertex records) ->
global-table tier for the partitions too large for one SM.  The default workload is chr14
(BASELINE.json configs[2], the largest configuration that fits one GPU).

``value`` is device-timed (CUDA events on the launching stream, L2 flushed before every step).
``e2e`` is the same workload through the public API with the paper's timing scope (P:L979-987:
"ends at the time all the subgraphs are constructed in main memory", transfers included): H2D of
the packed reads from pinned memory (overlapped with MSP), the device path, and the D2H of every
vertex record into pinned host memory.

N > 1 (``--gpus N``; re-launches itself under torch.distributed.run when started without it):
strong scaling -- the configuration's reads are split into N contiguous ranges, one per rank; each
step is multi.ShardedBuilder.step (local MSP, emission of the records into their owners' buffers
through peer pointers, Step 2 of the owned partitions); times are the max over ranks.

Prints ONE JSON line (rank 0).  DESIGN.md Sec. 7 has the roofline arithmetic.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "K-mers hashed/sec (graph build, device-timed) at 1/2/4/8 B200; HBM roofline %"
UNIT = "kmers/s"
# algorithmic bytes per K-mer occurrence of the hot path -- one 32-B sector read +
# write-back of the vertex's table entry (64 B, the random-access HBM table the north star's
# roofline assumes) + ~4 B of streaming (packed reads, superkmer records written and read back)
ALG_BYTES_PER_KMER = 68
# version tag of the on-chip kernel: profiles/traffic.json (ncu --set full) is quoted only when it
# was captured on this version and workload
KERNEL_VERSION = "smem-v14"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region (B200_PROFILING.md), in-process
    through NVML on a background thread (an nvidia-smi subprocess starting inside the timed region
    stalls the driver and was measured to inflate the step time)."""

    REASONS = {  # nvmlClocksEventReason* bits
        "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
        "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4,
    }

    def __init__(self, index: int, interval: float = 0.02):
        self.index, self.interval = index, interval
        self.rows = []
        self._stop = threading.Event()
        self.ok = False

    def __enter__(self):
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nvml = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
            self.thread = threading.Thread(target=self._run, daemon=True)
            self.thread.start()
            time.sleep(0.2)  # sampler warm before the timed region starts
        except Exception:
            self.ok = False
        self.t0 = time.time()
        return self

    def _run(self):
        nv = self.nvml
        while not self._stop.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                try:
                    rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                except Exception:
                    rs = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                self.rows.append((time.time(), sm, rs))
            except Exception:
                pass
            time.sleep(self.interval)

    def __exit__(self, *a):
        self.t1 = time.time()
        self._stop.set()
        if self.ok:
            self.thread.join(timeout=2)
        return False

    def summary(self):
        rows = [r for r in self.rows if self.t0 <= r[0] <= self.t1] or self.rows[-3:]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        reasons = sorted({n for _, _, rs in rows for n, bit in self.REASONS.items() if rs & bit})
        return {"sm_mhz": statistics.median(r[1] for r in rows), "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(rows), "source": "nvml"}


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _relaunch_under_torchrun(n: int) -> int:
    """`python bench.py --gpus N` without a launcher: start N ranks (one per GPU) ourselves."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    import subprocess

    return subprocess.call(cmd)


def _config_kmers(name: str, scale: float) -> tuple[int, int]:
    """(reads, K-mer occurrences) of a configuration without generating it (fixed read length)."""
    from synth import CONFIGS

    c = CONFIGS[name]
    n = max(int(c["reads"] * scale), 1)
    return n, n * max(c["read_len"] - c["k"] + 1, 0)


def _config_json(rs, args, n_reads_total: int, n_kmers_total: int, extra=None):
    c = {"workload": rs.name, "desc": rs.meta["desc"], "genome_bp": rs.meta["genome"], "reads": n_reads_total,
         "read_len": rs.meta["read_len"], "error_rate": rs.meta["error"], "k": rs.k, "p": rs.p,
         "num_partitions": rs.num_partitions, "lambda": args.lam, "alpha": args.alpha,
         "kmers_per_step": n_kmers_total, "scale": args.scale,
         "l2": "flushed between timed steps (512 MiB write); step working set > L2",
         "parallelism": "one GPU" if args.gpus == 1 else
         f"dp{args.gpus}: reads split by range, fine partitions owned by rank (emission into peer buffers)"}
    if extra:
        c.update(extra)
    return c


# ------------------------------------------------------------------------------- oracle arm
def _oracle_rate(rs, seconds: float, threads: int):
    """Times the oracle (as it stands) on a bounded prefix of the workload's reads."""
    import oracle

    oracle.build()
    n = min(rs.n_reads, 2000)
    for _ in range(2):  # calibrate on a sample that takes ~10 % of the budget (thread start-up amortised)
        t = time.time()
        sub = rs.subset(0, n)
        oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
        dt = max(time.time() - t, 1e-3)
        if dt > 0.1 * seconds or n == rs.n_reads:
            break
        n = int(min(rs.n_reads, n * 0.1 * seconds / dt))
    n2 = int(min(rs.n_reads, max(n, n * seconds / dt)))
    sub = rs.subset(0, n2)
    t = time.time()
    oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
    dt = time.time() - t
    return sub.n_kmers() / dt, sub, dt


def _oracle_single_thread_ecoli(seconds: float = 4.0) -> dict:
    """the oracle's single-thread K-mer rate on the E. coli-shaped config (configs[1])."""
    from synth import make_config

    rs = make_config("ecoli")
    rate, sub, dt = _oracle_rate(rs, seconds, 1)
    return {"value": rate, "unit": UNIT, "cores": 1, "workload": "ecoli",
            "sample": f"first {sub.n_reads} of {rs.n_reads} reads ({sub.n_kmers()} K-mers), {dt:.1f} s"}


def run_reference(args):
    ws, rank, _ = _dist()
    if rank != 0:
        return 0
    from synth import make_config

    rs = make_config(args.config, scale=args.scale, num_partitions=args.np)
    threads = os.cpu_count() or 1
    import oracle

    oracle.build()
    per_step = max(1.0, min(20.0, 120.0 / max(1, args.steps + args.warmup)))
    _, sub, _ = _oracle_rate(rs, per_step, threads)
    for _ in range(args.warmup):
        oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
    times = []
    for _ in range(args.steps):
        t = time.time()
        oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
        times.append(time.time() - t)
    total = sum(times)
    value = sub.n_kmers() * args.steps / total
    sample = f"first {sub.n_reads} of {rs.n_reads} reads ({sub.n_kmers()} K-mers) per step"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "config": _config_json(rs, args, rs.n_reads, rs.n_kmers()),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------- our arm
def _placement(b) -> dict:
    """Share of the K-mers whose partition is grouped on chip, split over several CTA tables, or
    built in the global tables (dbg_smem_onchip)."""
    from paper_conf_icdcs_qiul17_b200 import _lib

    pk = b.part_kmers
    uniq, inv = np.unique(pk, return_inverse=True)
    place = np.array([_lib.dbg_smem_onchip(b.prm, int(n)) for n in uniq])[inv]
    tot = max(int(pk.sum()), 1)
    return {"grouped": float(pk[place == 1].sum()) / tot, "split": float(pk[place >= 2].sum()) / tot,
            "global": float(pk[place == 0].sum()) / tot, "split_ctas": int(place[place >= 2].sum())}


def _profile_facts(workload: str) -> dict:
    """ncu facts of the dominant kernel for this workload (profiles/traffic.json, written from a
    committed `ncu --set full` capture); stale=True when captured on another kernel version."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f).get(workload)
    except Exception:
        tr = None
    if not tr:
        return {"stale": True, "source": None}
    return dict(tr, stale=tr.get("kernel_version") != KERNEL_VERSION)


def run_ours(args):
    """Our arm (module docstring)."""
    import torch

    ws, rank, local = _dist()
    if ws != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={ws}: launch with torchrun --nproc-per-node {args.gpus}")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_icdcs_qiul17_b200 import encode_reads, launch_builder, _lib
    from synth import make_config

    dist = None
    if ws > 1:
        import torch.distributed as dist
        from paper_conf_icdcs_qiul17_b200.multi import ShardedBuilder

        dist.init_process_group("nccl", device_id=dev)
    n_reads_total, n_kmers_total = _config_kmers(args.config, args.scale)
    t = time.time()
    rs = make_config(args.config, scale=args.scale, num_partitions=args.np, shard=(rank, ws) if ws > 1 else None)
    gen_s = time.time() - t
    packed = encode_reads(rs.seq, pin=True)
    offsets = torch.from_numpy(rs.offsets.view(np.int64)).pin_memory()
    stream = torch.cuda.current_stream(dev)
    kw = {}
    if args.refine:
        kw["refine"] = args.refine
    if args.fine_p:
        kw["fine_p"] = args.fine_p
    if ws > 1:
        sb = ShardedBuilder(rs.k, rs.p, rs.num_partitions, n_kmers_total, dev, lam=args.lam, alpha=args.alpha,
                            min_count=args.min_count, **kw)
        src, b = sb.src, sb.dst
    else:
        b = src = launch_builder(rs.k, rs.p, rs.num_partitions, n_kmers_total, args.lam, args.alpha, device=dev,
                                 min_count=args.min_count, **kw)
    if args.scatter == "one":  # A/B: pass 2 in one level
        src.two_level = False
    elif args.scatter == "two":  # A/B: two levels at any size and record width
        src.two_level_words, src.two_level_min_bytes = (4, 8, 16), 0
    d_bases, d_off = src.upload(packed, offsets, stream)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    E = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    # output capacity: distinct vertices <= K-mers; 0.4 x covers the configs' error rates (a build
    # that overflows it reports DBG_ENOSPACE and the invariant check fails loudly)
    out_cap = int(args.out_frac * n_kmers_total / ws) + (1 << 20)

    def step(db, do):
        """One pass of rows a2-a7 on this rank."""
        if ws > 1:
            sb.step(db, do, stream, out_cap)
            return
        b.msp(db, do, stream)
        b.plan(stream)
        b.reset_output(out_cap, stream)
        b.step2(stream)

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier(device_ids=[local])

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    for _ in range(args.warmup):
        step(d_bases, d_off)
    st = _lib.dbg_sync_status(b.d_status, stream)
    assert st == 0, _lib.dbg_status_string(st)

    src.timer = b.timer = {}
    step_ms = []
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            flush.zero_()
            barrier()
            e0, e1 = E(), E()
            e0.record(stream)
            step(d_bases, d_off)
            e1.record(stream)
            barrier()
            step_ms.append(e0.elapsed_time(e1))
    phases = {k: statistics.mean(a.elapsed_time(c) for a, c in v) for k, v in b.timer.items()}
    src.timer = b.timer = None
    st = _lib.dbg_sync_status(b.d_status, stream)
    stats = b.stats()
    n_out = int(b.d_n_out.item())
    L = rs.lengths()
    tot = torch.tensor([rs.n_kmers(), stats["sum_count"], stats["sum_edges"], stats["distinct"],
                        2 * int(np.maximum(L - rs.k, 0).sum()), int(st == 0),
                        int(np.array(stats["checksum"], dtype=np.uint64).view(np.int64))],
                       dtype=torch.int64, device=dev)
    if dist is not None:
        dist.all_reduce(tot)  # int64 sums wrap: the checksum sum stays exact mod 2^64
    total_kmers, sum_count, sum_edges, distinct, want_edges, ok_ranks, checksum = (int(x) for x in tot.cpu())
    checksum &= (1 << 64) - 1
    assert total_kmers == n_kmers_total, (total_kmers, n_kmers_total)
    inv_ok = ok_ranks == ws and sum_count == total_kmers and sum_edges == want_edges

    # e2e through the public API with the paper's timing scope: H2D of the packed reads (pinned;
    # N = 1: overlapped with MSP, DbgBuilder.msp_overlapped), the path, the readback of the vertex
    # count, and the D2H of every vertex record (n_out x 56 B) into pinned host memory
    e2e_ms, h2d_ms, d2h_ms = [], [], []
    db = torch.empty_like(d_bases)
    do = torch.empty_like(d_off)
    vbytes = b.vdtype.itemsize
    host_out = torch.empty(int(n_out * 1.02 + 1024) * vbytes, dtype=torch.uint8, pin_memory=True)
    host_n = torch.empty(1, dtype=torch.int64, pin_memory=True)
    host_stats = torch.empty(4, dtype=torch.int64, pin_memory=True)
    cs = torch.cuda.Stream(dev)
    d2h_bytes = 0
    for _ in range(max(3, min(args.steps, 5))):
        flush.zero_()
        barrier()
        e0, e1, eh, ed = E(), E(), E(), E()
        e0.record(stream)
        if ws == 1:
            b.msp_overlapped(packed, offsets, db, do, 8, stream, cs)
            eh.record(cs)
            b.plan(stream)
            b.reset_output(out_cap, stream)
            b.step2(stream)
        else:
            db.copy_(packed, non_blocking=True)   # H2D of this rank's reads from pinned memory
            do.copy_(offsets, non_blocking=True)
            eh.record(stream)
            step(db, do)
        host_n.copy_(b.d_n_out, non_blocking=True)
        stream.synchronize()                      # the host needs the vertex count to size the copy
        n = int(host_n.item())
        ed.record(stream)
        if n * vbytes > host_out.numel():
            raise RuntimeError(f"{n} vertices exceed the pinned output buffer")
        host_out[:n * vbytes].copy_(b.out[:n * vbytes], non_blocking=True)   # the subgraphs in host memory
        host_stats.copy_(b.d_stats, non_blocking=True)
        e1.record(stream)
        barrier()
        e2e_ms.append(max_over_ranks(e0.elapsed_time(e1)))
        h2d_ms.append(e0.elapsed_time(eh))
        d2h_ms.append(ed.elapsed_time(e1))
        d2h_bytes = n * vbytes + 8 + 32
    h2d = packed.numel() * 8 + offsets.numel() * 8

    ms = max_over_ranks(statistics.mean(step_ms))
    hash_ms = phases.get("step2_smem", 0.0) + phases.get("hash_build", 0.0) + phases.get("extract", 0.0)
    my_kmers = int(b.part_kmers.sum())         # this rank's Step-2 K-mers (its owned partitions)
    n_records = int(b.part_records.sum())
    peak, peak_kind = _peaks()
    alg_bytes = ALG_BYTES_PER_KMER * my_kmers
    achieved = alg_bytes / (hash_ms * 1e-3) / 1e9
    # the r01 byte model (table RMW + records read + vertex records written), kept for comparison
    detailed = my_kmers * 64 + n_records * 4 * b.rec_words + n_out * 56
    prof = _profile_facts(rs.name) if ws == 1 else {"stale": True, "source": None}
    cpu = None
    if not args.no_cpu_baseline and ws == 1:
        threads = os.cpu_count() or 1
        rate, sub, dt = _oracle_rate(rs, args.cpu_seconds, threads)
        cpu = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle",
               "sample": f"first {sub.n_reads} of {rs.n_reads} reads ({sub.n_kmers()} K-mers), {dt:.1f} s",
               "single_thread_ecoli": _oracle_single_thread_ecoli()}
    scan = 1 if b.np <= 16384 else 3  # scan.cuh: one CTA, or tile sums + tile scan + apply
    # Step 1: msp kernel + its scan + the scatter (one kernel, or the two-level one: bucket counts,
    # bucket scan, level A, level B); Step 2: the on-chip plan (8 kernels incl. the greedy group
    # packing) + the on-chip kernel (+ per global-tier batch: its plan scan once, hash_build_list +
    # extract_kernel); multi-GPU adds the exchange plan (scan + 1)
    nb = len(b.batches)
    scatter = 4 if src.use_two_level() else 1
    launches_per_step = 1 + scan + scatter + 9 + 2 * nb + (scan if nb else 0) + (scan + 1 if ws > 1 else 0)
    placement = _placement(b)
    # Fig. 6 / Table II analogue (row f1): the paper's partitions (the vertices' pid, reading V; K-mers
    # = sum of their counts) -- skew and the table size lambda/(4 alpha) N^i_kmer x slot bytes of the
    # largest one (this rank's vertices)
    rec = b.out[:n_out * b.vdtype.itemsize].view(torch.int32).view(n_out, b.vdtype.itemsize // 4)
    paper_parts = np.zeros(rs.num_partitions, dtype=np.float64)
    for c0 in range(0, n_out, 1 << 26):  # chunks: the conversions of 1.8 G rows would not fit
        c = rec[c0:c0 + (1 << 26)]
        paper_parts += torch.bincount(c[:, -1].long(), weights=c[:, -10].double(),
                                      minlength=rs.num_partitions).cpu().numpy()
    del rec, c
    psizes = {"max_over_mean": float(paper_parts.max() / max(paper_parts.mean(), 1e-9)),
              "max_kmers": int(paper_parts.max()), "mean_kmers": float(paper_parts.mean()),
              "max_table_mb": _lib.dbg_table_bytes(b.prm, int(paper_parts.max())) / 1e6,
              "fine_max_over_mean": float(b.part_kmers.max() / max(b.part_kmers.mean(), 1e-9))}
    if rank != 0:
        dist.barrier(device_ids=[local])
        dist.destroy_process_group()
        return 0
    cfg_extra = {"refine": b.refine, "fine_partitions": b.np, "fine_p": b.fine_p or rs.p, "records": n_records,
                 "vertices": n_out,
                 "smem_slots": _lib.dbg_smem_table_slots(b.prm), "kmer_placement": placement,
                 "kernel_version": KERNEL_VERSION, "partition_sizes": psizes}
    if ws > 1:
        cfg_extra["reads_per_rank"] = rs.n_reads
    if args.min_count > 1:
        cfg_extra["min_count"] = args.min_count
    onchip = {k: prof.get(k) for k in ("issue_active_pct", "warp_inst_per_kmer", "dram_bytes_per_kmer",
                                       "l2_hit_pct", "bank_conflict_pct", "source", "kernel_version")}
    onchip["stale"] = prof.get("stale", True)
    line = {
        "metric": METRIC, "value": total_kmers / (ms * 1e-3), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u64", "data": "synthetic (seeded genome + reads, DESIGN.md Sec. 4)",
        "config": _config_json(rs, args, n_reads_total, n_kmers_total, cfg_extra),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak,
                     "traffic": None if prof.get("stale", True) else prof.get("dram_bytes_per_launch"),
                     "kernel": "smem_subgraph_kernel (+ global tier)", "peak_kind": peak_kind,
                     "model": f"random-access HBM table, {ALG_BYTES_PER_KMER} B per K-mer occurrence "
                              "(SURVEY.md 8(d)) x this rank's Step-2 K-mers / Step-2 kernel time; the tables "
                              "are on chip, so measured DRAM traffic is far below the model (onchip)",
                     "alg_bytes_per_launch": alg_bytes, "kernel_ms": hash_ms,
                     "kernel_kmers_per_s": my_kmers / (hash_ms * 1e-3),
                     "detailed_model_frac": detailed / (hash_ms * 1e-3) / 1e9 / peak,
                     "onchip": onchip, "rank": 0},
        "cpu_baseline": cpu,
        "e2e": {"value": total_kmers / (statistics.median(e2e_ms) * 1e-3), "unit": UNIT,
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h_bytes, "ms": statistics.median(e2e_ms),
                "h2d_ms": statistics.median(h2d_ms), "d2h_ms": statistics.median(d2h_ms),
                "all_ms": [round(x, 3) for x in e2e_ms],
                "scope": "H2D of the packed reads + path + D2H of all vertex records to pinned host memory "
                         "(P:L979-987)" + (", H2D overlapped with MSP in 8 read ranges" if ws == 1 else "")},
        "gpu_launches": args.steps * launches_per_step,
        "clocks": clk.summary(),
        "breakdown_ms": phases,
        "stats": {"distinct": distinct, "sum_count": sum_count, "sum_edges": sum_edges,
                  "checksum": checksum},
        "invariants_ok": bool(inv_ok), "gen_s": gen_s,
    }
    print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier(device_ids=[local])
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="chr14")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--np", type=int, default=None, help="override the number of partitions")
    ap.add_argument("--lam", type=float, default=2.0)
    ap.add_argument("--alpha", type=float, default=0.5)
    ap.add_argument("--refine", type=int, default=None, help="fine partitions per partition (default: auto)")
    ap.add_argument("--fine-p", type=int, default=None,
                    help="minimizer length of the fine partitioning (default: auto; dbg_params.fine_p)")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--out-frac", type=float, default=0.4, help="output capacity / K-mers")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--scatter", choices=["auto", "one", "two"], default="auto", help="A/B: pass-2 scatter levels")
    ap.add_argument("--min-count", type=int, default=0, help="row f4 low-count filter (0: the full graph)")
    args = ap.parse_args()
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return _relaunch_under_torchrun(args.gpus)
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
