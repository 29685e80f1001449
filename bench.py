#!/usr/bin/env python
"""Benchmark of the ParaHash hot path on B200: K-mers hashed per second (graph build, device-timed).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config ecoli] [--impl ours|reference]

One step = one pass of the whole hot path over the synthetic read set
of the chosen configuration: MSP count pass -> size readback -> MSP emit pass -> table plan ->
table zero-fill -> hash build.  Extraction (a7) is timed separately (``extract_ms``) and is part of
the ``e2e`` number, which also includes the H2D of the packed reads and the D2H of the stats.

Prints ONE JSON line (rank 0).  See DESIGN.md Sec. 7 for the roofline arithmetic.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "K-mers hashed/sec (graph build, device-timed) at 1/2/4/8 B200; HBM roofline %"
UNIT = "kmers/s"
# version tag of the on-chip kernel: profiles/traffic.json (ncu --set full) is quoted only when it
# was captured on this version
KERNEL_VERSION = "smem-v11"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


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


def _workload(args):
    from synth import make_config

    t = time.time()
    rs = make_config(args.config, scale=args.scale, num_partitions=args.np)
    if args.p is not None:
        rs.p = args.p
    return rs, time.time() - t


def _config_json(rs, args, extra=None):
    c = {"workload": rs.name, "genome_bp": rs.meta["genome"], "reads": rs.n_reads,
         "read_len": rs.meta["read_len"], "error_rate": rs.meta["error"], "k": rs.k, "p": rs.p,
         "num_partitions": rs.num_partitions, "lambda": args.lam, "alpha": args.alpha,
         "kmers_per_step": rs.n_kmers(), "scale": args.scale,
         "l2": "flushed between timed steps (512 MiB write); step working set > L2",
         "parallelism": f"partitions sharded over {args.gpus} GPU(s)"}
    if extra:
        c.update(extra)
    return c


# ------------------------------------------------------------------------------- oracle arm
def _oracle_rate(rs, seconds: float, threads: int):
    """Times the oracle (as it stands) on a bounded prefix of the workload's reads."""
    import oracle

    oracle.build()
    n = min(rs.n_reads, 2000)
    t = time.time()
    sub = rs.subset(0, n)
    oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
    dt = max(time.time() - t, 1e-3)
    rate = sub.n_kmers() / dt
    n2 = int(min(rs.n_reads, max(n, n * seconds / dt)))
    sub = rs.subset(0, n2)
    t = time.time()
    oracle.graph(sub.seq, sub.offsets, rs.k, rs.p, rs.num_partitions, n_threads=threads)
    dt = time.time() - t
    return sub.n_kmers() / dt, sub, dt


def run_reference(args):
    ws, rank, _ = _dist()
    if rank != 0:
        return 0
    rs, _ = _workload(args)
    threads = os.cpu_count() or 1
    import oracle

    oracle.build()
    per_step = max(2.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
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
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "config": _config_json(rs, args),
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


def run_ours(args):
    """Our arm.  N = 1: the whole path on one GPU.  N > 1 (torchrun): one process per GPU, weak
    scaling -- every rank owns a read set of the configuration's size (same genome, its own reads);
    a step is multi.distributed_step (local MSP, one record exchange to the partition owners,
    owned-partition Step 2, NCCL reduces), timed on each rank's stream, max over ranks."""
    import torch

    ws, rank, local = _dist()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_icdcs_qiul17_b200 import DbgBuilder, auto_fine_p, auto_refine, encode_reads, _lib

    dist = None
    if ws > 1:
        import torch.distributed as dist
        from paper_conf_icdcs_qiul17_b200 import multi

        dist.init_process_group("nccl", device_id=dev)
    t = time.time()
    from synth import make_config

    rs = make_config(args.config, scale=args.scale, num_partitions=args.np, read_seed_offset=7919 * rank)
    if args.p is not None:
        rs.p = args.p
    gen_s = time.time() - t
    packed = encode_reads(rs.seq, pin=True)
    offsets = torch.from_numpy(rs.offsets.view(np.int64)).pin_memory()
    n_kmers = rs.n_kmers()
    stream = torch.cuda.current_stream(dev)
    refine = args.refine
    if refine is None:
        refine = auto_refine(n_kmers, rs.k, rs.p, rs.num_partitions, args.lam, args.alpha) if args.mode == "smem" else 1
    fine_p = args.fine_p
    if fine_p is None:
        fine_p = auto_fine_p(n_kmers, rs.k, rs.p, args.lam, args.alpha) if args.mode == "smem" else 0
    if ws > 1 and args.mode != "smem":
        raise SystemExit("multi-GPU runs use mode smem")
    b = DbgBuilder(rs.k, rs.p, rs.num_partitions, args.lam, args.alpha, dev, args.table_budget, args.mode,
                   args.group_slots, refine, args.smem_split, fine_p, args.min_count)
    d_bases, d_off = b.upload(packed, offsets, stream)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    E = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    # output capacity: distinct vertices <= K-mers; 0.4 x covers the configs' error rates (a build
    # that overflows it reports DBG_ENOSPACE and the invariant check fails loudly)
    out_cap = int(args.out_frac * n_kmers) + 1024

    host_ms = {"msp": [], "plan": [], "reset": [], "step2": []}

    def step(db, do):
        """One pass of rows a2-a7 (MSP, sizing, on-chip / global Step 2) on this rank."""
        if ws > 1:
            multi.distributed_step(b, db, do, stream, out_cap)
            return
        t = time.perf_counter()
        b.msp(db, do, stream)
        t1 = time.perf_counter()
        b.plan(stream)
        t2 = time.perf_counter()
        b.reset_output(out_cap, stream)
        t3 = time.perf_counter()
        b.step2(stream)
        t4 = time.perf_counter()
        for k, v in zip(("msp", "plan", "reset", "step2"), (t1 - t, t2 - t1, t3 - t2, t4 - t3)):
            host_ms[k].append(1e3 * v)

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()

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

    b.timer = {}
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
    b.timer = None
    st = _lib.dbg_sync_status(b.d_status, stream)
    stats = b.stats()
    L = rs.lengths()
    tot = torch.tensor([n_kmers, stats["sum_count"], stats["sum_edges"], stats["distinct"],
                        2 * int(np.maximum(L - rs.k, 0).sum()), int(st == 0)], dtype=torch.int64, device=dev)
    if dist is not None:
        dist.all_reduce(tot)
    total_kmers, sum_count, sum_edges, distinct, want_edges, ok_ranks = (int(x) for x in tot.cpu())
    inv_ok = ok_ranks == ws and sum_count == total_kmers and sum_edges == want_edges

    # e2e through the public API: H2D of the packed reads (pinned) + path + D2H of the stats.
    # N = 1: DbgBuilder.msp_overlapped uploads the reads in 8 read ranges on a copy stream and
    # starts MSP on each range as soon as it has arrived (the f2 overlap of transfer and compute).
    e2e_ms, h2d_ms = [], []
    db = torch.empty_like(d_bases)
    do = torch.empty_like(d_off)
    host_stats = torch.empty(4, dtype=torch.int64, pin_memory=True)
    cs = torch.cuda.Stream(dev)
    for _ in range(max(3, min(args.steps, 5))):
        flush.zero_()
        barrier()
        e0, e1, eh = E(), E(), E()
        e0.record(stream)
        if ws == 1:
            b.msp_overlapped(packed, offsets, db, do, 8, stream, cs)
            eh.record(cs)
            b.plan(stream)
            b.reset_output(out_cap, stream)
            b.step2(stream)
        else:
            db.copy_(packed, non_blocking=True)   # H2D of the step's input from pinned memory
            do.copy_(offsets, non_blocking=True)
            eh.record(stream)
            step(db, do)
        host_stats.copy_(b.d_stats, non_blocking=True)  # D2H of the step's result
        e1.record(stream)
        barrier()
        e2e_ms.append(max_over_ranks(e0.elapsed_time(e1)))
        h2d_ms.append(e0.elapsed_time(eh))
    h2d = packed.numel() * 8 + offsets.numel() * 8
    d2h = 32

    ms = max_over_ranks(statistics.mean(step_ms))
    key = {"fused": "step2", "resident": "hash_build", "smem": "step2_smem"}[args.mode]
    hash_ms = phases.get(key, float("nan")) + (phases.get("hash_build", 0.0) + phases.get("extract", 0.0)
                                               if args.mode == "smem" else 0.0)
    # this rank's Step-2 work (after the exchange: the K-mers of its own partitions)
    my_kmers = int(b.part_kmers.sum())
    n_records = int(b.part_records.sum())
    # one 32-B sector read + write-back per K-mer occurrence (the paper's
    # random-access table RMW) + the records read + the vertex records written
    alg_bytes = my_kmers * 64 + n_records * 4 * b.rec_words + stats["distinct"] * 56
    peak, peak_kind = _peaks()
    achieved = alg_bytes / (hash_ms * 1e-3) / 1e9
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f).get(rs.name, {})
            if ws == 1 and tr.get("kernel_version") == KERNEL_VERSION:
                traffic = tr.get("dram_bytes_per_launch")
    except Exception:
        pass
    cpu = None
    if not args.no_cpu_baseline and ws == 1:
        threads = os.cpu_count() or 1
        rate, sub, dt = _oracle_rate(rs, args.cpu_seconds, threads)
        cpu = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle",
               "sample": f"first {sub.n_reads} of {rs.n_reads} reads ({sub.n_kmers()} K-mers), {dt:.1f} s"}
    scan = 1 if b.np <= 16384 else 3  # scan.cuh: one CTA, or tile sums + tile scan + apply
    # msp_block_kernel + its scan + scatter_kernel (+ bucket_scatter_kernel when two-level), then
    # Step 2: the on-chip plan (8 kernels incl. the greedy group packing) + the on-chip kernel
    # (+ per global-tier batch: its plan scan once, hash_build_list + extract_kernel)
    nb = len(b.batches)
    launches_per_step = 2 + scan + int(b.two_level) + {"fused": scan + 2, "resident": scan + 2 * nb,
                                                       "smem": 9 + 2 * nb + (scan if nb else 0)}[args.mode]
    placement = _placement(b) if args.mode == "smem" else None
    # Fig. 6 / Table II analogue (row f1): the paper's partitions (fine pid mod NP) -- skew and the
    # table size lambda/(4 alpha) N^i_kmer x slot bytes of the largest one
    paper_parts = np.bincount(np.arange(b.np) % rs.num_partitions, weights=b.part_kmers,
                              minlength=rs.num_partitions)
    psizes = {"max_over_mean": float(paper_parts.max() / max(paper_parts.mean(), 1e-9)),
              "max_kmers": int(paper_parts.max()), "mean_kmers": float(paper_parts.mean()),
              "max_table_mb": _lib.dbg_table_capacity(b.prm, int(paper_parts.max())) * b.slot_bytes / 1e6,
              "fine_max_over_mean": float(b.part_kmers.max() / max(b.part_kmers.mean(), 1e-9))}
    if rank != 0:
        dist.barrier()
        dist.destroy_process_group()
        return 0
    cfg_extra = {"mode": args.mode, "batches": len(b.batches), "group_slots": args.group_slots, "refine": refine,
                 "fine_partitions": b.np, "smem_split": args.smem_split, "fine_p": fine_p or rs.p,
                 "smem_slots": _lib.dbg_smem_table_slots(b.prm), "kmer_placement": placement,
                 "kernel_version": KERNEL_VERSION, "partition_sizes": psizes}
    if ws > 1:
        cfg_extra.update({"reads_per_rank": rs.n_reads, "kmers_total": total_kmers,
                          "parallelism": f"reads sharded; fine partitions owned by rank (one all_to_all of "
                                         f"records over NCCL); {ws} GPUs"})
    if args.min_count > 1:
        cfg_extra["min_count"] = args.min_count
    line = {
        "metric": METRIC, "value": total_kmers / (ms * 1e-3), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": _config_json(rs, args, cfg_extra),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "kernel": {"fused": "subgraph_kernel", "resident": "hash_build_kernel",
                                "smem": "smem_subgraph_kernel"}[args.mode],
                     "peak_kind": peak_kind, "alg_bytes_per_launch": alg_bytes,
                     "kernel_ms": hash_ms, "kernel_kmers_per_s": my_kmers / (hash_ms * 1e-3),
                     "rank": 0},
        "cpu_baseline": cpu,
        "e2e": {"value": total_kmers / (statistics.median(e2e_ms) * 1e-3), "unit": UNIT,
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "ms": statistics.median(e2e_ms),
                "h2d_ms": statistics.median(h2d_ms), "all_ms": [round(x, 3) for x in e2e_ms],
                "h2d_overlap": "8 read ranges H2D on a copy stream, MSP per range as it arrives" if ws == 1 else None},
        "gpu_launches": args.steps * launches_per_step,
        "clocks": clk.summary(),
        "breakdown_ms": phases,
        "host_ms": {k: round(statistics.mean(v[-args.steps:]), 3) for k, v in host_ms.items() if v},
        "stats": {"distinct": distinct, "sum_count": sum_count, "sum_edges": sum_edges,
                  "checksum": stats["checksum"] if ws == 1 else None},
        "invariants_ok": bool(inv_ok), "gen_s": gen_s,
    }
    print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="ecoli")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--np", type=int, default=None, help="override the number of partitions")
    ap.add_argument("--p", type=int, default=None, help="override the minimizer length P")
    ap.add_argument("--lam", type=float, default=2.0)
    ap.add_argument("--alpha", type=float, default=0.5)
    ap.add_argument("--table-budget", type=int, default=None)
    ap.add_argument("--mode", choices=["smem", "fused", "resident"], default="smem")
    ap.add_argument("--refine", type=int, default=None, help="fine partitions per partition (default: auto)")
    ap.add_argument("--group-slots", type=int, default=1 << 19)
    ap.add_argument("--fine-p", type=int, default=None,
                    help="minimizer length of the fine partitioning (default: auto; dbg_params.fine_p)")
    ap.add_argument("--smem-split", type=int, default=0,
                    help="most CTAs an oversize partition is split over on chip (0: default, 1: none)")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--out-frac", type=float, default=0.4, help="output capacity / K-mers")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--min-count", type=int, default=0, help="row f4 low-count filter (0: the full graph)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
