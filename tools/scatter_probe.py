#!/usr/bin/env python
"""Microbenchmark of the scatter's ingredients on B200 (torch kernels, timing only): where do the
14 ms of chr14's pass 2 go?  n 16-byte records, NP partitions (chr14: 295 M, 1.58 M).

  copy      sequential read + write of the records (the bandwidth floor)
  perm      records written to random positions of a uniform permutation
  frontier  records written to rec_off[pid] + rank (the scatter's pattern: one advancing
            cursor per partition, partitions chosen uniformly)
  sorted    the same destinations, but the writes issued in destination order (coalesced)
  atom      index_add_ of 1 into NP 64-bit counters (atomics without return)
"""
import sys
import time

import torch


def t(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


def main():
    n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 295_000_000
    NP = int(float(sys.argv[2])) if len(sys.argv) > 2 else 1_579_008
    dev = torch.device("cuda")
    g = torch.Generator(device=dev).manual_seed(1)
    rec = torch.randint(0, 2 ** 31, (n, 4), dtype=torch.int32, device=dev, generator=g)
    out = torch.empty_like(rec)
    pid = torch.randint(0, NP, (n,), dtype=torch.int64, device=dev, generator=g)
    # the scatter's destinations: rec_off[pid] + rank of the record among its partition's records
    order = torch.argsort(pid, stable=True)
    dest = torch.empty(n, dtype=torch.int64, device=dev)
    dest[order] = torch.arange(n, device=dev)
    perm = torch.randperm(n, device=dev, generator=g)
    res = {"n": n, "NP": NP}
    res["copy_ms"] = t(lambda: out.copy_(rec))
    res["perm_ms"] = t(lambda: out.index_copy_(0, perm, rec))
    res["frontier_ms"] = t(lambda: out.index_copy_(0, dest, rec))
    sdest = dest[order]
    srec = rec[order]
    res["sorted_ms"] = t(lambda: out.index_copy_(0, sdest, srec))
    cnt = torch.zeros(NP, dtype=torch.int64, device=dev)
    ones = torch.ones(n, dtype=torch.int64, device=dev)
    res["atom_ms"] = t(lambda: cnt.index_add_(0, pid, ones))
    print(res, flush=True)


if __name__ == "__main__":
    main()
