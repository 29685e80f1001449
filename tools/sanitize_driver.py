#!/usr/bin/env python
"""Small end-to-end runs of every kernel tier for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck), each checked against the oracle:

    compute-sanitizer --tool racecheck python tools/sanitize_driver.py

  * on-chip Step 2 (smem_subgraph_kernel), K = 31 and K = 63, with split and global-tier
    partitions (small refine so some partitions exceed a CTA table);
  * resident tables (hash_build_kernel / extract_kernel);
  * K = 65 / 101 (wide.cu, the empty -> locked -> occupied protocol, with a hot key);
  * the MSP kernels: register-blocked K = 31 (P = 11, 13), generic otherwise (K = 63: 40-bit row);
  * the two-level scatter (more than 8192 fine partitions).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, build_graph, encode_reads  # noqa: E402
from synth import ReadSet, genome, make_reads, random_reads  # noqa: E402


def _check(tag, rs, k, p, np_, two_level_min_bytes=None, **kw):
    if two_level_min_bytes is None:
        res = build_graph(rs.seq, rs.offsets, k, p, np_, **kw)
    else:  # the two-level scatter at a size where the builder would not pick it
        b = DbgBuilder(k, p, np_, **kw)
        b.two_level_min_bytes, b.two_level_words = two_level_min_bytes, (4, 8, 16)
        d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
        res = b.build(d_bases, d_off)
    if k > 63:
        orc = oracle.graph_wide(rs.seq, rs.offsets, k, p, np_)
        ok = len(orc) == len(res.vertices) and np.array_equal(res.vertices["kmer"], orc["key"]) and \
            all(np.array_equal(res.vertices[f], orc[f]) for f in ("count", "out", "in", "pid"))
    else:
        orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=os.cpu_count() or 1)
        g = res.vertices
        ok = len(orc) == len(g) and np.array_equal(g["kmer_lo"], orc["key_lo"]) and \
            np.array_equal(g["kmer_hi"], orc["key_hi"]) and \
            all(np.array_equal(g[f], orc[f]) for f in ("count", "out", "in", "pid"))
    print(f"{tag}: {len(res.vertices)} vertices, parity {'ok' if ok else 'FAILED'}", flush=True)
    return ok


def main():
    g = genome(30_000, seed=31)
    seq, offs = make_reads(g, 1500, 100, 0.01, seed=32)
    rs = ReadSet(seq, offs)
    hot = ReadSet(np.frombuffer(b"ACGT" * 40 * 60, dtype=np.uint8).copy(),
                  np.arange(61, dtype=np.uint64) * np.uint64(160))
    ok = True
    ok &= _check("smem K=31 P=11 (register MSP, split + global tier)", rs, 31, 11, 2, refine=1)
    ok &= _check("smem K=31 P=11 fine_p 13 (reading V)", rs, 31, 11, 8, refine=4, fine_p=13)
    ok &= _check("smem K=63 P=19 (warp MSP, TMA-staged reads)", rs, 63, 19, 4, refine=2)
    ok &= _check("smem K=41 P=17 (warp MSP)", rs, 41, 17, 4, refine=2)
    ok &= _check("smem two-level scatter (10000 fine partitions)", rs, 31, 11, 16, refine=625, two_level_min_bytes=0)
    ok &= _check("smem two-level scatter, 8-word records", rs, 63, 19, 16, refine=625, two_level_min_bytes=0)
    ok &= _check("resident K=31", rs, 31, 11, 4, mode="resident")
    ok &= _check("wide K=65 (locked state)", rs, 65, 21, 3)
    ok &= _check("wide K=101 hot key", hot, 101, 19, 2)
    ok &= _check("ragged reads K=21", random_reads(300, 1, 200, seed=33, n_rate=0.01), 21, 9, 5)
    print("ALL OK" if ok else "PARITY FAILURE", flush=True)
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
