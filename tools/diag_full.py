"""Diagnose table-full status: run smem and resident tiers separately on a scaled config."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from synth import make_config
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, encode_reads, _lib

scale = float(sys.argv[1]) if len(sys.argv) > 1 else 0.1
refine = int(sys.argv[2]) if len(sys.argv) > 2 else 16
rs = make_config("ecoli", scale=scale)
b = DbgBuilder(rs.k, rs.p, rs.num_partitions, refine=refine)
d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
b.msp(d_bases, d_off)
b.plan()
slots = _lib.dbg_smem_table_slots(b.prm)
caps_all = np.array([_lib.dbg_table_capacity(b.prm, int(n)) for n in b.part_kmers])
print("fine", b.np, "slots", slots, "max cap", caps_all.max(), "big", int((caps_all > slots).sum()),
      "mean", caps_all.mean())
b.reset_output(rs.n_kmers())
_lib.dbg_build_subgraphs_smem(b.prm, b.part_set(True), b.d_work, b.out, b.out_cap(), b.d_n_out, b.d_stats,
                              b.d_status, None)
print("after smem:", _lib.dbg_sync_status(b.d_status), "n_out", int(b.d_n_out.item()))
for (lo, hi) in b.batches:
    _lib.dbg_hash_build(b.prm, b.part_set(True), lo, hi, b.table, b.d_tab_off, b.d_status, None)
    print("after hash batch", lo, hi, _lib.dbg_sync_status(b.d_status))
    _lib.dbg_extract_graph(b.prm, b.table, b.d_tab_off, lo, hi, b.out, b.out_cap(), b.d_n_out, b.d_stats,
                           b.d_status, None)
print("final", _lib.dbg_sync_status(b.d_status), b.stats(), rs.n_kmers())

# repeat the bench's step sequence
for it in range(3):
    b.msp(d_bases, d_off)
    b.plan()
    b.reset_output(rs.n_kmers() // 2 + 1024)
    b.step2()
    print("step", it, _lib.dbg_sync_status(b.d_status), b.stats()["checksum"], len(b.batches))
