"""Full-size GPU parity at BASELINE.json's configs, in the launch configuration bench.py times.

* E. coli (configs[1]): the WHOLE graph against the full oracle, record by record (54 M vertices).
* chr14 (configs[2]) and bumblebee (configs[3], K = 63 two-word keys): the GPU output restricted
  to 16 seeded paper partitions against oracle.graph(pids=...) over ALL reads -- unbiased (the
  partitions are drawn before the GPU runs, and a vertex the GPU never emitted is still in the
  oracle's output) -- plus, over every record: I1 (sum of counts = sum(L-K+1)), I2 (sum of edges
  = 2 sum(L-K)), unique keys, the device checksum equal to the oracle's checksum of the same
  records, and I4 placement on a sample (pid = fmix64(canonical P-minimizer) mod NP, by the
  oracle's brute-force minimizer).

Bit-exact (integer work).  PAPER.md Def. 3 (L232-237) is the graph; Sec. III-B L463-467 why a
vertex lives in exactly one partition.
"""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import VERTEX_DTYPE, build_graph, encode_reads, launch_builder, _lib  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import build as _build  # noqa: E402
from synth import make_config  # noqa: E402

from gpu_helpers import compare_vertices  # noqa: E402

NT = os.cpu_count() or 1
OUT_FRAC = 0.4          # bench.py --out-frac default
REC_I32 = VERTEX_DTYPE.itemsize // 4
_build.build()


def _free():
    import gc

    gc.collect()
    torch.cuda.empty_cache()


def test_ecoli_full_graph_equals_oracle():
    """configs[1] at full size: every vertex record equals the oracle's (no sampling)."""
    rs = make_config("ecoli")
    k, p, np_ = rs.k, rs.p, rs.num_partitions
    b = launch_builder(k, p, np_, rs.n_kmers(), device="cuda")
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    res = b.build(d_bases, d_off, out_cap=int(OUT_FRAC * rs.n_kmers()) + 1024)
    del b, d_bases, d_off
    _free()
    orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT)
    compare_vertices(res.vertices, orc)
    st = res.stats
    assert st["distinct"] == len(orc)
    assert st["sum_count"] == int(orc["count"].sum()) == rs.n_kmers()
    assert st["sum_edges"] == int(orc["out"].sum() + orc["in"].sum())
    assert st["checksum"] == oracle.checksum(orc)


def _code_string(hi: int, lo: int, k: int) -> str:
    code = (hi << 64) | lo
    return "".join("ACGT"[(code >> (2 * (k - 1 - t))) & 3] for t in range(k))


@pytest.mark.parametrize("name", ["chr14", "bumblebee"])
def test_full_size_sampled_partitions_equal_oracle(name):
    rs = make_config(name)
    k, p, np_ = rs.k, rs.p, rs.num_partitions
    n_kmers = rs.n_kmers()
    rng = np.random.default_rng(20261017 + np_ + k)
    pids = np.sort(rng.choice(np_, size=16, replace=False))   # drawn before the GPU runs

    b = launch_builder(k, p, np_, n_kmers, device="cuda")
    d_bases, d_off = b.upload(encode_reads(rs.seq, pin=True), rs.offsets)
    res = b.build(d_bases, d_off, out_cap=int(OUT_FRAC * n_kmers) + 1024, want_vertices=False)
    # free Step 1's buffers before the checks
    b.staging = b.records = b.work = b.table = torch.empty(0, dtype=torch.int32, device="cuda")
    del d_bases, d_off
    _free()
    n = res.n_vertices
    st = res.stats
    L = rs.lengths()
    assert st["sum_count"] == int(np.maximum(L - k + 1, 0).sum())                        # I1
    assert st["sum_edges"] == 2 * int(np.maximum(L - k, 0).sum())                        # I2
    assert st["distinct"] == n
    rec = b.out[:n * VERTEX_DTYPE.itemsize].view(torch.int32).view(n, REC_I32)
    pid = rec[:, REC_I32 - 1]
    assert int(pid.min()) >= 0 and int(pid.max()) < np_

    # sampled partitions, bit-exact against the oracle over all reads
    m = torch.isin(pid, torch.from_numpy(pids.astype(np.int32)).cuda())
    sel = rec[m].contiguous().cpu().numpy().view(VERTEX_DTYPE).reshape(-1)
    sel = sel[np.lexsort((sel["kmer_lo"], sel["kmer_hi"]))]
    orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT, pids=pids.tolist())
    assert len(orc) > 0
    compare_vertices(sel, orc)

    # every record: unique keys (checked per block of 32 paper partitions: a key's partition is a
    # function of the key, I4) and the checksum of the records by the oracle's code
    for a in range(0, np_, 32):
        mm = (pid >= a) & (pid < a + 32)
        keys = rec[mm][:, :4].contiguous().view(torch.int64)
        assert torch.unique(keys, dim=0).shape[0] == keys.shape[0], f"duplicate vertex in partitions {a}..{a + 31}"
        del keys, mm
    cs = 0
    step = 50_000_000
    for c0 in range(0, n, step):
        cs += oracle.checksum(rec[c0:c0 + step].contiguous().cpu().numpy().view(VERTEX_DTYPE).reshape(-1))
    assert cs % (1 << 64) == st["checksum"]

    # I4 placement on 2,000 records: pid = fmix64(canonical P-minimizer of the vertex) mod NP
    idx = torch.from_numpy(np.sort(rng.choice(n, size=2000, replace=False))).cuda()
    smp = rec[idx].contiguous().cpu().numpy().view(VERTEX_DTYPE).reshape(-1)
    for r in smp:
        s = _code_string(int(r["kmer_hi"]), int(r["kmer_lo"]), k)
        assert oracle.fmix64(oracle.kmer_minimizer(s, p)) % np_ == int(r["pid"]), s
    del rec, pid, b
    _free()
