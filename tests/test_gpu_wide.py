"""Row f3 (Sec. III-C3): K-mers longer than 63 bases -- four-word keys inserted
with the paper's empty -> locked -> occupied state protocol in the resident tables -- give the
oracle's graph bit-exact (oracle.graph_wide, string-keyed)."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, build as _build, build_graph, encode_reads  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import _lib  # noqa: E402
from synth import ReadSet, genome, make_reads, random_reads  # noqa: E402

_build.build()


def _compare(res, orc):
    v = res.vertices
    assert len(v) == len(orc), (len(v), len(orc))
    assert np.array_equal(v["kmer"], orc["key"])
    for f in ("count", "out", "in", "pid"):
        assert np.array_equal(v[f], orc[f]), f


@pytest.mark.parametrize("k,p,np_,seed", [(65, 21, 7, 1), (71, 13, 3, 2), (99, 31, 16, 3), (127, 19, 5, 4),
                                           (65, 1, 1, 5), (101, 27, 64, 6)])
def test_wide_random_reads(k, p, np_, seed):
    rs = random_reads(400, 1, 2 * k + 120, seed=seed, n_rate=0.01)
    res = build_graph(rs.seq, rs.offsets, k, p, np_)
    orc = oracle.graph_wide(rs.seq, rs.offsets, k, p, np_)
    _compare(res, orc)
    assert res.stats["distinct"] == len(orc)
    assert res.stats["sum_count"] == int(orc["count"].sum())
    assert res.stats["sum_edges"] == int(orc["out"].sum() + orc["in"].sum())


def test_wide_genome_reads_with_errors_and_filter():
    g = genome(20_000, seed=7)
    seq, offs = make_reads(g, 2500, 150, 0.01, seed=8)
    rs = ReadSet(seq, offs)
    res = build_graph(rs.seq, rs.offsets, 81, 19, 8)
    orc = oracle.graph_wide(rs.seq, rs.offsets, 81, 19, 8)
    _compare(res, orc)
    f = build_graph(rs.seq, rs.offsets, 81, 19, 8, min_count=3)
    keep = orc[orc["count"] >= 3]
    _compare(f, keep)


def test_wide_locked_state_contention():
    """The same 127-mer occurs thousands of times at once (identical reads): every occurrence but one
    meets the entry locked or occupied; the count must be exact (no lost or duplicated insertion)."""
    rng = np.random.default_rng(3)
    r = "".join("ACGT"[x] for x in rng.integers(0, 4, 160))
    reads = [r] * 3000 + ["".join("ACGT"[x] for x in rng.integers(0, 4, 140)) for _ in range(200)]
    b = "".join(reads).encode()
    offs = np.zeros(len(reads) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(x) for x in reads])
    rs = ReadSet(np.frombuffer(b, dtype=np.uint8).copy(), offs)
    res = build_graph(rs.seq, rs.offsets, 127, 23, 2)
    orc = oracle.graph_wide(rs.seq, rs.offsets, 127, 23, 2)
    _compare(res, orc)
    assert int(res.vertices["count"].max()) >= 3000


def test_wide_table_overflow_detected_and_rebuilt():
    """Reading O with four-word keys: an undersized table reports DBG_ETABLEFULL, the rebuild at
    capacity N^i_kmer gives the oracle's graph."""
    rs = random_reads(300, 90, 200, seed=9)
    b = DbgBuilder(75, 21, 3, lam=0.04, alpha=0.5, mode="resident")
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.msp(d_bases, d_off)
    assert b.sync_sizes()
    b.plan()
    b.reset_output(1 << 18)
    b.step2()
    assert _lib.dbg_sync_status(b.d_status) == _lib.DBG_ETABLEFULL
    res = build_graph(rs.seq, rs.offsets, 75, 21, 3, lam=0.04, alpha=0.5)
    _compare(res, oracle.graph_wide(rs.seq, rs.offsets, 75, 21, 3))
