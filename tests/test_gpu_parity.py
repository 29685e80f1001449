"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar: bit-exact -- integer work.  Sorted (kmer_hi, kmer_lo, count, out[4], in[4],
pid) records must equal the oracle's; totals and the order-independent checksum too.
"""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, build_graph, encode_reads, _lib  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import build as _build  # noqa: E402
from synth import ReadSet, genome, make_config, make_reads, random_reads  # noqa: E402

from gpu_helpers import (compare_vertices, decode_records, occurrences_from_oracle_msp,  # noqa: E402
                         occurrences_from_records)

NT = os.cpu_count() or 1
_build.build()


def _readset(reads):
    b = "".join(reads).encode()
    offs = np.zeros(len(reads) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(r) for r in reads])
    return ReadSet(np.frombuffer(b, dtype=np.uint8).copy(), offs)


def _check(rs, k, p, np_, **kw):
    res = build_graph(rs.seq, rs.offsets, k, p, np_, **kw)
    orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT)
    compare_vertices(res.vertices, orc)
    st = res.stats
    assert st["distinct"] == len(orc)
    assert st["sum_count"] == int(orc["count"].sum())
    assert st["sum_edges"] == int(orc["out"].sum() + orc["in"].sum())
    assert st["checksum"] == oracle.checksum(orc)
    return res, orc


def test_tiny_config_bitexact():
    rs = make_config("tiny")
    res, orc = _check(rs, rs.k, rs.p, rs.num_partitions)
    # I1: sum of counts = sum(L-K+1)
    assert res.stats["sum_count"] == rs.n_kmers()
    assert res.n_kmers == rs.n_kmers()
    fine = np.arange(len(res.part_kmers)) % rs.num_partitions  # fine pid -> the paper's pid
    assert np.array_equal(np.bincount(fine, weights=res.part_kmers, minlength=rs.num_partitions).astype(np.int64),
                          np.bincount(orc["pid"], weights=orc["count"], minlength=rs.num_partitions).astype(np.int64))


CASES = [(3, 1, 1), (5, 3, 3), (7, 7, 16), (11, 4, 5), (31, 11, 16), (31, 31, 3), (31, 1, 7),
         (33, 13, 7), (39, 15, 9), (41, 17, 11), (63, 19, 16), (63, 1, 4), (63, 31, 64), (21, 9, 1)]


@pytest.mark.parametrize("k,p,np_", CASES)
def test_ragged_random_reads(k, p, np_):
    rs = random_reads(400, 1, 2 * k + 150, seed=k * 100 + p, n_rate=0.01, lower_rate=0.02)
    _check(rs, k, p, np_)


@pytest.mark.parametrize("k,p", [(31, 11), (63, 19), (31, 31), (9, 3)])
def test_long_reads_and_repeats(k, p):
    rs = random_reads(20, 300, 3000, seed=7 + k)
    reads = rs.reads()
    reads += ["A" * 700, "AC" * 400, "ACGTTGCA" * 90, "T" * (k + 1), "G" * k, "ACG"]
    _check(_readset(reads), k, p, 13)


def test_hot_key_stress():
    """One K-mer repeated ~10^5 times (poly-A), plus its reverse complement."""
    reads = ["A" * 2000] * 30 + ["T" * 2000] * 30 + ["C" * 200]
    res, orc = _check(_readset(reads), 31, 11, 8)
    assert res.vertices["count"].max() == 60 * (2000 - 31 + 1)


def test_edge_cases_empty_short():
    empty = ReadSet(np.zeros(0, np.uint8), np.zeros(1, np.uint64))
    res = build_graph(empty.seq, empty.offsets, 31, 11, 16)
    assert res.n_vertices == 0 and res.stats["distinct"] == 0
    _check(_readset(["ACGT", "", "ACGTACGTA", "TTTTTTTTT"]), 9, 3, 4)
    _check(_readset(["A" * 31]), 31, 11, 16)


def test_msp_records_vs_oracle_superkmers():
    """Kernel (a): per-partition multisets of (K-mer, pred, succ) occurrences from the emitted
    records equal the oracle's MSP superkmers (reading S: buffer order is not unique)."""
    for (k, p, np_, seed) in [(31, 11, 16, 1), (63, 19, 8, 2), (15, 5, 3, 3), (31, 31, 5, 4)]:
        rs = random_reads(200, 1, 300, seed=seed, n_rate=0.01)
        b = DbgBuilder(k, p, np_)
        d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
        b.msp(d_bases, d_off)
        assert b.sync_sizes()
        torch.cuda.synchronize()
        nrec = int(b.part_records.sum())
        words = b.records[: nrec * b.rec_words].cpu().numpy().view(np.uint32)
        recs = decode_records(words, b.rec_words, k)
        sk = oracle.msp(rs.seq, rs.offsets, k, p, np_)
        nmax = _lib.dbg_record_max_kmers(b.prm)
        # sizes per partition (count pass)
        want_k = np.bincount(sk["pid"], weights=sk["n_kmers"], minlength=np_).astype(np.int64)
        want_r = np.bincount(sk["pid"], weights=(sk["n_kmers"] + nmax - 1) // nmax,
                             minlength=np_).astype(np.int64)
        assert np.array_equal(b.part_kmers, want_k)
        assert np.array_equal(b.part_records, want_r)
        # records sit in their partition's range
        off = b.d_rec_off.cpu().numpy()
        pids = np.array([r[0] for r in recs])
        for q in range(np_):
            assert (pids[off[q]:off[q + 1]] == q).all()
        assert occurrences_from_records(recs, k) == occurrences_from_oracle_msp(sk, rs.reads(), k)


@pytest.mark.parametrize("mode", ["smem", "resident"])
def test_table_overflow_detected_and_rebuilt(mode):
    """Reading O: an undersized table (lambda/(4 alpha) << distinct/N) overflows; the status word
    reports DBG_ETABLEFULL and the builder rebuilds at capacity N^i_kmer with the same result."""
    g = genome(20_000, seed=5)
    seq, offs = make_reads(g, 3000, 100, 0.01, seed=6)
    rs = ReadSet(seq, offs)
    b = DbgBuilder(31, 11, 4, lam=0.04, alpha=0.5, mode=mode)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.msp(d_bases, d_off)
    assert b.sync_sizes()
    b.plan()
    b.reset_output(1 << 20)
    b.step2()
    assert _lib.dbg_sync_status(b.d_status) == _lib.DBG_ETABLEFULL
    _check(rs, 31, 11, 4, lam=0.04, alpha=0.5, mode=mode)


def test_resident_batches_give_same_graph():
    rs = make_config("tiny", scale=0.5)
    a = build_graph(rs.seq, rs.offsets, 31, 11, 16)
    b = build_graph(rs.seq, rs.offsets, 31, 11, 16, table_budget_bytes=48 * 2000, mode="resident")
    assert len(b.batches) > 4
    assert a.vertices.tobytes() == b.vertices.tobytes()
    assert a.stats == b.stats


@pytest.mark.parametrize("k,p,np_", [(31, 11, 16), (63, 19, 8), (41, 17, 5), (7, 3, 3)])
def test_resident_mode_parity(k, p, np_):
    rs = random_reads(300, 1, 2 * k + 100, seed=k + np_, n_rate=0.01)
    _check(rs, k, p, np_, mode="resident")


@pytest.mark.parametrize("k,p,np_,refine", [(31, 11, 1, 1), (31, 11, 3, 1), (63, 19, 2, 1), (31, 11, 4, 8),
                                             (41, 13, 3, 16), (21, 7, 5, 64)])
def test_smem_with_global_tier(k, p, np_, refine):
    """On-chip tables for partitions that fit one SM, the global-table path for the rest (here NP is
    small, so some partitions exceed dbg_smem_table_slots), and refined partitions whose pid is
    reported modulo NP -- all equal to the oracle."""
    g = genome(60_000, seed=k + np_)
    seq, offs = make_reads(g, 4000, 100, 0.01, seed=refine + 3)
    rs = ReadSet(seq, offs)
    res, _ = _check(rs, k, p, np_, refine=refine, smem_split=1)
    if refine == 1 and np_ <= 3:
        assert res.batches, "expected some partitions on the global-table path"


@pytest.mark.parametrize("k,p,np_,refine,split", [(31, 11, 3, 1, 0), (31, 11, 1, 2, 0), (63, 19, 2, 1, 0),
                                                   (41, 13, 12, 1, 3), (21, 7, 4, 2, 64), (31, 11, 12, 1, 2)])
def test_smem_split_partitions(k, p, np_, refine, split):
    """Partitions larger than one CTA table built on chip over several sub-tables (dbg.h
    dbg_smem_onchip), next to grouped ones and (with a small split limit) global ones.  1500 reads
    of 100 bp: partitions of ~10^4 K-mers, above one CTA table and below the 65535 bound."""
    g = genome(60_000, seed=k + np_ + 1)
    seq, offs = make_reads(g, 1500, 100, 0.01, seed=refine + 5)
    rs = ReadSet(seq, offs)
    res, _ = _check(rs, k, p, np_, refine=refine, smem_split=split)
    prm = _lib.params(k, p, np_, refine=refine, smem_split=split)
    place = np.array([_lib.dbg_smem_onchip(prm, int(n)) for n in res.part_kmers])
    assert (place >= 2).any(), "expected split partitions"
    assert bool(res.batches) == bool((place[res.part_kmers > 0] == 0).any())


@pytest.mark.parametrize("k,p,np_,fine_p,refine", [(31, 11, 16, 13, 1), (31, 11, 7, 19, 4), (63, 19, 8, 25, 2),
                                                   (41, 13, 5, 31, 1), (31, 11, 9, 7, 3), (21, 9, 3, 21, 1)])
def test_fine_minimizer_partitioning(k, p, np_, fine_p, refine):
    """dbg_params.fine_p (reading V): the device partitions by a P'-minimizer; the graph and every
    vertex's pid (the partition of its P-minimizer) still equal the oracle's at P."""
    g = genome(30_000, seed=k + fine_p)
    seq, offs = make_reads(g, 2000, 100, 0.01, seed=fine_p)
    rs = ReadSet(seq, offs)
    _check(rs, k, p, np_, refine=refine, fine_p=fine_p)
    rr = random_reads(300, 1, 2 * k + 80, seed=fine_p, n_rate=0.01)
    _check(rr, k, p, np_, refine=refine, fine_p=fine_p)


def test_fine_minimizer_records_vs_oracle_msp():
    """Kernel (a) with fine_p: the records are the oracle's MSP superkmers at P' (Defs. 1-2)."""
    for (k, p, q, np_, seed) in [(31, 11, 15, 16, 1), (63, 19, 27, 8, 2), (15, 5, 9, 3, 3)]:
        rs = random_reads(200, 1, 300, seed=seed, n_rate=0.01)
        b = DbgBuilder(k, p, np_, fine_p=q)
        d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
        b.msp(d_bases, d_off)
        assert b.sync_sizes()
        torch.cuda.synchronize()
        nrec = int(b.part_records.sum())
        recs = decode_records(b.records[: nrec * b.rec_words].cpu().numpy().view(np.uint32), b.rec_words, k)
        sk = oracle.msp(rs.seq, rs.offsets, k, q, np_)
        assert np.array_equal(b.part_kmers, np.bincount(sk["pid"], weights=sk["n_kmers"],
                                                         minlength=np_).astype(np.int64))
        assert occurrences_from_records(recs, k) == occurrences_from_oracle_msp(sk, rs.reads(), k)


def test_split_partition_hot_key_over_16_bits():
    """A vertex seen more than 65535 times sits in a partition with N^i_kmer > 65535: it must take
    the global tables (32-bit counters), not a 16-bit on-chip table."""
    reads = ["A" * 1200] * 60 + ["ACGT" * 300] * 5
    res, orc = _check(_readset(reads), 31, 11, 4)
    assert res.vertices["count"].max() == 60 * (1200 - 31 + 1) > 65535


def test_auto_refine_small_partitions():
    from paper_conf_icdcs_qiul17_b200 import auto_refine
    rs = make_config("tiny")
    f = auto_refine(rs.n_kmers(), 31, 11, 16)
    assert f >= 2
    res, _ = _check(rs, 31, 11, 16, refine=f)
    assert int(res.part_kmers.sum()) == rs.n_kmers()


def test_repeat_runs_deterministic():
    rs = random_reads(2000, 50, 150, seed=99)
    b = DbgBuilder(31, 11, 32)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    r1 = b.build(d_bases, d_off)
    r2 = b.build(d_bases, d_off)
    assert r1.vertices.tobytes() == r2.vertices.tobytes() and r1.stats == r2.stats


def test_strand_symmetry_on_gpu():
    """I5: graph(R) = graph(rc(R)) on the GPU output alone."""
    rs = random_reads(300, 40, 200, seed=3)
    comp = str.maketrans("ACGT", "TGCA")
    rr = _readset([r.translate(comp)[::-1] for r in rs.reads()])
    a = build_graph(rs.seq, rs.offsets, 31, 11, 16)
    b = build_graph(rr.seq, rr.offsets, 31, 11, 16)
    assert a.vertices.tobytes() == b.vertices.tobytes()


def test_smem_global_tier_in_several_batches():
    """Oversize partitions whose global tables do not fit the table budget at once are built in
    several batches (each batch's table block starts at its first partition)."""
    g = genome(60_000, seed=12)
    seq, offs = make_reads(g, 4000, 100, 0.01, seed=13)
    rs = ReadSet(seq, offs)
    res, _ = _check(rs, 31, 11, 3, refine=1, table_budget_bytes=48 * 20_000, smem_split=1)
    assert len(res.batches) >= 2


def test_staging_overflow_repeats_the_step():
    """dbg.h pass 2: after a staging overflow, pass 2 and the on-chip kernel do nothing (no write
    past the buffers); the builder grows the staging and the repeated step is exact."""
    rs = random_reads(3000, 60, 200, seed=31)
    b = DbgBuilder(31, 11, 16, refine=4)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.staging = torch.empty(64 * b.rec_words, dtype=torch.int32, device=b.device)  # far too small
    b.msp(d_bases, d_off)
    b.plan()
    b.reset_output(1 << 20)
    b.step2()
    assert b.overflowed and int(b.d_n_out.item()) == 0
    assert b.staging.numel() // b.rec_words >= int(b.part_records.sum())
    res = b.build(d_bases, d_off)
    orc = oracle.graph(rs.seq, rs.offsets, 31, 11, 16, n_threads=NT)
    compare_vertices(res.vertices, orc)


@pytest.mark.parametrize("mode,k,p,np_,refine,split", [("smem", 31, 11, 4, 8, 0), ("smem", 31, 11, 2, 1, 1),
                                                       ("smem", 63, 19, 3, 2, 0),
                                                       ("resident", 63, 19, 8, 1, 0)])
@pytest.mark.parametrize("min_count", [2, 3])
def test_low_count_filter(mode, k, p, np_, refine, split, min_count):
    """Row f4: extraction drops vertices with count < min_count, in every Step-2 tier
    (grouped and split on-chip tables, global tables), and equals oracle.filter_low_count."""
    g = genome(30_000, seed=21)
    seq, offs = make_reads(g, 6000, 100, 0.01, seed=22)
    rs = ReadSet(seq, offs)
    b = DbgBuilder(k, p, np_, mode=mode, refine=refine, smem_split=split, min_count=min_count)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    res = b.build(d_bases, d_off)
    full = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT)
    orc = oracle.filter_low_count(full, min_count)
    assert 0 < len(orc) < len(full)
    compare_vertices(res.vertices, orc)
    assert res.stats["distinct"] == len(orc)
    assert res.stats["sum_count"] == int(orc["count"].sum())
    assert res.stats["checksum"] == oracle.checksum(orc)
    # the resident tables were cleaned, filtered slots included: an unfiltered rebuild with the same
    # builder (same table buffers) is exact
    b.prm.min_count = b.min_count = 0
    compare_vertices(b.build(d_bases, d_off).vertices, full)


@pytest.mark.parametrize("n_batches", [1, 3, 8])
def test_msp_overlapped_upload_equals_single_pass(n_batches):
    """DbgBuilder.msp_overlapped (read ranges uploaded on a copy stream, MSP appended per range)
    builds the same graph as the single upload + MSP, ragged reads included."""
    rs = random_reads(3000, 1, 300, seed=51, n_rate=0.01)
    b = DbgBuilder(31, 11, 16, refine=4)
    packed = encode_reads(rs.seq, pin=True)
    offs = torch.from_numpy(rs.offsets.view(np.int64)).pin_memory()
    db = torch.empty(packed.numel(), dtype=torch.int64, device="cuda")
    do = torch.empty(offs.numel(), dtype=torch.int64, device="cuda")
    b.msp_overlapped(packed, offs, db, do, n_batches)
    assert b.sync_sizes()
    b.plan()
    b.reset_output(1 << 20)
    b.step2()
    assert _lib.dbg_sync_status(b.d_status) == 0
    orc = oracle.graph(rs.seq, rs.offsets, 31, 11, 16, n_threads=NT)
    compare_vertices(b.vertices(), orc)


@pytest.mark.parametrize("p", [11, 12, 13, 14, 15])
def test_register_blocked_msp_variants(p):
    """K = 31, P = 11..15 run msp_block_kernel<W, P> (van Herk blocks in registers): ragged reads
    (shorter than K, one K-mer, many blocks), N bases; MSP records vs the oracle's superkmers and
    the whole graph vs the oracle."""
    rs = random_reads(2500, 1, 420, seed=60 + p, n_rate=0.02)
    _check(rs, 31, p, 13)
    b = DbgBuilder(31, p, 13)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.msp(d_bases, d_off)
    assert b.sync_sizes()
    torch.cuda.synchronize()
    n = int(b.part_records.sum())
    words = b.records[:n * b.rec_words].cpu().numpy().view(np.uint32)
    got = occurrences_from_records(decode_records(words, b.rec_words, 31), 31)
    sk = oracle.msp(rs.seq, rs.offsets, 31, p, 13)
    assert got == occurrences_from_oracle_msp(sk, rs.reads(), 31)


@pytest.mark.parametrize("k,p,refine", [(31, 11, 1024), (31, 11, 4096), (31, 11, 40000), (31, 11, 1_000_000),
                                         (63, 19, 4096), (63, 19, 300_000)])
def test_two_level_scatter_partition_order(k, p, refine):
    """More than 8192 fine partitions: pass 2 scatters through d_scratch in two counting-sort
    levels (buckets of 2^s consecutive partitions, <= 2048 buckets; then partitions inside a
    bucket, up to 8192 per bucket at 16 M fine partitions).  Every record must land in its own
    partition's range [rec_off[p], rec_off[p+1]), the per-partition record multisets must equal the
    one-level scatter's, and the graph must equal the oracle's."""
    rs = ReadSet(*make_reads(genome(60_000, 5), 6000, 100, 0.01, 105))
    np_ = 16

    def records(two):
        b = DbgBuilder(k, p, np_, refine=refine)
        assert b.two_level
        b.two_level = two
        b.two_level_min_bytes, b.two_level_words = 0, (4, 8, 16)  # at every size here
        d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
        b.msp(d_bases, d_off)
        assert b.sync_sizes()
        torch.cuda.synchronize()
        n = int(b.part_records.sum())
        w = b.records[:n * b.rec_words].cpu().numpy().view(np.uint32).reshape(n, b.rec_words)
        off = np.concatenate([[0], np.cumsum(b.part_records)])
        pid = w[:, 0] >> 8
        assert np.array_equal(pid, np.repeat(np.arange(len(b.part_records)), b.part_records))
        rows = [tuple(r) for r in w]
        return off, sorted(rows)

    off2, rows2 = records(True)
    off1, rows1 = records(False)
    assert np.array_equal(off1, off2)
    assert rows1 == rows2
    # and the graph through the two-level path
    b = DbgBuilder(k, p, np_, refine=refine)
    b.two_level_min_bytes, b.two_level_words = 0, (4, 8, 16)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    res = b.build(d_bases, d_off)
    compare_vertices(res.vertices, oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT))


@pytest.mark.parametrize("k,p", [(63, 19), (21, 7), (45, 30)])
def test_warp_msp_chunks_pieces_and_fallback(k, p):
    """msp_warp_kernel (every (K, P) but K = 31 with P = 11..15): chunks of 32 reads whose words
    fit the TMA-staged buffer next to chunks that do not (long reads: global-memory windows),
    reads longer than one piece of 32R P-mer positions (the open superkmer carried across
    pieces), reads of exactly K bases, superkmers longer than a record (pieces), and P + R - 1 >
    32 (two-window codes, P = 30).  Records vs the oracle's superkmers (per-partition sizes and
    record counts) and the whole graph vs the oracle."""
    rng = np.random.default_rng(1000 + k + p)
    reads = []
    for q in range(7):  # chunks: short, long (unstaged), mixed, ...
        for t in range(32):
            if q == 1 or (q == 4 and t % 5 == 0):
                n = int(rng.integers(400, 1500))
            elif q == 5 and t % 3 == 0:
                n = k
            else:
                n = int(rng.integers(k, 160))
            reads.append("".join(rng.choice(list("ACGT"), n)))
    reads[40] = "A" * 900          # one minimizer over the whole read: superkmer pieces
    reads[70] = "AC" * 300
    rs = _readset(reads)
    _check(rs, k, p, 11)
    b = DbgBuilder(k, p, 11)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.msp(d_bases, d_off)
    assert b.sync_sizes()
    torch.cuda.synchronize()
    sk = oracle.msp(rs.seq, rs.offsets, k, p, 11)
    nmax = _lib.dbg_record_max_kmers(b.prm)
    want_k = np.bincount(sk["pid"], weights=sk["n_kmers"], minlength=11).astype(np.int64)
    want_r = np.bincount(sk["pid"], weights=(sk["n_kmers"] + nmax - 1) // nmax, minlength=11).astype(np.int64)
    assert np.array_equal(b.part_kmers, want_k)
    assert np.array_equal(b.part_records, want_r)
    n = int(b.part_records.sum())
    words = b.records[:n * b.rec_words].cpu().numpy().view(np.uint32)
    assert occurrences_from_records(decode_records(words, b.rec_words, k), k) == \
        occurrences_from_oracle_msp(sk, rs.reads(), k)


@pytest.mark.parametrize("k,p,np_,refine", [(31, 13, 16, 300_000), (63, 19, 7, 2_396_745)])
def test_fine_pids_beyond_22_bits(k, p, np_, refine):
    """dbg.h: the record header's 24-bit fine pid -- NP * refine above 2^22 (4.8 M and 16.8 M - 1
    fine partitions, almost all empty): multi-tile scans, the on-chip plan over millions of
    partitions, the two-level scatter, and the paper's pid (fine pid mod NP) of every vertex."""
    g = genome(30_000, seed=k + 1)
    seq, offs = make_reads(g, 3000, 120, 0.01, seed=k + 2)
    _check(ReadSet(seq, offs), k, p, np_, refine=refine)
