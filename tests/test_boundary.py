"""C-ABI library (libdbg.so): loads, exports every symbol include/dbg.h declares, and its host-only
entry points behave (no GPU needed: no compute call launches a kernel here)."""
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = os.path.join(ROOT, "tests", "golden")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icdcs_qiul17_b200 import build

    build.build()
    from paper_conf_icdcs_qiul17_b200 import _lib

    _lib.load()
    return _lib


def _declared():
    src = open(os.path.join(ROOT, "include", "dbg.h")).read()
    return re.findall(r"DBG_API\s+[\w\s\*]+?\b(dbg_\w+)\s*\(", src)


def test_exports_every_declared_symbol(lib):
    names = _declared()
    assert sorted(names) == sorted(lib.SIGNATURES)   # the binding mirrors the header exactly
    raw = lib.load()
    for n in names:
        assert hasattr(raw, n), n
        assert n in lib.SIGNATURES, n


def test_abi_and_sizes(lib):
    assert lib.dbg_abi_version() == 12
    p31 = lib.params(31, 11, 16)
    p63 = lib.params(63, 19, 16)
    assert lib.dbg_record_words(p31) == 4 and lib.dbg_record_max_kmers(p31) == 16
    assert lib.dbg_record_words(p63) == 8 and lib.dbg_record_max_kmers(p63) == 48
    assert lib.dbg_slot_bytes(p31) == 48 and lib.dbg_key_bytes(p31) == 16
    assert lib.dbg_slot_bytes(p63) == 64 and lib.dbg_key_bytes(p63) == 32
    assert lib.dbg_packed_words(0) == 1 and lib.dbg_packed_words(32) == 2 and lib.dbg_packed_words(33) == 3
    # the record header's 6-bit K-mer count caps long records at 63 K-mers (dbg.h)
    assert lib.dbg_record_words(lib.params(41, 11, 16)) == 8 and lib.dbg_record_max_kmers(lib.params(41, 11, 16)) == 63
    assert lib.dbg_record_words(lib.params(65, 11, 16)) == 16 and lib.dbg_record_max_kmers(lib.params(65, 11, 16)) == 63
    # fine partitions: NP * refine <= 2^24 - 1 (the header's 24-bit pid field); whole human (65.1 G
    # K-mers, NP = 960) wants ~39 M and is clamped there
    # two-level scatter workspace: fill, offsets and tile counts of the <= 2048 buckets (<= 4096 at
    # 2^24 - 1 fine partitions, 4096 partitions a bucket) that msp.cu's ts_shift picks
    def buckets(np_):
        sh = 0
        while sh < 12 and -(-np_ // (1 << sh)) > 2048:
            sh += 1
        return -(-np_ // (1 << sh))
    for np_, ref in ((16, 1), (16, 625), (512, 3084), (512, 7444), (960, 17476)):
        nb = buckets(np_ * ref)
        assert nb <= 4096
        assert lib.dbg_scatter_work_words(lib.params(31, 11, np_, refine=ref)) == 3 * nb + 2
    from paper_conf_icdcs_qiul17_b200.graph import MAX_FINE_PARTITIONS, auto_refine
    assert MAX_FINE_PARTITIONS == (1 << 24) - 1
    assert auto_refine(65_100_000_000, 31, 11, 960) == MAX_FINE_PARTITIONS // 960


def test_table2_sizing_pin(lib):
    """Table II (L1005-1013): with lambda=2, alpha=0.5 the capacity is N^i_kmer, so at the 32 B per
    entry of L1242 the max table per partition is 32 B x (2725 M / NP) within 7 %."""
    prm = lib.params(27, 11, 16, 2.0, 0.5)
    for l in open(os.path.join(GOLD, "table1_table2.txt")):
        f = l.split()
        if f and f[0] == "TABLE2":
            np_, kmers_m, size_mb = int(f[1]), float(f[2]), float(f[3])
            n_i = int(2725e6 / np_)
            assert abs(n_i / 1e6 - kmers_m) <= 0.5 + 0.01 * kmers_m
            cap = lib.dbg_table_capacity(prm, n_i)
            assert cap == n_i
            assert abs(cap * 32 / 1e6 - size_mb) / size_mb < 0.07
    # lambda/(4 alpha) scaling (L783-788)
    assert lib.dbg_table_capacity(lib.params(31, 11, 16, 2.0, 0.8), 1000) == 625
    assert lib.dbg_table_capacity(lib.params(31, 11, 16, 1.0, 0.5), 1001) == 501
    assert lib.dbg_table_capacity(prm, 0) == 0
    assert lib.dbg_table_capacity(lib.params(31, 11, 16, 0.001, 0.5), 10) == 1
    # dbg_table_bytes = capacity x slot bytes (the d_table block dbg_hash_build takes)
    for k, n in ((31, 1000), (63, 12345), (27, 2725 * 10 ** 6 // 512)):
        q = lib.params(k, 11, 16, 2.0, 0.8)
        assert lib.dbg_table_bytes(q, n) == lib.dbg_table_capacity(q, n) * lib.dbg_slot_bytes(q)
    assert lib.dbg_table_bytes(prm, 0) == 0


def test_onchip_placement_rule(lib):
    """dbg.h dbg_smem_onchip: grouped (1) while the Property-1 capacity fits a CTA table, split over
    ceil(1.25 c / slots) <= smem_split CTAs above that, global (0) past the split limit or when
    N^i_kmer > 65535 (16-bit on-chip counters)."""
    prm = lib.params(31, 11, 16)              # capacity = N^i_kmer
    S = lib.dbg_smem_table_slots(prm)
    assert S >= 1024 and S % 64 == 0
    on = lambda prm, n: lib.dbg_smem_onchip(prm, n)
    assert on(prm, 0) == 0 and on(prm, 1) == 1 and on(prm, S) == 1
    assert on(prm, S + 1) == 2                 # ceil(1.25 (S+1) / S)
    assert on(prm, 2 * S) == 3 and on(prm, (8 * S) // 5) == 2 and on(prm, (8 * S) // 5 + 1) == 3
    assert on(prm, 65535) == -(-5 * 65535 // (4 * S)) and on(prm, 65536) == 0
    assert on(lib.params(31, 11, 16, smem_split=1), S + 1) == 0
    two = lib.params(31, 11, 16, smem_split=2)
    assert on(two, (8 * S) // 5) == 2 and on(two, (8 * S) // 5 + 1) == 0
    half = lib.params(31, 11, 16, 1.0, 0.5)   # capacity = ceil(N / 2)
    assert on(half, 2 * S) == 1 and on(half, 2 * S + 1) == 2
    assert on(lib.params(30, 11, 16), 10) == -1


def test_auto_fine_p_rule(lib):
    """graph.auto_fine_p: the smallest P' >= P with 4^P' >= 4 (K-P'+1) N lambda/(4 alpha) / slots."""
    from paper_conf_icdcs_qiul17_b200 import auto_fine_p

    S = lib.dbg_smem_table_slots(lib.params(31, 11, 1))
    assert auto_fine_p(1000, 31, 11) == 11
    for n in (276_000_000, 2_627_000_000, 28_000_000_000, 10 ** 15):
        q = auto_fine_p(n, 31, 11)
        assert 4.0 ** q >= 4 * (31 - q + 1) * n / S
        assert q == 11 or 4.0 ** (q - 1) < 4 * (31 - q + 2) * n / S
    assert auto_fine_p(2_627_000_000, 31, 11) > 11          # chr14-sized input: longer minimizer
    assert auto_fine_p(10 ** 9, 63, 19) == 19


def test_encoder_fig4_and_rules(lib):
    """Fig. 4 (L598-606) bits; unknown -> A and lower case (L205-206)."""
    lines = dict(l.split() for l in open(os.path.join(GOLD, "fig4_encoding.txt")) if l.strip() and l[0] != "#")
    seq = np.frombuffer(lines["KMER"].encode(), dtype=np.uint8)
    out = np.zeros(lib.dbg_packed_words(len(seq)), dtype=np.uint64)
    lib.dbg_encode_ascii(seq, out)
    assert int(out[0]) >> 48 == int(lines["BITS"], 2)
    s = np.frombuffer(b"acgtNRYX" * 5, dtype=np.uint8)
    o1 = np.zeros(lib.dbg_packed_words(len(s)), dtype=np.uint64)
    lib.dbg_encode_ascii(s, o1)
    t = np.frombuffer(b"ACGTAAAA" * 5, dtype=np.uint8)
    o2 = np.zeros(lib.dbg_packed_words(len(t)), dtype=np.uint64)
    lib.dbg_encode_ascii(t, o2)
    assert (o1 == o2).all()
    # base i at word i/32, most significant first; pad word zero
    rng = np.random.default_rng(0)
    codes = rng.integers(0, 4, 1000)
    seq = np.frombuffer(b"ACGT", dtype=np.uint8)[codes]
    w = np.zeros(lib.dbg_packed_words(1000), dtype=np.uint64)
    lib.dbg_encode_ascii(seq, w)
    for i in range(0, 1000, 7):
        assert (int(w[i // 32]) >> (62 - 2 * (i % 32))) & 3 == codes[i]
    assert int(w[-1]) == 0


def test_invalid_arguments_return_before_launch(lib):
    from paper_conf_icdcs_qiul17_b200._lib import DbgError, partition_set

    part = partition_set(1, 1, 1, 1, 1, None, 0, None)
    for prm in (lib.params(30, 11, 16), lib.params(31, 0, 16), lib.params(31, 32, 16), lib.params(31, 11, 0),
                lib.params(129, 11, 16), lib.params(64, 11, 16), lib.params(65, 11, 16, fine_p=13),
                lib.params(31, 11, 16, fine_p=32), lib.params(21, 11, 16, fine_p=23),
                lib.params(31, 11, 16, fine_p=-1)):
        with pytest.raises(DbgError) as e:
            lib.dbg_msp_partition(prm, 1, 1, 1, 1, part, None)
        assert e.value.status == lib.DBG_EINVAL
    with pytest.raises(DbgError):
        lib.dbg_hash_build(lib.params(31, 11, 16), partition_set(1, 1, 1, 1, 1, None, 0, 1), 5, 2, 1, 1, 1, None)
    assert lib.dbg_status_string(lib.DBG_ETABLEFULL).startswith("hash table full")
    # row f3: K > 63 runs through the resident tables only
    p65 = lib.params(65, 21, 4)
    assert lib.dbg_record_words(p65) == 16 and lib.dbg_record_max_kmers(p65) == 63  # 6-bit header count
    assert lib.dbg_key_bytes(p65) == 48 and lib.dbg_slot_bytes(p65) == 80
    assert lib.dbg_smem_onchip(p65, 100) == 0 and lib.dbg_smem_table_slots(p65) == 0
    with pytest.raises(DbgError) as e:
        lib.dbg_table_plan_split(p65, 1, 1, None, None)
    assert e.value.status == lib.DBG_EINVAL


def test_product_has_no_oracle_dependency():
    """The product package never imports, loads or calls anything under oracle/ (DESIGN.md Sec. 3)."""
    pkg = os.path.join(ROOT, "paper_conf_icdcs_qiul17_b200")
    bad = re.compile(r"(import\s+oracle|from\s+oracle|liboracle|oracle_\w+\s*\(|oracle/\w+\.(cpp|py))")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert not bad.search(src), f


def test_graph_writer_roundtrip(lib, tmp_path):
    """Row f4 graph writer (host-only entry point): header + records, append updates the count."""
    from paper_conf_icdcs_qiul17_b200 import read_graph, write_graph

    rng = np.random.default_rng(3)
    v = np.zeros(1000, dtype=lib.VERTEX_DTYPE)
    v["kmer_lo"] = rng.integers(0, 1 << 62, 1000, dtype=np.uint64)
    v["count"] = rng.integers(1, 50, 1000)
    v["out"] = rng.integers(0, 9, (1000, 4))
    v["pid"] = rng.integers(0, 16, 1000)
    prm = lib.params(31, 11, 16, min_count=2)
    path = str(tmp_path / "g.dbg")
    write_graph(path, prm, v[:600])
    write_graph(path, prm, v[600:], append=True)
    write_graph(path, prm, v[:0], append=True)
    h, got = read_graph(path)
    assert h == {"k": 31, "p": 11, "num_partitions": 16, "min_count": 2, "n_vertices": 1000}
    assert got.tobytes() == v.tobytes()
    assert os.path.getsize(path) == 64 + 56 * 1000
    with pytest.raises(lib.DbgError):  # append with another K: header mismatch
        write_graph(path, lib.params(33, 11, 16), v[:1], append=True)
    write_graph(path, prm, v[:5])  # no append: truncates
    assert read_graph(path)[0]["n_vertices"] == 5
