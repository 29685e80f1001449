"""Pins for the CPU oracle (oracle/dbg_oracle.cpp) against what the paper and the mathematics fix.

None of these re-types the oracle's own formula: each one checks it against a value printed in
the paper (tests/golden/), an independent closed form, an invariant, or a string brute force.
"""
import math
import os

import numpy as np
import pytest

from oracle import brute
from synth import genome, make_reads, random_reads, ReadSet

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _as_dict(recs, k):
    d = {}
    for r in recs:
        code = (int(r["key_hi"]) << 64) | int(r["key_lo"])
        s = "".join("ACGT"[(code >> (2 * (k - 1 - t))) & 3] for t in range(k))
        d[s] = [int(r["count"]), [int(x) for x in r["out"]], [int(x) for x in r["in"]], int(r["pid"])]
    return d


def _readset(reads):
    b = "".join(reads).encode()
    offs = np.zeros(len(reads) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(r) for r in reads])
    return ReadSet(np.frombuffer(b, dtype=np.uint8).copy(), offs)


# ---------------------------------------------------------------- paper-printed values


def test_fig1_worked_example(oracle_lib):
    """PAPER.md Fig. 1 (L186-197): edge multiplicities 2 and 1 (tests/golden/fig1_edges.txt)."""
    lines = [l.split() for l in open(os.path.join(GOLD, "fig1_edges.txt")) if l.strip() and l[0] != "#"]
    k = int(lines[0][1])
    np_ = int(lines[1][1])
    reads = lines[2][1:]
    expect = {l[0]: [int(l[1]), [int(x) for x in l[2:6]], [int(x) for x in l[6:10]]] for l in lines[3:]}
    rs = _readset(reads)
    got = _as_dict(oracle_lib.graph(rs.seq, rs.offsets, k, 3, np_), k)
    assert {v: e[:3] for v, e in got.items()} == expect


def test_fig1_kmer_count():
    """Fig. 1: reads of length 23 with K=5 give 19 K-mers each (L187-190); N(L-K+1) (L176-177)."""
    rs = random_reads(7, 23, 23, seed=11)
    import oracle

    recs = oracle.graph(rs.seq, rs.offsets, 5, 3, 4)
    assert int(recs["count"].sum()) == 7 * 19


def test_fig4_encoding(oracle_lib):
    """Fig. 4 (L598-606): the 2-word K-mer "00100101,01110011" is AGCCCTAT under reading A."""
    lines = dict(l.split() for l in open(os.path.join(GOLD, "fig4_encoding.txt")) if l.strip() and l[0] != "#")
    assert oracle_lib.canonical(lines["KMER"]) == int(lines["BITS"], 2)


def test_table1_occurrence_formula():
    """Table I (L925-935): # duplicate vertices = N (L-K+1) within the 2 % rounding of N."""
    for l in open(os.path.join(GOLD, "table1_table2.txt")):
        f = l.split()
        if f and f[0] == "TABLE1":
            L, n_m, dup_m = int(f[2]), float(f[3]), float(f[4])
            assert abs(n_m * (L - 27 + 1) - dup_m) / dup_m < 0.02


def test_table1_occurrences_on_oracle(oracle_lib):
    """I1 at a Table-I read length: sum of vertex counts = N (L-K+1) (K=27, L=101)."""
    g = genome(20_000, seed=7)
    seq, offs = make_reads(g, 300, 101, 0.005, seed=8)
    recs = oracle_lib.graph(seq, offs, 27, 11, 8)
    assert int(recs["count"].sum()) == 300 * (101 - 27 + 1)


def test_property1_appendix_closed_form():
    """Appendix, Eqs. (4)/(5) (L1349-1434): E[#erroneous K-mers | one error] by enumeration."""
    for L in (23, 50, 100, 101, 124):
        for K in range(1, L + 1):
            # exact: average over the error position of the K-mers covering it
            cover = [min(e, L - K) - max(0, e - K + 1) + 1 for e in range(L)]
            exact = sum(cover) / L
            if K <= (L + 1) // 2:
                paper = K * (L - 2 * K + 2) / L + sum(m * 2 / L for m in range(1, K))
            else:
                paper = (L - K + 1) * (2 * K - L) / L + sum(m * 2 / L for m in range(1, L - K + 1))
            assert math.isclose(exact, paper, rel_tol=1e-12), (L, K)
            assert math.isclose(exact, K * (L - K + 1) / L, rel_tol=1e-12)
            assert exact <= (L + 1) ** 2 / (4 * L) + 1e-12  # the Theta(L/4) bound of (4)/(5)


def test_property1_distinct_vertices_statistical(oracle_lib):
    """Property 1 (L540-555): distinct vertices ~ covered genome K-mers + erroneous K-mers."""
    G, N, L, K, e = 40_000, 4_000, 100, 31, 0.01
    g = genome(G, seed=21)
    seq, offs = make_reads(g, N, L, e, seed=22)
    recs = oracle_lib.graph(seq, offs, K, 11, 4, n_threads=4)
    p_ok = (1 - e) ** K
    starts = G - L + 1
    covered = 0.0
    for x in range(G - K + 1):
        n_cov = min(x, G - L) - max(0, x + K - L) + 1
        q = n_cov / starts
        covered += 1 - (1 - q * p_ok) ** N
    erroneous = N * (L - K + 1) * (1 - p_ok)
    expect = covered + erroneous
    assert abs(len(recs) - expect) / expect < 0.01, (len(recs), expect)


# ---------------------------------------------------------------- brute force


@pytest.mark.parametrize(
    "k,p,np_,seed",
    [(3, 1, 1, 1), (3, 3, 3, 2), (5, 3, 3, 3), (5, 5, 16, 4), (7, 1, 16, 5), (7, 3, 2, 6),
     (31, 11, 16, 7), (31, 31, 3, 8), (9, 4, 5, 9), (33, 13, 7, 10), (63, 19, 16, 11),
     (63, 1, 4, 12)],
)
def test_oracle_vs_string_brute_force(oracle_lib, k, p, np_, seed):
    rs = random_reads(40, 1, 2 * k + 40, seed=seed, n_rate=0.02, lower_rate=0.05)
    got = _as_dict(oracle_lib.graph(rs.seq, rs.offsets, k, p, np_), k)
    want = brute.graph(rs.reads(), k, p, np_)
    assert got == want


@pytest.mark.parametrize("k,p", [(5, 3), (31, 11), (31, 13), (63, 19), (21, 21), (9, 1)])
def test_oracle_helpers_vs_string_brute_force(oracle_lib, k, p):
    """oracle.kmer_minimizer (Def. 1, readings D, E) and oracle.canonical against the
    string brute force: the lexicographically smallest of all P-substrings of the K-mer and of its
    reverse complement, and the smaller of the K-mer and its reverse complement."""
    rng = np.random.default_rng(k * 100 + p)
    for _ in range(200):
        x = "".join("ACGT"[c] for c in rng.integers(0, 4, k))
        m = brute.minimizer_string(x, p)
        assert oracle_lib.kmer_minimizer(x, p) == brute.code(m)
        assert oracle_lib.canonical(x) == brute.code(brute.canonical_string(x))


def test_oracle_threads_equal(oracle_lib):
    rs = random_reads(300, 20, 120, seed=13)
    a = oracle_lib.graph(rs.seq, rs.offsets, 11, 5, 7, n_threads=1)
    b = oracle_lib.graph(rs.seq, rs.offsets, 11, 5, 7, n_threads=5)
    assert a.tobytes() == b.tobytes()


def test_oracle_msp_vs_brute(oracle_lib):
    for (k, p, np_, seed) in [(5, 3, 4, 1), (31, 11, 16, 2), (21, 7, 3, 3), (9, 9, 5, 4)]:
        rs = random_reads(30, 1, 90, seed=seed)
        sk = oracle_lib.msp(rs.seq, rs.offsets, k, p, np_)
        want = brute.superkmers(rs.reads(), k, p, np_)
        got = [(int(s["read"]), int(s["start"]), int(s["n_kmers"]), int(s["pid"]), int(s["has_left"]),
                int(s["has_right"])) for s in sk]
        assert got == [w[:6] for w in want]
        assert [int(s["minimizer"]) for s in sk] == [brute.code(w[6]) for w in want]


# ---------------------------------------------------------------- closed form and invariants


@pytest.mark.parametrize("k,seed", [(3, 1), (5, 2), (7, 3), (11, 4), (31, 5)])
def test_kplus1_closed_form(oracle_lib, k, seed):
    """Edge multiplicities equal (K+1)-mer counts (north star; odd K, no palindromes)."""
    rs = random_reads(60, 1, 80, seed=seed, alphabet=b"ACGT" if k > 5 else b"ACGTAC")
    got = {v: e[:3] for v, e in _as_dict(oracle_lib.graph(rs.seq, rs.offsets, k, 1, 1), k).items()}
    assert got == brute.kplus1_closed_form(rs.reads(), k)


def test_kplus1_closed_form_with_palindromic_kplus1mers(oracle_lib):
    """A palindromic (K+1)-mer (even length) increments the same counter twice (reading K)."""
    reads = ["ACGT", "AACGTT", "TTAA", "GAATTC", "ACGTACGT"]
    rs = _readset(reads)
    got = {v: e[:3] for v, e in _as_dict(oracle_lib.graph(rs.seq, rs.offsets, 3, 1, 1), 3).items()}
    assert got == brute.kplus1_closed_form(reads, 3)


def _tiny_erroneous():
    g = genome(30_000, seed=31)
    seq, offs = make_reads(g, 2_000, 100, 0.01, seed=32)
    return ReadSet(seq, offs)


def test_invariants_I1_I2_I3_I4(oracle_lib):
    rs = _tiny_erroneous()
    K, P, NP = 31, 11, 16
    recs = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP, n_threads=4)
    L = rs.lengths()
    # I1: total vertex occurrences
    assert int(recs["count"].sum()) == int(np.maximum(L - K + 1, 0).sum())
    # I2: every adjacent K-mer pair counts once at each endpoint
    assert int(recs["out"].sum() + recs["in"].sum()) == 2 * int(np.maximum(L - K, 0).sum())
    d = _as_dict(recs, K)
    # I3 mirror: out_v[c] > 0 -> w = v[1:]+c has the matching in-edge (or out-edge if w is not canonical)
    for v, (cnt, out, inn, pid) in d.items():
        for ci, c in enumerate("ACGT"):
            if out[ci]:
                w = v[1:] + c
                cw = brute.canonical_string(w)
                if cw == w:
                    assert d[cw][2]["ACGT".index(v[0])] == out[ci]
                else:
                    assert d[cw][1][3 - "ACGT".index(v[0])] == out[ci]
            if inn[ci]:
                w = c + v[:-1]
                cw = brute.canonical_string(w)
                if cw == w:
                    assert d[cw][1]["ACGT".index(v[-1])] == inn[ci]
                else:
                    assert d[cw][2][3 - "ACGT".index(v[-1])] == inn[ci]
    # I4 placement, recomputed from the vertex string alone with the string brute force
    for v, e in list(d.items())[:3000]:
        assert e[3] == brute.partition(v, P, NP)


def test_invariant_I5_strand_symmetry(oracle_lib):
    rs = random_reads(100, 10, 90, seed=41)
    reads = rs.reads()
    a = oracle_lib.graph(rs.seq, rs.offsets, 15, 5, 9)
    rr = _readset([brute.rc(r) for r in reads])
    b = oracle_lib.graph(rr.seq, rr.offsets, 15, 5, 9)
    assert a.tobytes() == b.tobytes()


def test_invariant_I6_partition_independence(oracle_lib):
    rs = _tiny_erroneous().subset(0, 600)
    base = None
    for P in (1, 5, 11, 31):
        for NP in (1, 16, 512):
            r = oracle_lib.graph(rs.seq, rs.offsets, 31, P, NP, n_threads=2)
            key = b"".join(r[f].tobytes() for f in ("key_hi", "key_lo", "count", "out", "in"))
            base = base or key
            assert key == base


def test_read_permutation_and_union(oracle_lib):
    rs = random_reads(80, 5, 70, seed=51)
    reads = rs.reads()
    perm = np.random.default_rng(3).permutation(len(reads))
    rp = _readset([reads[i] for i in perm])
    a = oracle_lib.graph(rs.seq, rs.offsets, 9, 3, 5)
    b = oracle_lib.graph(rp.seq, rp.offsets, 9, 3, 5)
    assert a.tobytes() == b.tobytes()
    # additivity under read-set union
    h1, h2 = _readset(reads[:40]), _readset(reads[40:])
    d1 = _as_dict(oracle_lib.graph(h1.seq, h1.offsets, 9, 3, 5), 9)
    d2 = _as_dict(oracle_lib.graph(h2.seq, h2.offsets, 9, 3, 5), 9)
    da = _as_dict(a, 9)
    for v, e in da.items():
        e1 = d1.get(v, [0, [0] * 4, [0] * 4, e[3]])
        e2 = d2.get(v, [0, [0] * 4, [0] * 4, e[3]])
        assert e[0] == e1[0] + e2[0]
        assert e[1] == [x + y for x, y in zip(e1[1], e2[1])]
        assert e[2] == [x + y for x, y in zip(e1[2], e2[2])]


def test_special_case_P_equals_K(oracle_lib):
    """P = K (L1101-1103): every superkmer holds one K-mer on random reads."""
    rs = random_reads(50, 100, 100, seed=61)
    sk = oracle_lib.msp(rs.seq, rs.offsets, 31, 31, 8)
    assert len(sk) == 50 * 70 and set(sk["n_kmers"].tolist()) == {1}


def test_superkmers_cover_all_kmers(oracle_lib):
    rs = _tiny_erroneous().subset(0, 300)
    sk = oracle_lib.msp(rs.seq, rs.offsets, 31, 11, 16)
    assert int(sk["n_kmers"].sum()) == rs.n_kmers(31)
    # Def. 2 with reading G: consecutive superkmers of a read have different minimizers
    same_read = sk["read"][1:] == sk["read"][:-1]
    assert np.all(sk["minimizer"][1:][same_read] != sk["minimizer"][:-1][same_read])
    # average superkmer length near the SURVEY.md simulation (8.85 K-mers, K=31 P=11)
    assert 7.0 < rs.n_kmers(31) / len(sk) < 11.0


def test_edge_cases_short_reads(oracle_lib):
    """Reading N: L<K gives nothing, L=K one vertex without edges; empty input."""
    rs = _readset(["ACG", "ACGTA", "", "TTTTT"])
    d = _as_dict(oracle_lib.graph(rs.seq, rs.offsets, 5, 2, 3), 5)
    assert d["ACGTA"][:3] == [1, [0] * 4, [0] * 4]
    assert d["AAAAA"][:3] == [1, [0] * 4, [0] * 4]
    assert len(d) == 2
    empty = oracle_lib.graph(np.zeros(0, np.uint8), np.zeros(1, np.uint64), 5, 2, 3)
    assert len(empty) == 0


def test_unknown_bases_become_A(oracle_lib):
    """L205-206: unknown bases -> A; lower case as upper (reading B)."""
    a = _readset(["ACGNNTRYacgt"])
    b = _readset(["ACGAATAAACGT"])
    ga = oracle_lib.graph(a.seq, a.offsets, 5, 3, 4)
    gb = oracle_lib.graph(b.seq, b.offsets, 5, 3, 4)
    assert ga.tobytes() == gb.tobytes()


def test_checksum_order_independent(oracle_lib):
    rs = random_reads(50, 30, 60, seed=71)
    r = oracle_lib.graph(rs.seq, rs.offsets, 11, 5, 4)
    c = oracle_lib.checksum(r)
    assert c == oracle_lib.checksum(r[::-1].copy())
    r2 = r.copy()
    r2["out"][0, 0] += 1
    assert oracle_lib.checksum(r2) != c
    # fmix64 (reading I) agrees with the string-side twin; the partition function is a free
    # choice (reading I), so this is consistency, not a pin -- placement is pinned by I4.
    for x in (0, 1, 2, 0xDEADBEEF, (1 << 64) - 1):
        assert oracle_lib.fmix64(x) == brute.fmix64(x)
    assert brute.fmix64(0) == 0


def _murmur3_x64_128(data: bytes, seed: int, fmix, c1: int, c2: int) -> bytes:
    """MurmurHash3_x64_128 (Appleby, SMHasher) with its finaliser taken from the oracle: body
    blocks of 16 bytes, tail, length, then fmix64 of both halves.  Only fmix64 is the oracle's."""
    M = (1 << 64) - 1

    def rotl(x, r):
        return ((x << r) | (x >> (64 - r))) & M

    n, nb = len(data), len(data) // 16
    h1 = h2 = seed
    for i in range(nb):
        k1 = int.from_bytes(data[16 * i:16 * i + 8], "little")
        k2 = int.from_bytes(data[16 * i + 8:16 * i + 16], "little")
        k1 = (rotl((k1 * c1) & M, 31) * c2) & M
        h1 ^= k1
        h1 = (((rotl(h1, 27) + h2) & M) * 5 + 0x52DCE729) & M
        k2 = (rotl((k2 * c2) & M, 33) * c1) & M
        h2 ^= k2
        h2 = (((rotl(h2, 31) + h1) & M) * 5 + 0x38495AB5) & M
    tail = data[16 * nb:]
    if len(tail) > 8:
        h2 ^= (rotl((int.from_bytes(tail[8:], "little") * c2) & M, 33) * c1) & M
    if len(tail) > 0:
        h1 ^= (rotl((int.from_bytes(tail[:8], "little") * c1) & M, 31) * c2) & M
    h1 ^= n
    h2 ^= n
    h1 = (h1 + h2) & M
    h2 = (h2 + h1) & M
    h1, h2 = fmix(h1), fmix(h2)
    h1 = (h1 + h2) & M
    h2 = (h2 + h1) & M
    return h1.to_bytes(8, "little") + h2.to_bytes(8, "little")


def test_fmix64_pinned_by_murmurhash3_verification_value(oracle_lib):
    """Reading I: the partition hash is MurmurHash3's finaliser fmix64.  Pinned by SMHasher's
    published verification value of MurmurHash3_x64_128 (tests/golden/murmur3_verification.txt),
    computed here with the oracle's fmix64 as the finaliser."""
    g = dict(l.split() for l in open(os.path.join(GOLD, "murmur3_verification.txt")) if l.strip() and l[0] != "#")
    c1, c2 = int(g["C1"], 16), int(g["C2"], 16)
    key = bytearray(256)
    hashes = b""
    for i in range(256):
        key[i] = i
        hashes += _murmur3_x64_128(bytes(key[:i]), 256 - i, oracle_lib.fmix64, c1, c2)
    final = _murmur3_x64_128(hashes, 0, oracle_lib.fmix64, c1, c2)
    assert int.from_bytes(final[:4], "little") == int(g["VERIFICATION"], 16)
    assert oracle_lib.fmix64(0) == 0  # the fixed point the checksum closed form below relies on


def test_checksum_closed_form_pins_field_order(oracle_lib):
    """SURVEY.md 8(d) checksum: per record h = 0, then h = fmix64(h ^ field) over the 11 fields
    key_hi, key_lo, count, out[0..3], in[0..3]; the checksum is the sum of h mod 2^64.  Because
    fmix64(0) = 0 (pinned above), a record whose only nonzero field is field j (0-based) with
    value x has h = fmix64 applied 11 - j times to x -- so the position of every field, the number
    of fields and the exclusion of pid are fixed by iterating the pinned fmix64, not by the
    checksum code.  Two nonzero fields i < j combine as fmix^(11-j)(fmix^(j-i)(a) ^ b)."""

    def it(x, n):
        for _ in range(n):
            x = oracle_lib.fmix64(x)
        return x

    slots = [("key_hi", None), ("key_lo", None), ("count", None)] + [("out", c) for c in range(4)] + \
            [("in", c) for c in range(4)]

    def rec(vals):
        r = np.zeros(1, dtype=oracle_lib.VERTEX_DTYPE)
        for j, v in vals.items():
            name, c = slots[j]
            if c is None:
                r[name] = v
            else:
                r[name][0, c] = v
        return r

    assert oracle_lib.checksum(np.zeros(3, dtype=oracle_lib.VERTEX_DTYPE)) == 0
    for j in range(11):
        x = 0x1234 + 977 * j
        assert oracle_lib.checksum(rec({j: x})) == it(x, 11 - j), j
    M = (1 << 64) - 1
    for i, j in ((0, 1), (1, 2), (2, 6), (3, 7), (6, 10), (0, 10)):
        a, b = 0xABCDEF + i, 0x31337 + j
        assert oracle_lib.checksum(rec({i: a, j: b})) == it(it(a, j - i) ^ b, 11 - j), (i, j)
    r = rec({0: 5, 2: 7})
    r2 = r.copy()
    r2["pid"] = 12345
    assert oracle_lib.checksum(r2) == oracle_lib.checksum(r)          # pid is not a checksum field
    both = np.concatenate([rec({1: 9}), rec({4: 3})])
    assert oracle_lib.checksum(both) == (it(9, 10) + it(3, 7)) & M    # sum over records mod 2^64


def test_oracle_filters_equal_the_unfiltered_graph_restricted(oracle_lib):
    """The pid and key filters (sampled parity at full size) only drop occurrences: the filtered
    graph is exactly the unfiltered graph restricted to those partitions / vertices."""
    rs = random_reads(400, 20, 150, seed=91, n_rate=0.01)
    K, P, NP = 21, 7, 16
    full = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP, n_threads=3)
    for pids in ([], [0], [3, 7, 11], list(range(NP))):
        got = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP, n_threads=2, pids=pids)
        assert got.tobytes() == full[np.isin(full["pid"], pids)].tobytes(), pids
    rng = np.random.default_rng(5)
    pick = full[rng.choice(len(full), 50, replace=False)]
    keys = np.stack([pick["key_hi"], pick["key_lo"]], 1)
    absent = np.array([[0, (1 << 42) + 12345], [0, 7]], dtype=np.uint64)  # codes not in the graph
    absent = absent[~np.isin(absent[:, 1], full["key_lo"])]
    got = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP, keys=np.concatenate([keys, absent]))
    assert got.tobytes() == np.sort(pick, order=["key_hi", "key_lo"]).tobytes()
    both = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP, pids=[int(pick["pid"][0])], keys=keys)
    assert both.tobytes() == np.sort(pick[pick["pid"] == pick["pid"][0]], order=["key_hi", "key_lo"]).tobytes()


# ---------------------------------------------------------------- row f4: low-count filtering


def test_filter_low_count_keeps_genome_kmers(oracle_lib):
    """Row f4: "a single error ... generates ... K erroneous kmers ... these
    erroneous vertices can only be filtered by the number of their occurrences".  Error-free reads
    tile a random genome (every interior K-mer covered >= 3 times) and 40 reads carry one distinct
    substitution each.  Filtering at 2 must keep exactly the K-mers occurring >= 2 times by a
    string count (collections.Counter over canonical strings), which are genome K-mers only, with
    their records unchanged; every erroneous K-mer (not in the genome on either strand) is gone."""
    import collections

    rng = np.random.default_rng(11)
    K, P, NP, L = 21, 7, 8, 80
    g = "".join("ACGT"[x] for x in rng.integers(0, 4, 2000))
    reads = [g[s:s + L] for s in range(0, len(g) - L + 1, 20)]
    errs = []
    for j in range(40):
        s = 25 * j + 3
        r = list(g[s:s + L])
        q = 40 + (j % 7)
        r[q] = "ACGT"[("ACGT".index(r[q]) + 1 + j % 3) % 4]
        errs.append("".join(r))
    rs = _readset(reads + errs)
    recs = oracle_lib.graph(rs.seq, rs.offsets, K, P, NP)
    kept = oracle_lib.filter_low_count(recs, 2)
    cnt = collections.Counter(brute.canonical_string(r[i:i + K]) for r in reads + errs for i in range(len(r) - K + 1))
    want = {v for v, c in cnt.items() if c >= 2}
    got = _as_dict(kept, K)
    assert set(got) == want
    genome_kmers = {brute.canonical_string(g[i:i + K]) for i in range(len(g) - K + 1)}
    assert want <= genome_kmers
    erroneous = set(cnt) - genome_kmers
    assert len(erroneous) > 40 * (K - 5) and not (erroneous & set(got))
    full = _as_dict(recs, K)
    assert all(full[v] == e for v, e in got.items())  # kept records are not edited
    assert len(oracle_lib.filter_low_count(recs, 1)) == len(recs)
    assert len(oracle_lib.filter_low_count(recs, 0)) == len(recs)


# ---------------------------------------------------------------- row f3: K up to 127


def _wide_as_dict(recs, k):
    d = {}
    for r in recs:
        code = 0
        for w in r["key"]:
            code = (code << 64) | int(w)
        s = "".join("ACGT"[(code >> (2 * (k - 1 - t))) & 3] for t in range(k))
        d[s] = [int(r["count"]), [int(x) for x in r["out"]], [int(x) for x in r["in"]], int(r["pid"])]
    return d


@pytest.mark.parametrize("k,p,np_,seed", [(65, 21, 7, 1), (71, 13, 3, 2), (99, 31, 16, 3), (127, 19, 5, 4),
                                           (101, 1, 2, 5)])
def test_wide_oracle_vs_string_brute_force(oracle_lib, k, p, np_, seed):
    """Row f3 (Sec. III-C3 L569-615 needs K > 63 keys): the string-keyed oracle equals the pure-Python
    string brute force (oracle/brute.py) on ragged reads with N bases and repeats, codes included."""
    rng = np.random.default_rng(seed)
    base = "".join("ACGT"[x] for x in rng.integers(0, 4, 400))
    reads = []
    for _ in range(40):
        L = int(rng.integers(k - 3, k + 90))
        s0 = int(rng.integers(0, 400 - min(L, 399)))
        r = base[s0:s0 + L]
        if rng.random() < 0.5:
            r = brute.rc(r)
        r = "".join(c if rng.random() > 0.01 else "N" for c in r)
        reads.append(r)
    reads.append(base[:k])  # L = K: one K-mer, no edges (reading N)
    rs = _readset(reads)
    got = _wide_as_dict(oracle_lib.graph_wide(rs.seq, rs.offsets, k, p, np_), k)
    want = brute.graph(reads, k, p, np_)
    assert got == want
    recs = oracle_lib.graph_wide(rs.seq, rs.offsets, k, p, np_)
    keys = [tuple(int(x) for x in r["key"]) for r in recs]
    assert keys == sorted(keys)  # reading Q: ascending canonical code


def test_wide_oracle_equals_two_word_oracle(oracle_lib):
    """For K <= 63 the string-keyed oracle and the 128-bit-keyed oracle are the same graph."""
    rs = random_reads(300, 1, 200, seed=12, n_rate=0.01)
    for k, p, np_ in [(31, 11, 16), (63, 19, 8), (5, 3, 3)]:
        a = oracle_lib.graph(rs.seq, rs.offsets, k, p, np_)
        b = oracle_lib.graph_wide(rs.seq, rs.offsets, k, p, np_)
        assert len(a) == len(b)
        assert np.array_equal(b["key"][:, 0], np.zeros(len(b), dtype=np.uint64))
        assert np.array_equal(b["key"][:, 1], np.zeros(len(b), dtype=np.uint64))
        assert np.array_equal(b["key"][:, 2], a["key_hi"]) and np.array_equal(b["key"][:, 3], a["key_lo"])
        for f in ("count", "out", "in", "pid"):
            assert np.array_equal(a[f], b[f])
