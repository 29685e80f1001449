"""Synthetic genomes and reads shaped like the paper's datasets (Table I).

Recipe:
  * genome: i.i.d. uniform A/C/G/T of length G (optional repeat-family knob);
  * reads: fixed length L, start uniform in [0, G-L], reverse-complemented
    with probability 1/2 (both strands are sequenced);
  * substitution errors: each base independently with probability e,
    replaced uniformly by one of the 3 other bases (Property 1's independent
    error model, L540-547);
  * optional N bases (rate n_rate) to exercise the "unknown -> A" rule (L205-206).

Generation is chunked (2**20 reads per chunk, each chunk seeded by
SeedSequence([seed, chunk])) so results do not depend on memory limits.
Output is ASCII bytes + uint64 read offsets; no encoding happens here.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

_ALPHA = np.frombuffer(b"ACGT", dtype=np.uint8)
_COMP = np.zeros(256, dtype=np.uint8)
for _a, _b in zip(b"ACGTN", b"TGCAN"):
    _COMP[_a] = _b
CHUNK = 1 << 20


@dataclass
class ReadSet:
    seq: np.ndarray          # uint8 ASCII, all reads concatenated
    offsets: np.ndarray      # uint64 [n_reads + 1], in bases
    name: str = "custom"
    k: int = 31
    p: int = 11
    num_partitions: int = 16
    meta: dict = field(default_factory=dict)

    @property
    def n_reads(self) -> int:
        return len(self.offsets) - 1

    @property
    def n_bases(self) -> int:
        return int(self.offsets[-1])

    def lengths(self) -> np.ndarray:
        return np.diff(self.offsets.astype(np.int64))

    def n_kmers(self, k: int | None = None) -> int:
        k = self.k if k is None else k
        return int(np.maximum(self.lengths() - k + 1, 0).sum())

    def reads(self):
        """Python strings (tiny inputs only)."""
        b = self.seq.tobytes()
        o = self.offsets
        return [b[o[i]:o[i + 1]].decode() for i in range(self.n_reads)]

    def subset(self, r0: int, r1: int) -> "ReadSet":
        o = self.offsets[r0:r1 + 1]
        return ReadSet(self.seq[o[0]:o[-1]].copy(), (o - o[0]).astype(np.uint64), self.name,
                       self.k, self.p, self.num_partitions, dict(self.meta))


def genome(length: int, seed: int, repeat_families: int = 0, repeat_len: int = 300,
           repeat_frac: float = 0.0, repeat_div: float = 0.10) -> np.ndarray:
    """i.i.d. uniform genome; optionally overwrite repeat_frac of it with diverged repeat copies."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0xB200])))
    g = _ALPHA[rng.integers(0, 4, size=length, dtype=np.uint8)]
    if repeat_families and repeat_frac > 0:
        fams = _ALPHA[rng.integers(0, 4, size=(repeat_families, repeat_len), dtype=np.uint8)]
        n_copies = int(length * repeat_frac) // repeat_len
        for _ in range(n_copies):
            f = fams[rng.integers(0, repeat_families)].copy()
            mut = rng.random(repeat_len) < repeat_div
            f[mut] = _ALPHA[rng.integers(0, 4, size=int(mut.sum()), dtype=np.uint8)]
            at = int(rng.integers(0, length - repeat_len))
            g[at:at + repeat_len] = f
    return g


def make_reads(g: np.ndarray, n_reads: int, read_len: int, error_rate: float, seed: int,
               both_strands: bool = True, n_rate: float = 0.0,
               read_range: tuple[int, int] | None = None) -> tuple[np.ndarray, np.ndarray]:
    """Reads [r0, r1) of the n_reads-read set (default: all of them).  Chunks are seeded by their
    index, so a read range is the same reads whether it is drawn alone or as part of the set
    (multi-GPU strong scaling: each rank draws only its own range)."""
    G = len(g)
    assert G >= read_len
    r0, r1 = read_range if read_range is not None else (0, n_reads)
    assert 0 <= r0 <= r1 <= n_reads
    seq = np.empty((r1 - r0) * read_len, dtype=np.uint8)
    cols = np.arange(read_len, dtype=np.int64)
    for c0 in range((r0 // CHUNK) * CHUNK, r1, CHUNK):
        c1 = min(n_reads, c0 + CHUNK)
        n = c1 - c0
        rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, c0 // CHUNK])))
        start = rng.integers(0, G - read_len + 1, size=n, dtype=np.int64)
        r = g[start[:, None] + cols[None, :]]
        if both_strands:
            flip = rng.random(n) < 0.5
            r[flip] = _COMP[r[flip][:, ::-1]]
        if error_rate > 0:
            err = rng.random((n, read_len)) < error_rate
            ne = int(err.sum())
            if ne:
                cur = r[err]
                # uniform over the 3 other bases
                idx = np.searchsorted(_ALPHA, cur)
                shift = rng.integers(1, 4, size=ne, dtype=np.int64)
                r[err] = _ALPHA[(idx + shift) % 4]
        if n_rate > 0:
            nm = rng.random((n, read_len)) < n_rate
            r[nm] = ord("N")
        a, z = max(c0, r0), min(c1, r1)
        seq[(a - r0) * read_len:(z - r0) * read_len] = r[a - c0:z - c0].reshape(-1)
    offsets = np.arange(r1 - r0 + 1, dtype=np.uint64) * np.uint64(read_len)
    return seq, offsets


def random_reads(n_reads: int, min_len: int, max_len: int, seed: int, n_rate: float = 0.0,
                 lower_rate: float = 0.0, alphabet: bytes = b"ACGT") -> ReadSet:
    """Ragged i.i.d. reads (edge-case tests): lengths uniform in [min_len, max_len]."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x5EED])))
    lens = rng.integers(min_len, max_len + 1, size=n_reads, dtype=np.int64)
    offsets = np.zeros(n_reads + 1, dtype=np.uint64)
    offsets[1:] = np.cumsum(lens).astype(np.uint64)
    total = int(offsets[-1])
    alpha = np.frombuffer(alphabet, dtype=np.uint8)
    seq = alpha[rng.integers(0, len(alpha), size=total)]
    if n_rate > 0:
        seq[rng.random(total) < n_rate] = ord("N")
    if lower_rate > 0:
        low = rng.random(total) < lower_rate
        seq[low] = seq[low] + 32  # ASCII lower case
    return ReadSet(seq, offsets, name="random")


# name: (genome bp, reads, read length, error rate, K, P, NP, genome seed, read seed)
CONFIGS = {
    "tiny": dict(genome=50_000, reads=5_000, read_len=100, error=0.0, k=31, p=11, np=16,
                 gseed=1, rseed=101,
                 desc="tiny synthetic genome 50 kbp, 100 bp error-free reads at 10x, K=31, p=11, "
                      "16 MSP partitions"),
    "ecoli": dict(genome=4_600_000, reads=2_760_000, read_len=100, error=0.01, k=31, p=11, np=2048,
                  gseed=2, rseed=102,
                  desc="E. coli-shaped synthetic: 4.6 Mbp genome, 100 bp reads at 60x with 1% "
                       "substitution errors, K=31"),
    "chr14": dict(genome=88_000_000, reads=37_000_000, read_len=101, error=0.005, k=31, p=11,
                  np=512, gseed=3, rseed=103,
                  desc="human chr14-shaped synthetic (GAGE-like): 88 Mbp genome, 101 bp reads at "
                       "~40x, K=31, 512 partitions"),
    "bumblebee": dict(genome=250_000_000, reads=80_645_161, read_len=124, error=0.006, k=63,
                      p=19, np=512, gseed=4, rseed=104,
                      desc="bumblebee-shaped synthetic: ~250 Mbp genome, 124 bp reads at ~40x, "
                           "K=63 (two-word keys)"),
    "human": dict(genome=3_100_000_000, reads=930_000_000, read_len=100, error=0.005, k=31,
                  p=11, np=960, gseed=5, rseed=105,
                  desc="whole-human-shaped synthetic: 3.1 Gbp genome, 100 bp reads at 30x, K=31"),
}


def make_config(name: str, scale: float = 1.0, num_partitions: int | None = None,
                read_seed_offset: int = 0, shard: tuple[int, int] | None = None) -> ReadSet:
    """The named configuration; ``scale`` < 1 shrinks genome and read count together
    (same coverage, error rate and read length) for quick runs; ``read_seed_offset`` draws a
    different read set from the same genome; ``shard`` = (rank, world) draws only the contiguous
    read range [rank N / world, (rank+1) N / world) of the configuration (multi-GPU strong
    scaling: the ranks' ranges together are exactly the configuration's reads)."""
    c = CONFIGS[name]
    G = max(int(c["genome"] * scale), c["read_len"] * 4)
    n = max(int(c["reads"] * scale), 1)
    rng_ = None
    if shard is not None:
        r, w = shard
        rng_ = (n * r // w, n * (r + 1) // w)
    g = genome(G, c["gseed"])
    seq, offsets = make_reads(g, n, c["read_len"], c["error"], c["rseed"] + read_seed_offset, read_range=rng_)
    return ReadSet(seq, offsets, name=name, k=c["k"], p=c["p"],
                   num_partitions=num_partitions or c["np"],
                   meta=dict(genome=G, reads=n, read_len=c["read_len"], error=c["error"],
                             scale=scale, desc=c["desc"], read_range=rng_ or (0, n)))
