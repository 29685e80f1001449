"""CPU oracle for ParaHash's De Bruijn graph construction -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  The product package
``paper_conf_icdcs_qiul17_b200`` never imports it, and it never imports the
product package: the two share no code ("Oracle").

Contents
  dbg_oracle.cpp  plain C++ std::map oracle of Definition 3,
                  loaded here through ctypes (``graph``, ``msp``, ``checksum``).
  brute.py        pure-Python string brute force for tiny inputs (a pin for the
                  C++ oracle, not a second implementation used by the product).

Pins: tests/test_oracle_pins.py.  Parity: unpinned parts are listed in
DESIGN.md "Parity pins" (none for the functions exported here).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dbg_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

VERTEX_DTYPE = np.dtype(
    [
        ("key_hi", "<u8"),
        ("key_lo", "<u8"),
        ("count", "<u4"),
        ("out", "<u4", (4,)),
        ("in", "<u4", (4,)),
        ("pid", "<u4"),
    ]
)
assert VERTEX_DTYPE.itemsize == 56

# Row f3 (K <= 127): four key words, most significant first
VERTEX_WIDE_DTYPE = np.dtype([("key", "<u8", (4,)), ("count", "<u4"), ("out", "<u4", (4,)), ("in", "<u4", (4,)),
                              ("pid", "<u4")])
assert VERTEX_WIDE_DTYPE.itemsize == 72

SUPERKMER_DTYPE = np.dtype(
    [
        ("read", "<u8"),
        ("minimizer", "<u8"),
        ("start", "<u4"),
        ("n_kmers", "<u4"),
        ("pid", "<u4"),
        ("has_left", "<u4"),
        ("has_right", "<u4"),
        ("pad", "<u4"),
    ]
)
assert SUPERKMER_DTYPE.itemsize == 40


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", tmp, _SRC]
        )
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        u64p = ctypes.POINTER(ctypes.c_uint64)
        lib.oracle_graph.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
            ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_void_p), u64p,
        ]
        lib.oracle_graph.restype = ctypes.c_int
        lib.oracle_graph_filtered.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
            ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
            ctypes.POINTER(ctypes.c_void_p), u64p,
        ]
        lib.oracle_graph_filtered.restype = ctypes.c_int
        lib.oracle_msp.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
            ctypes.c_int, ctypes.POINTER(ctypes.c_void_p), u64p,
        ]
        lib.oracle_msp.restype = ctypes.c_int
        lib.oracle_checksum.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
        lib.oracle_checksum.restype = ctypes.c_uint64
        lib.oracle_fmix64.argtypes = [ctypes.c_uint64]
        lib.oracle_fmix64.restype = ctypes.c_uint64
        lib.oracle_canonical.argtypes = [ctypes.c_char_p, ctypes.c_int, u64p, u64p]
        lib.oracle_canonical.restype = None
        lib.oracle_kmer_minimizer.argtypes = [ctypes.c_char_p, ctypes.c_int, ctypes.c_int]
        lib.oracle_kmer_minimizer.restype = ctypes.c_uint64
        lib.oracle_graph_wide.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
                                          ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_void_p), u64p]
        lib.oracle_graph_wide.restype = ctypes.c_int
        lib.oracle_free.argtypes = [ctypes.c_void_p]
        lib.oracle_free.restype = None
        _lib = lib
    return _lib


def _as_inputs(seq, offsets):
    seq = np.ascontiguousarray(seq, dtype=np.uint8)
    offsets = np.ascontiguousarray(offsets, dtype=np.uint64)
    return seq, offsets


def graph(seq, offsets, k: int, p: int, num_partitions: int, n_threads: int = 1, pids=None,
          keys=None):
    """Sorted vertex records (VERTEX_DTYPE) of the reads ``seq[offsets[r]:offsets[r+1]]``.

    ``pids``: optional iterable of partition ids to keep; ``keys``: optional
    (hi, lo) uint64 pairs of canonical codes to keep (sampled parity at full size).
    """
    lib = _load()
    seq, offsets = _as_inputs(seq, offsets)
    n_reads = len(offsets) - 1
    filt = None
    if pids is not None:
        filt = np.zeros(num_partitions, dtype=np.uint8)
        filt[np.asarray(list(pids), dtype=np.int64)] = 1
    kf = None
    if keys is not None:
        kf = np.ascontiguousarray(np.asarray(keys, dtype=np.uint64).reshape(-1, 2))
        order = np.lexsort((kf[:, 1], kf[:, 0]))
        kf = np.ascontiguousarray(kf[order])
    out = ctypes.c_void_p()
    n = ctypes.c_uint64()
    rc = lib.oracle_graph_filtered(
        seq.ctypes.data if seq.size else None, offsets.ctypes.data, n_reads, k, p,
        num_partitions, n_threads, filt.ctypes.data if filt is not None else None,
        kf.ctypes.data if kf is not None else None, 0 if kf is None else len(kf),
        ctypes.byref(out), ctypes.byref(n),
    )
    if rc != 0:
        raise RuntimeError(f"oracle_graph failed with code {rc}")
    try:
        buf = (ctypes.c_char * (n.value * VERTEX_DTYPE.itemsize)).from_address(out.value)
        arr = np.frombuffer(buf, dtype=VERTEX_DTYPE).copy()
    finally:
        lib.oracle_free(out)
    return arr


def msp(seq, offsets, k: int, p: int, num_partitions: int):
    """Superkmers (SUPERKMER_DTYPE) in read order (Def. 2 + Sec. III-B)."""
    lib = _load()
    seq, offsets = _as_inputs(seq, offsets)
    out = ctypes.c_void_p()
    n = ctypes.c_uint64()
    rc = lib.oracle_msp(
        seq.ctypes.data if seq.size else None, offsets.ctypes.data, len(offsets) - 1, k, p,
        num_partitions, ctypes.byref(out), ctypes.byref(n),
    )
    if rc != 0:
        raise RuntimeError(f"oracle_msp failed with code {rc}")
    try:
        buf = (ctypes.c_char * (n.value * SUPERKMER_DTYPE.itemsize)).from_address(out.value)
        arr = np.frombuffer(buf, dtype=SUPERKMER_DTYPE).copy()
    finally:
        lib.oracle_free(out)
    return arr


def checksum(records) -> int:
    """Order-independent 64-bit checksum of VERTEX_DTYPE records."""
    lib = _load()
    rec = np.ascontiguousarray(records, dtype=VERTEX_DTYPE)
    return int(lib.oracle_checksum(rec.ctypes.data if rec.size else None, len(rec)))


def fmix64(x: int) -> int:
    return int(_load().oracle_fmix64(x))


def canonical(kmer: str):
    hi, lo = ctypes.c_uint64(), ctypes.c_uint64()
    _load().oracle_canonical(kmer.encode(), len(kmer), ctypes.byref(hi), ctypes.byref(lo))
    return (hi.value << 64) | lo.value


def kmer_minimizer(kmer: str, p: int) -> int:
    return int(_load().oracle_kmer_minimizer(kmer.encode(), len(kmer), p))


def filter_low_count(records, min_count: int):
    """Row f4 (Sec. III-C1: "these erroneous vertices can only be filtered by
    the number of their occurrences after the graph is constructed"): the records whose vertex
    count is at least ``min_count``, unchanged and in the same order (reading R: the
    edge multiplicities of a kept vertex are not edited).  ``min_count`` <= 1 keeps every record."""
    rec = np.asarray(records, dtype=VERTEX_DTYPE)
    if min_count <= 1:
        return rec.copy()
    return rec[rec["count"] >= min_count].copy()


def graph_wide(seq, offsets, k: int, p: int, num_partitions: int):
    """Row f3: sorted vertex records (VERTEX_WIDE_DTYPE) for K up to 127 -- the definition with the
    canonical K-mer held as a string (oracle_graph_wide), single-threaded."""
    lib = _load()
    seq, offsets = _as_inputs(seq, offsets)
    out = ctypes.c_void_p()
    n = ctypes.c_uint64()
    rc = lib.oracle_graph_wide(seq.ctypes.data if seq.size else None, offsets.ctypes.data, len(offsets) - 1, k, p,
                               num_partitions, ctypes.byref(out), ctypes.byref(n))
    if rc != 0:
        raise RuntimeError(f"oracle_graph_wide failed with code {rc}")
    try:
        buf = (ctypes.c_char * (n.value * VERTEX_WIDE_DTYPE.itemsize)).from_address(out.value)
        arr = np.frombuffer(buf, dtype=VERTEX_WIDE_DTYPE).copy()
    finally:
        lib.oracle_free(out)
    return arr
