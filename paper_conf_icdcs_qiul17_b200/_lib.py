"""ctypes binding of libdbg.so (include/dbg.h) -- argument marshalling only.

Every function here has the name of the C entry point it calls and only turns
torch tensors / numpy arrays into pointers; all work runs in libdbg.so.  The
library is loaded from this package's lib/ directory (built in-tree by
``paper_conf_icdcs_qiul17_b200.build``); if it is missing, loading fails
loudly -- there is no fallback path.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# DBG_LIB_PATH: an A/B kernel-variant build (tools/build_variants.py); default: the in-tree build
LIB_PATH = os.environ.get("DBG_LIB_PATH") or os.path.join(_PKG, "lib", "libdbg.so")

DBG_OK, DBG_EINVAL, DBG_ENOSPACE, DBG_ETABLEFULL, DBG_ECUDA = range(5)


class DbgError(RuntimeError):
    def __init__(self, name: str, status: int, msg: str):
        super().__init__(f"{name} failed: status {status} ({msg})")
        self.status = status


class dbg_params(ctypes.Structure):
    _fields_ = [("k", ctypes.c_int32), ("p", ctypes.c_int32), ("num_partitions", ctypes.c_int32),
                ("lambda_", ctypes.c_float), ("alpha", ctypes.c_float), ("refine", ctypes.c_int32),
                ("smem_split", ctypes.c_int32), ("fine_p", ctypes.c_int32), ("min_count", ctypes.c_uint32)]


class dbg_partition_set(ctypes.Structure):
    _fields_ = [("d_n_records", ctypes.c_void_p), ("d_n_kmers", ctypes.c_void_p),
                ("d_record_offset", ctypes.c_void_p), ("d_fill", ctypes.c_void_p),
                ("d_staged", ctypes.c_void_p), ("d_staging", ctypes.c_void_p),
                ("staging_cap", ctypes.c_uint64), ("d_records", ctypes.c_void_p),
                ("d_scratch", ctypes.c_void_p),
                ("d_peer_records", ctypes.c_void_p), ("d_peer_bounds", ctypes.c_void_p), ("n_peers", ctypes.c_int32),
                ("d_work", ctypes.c_void_p)]


# dbg_vertex (56 B) and dbg_stats (32 B) as numpy dtypes
VERTEX_DTYPE = np.dtype([("kmer_hi", "<u8"), ("kmer_lo", "<u8"), ("count", "<u4"),
                         ("out", "<u4", (4,)), ("in", "<u4", (4,)), ("pid", "<u4")])
# row f3 (K > 63): dbg_vertex_wide, four key words most significant first (72 B)
VERTEX_WIDE_DTYPE = np.dtype([("kmer", "<u8", (4,)), ("count", "<u4"), ("out", "<u4", (4,)), ("in", "<u4", (4,)),
                              ("pid", "<u4")])
assert VERTEX_WIDE_DTYPE.itemsize == 72
STATS_FIELDS = ("distinct", "sum_count", "sum_edges", "checksum")
assert VERTEX_DTYPE.itemsize == 56

_P = ctypes.c_void_p
_U64 = ctypes.c_uint64
_I32 = ctypes.c_int32
_PRM = ctypes.POINTER(dbg_params)
_PART = ctypes.POINTER(dbg_partition_set)

# name -> (restype, argtypes); mirrors include/dbg.h
SIGNATURES = {
    "dbg_abi_version": (ctypes.c_int, []),
    "dbg_record_words": (ctypes.c_uint32, [_PRM]),
    "dbg_record_max_kmers": (ctypes.c_uint32, [_PRM]),
    "dbg_scatter_work_words": (ctypes.c_uint64, [_PRM]),
    "dbg_slot_bytes": (ctypes.c_uint32, [_PRM]),
    "dbg_key_bytes": (ctypes.c_uint32, [_PRM]),
    "dbg_table_capacity": (_U64, [_PRM, _U64]),
    "dbg_table_bytes": (_U64, [_PRM, _U64]),
    "dbg_exchange_plan": (ctypes.c_int, [_PRM, _P, _P, _I32, _I32, _P, _P, _P, _P, _P, _P, _P, _P]),
    "dbg_enable_peer_access": (ctypes.c_int, [_I32]),
    "dbg_packed_words": (_U64, [_U64]),
    "dbg_encode_ascii": (ctypes.c_int, [_P, _U64, _P]),
    "dbg_msp_partition": (ctypes.c_int, [_PRM, _P, _U64, _P, _U64, _PART, _P]),
    "dbg_msp_partition_range": (ctypes.c_int, [_PRM, _P, _U64, _P, _U64, _PART, _I32, _I32, ctypes.c_int, _P]),
    "dbg_table_plan": (ctypes.c_int, [_PRM, _P, _P, _P, _P]),
    "dbg_smem_table_slots": (_U64, [_PRM]),
    "dbg_smem_onchip": (ctypes.c_int32, [_PRM, _U64]),
    "dbg_smem_workspace_bytes": (_U64, [_PRM]),
    "dbg_build_subgraphs_smem": (ctypes.c_int, [_PRM, _PART, _I32, _I32, _P, _U64, _P, _U64, _P, _P, _P, _P]),
    "dbg_table_plan_split": (ctypes.c_int, [_PRM, _P, _P, _P, _P]),
    "dbg_hash_build": (ctypes.c_int, [_PRM, _PART, _I32, _I32, _P, _P, _P, _P]),
    "dbg_hash_build_list": (ctypes.c_int, [_PRM, _PART, _I32, _I32, _P, _P, _I32, _P, _P, _P, _P]),
    "dbg_extract_graph": (ctypes.c_int, [_PRM, _P, _P, _I32, _I32, _P, _U64, _P, _P, _P, _P]),
    "dbg_sort_workspace_bytes": (_U64, [_PRM, _U64]),
    "dbg_sort_vertices": (ctypes.c_int, [_PRM, _P, _P, _U64, _P, _U64, _P]),
    "dbg_checksum_vertices": (ctypes.c_int, [_PRM, _P, _U64, _P, _P]),
    "dbg_write_graph": (ctypes.c_int, [ctypes.c_char_p, _PRM, _P, _U64, ctypes.c_int]),
    "dbg_sync_status": (ctypes.c_int, [_P, _P]),
    "dbg_status_string": (ctypes.c_char_p, [ctypes.c_int]),
}

_lib = None
ABI_VERSION = 12


def load():
    """Loads libdbg.so; raises if it has not been built."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_icdcs_qiul17_b200.build` "
                              "(there is no CPU fallback)")
        lib = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        if lib.dbg_abi_version() != ABI_VERSION:
            raise ImportError("libdbg.so ABI version mismatch")
        _lib = lib
    return _lib


def _ptr(x) -> int | None:
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    raise TypeError(type(x))


def _check(name: str, status: int):
    if status != DBG_OK:
        raise DbgError(name, status, load().dbg_status_string(status).decode())


def _stream(stream) -> int | None:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def params(k: int, p: int, num_partitions: int, lam: float = 2.0, alpha: float = 0.5,
           refine: int = 1, smem_split: int = 0, fine_p: int = 0, min_count: int = 0) -> dbg_params:
    return dbg_params(k, p, num_partitions, lam, alpha, refine, smem_split, fine_p, min_count)


def fine_partitions(prm: dbg_params) -> int:
    return prm.num_partitions * max(1, prm.refine)


def partition_set(n_records, n_kmers, record_offset, fill, staged, staging=None, staging_cap: int = 0,
                  records=None, scratch=None, peer_records=None, peer_bounds=None,
                  n_peers: int = 0, work=None) -> dbg_partition_set:
    return dbg_partition_set(_ptr(n_records), _ptr(n_kmers), _ptr(record_offset), _ptr(fill), _ptr(staged),
                             _ptr(staging), staging_cap, _ptr(records), _ptr(scratch),
                             _ptr(peer_records), _ptr(peer_bounds), n_peers, _ptr(work))


# --------------------------------------------------------------------------- entry points


def dbg_abi_version() -> int:
    return load().dbg_abi_version()


def dbg_record_words(prm: dbg_params) -> int:
    return load().dbg_record_words(ctypes.byref(prm))


def dbg_record_max_kmers(prm: dbg_params) -> int:
    return load().dbg_record_max_kmers(ctypes.byref(prm))


def dbg_scatter_work_words(prm: dbg_params) -> int:
    return load().dbg_scatter_work_words(ctypes.byref(prm))


def dbg_slot_bytes(prm: dbg_params) -> int:
    return load().dbg_slot_bytes(ctypes.byref(prm))


def dbg_key_bytes(prm: dbg_params) -> int:
    return load().dbg_key_bytes(ctypes.byref(prm))


def dbg_table_capacity(prm: dbg_params, n_kmers: int) -> int:
    return load().dbg_table_capacity(ctypes.byref(prm), n_kmers)


def dbg_table_bytes(prm: dbg_params, n_kmers: int) -> int:
    return load().dbg_table_bytes(ctypes.byref(prm), n_kmers)


def dbg_exchange_plan(prm, d_counts, d_kmers_sum, world: int, rank: int, d_bounds, d_dest_offset, d_owned_n_records,
                      d_owned_n_kmers, d_owned_record_offset, d_prefix, d_scratch, stream=None) -> None:
    _check("dbg_exchange_plan", load().dbg_exchange_plan(
        ctypes.byref(prm), _ptr(d_counts), _ptr(d_kmers_sum), world, rank, _ptr(d_bounds), _ptr(d_dest_offset),
        _ptr(d_owned_n_records), _ptr(d_owned_n_kmers), _ptr(d_owned_record_offset), _ptr(d_prefix),
        _ptr(d_scratch), _stream(stream)))


def dbg_enable_peer_access(peer_device: int) -> None:
    _check("dbg_enable_peer_access", load().dbg_enable_peer_access(peer_device))


def dbg_packed_words(n_bases: int) -> int:
    return load().dbg_packed_words(n_bases)


def dbg_encode_ascii(seq, h_words) -> None:
    """seq: uint8 ASCII array (numpy or CPU tensor); h_words: uint64 host buffer of
    dbg_packed_words(len(seq)) words (numpy or pinned CPU tensor)."""
    n = seq.numel() if hasattr(seq, "numel") else len(seq)
    _check("dbg_encode_ascii", load().dbg_encode_ascii(_ptr(seq), n, _ptr(h_words)))


def dbg_msp_partition(prm, d_bases, n_words: int, d_offsets, n_reads: int, part: dbg_partition_set,
                      stream=None) -> None:
    _check("dbg_msp_partition", load().dbg_msp_partition(
        ctypes.byref(prm), _ptr(d_bases), n_words, _ptr(d_offsets), n_reads, ctypes.byref(part),
        _stream(stream)))


def dbg_msp_partition_range(prm, d_bases, n_words: int, d_offsets, n_reads: int, part: dbg_partition_set,
                            pid_lo: int, pid_hi: int, append: bool, stream=None) -> None:
    _check("dbg_msp_partition_range", load().dbg_msp_partition_range(
        ctypes.byref(prm), _ptr(d_bases), n_words, _ptr(d_offsets), n_reads, ctypes.byref(part), pid_lo, pid_hi,
        int(bool(append)), _stream(stream)))


def dbg_table_plan(prm, d_n_kmers, d_table_offset, d_scratch=None, stream=None) -> None:
    _check("dbg_table_plan", load().dbg_table_plan(ctypes.byref(prm), _ptr(d_n_kmers),
                                                   _ptr(d_table_offset), _ptr(d_scratch), _stream(stream)))


def dbg_smem_table_slots(prm) -> int:
    return load().dbg_smem_table_slots(ctypes.byref(prm))


def dbg_smem_onchip(prm, n_kmers: int) -> int:
    return load().dbg_smem_onchip(ctypes.byref(prm), n_kmers)


def dbg_smem_workspace_bytes(prm) -> int:
    return load().dbg_smem_workspace_bytes(ctypes.byref(prm))


def dbg_build_subgraphs_smem(prm, part, pid_begin: int, pid_end: int, d_work, work_bytes: int, d_out, out_cap: int,
                             d_n_out, d_stats, d_status, stream=None) -> None:
    _check("dbg_build_subgraphs_smem", load().dbg_build_subgraphs_smem(
        ctypes.byref(prm), ctypes.byref(part), pid_begin, pid_end, _ptr(d_work), work_bytes, _ptr(d_out), out_cap,
        _ptr(d_n_out), _ptr(d_stats), _ptr(d_status), _stream(stream)))


def dbg_table_plan_split(prm, d_n_kmers, d_table_offset, d_scratch=None, stream=None) -> None:
    _check("dbg_table_plan_split", load().dbg_table_plan_split(ctypes.byref(prm), _ptr(d_n_kmers),
                                                               _ptr(d_table_offset), _ptr(d_scratch),
                                                               _stream(stream)))


def dbg_hash_build(prm, part, pid_begin: int, pid_end: int, d_table, d_table_offset, d_status,
                   stream=None) -> None:
    _check("dbg_hash_build", load().dbg_hash_build(
        ctypes.byref(prm), ctypes.byref(part), pid_begin, pid_end, _ptr(d_table), _ptr(d_table_offset),
        _ptr(d_status), _stream(stream)))


def dbg_hash_build_list(prm, part, pid_begin: int, pid_end: int, d_pids, d_chunk_prefix, n_pids: int, d_table,
                        d_table_offset, d_status, stream=None) -> None:
    _check("dbg_hash_build_list", load().dbg_hash_build_list(
        ctypes.byref(prm), ctypes.byref(part), pid_begin, pid_end, _ptr(d_pids), _ptr(d_chunk_prefix), n_pids,
        _ptr(d_table), _ptr(d_table_offset), _ptr(d_status), _stream(stream)))


def dbg_extract_graph(prm, d_table, d_table_offset, pid_begin: int, pid_end: int, d_out, out_cap: int, d_n_out,
                      d_stats, d_status, stream=None) -> None:
    _check("dbg_extract_graph", load().dbg_extract_graph(
        ctypes.byref(prm), _ptr(d_table), _ptr(d_table_offset), pid_begin, pid_end, _ptr(d_out), out_cap,
        _ptr(d_n_out), _ptr(d_stats), _ptr(d_status), _stream(stream)))


def dbg_sort_workspace_bytes(prm, n: int) -> int:
    return load().dbg_sort_workspace_bytes(ctypes.byref(prm), n)


def dbg_sort_vertices(prm, d_in, d_out, n: int, d_workspace, workspace_bytes: int, stream=None) -> None:
    _check("dbg_sort_vertices", load().dbg_sort_vertices(
        ctypes.byref(prm), _ptr(d_in), _ptr(d_out), n, _ptr(d_workspace), workspace_bytes,
        _stream(stream)))


def dbg_checksum_vertices(prm, d_vertices, n: int, d_stats, stream=None) -> None:
    _check("dbg_checksum_vertices", load().dbg_checksum_vertices(ctypes.byref(prm), _ptr(d_vertices), n,
                                                                 _ptr(d_stats), _stream(stream)))


def dbg_write_graph(path: str, prm, h_vertices, n: int, append: bool = False) -> None:
    _check("dbg_write_graph", load().dbg_write_graph(os.fsencode(path), ctypes.byref(prm), _ptr(h_vertices), n,
                                                     int(bool(append))))


def dbg_sync_status(d_status, stream=None) -> int:
    return load().dbg_sync_status(_ptr(d_status), _stream(stream))


def dbg_status_string(status: int) -> str:
    return load().dbg_status_string(status).decode()
