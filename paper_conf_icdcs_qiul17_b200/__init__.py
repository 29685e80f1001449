"""B200-native hot path of ParaHash (Qiu & Luo, ICDCS 2017): MSP partitioning + per-partition
hash-table De Bruijn graph construction, behind the C ABI of include/dbg.h (libdbg.so, sm_100a).

The Python layer only marshals arguments and owns device memory (PyTorch); there is no CPU
fallback -- if libdbg.so is missing, calls raise.
"""
from . import _lib
from ._lib import VERTEX_DTYPE, DbgError, load
from .stream import StreamingBuilder, build_graph_streamed, plan_ranges
from .graph import (DbgBuilder, GraphResult, auto_fine_p, auto_refine, build_graph, encode_reads, launch_builder, read_graph,
                    write_graph)

__all__ = ["_lib", "VERTEX_DTYPE", "DbgError", "load", "DbgBuilder", "GraphResult", "auto_fine_p", "auto_refine",
           "build_graph", "encode_reads", "launch_builder", "read_graph", "write_graph",
           "StreamingBuilder", "build_graph_streamed", "plan_ranges"]
