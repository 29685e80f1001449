"""Row f2 (Sec. III-E): the overlapped ingest pipeline -- read batches streamed
H2D per partition range, Step 1 appended per batch, Step 2 per range, output D2H overlapped --
gives the oracle's graph bit-exact, whatever the batch size, range count and residency."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import build as _build, build_graph_streamed  # noqa: E402
from synth import ReadSet, genome, make_reads, random_reads  # noqa: E402

from gpu_helpers import compare_vertices  # noqa: E402

NT = os.cpu_count() or 1
_build.build()


@pytest.mark.parametrize("k,p,np_,batch_reads,budget,resident", [
    (31, 11, 16, 700, 3000, False),    # several batches and several ranges
    (31, 11, 16, 700, 3000, True),     # read batches resident in HBM, ranges only
    (63, 19, 8, 1000, 2500, False),    # two-word keys
    (31, 11, 4, 100000, 1 << 30, False),  # one batch, one range (degenerate pipeline)
    (21, 9, 32, 333, 1, False),        # budget below one partition: a range per partition
])
def test_streamed_equals_oracle(k, p, np_, batch_reads, budget, resident):
    g = genome(40_000, seed=31)
    seq, offs = make_reads(g, 4000, 100, 0.01, seed=32)
    rs = ReadSet(seq, offs)
    res = build_graph_streamed(rs.seq, rs.offsets, k, p, np_, batch_reads=batch_reads,
                               staging_budget_records=budget, resident=resident)
    orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=NT)
    compare_vertices(res.vertices, orc)
    assert res.stats["distinct"] == len(orc)
    assert res.stats["sum_count"] == int(orc["count"].sum()) == res.n_kmers
    assert res.batches == (len(rs.offsets) - 2) // batch_reads + 1
    if budget < 1 << 20:
        assert len(res.ranges) > 1
    # every read batch crossed the bus once per range plus once for the sizing pass (resident: once)
    packed = 8 * sum((int(rs.offsets[min(r + batch_reads, len(rs.offsets) - 1)] - rs.offsets[r]) + 31) // 32 + 1
                     + min(batch_reads, len(rs.offsets) - 1 - r) + 1
                     for r in range(0, len(rs.offsets) - 1, batch_reads))
    assert res.h2d_bytes == packed * (1 if resident else len(res.ranges) + 1)


def test_streamed_ragged_reads_and_filter():
    rs = random_reads(3000, 1, 260, seed=41, n_rate=0.01)
    res = build_graph_streamed(rs.seq, rs.offsets, 31, 11, 7, batch_reads=257, staging_budget_records=700,
                               min_count=2)
    orc = oracle.filter_low_count(oracle.graph(rs.seq, rs.offsets, 31, 11, 7, n_threads=NT), 2)
    compare_vertices(res.vertices, orc)
