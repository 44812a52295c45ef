"""Online trace mode ("SASSI traces driving other tools"): an
instrumented kernel traced one block-range segment at a time into a two-slot ring, each segment
folded by sassi_consume on a second stream while the next is traced. Every table is an
order-independent fold, so the result must equal the oracle on the whole-kernel trace bit for bit
(record diagnostics included), for any segment size, overlapped or serial."""
import numpy as np
import pytest

import oracle
from gpu_helpers import diff_tables
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

# sizes with several thread blocks (vecadd 2^20: 1,184 blocks; the others 16 blocks)
SIZES = {"vecadd": 1 << 20, "bfs": 4096, "sgemm": 64, "stencil": 64}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def whole_trace_oracle(ik, mask):
    ctx = ik.context(mask)
    rec = ik.trace(ctx)
    ctx.close()
    h = gen.to_host(rec)
    return rec, oracle.run(h["sites"], ik.n_warps, mask, h["hdr"], h["addr"], h["val"])


@pytest.mark.parametrize("name", list(SIZES))
@pytest.mark.parametrize("bps,serial", [(1, False), (3, False), (0, False), (5, True)])
def test_online_fold_equals_oracle_on_whole_trace(name, bps, serial):
    ik = sassi.InstrumentedKernel(name, SIZES[name])
    mask = sassi.SASSI_H_EVERY
    rec, t_or = whole_trace_oracle(ik, mask)
    ctx = ik.context(mask)
    st = ik.trace_fold(ctx, blocks_per_segment=bps, serial=serial)
    t = ctx.read_tables()
    ctx.close()
    S, W = len(ik.sites), ik.n_warps
    assert diff_tables(t, t_or, S, W) is None
    assert (st["n_records"], st["n_addr_rows"], st["n_val_rows"]) == (
        rec["n"], rec["n_addr_rows"], rec["n_val_rows"])
    assert int(t[0]) == rec["n"]
    if bps:
        assert st["blocks_per_segment"] == bps
        assert st["segments"] >= 1 and st["max_segment_records"] <= rec["n"]
    ik.close()


@pytest.mark.parametrize("mask", [1, 2, 4, 8, 16, 15])
def test_online_single_handlers(mask):
    ik = sassi.InstrumentedKernel("bfs", SIZES["bfs"])
    _, t_or = whole_trace_oracle(ik, mask)
    ctx = ik.context(mask)
    ik.trace_fold(ctx, blocks_per_segment=2)
    t = ctx.read_tables()
    ctx.close()
    assert diff_tables(t, t_or, len(ik.sites), ik.n_warps) is None
    ik.close()


@pytest.mark.parametrize("name,size", [("bfs", 1 << 16), ("stencil", 1024), ("sgemm", 256),
                                       ("vecadd", 1 << 22)])
def test_online_equals_inline_at_larger_sizes(name, size):
    """Sizes whose whole trace the oracle would take long on: the online fold equals the inline
    handlers' tables (themselves equal to the oracle at the small sizes, test_gpu_inline.py) except
    the record diagnostics, which only a record stream has; the tables accumulate across repeated
    runs exactly twice over."""
    ik = sassi.InstrumentedKernel(name, size)
    mask = sassi.SASSI_H_EVERY
    S, W = len(ik.sites), ik.n_warps
    ctx = ik.context(mask)
    ik.run(mask, ctx)
    t_inline = ctx.read_tables()
    ctx.close()
    ctx = ik.context(mask)
    st = ik.trace_fold(ctx, blocks_per_segment=37)
    t = ctx.read_tables()
    assert int(t[0]) == st["n_records"] > 0 and int(t[2]) == 0
    t_cmp = t.copy()
    t_cmp[0:4] = 0
    assert diff_tables(t_cmp, t_inline, S, W) is None
    ik.trace_fold(ctx)  # default segment size, accumulating into the same tables
    t2 = ctx.read_tables()
    ctx.close()
    sec1, sec2 = oracle.sections(t, S, W), oracle.sections(t2, S, W)
    for k in ("br", "mem", "val", "counts", "h32", "h128", "mix"):
        assert np.array_equal(sec2[k], 2 * sec1[k]), k
    for k in ("ones", "zeros", "scalar"):
        assert np.array_equal(sec2[k], sec1[k]), k
    ik.close()


def test_online_preserves_output_and_rejects_bad_arguments():
    ik = sassi.InstrumentedKernel("stencil", 64)
    ik.run(sassi.SASSI_IK_NONE)
    torch.cuda.synchronize()
    base = ik.checksum()
    ctx = ik.context(sassi.SASSI_H_ALL)
    ik.trace_fold(ctx, blocks_per_segment=4)
    assert ik.checksum() == base
    with pytest.raises(sassi.SassiError):
        sassi.sassi_ik_trace_fold(ik.handle, ctx.handle, 1, 2)  # unknown flag
    other = sassi.InstrumentedKernel("bfs", 4096)
    with pytest.raises(sassi.SassiError):
        other.trace_fold(ctx)  # ctx holds another kernel's sites
    ctx.close()
    other.close()
    ik.close()
