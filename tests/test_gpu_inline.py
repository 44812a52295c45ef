"""Inline handlers in instrumented kernels: for each synthetic kernel, the tables the
inline handlers build during execution equal the fold (sassi_consume) of the same kernel's trace,
which equals the oracle on that trace; instrumentation never changes the kernel's output; the
instrumented vector add reproduces c1's closed forms."""
import numpy as np
import pytest

import oracle
from gpu_helpers import diff_tables
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

SMALL = {"vecadd": 12800, "bfs": 4096, "sgemm": 64, "stencil": 64}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def no_diag(t):
    """Inline handlers see no record stream, so the record diagnostics diag[0..3] stay 0."""
    t = t.copy()
    t[0:4] = 0
    return t


def trace_and_fold(ik, mask):
    ctx = ik.context(mask)
    rec = ik.trace(ctx)
    ctx.consume(rec)
    t = ctx.read_tables()
    ctx.close()
    return rec, t


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("mask", [sassi.SASSI_H_ALL, sassi.SASSI_H_EVERY])
@pytest.mark.parametrize("smem", [0, sassi.SASSI_IK_SMEM])
def test_inline_equals_trace_fold_equals_oracle(name, mask, smem):
    ik = sassi.InstrumentedKernel(name, SMALL[name])
    S, W = len(ik.sites), ik.n_warps
    ctx = ik.context(mask)
    ik.run(mask | smem, ctx)
    t_inline = ctx.read_tables()
    ctx.close()
    rec, t_fold = trace_and_fold(ik, mask)
    assert rec["n"] > 0
    h = gen.to_host(rec)
    t_or = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(t_fold, t_or, S, W) is None
    assert int(t_inline[0]) == 0
    assert diff_tables(t_inline, no_diag(t_or), S, W) is None
    ik.close()


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("mask", [1, 2, 4, 8, 16])
@pytest.mark.parametrize("smem", [0, sassi.SASSI_IK_SMEM])
def test_single_handler_inline(name, mask, smem):
    ik = sassi.InstrumentedKernel(name, SMALL[name])
    ctx = ik.context(mask)
    ik.run(mask | smem, ctx)
    t_inline = ctx.read_tables()
    ctx.close()
    _, t_fold = trace_and_fold(ik, mask)
    assert diff_tables(t_inline, no_diag(t_fold), len(ik.sites), ik.n_warps) is None
    ik.close()


@pytest.mark.parametrize("name", list(SMALL))
def test_instrumentation_preserves_output(name):
    ik = sassi.InstrumentedKernel(name, SMALL[name])
    ik.run(sassi.SASSI_IK_NONE)
    torch.cuda.synchronize()
    base = ik.checksum()
    ctx = ik.context(sassi.SASSI_H_EVERY)
    for mode in (sassi.SASSI_IK_NULL_ABI, sassi.SASSI_H_ALL, 1, 2, 4, 8, 16, sassi.SASSI_H_EVERY):
        ik.run(mode, ctx if mode & sassi.SASSI_H_EVERY else None)
        torch.cuda.synchronize()
        assert ik.checksum() == base, mode
    ik.trace(ctx)
    assert ik.checksum() == base
    ctx.close()
    ik.close()


def test_instrumented_vecadd_is_config_c1():
    """The instrumented vector add (1 CTA x 128 threads, n = 12,800) is config c1's program: its
    divergent i%3 branch, loop branch and unit-stride loads give c1's closed forms."""
    ik = sassi.InstrumentedKernel("vecadd", 12800)
    assert ik.n_warps == 4
    ctx = ik.context(sassi.SASSI_H_ALL)
    ik.run(sassi.SASSI_H_ALL, ctx)
    sec = ctx.sections()
    n3 = len(range(0, 12800, 3))
    assert list(map(int, sec["br"][4])) == [400, 12800, n3, 12800 - n3, 400]
    assert list(map(int, sec["br"][7])) == [400, 12800, 4 * 99 * 32, 128, 0]
    for s in (0, 1, 3):
        assert list(map(int, sec["mem"][s])) == [400, 12800, 1600, 400]
    assert list(map(int, sec["mem"][5])) == [400, n3, n3, n3]
    # per-thread counts: 7 eligible sites per iteration (IMAD.WIDE, IADD.CC, 2 LDG, FADD, STG,
    # ISETP) + the x load and the running sum in iterations where i % 3 == 0
    expect = 7 * 100 + 2 * np.array([sum(1 for it in range(100) if (128 * it + t) % 3 == 0)
                                      for t in range(128)])
    assert np.array_equal(sec["counts"].astype(np.int64), expect)
    ctx.close()
    ik.close()
