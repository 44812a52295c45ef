"""Inline handlers at the sizes the slowdown K is quoted on (bench.py `instrumented_slowdown`:
vecadd 2^25 floats, BFS 2^21 nodes, stencil 8192^2, SGEMM 2048^3): thousands of CTAs, all 256
%smid table stripes and long per-warp runs, with every handler attached (default and SMEM modes).

vecadd / BFS / stencil: the inline tables equal the fold of the same kernel's whole trace, which
equals the oracle over that trace (11-19 million records each). SGEMM 2048's trace is ~1.2x10^9
records, beyond a host oracle pass here: its inline tables equal the online trace-mode fold of the
whole kernel (segment by segment; that fold is itself oracle-exact, tests/test_gpu_online.py),
and its per-thread counts and loop-branch counters equal their closed forms."""
import numpy as np
import pytest

import oracle
from gpu_helpers import diff_tables
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def no_diag(t):
    t = t.copy()
    t[0:4] = 0
    return t


@pytest.mark.parametrize("name", ["vecadd", "bfs", "stencil"])
def test_inline_equals_trace_fold_equals_oracle_at_timing_size(name):
    ik = sassi.InstrumentedKernel(name, 0)          # size 0 = the timing size
    S, W = len(ik.sites), ik.n_warps
    mask = sassi.SASSI_H_EVERY
    inline = {}
    for smem in (0, sassi.SASSI_IK_SMEM):
        ctx = ik.context(mask)
        ik.run(mask | smem, ctx)
        inline[smem] = ctx.read_tables()
        ctx.close()
    ctx = ik.context(mask)
    rec = ik.trace(ctx)
    ctx.consume(rec)
    t_fold = ctx.read_tables()
    ctx.close()
    assert rec["n"] > 10_000_000
    h = gen.to_host(rec)
    del rec
    torch.cuda.empty_cache()
    t_or = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(t_fold, t_or, S, W) is None
    for smem, t in inline.items():
        assert diff_tables(t, no_diag(t_or), S, W) is None, smem
    ik.close()


def test_sgemm_2048_inline_equals_online_fold_and_closed_forms():
    n = 2048
    ik = sassi.InstrumentedKernel("sgemm", n)
    S, W = len(ik.sites), ik.n_warps
    mask = sassi.SASSI_H_EVERY
    ctx = ik.context(mask)
    st = ik.trace_fold(ctx)
    t_fold = ctx.read_tables()
    ctx.close()
    assert st["n_records"] > 10**9
    for smem in (0, sassi.SASSI_IK_SMEM):
        ctx = ik.context(mask)
        ik.run(mask | smem, ctx)
        t = ctx.read_tables()
        ctx.close()
        assert diff_tables(t, no_diag(t_fold), S, W) is None, smem
    sec = oracle.sections(t_fold, S, W)
    # closed forms: per tile a thread executes 2 LDG + 2 STS + 16 x (2 LDS + FFMA) eligible
    # instructions, over n / 16 tiles, plus the final STG
    nt = n // 16
    assert (sec["counts"] == nt * (4 + 16 * 3) + 1).all()
    assert len(sec["counts"]) == n * n
    # the k-loop branch (s7) runs 16 times per tile per warp, taken 15 of 16, never divergent
    warps = n * n // 32
    assert list(map(int, sec["br"][7])) == [16 * nt * warps, 16 * nt * n * n, 15 * nt * n * n,
                                           nt * n * n, 0]
    ik.close()
