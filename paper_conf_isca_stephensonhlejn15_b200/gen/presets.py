"""Workload presets c1..c5 (BASELINE.json ``configs``; recipe in DESIGN.md §5).

Each preset is a synthetic instrumented kernel shaped like the paper's workloads:
  c1  tiny vector add (4 warps, 12,800 floats, grid-stride) + one divergent branch + one strided load
  c2  Rodinia/Parboil-BFS-shaped irregular trace (10^7 records, 10^6 threads, gathers, frontier masks,
      data-dependent branches ~10 % divergent — Table 1 bfs 4-15 %, L265/L271)
  c3  SGEMM/stencil-shaped regular trace (10^8 records, coalesced / broadcast / 16 B vector loads,
      uniform loop branches — sgemm 0 % divergent, L265 — value handler on all register writes)
  c4  error-injection profiling pass (10^8 records, 10^6 threads, 85 % eligible sites, 25 % partial
      masks, 5 % guard-false lanes; then 1,000 site draws, L629)
  c5  mixed c2/c3 warps (alternating by warp id), 131,072 warps, ~4x10^9 records, sharded by warp
"""
from __future__ import annotations

from . import (Program, prob, TRIP_FIXED, TRIP_HEAVY, BASE_FULL, BASE_FRONTIER, T_ALL, T_UNIFORM,
               T_DIVERGE, T_MOD, T_LOOP, T_WARPMOD, G_ALL, G_BERN, A_UNIT, A_BCAST, A_STRIDE,
               A_GATHER, A_WINDOW, V_CONST, V_ELEM, V_SMALL, V_RAND, V_FLOAT, V_ITER, V_LANE,
               V_BOOL, V_WSCALAR, V_ADDR_LO, V_ADDR_HI, F_COND_BRANCH, F_CTRL, F_MEM, F_MEM_READ,
               F_MEM_WRITE, F_NUMERIC, F_SYNC, F_WRITES_PRED, D_GLOBAL, D_SHARED)

GB = 1 << 30
VA = 0x7F0000000000  # base of synthetic device allocations (2^40-aligned)
BR = F_COND_BRANCH | F_CTRL
LD = F_MEM | F_MEM_READ
ST = F_MEM | F_MEM_WRITE
ALU = F_NUMERIC
H_ALL = 15


def c1_vecadd(seed: int = 20150613) -> Program:
    """4 warps x 100 grid-stride iterations of c[i] = a[i] + b[i] (n = 12,800) with a divergent
    `if (i % 3 == 0) s += x[32*i]` (128 B stride -> 32 sectors / 32 lines)."""
    P = Program("c1-vecadd", seed, total_warps=4, trip=(TRIP_FIXED, 100, 0, 0))
    A, B, C, X = VA, VA + GB, VA + 2 * GB, VA + 3 * GB
    P.op(0, flags=ALU, n_dst=1, vals=[(V_LANE, 0, 0)], regs=[0])                      # S2R R0, SR_TID.X
    P.op(0, flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 0)], regs=[3])                      # IMAD R3 = gtid
    P.op(1, flags=ALU, n_dst=2, addr=(A_UNIT, A, 4), vals=[(V_ADDR_LO, 0, 0), (V_ADDR_HI, 0, 0)],
         regs=[4, 5])                                                                  # IMAD.WIDE R4 = &a[i]
    P.op(1, flags=ALU, n_dst=2, addr=(A_UNIT, B, 4), vals=[(V_ADDR_LO, 0, 0), (V_ADDR_HI, 0, 0)],
         regs=[6, 7])                                                                  # IMAD.WIDE R6 = &b[i]
    P.op(1, flags=LD, n_dst=1, width=4, addr=(A_UNIT, A, 4), vals=[(V_FLOAT, 23, 0)], regs=[8])
    P.op(1, flags=LD, n_dst=1, width=4, addr=(A_UNIT, B, 4), vals=[(V_FLOAT, 23, 0)], regs=[9])
    P.op(1, flags=ALU, n_dst=1, vals=[(V_RAND, 0, 0)], regs=[10])                     # FADD R10
    P.op(1, flags=ST, width=4, addr=(A_UNIT, C, 4))                                    # STG.E [c+i]
    P.op(1, flags=ALU | F_WRITES_PRED)                                                 # ISETP P0 = i%3==0
    br = P.op(1, flags=BR, mask=(T_MOD, 3, 0))                                         # @P0 BRA
    P.op(1, flags=LD, n_dst=1, width=4, addr=(A_STRIDE, X, 128), vals=[(V_SMALL, 20, 0)],
         parent=br, regs=[11])                                                         # LDG x[32*i]
    P.op(1, flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 128)], regs=[3])                    # IADD R3 += 128
    P.op(1, flags=ALU | F_WRITES_PRED)                                                 # ISETP P1 = i<n
    P.op(1, flags=BR, mask=(T_LOOP, 0, 0))                                             # @P1 BRA loop
    P.op(2, flags=F_CTRL)                                                              # EXIT
    return P


def _bfs_block(P: Program, sec: int, k: int, parent: int = -1, diverge_q: float = 0.35):
    """One 25-instruction BFS edge-relaxation block (Parboil/Rodinia bfs inner loop shape):
    unit-stride edge loads, random gathers into 64 MB node arrays, a data-dependent branch."""
    E = VA + (4 + 4 * k) * GB       # edge array (unit stride)
    COST = VA + (5 + 4 * k) * GB    # node arrays, 64 MB = 16 M x 4 B, random gathers
    VIS = VA + (6 + 4 * k) * GB
    NODE = VA + (7 + 4 * k) * GB
    NE = (64 << 20) // 4
    pa = parent

    def op(**kw):
        kw.setdefault("parent", pa)
        return P.op(sec, **kw)

    op(flags=ALU, n_dst=2, addr=(A_UNIT, E, 4), vals=[(V_ADDR_LO, 0, 0), (V_ADDR_HI, 0, 0)])
    op(flags=LD, n_dst=1, width=4, addr=(A_UNIT, E, 4), vals=[(V_SMALL, 20, 0)])     # nbr = edges[j]
    op(flags=ALU, n_dst=2, addr=(A_GATHER, COST, NE, 4), vals=[(V_ADDR_LO, 0, 0), (V_ADDR_HI, 0, 0)])
    op(flags=LD, n_dst=1, width=4, addr=(A_GATHER, COST, NE, 4), vals=[(V_SMALL, 8, 0)])
    op(flags=LD, n_dst=1, width=4, addr=(A_GATHER, VIS, NE, 4), vals=[(V_BOOL, prob(0.3), 0)])
    op(flags=ALU | F_WRITES_PRED)
    b = op(flags=BR, mask=(T_DIVERGE, prob(diverge_q), prob(0.5)))
    op(flags=ALU, n_dst=1, vals=[(V_SMALL, 8, 0)], parent=b)                            # cost + 1
    op(flags=ST, width=4, addr=(A_GATHER, COST, NE, 4), parent=b)
    op(flags=ST, width=4, addr=(A_GATHER, VIS, NE, 4), parent=b)
    op(flags=ALU, n_dst=1, vals=[(V_WSCALAR, 1, 0)], parent=b)                         # over = true
    op(flags=ALU, n_dst=1, vals=[(V_BOOL, prob(0.5), 0)])
    op(flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 0)])                                       # j++
    op(flags=ALU | F_WRITES_PRED)
    b2 = op(flags=BR, mask=(T_UNIFORM, prob(0.9), 0))
    op(flags=LD, n_dst=1, width=4, addr=(A_GATHER, NODE, NE, 8), vals=[(V_SMALL, 20, 0)], parent=b2)
    op(flags=LD, n_dst=1, width=4, addr=(A_GATHER, NODE + 4, NE, 8), vals=[(V_SMALL, 4, 0)],
       parent=b2)
    op(flags=ALU, n_dst=1, vals=[(V_SMALL, 20, 0)], parent=b2)
    op(flags=ALU, n_dst=1, vals=[(V_CONST, 0xFFFFFFFF, 0)])                             # MOV -1
    op(flags=ALU, n_dst=1, vals=[(V_ITER, 1, 0)])                                       # level
    op(flags=ALU, n_dst=1, vals=[(V_SMALL, 16, 0)])
    op(flags=LD, n_dst=1, width=4, addr=(A_UNIT, NODE, 4), vals=[(V_SMALL, 20, 0)])
    op(flags=ALU | F_WRITES_PRED)
    op(flags=BR, mask=(T_UNIFORM, prob(0.5), 0))
    op(flags=ALU, n_dst=1, vals=[(V_SMALL, 8, 0)])


def c2_bfs(seed: int = 20150614) -> Program:
    P = Program("c2-bfs", seed, total_warps=31250, trip=(TRIP_HEAVY, 1, 2, 4),
                base=(BASE_FRONTIER, prob(0.4)))
    P.op(0, flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 0)], regs=[0])                      # tid
    P.op(0, flags=LD, n_dst=2, width=8, addr=(A_UNIT, VA, 8),
         vals=[(V_SMALL, 20, 0), (V_SMALL, 6, 0)])                                     # node {start, deg}
    for k in range(4):
        _bfs_block(P, 1, k)
    P.op(1, flags=ALU | F_WRITES_PRED)
    P.op(1, flags=BR, mask=(T_LOOP, 0, 0))
    P.op(2, flags=F_CTRL)
    return P


def _sgemm_block(P: Program, sec: int, k: int, parent: int = -1):
    """One 50-instruction SGEMM/stencil inner-loop block: unit-stride, broadcast and 16 B vector
    global loads, shared-memory tile traffic, FFMA chains, affine address math, loop counters."""
    Abase, Bbase, Cbase = VA + (40 + 3 * k) * GB, VA + (41 + 3 * k) * GB, VA + (42 + 3 * k) * GB
    SH = 0x10000 * (k + 1)
    pa = parent

    def op(**kw):
        kw.setdefault("parent", pa)
        return P.op(sec, **kw)

    for i in range(2):
        op(flags=LD, n_dst=1, width=4, addr=(A_UNIT, Abase + i * 0x100000, 4), vals=[(V_FLOAT, 23, 0)])
    op(flags=LD, n_dst=1, width=4, addr=(A_BCAST, Bbase, 4), vals=[(V_WSCALAR, 32, 0)])
    op(flags=LD, n_dst=4, width=16, addr=(A_UNIT, Bbase + 0x4000000, 16),
       vals=[(V_FLOAT, 23, 0)] * 4)                                                     # LDG.128
    for i in range(3):
        op(flags=ST, width=4, domain=D_SHARED,
           addr=(A_UNIT, SH + i * 0x1000, 4))                                            # STS tile
    for i in range(3):
        op(flags=LD, n_dst=1, width=4, domain=D_SHARED, addr=(A_BCAST, SH + i * 0x1000, 4),
           vals=[(V_FLOAT, 23, 0)])                                                      # LDS
    for i in range(20):
        op(flags=ALU, n_dst=1, vals=[(V_FLOAT, 23 if i % 4 else 20, 0)])                 # FFMA
    for i in range(5):
        op(flags=ALU, n_dst=1, vals=[(V_ELEM, 4, 0x1000 * i)])                          # IMAD addr
    for i in range(5):
        op(flags=ALU, n_dst=1, vals=[(V_ITER, 1 + i, 0)])                               # counters
    op(flags=ALU, n_dst=1, vals=[(V_CONST, 0x3F800000, 0)])
    op(flags=ALU, n_dst=1, vals=[(V_LANE, 0, 0)])
    op(flags=ALU | F_WRITES_PRED)
    op(flags=ALU | F_WRITES_PRED)
    op(flags=ALU | F_WRITES_PRED, mask=(G_BERN, prob(0.01), 0))
    op(flags=ST, width=4, addr=(A_UNIT, Cbase, 4), mask=(G_BERN, prob(0.01), 0))     # STG
    op(flags=LD, n_dst=1, width=4, addr=(A_BCAST, Cbase + 0x8000000, 4),
       vals=[(V_WSCALAR, 32, 0)])
    op(flags=F_SYNC)                                                                     # BAR.SYNC
    op(flags=BR, mask=(T_ALL, 0, 0))                                                     # k-loop edge


def c3_sgemm(seed: int = 20150615) -> Program:
    P = Program("c3-sgemm", seed, total_warps=32768, trip=(TRIP_FIXED, 31, 0, 0))
    P.op(0, flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 0)], regs=[0])
    P.op(0, flags=ALU, n_dst=1, vals=[(V_LANE, 0, 0)], regs=[1])
    for k in range(2):
        _sgemm_block(P, 1, k)
    P.op(1, flags=ALU | F_WRITES_PRED)
    P.op(1, flags=BR, mask=(T_LOOP, 0, 0))
    P.op(2, flags=ST, width=4, addr=(A_UNIT, VA + 60 * GB, 4))
    P.op(2, flags=F_CTRL)
    return P


def c4_inject(seed: int = 20150616) -> Program:
    """32 iterations x 100 instructions per warp: 85 eligible (60 ALU with a GPR result, 10 ISETP,
    10 loads, 5 stores with 5 % guard-false lanes), 15 not eligible (branches, barriers)."""
    P = Program("c4-inject", seed, total_warps=31250, trip=(TRIP_FIXED, 32, 0, 0),
                base=(BASE_FRONTIER, prob(0.25)))
    bern = (G_BERN, prob(0.05), 0)
    for i in range(100):
        r = i % 20
        if r < 12:
            P.op(1, flags=ALU, n_dst=1, vals=[(V_SMALL, 12 + r, 0)], mask=bern)
        elif r < 14:
            P.op(1, flags=ALU | F_WRITES_PRED, mask=bern)
        elif r < 16:
            P.op(1, flags=LD, n_dst=1, width=4, addr=(A_UNIT, VA + (70 + i) * GB, 4),
                 vals=[(V_FLOAT, 23, 0)], mask=bern)
        elif r < 17:
            P.op(1, flags=ST, width=4, addr=(A_UNIT, VA + (70 + i) * GB, 4), mask=bern)
        elif r < 19:
            P.op(1, flags=BR, mask=(T_UNIFORM, prob(0.5), 0))
        else:
            P.op(1, flags=F_SYNC)
    return P


def c5_mixed(seed: int = 20150617) -> Program:
    """Warps alternate a BFS-shaped and an SGEMM-shaped body (selected by warp id), 305 trips."""
    P = Program("c5-mixed", seed, total_warps=131072, trip=(TRIP_FIXED, 305, 0, 0),
                base=(BASE_FULL, 0))
    P.op(0, flags=ALU, n_dst=1, vals=[(V_ELEM, 1, 0)], regs=[0])
    a = P.op(1, flags=BR, mask=(T_WARPMOD, 2, 0))
    for k in range(4):
        _bfs_block(P, 1, k, parent=a)
    b = P.op(1, flags=BR, mask=(T_WARPMOD, 2, 1))
    _sgemm_block(P, 1, 0, parent=b)
    _sgemm_block(P, 1, 1, parent=b)
    P.op(1, flags=ALU | F_WRITES_PRED)
    P.op(1, flags=BR, mask=(T_LOOP, 0, 0))
    P.op(2, flags=F_CTRL)
    return P


PRESETS = {
    # name: (builder, record limit, handler mask, description)
    "c1": (c1_vecadd, None, H_ALL, "tiny hand-written trace: 4 warps, vector-add plus one "
           "divergent branch and one strided load, ~5k warp-instruction records"),
    "c2": (c2_bfs, 10_000_000, H_ALL, "Rodinia-BFS-shaped irregular trace: 10^7 records"),
    "c3": (c3_sgemm, 100_000_000, H_ALL, "SGEMM/stencil-shaped regular trace: 10^8 records"),
    "c4": (c4_inject, 100_000_000, 8, "error-injection profiling pass: 10^8 records, 10^6 threads"),
    "c5": (c5_mixed, 4_000_000_000, H_ALL, "all four handlers on a 4x10^9-record mixed trace"),
}


def preset(name: str):
    """-> (Program, record limit, handler mask, description)"""
    b, lim, mask, desc = PRESETS[name]
    return b(), lim, mask, desc
