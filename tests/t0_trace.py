"""T0 — the hand-worked tiny trace with its expected tables written by hand.

Every expected number below was computed on paper from the handler listings, not by any code:
  Fig.4 (L237-L243) branch, Fig.6 (L361-L369) memory divergence, Fig.9 (L549-L563) value profile,
  §8.1 (L625-L627) per-thread counts, Fig.3 (L193-L199) instruction mix; readings R1-R13 and R22
  of DESIGN.md §3.
"""
import numpy as np

from oracle import SITE_DTYPE, HDR_DTYPE, F_COND_BRANCH, F_CTRL, F_MEM, F_MEM_READ, F_MEM_WRITE, \
    F_NUMERIC, F_SYNC, F_WRITES_PRED, D_GLOBAL, D_SHARED

FULL = 0xFFFFFFFF
BASE = 0x7F0000001000          # 128 B aligned
N_WARPS = 2


def sites():
    s = np.zeros(7, dtype=SITE_DTYPE)
    rows = [
        (0x10, F_COND_BRANCH | F_CTRL, 0, D_GLOBAL, 0, [0, 0, 0, 0]),             # s0 BRA
        (0x20, F_MEM | F_MEM_READ, 4, D_GLOBAL, 1, [12, 0, 0, 0]),               # s1 LDG R12
        (0x30, F_MEM | F_MEM_WRITE, 8, D_GLOBAL, 0, [0, 0, 0, 0]),               # s2 STG.64
        (0x40, F_NUMERIC, 0, D_GLOBAL, 1, [13, 0, 0, 0]),                        # s3 IADD R13
        (0x50, F_MEM | F_MEM_READ, 4, D_SHARED, 1, [14, 0, 0, 0]),               # s4 LDS R14
        (0x60, F_NUMERIC | F_WRITES_PRED, 0, D_GLOBAL, 0, [0, 0, 0, 0]),         # s5 ISETP
        (0x70, F_SYNC, 0, D_GLOBAL, 0, [0, 0, 0, 0]),                            # s6 BAR
    ]
    for i, (pc, fl, w, dom, nd, regs) in enumerate(rows):
        s[i]["pc"], s[i]["flags"], s[i]["mem_width"], s[i]["domain"] = pc, fl, w, dom
        s[i]["n_gpr_dst"], s[i]["reg_num"] = nd, regs
    return s


def records():
    """-> hdr [15], addr rows [6,32], val rows [8,32] (garbage outside the masks on purpose)."""
    lanes = np.arange(32, dtype=np.uint64)
    junk64 = np.uint64(0x0123456789ABCDEF) * (lanes + np.uint64(7))
    junk32 = (np.arange(32, dtype=np.uint32) * np.uint32(2654435761)) ^ np.uint32(0xDEADBEEF)
    H, A, V = [], [], []

    def rec(pc, warp, active, mask2, addr=None, vals=()):
        H.append((pc, warp, active, mask2))
        if addr is not None:
            A.append(addr)
        for v in vals:
            V.append(v)

    # r0-r2: s0 branch (R1: taken = mask2 & active)
    rec(0x10, 0, FULL, FULL)                          # converged taken
    rec(0x10, 0, FULL, 0)                             # converged not taken
    rec(0x10, 1, 0x0000FFFF, 0xFF0000FF)              # 8 taken + 8 not taken -> divergent
    # r3: s1 unit-stride 4 B at a 128 B-aligned base: 32 lanes, 4 sectors, 1 line; value = lane
    rec(0x20, 0, FULL, FULL, BASE + 4 * lanes, [np.arange(32, dtype=np.uint32)])
    # r4: s1 broadcast load: 1 sector, 1 line; value == 1 (scalar)
    rec(0x20, 0, FULL, FULL, np.full(32, BASE + 64, np.uint64), [np.ones(32, np.uint32)])
    # r5: s1 4 active lanes, unit stride: 1 sector, 1 line; value 1 on the 4 lanes, junk elsewhere
    v5 = junk32.copy()
    v5[:4] = 1
    a5 = junk64.copy()
    a5[:4] = BASE + 4 * lanes[:4]
    rec(0x20, 1, 0x0000000F, FULL, a5, [v5])
    # r6: s2 store, 128 B stride, lane 5 predicated off (R2): 31 lanes / 31 sectors / 31 lines
    a6 = BASE + 128 * lanes
    a6[5] = a6[4]                                     # would merge with lane 4 if not excluded
    rec(0x30, 1, FULL, FULL & ~(1 << 5), a6)
    # r7: s3 value == 1 on all lanes -> "R13* <- [0...01]"
    rec(0x40, 0, FULL, FULL, None, [np.ones(32, np.uint32)])
    # r8: s3 active lanes {0,1}, lane 1 predicated off (R3); lane 1 holds junk 0xFFFFFFFF
    v8 = junk32.copy()
    v8[0] = 1
    v8[1] = 0xFFFFFFFF
    rec(0x40, 1, 0x3, 0x1, None, [v8])
    # r9: s4 shared-memory load: ignored by memdiv (R7), counted by instcount, value 7 (scalar)
    rec(0x50, 0, FULL, FULL, BASE + 4 * lanes, [np.full(32, 7, np.uint32)])
    # r10: s5 predicate write, guard true on lanes 16..31 of warp 1
    rec(0x60, 1, FULL, 0xFFFF0000)
    # r11: s6 barrier: not eligible for instcount
    rec(0x70, 0, FULL, FULL)
    # r12: unregistered pc: no rows, n_unknown_pc
    rec(0x999, 0, FULL, FULL)
    # r13: s3 with no active lane: n_invalid; its value row exists and is skipped
    rec(0x40, 0, 0, FULL, None, [junk32])
    # r14: s1, lanes 0-15 8 B unit stride (4 sectors, 1 line), lanes 16-31 the same 2^40 B higher
    #      (4 more sectors, 1 more line; high words differ -> wide-window path): 8 sectors / 2 lines
    a14 = np.where(lanes < 16, BASE + 8 * lanes, BASE + (1 << 40) + 8 * (lanes - 16)).astype(np.uint64)
    rec(0x20, 1, FULL, FULL, a14, [np.arange(32, dtype=np.uint32)])

    hdr = np.array(H, dtype=np.uint32).view(HDR_DTYPE).reshape(-1)
    addr = np.array(A, dtype=np.uint64).reshape(-1, 32)
    val = np.array(V, dtype=np.uint32).reshape(-1, 32)
    return hdr, addr, val


# ---- expected tables, by hand ------------------------------------------------------------------
EXPECT_DIAG = [15, 1, 1, 0]                        # n_records, n_invalid, n_unknown_pc, n_bad_warp
EXPECT_BR = {0: [3, 80, 40, 40, 1]}                # totals: 32+32+16 active, 32+0+8 taken
EXPECT_MEM = {1: [4, 100, 14, 5], 2: [1, 31, 31, 31]}
EXPECT_H32 = {(31, 3): 1, (31, 0): 1, (3, 0): 1, (30, 30): 1, (31, 7): 1}
EXPECT_H128 = {(31, 0): 2, (3, 0): 1, (30, 30): 1, (31, 1): 1}
EXPECT_VAL = {1: [4, 100], 3: [2, 33], 4: [1, 32]}
EXPECT_ONES = {1: 0x0, 3: 0x1, 4: 0x7}
EXPECT_ZEROS = {1: 0xFFFFFFE0, 3: 0xFFFFFFFE, 4: 0xFFFFFFF8}
EXPECT_SCALAR = {1: 0, 3: 1, 4: 1}


def expect_counts():
    c = np.zeros(32 * N_WARPS, dtype=np.uint64)
    c[0:32] = 4                                     # r3, r4, r7, r9
    w1 = np.zeros(32, np.uint64)
    w1[0] = 4                                       # r5, r6, r8, r14
    w1[1:4] = 3                                     # r5, r6, r14
    w1[4] = 2                                       # r6, r14
    w1[5] = 1                                       # r14 (predicated off in r6)
    w1[6:16] = 2                                    # r6, r14
    w1[16:32] = 3                                   # r6, r10, r14
    c[32:64] = w1
    return c


# Fig.3 (R22): every ACTIVE thread counts (guard-false lanes too), per site Σ popc(active):
#   s0 32+32+16, s1 32+32+4+32, s2 32 (lane 5 guard-false still counts), s3 32+2 (+0 for r13),
#   s4 32, s5 32, s6 32; r12 is unregistered.
EXPECT_MIX = [80, 100, 32, 34, 32, 32, 32]
# memory = s1+s2+s4 = 164; extended (width > 4) = s2 = 32; controlxfer = s0 = 80; sync = s6 = 32;
# numeric = s3+s5 = 66; texture = 0; total = 342
EXPECT_IMIX = [164, 32, 80, 32, 66, 0, 342, 0]

EXPECT_VALUE_LINES = {
    0x20: ["R12 <- [000000000000000000000000000TTTTT]"],
    0x40: ["R13* <- [00000000000000000000000000000001]"],
    0x50: ["R14* <- [00000000000000000000000000000111]"],
}


def check_table(t, sec, mask=15):
    """Assert a table image (dict of sections) equals the hand-worked expectation (handlers 1-8
    always; the Fig.3 sections when mask has 16, else they stay 0)."""
    assert list(map(int, sec["diag"][:4])) == EXPECT_DIAG
    S = 7
    for s in range(S):
        assert list(map(int, sec["br"][s])) == EXPECT_BR.get(s, [0] * 5), ("br", s)
        assert list(map(int, sec["mem"][s])) == EXPECT_MEM.get(s, [0] * 4), ("mem", s)
        assert list(map(int, sec["val"][s])) == EXPECT_VAL.get(s, [0, 0]), ("val", s)
        assert int(sec["ones"][s, 0]) == EXPECT_ONES.get(s, 0xFFFFFFFF), ("ones", s)
        assert int(sec["zeros"][s, 0]) == EXPECT_ZEROS.get(s, 0xFFFFFFFF), ("zeros", s)
        assert int(sec["scalar"][s, 0]) == EXPECT_SCALAR.get(s, 1), ("scalar", s)
        for d in range(1, 4):
            assert int(sec["ones"][s, d]) == 0xFFFFFFFF and int(sec["zeros"][s, d]) == 0xFFFFFFFF
            assert int(sec["scalar"][s, d]) == 1
    h32 = np.zeros((32, 32), np.uint64)
    for k, v in EXPECT_H32.items():
        h32[k] = v
    h128 = np.zeros((32, 32), np.uint64)
    for k, v in EXPECT_H128.items():
        h128[k] = v
    assert np.array_equal(sec["h32"], h32)
    assert np.array_equal(sec["h128"], h128)
    assert np.array_equal(sec["counts"], expect_counts())
    mix = EXPECT_MIX if mask & 16 else [0] * 7
    imix = EXPECT_IMIX if mask & 16 else [0] * 8
    assert list(map(int, sec["mix"])) == mix
    assert list(map(int, sec["imix"])) == imix
