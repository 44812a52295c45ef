"""Randomised parity fuzz (GPU): random traces (tests/test_oracle.random_trace) under random handler
masks, per-PC matrix selections, dynamic-pc tables, split / host-buffer consumption, the GLOBAL-only
address-row layout, forced global mode, and warp shards merged with sassi_merge_local; every table
(and dynamic table, and draw) must equal the oracle's bit for bit.
usage: python tools/fuzz_parity.py [N_CASES] [SEED]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from gpu_helpers import to_device, diff_tables  # noqa: E402
from test_oracle import random_trace  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

n_cases = int(sys.argv[1]) if len(sys.argv) > 1 else 200
rng = np.random.default_rng(int(sys.argv[2]) if len(sys.argv) > 2 else 1)
fails = 0
for case in range(n_cases):
    seed = int(rng.integers(0, 2**31))
    n = int(rng.choice([1, 7, 255, 256, 257, 1000, 4096, 20000, 65536]))
    W = int(rng.integers(1, 40))
    s, W, hdr, addr, val = random_trace(seed, n=n, n_warps=W)
    mask = int(rng.integers(1, 32))
    # optionally unregister some row-less sites (dynamic pcs then count them)
    dyn = bool(rng.integers(0, 2))
    if dyn:
        rowless = [i for i in range(len(s)) if not (s[i]["flags"] & oracle.F_MEM) and s[i]["n_gpr_dst"] == 0]
        drop = rng.choice(rowless, size=min(len(rowless), int(rng.integers(0, 3))), replace=False)
        s = s[~np.isin(np.arange(len(s)), drop)]
    glob = [i for i in range(len(s)) if (s[i]["flags"] & oracle.F_MEM) and s[i]["domain"] == oracle.D_GLOBAL]
    sel = list(rng.choice(glob, size=min(len(glob), int(rng.integers(0, 5))), replace=False)) if glob else []
    d = to_device(s, hdr, addr, val)
    gmode = bool(rng.integers(0, 2))
    os.environ["SASSI_FORCE_GLOBAL_MODE"] = "1" if gmode else "0"
    rows_g = bool(rng.integers(0, 3) == 0)
    if rows_g:
        d = gen.split_global_rows(dict(d, sites=s))
    ctx = sassi.Context(s, W, mask)
    if rows_g:
        ctx.set_addr_rows(sassi.SASSI_ADDR_ROWS_GLOBAL)
    if sel:
        ctx.select_memdiv_pcs([int(s[i]["pc"]) for i in sel])
    if dyn:
        ctx.enable_dynamic_pcs(64)
    # consume in one piece, in two chunk-aligned pieces, from pinned host buffers, or as P warp
    # shards in P contexts merged with sassi_merge_local
    how = int(rng.integers(0, 4))
    if how == 3 and not rows_g:
        P = int(rng.integers(2, 6))
        others = []
        site = {int(x["pc"]): x for x in s}
        na = np.cumsum([0] + [1 if int(q) in site and int(site[int(q)]["flags"]) & oracle.F_MEM else 0
                              for q in hdr["pc"]])
        nv = np.cumsum([0] + [int(site[int(q)]["n_gpr_dst"]) if int(q) in site else 0 for q in hdr["pc"]])
        for r in range(P):
            idx = np.nonzero(hdr["warp"] % P == r)[0]
            c = ctx if r == 0 else sassi.Context(s, W, mask)
            if r and sel:
                c.select_memdiv_pcs([int(s[i]["pc"]) for i in sel])
            if r and dyn:
                c.enable_dynamic_pcs(64)
            if len(idx):
                ar = np.concatenate([np.arange(na[i], na[i + 1]) for i in idx]).astype(np.int64)
                vr = np.concatenate([np.arange(nv[i], nv[i + 1]) for i in idx]).astype(np.int64)
                c.consume(to_device(s, hdr[idx], addr.reshape(-1, 32)[ar], val.reshape(-1, 32)[vr]))
            if r:
                others.append(c)
        sassi.sassi_merge_local([ctx] + others)
        for c in others:
            c.close()
    elif how == 2:
        ctx.consume_host({k: (v.cpu().pin_memory() if hasattr(v, "cpu") else v) for k, v in d.items()})
    elif n > 512 and how == 1:
        half = (n // 2) // 256 * 256
        ctx.consume(dict(d, hdr=d["hdr"][:half], chunk_base=d["chunk_base"][: half // 256 + 1], n=half))
        ctx.consume(dict(d, hdr=d["hdr"][half:], chunk_base=d["chunk_base"][half // 256:], n=n - half))
    else:
        ctx.consume(d)
    t = ctx.read_tables()
    o = oracle.run(s, W, mask, hdr, addr, val, pcs=[int(i) for i in sel])  # pcsel: configuration
    msg = diff_tables(t, o, len(s), W)
    if msg is None and dyn:
        dynt, dropped = ctx.read_dynamic_pcs()
        odyn, odrop = oracle.dynamic_pcs(s, hdr)
        got = [[int(e["pc"]), int(e["warp_execs"]), int(e["thread_execs"])] for e in dynt]
        if got != odyn.tolist() or dropped != odrop:
            msg = "dynamic table differs"
    if msg is None and (mask & 8):  # injection-site draws over the per-thread counts (L629)
        sec = oracle.sections(o, len(s), W)
        if int(sec["counts"].sum()) > 0:
            k, sd = int(rng.integers(1, 300)), int(rng.integers(0, 2**62))
            if not np.array_equal(ctx.sample(k, sd), oracle.sample(sec["counts"], k, sd)):
                msg = "sampling differs"
    ctx.close()
    if msg is not None:
        fails += 1
        print("FAIL case %d seed %d n %d W %d mask %d dyn %d sel %s how %d gmode %d rows_g %d: %s" % (
            case, seed, n, W, mask, dyn, sel, how, gmode, rows_g, msg), flush=True)
print("fuzz: %d cases, %d failures" % (n_cases, fails))
sys.exit(1 if fails else 0)
