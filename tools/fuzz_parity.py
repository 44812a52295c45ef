"""Randomised parity fuzz (GPU): random traces (tests/test_oracle.random_trace) under random handler
masks, per-PC matrix selections, dynamic-pc tables and split consumption; every table (and dynamic
table) must equal the oracle's bit for bit. usage: python tools/fuzz_parity.py [N_CASES] [SEED]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from gpu_helpers import to_device, diff_tables  # noqa: E402
from test_oracle import random_trace  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import sassi  # noqa: E402

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
    ctx = sassi.Context(s, W, mask)
    if sel:
        ctx.select_memdiv_pcs([int(s[i]["pc"]) for i in sel])
    if dyn:
        ctx.enable_dynamic_pcs(64)
    # consume in one piece, in two chunk-aligned pieces, or from pinned host buffers
    how = int(rng.integers(0, 3))
    if how == 2:
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
        print("FAIL case %d seed %d n %d W %d mask %d dyn %d sel %s: %s" % (case, seed, n, W, mask, dyn, sel, msg),
              flush=True)
print("fuzz: %d cases, %d failures" % (n_cases, fails))
sys.exit(1 if fails else 0)
