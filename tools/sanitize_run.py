"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): T0 under
every handler set, a random edge trace, c1, the four instrumented kernels in every mode (inline,
trace, null ABI, injection), sampling and a 1-rank merge. Exits non-zero on any mismatch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import t0_trace as T0  # noqa: E402
from gpu_helpers import to_device, gpu_table  # noqa: E402
from test_oracle import random_trace  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

PART = os.environ.get("SANITIZE_PART", "all")  # all | base | online | dynamic | r2
s = T0.sites()
hdr, addr, val = T0.records()
d = to_device(s, hdr, addr, val)
if PART in ("all", "base"):
    for mask in (1, 2, 4, 8, 15, 16, 31):
        t = gpu_table(s, T0.N_WARPS, mask, d)
        assert np.array_equal(t, oracle.run(s, T0.N_WARPS, mask, hdr, addr, val)), mask
    s2, W, h2, a2, v2 = random_trace(4321, n=3000)
    t = gpu_table(s2, W, 31, to_device(s2, h2, a2, v2))
    assert np.array_equal(t, oracle.run(s2, W, 31, h2, a2, v2))
    t = gpu_table(s2, W, 31, to_device(s2, h2, a2, v2), pcs=[int(s2[1]["pc"]), int(s2[7]["pc"])])
    assert np.array_equal(t, oracle.run(s2, W, 31, h2, a2, v2, pcs=[1, 7]))
    P, lim, mask, _ = gen.preset("c1")
    dc = gen.generate_device(P, lim)
    ctx = sassi.Context(dc["sites"], P.total_warps, 31)
    ctx.consume(dc)
    ctx.sample(50, 7)
    ctx.close()
    for name, size in (("vecadd", 12800), ("bfs", 4096), ("sgemm", 32), ("stencil", 64)):
        ik = sassi.InstrumentedKernel(name, size)
        ctx = ik.context(sassi.SASSI_H_EVERY)
        for mode in (0, 1, 2, 4, 8, 16, 15, 31, sassi.SASSI_IK_NULL_ABI, 1024 | 1, 1024 | 2, 1024 | 15, 1024 | 31):
            ctx.reset()
            ik.run(mode, ctx if mode & 31 else None)
        ik.trace(ctx)
        ctx.close()
        ik.injection_campaign(k=20, seed=3)
        ik.close()

if PART in ("all", "online"):
    # online trace mode (count pass, placed trace into the ring, index + fold on the consumer stream)
    for name, size in (("vecadd", 1 << 16), ("bfs", 4096), ("sgemm", 64), ("stencil", 64)):
        ik = sassi.InstrumentedKernel(name, size)
        ctx = ik.context(sassi.SASSI_H_EVERY)
        rec = ik.trace(ctx)
        h = gen.to_host(rec)
        want = oracle.run(h["sites"], ik.n_warps, 31, h["hdr"], h["addr"], h["val"])
        for bps, serial in ((0, True), (3, False)):
            ctx.reset()
            ik.trace_fold(ctx, blocks_per_segment=bps, serial=serial)
            assert np.array_equal(ctx.read_tables(), want), (name, bps)
        ctx.close()
        ik.close()

if PART in ("all", "dynamic"):
    # dynamic sites: an empty site table (every record inserted on miss) and a 1-rank merge
    hs = np.zeros((5000, 4), np.uint32)
    rng = np.random.default_rng(5)
    hs[:, 0] = 0x1000 + 16 * rng.integers(0, 300, 5000)
    hs[:, 2] = rng.integers(0, 2**32, 5000, dtype=np.uint64).astype(np.uint32)
    hs = hs.view(oracle.HDR_DTYPE).reshape(-1)
    s0 = np.zeros(0, dtype=oracle.SITE_DTYPE)
    ctx = sassi.Context(s0, 4, 15)
    ctx.enable_dynamic_pcs(300)
    ctx.consume(to_device(s0, hs, None, None))
    uid = sassi.sassi_nccl_get_unique_id()
    comm = sassi.sassi_nccl_comm_create(1, 0, uid, 0)
    ctx.merge(comm)
    sassi.sassi_nccl_comm_destroy(comm)
    dyn, dropped = ctx.read_dynamic_pcs()
    odyn, odrop = oracle.dynamic_pcs(s0, hs)
    assert [[int(e["pc"]), int(e["warp_execs"]), int(e["thread_execs"])] for e in dyn] == odyn.tolist()
    ctx.close()

if PART in ("all", "r2"):
    # round 2: global mode (site table beyond shared memory), the merge kernels for 3 contexts on
    # one device, GLOBAL-only address rows, top-K selection, repeated NCCL merges (device check)
    s3 = np.zeros(5000, dtype=oracle.SITE_DTYPE)
    s3["pc"] = 0x1000 + 16 * np.arange(5000)
    s3["flags"] = oracle.F_NUMERIC
    s3["n_gpr_dst"] = 4
    rng = np.random.default_rng(9)
    h3 = np.zeros((4000, 4), np.uint32)
    h3[:, 0] = s3["pc"][rng.integers(0, 5000, 4000)]
    h3[:, 1] = rng.integers(0, 8, 4000)
    h3[:, 2] = rng.integers(0, 2**32, 4000, dtype=np.uint64).astype(np.uint32)
    h3[:, 3] = 0xFFFFFFFF
    h3 = h3.view(oracle.HDR_DTYPE).reshape(-1)
    v3 = rng.integers(0, 64, (16000, 32)).astype(np.uint32)
    t = gpu_table(s3, 8, 31, to_device(s3, h3, None, v3))
    assert np.array_equal(t, oracle.run(s3, 8, 31, h3, None, v3))
    s2, W, h2, a2, v2 = random_trace(777, n=3000, n_warps=6)
    ctxs = []
    for r in range(3):
        keep = h2["warp"] % 3 == r
        sel = np.nonzero(keep)[0]
        site = {int(x["pc"]): x for x in s2}
        na = np.cumsum([0] + [1 if int(p) in site and int(site[int(p)]["flags"]) & oracle.F_MEM else 0 for p in h2["pc"]])
        nv = np.cumsum([0] + [int(site[int(p)]["n_gpr_dst"]) if int(p) in site else 0 for p in h2["pc"]])
        ar = np.concatenate([np.arange(na[i], na[i + 1]) for i in sel]).astype(np.int64)
        vr = np.concatenate([np.arange(nv[i], nv[i + 1]) for i in sel]).astype(np.int64)
        c = sassi.Context(s2, W, 31)
        c.consume(to_device(s2, h2[sel], a2[ar], v2[vr]))
        ctxs.append(c)
    sassi.sassi_merge_local(ctxs)
    want = oracle.run(s2, W, 31, h2, a2, v2)
    for c in ctxs:
        assert np.array_equal(c.read_tables(), want)
    d2 = gen.split_global_rows(dict(to_device(s2, h2, a2, v2), sites=s2))
    c = ctxs[0]
    c.reset()
    c.set_addr_rows(sassi.SASSI_ADDR_ROWS_GLOBAL)
    c.consume(d2)
    assert np.array_equal(c.read_tables(), want)
    c.select_memdiv_topk(2)
    uid = sassi.sassi_nccl_get_unique_id()
    comm = sassi.sassi_nccl_comm_create(1, 0, uid, 0)
    for _ in range(2):
        ctxs[1].reset()
        ctxs[1].consume(to_device(s2, h2, a2, v2))
        ctxs[1].merge(comm)
        assert np.array_equal(ctxs[1].read_tables(), want)
    sassi.sassi_nccl_comm_destroy(comm)
    for c in ctxs:
        c.close()

torch.cuda.synchronize()
print("sanitize workload ok")
