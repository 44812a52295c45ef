"""GPU: the multi-GPU merge kernels at nranks > 1, bit-exact against the single-pass oracle.

sassi_merge packs each rank's table image (AND masks byte-expanded, isScalar as 0/1), sums the
packed images with one ncclAllReduce and unpacks them with `byte == nranks` (north_star subsystem 5,
DESIGN.md §9). NCCL cannot put two ranks on one GPU, so sassi_merge_local runs the same pack and
unpack kernels for P contexts on this GPU with the allreduce replaced by a device sum: P warp shards
folded into P contexts, merged, must equal the oracle's fold of the whole trace in every context
(every table section, the per-PC matrices and the dynamic-pc table), for P = 2, 3 and 8."""
import numpy as np
import pytest

import oracle
from gpu_helpers import to_device, diff_tables
from test_oracle import random_trace
from paper_conf_isca_stephensonhlejn15_b200 import sassi

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def shard_by_warp(s, hdr, addr, val, P):
    """The records of warps w with w % P == r (rows kept with their records), r = 0..P-1."""
    site = {int(x["pc"]): x for x in s}
    na = np.array([1 if int(p) in site and int(site[int(p)]["flags"]) & oracle.F_MEM else 0
                   for p in hdr["pc"]], np.int64)
    nv = np.array([int(site[int(p)]["n_gpr_dst"]) if int(p) in site else 0 for p in hdr["pc"]], np.int64)
    a0 = np.concatenate([[0], np.cumsum(na)])
    v0 = np.concatenate([[0], np.cumsum(nv)])
    out = []
    for r in range(P):
        idx = np.nonzero(hdr["warp"] % P == r)[0]
        ar = np.concatenate([np.arange(a0[i], a0[i] + na[i]) for i in idx] or [np.zeros(0, np.int64)])
        vr = np.concatenate([np.arange(v0[i], v0[i] + nv[i]) for i in idx] or [np.zeros(0, np.int64)])
        out.append((hdr[idx], addr[ar.astype(np.int64)].reshape(-1, 32), val[vr.astype(np.int64)].reshape(-1, 32)))
    return out


def _global_mem_sites(s):
    return [i for i in range(len(s)) if (int(s[i]["flags"]) & oracle.F_MEM)
            and int(s[i]["domain"]) == oracle.D_GLOBAL]


@pytest.mark.parametrize("P", [2, 3, 8])
def test_merge_local_equals_single_pass(P):
    s, W, hdr, addr, val = random_trace(7000 + P, n=12000, n_warps=24)
    sel = _global_mem_sites(s)[:4]
    pcs = [int(s[i]["pc"]) for i in sel]
    ctxs = []
    for h, a, v in shard_by_warp(s, hdr, addr, val, P):
        c = sassi.Context(s, W, sassi.SASSI_H_EVERY)
        c.select_memdiv_pcs(pcs)
        c.enable_dynamic_pcs(16)
        if len(h):
            c.consume(to_device(s, h, a, v))
        ctxs.append(c)
    parts = [c.read_tables() for c in ctxs]
    sassi.sassi_merge_local(ctxs)
    o = oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val, pcs=sel)
    dyn, dropped = oracle.dynamic_pcs(s, hdr)
    for c in ctxs:
        t = c.read_tables()
        assert diff_tables(t, o, len(s), W) is None
        d, nd = c.read_dynamic_pcs()
        assert nd == dropped
        assert np.array_equal(np.stack([d["pc"], d["warp_execs"], d["thread_execs"]], 1).astype(np.uint64), dyn)
    # the shards really differ (the merge did work), and the oracle's own merge agrees
    acc = parts[0].copy()
    for t in parts[1:]:
        oracle.merge(acc, t, len(s), W)
    assert not np.array_equal(parts[0], o) and np.array_equal(acc, o)
    for c in ctxs:
        c.close()


@pytest.mark.parametrize("P", [2, 3, 8])
def test_merge_local_mask_byte_levels(P):
    """One value site whose ones / zeros bits are set in exactly k of the P shards for every k:
    shard r < P - 1 writes the constant v_r with bit b set iff r < b % P, shard P - 1 never executes
    the site (its masks stay all-ones, the AND identity), so after the sum every byte level 1..P
    occurs; a bit survives only at level P. A second site is scalar in every shard but one."""
    s = np.zeros(2, dtype=oracle.SITE_DTYPE)
    s["pc"] = [0x10, 0x20]
    s["flags"] = oracle.F_NUMERIC
    s["n_gpr_dst"] = [1, 1]
    W = P
    H, V = [], []
    for r in range(P - 1):
        v_r = sum(1 << b for b in range(32) if r < b % P)
        for rep in range(3):
            H.append((0x10, r, 0xFFFFFFFF, 0xFFFFFFFF))
            V.append(np.full(32, v_r, np.uint32))
    for r in range(P):
        H.append((0x20, r, 0xFFFFFFFF, 0xFFFFFFFF))
        V.append(np.arange(32, dtype=np.uint32) if r == P // 2 else np.full(32, 7, np.uint32))
    hdr = np.array(H, dtype=oracle.HDR_DTYPE)
    val = np.stack(V)
    addr = np.zeros((0, 32), np.uint64)
    o = oracle.run(s, W, sassi.SASSI_H_VALUE, hdr, addr, val)
    so = oracle.sections(o, 2, W)
    ones = int(so["ones"][0, 0])
    assert ones == sum(1 << b for b in range(32) if b % P == P - 1)      # survives only at level P
    assert int(so["zeros"][0, 0]) == sum(1 << b for b in range(32) if b % P == 0)
    assert int(so["scalar"][0, 0]) == 1 and int(so["scalar"][1, 0]) == 0
    ctxs = []
    for h, a, v in shard_by_warp(s, hdr, addr, val, P):
        c = sassi.Context(s, W, sassi.SASSI_H_VALUE)
        c.consume(to_device(s, h, a, v))
        ctxs.append(c)
    sassi.sassi_merge_local(ctxs)
    for c in ctxs:
        assert diff_tables(c.read_tables(), o, 2, W) is None
        c.close()


def test_merge_local_rejects_different_site_tables():
    s, W, hdr, addr, val = random_trace(11, n=500)
    s2 = s.copy()
    s2["pc"][0] += 4
    a, b = sassi.Context(s, W, 15), sassi.Context(s2, W, 15)
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_merge_local([a, b])
    assert e.value.status == sassi.SASSI_EMISMATCH
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_merge_local([a, a])
    assert e.value.status == sassi.SASSI_EINVAL
    a.select_memdiv_pcs([int(s[i]["pc"]) for i in _global_mem_sites(s)[:1]])
    c = sassi.Context(s, W, 15)
    with pytest.raises(sassi.SassiError) as e:     # same sites, another pc selection
        sassi.sassi_merge_local([a, c])
    assert e.value.status == sassi.SASSI_EMISMATCH
    for x in (a, b, c):
        x.close()


def test_nccl_merge_repeated_uses_device_side_check():
    """sassi_merge checks the ranks' checksums on the host the first time a context merges over a
    communicator and on the device afterwards: repeated 1-rank merges (fold, merge, reset, ...)
    keep giving the oracle's tables, with no EMISMATCH."""
    s, W, hdr, addr, val = random_trace(555, n=6000)
    d = to_device(s, hdr, addr, val)
    ctx = sassi.Context(s, W, sassi.SASSI_H_EVERY)
    uid = sassi.sassi_nccl_get_unique_id()
    comm = sassi.sassi_nccl_comm_create(1, 0, uid, torch.cuda.current_device())
    o = oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val)
    for _ in range(3):
        ctx.reset()
        ctx.consume(d)
        ctx.merge(comm)
        assert np.array_equal(ctx.read_tables(), o)
    sassi.sassi_nccl_comm_destroy(comm)
    ctx.close()
