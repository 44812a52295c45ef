"""Multi-rank host logic on CPU (gloo, world size 2): the warp-shard split, the packed-image merge
protocol that sassi_merge implements with one sum-allreduce (byte-expanded AND masks, isScalar as
0/1 sums), and the max-over-ranks timing reduction used by bench.py. The per-rank folds use the
oracle; the merged result must equal the single-pass oracle bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen


def pack(t, S, W):
    """The packed image documented in csrc/merge.cu."""
    L = oracle.layout(S, W)
    masks = t[L["ones"]:L["scalar"]].astype(np.uint32)               # ones[S][4], zeros[S][4]
    bits = np.unpackbits(masks.view(np.uint8).reshape(-1, 4), axis=1, bitorder="little")
    expanded = bits.astype(np.uint8).reshape(-1, 32).view(np.uint64).reshape(-1)  # 4 words / mask
    return np.concatenate([t[0:4], t[L["br"]:L["ones"]], t[L["h32"]:L["pcsel"]],
                           t[L["pcmat"]:L["total"]], t[L["scalar"]:L["h32"]],
                           expanded]).astype(np.uint64)


def unpack(pk, t, S, W, nranks):
    L = oracle.layout(S, W)
    out = t.copy()
    a = L["ones"] - L["br"]
    b1 = L["pcsel"] - L["h32"]
    b = b1 + (L["total"] - L["pcmat"])               # the pc selection (pcsel) is not summed
    out[0:4] = pk[0:4]
    out[L["br"]:L["ones"]] = pk[4:4 + a]
    out[L["h32"]:L["pcsel"]] = pk[4 + a:4 + a + b1]
    out[L["pcmat"]:L["total"]] = pk[4 + a + b1:4 + a + b]
    out[L["scalar"]:L["h32"]] = (pk[4 + a + b:4 + a + b + 4 * S] == nranks).astype(np.uint64)
    bytes_ = pk[4 + a + b + 4 * S:].view(np.uint8).reshape(-1, 32)
    bits = (bytes_ == nranks).astype(np.uint8)
    out[L["ones"]:L["scalar"]] = np.packbits(bits, axis=1, bitorder="little").view(np.uint32).reshape(-1)
    return out


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    P, _, mask, _ = gen.preset("c5")
    per = 3                                          # tiny: 3 warps per rank
    P.total_warps = per * world
    r = gen.generate_host(P, None, rank * per, per)
    S, W = len(r["sites"]), P.total_warps
    t = oracle.run(r["sites"], W, mask, r["hdr"], r["addr"], r["val"])
    pk = torch.from_numpy(pack(t, S, W).view(np.int64).copy())
    dist.all_reduce(pk, op=dist.ReduceOp.SUM)        # the single collective of sassi_merge
    merged = unpack(pk.numpy().view(np.uint64), t, S, W, world)
    # max-over-ranks timing, as bench.py reports it
    tt = torch.tensor([float(rank + 1)])
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    q.put((rank, merged, float(tt.item())))
    dist.destroy_process_group()


def test_two_rank_merge_equals_single_pass():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    P, _, mask, _ = gen.preset("c5")
    P.total_warps = 3 * world
    whole = gen.generate_host(P, None, 0, 3 * world)
    S, W = len(whole["sites"]), P.total_warps
    single = oracle.run(whole["sites"], W, mask, whole["hdr"], whole["addr"], whole["val"])
    for rank, merged, tmax in res:
        assert np.array_equal(merged, single), rank
        assert tmax == float(world)


def test_pack_roundtrip_single_rank():
    s = oracle.SITE_DTYPE
    import t0_trace as T0
    sites = T0.sites()
    hdr, addr, val = T0.records()
    t = oracle.run(sites, T0.N_WARPS, oracle.H_ALL, hdr, addr, val)
    assert np.array_equal(unpack(pack(t, 7, 2), t, 7, 2, 1), t)
