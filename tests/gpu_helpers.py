"""Helpers for the GPU parity tests: move a host record stream to the device, run the CUDA fold
through the C ABI, run the oracle on the same bytes."""
import numpy as np

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

CHUNK = 256


def host_chunk_base(sites, hdr):
    """Chunk index computed on the host from the site table (independent of the device code)."""
    pcs = {int(s["pc"]): s for s in sites}
    n = len(hdr)
    nch = (n + CHUNK - 1) // CHUNK
    cb = np.zeros((nch + 1, 2), np.uint64)
    a = v = 0
    for i, h in enumerate(hdr):
        if i % CHUNK == 0:
            cb[i // CHUNK] = (a, v)
        s = pcs.get(int(h["pc"]))
        if s is not None:
            a += 1 if int(s["flags"]) & gen.F_MEM else 0
            v += int(s["n_gpr_dst"])
    cb[nch] = (a, v)
    return cb


def to_device(sites, hdr, addr, val, chunk_base=None):
    import torch
    hdr = np.ascontiguousarray(hdr).view(np.uint32).reshape(-1, 4)
    addr = np.zeros((0, 32), np.uint64) if addr is None else np.ascontiguousarray(addr, np.uint64)
    val = np.zeros((0, 32), np.uint32) if val is None else np.ascontiguousarray(val, np.uint32)
    if chunk_base is None:
        chunk_base = host_chunk_base(sites, hdr.view(gen.HDR_DTYPE).reshape(-1))
    d = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).cuda()
    return dict(hdr=d(hdr, np.int32), addr=d(addr.reshape(-1, 32), np.int64),
                val=d(val.reshape(-1, 32), np.int32), chunk_base=d(chunk_base, np.int64),
                n=len(hdr), n_addr_rows=len(addr), n_val_rows=len(val))


def gpu_table(sites, n_warps, mask, drec, n=None, pcs=()):
    """One consume through the C ABI; `pcs` = pcs of the per-PC memdiv matrices to keep."""
    ctx = sassi.Context(sites, n_warps, mask)
    try:
        if len(pcs):
            ctx.select_memdiv_pcs(pcs)
        ctx.consume(drec, n)
        return ctx.read_tables()
    finally:
        ctx.close()


def oracle_table(sites, n_warps, mask, hdr, addr, val):
    return oracle.run(sites, n_warps, mask, hdr, addr, val)


def diff_tables(a, b, S, W):
    """Readable first difference between two table images (None if identical)."""
    if np.array_equal(a, b):
        return None
    sa, sb = oracle.sections(a, S, W), oracle.sections(b, S, W)
    for k in sa:
        if not np.array_equal(sa[k], sb[k]):
            idx = np.argwhere(sa[k] != sb[k])[:5]
            return "%s differs at %s: gpu %s oracle %s" % (
                k, idx.tolist(), [int(sa[k][tuple(i)]) for i in idx], [int(sb[k][tuple(i)]) for i in idx])
    return "differs"
