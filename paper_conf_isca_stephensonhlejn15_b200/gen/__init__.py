"""Seeded synthetic SASSI record streams (SRF1) — the input generator shared by tests and bench.

This module holds NONE of the handler arithmetic: it only builds site tables and record streams
(headers, address rows, value rows, chunk index) from a program model, on the host
(``libsassi_gen_host.so``, gcc) or on the device (``libsassi_gen.so``, nvcc) from ONE C source
(``sassi_gen.h``), so both produce identical bytes. Workload presets c1..c5 follow
BASELINE.json ``configs`` and DESIGN.md §5 ("Input recipe").
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_PKG = os.path.dirname(_HERE)
HOST_LIB = os.path.join(_PKG, "lib", "libsassi_gen_host.so")
DEV_LIB = os.path.join(_PKG, "lib", "libsassi_gen.so")

CHUNK = 256  # SASSI_CHUNK

# --- SRF1 site record (format spec include/sassi.h) ----------------------------------------------
SITE_DTYPE = np.dtype([("pc", "<u4"), ("flags", "<u2"), ("mem_width", "u1"), ("domain", "u1"),
                       ("n_gpr_dst", "u1"), ("reg_num", "u1", (4,)), ("reserved", "u1", (3,))])
HDR_DTYPE = np.dtype([("pc", "<u4"), ("warp", "<u4"), ("active", "<u4"), ("mask2", "<u4")])

F_COND_BRANCH, F_CTRL, F_MEM, F_MEM_READ, F_MEM_WRITE = 1, 2, 4, 8, 16
F_ATOMIC, F_SYNC, F_NUMERIC, F_TEXTURE, F_WRITES_PRED, F_WRITES_CC = 32, 64, 128, 256, 512, 1024
D_GLOBAL, D_SHARED, D_LOCAL, D_CONST, D_TEX = 0, 1, 2, 3, 4

# --- generator structs (sassi_gen.h) -------------------------------------------------------------
OP_DTYPE = np.dtype([("pc", "<u4"), ("parent", "<i4"), ("is_branch", "u1"), ("is_mem", "u1"),
                     ("n_dst", "u1"), ("mask_model", "u1"), ("addr_model", "u1"),
                     ("val_model", "u1", (4,)), ("pad0", "u1", (3,)), ("mask_p0", "<u4"),
                     ("mask_p1", "<u4"), ("pad1", "<u4"), ("addr_base", "<u8"), ("addr_p0", "<u8"),
                     ("addr_p1", "<u8"), ("val_p0", "<u4", (4,)), ("val_p1", "<u4", (4,))])
PROG_DTYPE = np.dtype([("seed", "<u8"), ("warp_base", "<u4"), ("n_warps", "<u4"),
                       ("total_warps", "<u4"), ("last_warp_lanes", "<u4"), ("trip_model", "<u4"),
                       ("trip_p0", "<u4"), ("trip_p1", "<u4"), ("trip_p2", "<u4"),
                       ("base_model", "<u4"), ("base_p0", "<u4"), ("n_pro", "<u4"),
                       ("n_body", "<u4"), ("n_epi", "<u4"), ("pad", "<u4")])
assert OP_DTYPE.itemsize == 88 and PROG_DTYPE.itemsize == 64

TRIP_FIXED, TRIP_UNIFORM, TRIP_HEAVY = 0, 1, 2
BASE_FULL, BASE_FRONTIER = 0, 1
T_NONE, T_ALL, T_UNIFORM, T_DIVERGE, T_MOD, T_LOOP, T_WARPMOD = 0, 1, 2, 3, 4, 5, 6
G_ALL, G_BERN, G_NOISE = 0, 1, 2
A_NONE, A_UNIT, A_BCAST, A_STRIDE, A_GATHER, A_FAR, A_WINDOW = 0, 1, 2, 3, 4, 5, 6
(V_CONST, V_ELEM, V_SMALL, V_RAND, V_FLOAT, V_ITER, V_LANE, V_BOOL, V_WSCALAR, V_ADDR_LO,
 V_ADDR_HI) = range(11)
MAX_OPS = 256


def prob(p: float) -> int:
    """Probability as a u32 threshold (x < prob(p) happens w.p. p for uniform u32 x)."""
    return int(min(max(p, 0.0), 1.0) * 4294967295.0)


class Program:
    """A synthetic instrumented kernel: prologue / body (x trips) / epilogue of static sites."""

    def __init__(self, name: str, seed: int, total_warps: int, last_warp_lanes: int = 32,
                 trip=(TRIP_FIXED, 1, 0, 0), base=(BASE_FULL, 0), pc0: int = 0x100):
        self.name = name
        self.seed = seed
        self.total_warps = total_warps
        self.last_warp_lanes = last_warp_lanes
        self.trip = trip
        self.base = base
        self.ops = {0: [], 1: [], 2: []}
        self._pc = pc0
        self._sites = []

    def op(self, sec: int, *, flags: int = 0, n_dst: int = 0, domain: int = D_GLOBAL,
           width: int = 0, mask=(0, 0, 0), addr=(A_NONE, 0, 0, 0), vals=(), parent: int = -1,
           regs=None, pc=None) -> int:
        """Append one static instruction to section sec (0 pro, 1 body, 2 epi); returns its index.
        mask=(model, p0, p1); addr=(model, base, p0, p1); vals=[(model, p0, p1)] * n_dst."""
        if pc is None:
            pc = self._pc
            self._pc += 16
        j = len(self.ops[sec])
        assert j < MAX_OPS
        if parent >= 0:
            assert parent < j and self.ops[sec][parent]["is_branch"], "parent must be an earlier branch"
        vals = list(vals) + [(V_CONST, 0, 0)] * (4 - len(vals))
        if regs is None:
            regs = [(len(self._sites) * 2 + d) % 250 for d in range(4)]
        o = dict(pc=pc, parent=parent, is_branch=int(bool(flags & F_COND_BRANCH)),
                 is_mem=int(bool(flags & F_MEM)), n_dst=n_dst, mask_model=mask[0],
                 mask_p0=mask[1], mask_p1=mask[2], addr_model=addr[0], addr_base=addr[1],
                 addr_p0=addr[2], addr_p1=addr[3] if len(addr) > 3 else 0,
                 val_model=[v[0] for v in vals], val_p0=[v[1] for v in vals],
                 val_p1=[v[2] for v in vals])
        self.ops[sec].append(o)
        self._sites.append(dict(pc=pc, flags=flags, mem_width=width, domain=domain, n_gpr_dst=n_dst,
                                reg_num=list(regs)[:4] + [0] * (4 - len(list(regs)[:4]))))
        return j

    # -- arrays for the C generator / the site registry --
    def sites(self) -> np.ndarray:
        s = np.zeros(len(self._sites), dtype=SITE_DTYPE)
        for i, d in enumerate(self._sites):
            for k, v in d.items():
                s[i][k] = v
        return s

    def op_array(self) -> np.ndarray:
        allops = self.ops[0] + self.ops[1] + self.ops[2]
        a = np.zeros(max(1, len(allops)), dtype=OP_DTYPE)
        for i, o in enumerate(allops):
            for k, v in o.items():
                a[i][k] = v
        return a

    def prog_array(self, warp_base: int = 0, n_warps=None) -> np.ndarray:
        p = np.zeros(1, dtype=PROG_DTYPE)
        p["seed"] = self.seed
        p["warp_base"] = warp_base
        p["n_warps"] = self.total_warps - warp_base if n_warps is None else n_warps
        p["total_warps"] = self.total_warps
        p["last_warp_lanes"] = self.last_warp_lanes
        p["trip_model"], p["trip_p0"], p["trip_p1"], p["trip_p2"] = self.trip
        p["base_model"], p["base_p0"] = self.base
        p["n_pro"], p["n_body"], p["n_epi"] = len(self.ops[0]), len(self.ops[1]), len(self.ops[2])
        return p


# --- host generator ------------------------------------------------------------------------------
_host = None
_dev = None


def _host_lib():
    global _host
    if _host is None:
        if not os.path.exists(HOST_LIB):
            raise RuntimeError("generator host library missing: run __graft_entry__.build()")
        L = ctypes.CDLL(HOST_LIB)
        vp, u64 = ctypes.c_void_p, ctypes.c_uint64
        L.sassi_gen_count_host.argtypes = [vp, vp, vp]
        L.sassi_gen_emit_host.argtypes = [vp, vp, vp, u64, vp, vp, vp, vp]
        L.sassi_gen_hash_host.argtypes = [u64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                          ctypes.c_uint32, ctypes.c_uint32]
        L.sassi_gen_hash_host.restype = u64
        assert L.sassi_gen_sizeof_op() == OP_DTYPE.itemsize
        assert L.sassi_gen_sizeof_prog() == PROG_DTYPE.itemsize
        _host = L
    return _host


def _dev_lib():
    global _dev
    if _dev is None:
        if not os.path.exists(DEV_LIB):
            raise RuntimeError("generator device library missing: run __graft_entry__.build()")
        L = ctypes.CDLL(DEV_LIB)
        vp, u64 = ctypes.c_void_p, ctypes.c_uint64
        L.sassi_gen_count.argtypes = [vp, vp, vp, vp]
        L.sassi_gen_emit.argtypes = [vp, vp, vp, u64, vp, vp, vp, vp, vp]
        _dev = L
    return _dev


def _offsets(counts: np.ndarray):
    offs = np.zeros_like(counts)
    offs[1:] = np.cumsum(counts, axis=0)[:-1]
    tot = counts.sum(axis=0)
    return offs, int(tot[0]), int(tot[1]), int(tot[2])


def count_host(program: Program, warp_base: int = 0, n_warps=None) -> np.ndarray:
    P = program.prog_array(warp_base, n_warps)
    ops = program.op_array()
    out = np.zeros((int(P["n_warps"][0]), 3), dtype=np.uint64)
    _host_lib().sassi_gen_count_host(P.ctypes.data, ops.ctypes.data, out.ctypes.data)
    return out


def generate_host(program: Program, limit=None, warp_base: int = 0, n_warps=None) -> dict:
    """Generate the stream of warps [warp_base, warp_base+n_warps) on the host (numpy)."""
    P = program.prog_array(warp_base, n_warps)
    ops = program.op_array()
    counts = count_host(program, warp_base, n_warps)
    offs, n_tot, a_tot, v_tot = _offsets(counts)
    n = n_tot if limit is None else min(int(limit), n_tot)
    nch = (n + CHUNK - 1) // CHUNK
    hdr = np.zeros((n, 4), dtype=np.uint32)
    cb = np.zeros((nch + 1, 2), dtype=np.uint64)
    # rows: allocate full totals, trim after the walk using the sentinel
    addr = np.zeros((a_tot, 32), dtype=np.uint64)
    val = np.zeros((v_tot, 32), dtype=np.uint32)
    if n == n_tot:
        cb[nch] = (a_tot, v_tot)
    _host_lib().sassi_gen_emit_host(P.ctypes.data, ops.ctypes.data, offs.ctypes.data, n,
                                    hdr.ctypes.data, addr.ctypes.data if a_tot else None,
                                    val.ctypes.data if v_tot else None, cb.ctypes.data)
    na, nv = int(cb[nch][0]), int(cb[nch][1])
    return dict(sites=program.sites(), n_warps_total=program.total_warps,
                hdr=hdr.view(HDR_DTYPE).reshape(n), addr=addr[:na], val=val[:nv], chunk_base=cb,
                n=n, n_addr_rows=na, n_val_rows=nv, counts=counts)


def generate_device(program: Program, limit=None, warp_base: int = 0, n_warps=None,
                    device=None) -> dict:
    """Generate on the GPU (torch tensors as plain device memory; generation is untimed)."""
    import torch
    dev = torch.device("cuda" if device is None else device)
    P = program.prog_array(warp_base, n_warps)
    ops = program.op_array()
    W = int(P["n_warps"][0])
    L = _dev_lib()
    with torch.cuda.device(dev):
        stream = torch.cuda.current_stream(dev).cuda_stream
        cnt_d = torch.zeros((W, 3), dtype=torch.int64, device=dev)
        rc = L.sassi_gen_count(P.ctypes.data, ops.ctypes.data, cnt_d.data_ptr(), stream)
        if rc != 0:
            raise RuntimeError("sassi_gen_count failed (%d)" % rc)
        counts = cnt_d.cpu().numpy().view(np.uint64)
        offs, n_tot, a_tot, v_tot = _offsets(counts)
        n = n_tot if limit is None else min(int(limit), n_tot)
        nch = (n + CHUNK - 1) // CHUNK
        offs_d = torch.from_numpy(offs.view(np.int64)).to(dev)
        if n < n_tot:  # rows needed: at most up to the end of the warp holding record n
            wl = int(np.searchsorted(offs[:, 0], n, side="right"))
            a_cap = int(offs[wl, 1]) if wl < len(offs) else a_tot
            v_cap = int(offs[wl, 2]) if wl < len(offs) else v_tot
        else:
            a_cap, v_cap = a_tot, v_tot
        hdr = torch.empty((max(n, 1), 4), dtype=torch.int32, device=dev)
        addr = torch.empty((max(a_cap, 1), 32), dtype=torch.int64, device=dev)
        val = torch.empty((max(v_cap, 1), 32), dtype=torch.int32, device=dev)
        cb = torch.zeros((nch + 1, 2), dtype=torch.int64, device=dev)
        if n == n_tot:
            cb[nch, 0] = a_tot
            cb[nch, 1] = v_tot
        rc = L.sassi_gen_emit(P.ctypes.data, ops.ctypes.data, offs_d.data_ptr(), n, hdr.data_ptr(),
                              addr.data_ptr(), val.data_ptr(), cb.data_ptr(), stream)
        if rc != 0:
            raise RuntimeError("sassi_gen_emit failed (%d)" % rc)
        tail = cb[nch].cpu().numpy()
        na, nv = int(tail[0]), int(tail[1])
    return dict(sites=program.sites(), n_warps_total=program.total_warps, hdr=hdr[:n],
                addr=addr[:na], val=val[:nv], chunk_base=cb, n=n, n_addr_rows=na, n_val_rows=nv,
                counts=counts)


def to_host(rec: dict) -> dict:
    """Device stream -> numpy arrays in the host layout (for the oracle)."""
    out = dict(rec)
    out["hdr"] = rec["hdr"].cpu().numpy().view(np.uint32).reshape(-1, 4).view(HDR_DTYPE).reshape(-1)[: rec["n"]]
    out["addr"] = rec["addr"].cpu().numpy().view(np.uint64).reshape(-1, 32)[: rec["n_addr_rows"]]
    out["val"] = rec["val"].cpu().numpy().view(np.uint32).reshape(-1, 32)[: rec["n_val_rows"]]
    out["chunk_base"] = rec["chunk_base"].cpu().numpy().view(np.uint64)
    return out


def split_global_rows(rec: dict) -> dict:
    """The producer-side split of SASSI_ADDR_ROWS_GLOBAL (include/sassi.h): keep only the address
    rows of GLOBAL memory sites (the rows of shared / local memory sites go to a stream of their own
    that the fold never reads) and rebuild chunk_base's addr_row column over the kept rows. Works on
    device (torch) and host (numpy) streams; input preparation only, no handler arithmetic."""
    sites = rec["sites"]
    order = np.argsort(sites["pc"].astype(np.int64))
    spc = sites["pc"].astype(np.int64)[order]
    mem = (sites["flags"][order].astype(np.int64) & F_MEM) != 0
    glob = mem & (sites["domain"][order] == D_GLOBAL)
    n = rec["n"]
    if isinstance(rec["hdr"], np.ndarray):
        pc = rec["hdr"]["pc"].astype(np.int64)[:n]
        idx = np.minimum(np.searchsorted(spc, pc), max(len(spc) - 1, 0))
        hit = (spc[idx] == pc) if len(spc) else np.zeros(n, bool)
        has_row, is_g = hit & mem[idx], hit & glob[idx]
        keep = is_g[has_row]
        cum = np.concatenate([[0], np.cumsum(is_g)]).astype(np.uint64)
        cb = rec["chunk_base"].copy()
        cb[:, 0] = cum[np.minimum(np.arange(len(cb)) * CHUNK, n)]
        addr = rec["addr"][keep]
    else:
        import torch
        dev = rec["hdr"].device
        tspc = torch.from_numpy(spc).to(dev)
        pc = rec["hdr"][:n, 0].to(torch.int64) & 0xFFFFFFFF
        idx = torch.clamp(torch.searchsorted(tspc, pc), max=max(len(spc) - 1, 0))
        hit = tspc[idx] == pc
        has_row = hit & torch.from_numpy(mem).to(dev)[idx]
        is_g = hit & torch.from_numpy(glob).to(dev)[idx]
        keep = is_g[has_row]
        cum = torch.cat([torch.zeros(1, dtype=torch.int64, device=dev), torch.cumsum(is_g.to(torch.int64), 0)])
        cb = rec["chunk_base"].clone()
        pos = torch.clamp(torch.arange(cb.shape[0], device=dev) * CHUNK, max=n)
        cb[:, 0] = cum[pos]
        addr = rec["addr"][: rec["n_addr_rows"]][keep]
    return dict(rec, addr=addr, chunk_base=cb, n_addr_rows=int(keep.sum()))


def stream_bytes(rec: dict, handler_mask: int) -> dict:
    """Algorithmic bytes the fold must read for this stream and handler mask:
    16 B per header + 256 B per addr row of a GLOBAL memory site when MEMDIV is attached +
    128 B per val row when VALUE is attached. Counted from the stream itself."""
    sites = rec["sites"]
    hdr = rec["hdr"] if isinstance(rec["hdr"], np.ndarray) else None
    out = {"hdr": 16 * rec["n"], "addr_global": 0, "addr_all": 256 * rec["n_addr_rows"],
           "val": 128 * rec["n_val_rows"]}
    if hdr is None:
        return out
    pcs = {int(s["pc"]): s for s in sites}
    glob = np.array([int(s["pc"]) for s in sites
                     if (int(s["flags"]) & F_MEM) and int(s["domain"]) == D_GLOBAL], dtype=np.uint32)
    out["addr_global"] = 256 * int(np.isin(hdr["pc"], glob).sum())
    return out


from .presets import preset, PRESETS  # noqa: E402,F401
