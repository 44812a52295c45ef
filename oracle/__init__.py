"""SASSI handler-fold ORACLE — test infrastructure only.

Plain single-threaded C++ (``oracle.cpp``) behind ctypes, plus host-side report formulas
(``reports.py``). Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package; the product package
``paper_conf_isca_stephensonhlejn15_b200`` never does. It shares no code with the CUDA path:
the record layout and table offsets below are re-declared from the written format spec
(``include/sassi.h`` comment block).

Paper: /root/reference/PAPER.md (SASSI, ISCA'15). See oracle.cpp for per-handler citations.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

# ---- record format (spec: include/sassi.h, re-declared) --------------------------------------
SITE_DTYPE = np.dtype([("pc", "<u4"), ("flags", "<u2"), ("mem_width", "u1"), ("domain", "u1"),
                       ("n_gpr_dst", "u1"), ("reg_num", "u1", (4,)), ("reserved", "u1", (3,))])
HDR_DTYPE = np.dtype([("pc", "<u4"), ("warp", "<u4"), ("active", "<u4"), ("mask2", "<u4")])
INJ_DTYPE = np.dtype([("kernel", "<u4"), ("invocation", "<u4"), ("thread", "<u4"),
                      ("reg_seed", "<u4"), ("bit_seed", "<u4"), ("reserved", "<u4"),
                      ("dyn_index", "<u8")])
assert SITE_DTYPE.itemsize == 16 and HDR_DTYPE.itemsize == 16 and INJ_DTYPE.itemsize == 32

F_COND_BRANCH, F_CTRL, F_MEM, F_MEM_READ, F_MEM_WRITE = 1, 2, 4, 8, 16
F_ATOMIC, F_SYNC, F_NUMERIC, F_TEXTURE, F_WRITES_PRED, F_WRITES_CC = 32, 64, 128, 256, 512, 1024
D_GLOBAL, D_SHARED, D_LOCAL, D_CONST, D_TEX = 0, 1, 2, 3, 4
H_BRANCH, H_MEMDIV, H_VALUE, H_INSTCOUNT, H_ALL = 1, 2, 4, 8, 15
H_INSTMIX = 16  # Fig.3 instruction-mix handler
# Fig.3's dynamic_instr_counts[7] order (L193): imix[0..6]
IMIX_NAMES = ("memory", "extended memory", "controlxfer", "sync", "numeric", "texture",
              "total executed")


def layout(n_sites: int, n_warps: int) -> dict:
    """Offsets (u64 words) of the table image, spec include/sassi.h 'TABLE IMAGE'."""
    S, W = int(n_sites), int(n_warps)
    L = {"diag": 0, "br": 8}
    L["mem"] = L["br"] + 5 * S
    L["val"] = L["mem"] + 4 * S
    L["ones"] = L["val"] + 2 * S
    L["zeros"] = L["ones"] + 4 * S
    L["scalar"] = L["zeros"] + 4 * S
    L["h32"] = L["scalar"] + 4 * S
    L["h128"] = L["h32"] + 1024
    L["counts"] = L["h128"] + 1024
    L["mix"] = L["counts"] + 32 * W
    L["imix"] = L["mix"] + S
    L["pcsel"] = L["imix"] + 8
    L["pcmat"] = L["pcsel"] + 4
    L["total"] = L["pcmat"] + 4 * 1024
    return L


def sections(table: np.ndarray, n_sites: int, n_warps: int) -> dict:
    """Named numpy views of a table image."""
    L = layout(n_sites, n_warps)
    S = int(n_sites)
    t = table
    return {
        "diag": t[0:8],
        "br": t[L["br"]:L["mem"]].reshape(S, 5),
        "mem": t[L["mem"]:L["val"]].reshape(S, 4),
        "val": t[L["val"]:L["ones"]].reshape(S, 2),
        "ones": t[L["ones"]:L["zeros"]].reshape(S, 4),
        "zeros": t[L["zeros"]:L["scalar"]].reshape(S, 4),
        "scalar": t[L["scalar"]:L["h32"]].reshape(S, 4),
        "h32": t[L["h32"]:L["h128"]].reshape(32, 32),
        "h128": t[L["h128"]:L["counts"]].reshape(32, 32),
        "counts": t[L["counts"]:L["mix"]],
        "mix": t[L["mix"]:L["imix"]],
        "imix": t[L["imix"]:L["pcsel"]],
        "pcsel": t[L["pcsel"]:L["pcmat"]],
        "pcmat": t[L["pcmat"]:L["total"]].reshape(4, 32, 32),
    }


def build(force: bool = False) -> str:
    """Compile oracle.cpp -> liboracle.so with g++ (plain -O2, no threads, no intrinsics)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        subprocess.check_call(["g++", "-O2", "-std=c++20", "-Wall", "-Wextra", "-shared", "-fPIC",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u32, u64, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p
        L.oracle_table_words.argtypes = [u32, u32]
        L.oracle_table_words.restype = u64
        L.oracle_table_init.argtypes = [u32, u32, u32, vp]
        L.oracle_table_init.restype = None
        L.oracle_consume.argtypes = [vp, u32, u32, u32, vp, u64, vp, u64, vp, u64, vp]
        L.oracle_consume.restype = ctypes.c_int
        L.oracle_merge.argtypes = [vp, vp, u32, u32]
        L.oracle_merge.restype = None
        L.oracle_sample.argtypes = [vp, u64, u32, u64, vp]
        L.oracle_sample.restype = ctypes.c_int
        L.oracle_sample_multi.argtypes = [vp, vp, vp, vp, u32, u32, u64, vp]
        L.oracle_sample_multi.restype = ctypes.c_int
        L.oracle_splitmix64.argtypes = [u64]
        L.oracle_splitmix64.restype = u64
        L.oracle_select_pcs.argtypes = [u32, u32, vp, u32, vp]
        L.oracle_select_pcs.restype = None
        L.oracle_dynamic_pcs.argtypes = [vp, u32, vp, u64, vp, u64, vp]
        L.oracle_dynamic_pcs.restype = u64
        L.oracle_memdiv_topk.argtypes = [vp, u32, u32, vp, u32, vp]
        L.oracle_memdiv_topk.restype = u32
        L.oracle_locate_injection.argtypes = [vp, u32, vp, u64, vp, u64, u64, u32, u32, vp]
        L.oracle_locate_injection.restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None or a.size == 0 else a.ctypes.data


def table_init(n_sites: int, n_warps: int, handler_mask: int, pcs=()) -> np.ndarray:
    """Fresh table; `pcs` = up to 4 site indices whose per-PC memdiv matrices are kept."""
    L = lib()
    t = np.zeros(int(L.oracle_table_words(n_sites, n_warps)), dtype=np.uint64)
    L.oracle_table_init(n_sites, n_warps, handler_mask, t.ctypes.data)
    if len(pcs):
        sel = np.ascontiguousarray(pcs, dtype=np.uint32)
        L.oracle_select_pcs(n_sites, n_warps, sel.ctypes.data, len(sel), t.ctypes.data)
    return t


def consume(table: np.ndarray, sites: np.ndarray, n_warps: int, handler_mask: int,
            hdr: np.ndarray, addr: np.ndarray | None, val: np.ndarray | None,
            n_addr_rows: int | None = None, n_val_rows: int | None = None) -> np.ndarray:
    """Fold records into ``table`` in place (and return it). addr: [rows,32] u64; val: [rows,32] u32.
    A row array may be None when no attached handler reads it; pass its row count instead."""
    sites = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    hdr = np.ascontiguousarray(hdr, dtype=HDR_DTYPE)
    na = (0 if addr is None else np.asarray(addr).reshape(-1, 32).shape[0]) if n_addr_rows is None else n_addr_rows
    nv = (0 if val is None else np.asarray(val).reshape(-1, 32).shape[0]) if n_val_rows is None else n_val_rows
    addr = None if addr is None else np.ascontiguousarray(addr, np.uint64)
    val = None if val is None else np.ascontiguousarray(val, np.uint32)
    assert table.dtype == np.uint64 and table.flags.c_contiguous
    rc = lib().oracle_consume(sites.ctypes.data, len(sites), n_warps, handler_mask,
                              _ptr(hdr), len(hdr), _ptr(addr), na, _ptr(val), nv,
                              table.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_consume: record stream inconsistent with its rows (rc=%d)" % rc)
    return table


def run(sites, n_warps, handler_mask, hdr, addr=None, val=None, pcs=()) -> np.ndarray:
    """Fresh table + one consume."""
    t = table_init(len(sites), n_warps, handler_mask, pcs)
    return consume(t, sites, n_warps, handler_mask, hdr, addr, val)


def merge(dst: np.ndarray, src: np.ndarray, n_sites: int, n_warps: int) -> np.ndarray:
    lib().oracle_merge(dst.ctypes.data, np.ascontiguousarray(src).ctypes.data, n_sites, n_warps)
    return dst


def sample(counts: np.ndarray, k: int, seed: int) -> np.ndarray:
    counts = np.ascontiguousarray(counts, dtype=np.uint64)
    out = np.zeros(k, dtype=INJ_DTYPE)
    rc = lib().oracle_sample(counts.ctypes.data, counts.size, k, seed & (2**64 - 1),
                             out.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_sample: no eligible dynamic instruction to sample")
    return out


def memdiv_topk(table: np.ndarray, sites, n_warps: int, k: int) -> list:
    """Site indices of the k most divergent GLOBAL memory sites of a table (reading R26)."""
    sites = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    out = np.zeros(max(k, 1), np.uint32)
    n = lib().oracle_memdiv_topk(sites.ctypes.data, len(sites), n_warps,
                                 np.ascontiguousarray(table).ctypes.data, k, out.ctypes.data)
    return [int(x) for x in out[:n]]


def sample_multi(profiles, k: int, seed: int) -> np.ndarray:
    """Draws over several kernel invocations: profiles = [(counts, kernel, invocation), ...]."""
    counts = np.ascontiguousarray(np.concatenate([np.asarray(c, np.uint64) for c, _, _ in profiles]))
    nt = np.array([len(c) for c, _, _ in profiles], np.uint64)
    ke = np.array([kk for _, kk, _ in profiles], np.uint32)
    iv = np.array([ii for _, _, ii in profiles], np.uint32)
    out = np.zeros(k, dtype=INJ_DTYPE)
    rc = lib().oracle_sample_multi(counts.ctypes.data, nt.ctypes.data, ke.ctypes.data, iv.ctypes.data,
                                   len(profiles), k, seed & (2**64 - 1), out.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_sample_multi: no eligible dynamic instruction to sample")
    return out


def splitmix64(x: int) -> int:
    return int(lib().oracle_splitmix64(x & (2**64 - 1)))


def locate_injection(sites, hdr, val, thread: int, dyn_index: int, reg_seed: int, bit_seed: int):
    """§8.1 step (3) (L631): the dyn_index-th eligible, not-predicated-out dynamic instruction of
    `thread` in a warp-major record stream -> dict(record, site, target ('gpr' | 'mem' | 'pred' |
    'cc'), before, bit), or None when the thread has fewer. See oracle.cpp (reading R23)."""
    sites = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    hdr = np.ascontiguousarray(hdr, dtype=HDR_DTYPE)
    val = None if val is None else np.ascontiguousarray(val, np.uint32)
    out = np.zeros(5, np.uint64)
    rc = lib().oracle_locate_injection(sites.ctypes.data, len(sites), _ptr(hdr), len(hdr), _ptr(val),
                                       thread, dyn_index, reg_seed & 0xFFFFFFFF,
                                       bit_seed & 0xFFFFFFFF, out.ctypes.data)
    if rc != 0:
        return None
    return {"record": int(out[0]), "site": int(out[1]),
            "target": ("gpr", "mem", "pred", "cc")[int(out[2])], "before": int(out[3]),
            "bit": int(out[4])}


def dynamic_pcs(sites, hdr):
    """Insert-on-miss table of the unregistered pcs (Fig.4 l.21-23, DESIGN R25), sorted by pc:
    -> (uint64 array [n][3] = pc, warp executions, thread executions; records with the reserved
    pc 0xFFFFFFFF)."""
    sites = np.ascontiguousarray(sites)
    hdr = np.ascontiguousarray(hdr)
    dropped = np.zeros(1, np.uint64)
    n = lib().oracle_dynamic_pcs(_ptr(sites), len(sites), _ptr(hdr), len(hdr), None, 0,
                                 _ptr(dropped))
    out = np.zeros((max(int(n), 1), 3), np.uint64)
    lib().oracle_dynamic_pcs(_ptr(sites), len(sites), _ptr(hdr), len(hdr), _ptr(out), int(n),
                             _ptr(dropped))
    return out[:int(n)], int(dropped[0])
