"""Thin ctypes binding of libsassi.so — same names as the C ABI (include/sassi.h).

Argument marshalling only: every step of the fold runs in the CUDA kernels of libsassi.so. Device
buffers are torch tensors (``data_ptr()``), streams are ``torch.cuda.Stream.cuda_stream``. There is
no CPU fallback: if the library or a CUDA device is missing, calls raise ``SassiError``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# SASSI_LIB selects another build of the same library (tools/build_variant.py A/B timing)
LIB_PATH = os.environ.get("SASSI_LIB") or os.path.join(_PKG, "lib", "libsassi.so")

SITE_DTYPE = np.dtype([("pc", "<u4"), ("flags", "<u2"), ("mem_width", "u1"), ("domain", "u1"),
                       ("n_gpr_dst", "u1"), ("reg_num", "u1", (4,)), ("reserved", "u1", (3,))])
INJ_DTYPE = np.dtype([("kernel", "<u4"), ("invocation", "<u4"), ("thread", "<u4"),
                      ("reg_seed", "<u4"), ("bit_seed", "<u4"), ("reserved", "<u4"),
                      ("dyn_index", "<u8")])

SASSI_OK, SASSI_EINVAL, SASSI_ECUDA, SASSI_ENCCL = 0, -1, -2, -3
SASSI_ENOSPC, SASSI_ESTATE, SASSI_EMISMATCH, SASSI_EFORMAT = -4, -5, -6, -7
SASSI_H_BRANCH, SASSI_H_MEMDIV, SASSI_H_VALUE, SASSI_H_INSTCOUNT, SASSI_H_ALL = 1, 2, 4, 8, 15
SASSI_H_INSTMIX, SASSI_H_EVERY = 16, 31
SASSI_CHUNK = 256
SASSI_ADDR_ROWS_ALL, SASSI_ADDR_ROWS_GLOBAL = 0, 1
SASSI_IK_VECADD, SASSI_IK_BFS, SASSI_IK_SGEMM, SASSI_IK_STENCIL = 0, 1, 2, 3
SASSI_IK_NONE, SASSI_IK_TRACE, SASSI_IK_NULL_ABI, SASSI_IK_SMEM = 0, 64, 128, 1024

# every function declared in include/*.h: name -> (restype, argtypes)
_vp, _u32, _u64, _i = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int


class SassiRecords(ctypes.Structure):
    _fields_ = [("hdr", _vp), ("addr", _vp), ("val", _vp), ("chunk_base", _vp),
                ("n_addr_rows", _u64), ("n_val_rows", _u64)]


class SassiLayout(ctypes.Structure):
    _fields_ = [(k, _u64) for k in ("diag", "br", "mem", "val", "ones", "zeros", "scalar", "h32",
                                    "h128", "counts", "mix", "imix", "pcsel", "pcmat", "total")]


SIGNATURES = {
    "sassi_table_layout": (_i, [_u32, _u32, ctypes.POINTER(SassiLayout)]),
    "sassi_ctx_create": (_i, [ctypes.POINTER(_vp), _i, _vp, _u32, _u32]),
    "sassi_ctx_destroy": (None, [_vp]),
    "sassi_attach_handler": (_i, [_vp, _u32]),
    "sassi_select_memdiv_pcs": (_i, [_vp, _vp, _u32]),
    "sassi_select_memdiv_topk": (_i, [_vp, _u32, _vp, ctypes.POINTER(_u32), _vp]),
    "sassi_set_addr_rows": (_i, [_vp, _u32]),
    "sassi_consume": (_i, [_vp, ctypes.POINTER(SassiRecords), _u64, _vp]),
    "sassi_consume_host": (_i, [_vp, ctypes.POINTER(SassiRecords), _u64, _vp]),
    "sassi_index_records": (_i, [_vp, _vp, _u64, _vp, _vp]),
    "sassi_reset": (_i, [_vp, _vp]),
    "sassi_read_tables": (_i, [_vp, _vp, _u64, _vp]),
    "sassi_tables_device": (_i, [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_u64)]),
    "sassi_sample_sites": (_i, [_vp, _u32, _u64, _vp, _vp]),
    "sassi_sample_sites_device": (_i, [_vp, _u32, _u64, _vp, _vp, _vp]),
    "sassi_sample_sites_multi": (_i, [_vp, _u32, _u32, _u64, _vp, _vp]),
    "sassi_merge": (_i, [_vp, _vp, _vp]),
    "sassi_merge_local": (_i, [_vp, _u32, _vp]),
    "sassi_nccl_get_unique_id": (_i, [_vp]),
    "sassi_nccl_comm_create": (_i, [ctypes.POINTER(_vp), _i, _i, _vp, _i]),
    "sassi_nccl_comm_destroy": (_i, [_vp]),
    "sassi_kernel_launches": (_i, [_vp, ctypes.POINTER(_u64)]),
    "sassi_enable_dynamic_pcs": (_i, [_vp, _u32]),
    "sassi_ipc_table_handle": (_i, [_vp, _vp]),
    "sassi_add_peer_table": (_i, [_vp, _vp]),
    "sassi_clear_peer_tables": (_i, [_vp]),
    "sassi_read_dynamic_pcs": (_i, [_vp, _vp, _u32, ctypes.POINTER(_u32), ctypes.POINTER(_u64), _vp]),
    "sassi_ik_create": (_i, [ctypes.POINTER(_vp), _i, _u32, _u64, _i]),
    "sassi_ik_destroy": (None, [_vp]),
    "sassi_ik_sites": (_i, [_vp, _vp, _u32, ctypes.POINTER(_u32), ctypes.POINTER(_u32)]),
    "sassi_ik_run": (_i, [_vp, _u32, _vp, _vp]),
    "sassi_ik_trace_totals": (_i, [_vp, ctypes.POINTER(_u64), ctypes.POINTER(_u64), ctypes.POINTER(_u64)]),
    "sassi_ik_trace_copy": (_i, [_vp, _vp, _vp, _vp, _vp]),
    "sassi_ik_output_checksum": (_i, [_vp, ctypes.POINTER(_u64)]),
    "sassi_ik_inject": (_i, [_vp, _vp, _u32, _vp, _vp]),
    "sassi_ik_trace_fold": (_i, [_vp, _vp, _u32, _u32, _vp, _vp]),
    "sassi_strerror": (ctypes.c_char_p, [_i]),
    "sassi_last_error": (ctypes.c_char_p, []),
}


class SassiError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__("%s (%d): %s" % (sassi_strerror(status), status, msg))
        self.status = status


_lib = None


def lib() -> ctypes.CDLL:
    """Load libsassi.so (fails loudly: there is no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError("libsassi.so not built (%s): run __graft_entry__.build()" % LIB_PATH)
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name, None)
            if f is None:  # an older build (SASSI_LIB A/B variants): calling it raises AttributeError
                continue
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def sassi_strerror(status: int) -> str:
    return lib().sassi_strerror(status).decode()


def sassi_last_error() -> str:
    return lib().sassi_last_error().decode()


def _check(rc: int) -> None:
    if rc != 0:
        raise SassiError(rc, sassi_last_error())


def _stream(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def _ptr(x) -> int | None:
    if x is None:
        return None
    if hasattr(x, "data_ptr"):
        return x.data_ptr() if x.numel() else None
    if isinstance(x, np.ndarray):
        return x.ctypes.data if x.size else None
    return int(x)


def _records(rec: dict) -> SassiRecords:
    r = SassiRecords()
    r.hdr = _ptr(rec["hdr"])
    r.addr = _ptr(rec["addr"]) if rec.get("n_addr_rows", 0) else None
    r.val = _ptr(rec["val"]) if rec.get("n_val_rows", 0) else None
    r.chunk_base = _ptr(rec["chunk_base"])
    r.n_addr_rows = int(rec.get("n_addr_rows", 0))
    r.n_val_rows = int(rec.get("n_val_rows", 0))
    return r


# ---- the C ABI, one Python function per C function --------------------------------------------
def sassi_table_layout(n_sites: int, n_warps: int) -> dict:
    L = SassiLayout()
    _check(lib().sassi_table_layout(n_sites, n_warps, ctypes.byref(L)))
    return {k: int(getattr(L, k)) for k, _ in SassiLayout._fields_}


def sassi_ctx_create(device: int, sites: np.ndarray, n_warps: int) -> int:
    sites = np.ascontiguousarray(sites).view(SITE_DTYPE)
    h = _vp()
    _check(lib().sassi_ctx_create(ctypes.byref(h), device, sites.ctypes.data if len(sites) else None,
                                  len(sites), n_warps))
    return h.value


def sassi_ctx_destroy(ctx: int) -> None:
    lib().sassi_ctx_destroy(ctx)


def sassi_attach_handler(ctx: int, kind_mask: int) -> None:
    _check(lib().sassi_attach_handler(ctx, kind_mask))


def sassi_select_memdiv_pcs(ctx: int, pcs) -> None:
    a = np.ascontiguousarray(pcs, dtype=np.uint32)
    _check(lib().sassi_select_memdiv_pcs(ctx, a.ctypes.data if a.size else None, a.size))


def sassi_set_addr_rows(ctx: int, which: int) -> None:
    _check(lib().sassi_set_addr_rows(ctx, which))


def sassi_select_memdiv_topk(ctx: int, k: int, stream=None) -> np.ndarray:
    """Rank GLOBAL memory sites by sectors per warp access in the tables so far, reset, and keep
    the per-PC matrices of the top k for the next pass -> their pcs in rank order."""
    out = np.zeros(max(k, 1), dtype=np.uint32)
    n = _u32()
    _check(lib().sassi_select_memdiv_topk(ctx, k, out.ctypes.data, ctypes.byref(n), _stream(stream)))
    return out[:n.value]


def sassi_consume(ctx: int, rec: dict, n=None, stream=None) -> None:
    n = rec["n"] if n is None else n
    r = _records(rec)
    _check(lib().sassi_consume(ctx, ctypes.byref(r), n, _stream(stream)))


def sassi_consume_host(ctx: int, rec: dict, n=None, stream=None) -> None:
    n = rec["n"] if n is None else n
    r = _records(rec)
    _check(lib().sassi_consume_host(ctx, ctypes.byref(r), n, _stream(stream)))


def sassi_index_records(ctx: int, hdr, n: int, chunk_base_out, stream=None) -> None:
    _check(lib().sassi_index_records(ctx, _ptr(hdr), n, _ptr(chunk_base_out), _stream(stream)))


def sassi_reset(ctx: int, stream=None) -> None:
    _check(lib().sassi_reset(ctx, _stream(stream)))


def sassi_read_tables(ctx: int, n_words: int, stream=None, out: np.ndarray | None = None) -> np.ndarray:
    out = np.zeros(n_words, dtype=np.uint64) if out is None else out
    _check(lib().sassi_read_tables(ctx, out.ctypes.data, out.size, _stream(stream)))
    return out


def sassi_tables_device(ctx: int):
    p, n = _vp(), _u64()
    _check(lib().sassi_tables_device(ctx, ctypes.byref(p), ctypes.byref(n)))
    return p.value, n.value


def sassi_sample_sites(ctx: int, k: int, seed: int, stream=None) -> np.ndarray:
    out = np.zeros(k, dtype=INJ_DTYPE)
    _check(lib().sassi_sample_sites(ctx, k, seed & (2**64 - 1), out.ctypes.data if k else None,
                                    _stream(stream)))
    return out


def sassi_sample_sites_device(ctx: int, k: int, seed: int, dev_out: int, dev_status: int,
                              stream=None) -> None:
    """Asynchronous form: k tuples to the device buffer at dev_out (32 B each), a u32 status at
    dev_status (1 = nothing to sample)."""
    _check(lib().sassi_sample_sites_device(ctx, k, seed & (2**64 - 1), dev_out or None, dev_status,
                                           _stream(stream)))


class SassiProfile(ctypes.Structure):
    _fields_ = [("ctx", _vp), ("kernel", _u32), ("invocation", _u32)]


def sassi_sample_sites_multi(profiles, k: int, seed: int, stream=None) -> np.ndarray:
    """profiles = [(Context or handle, kernel id, invocation id), ...] -> k tuples (INJ_DTYPE)."""
    arr = (SassiProfile * len(profiles))(*[SassiProfile(getattr(c, "handle", c), kk, ii)
                                           for c, kk, ii in profiles])
    out = np.zeros(k, dtype=INJ_DTYPE)
    _check(lib().sassi_sample_sites_multi(arr, len(profiles), k, seed & (2**64 - 1),
                                          out.ctypes.data if k else None, _stream(stream)))
    return out


def sassi_merge(ctx: int, comm: int, stream=None) -> None:
    _check(lib().sassi_merge(ctx, comm, _stream(stream)))


def sassi_merge_local(ctxs, stream=None) -> None:
    """Merge n contexts of one device in place (each ends with the merged tables)."""
    arr = (_vp * len(ctxs))(*[getattr(c, "handle", c) for c in ctxs])
    _check(lib().sassi_merge_local(arr, len(ctxs), _stream(stream)))


def sassi_nccl_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().sassi_nccl_get_unique_id(buf))
    return buf.raw


def sassi_nccl_comm_create(nranks: int, rank: int, unique_id: bytes, device: int) -> int:
    comm = _vp()
    uid = ctypes.create_string_buffer(bytes(unique_id), 128)
    _check(lib().sassi_nccl_comm_create(ctypes.byref(comm), nranks, rank, uid, device))
    return comm.value


def sassi_nccl_comm_destroy(comm: int) -> None:
    _check(lib().sassi_nccl_comm_destroy(comm))


DYN_PC_DTYPE = np.dtype([("pc", "<u4"), ("reserved", "<u4"), ("warp_execs", "<u8"),
                         ("thread_execs", "<u8")])
assert DYN_PC_DTYPE.itemsize == 24


def sassi_enable_dynamic_pcs(ctx: int, capacity: int) -> None:
    _check(lib().sassi_enable_dynamic_pcs(ctx, capacity))


def sassi_read_dynamic_pcs(ctx: int, stream=None):
    """-> (DYN_PC_DTYPE array sorted by pc, dropped records)."""
    n, dropped = _u32(), _u64()
    _check(lib().sassi_read_dynamic_pcs(ctx, None, 0, ctypes.byref(n), None, _stream(stream)))
    out = np.zeros(n.value, dtype=DYN_PC_DTYPE)
    _check(lib().sassi_read_dynamic_pcs(ctx, out.ctypes.data if n.value else None, n.value,
                                        ctypes.byref(n), ctypes.byref(dropped), _stream(stream)))
    return out[:n.value], dropped.value


def sassi_ipc_table_handle(ctx: int) -> bytes:
    buf = ctypes.create_string_buffer(64)
    _check(lib().sassi_ipc_table_handle(ctx, buf))
    return buf.raw


def sassi_add_peer_table(ctx: int, handle: bytes) -> None:
    buf = ctypes.create_string_buffer(bytes(handle), 64)
    _check(lib().sassi_add_peer_table(ctx, buf))


def sassi_clear_peer_tables(ctx: int) -> None:
    _check(lib().sassi_clear_peer_tables(ctx))


def sassi_kernel_launches(ctx: int) -> int:
    n = _u64()
    _check(lib().sassi_kernel_launches(ctx, ctypes.byref(n)))
    return n.value


# ---- convenience wrapper -----------------------------------------------------------------------
class Context:
    """One SASSI analysis context on one device: sites registered once, tables accumulate."""

    def __init__(self, sites: np.ndarray, n_warps: int, handlers: int = SASSI_H_ALL, device: int = 0):
        self.sites = np.ascontiguousarray(sites).view(SITE_DTYPE)
        self.n_sites = len(self.sites)
        self.n_warps = int(n_warps)
        self.device = device
        self.layout = sassi_table_layout(self.n_sites, self.n_warps)
        self.handle = sassi_ctx_create(device, self.sites, self.n_warps)
        sassi_attach_handler(self.handle, handlers)
        self.handlers = handlers

    def consume(self, rec: dict, n=None, stream=None):
        sassi_consume(self.handle, rec, n, stream)

    def consume_host(self, rec: dict, n=None, stream=None):
        sassi_consume_host(self.handle, rec, n, stream)

    def reset(self, stream=None):
        sassi_reset(self.handle, stream)

    def select_memdiv_pcs(self, pcs) -> None:
        """Keep per-PC memory-divergence matrices (pcmat) for up to 4 GLOBAL memory sites."""
        sassi_select_memdiv_pcs(self.handle, pcs)

    def set_addr_rows(self, which: int) -> None:
        """SASSI_ADDR_ROWS_GLOBAL: the streams carry the address rows of GLOBAL memory sites only."""
        sassi_set_addr_rows(self.handle, which)

    def select_memdiv_topk(self, k: int, stream=None) -> np.ndarray:
        """Top-k most divergent GLOBAL pcs of the folds so far; resets and keeps their matrices."""
        return sassi_select_memdiv_topk(self.handle, k, stream)

    def read_tables(self, stream=None) -> np.ndarray:
        return sassi_read_tables(self.handle, self.layout["total"], stream)

    def sections(self, table: np.ndarray | None = None) -> dict:
        t = self.read_tables() if table is None else table
        L, S = self.layout, self.n_sites
        return {"diag": t[0:8], "br": t[L["br"]:L["mem"]].reshape(S, 5),
                "mem": t[L["mem"]:L["val"]].reshape(S, 4), "val": t[L["val"]:L["ones"]].reshape(S, 2),
                "ones": t[L["ones"]:L["zeros"]].reshape(S, 4),
                "zeros": t[L["zeros"]:L["scalar"]].reshape(S, 4),
                "scalar": t[L["scalar"]:L["h32"]].reshape(S, 4),
                "h32": t[L["h32"]:L["h128"]].reshape(32, 32),
                "h128": t[L["h128"]:L["counts"]].reshape(32, 32), "counts": t[L["counts"]:L["mix"]],
                "mix": t[L["mix"]:L["imix"]], "imix": t[L["imix"]:L["pcsel"]],
                "pcsel": t[L["pcsel"]:L["pcmat"]],
                "pcmat": t[L["pcmat"]:L["total"]].reshape(4, 32, 32)}

    def sample(self, k: int, seed: int, stream=None) -> np.ndarray:
        return sassi_sample_sites(self.handle, k, seed, stream)

    def sample_device(self, out, status, k: int, seed: int, stream=None) -> None:
        """Draws into `out` (a device tensor of >= 32*k bytes) and the status into `status` (a
        device tensor of >= 4 bytes); no synchronisation."""
        sassi_sample_sites_device(self.handle, k, seed, out.data_ptr() if k else 0,
                                  status.data_ptr(), stream)

    def merge(self, comm: int, stream=None):
        sassi_merge(self.handle, comm, stream)

    def enable_dynamic_pcs(self, capacity: int) -> None:
        """Insert-on-miss table of unregistered pcs (Fig.4 l.21-23)."""
        sassi_enable_dynamic_pcs(self.handle, capacity)

    def read_dynamic_pcs(self, stream=None):
        return sassi_read_dynamic_pcs(self.handle, stream)

    def ipc_table_handle(self) -> bytes:
        """CUDA IPC handle of this context's table image (for the fused merge)."""
        return sassi_ipc_table_handle(self.handle)

    def add_peer_table(self, handle: bytes) -> None:
        """Fold into a peer's table image too (fused fold + merge over peer memory)."""
        sassi_add_peer_table(self.handle, handle)

    def clear_peer_tables(self) -> None:
        sassi_clear_peer_tables(self.handle)

    def kernel_launches(self) -> int:
        return sassi_kernel_launches(self.handle)

    def close(self):
        if self.handle:
            sassi_ctx_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---- instrumented synthetic kernels (include/sassi_ik.h) ---------------------------------------
def sassi_ik_create(kernel: int, size: int = 0, seed: int = 20150613, device: int = 0) -> int:
    h = _vp()
    _check(lib().sassi_ik_create(ctypes.byref(h), kernel, size, seed, device))
    return h.value


def sassi_ik_destroy(ik: int) -> None:
    lib().sassi_ik_destroy(ik)


def sassi_ik_sites(ik: int):
    n, w = _u32(), _u32()
    _check(lib().sassi_ik_sites(ik, None, 0, ctypes.byref(n), ctypes.byref(w)))
    out = np.zeros(n.value, dtype=SITE_DTYPE)
    _check(lib().sassi_ik_sites(ik, out.ctypes.data, n.value, ctypes.byref(n), ctypes.byref(w)))
    return out, w.value


def sassi_ik_run(ik: int, mode: int, ctx: int | None = None, stream=None) -> None:
    _check(lib().sassi_ik_run(ik, mode, ctx, _stream(stream)))


def sassi_ik_trace_totals(ik: int):
    a, b, c = _u64(), _u64(), _u64()
    _check(lib().sassi_ik_trace_totals(ik, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
    return a.value, b.value, c.value


def sassi_ik_trace_copy(ik: int, hdr, addr, val, stream=None) -> None:
    _check(lib().sassi_ik_trace_copy(ik, _ptr(hdr), _ptr(addr), _ptr(val), _stream(stream)))


def sassi_ik_output_checksum(ik: int) -> int:
    c = _u64()
    _check(lib().sassi_ik_output_checksum(ik, ctypes.byref(c)))
    return c.value


SASSI_IK_SERIAL = 1
TRACE_STATS_DTYPE = np.dtype([("n_records", "<u8"), ("n_addr_rows", "<u8"), ("n_val_rows", "<u8"),
                              ("max_segment_records", "<u8"), ("ring_bytes", "<u8"),
                              ("segments", "<u4"), ("blocks_per_segment", "<u4")])
assert TRACE_STATS_DTYPE.itemsize == 48


def sassi_ik_trace_fold(ik: int, ctx: int, blocks_per_segment: int = 0, flags: int = 0,
                        stream=None) -> dict:
    st = np.zeros(1, dtype=TRACE_STATS_DTYPE)
    _check(lib().sassi_ik_trace_fold(ik, ctx, blocks_per_segment, flags, st.ctypes.data,
                                     _stream(stream)))
    return {k: int(st[0][k]) for k in TRACE_STATS_DTYPE.names}


# error-injection outcomes (include/sassi_ik.h)
SASSI_INJ_MASKED, SASSI_INJ_SDC, SASSI_INJ_DUE, SASSI_INJ_HANG, SASSI_INJ_NOT_REACHED = range(5)
INJ_OUTCOME_NAMES = ("masked", "sdc", "due", "hang", "not_reached")
OUTCOME_DTYPE = np.dtype([("outcome", "<u4"), ("site", "<u4"), ("target", "<u4"), ("bit", "<u4"),
                          ("before", "<u4"), ("after", "<u4"), ("reserved", "<u4", (2,))])
assert OUTCOME_DTYPE.itemsize == 32


def sassi_ik_inject(ik: int, sites: np.ndarray, stream=None) -> np.ndarray:
    sites = np.ascontiguousarray(sites, dtype=INJ_DTYPE)
    out = np.zeros(len(sites), dtype=OUTCOME_DTYPE)
    _check(lib().sassi_ik_inject(ik, sites.ctypes.data if len(sites) else None, len(sites),
                                 out.ctypes.data if len(sites) else None, _stream(stream)))
    return out


class InstrumentedKernel:
    """A synthetic kernel with hand-placed SASSI sites (vecadd / bfs / sgemm / stencil)."""

    NAMES = {"vecadd": SASSI_IK_VECADD, "bfs": SASSI_IK_BFS, "sgemm": SASSI_IK_SGEMM,
             "stencil": SASSI_IK_STENCIL}

    def __init__(self, kernel, size: int = 0, seed: int = 20150613, device: int = 0):
        kid = self.NAMES[kernel] if isinstance(kernel, str) else kernel
        self.handle = sassi_ik_create(kid, size, seed, device)
        self.device = device
        self.sites, self.n_warps = sassi_ik_sites(self.handle)

    def context(self, handlers: int = SASSI_H_ALL) -> Context:
        return Context(self.sites, self.n_warps, handlers, self.device)

    def run(self, mode: int, ctx: Context | None = None, stream=None) -> None:
        sassi_ik_run(self.handle, mode, ctx.handle if ctx is not None else None, stream)

    def inject(self, sites: np.ndarray, stream=None) -> np.ndarray:
        """One error-injection run per site tuple (§8.1) -> OUTCOME_DTYPE records."""
        return sassi_ik_inject(self.handle, sites, stream)

    def injection_campaign(self, k: int = 1000, seed: int = 20150616, stream=None):
        """§8.1's three steps on this kernel: (1) profile the per-thread eligible counts,
        (2) draw k injection sites, (3) one injection run per site. -> (sites, outcomes)."""
        ctx = self.context(SASSI_H_INSTCOUNT)
        try:
            self.run(SASSI_H_INSTCOUNT, ctx, stream)
            sites = ctx.sample(k, seed, stream)
        finally:
            ctx.close()
        return sites, self.inject(sites, stream)

    def checksum(self) -> int:
        return sassi_ik_output_checksum(self.handle)

    def trace(self, ctx: Context, stream=None) -> dict:
        """Run in trace mode; return the warp-major SRF1 stream as device tensors (+ chunk index)."""
        import torch
        sassi_ik_run(self.handle, SASSI_IK_TRACE, None, stream)
        n, na, nv = sassi_ik_trace_totals(self.handle)
        dev = torch.device("cuda", self.device)
        hdr = torch.empty((max(n, 1), 4), dtype=torch.int32, device=dev)
        addr = torch.empty((max(na, 1), 32), dtype=torch.int64, device=dev)
        val = torch.empty((max(nv, 1), 32), dtype=torch.int32, device=dev)
        sassi_ik_trace_copy(self.handle, hdr, addr, val, stream)
        cb = torch.zeros(((n + SASSI_CHUNK - 1) // SASSI_CHUNK + 1, 2), dtype=torch.int64, device=dev)
        sassi_index_records(ctx.handle, hdr, n, cb, stream)
        torch.cuda.synchronize(dev)
        return dict(hdr=hdr[:n], addr=addr[:na], val=val[:nv], chunk_base=cb, n=n, n_addr_rows=na,
                    n_val_rows=nv, sites=self.sites)

    def trace_fold(self, ctx: Context, blocks_per_segment: int = 0, serial: bool = False,
                   stream=None) -> dict:
        """Online trace mode: trace segment by segment into a two-slot ring and fold each segment
        into ctx on a second stream while the next one is traced."""
        return sassi_ik_trace_fold(self.handle, ctx.handle, blocks_per_segment,
                                   SASSI_IK_SERIAL if serial else 0, stream)

    def close(self):
        if self.handle:
            sassi_ik_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
