"""Site tables from a handful of sites up to SASSI_MAX_SITES = 65,536. When the pc hash, the value
state and the per-site counters fit one SM's shared memory the fold keeps them there; larger site
tables run in global mode (hash lookups from global memory, per-record u64 atomics into the table
image: Fig.4 / Fig.9's device-global tables, L239 / L595). Both must equal the oracle bit for bit:
4,096 and 65,536 header-handler sites, 16,384 sites with four value destinations each (all five
handlers, memory sites among them, per-PC matrices and dynamic pcs on), and one site more than the
maximum is ENOSPC at create."""
import time

import numpy as np
import pytest

import oracle
from gpu_helpers import to_device, diff_tables
from paper_conf_isca_stephensonhlejn15_b200 import sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _sites(n, flags, ndst=0):
    s = np.zeros(n, dtype=oracle.SITE_DTYPE)
    s["pc"] = 0x1000 + 16 * np.arange(n)
    s["flags"] = flags
    s["n_gpr_dst"] = ndst
    return s


def _headers(pcs, W, n, rng):
    H = np.stack([pcs[rng.integers(0, len(pcs), n)], rng.integers(0, W, n).astype(np.uint32),
                  rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32),
                  rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)], 1).astype(np.uint32)
    return np.ascontiguousarray(H).view(oracle.HDR_DTYPE).reshape(-1)


@pytest.mark.parametrize("n_sites", [4096, 65536])
def test_max_sites_header_handlers(n_sites):
    mask = sassi.SASSI_H_BRANCH | sassi.SASSI_H_INSTCOUNT | sassi.SASSI_H_INSTMIX
    W, n = 64, 400_000
    half = n_sites // 2
    s = np.concatenate([_sites(half, oracle.F_COND_BRANCH | oracle.F_CTRL),
                        _sites(half, oracle.F_NUMERIC | oracle.F_WRITES_PRED)])
    s["pc"] = 0x1000 + 16 * np.arange(n_sites)
    hdr = _headers(s["pc"], W, n, np.random.default_rng(n_sites))
    ctx = sassi.Context(s, W, mask)
    ctx.consume(to_device(s, hdr, None, None))
    t = ctx.read_tables()
    ctx.close()
    assert diff_tables(t, oracle.run(s, W, mask, hdr), n_sites, W) is None


def _big_trace(n_sites, W, n, seed):
    """n_sites sites: a quarter conditional branches, a quarter GLOBAL loads (1 destination), a
    quarter SHARED loads, a quarter 4-destination ALU sites; n records over W warps plus 2 % of
    unregistered pcs; address rows unit-stride / broadcast / gathers, value rows constant / small /
    random."""
    rng = np.random.default_rng(seed)
    q = n_sites // 4
    s = np.concatenate([_sites(q, oracle.F_COND_BRANCH | oracle.F_CTRL),
                        _sites(q, oracle.F_MEM | oracle.F_MEM_READ, 1),
                        _sites(q, oracle.F_MEM | oracle.F_MEM_READ, 1),
                        _sites(n_sites - 3 * q, oracle.F_NUMERIC, 4)])
    s["pc"] = 0x1000 + 16 * np.arange(n_sites)
    s["domain"][2 * q:3 * q] = oracle.D_SHARED
    s["mem_width"][q:3 * q] = 4
    pcs = np.concatenate([s["pc"], 0x9000000 + 16 * np.arange(64)]).astype(np.uint32)
    hdr = _headers(pcs[np.r_[np.arange(n_sites), np.arange(n_sites, n_sites + 64)[:(n_sites // 50)]]],
                   W, n, rng)
    idx = {int(p): i for i, p in enumerate(s["pc"])}
    site_of = np.array([idx.get(int(p), -1) for p in hdr["pc"]])
    is_mem = (site_of >= q) & (site_of < 3 * q)
    nd = np.where(site_of < 0, 0, s["n_gpr_dst"][np.maximum(site_of, 0)]).astype(np.int64)
    na = int(is_mem.sum())
    l = np.arange(32, dtype=np.uint64)
    base = (rng.integers(0, 2**30, na).astype(np.uint64) << np.uint64(7)) + np.uint64(0x7F0000000000)
    style = rng.integers(0, 3, na)
    addr = np.where(style[:, None] == 0, base[:, None] + 4 * l,
                    np.where(style[:, None] == 1, base[:, None] + np.uint64(64),
                             base[:, None] + 4 * rng.integers(0, 1 << 22, (na, 32)).astype(np.uint64)))
    nv = int(nd.sum())
    vs = rng.integers(0, 3, nv)
    val = np.where(vs[:, None] == 0, rng.integers(0, 2**32, nv, dtype=np.uint64)[:, None].astype(np.uint32),
                   np.where(vs[:, None] == 1, rng.integers(0, 256, (nv, 32)).astype(np.uint32),
                            rng.integers(0, 2**32, (nv, 32), dtype=np.uint64).astype(np.uint32)))
    return s, hdr, addr.astype(np.uint64), val.astype(np.uint32), q


def test_global_mode_16k_sites_four_destinations_all_handlers():
    n_sites, W, n = 16384, 512, 1_000_000
    s, hdr, addr, val, q = _big_trace(n_sites, W, n, 16384)
    mask = sassi.SASSI_H_EVERY
    sel = [q, q + 1, q + 7, 2 * q - 1]                  # four GLOBAL load sites
    d = to_device(s, hdr, addr, val)
    ctx = sassi.Context(s, W, mask)
    ctx.select_memdiv_pcs([int(s["pc"][i]) for i in sel])
    ctx.enable_dynamic_pcs(64)
    torch.cuda.synchronize()
    ctx.consume(d)
    t = ctx.read_tables()
    o = oracle.run(s, W, mask, hdr, addr, val, pcs=sel)
    assert diff_tables(t, o, n_sites, W) is None
    dyn, dropped = oracle.dynamic_pcs(s, hdr)
    got, nd = ctx.read_dynamic_pcs()
    assert nd == dropped and np.array_equal(
        np.stack([got["pc"], got["warp_execs"], got["thread_execs"]], 1).astype(np.uint64), dyn)
    # throughput of the global-mode fold on this stream (reported, not asserted)
    reps, t0 = 5, time.perf_counter()
    for _ in range(reps):
        ctx.reset()
        ctx.consume(d)
    torch.cuda.synchronize()
    el = (time.perf_counter() - t0) / reps
    print("global mode, 16384 sites x 4 dst: %.3f ms per fold of %d records (%.2e records/s)"
          % (1e3 * el, n, n / el))
    ctx.close()


def test_value_state_beyond_shared_memory_uses_global_mode():
    """4,096 sites with four destinations each: the value state alone (256 KB) exceeds shared
    memory, which was ENOSPC before global mode; now it folds exactly."""
    n_sites, W, n = 4096, 64, 100_000
    s = _sites(n_sites, oracle.F_NUMERIC, 4)
    rng = np.random.default_rng(7)
    hdr = _headers(s["pc"], W, n, rng)
    val = rng.integers(0, 16, (4 * n, 32)).astype(np.uint32)
    ctx = sassi.Context(s, W, sassi.SASSI_H_VALUE)
    ctx.consume(to_device(s, hdr, None, val))
    t = ctx.read_tables()
    ctx.close()
    assert diff_tables(t, oracle.run(s, W, sassi.SASSI_H_VALUE, hdr, None, val), n_sites, W) is None


def test_one_site_too_many_is_enospc():
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, _sites(65537, oracle.F_NUMERIC), 8)
    assert e.value.status == sassi.SASSI_ENOSPC


@pytest.mark.parametrize("seed,n", [(1, 257), (2, 5000), (3, 20000)])
@pytest.mark.parametrize("mask", [sassi.SASSI_H_ALL, sassi.SASSI_H_EVERY, sassi.SASSI_H_INSTMIX | 1])
def test_forced_global_mode_random_traces(monkeypatch, seed, n, mask):
    """Every handler path of global mode on the random edge-case traces (SASSI_FORCE_GLOBAL_MODE=1
    puts small site tables through it), with per-PC matrices and dynamic pcs."""
    from test_oracle import random_trace
    monkeypatch.setenv("SASSI_FORCE_GLOBAL_MODE", "1")
    s, W, hdr, addr, val = random_trace(8800 + seed, n=n)
    glob = [i for i in range(len(s)) if (int(s[i]["flags"]) & oracle.F_MEM) and int(s[i]["domain"]) == 0]
    ctx = sassi.Context(s, W, mask)
    ctx.select_memdiv_pcs([int(s[i]["pc"]) for i in glob[:2]])
    ctx.enable_dynamic_pcs(8)
    ctx.consume(to_device(s, hdr, addr, val))
    t = ctx.read_tables()
    dyn, dropped = ctx.read_dynamic_pcs()
    ctx.close()
    assert diff_tables(t, oracle.run(s, W, mask, hdr, addr, val, pcs=glob[:2]), len(s), W) is None
    odyn, odrop = oracle.dynamic_pcs(s, hdr)
    assert dropped == odrop and [[int(e["pc"]), int(e["warp_execs"]), int(e["thread_execs"])] for e in dyn] == odyn.tolist()
