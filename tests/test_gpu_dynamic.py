"""Dynamic sites (Fig.4 l.21-23 "Create a new entry if one does not exist";
DESIGN R25): records whose pc is not registered update an insert-on-miss device hash table keyed
by pc. Its canonical read-out (sorted by pc) must equal the oracle's ordered map bit for bit, the
registered-site tables must be unaffected, and a full table must drop whole pcs, never miscount."""
import numpy as np
import pytest

import oracle
import t0_trace as T0
from gpu_helpers import to_device, diff_tables
from test_oracle import random_trace
from paper_conf_isca_stephensonhlejn15_b200 import sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
FULL = 0xFFFFFFFF


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def as_list(dyn):
    return [[int(e["pc"]), int(e["warp_execs"]), int(e["thread_execs"])] for e in dyn]


def fold(sites, W, mask, drec, capacity, consumes=1):
    ctx = sassi.Context(sites, W, mask)
    ctx.enable_dynamic_pcs(capacity)
    for _ in range(consumes):
        ctx.consume(drec)
    t = ctx.read_tables()
    dyn, dropped = ctx.read_dynamic_pcs()
    ctx.close()
    return t, as_list(dyn), dropped


def header_stream(seed, n, pcs, n_warps=64):
    """Header-only records (every pc unregistered, so no rows) with heavy-tailed pc frequencies,
    random active masks (some empty) and a sprinkling of the reserved pc."""
    rng = np.random.default_rng(seed)
    z = rng.zipf(1.3, n) % len(pcs)
    pc = np.asarray(pcs, np.uint32)[z]
    pc[rng.random(n) < 0.001] = FULL
    act = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    act[rng.random(n) < 0.5] = FULL
    act[rng.random(n) < 0.01] = 0
    H = np.stack([pc, rng.integers(0, n_warps, n).astype(np.uint32), act,
                  rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)], 1)
    return np.ascontiguousarray(H, np.uint32).view(oracle.HDR_DTYPE).reshape(-1)


def test_t0_dynamic_table_and_unchanged_tables():
    s = T0.sites()
    hdr, addr, val = T0.records()
    t, dyn, dropped = fold(s, T0.N_WARPS, sassi.SASSI_H_EVERY, to_device(s, hdr, addr, val), 16)
    assert dyn == [[0x999, 1, 32]] and dropped == 0
    assert np.array_equal(t, oracle.run(s, T0.N_WARPS, sassi.SASSI_H_EVERY, hdr, addr, val))


@pytest.mark.parametrize("seed,n", [(7, 1000), (8, 20000)])
@pytest.mark.parametrize("mask", [sassi.SASSI_H_ALL, sassi.SASSI_H_INSTCOUNT])
def test_random_traces_with_unregistered_sites(seed, n, mask):
    s, W, hdr, addr, val = random_trace(seed, n=n)
    rowless = np.array([not (s[i]["flags"] & oracle.F_MEM) and s[i]["n_gpr_dst"] == 0
                        for i in range(len(s))])
    s2 = s[~np.isin(s["pc"], s["pc"][rowless][:3])]
    t, dyn, dropped = fold(s2, W, mask, to_device(s2, hdr, addr, val), 64)
    o = oracle.run(s2, W, mask, hdr, addr, val)
    assert diff_tables(t, o, len(s2), W) is None
    odyn, odrop = oracle.dynamic_pcs(s2, hdr)
    assert dyn == odyn.tolist() and dropped == odrop


@pytest.mark.parametrize("n_pcs,n", [(5, 100000), (3000, 1 << 20)])
@pytest.mark.parametrize("mask", [sassi.SASSI_H_INSTCOUNT, sassi.SASSI_H_EVERY])
def test_discovery_with_no_registered_sites(n_pcs, n, mask):
    """An empty site table: every record goes to the dynamic table (the 'which pcs ran' pass)."""
    pcs = 0x1000 + 16 * np.arange(n_pcs)
    hdr = header_stream(n_pcs, n, pcs)
    s = np.zeros(0, dtype=oracle.SITE_DTYPE)
    t, dyn, dropped = fold(s, 64, mask, to_device(s, hdr, None, None), n_pcs)
    odyn, odrop = oracle.dynamic_pcs(s, hdr)
    assert dyn == odyn.tolist() and dropped == odrop > 0
    assert int(t[0]) == n and int(t[2]) == n


def test_full_table_drops_whole_pcs_only():
    """Capacity 16 -> 32 slots for 200 distinct pcs: exactly 32 pcs get entries, each with its exact
    count (a pc is inserted at its first record and then always found); the rest are dropped."""
    pcs = 0x2000 + 16 * np.arange(200)
    hdr = header_stream(5, 200000, pcs)
    s = np.zeros(0, dtype=oracle.SITE_DTYPE)
    _, dyn, dropped = fold(s, 64, sassi.SASSI_H_INSTCOUNT, to_device(s, hdr, None, None), 16)
    odyn, odrop = oracle.dynamic_pcs(s, hdr)
    exact = {int(r[0]): r.tolist() for r in odyn}
    assert len(dyn) == 32
    for e in dyn:
        assert e == exact[e[0]]
    assert sum(e[1] for e in dyn) + dropped == int(odyn[:, 1].sum()) + odrop


def test_accumulate_reset_and_state_errors():
    pcs = 0x3000 + 16 * np.arange(50)
    hdr = header_stream(11, 50000, pcs)
    s = np.zeros(0, dtype=oracle.SITE_DTYPE)
    d = to_device(s, hdr, None, None)
    _, dyn2, drop2 = fold(s, 64, sassi.SASSI_H_BRANCH, d, 50, consumes=2)
    odyn, odrop = oracle.dynamic_pcs(s, hdr)
    assert dyn2 == [[p, 2 * w, 2 * t] for p, w, t in odyn.tolist()] and drop2 == 2 * odrop
    ctx = sassi.Context(s, 64, sassi.SASSI_H_BRANCH)
    with pytest.raises(sassi.SassiError):
        ctx.read_dynamic_pcs()          # not enabled
    ctx.enable_dynamic_pcs(50)
    ctx.consume(d)
    with pytest.raises(sassi.SassiError):
        ctx.enable_dynamic_pcs(60)      # after consume
    ctx.reset()
    dyn, dropped = ctx.read_dynamic_pcs()
    assert len(dyn) == 0 and dropped == 0
    ctx.enable_dynamic_pcs(60)          # allowed again after reset
    ctx.consume(d)
    assert as_list(ctx.read_dynamic_pcs()[0]) == odyn.tolist()
    ctx.close()


def test_merge_single_rank_nccl_rebuilds_dynamic_table():
    """sassi_merge gathers every rank's dynamic table and re-inserts all entries into a cleared
    table; over one rank that must reproduce the table exactly (and leave the rest unchanged)."""
    s, W, hdr, addr, val = random_trace(77, n=6000)
    rowless = np.array([not (s[i]["flags"] & oracle.F_MEM) and s[i]["n_gpr_dst"] == 0
                        for i in range(len(s))])
    s2 = s[~np.isin(s["pc"], s["pc"][rowless][:3])]
    ctx = sassi.Context(s2, W, sassi.SASSI_H_EVERY)
    ctx.enable_dynamic_pcs(8)
    ctx.consume(to_device(s2, hdr, addr, val))
    before = ctx.read_tables()
    uid = sassi.sassi_nccl_get_unique_id()
    comm = sassi.sassi_nccl_comm_create(1, 0, uid, torch.cuda.current_device())
    ctx.merge(comm)
    sassi.sassi_nccl_comm_destroy(comm)
    after = ctx.read_tables()
    dyn, dropped = ctx.read_dynamic_pcs()
    ctx.close()
    assert np.array_equal(after, before)
    odyn, odrop = oracle.dynamic_pcs(s2, hdr)
    assert as_list(dyn) == odyn.tolist() and dropped == odrop


@pytest.mark.parametrize("mask", [sassi.SASSI_H_INSTCOUNT, sassi.SASSI_H_BRANCH | sassi.SASSI_H_INSTMIX])
def test_c4_prefix_half_the_sites_unregistered(mask):
    """The error-injection profiling stream (c4) at scale: its first 10^7 records with every other
    site unregistered, under header-only handler sets (rows are never read, so the stream stays
    valid). The registered-site tables and the dynamic table both equal the oracle's."""
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    P, lim, _, _ = gen.preset("c4")
    d = gen.generate_device(P, 10_000_000)
    s_all = d["sites"]
    s2 = s_all[::2].copy()
    W = P.total_warps
    hdr = d["hdr"][: d["n"]].cpu().numpy().view(np.uint32).reshape(-1, 4).view(oracle.HDR_DTYPE).reshape(-1)
    rec = dict(hdr=d["hdr"], addr=d["addr"][:0], val=d["val"][:0], chunk_base=d["chunk_base"],
               n=d["n"], n_addr_rows=0, n_val_rows=0)
    t, dyn, dropped = fold(s2, W, mask, rec, len(s_all))
    # header-only handlers read no rows (c4 is generated without them): the oracle gets the row
    # counts its registered sites imply (SRF1) and never dereferences a row
    order = np.argsort(s2["pc"])
    pos = np.searchsorted(s2["pc"][order], hdr["pc"])
    pos = np.minimum(pos, len(s2) - 1)
    idx = order[pos]
    reg = s2["pc"][idx] == hdr["pc"]
    na = int(((s2["flags"][idx] & oracle.F_MEM) != 0)[reg].sum())
    nv = int(s2["n_gpr_dst"][idx][reg].astype(np.int64).sum())
    o = oracle.consume(oracle.table_init(len(s2), W, mask), s2, W, mask, hdr, None, None,
                       n_addr_rows=na, n_val_rows=nv)
    assert diff_tables(t, o, len(s2), W) is None
    odyn, odrop = oracle.dynamic_pcs(s2, hdr)
    assert dyn == odyn.tolist() and dropped == odrop == 0
    assert len(dyn) == len(s_all) - len(s2)


def test_host_buffers_with_dynamic_pcs():
    """sassi_consume_host (pinned host buffers, staged copies) takes the same extended kernel:
    tables and dynamic table equal the oracle's."""
    s, W, hdr, addr, val = random_trace(91, n=20000)
    rowless = np.array([not (s[i]["flags"] & oracle.F_MEM) and s[i]["n_gpr_dst"] == 0
                        for i in range(len(s))])
    s2 = s[~np.isin(s["pc"], s["pc"][rowless][:3])]
    d = to_device(s2, hdr, addr, val)
    h = {k: (v.cpu().pin_memory() if hasattr(v, "cpu") else v) for k, v in d.items()}
    ctx = sassi.Context(s2, W, sassi.SASSI_H_EVERY)
    ctx.enable_dynamic_pcs(64)
    ctx.consume_host(h)
    t = ctx.read_tables()
    dyn, dropped = ctx.read_dynamic_pcs()
    ctx.close()
    assert diff_tables(t, oracle.run(s2, W, sassi.SASSI_H_EVERY, hdr, addr, val), len(s2), W) is None
    odyn, odrop = oracle.dynamic_pcs(s2, hdr)
    assert as_list(dyn) == odyn.tolist() and dropped == odrop
