"""GPU parity: the CUDA fold (through the C ABI) equals the oracle bit for bit — hand-worked T0,
random edge-case traces for every handler combination, and every BASELINE config in full: c1 and
c2 with a single oracle pass; c3 and c4 (10^8 records) and one whole c5 shard (~4.9x10^8 records)
in the bench's launch configuration, against the oracle run over host-generated warp shards in
parallel processes and merged (tests/oracle_shards.py), plus properties that hold at any size."""
import numpy as np
import pytest

import oracle
import t0_trace as T0
from gpu_helpers import to_device, gpu_table, diff_tables, host_chunk_base
from test_oracle import random_trace
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.init()


def test_t0_hand_worked_on_gpu():
    s = T0.sites()
    hdr, addr, val = T0.records()
    t = gpu_table(s, T0.N_WARPS, sassi.SASSI_H_ALL, to_device(s, hdr, addr, val))
    T0.check_table(t, oracle.sections(t, len(s), T0.N_WARPS))
    assert np.array_equal(t, oracle.run(s, T0.N_WARPS, oracle.H_ALL, hdr, addr, val))


@pytest.mark.parametrize("mask", list(range(1, 32)))
def test_t0_every_handler_mask(mask):
    s = T0.sites()
    hdr, addr, val = T0.records()
    t = gpu_table(s, T0.N_WARPS, mask, to_device(s, hdr, addr, val))
    o = oracle.run(s, T0.N_WARPS, mask, hdr, addr, val)
    assert diff_tables(t, o, len(s), T0.N_WARPS) is None
    if mask == sassi.SASSI_H_EVERY:       # every handler, hand-worked values included
        T0.check_table(t, oracle.sections(t, len(s), T0.N_WARPS), mask)


@pytest.mark.parametrize("seed,n", [(0, 1), (1, 31), (2, 257), (3, 1000), (4, 5000), (5, 20000)])
@pytest.mark.parametrize("mask", [sassi.SASSI_H_ALL, sassi.SASSI_H_EVERY, sassi.SASSI_H_INSTMIX])
def test_random_traces(seed, n, mask):
    s, W, hdr, addr, val = random_trace(1000 + seed, n=n)
    o = oracle.run(s, W, mask, hdr, addr, val)
    t = gpu_table(s, W, mask, to_device(s, hdr, addr, val))
    assert diff_tables(t, o, len(s), W) is None


def test_reserved_pc_record_is_unknown():
    """A record whose pc is the reserved empty-slot key 0xFFFFFFFF is an unregistered pc."""
    s, W, hdr, addr, val = random_trace(31337, n=700)
    hdr = hdr.copy()
    hdr["pc"][::7] = np.where(np.isin(hdr["pc"][::7], s["pc"]), hdr["pc"][::7], 0xFFFFFFFF)
    o = oracle.run(s, W, oracle.H_ALL, hdr, addr, val)
    assert int(oracle.sections(o, len(s), W)["diag"][2]) > 0
    t = gpu_table(s, W, sassi.SASSI_H_ALL, to_device(s, hdr, addr, val))
    assert diff_tables(t, o, len(s), W) is None


def test_empty_stream():
    s = T0.sites()
    hdr, addr, val = T0.records()
    d = to_device(s, hdr, addr, val)
    t = gpu_table(s, T0.N_WARPS, sassi.SASSI_H_ALL, d, n=0)
    assert np.array_equal(t, oracle.table_init(len(s), T0.N_WARPS, oracle.H_ALL))


def test_misaligned_buffers_are_rejected():
    """Headers are vector-loaded, value rows TMA-copied and address rows bulk-prefetched: every
    buffer must be 16-byte aligned, and an 8-byte offset one is refused with EINVAL up front."""
    import torch
    s = T0.sites()
    hdr, addr, val = T0.records()
    d = to_device(s, hdr, addr, val)
    ctx = sassi.Context(s, T0.N_WARPS, sassi.SASSI_H_ALL)
    for key in ("hdr", "addr", "val", "chunk_base"):
        t = d[key]
        buf = torch.empty(t.numel() * t.element_size() + 8, dtype=torch.uint8, device=t.device)
        moved = buf[8:].view(t.dtype).reshape(t.shape)
        moved.copy_(t)
        with pytest.raises(sassi.SassiError) as ei:
            ctx.consume(dict(d, **{key: moved}))
        assert ei.value.status == sassi.SASSI_EINVAL and "aligned" in str(ei.value)
    ctx.consume(d)  # the aligned originals still fold
    assert np.array_equal(ctx.read_tables(),
                          oracle.run(s, T0.N_WARPS, oracle.H_ALL, hdr, addr, val))
    ctx.close()


def test_inconsistent_chunk_index_is_reported():
    s, W, hdr, addr, val = random_trace(77, n=3000)
    cb = host_chunk_base(s, hdr)
    cb[3, 1] += 1                                   # corrupt one chunk's val-row base
    d = to_device(s, hdr, addr, val, cb)
    ctx = sassi.Context(s, W, sassi.SASSI_H_ALL)
    ctx.consume(d)
    with pytest.raises(sassi.SassiError) as e:
        ctx.read_tables()
    assert e.value.status == sassi.SASSI_EFORMAT
    ctx.close()


def test_index_records_matches_generator():
    P, _, _, _ = gen.preset("c2")
    r = gen.generate_device(P, None, 0, 3000)
    ctx = sassi.Context(r["sites"], P.total_warps, sassi.SASSI_H_ALL)
    out = torch.zeros_like(r["chunk_base"])
    sassi.sassi_index_records(ctx.handle, r["hdr"], r["n"], out)
    torch.cuda.synchronize()
    assert torch.equal(out, r["chunk_base"])
    ctx.close()


def test_device_generator_equals_host_generator():
    for name, warps in (("c1", None), ("c2", 500), ("c3", 40), ("c4", 40), ("c5", 6)):
        P, _, _, _ = gen.preset(name)
        h = gen.generate_host(P, None, 0, warps)
        d = gen.to_host(gen.generate_device(P, None, 0, warps))
        assert np.array_equal(h["hdr"], d["hdr"]), name
        assert np.array_equal(h["addr"], d["addr"]), name
        assert np.array_equal(h["val"], d["val"]), name
        assert np.array_equal(h["chunk_base"], d["chunk_base"]), name


def _gen(name, limit=None, warp_base=0, n_warps=None):
    P, lim, mask, _ = gen.preset(name)
    lim = lim if limit is None else limit
    return P, mask, gen.generate_device(P, lim, warp_base, n_warps)


@pytest.mark.parametrize("every", [False, True])
def test_c1_full(every):
    P, mask, d = _gen("c1")
    mask = sassi.SASSI_H_EVERY if every else mask
    h = gen.to_host(d)
    t = gpu_table(h["sites"], P.total_warps, mask, d)
    o = oracle.run(h["sites"], P.total_warps, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(t, o, len(h["sites"]), P.total_warps) is None


@pytest.mark.parametrize("every", [False, True])
def test_c2_full(every):
    """Config 2 at its full size (10^7 records), bit-exact against the oracle (its four handlers,
    and with the Fig.3 instruction mix added)."""
    P, mask, d = _gen("c2")
    mask = sassi.SASSI_H_EVERY if every else mask
    assert d["n"] == 10_000_000
    h = gen.to_host(d)
    t = gpu_table(h["sites"], P.total_warps, mask, d)
    o = oracle.run(h["sites"], P.total_warps, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(t, o, len(h["sites"]), P.total_warps) is None


def test_c2_back_to_back_launches_dynamic_schedule():
    """The payload fold hands out its last rounds of chunks from a launch-wide counter that the
    launch's last CTA resets: three back-to-back folds of c2 (every item claimed
    dynamically at this size) on one context, without a reset in between, equal three oracle
    passes; a counter left non-zero would skip items in the second launch."""
    P, mask, d = _gen("c2")
    h = gen.to_host(d)
    S, W = len(h["sites"]), P.total_warps
    ctx = sassi.Context(h["sites"], W, mask)
    o = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    for k in range(3):
        ctx.consume(d)
        if k:
            oracle.consume(o, h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
        assert diff_tables(ctx.read_tables(), o, S, W) is None
    ctx.close()


def test_concurrent_folds_on_two_streams():
    """Two folds of c2 into one context on two unordered streams (each launch has its own
    chunk-scheduler words): the tables equal two oracle passes."""
    import torch
    P, mask, d = _gen("c2", limit=3_000_000)
    h = gen.to_host(d)
    S, W = len(h["sites"]), P.total_warps
    ctx = sassi.Context(h["sites"], W, mask)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    for _ in range(3):
        ctx.consume(d, stream=s1)
        ctx.consume(d, stream=s2)
    torch.cuda.synchronize()
    o = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    for _ in range(5):
        oracle.consume(o, h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(ctx.read_tables(), o, S, W) is None
    ctx.close()


def _prefix(d, n):
    """First n records of a device stream (n a multiple of SASSI_CHUNK) with their rows."""
    assert n % 256 == 0
    cb = d["chunk_base"][n // 256].cpu().numpy().view(np.uint64)
    na, nv = int(cb[0]), int(cb[1])
    return dict(hdr=d["hdr"][:n], addr=d["addr"][:na], val=d["val"][:nv],
                chunk_base=d["chunk_base"][: n // 256 + 1], n=n, n_addr_rows=na, n_val_rows=nv,
                sites=d["sites"])


def _properties(sec, n):
    br = sec["br"].astype(np.int64)
    assert (br[:, 2] + br[:, 3] == br[:, 1]).all()
    m = sec["mem"].astype(np.int64)
    assert (m[:, 3] <= m[:, 2]).all() and (m[:, 2] <= m[:, 1]).all() and (4 * m[:, 3] >= m[:, 2]).all()
    assert sec["h32"].sum() == sec["h128"].sum() == m[:, 0].sum()
    for k in range(32):
        assert sec["h32"][k, k + 1:].sum() == 0
    assert int(sec["diag"][0]) == n


@pytest.mark.parametrize("name", ["c3", "c4"])
def test_full_size_exact_and_properties(name):
    """10^8 records in the bench's launch configuration: the whole stream folded on the GPU equals
    the oracle over the whole stream in every table section (the oracle runs over host-generated
    warp shards in parallel processes, merged with its own merge: tests/oracle_shards.py); the
    invariants hold, and consuming the stream in two pieces equals consuming it at once."""
    from oracle_shards import oracle_full
    P, mask, d = _gen(name)
    assert d["n"] == 100_000_000
    S, W = len(d["sites"]), P.total_warps
    full = gpu_table(d["sites"], W, mask, d)
    sec = oracle.sections(full, S, W)
    _properties(sec, d["n"])
    o, n = oracle_full(name, mask, limit=d["n"])
    assert n == d["n"]
    assert diff_tables(full, o, S, W) is None
    # split consumption == single pass (chunk-aligned split; rows addressed absolutely)
    ctx = sassi.Context(d["sites"], W, mask)
    half = (d["n"] // 2) // 256 * 256
    hdr = d["hdr"]
    a = dict(d, hdr=hdr[:half], chunk_base=d["chunk_base"][: half // 256 + 1], n=half)
    b = dict(d, hdr=hdr[half:], chunk_base=d["chunk_base"][half // 256:], n=d["n"] - half)
    ctx.consume(a)
    ctx.consume(b)
    assert np.array_equal(ctx.read_tables(), full)
    ctx.close()


def test_c4_full_instcount_exact_and_sampling():
    """Config 4 in full: per-thread counts over 10^8 records for 10^6 threads, bit-exact, then
    1,000 injection-site draws (L629) equal the oracle's draws on the same counts."""
    P, mask, d = _gen("c4")
    W = P.total_warps
    ctx = sassi.Context(d["sites"], W, mask)
    ctx.consume(d)
    t = ctx.read_tables()
    hdr = d["hdr"].cpu().numpy().view(np.uint32).reshape(-1, 4).view(gen.HDR_DTYPE).reshape(-1)
    o = oracle.table_init(len(d["sites"]), W, mask)
    oracle.consume(o, d["sites"], W, mask, hdr, None, None, d["n_addr_rows"], d["n_val_rows"])
    s2 = d["sites"]
    so, st = oracle.sections(o, len(s2), W), oracle.sections(t, len(s2), W)
    assert np.array_equal(st["counts"], so["counts"])
    assert np.array_equal(st["diag"][:4], so["diag"][:4])
    assert int(so["counts"].sum()) > 0
    got = ctx.sample(1000, 20150616)
    exp = oracle.sample(so["counts"], 1000, 20150616)
    assert np.array_equal(got, exp)
    ctx.close()


def test_multi_launch_split_equals_single_launch(monkeypatch):
    """sassi_consume splits n records into launches of at most 2^29 (32-bit indices inside a
    launch). Lowering the split to 4,096 / 65,536 records (SASSI_MAX_LAUNCH_RECORDS) must give the
    single-launch tables bit for bit on c2 (every handler, payload rows addressed per launch)."""
    P, mask, d = _gen("c2")
    S, W = len(d["sites"]), P.total_warps
    full = gpu_table(d["sites"], W, sassi.SASSI_H_EVERY, d)
    for per in ("4096", "65536"):
        monkeypatch.setenv("SASSI_MAX_LAUNCH_RECORDS", per)
        ctx = sassi.Context(d["sites"], W, sassi.SASSI_H_EVERY)
        n0 = ctx.kernel_launches()
        ctx.consume(d)
        assert ctx.kernel_launches() - n0 == -(-d["n"] // int(per))
        assert diff_tables(ctx.read_tables(), full, S, W) is None
        ctx.close()


@pytest.mark.parametrize("seed,n,n_warps", [(1, 1, 1), (2, 40, 1), (3, 700, 33), (4, 3000, 300),
                                             (5, 20000, 1500)])
def test_sampling_edge_cases(seed, n, n_warps):
    """Injection-site draws (L629) against the oracle's upper_bound on the same counts: one warp
    (33 prefix entries: the 32-ary search's last round only), prefix lengths just above a multiple
    of 32, thousands of threads with most counts zero; k = 0 and a zero total (ESTATE)."""
    s, W, hdr, addr, val = random_trace(3000 + seed, n=n, n_warps=n_warps)
    mask = sassi.SASSI_H_INSTCOUNT
    so = oracle.sections(oracle.run(s, W, mask, hdr, addr, val), len(s), W)
    ctx = sassi.Context(s, W, mask)
    ctx.consume(to_device(s, hdr, addr, val))
    if int(so["counts"].sum()) == 0:
        with pytest.raises(sassi.SassiError) as e:
            ctx.sample(10, seed)
        assert e.value.status == sassi.SASSI_ESTATE
    else:
        for k in (0, 1, 33, 1000):
            assert np.array_equal(ctx.sample(k, seed), oracle.sample(so["counts"], k, seed))
    ctx.reset()
    with pytest.raises(sassi.SassiError) as e:   # nothing counted since the reset
        ctx.sample(5, seed)
    assert e.value.status == sassi.SASSI_ESTATE
    ctx.close()


def test_sampling_device_output_matches_host_output():
    """sassi_sample_sites_device (no synchronisation, draws in device memory) == the host-output
    form == the oracle; status 1 and outputs untouched when nothing was counted."""
    s, W, hdr, addr, val = random_trace(5151, n=4000, n_warps=40)
    mask = sassi.SASSI_H_INSTCOUNT
    so = oracle.sections(oracle.run(s, W, mask, hdr, addr, val), len(s), W)
    ctx = sassi.Context(s, W, mask)
    ctx.consume(to_device(s, hdr, addr, val))
    out = torch.full((300 * 32,), 0xAB, dtype=torch.uint8, device="cuda")
    status = torch.full((1,), 7, dtype=torch.int32, device="cuda")
    ctx.sample_device(out, status, 300, 77)
    torch.cuda.synchronize()
    assert int(status.item()) == 0
    got = np.frombuffer(out.cpu().numpy().tobytes(), dtype=sassi.INJ_DTYPE)
    assert np.array_equal(got, ctx.sample(300, 77))
    assert np.array_equal(got, oracle.sample(so["counts"], 300, 77))
    ctx.reset()
    out.fill_(0xAB)
    ctx.sample_device(out, status, 300, 77)
    torch.cuda.synchronize()
    assert int(status.item()) == 1 and bool((out == 0xAB).all())
    ctx.close()


def test_sampling_one_thread_holds_every_count():
    """All eligible instructions on the last thread: every draw must pick it (upper_bound at the
    very end of the prefix), dyn_index = k itself."""
    s, W, hdr, addr, val = random_trace(4242, n=2000, n_warps=64)
    elig = [i for i, x in enumerate(s) if int(x["n_gpr_dst"]) > 0 and not int(x["flags"]) & gen.F_MEM]
    hdr = hdr.copy()
    hdr["pc"] = s["pc"][elig[0]]
    hdr["warp"] = W - 1
    hdr["active"] = 0x80000000
    hdr["mask2"] = 0xFFFFFFFF
    addr = np.zeros((0, 32), np.uint64)
    val = np.zeros((len(hdr) * int(s["n_gpr_dst"][elig[0]]), 32), np.uint32)
    so = oracle.sections(oracle.run(s, W, sassi.SASSI_H_INSTCOUNT, hdr, addr, val), len(s), W)
    assert int(so["counts"][-1]) == len(hdr) and int(so["counts"].sum()) == len(hdr)
    ctx = sassi.Context(s, W, sassi.SASSI_H_INSTCOUNT)
    ctx.consume(to_device(s, hdr, addr, val))
    got = ctx.sample(500, 99)
    assert np.array_equal(got, oracle.sample(so["counts"], 500, 99))
    assert (got["thread"] == 32 * W - 1).all()
    ctx.close()


def test_c5_sampled_shards():
    """Config 5 (4x10^9 records over 8 shards of 16,384 warps): each of two shards is generated
    with its global warp ids; a 3x10^6-record prefix of each is exact against the oracle, and the
    merged tables of the two prefixes equal the oracle's merge."""
    P, _, mask, _ = gen.preset("c5")
    W = P.total_warps
    acc = None
    for shard in (0, 5):
        d = gen.generate_device(P, 3_000_000, shard * 16384, 16384)
        h = gen.to_host(d)
        S = len(h["sites"])
        o = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
        t = gpu_table(h["sites"], W, mask, d)
        assert diff_tables(t, o, S, W) is None
        acc = o if acc is None else oracle.merge(acc, o, S, W)
    assert int(oracle.sections(acc, S, W)["counts"].sum()) > 0


def test_reset_and_accumulate():
    s, W, hdr, addr, val = random_trace(4242, n=4000)
    d = to_device(s, hdr, addr, val)
    ctx = sassi.Context(s, W, sassi.SASSI_H_ALL)
    ctx.consume(d)
    once = ctx.read_tables()
    ctx.consume(d)
    twice = ctx.read_tables()
    o = oracle.run(s, W, oracle.H_ALL, hdr, addr, val)
    oracle.consume(o, s, W, oracle.H_ALL, hdr, addr, val)
    assert np.array_equal(twice, o)
    ctx.reset()
    ctx.consume(d)
    assert np.array_equal(ctx.read_tables(), once)
    with pytest.raises(sassi.SassiError):
        sassi.sassi_attach_handler(ctx.handle, 1)    # after consume: ESTATE
    ctx.close()


@pytest.mark.parametrize("mask", [15, 1, 2, 4, 6, 8, 31])
def test_consume_host_equals_device(mask):
    """sassi_consume_host copies only what the attached handlers read (address rows for memdiv,
    value rows for value, the chunk index for either): every handler set folds from host buffers
    to the device fold's tables."""
    P, _, d = _gen("c2", limit=3_000_000)
    h = gen.to_host(d)
    t_dev = gpu_table(h["sites"], P.total_warps, mask, d)
    ctx = sassi.Context(h["sites"], P.total_warps, mask)
    hrec = dict(hdr=np.ascontiguousarray(h["hdr"]), addr=h["addr"], val=h["val"],
                chunk_base=h["chunk_base"], n=h["n"], n_addr_rows=h["n_addr_rows"],
                n_val_rows=h["n_val_rows"])
    ctx.consume_host(hrec)
    assert np.array_equal(ctx.read_tables(), t_dev)
    ctx.close()


def test_consume_host_header_only_reads_no_rows():
    """A header-only handler set (per-thread counts, the injection-profiling pass) folds from the
    headers alone: the host row buffers passed here hold one row each while the record counts
    say millions, so any copy of rows would read far past them."""
    P, _, d = _gen("c2", limit=3_000_000)
    h = gen.to_host(d)
    mask = sassi.SASSI_H_INSTCOUNT
    t_dev = gpu_table(h["sites"], P.total_warps, mask, d)
    ctx = sassi.Context(h["sites"], P.total_warps, mask)
    hrec = dict(hdr=np.ascontiguousarray(h["hdr"]), addr=np.zeros((1, 32), np.uint64),
                val=np.zeros((1, 32), np.uint32), chunk_base=h["chunk_base"], n=h["n"],
                n_addr_rows=h["n_addr_rows"], n_val_rows=h["n_val_rows"])
    ctx.consume_host(hrec)
    assert np.array_equal(ctx.read_tables(), t_dev)
    ctx.close()


def test_merge_single_rank_nccl():
    """sassi_merge through a real 1-rank NCCL communicator: pack -> ncclAllReduce -> unpack must
    leave the tables unchanged (sums over one rank; masks survive the byte-expansion round trip)."""
    s, W, hdr, addr, val = random_trace(555, n=6000)
    d = to_device(s, hdr, addr, val)
    ctx = sassi.Context(s, W, sassi.SASSI_H_EVERY)
    sel = [i for i in range(len(s)) if (int(s[i]["flags"]) & oracle.F_MEM)
           and int(s[i]["domain"]) == oracle.D_GLOBAL][:4]
    ctx.select_memdiv_pcs([int(s[i]["pc"]) for i in sel])
    ctx.consume(d)
    before = ctx.read_tables()
    uid = sassi.sassi_nccl_get_unique_id()
    comm = sassi.sassi_nccl_comm_create(1, 0, uid, torch.cuda.current_device())
    ctx.merge(comm)
    after = ctx.read_tables()
    sassi.sassi_nccl_comm_destroy(comm)
    ctx.close()
    assert np.array_equal(after, before)
    assert np.array_equal(after, oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val, pcs=sel))


def test_c5_full_shard_exact():
    """One full c5 shard (16,384 warps, ~4.9x10^8 records, ~90 GB in HBM) folded in the bench's
    launch configuration equals the oracle over the whole shard in every table section (parallel
    host oracle over warp sub-shards, merged); the per-PC tables also satisfy the invariants and
    two chunk-aligned halves accumulate to the single pass."""
    from oracle_shards import oracle_full
    P, _, mask, _ = gen.preset("c5")
    W = P.total_warps
    shard = 3
    d = gen.generate_device(P, None, shard * 16384, 16384)
    S = len(d["sites"])
    assert d["n"] > 4 * 10**8
    full = gpu_table(d["sites"], W, mask, d)
    sec = oracle.sections(full, S, W)
    _properties(sec, d["n"])
    o, n = oracle_full("c5", mask, warp_base=shard * 16384, n_warps=16384, warps_per_job=512)
    assert n == d["n"]
    assert diff_tables(full, o, S, W) is None
    # two chunk-aligned halves accumulate to the single pass
    half = (d["n"] // 2) // 256 * 256
    ctx = sassi.Context(d["sites"], W, mask)
    ctx.consume(dict(d, hdr=d["hdr"][:half], chunk_base=d["chunk_base"][: half // 256 + 1], n=half))
    ctx.consume(dict(d, hdr=d["hdr"][half:], chunk_base=d["chunk_base"][half // 256:], n=d["n"] - half))
    assert np.array_equal(ctx.read_tables(), full)
    ctx.close()


def test_permuted_records_give_identical_tables():
    """§4.2 item 5: every table is a commutative fold — shuffling whole records (with their rows)
    across chunks and batches changes nothing, on the GPU as in the oracle."""
    from test_oracle import permute_records
    s, W, hdr, addr, val = random_trace(2024, n=6000)
    o = oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val)
    for seed in (1, 2):
        h2, a2, v2 = permute_records(s, hdr, addr, val, seed)
        t = gpu_table(s, W, sassi.SASSI_H_EVERY, to_device(s, h2, a2, v2))
        assert diff_tables(t, o, len(s), W) is None


def test_virtual_ranks_merged_on_host_equal_single_pass():
    """§4.2 item 8 (multi-GPU without a cluster): P shards consumed into P contexts on one GPU,
    merged with the oracle's merge, equal the unsharded fold."""
    from test_oracle import _split
    s, W, hdr, addr, val = random_trace(99, n=9000)
    single = gpu_table(s, W, sassi.SASSI_H_EVERY, to_device(s, hdr, addr, val))
    acc = oracle.table_init(len(s), W, sassi.SASSI_H_EVERY)
    parts = []
    for half in _split(s, hdr, addr, val, 4000):
        parts += _split(s, *half, len(half[0]) // 3)
    for h, a, v in parts:
        t = gpu_table(s, W, sassi.SASSI_H_EVERY, to_device(s, h, a, v))
        oracle.merge(acc, t, len(s), W)
    assert diff_tables(acc, single, len(s), W) is None
    assert np.array_equal(single, oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val))


def _global_mem_sites(s):
    return [i for i in range(len(s)) if (int(s[i]["flags"]) & oracle.F_MEM)
            and int(s[i]["domain"]) == oracle.D_GLOBAL]


@pytest.mark.parametrize("mask", [2, 15, 31])
def test_per_pc_memdiv_matrices_t0(mask):
    s = T0.sites()
    hdr, addr, val = T0.records()
    t = gpu_table(s, T0.N_WARPS, mask, to_device(s, hdr, addr, val), pcs=[0x30, 0x20])
    o = oracle.run(s, T0.N_WARPS, mask, hdr, addr, val, pcs=[2, 1])
    assert diff_tables(t, o, len(s), T0.N_WARPS) is None
    sec = oracle.sections(t, len(s), T0.N_WARPS)
    assert list(map(int, sec["pcsel"])) == [3, 2, 0, 0]
    assert np.array_equal(sec["pcmat"][0] + sec["pcmat"][1], sec["h32"])


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_per_pc_memdiv_matrices_random(seed):
    s, W, hdr, addr, val = random_trace(3000 + seed, n=8000)
    sel = _global_mem_sites(s)[:4]
    o = oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val, pcs=sel)
    t = gpu_table(s, W, sassi.SASSI_H_EVERY, to_device(s, hdr, addr, val),
                  pcs=[int(s[i]["pc"]) for i in sel])
    assert diff_tables(t, o, len(s), W) is None


def test_per_pc_memdiv_matrices_c2_full():
    """c2 (10^7 records) with four selected gather / unit-stride sites."""
    P, mask, d = _gen("c2")
    h = gen.to_host(d)
    sel = _global_mem_sites(h["sites"])[:4]
    t = gpu_table(h["sites"], P.total_warps, mask, d, pcs=[int(h["sites"][i]["pc"]) for i in sel])
    o = oracle.run(h["sites"], P.total_warps, mask, h["hdr"], h["addr"], h["val"], pcs=sel)
    assert diff_tables(t, o, len(h["sites"]), P.total_warps) is None
    assert oracle.sections(t, len(h["sites"]), P.total_warps)["pcmat"].sum() > 0


def test_select_memdiv_pcs_errors():
    s = T0.sites()
    ctx = sassi.Context(s, T0.N_WARPS, 2)
    for bad in ([0x40], [0x50], [0x999], [0x20, 0x20], [0x20, 0x30, 0x20, 0x30, 0x20]):
        with pytest.raises(sassi.SassiError) as e:   # ALU, shared-memory, unregistered, twice, > 4
            ctx.select_memdiv_pcs(bad)
        assert e.value.status == sassi.SASSI_EINVAL
    hdr, addr, val = T0.records()
    ctx.consume(to_device(s, hdr, addr, val))
    with pytest.raises(sassi.SassiError) as e:
        ctx.select_memdiv_pcs([0x20])
    assert e.value.status == sassi.SASSI_ESTATE
    ctx.reset()
    ctx.select_memdiv_pcs([0x20])
    ctx.select_memdiv_pcs([])
    ctx.close()


@pytest.mark.parametrize("k", [1, 4])
def test_memdiv_topk_two_pass(k):
    """sassi_select_memdiv_topk: pass 1 folds c2 (10^7 records), the k most
    divergent GLOBAL pcs by sectors per warp access are picked (== the oracle's ranking of the
    oracle's table, reading R26), the context is reset, and pass 2 keeps their matrices: every
    table equals the oracle run with that selection."""
    P, mask, d = _gen("c2", limit=2_000_000)
    h = gen.to_host(d)
    S, W = len(h["sites"]), P.total_warps
    o1 = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    want = oracle.memdiv_topk(o1, h["sites"], W, k)
    ctx = sassi.Context(h["sites"], W, mask)
    ctx.consume(d)
    got = ctx.select_memdiv_topk(k)
    assert [int(x) for x in got] == [int(h["sites"]["pc"][i]) for i in want]
    assert np.array_equal(ctx.read_tables(), oracle.table_init(S, W, mask, pcs=want))  # reset
    ctx.consume(d)
    t = ctx.read_tables()
    ctx.close()
    o2 = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"], pcs=want)
    assert diff_tables(t, o2, S, W) is None
    assert oracle.sections(t, S, W)["pcmat"][:k].sum() > 0


@pytest.mark.parametrize("seed", [0, 1])
def test_global_only_address_rows_random(seed):
    """SASSI_ADDR_ROWS_GLOBAL: the same records with only the GLOBAL sites' address rows (the
    shared-memory rows split off by the producer) fold to the oracle's tables of the full stream;
    sassi_index_records follows the layout."""
    s, W, hdr, addr, val = random_trace(6100 + seed, n=20000)
    o = oracle.run(s, W, sassi.SASSI_H_EVERY, hdr, addr, val)
    full = to_device(s, hdr, addr, val)
    d = gen.split_global_rows(dict(full, sites=s))
    assert d["n_addr_rows"] < full["n_addr_rows"]
    ctx = sassi.Context(s, W, sassi.SASSI_H_EVERY)
    ctx.set_addr_rows(sassi.SASSI_ADDR_ROWS_GLOBAL)
    cb = torch.zeros_like(d["chunk_base"])
    sassi.sassi_index_records(ctx.handle, d["hdr"], d["n"], cb)
    torch.cuda.synchronize()
    assert torch.equal(cb, d["chunk_base"])
    ctx.consume(d)
    assert diff_tables(ctx.read_tables(), o, len(s), W) is None
    ctx.close()


def test_global_only_address_rows_c3_host_consume():
    """c3 (2x10^6-record prefix, 12 % shared-memory records) from HOST buffers with the shared rows
    split off: sassi_consume_host copies only the GLOBAL rows and the tables equal the oracle."""
    P, mask, d = _gen("c3", limit=2_000_128)
    h = gen.to_host(d)
    g = gen.split_global_rows(h)
    S, W = len(h["sites"]), P.total_warps
    ctx = sassi.Context(h["sites"], W, mask)
    ctx.set_addr_rows(sassi.SASSI_ADDR_ROWS_GLOBAL)
    ctx.consume_host(dict(hdr=np.ascontiguousarray(g["hdr"]), addr=g["addr"], val=g["val"],
                          chunk_base=g["chunk_base"], n=g["n"], n_addr_rows=g["n_addr_rows"],
                          n_val_rows=g["n_val_rows"]))
    t = ctx.read_tables()
    with pytest.raises(sassi.SassiError):
        ctx.set_addr_rows(sassi.SASSI_ADDR_ROWS_ALL)          # after a consume: ESTATE
    ctx.close()
    o = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    assert diff_tables(t, o, S, W) is None
    assert g["n_addr_rows"] < h["n_addr_rows"]


def test_sample_sites_multi_random_profiles():
    """sassi_sample_sites_multi over five random-trace profiles of different warp counts equals the
    oracle's draws over the concatenated counts; a profile with nothing counted contributes none."""
    profs, oprofs, ctxs = [], [], []
    for i, (n, w) in enumerate([(3000, 5), (500, 1), (7000, 40), (1, 3), (20000, 70)]):
        s, W, hdr, addr, val = random_trace(9100 + i, n=n, n_warps=w)
        ctx = sassi.Context(s, W, sassi.SASSI_H_INSTCOUNT)
        ctx.consume(to_device(s, hdr, addr, val))
        c = oracle.sections(oracle.run(s, W, sassi.SASSI_H_INSTCOUNT, hdr, addr, val), len(s), W)["counts"]
        profs.append((ctx, 10 + i, i))
        oprofs.append((c, 10 + i, i))
        ctxs.append(ctx)
    for k, seed in ((1, 0), (33, 5), (1000, 2**40 + 3)):
        assert np.array_equal(sassi.sassi_sample_sites_multi(profs, k, seed), oracle.sample_multi(oprofs, k, seed))
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_sample_sites_multi([profs[0], profs[0]], 4, 1)
    assert e.value.status == sassi.SASSI_EINVAL
    for c in ctxs:
        c.close()
