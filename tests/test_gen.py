"""Generator tests (CPU): the c1 stream equals a literal builder written from the c1 recipe, the
oracle reproduces c1's closed-form tables, and the chunk index is consistent with the rows."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen
from paper_conf_isca_stephensonhlejn15_b200.gen import presets

FULL = 0xFFFFFFFF
VA, GB = presets.VA, presets.GB


def c1_literal():
    """c1 = vecadd over n = 12,800 floats by 4 warps (128 threads), grid-stride i += 128, with
    `if (i % 3 == 0) load x[32*i]`; written out instruction by instruction."""
    A, B, C, X = VA, VA + GB, VA + 2 * GB, VA + 3 * GB
    H, Arows, Vdet = [], [], []
    for w in range(4):
        lanes = np.arange(32, dtype=np.uint64)
        H.append((0x100, w, FULL, FULL))                 # S2R R0 = lane
        Vdet.append(("lane", lanes.astype(np.uint32)))
        H.append((0x110, w, FULL, FULL))                 # IMAD R3 = global tid
        Vdet.append(("e", (32 * w + lanes).astype(np.uint32)))
        for it in range(100):
            e = (128 * it + 32 * w + lanes).astype(np.uint64)
            H.append((0x120, w, FULL, FULL))             # IMAD.WIDE &a[i]
            Vdet += [("lo", ((A + 4 * e) & 0xFFFFFFFF).astype(np.uint32)),
                     ("hi", ((A + 4 * e) >> 32).astype(np.uint32))]
            H.append((0x130, w, FULL, FULL))             # IMAD.WIDE &b[i]
            Vdet += [("lo", ((B + 4 * e) & 0xFFFFFFFF).astype(np.uint32)),
                     ("hi", ((B + 4 * e) >> 32).astype(np.uint32))]
            H.append((0x140, w, FULL, FULL)); Arows.append(A + 4 * e); Vdet.append(("rand", None))
            H.append((0x150, w, FULL, FULL)); Arows.append(B + 4 * e); Vdet.append(("rand", None))
            H.append((0x160, w, FULL, FULL)); Vdet.append(("rand", None))          # FADD
            H.append((0x170, w, FULL, FULL)); Arows.append(C + 4 * e)              # STG
            H.append((0x180, w, FULL, FULL))                                       # ISETP
            m3 = int(sum(1 << l for l in range(32) if int(e[l]) % 3 == 0))
            H.append((0x190, w, FULL, m3))                                         # @P0 BRA
            H.append((0x1A0, w, m3, m3)); Arows.append(X + 128 * e); Vdet.append(("rand", None))
            H.append((0x1B0, w, FULL, FULL)); Vdet.append(("e", (e + 128).astype(np.uint32)))
            H.append((0x1C0, w, FULL, FULL))                                       # ISETP
            H.append((0x1D0, w, FULL, FULL if it < 99 else 0))                     # loop BRA
        H.append((0x1E0, w, FULL, FULL))                                           # EXIT
    return np.array(H, np.uint32).view(gen.HDR_DTYPE).reshape(-1), Arows, Vdet


def test_c1_matches_literal_builder():
    P, lim, mask, _ = gen.preset("c1")
    r = gen.generate_host(P, lim)
    hdr, arows, vdet = c1_literal()
    assert r["n"] == len(hdr) == 4 * (2 + 100 * 12 + 1)
    assert np.array_equal(r["hdr"], hdr)
    assert r["n_addr_rows"] == len(arows) and r["n_val_rows"] == len(vdet)
    # addresses on the lanes whose payload is meaningful (active & mask2) — mem records in order
    mem_hdr = hdr[np.isin(hdr["pc"], [0x140, 0x150, 0x170, 0x1A0])]
    for k, (h, row) in enumerate(zip(mem_hdr, arows)):
        m = int(h["active"]) & int(h["mask2"])
        for l in range(32):
            if (m >> l) & 1:
                assert int(r["addr"][k, l]) == int(row[l])
    for k, (kind, v) in enumerate(vdet):
        if v is not None:
            assert np.array_equal(r["val"][k], v), (k, kind)


def test_c1_oracle_closed_forms():
    """c1's tables in closed form: the i%3 branch splits every warp (10 or 11 of 32 lanes have
    i % 3 == 0), the loop branch diverges never, unit-stride loads give 4 sectors / 1 line."""
    P, lim, mask, _ = gen.preset("c1")
    r = gen.generate_host(P, lim)
    s = r["sites"]
    t = oracle.run(s, 4, oracle.H_ALL, r["hdr"], r["addr"], r["val"])
    sec = oracle.sections(t, len(s), 4)
    idx = {int(x["pc"]): i for i, x in enumerate(s)}
    n3 = len(range(0, 12800, 3))                                    # 4267 elements with i%3==0
    assert list(sec["br"][idx[0x190]]) == [400, 12800, n3, 12800 - n3, 400]
    assert list(sec["br"][idx[0x1D0]]) == [400, 12800, 4 * 99 * 32, 128, 0]
    for pc in (0x140, 0x150, 0x170):
        assert list(sec["mem"][idx[pc]]) == [400, 12800, 1600, 400]
    assert list(sec["mem"][idx[0x1A0]]) == [400, n3, n3, n3]
    h32 = np.zeros((32, 32), np.int64)
    h32[31, 3] = 1200
    for w in range(4):
        for it in range(100):
            c = len([l for l in range(32) if (128 * it + 32 * w + l) % 3 == 0])
            h32[c - 1, c - 1] += 1
    assert np.array_equal(sec["h32"].astype(np.int64), h32)
    # per-thread counts: prologue 2 + 9 eligible per iteration (2 IMAD.WIDE, 2 LDG, FADD, STG,
    # 2 ISETP, IADD) + the x[32 i] load in iterations where i % 3 == 0
    e0 = np.arange(128)
    expect = 2 + 900 + np.array([sum(1 for it in range(100) if (128 * it + t) % 3 == 0)
                                  for t in e0])
    assert np.array_equal(sec["counts"].astype(np.int64), expect)
    assert list(map(int, sec["diag"][:4])) == [4812, 0, 0, 0]


def test_c1_instmix_closed_form():
    """Fig.3 on c1 by hand: 128 threads; prologue 2 numeric; per iteration 6 numeric (2 IMAD.WIDE,
    FADD, 2 ISETP, IADD), 3 memory (2 LDG, STG, all 4 B), 2 control transfers (2 BRA), and the
    x[32 i] load on the 4,267 (thread, iteration) pairs with i % 3 == 0; EXIT is one more control
    transfer per thread."""
    P, lim, mask, _ = gen.preset("c1")
    r = gen.generate_host(P, lim)
    s = r["sites"]
    t = oracle.run(s, 4, oracle.H_INSTMIX, r["hdr"], r["addr"], r["val"])
    sec = oracle.sections(t, len(s), 4)
    n3 = len(range(0, 12800, 3))
    numeric = 2 * 128 + 6 * 12800
    memory = 3 * 12800 + n3
    ctrl = 2 * 12800 + 128
    assert list(map(int, sec["imix"])) == [memory, 0, ctrl, 0, numeric, 0,
                                           numeric + memory + ctrl, 0]
    idx = {int(x["pc"]): i for i, x in enumerate(s)}
    assert int(sec["mix"][idx[0x1A0]]) == n3 and int(sec["mix"][idx[0x140]]) == 12800


def _walk_rows(sites, hdr):
    """(addr rows, val rows) before each record, from the site table only."""
    pcs = {int(x["pc"]): x for x in sites}
    na = np.zeros(len(hdr) + 1, np.int64)
    nv = np.zeros(len(hdr) + 1, np.int64)
    for i, h in enumerate(hdr):
        s = pcs.get(int(h["pc"]))
        na[i + 1] = na[i] + (1 if s is not None and int(s["flags"]) & gen.F_MEM else 0)
        nv[i + 1] = nv[i] + (int(s["n_gpr_dst"]) if s is not None else 0)
    return na, nv


@pytest.mark.parametrize("name,warps,limit", [("c1", None, None), ("c1", None, 1000),
                                              ("c2", 60, None), ("c2", 60, 5000),
                                              ("c3", 3, None), ("c4", 3, 7777), ("c5", 2, None)])
def test_chunk_index_consistent(name, warps, limit):
    P, _, _, _ = gen.preset(name)
    r = gen.generate_host(P, limit, 0, warps)
    na, nv = _walk_rows(r["sites"], r["hdr"])
    n = r["n"]
    if limit is not None:
        assert n == limit
    nch = (n + gen.CHUNK - 1) // gen.CHUNK
    cb = r["chunk_base"]
    assert cb.shape == (nch + 1, 2)
    for c in range(nch):
        assert (int(cb[c, 0]), int(cb[c, 1])) == (na[c * gen.CHUNK], nv[c * gen.CHUNK])
    assert (int(cb[nch, 0]), int(cb[nch, 1])) == (na[n], nv[n]) == (r["n_addr_rows"], r["n_val_rows"])
    # the oracle accepts the stream (rows consistent with records)
    oracle.run(r["sites"], P.total_warps, oracle.H_ALL, r["hdr"], r["addr"], r["val"])


def test_shards_concatenate_to_whole():
    P, _, _, _ = gen.preset("c2")
    whole = gen.generate_host(P, None, 0, 40)
    a = gen.generate_host(P, None, 0, 17)
    b = gen.generate_host(P, None, 17, 23)
    assert np.array_equal(np.concatenate([a["hdr"], b["hdr"]]), whole["hdr"])
    assert np.array_equal(np.concatenate([a["addr"], b["addr"]]), whole["addr"])
    assert np.array_equal(np.concatenate([a["val"], b["val"]]), whole["val"])


def test_c2_shape():
    """BFS-shaped mix: ~12 % conditional branches, ~10 % of them divergent, ~30 %
    memory records mostly random gathers, ~75 % register-writing rows, 40 % frontier iterations."""
    P, _, _, _ = gen.preset("c2")
    r = gen.generate_host(P, None, 0, 400)
    s = r["sites"]
    t = oracle.run(s, P.total_warps, oracle.H_ALL, r["hdr"], r["addr"], r["val"])
    sec = oracle.sections(t, len(s), P.total_warps)
    n = r["n"]
    nbr = int(sec["br"][:, 0].sum())
    assert 0.08 < nbr / n < 0.16
    assert 0.04 < int(sec["br"][:, 4].sum()) / nbr < 0.20
    assert 0.2 < r["n_addr_rows"] / n < 0.4
    assert 0.6 < r["n_val_rows"] / n < 0.9


def test_split_global_rows_host():
    """SASSI_ADDR_ROWS_GLOBAL input preparation: the kept rows are exactly the rows of the records
    at GLOBAL memory sites, in record order, and chunk_base's addr_row counts them."""
    P, _, _, _ = gen.preset("c3")
    r = gen.generate_host(P, 5000, 0, 4)
    g = gen.split_global_rows(r)
    site = {int(x["pc"]): x for x in r["sites"]}
    rows, kept, cnt = 0, [], [0]
    for i, h in enumerate(r["hdr"]):
        st = site.get(int(h["pc"]))
        if st is not None and int(st["flags"]) & gen.F_MEM:
            if int(st["domain"]) == gen.D_GLOBAL:
                kept.append(rows)
            rows += 1
        cnt.append(len(kept))
    assert g["n_addr_rows"] == len(kept) < r["n_addr_rows"]
    assert np.array_equal(g["addr"], r["addr"][kept])
    assert [int(x) for x in g["chunk_base"][:, 0]] == [cnt[min(256 * c, r["n"])] for c in range(len(g["chunk_base"]))]
    assert np.array_equal(g["chunk_base"][:, 1], r["chunk_base"][:, 1])
