"""Error injection on the instrumented kernels (§8.1):
profile -> draw sites -> one injection run per site. The injected instruction, target kind (a GPR
destination chosen by reg_seed % n_gpr_dst, the stored word, the written predicate or one of the 4
condition-code bits, L621 / L629), register value and bit of every run equal what the oracle
locates in the same kernel's trace (the dyn-th eligible, not-predicated-out dynamic instruction of
the thread, reading R23); outcomes follow their rules."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

SMALL = {"vecadd": 12800, "bfs": 4096, "sgemm": 64, "stencil": 64}
TARGET_CODE = {"gpr": 0, "mem": 1, "pred": 2, "cc": 3}
# target kinds a campaign reaches: vecadd has GPR (1 and 2 destinations), stores, a predicate and a
# condition-code site; bfs and stencil a predicate site; sgemm GPRs and stores only
EXPECTED_KINDS = {"vecadd": {0, 1, 2, 3}, "bfs": {0, 1, 2}, "sgemm": {0, 1}, "stencil": {0, 1, 2}}
# the global stores into the kernels' outputs (a flipped stored word is always visible)
OUTPUT_STORES = {"vecadd": {3}, "bfs": {8}, "sgemm": {9}, "stencil": {7}}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@pytest.mark.parametrize("name", list(SMALL))
def test_injection_targets_equal_oracle_locate(name):
    ik = sassi.InstrumentedKernel(name, SMALL[name])
    sites, outs = ik.injection_campaign(k=300, seed=77)
    ctx = ik.context(sassi.SASSI_H_INSTCOUNT)
    rec = ik.trace(ctx)
    ctx.close()
    h = gen.to_host(rec)
    assert (outs["outcome"] != sassi.SASSI_INJ_NOT_REACHED).all()
    for st, o in zip(sites, outs):
        loc = oracle.locate_injection(h["sites"], h["hdr"], h["val"], int(st["thread"]),
                                      int(st["dyn_index"]), int(st["reg_seed"]), int(st["bit_seed"]))
        assert loc is not None
        assert int(o["site"]) == loc["site"]
        assert int(o["bit"]) == loc["bit"]
        assert int(o["target"]) == TARGET_CODE[loc["target"]]
        if loc["target"] == "gpr":   # the chosen destination's value (reg_seed % n_gpr_dst)
            assert int(o["before"]) == loc["before"]
        if loc["target"] == "pred":
            assert int(o["before"]) in (0, 1) and int(o["bit"]) == 0
        if loc["target"] == "cc":
            assert int(o["before"]) < 16 and int(o["bit"]) < 4
        assert int(o["after"]) == int(o["before"]) ^ (1 << int(o["bit"]))
    kinds = set(int(t) for t in outs["target"])
    assert kinds == EXPECTED_KINDS[name], kinds
    ik.close()


def test_injection_two_destination_choice():
    """vecadd's IMAD.WIDE site (s8) writes R4:R5: reg_seed picks the destination (L629), so the
    flipped value is the low or the high half of the 64-bit address, as the oracle locates."""
    ik = sassi.InstrumentedKernel("vecadd", SMALL["vecadd"])
    ctx = ik.context(sassi.SASSI_H_INSTCOUNT)
    rec = ik.trace(ctx)
    ctx.close()
    h = gen.to_host(rec)
    s8 = [i for i, r in enumerate(h["hdr"]) if r["pc"] == h["sites"][8]["pc"] and r["warp"] == 0][0]
    # thread 0's eligible instructions before its first s8 record: count them from the trace
    dyn = sum(1 for r in h["hdr"][:s8] if r["warp"] == 0 and r["pc"] in h["sites"]["pc"] and
              (h["sites"][list(h["sites"]["pc"]).index(r["pc"])]["n_gpr_dst"] > 0 or
               h["sites"][list(h["sites"]["pc"]).index(r["pc"])]["flags"] & (gen.F_MEM | gen.F_WRITES_PRED | gen.F_WRITES_CC))
              and (r["active"] & r["mask2"]) & 1)
    st = np.zeros(2, dtype=sassi.INJ_DTYPE)
    st["thread"] = 0
    st["dyn_index"] = dyn
    st["reg_seed"] = [4, 7]                         # destination 0 (low half), then 1 (high half)
    st["bit_seed"] = [3, 3]
    outs = ik.inject(st)
    for t, o in zip(st, outs):
        loc = oracle.locate_injection(h["sites"], h["hdr"], h["val"], 0, dyn, int(t["reg_seed"]), 3)
        assert loc["site"] == 8 == int(o["site"]) and loc["target"] == "gpr"
        assert int(o["before"]) == loc["before"]
    assert int(outs["before"][0]) != int(outs["before"][1])   # the two halves of the address
    # a flipped high-half bit sends the load far outside A: the crash symptom (DUE)
    assert int(outs["outcome"][1]) == sassi.SASSI_INJ_DUE
    ik.close()


@pytest.mark.parametrize("name", list(SMALL))
def test_injection_outcome_rules(name):
    ik = sassi.InstrumentedKernel(name, SMALL[name])
    ik.run(sassi.SASSI_IK_NONE)
    torch.cuda.synchronize()
    golden = ik.checksum()
    sites, outs = ik.injection_campaign(k=400, seed=5)
    oc = outs["outcome"]
    assert ((oc >= sassi.SASSI_INJ_MASKED) & (oc <= sassi.SASSI_INJ_HANG)).all()
    # a flipped word stored to the output is always an SDC
    stores = np.isin(outs["site"], list(OUTPUT_STORES[name]))
    assert stores.any() and (oc[stores] == sassi.SASSI_INJ_SDC).all()
    # hangs need data-dependent trip counts (bfs); crashes need a corruptible address or index:
    # bfs indices, vecadd's 64-bit addresses (IMAD.WIDE / IADD.CC carry), stencil's border points
    # reached through a flipped predicate; sgemm has neither
    if name != "bfs":
        assert not (oc == sassi.SASSI_INJ_HANG).any()
    if name == "sgemm":
        assert not (oc == sassi.SASSI_INJ_DUE).any()
    # a flipped predicate or condition code changes control or the address, or nothing (masked)
    pcc = np.isin(outs["target"], [2, 3])
    if pcc.any():
        assert np.isin(oc[pcc], [sassi.SASSI_INJ_MASKED, sassi.SASSI_INJ_SDC, sassi.SASSI_INJ_DUE]).all()
    # the same tuples give the same outcomes, and the outputs are left error-free
    again = ik.inject(sites)
    assert np.array_equal(again, outs)
    assert ik.checksum() == golden
    ik.close()


def test_injection_beyond_the_profile_is_not_reached():
    ik = sassi.InstrumentedKernel("vecadd", 12800)
    ctx = ik.context(sassi.SASSI_H_INSTCOUNT)
    ik.run(sassi.SASSI_H_INSTCOUNT, ctx)
    counts = ctx.sections()["counts"]
    ctx.close()
    st = np.zeros(2, dtype=sassi.INJ_DTYPE)
    st["thread"] = [5, 5]
    st["dyn_index"] = [int(counts[5]), int(counts[5]) - 1]
    outs = ik.inject(st)
    assert outs["outcome"][0] == sassi.SASSI_INJ_NOT_REACHED and outs["site"][0] == 0xFFFFFFFF
    assert outs["outcome"][1] != sassi.SASSI_INJ_NOT_REACHED
    ik.close()


def test_campaign_across_kernels_and_invocations():
    """§8.1 (L627, L629): one campaign over several kernel invocations — vecadd, stencil and two
    invocations of BFS (different graphs) — drawn uniformly over all their eligible dynamic
    instructions (sassi_sample_sites_multi == the oracle's draws over the concatenated profiles);
    each tuple goes to its kernel invocation and hits what the oracle locates in that trace."""
    kernels = [("vecadd", 12800, 20150613, 0, 0), ("stencil", 64, 20150613, 1, 0),
               ("bfs", 4096, 20150613, 2, 0), ("bfs", 4096, 77, 2, 1)]
    iks, ctxs, profiles, oprof, traces = [], [], [], [], []
    for name, size, seed, kid, inv in kernels:
        ik = sassi.InstrumentedKernel(name, size, seed=seed)
        ctx = ik.context(sassi.SASSI_H_INSTCOUNT)
        ik.run(sassi.SASSI_H_INSTCOUNT, ctx)
        profiles.append((ctx, kid, inv))
        oprof.append((ctx.sections()["counts"], kid, inv))
        tctx = ik.context(sassi.SASSI_H_INSTCOUNT)
        traces.append(gen.to_host(ik.trace(tctx)))
        tctx.close()
        iks.append(ik)
        ctxs.append(ctx)
    sites = sassi.sassi_sample_sites_multi(profiles, 400, 2024)
    assert np.array_equal(sites, oracle.sample_multi(oprof, 400, 2024))
    assert len(set(zip(sites["kernel"].tolist(), sites["invocation"].tolist()))) == 4
    # one profile with ids 0 / 0 is sassi_sample_sites
    assert np.array_equal(sassi.sassi_sample_sites_multi([(ctxs[0], 0, 0)], 50, 3), ctxs[0].sample(50, 3))
    for i, (name, size, seed, kid, inv) in enumerate(kernels):
        mine = sites[(sites["kernel"] == kid) & (sites["invocation"] == inv)]
        outs = iks[i].inject(mine)
        h = traces[i]
        for st, o in zip(mine, outs):
            loc = oracle.locate_injection(h["sites"], h["hdr"], h["val"], int(st["thread"]),
                                          int(st["dyn_index"]), int(st["reg_seed"]), int(st["bit_seed"]))
            assert loc is not None and int(o["site"]) == loc["site"] and int(o["bit"]) == loc["bit"]
            assert int(o["target"]) == TARGET_CODE[loc["target"]]
    for c in ctxs:
        c.close()
    for ik in iks:
        ik.close()
