"""Error injection on the instrumented kernels (§8.1):
profile -> draw sites -> one injection run per site. The injected instruction, register value and
bit of every run equal what the oracle locates in the same kernel's trace (the dyn-th eligible,
not-predicated-out dynamic instruction of the thread, reading R23); outcomes follow their rules."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

SMALL = {"vecadd": 12800, "bfs": 4096, "sgemm": 64, "stencil": 64}
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
        assert int(o["target"]) == {"gpr": 0, "mem": 1}[loc["target"]]
        if loc["target"] == "gpr":
            assert int(o["before"]) == loc["before"]
        assert int(o["after"]) == int(o["before"]) ^ (1 << int(o["bit"]))
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
    # only the kernel with data-dependent indices and trip counts shows crash / hang symptoms
    if name != "bfs":
        assert not np.isin(oc, [sassi.SASSI_INJ_DUE, sassi.SASSI_INJ_HANG]).any()
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
