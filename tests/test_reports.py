"""The product's report module (paper_conf_isca_stephensonhlejn15_b200/reports.py) against the
oracle's independent report formulas and the paper's worked example, on oracle-built tables."""
import os

import numpy as np
import pytest

import oracle
from oracle import reports as oreports
import t0_trace as T0
from test_oracle import random_trace
from paper_conf_isca_stephensonhlejn15_b200 import reports, sassi

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _tables():
    s = T0.sites()
    hdr, addr, val = T0.records()
    yield s, T0.N_WARPS, oracle.run(s, T0.N_WARPS, 31, hdr, addr, val, pcs=[1, 2])
    for seed in (11, 12, 13):
        s, W, hdr, addr, val = random_trace(seed, n=800)
        yield s, W, oracle.run(s, W, 31, hdr, addr, val, pcs=[1, 7])


@pytest.mark.parametrize("k", range(4))
def test_reports_match_oracle_formulas(k):
    s, W, t = list(_tables())[k]
    sec = oracle.sections(t, len(s), W)
    assert reports.branch_table1(t, s, W) == pytest.approx(oreports.table1_percent(sec["br"]))
    assert np.allclose(reports.memdiv_pmf(sec["h32"]), oreports.fig7_pmf(sec["h32"]))
    assert reports.value_dump(t, s, W) == dict(oreports.value_profile_lines(t, s, W))
    assert reports.value_table2(t, s, W) == pytest.approx(oreports.table2_percent(t, s, W))
    assert [(a, b) for a, b, _ in reports.instruction_mix(t, len(s), W)] == \
        [(a, b) for a, b, _ in oreports.instmix_report(t, len(s), W)]
    hm = reports.memdiv_heatmap(sec["h32"])
    assert hm.sum() == pytest.approx(1.0) and np.allclose(hm * sec["h32"].sum(), sec["h32"])
    prof = reports.branch_profile(t, s, W)
    assert [r[1] for r in prof] == sorted((r[1] for r in prof), reverse=True)
    assert sum(r[1] for r in prof) == int(sec["br"][:, 0].sum())


def test_value_dump_reproduces_the_paper_example():
    """§7.2 (L601-L609): R12 with 18 toggling low bits, R13 always 1 and scalar."""
    golden = [l.rstrip("\n") for l in open(os.path.join(GOLDEN, "value_profile_L601_L609.txt"))
              if not l.startswith("#") and l.strip()]
    s = np.zeros(1, dtype=oracle.SITE_DTYPE)
    s[0]["pc"], s[0]["flags"], s[0]["n_gpr_dst"] = 0x40, oracle.F_MEM | oracle.F_MEM_READ, 2
    s[0]["domain"], s[0]["reg_num"] = oracle.D_GLOBAL, [12, 13, 0, 0]
    rng = np.random.default_rng(3)
    H, A, V = [], [], []
    for _ in range(64):
        H.append((0x40, 0, 0xFFFFFFFF, 0xFFFFFFFF))
        A.append(np.arange(32, dtype=np.uint64) * 8 + 0x10000)
        V.append(rng.integers(0, 2**18, 32).astype(np.uint32))
        V.append(np.ones(32, np.uint32))
    hdr = np.array(H, np.uint32).view(oracle.HDR_DTYPE).reshape(-1)
    t = oracle.run(s, 1, oracle.H_VALUE, hdr, np.array(A).reshape(-1, 32), np.array(V).reshape(-1, 32))
    assert reports.value_dump(t, s, 1)[0x40] == golden


def test_injection_outcome_percentages():
    o = np.zeros(8, dtype=sassi.OUTCOME_DTYPE)
    o["outcome"] = [0, 0, 0, 1, 1, 2, 3, 0]
    r = reports.injection_outcomes(o)
    assert r == {"masked": 50.0, "sdc": 25.0, "due": 12.5, "hang": 12.5, "not_reached": 0.0}
