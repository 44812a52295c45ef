"""Maximum sizes of the site table (SASSI_MAX_SITES = 4096): with branch / instcount / instmix
handlers every site fits (the per-warp private counters fall back to one shared set) and the fold
equals the oracle on a trace touching all of them; 4096 sites with four value destinations each
need more shared memory than an SM has, which attach reports as ENOSPC instead of failing later;
one site more than the maximum is ENOSPC at create."""
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


@pytest.mark.parametrize("mask", [sassi.SASSI_H_BRANCH | sassi.SASSI_H_INSTCOUNT | sassi.SASSI_H_INSTMIX])
def test_max_sites_header_handlers(mask):
    n_sites, W, n = 4096, 64, 200_000
    half = n_sites // 2
    s = np.concatenate([_sites(half, oracle.F_COND_BRANCH | oracle.F_CTRL),
                        _sites(half, oracle.F_NUMERIC | oracle.F_WRITES_PRED)])
    s["pc"] = 0x1000 + 16 * np.arange(n_sites)
    rng = np.random.default_rng(4096)
    H = np.stack([s["pc"][rng.integers(0, n_sites, n)], rng.integers(0, W, n).astype(np.uint32),
                  rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32),
                  rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)], 1).astype(np.uint32)
    hdr = np.ascontiguousarray(H).view(oracle.HDR_DTYPE).reshape(-1)
    ctx = sassi.Context(s, W, mask)
    ctx.consume(to_device(s, hdr, None, None))
    t = ctx.read_tables()
    ctx.close()
    assert diff_tables(t, oracle.run(s, W, mask, hdr), n_sites, W) is None


def test_value_state_beyond_shared_memory_is_enospc():
    s = _sites(4096, oracle.F_NUMERIC, ndst=4)
    with pytest.raises(sassi.SassiError) as e:
        sassi.Context(s, 8, sassi.SASSI_H_VALUE)
    assert e.value.status == sassi.SASSI_ENOSPC


def test_one_site_too_many_is_enospc():
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, _sites(4097, oracle.F_NUMERIC), 8)
    assert e.value.status == sassi.SASSI_ENOSPC
