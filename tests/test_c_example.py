"""The boundary is a plain C ABI: `examples/sassi_fold.c` (C99, no C++ and no torch) includes the
headers, links libsassi.so and folds record files through the C calls only. CPU: it compiles and
links with -Wall -Wextra -Werror, and sassi_ik.h compiles as C. GPU: its table image and draws on
the hand-worked T0 trace and on c1 equal the oracle's bit for bit."""
import os
import shutil
import subprocess

import numpy as np
import pytest

import oracle
import t0_trace as T0
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CUDA = "/usr/local/cuda"
pytestmark = pytest.mark.skipif(shutil.which("gcc") is None, reason="no gcc")


def build_example(tmp_path):
    exe = str(tmp_path / "sassi_fold")
    libdir = os.path.dirname(sassi.LIB_PATH)
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Wextra", "-Werror",
                           "-I", os.path.join(ROOT, "include"), "-I", os.path.join(CUDA, "include"),
                           os.path.join(ROOT, "examples", "sassi_fold.c"), "-o", exe,
                           "-L", libdir, "-lsassi", "-L", os.path.join(CUDA, "lib64"), "-lcudart",
                           "-Wl,-rpath," + libdir + ":" + os.path.join(CUDA, "lib64")])
    return exe


def test_example_compiles_and_links_as_c99(tmp_path):
    assert os.access(build_example(tmp_path), os.X_OK)
    src = tmp_path / "ik.c"
    src.write_text('#include "sassi_ik.h"\nint main(void) { sassi_ik* k = 0; (void)k; return 0; }\n')
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Wextra", "-Werror", "-fsyntax-only",
                           "-I", os.path.join(ROOT, "include"), str(src)])


def _files(tmp_path, sites, hdr, addr, val):
    paths = []
    for name, a in (("sites", sites), ("hdr", hdr), ("addr", addr), ("val", val)):
        p = tmp_path / (name + ".bin")
        np.ascontiguousarray(a).tofile(p)
        paths.append(str(p))
    return paths


@pytest.mark.gpu
@pytest.mark.parametrize("case", ["t0", "c1"])
def test_example_run_equals_oracle(tmp_path, case):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    exe = build_example(tmp_path)
    if case == "t0":
        sites, (hdr, addr, val), W, mask = T0.sites(), T0.records(), T0.N_WARPS, sassi.SASSI_H_EVERY
    else:
        P, lim, mask, _ = gen.preset("c1")
        h = gen.generate_host(P, lim)
        sites, hdr, addr, val, W = h["sites"], h["hdr"], h["addr"], h["val"], P.total_warps
    files = _files(tmp_path, sites, hdr, np.asarray(addr, np.uint64), np.asarray(val, np.uint32))
    out, draws = str(tmp_path / "table.bin"), str(tmp_path / "draws.bin")
    r = subprocess.run([exe] + files + [str(W), str(mask), out, "100", "7", draws],
                       capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    t = np.fromfile(out, dtype=np.uint64)
    o = oracle.run(sites, W, mask, hdr, addr, val)
    assert np.array_equal(t, o)
    d = np.fromfile(draws, dtype=sassi.INJ_DTYPE)
    so = oracle.sections(o, len(sites), W)
    assert np.array_equal(d, oracle.sample(so["counts"], 100, 7))
