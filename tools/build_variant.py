"""Build a variant of libsassi.so with extra nvcc defines, for A/B timing on one GPU call:
    python tools/build_variant.py NAME -DFOO=1 ...   ->  <pkg>/lib/variants/NAME/libsassi.so
    SASSI_LIB=paper_conf_isca_stephensonhlejn15_b200/lib/variants/NAME/libsassi.so python tools/time_masks.py c2 15,2"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_stephensonhlejn15_b200 import _build as B  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
csrc, inc = B.CSRC, B.INCLUDE
if defs and defs[0].startswith("--src="):   # build another source tree (e.g. a git-archived commit)
    csrc, defs = defs[0][6:], defs[1:]
if defs and defs[0].startswith("--inc="):   # ... with its own include/ (sassi.h of that commit)
    inc, defs = defs[0][6:], defs[1:]
out = os.path.join(B.ROOT, "build", "variants", name)
os.makedirs(out, exist_ok=True)
srcs = sorted(f for f in os.listdir(csrc) if f.endswith(".cu"))
objs = []
procs = []
for f in srcs:
    o = os.path.join(out, f + ".o")
    objs.append(o)
    procs.append(subprocess.Popen([B.NVCC] + B.NVFLAGS + defs + ["-I", inc, "-I", csrc, "-c",
                                                                  "-o", o, os.path.join(csrc, f)]))
assert all(p.wait() == 0 for p in procs)
lib = os.path.join(B.LIB, "variants", name)
os.makedirs(lib, exist_ok=True)
subprocess.check_call([B.NVCC] + B.ARCH + ["-shared", "-o", os.path.join(lib, "libsassi.so")] + objs +
                      ["-ldl", "-lpthread"])
print(os.path.join(lib, "libsassi.so"))
