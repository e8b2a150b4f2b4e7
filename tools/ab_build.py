"""Build a variant of libearapsp.so with one csrc file replaced (A/B timing on one box via EAR_LIB).

    python tools/ab_build.py NAME csrc_file_variant.cu [replaced_file.cu]

Objects of the other sources are reused from the in-tree build (paper_conf_ipps_duttackb17_b200/build);
the result is paper_conf_ipps_duttackb17_b200/libearapsp_NAME.so.
"""
import os
import shutil
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_duttackb17_b200 import _build  # noqa: E402

name, variant = sys.argv[1], os.path.abspath(sys.argv[2])
replaced = sys.argv[3] if len(sys.argv) > 3 else os.path.basename(variant)
_build.build()
tmpdir = os.path.join("/tmp", f"ab_{name}")
os.makedirs(tmpdir, exist_ok=True)
src = os.path.join(tmpdir, replaced)
shutil.copy(variant, src)
for h in os.listdir(_build.CSRC):
    if h.endswith(".cuh"):
        shutil.copy(os.path.join(_build.CSRC, h), tmpdir)
obj = os.path.join(tmpdir, replaced[:-3] + ".o")
subprocess.check_call(["nvcc", "-gencode", _build.GENCODE, "-O3", "-lineinfo", "-std=c++17", "-c", "-Xcompiler", "-fPIC",
                       "-I", os.path.join(_build.ROOT, "include"), src, "-o", obj])
objs = [obj if os.path.basename(s) == replaced else _build._obj(s) for s in _build.sources()]
out = os.path.join(_build.HERE, f"libearapsp_{name}.so")
subprocess.check_call(["nvcc", "-gencode", _build.GENCODE, "-shared", "-Xcompiler", "-fPIC", *objs, "-o", out])
print(out)
