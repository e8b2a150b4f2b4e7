"""Build libearapsp.so in-tree with nvcc for sm_100a (called by __graft_entry__.build()).

Every csrc/*.cu is compiled to its own object in parallel (build/), then linked into the shared
library; an object is rebuilt when its source, a csrc header or include/ear_apsp.h is newer.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libearapsp.so")
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "build")
GENCODE = "arch=compute_100a,code=sm_100a"


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _headers():
    return glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "ear_apsp.h")]


def _obj(src: str) -> str:
    return os.path.join(OBJ, os.path.basename(src)[:-3] + ".o")


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def needs_build() -> bool:
    return _stale(LIB, sources() + _headers())


def _compile(src: str, verbose: bool) -> tuple[str, int, str]:
    out = _obj(src)
    tmp = out + f".tmp{os.getpid()}"
    cmd = ["nvcc", "-gencode", GENCODE, "-O3", "-lineinfo", "-std=c++17", "-c", "-Xcompiler", "-fPIC",
           "-Xptxas", "-v" if verbose else "-O3", "-I", os.path.join(ROOT, "include"), src, "-o", tmp]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode == 0:
        os.replace(tmp, out)
    return src, res.returncode, res.stdout + res.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    hdr = _headers()
    todo = [s for s in sources() if force or _stale(_obj(s), [s] + hdr)]
    with ThreadPoolExecutor(max_workers=max(1, min(len(todo), os.cpu_count() or 4))) as ex:
        results = list(ex.map(lambda s: _compile(s, verbose), todo))
    failed = [r for r in results if r[1] != 0]
    for src, rc, log in results:
        if rc != 0 or verbose:
            sys.stderr.write(f"--- {os.path.basename(src)}\n{log}")
    if failed:
        raise RuntimeError("nvcc failed: " + ", ".join(os.path.basename(r[0]) for r in failed))
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = ["nvcc", "-gencode", GENCODE, "-shared", "-Xcompiler", "-fPIC", *[_obj(s) for s in sources()], "-o", tmp]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed linking libearapsp.so")
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="-f" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
