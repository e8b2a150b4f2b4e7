"""CPU-side checks of the boundary: the C-ABI library loads and exports every symbol that
include/ear_apsp.h declares (no compute calls without a GPU), plus host-only entry points."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ear_apsp.h")


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    names = re.findall(r"^\s*(?!typedef)(?:const\s+)?[a-z_0-9]+\s*\*?\s*([a-z_0-9]+)\s*\(", text, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def L():
    from paper_conf_ipps_duttackb17_b200 import _build, ear_apsp
    _build.build()
    return ear_apsp.lib()


def test_header_declares_the_north_star_entry_points():
    names = declared_functions()
    for n in ["ear_decompose", "apsp_reduced", "expand_ears", "apsp_full"]:
        assert n in names


def test_library_exports_every_declared_symbol(L):
    names = declared_functions()
    assert len(names) >= 15
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing


def test_binding_covers_every_declared_symbol():
    from paper_conf_ipps_duttackb17_b200 import ear_apsp
    assert sorted(ear_apsp.SIGNATURES) == declared_functions()


def test_host_only_calls(L):
    from paper_conf_ipps_duttackb17_b200 import ear_apsp
    assert ear_apsp.version().startswith("earapsp")
    assert L.ear_status_string(-1) == b"EAR_EINVAL"
    # ear_row_block: contiguous, near-equal, covering split
    for rows in [0, 1, 7, 100000]:
        for P in [1, 2, 3, 8]:
            blocks = [ear_apsp.row_block(rows, P, r) for r in range(P)]
            assert blocks[0][0] == 0 and blocks[-1][1] == rows
            assert all(blocks[i][1] == blocks[i + 1][0] for i in range(P - 1))
            sizes = [e - b for b, e in blocks]
            assert max(sizes) - min(sizes) <= 1


def test_bad_arguments_fail_without_a_gpu(L):
    h = ctypes.c_void_p()
    # n < 1 is rejected before any CUDA call
    assert L.ear_decompose(0, 0, None, None, None, 0, None, ctypes.byref(h)) == -1
    assert b"bad sizes" in L.ear_last_error()
    assert L.apsp_full(5, 0, None, None, None, 0, 3, 2, None, 5, None, None) == -1


def test_no_cpu_fallback_when_library_missing(tmp_path, monkeypatch):
    from paper_conf_ipps_duttackb17_b200 import _build, ear_apsp
    monkeypatch.setattr(_build, "LIB", str(tmp_path / "missing.so"))
    monkeypatch.setattr(ear_apsp, "_lib", None)
    with pytest.raises(ear_apsp.EarError):
        ear_apsp.lib()


def test_product_package_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_duttackb17_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src and "apsp_oracle" not in src, f


def test_only_test_infrastructure_uses_the_oracle():
    """oracle/ is test infrastructure: only tests/, bench.py (cpu_baseline / reference arm) and
    __graft_entry__.smoke() may import it -- not the package, tools/ or microbench/."""
    for sub in ("paper_conf_ipps_duttackb17_b200", "tools", "microbench"):
        for dirpath, _, files in os.walk(os.path.join(ROOT, sub)):
            for f in files:
                if f.endswith((".py", ".cu", ".cuh", ".h", ".sh")):
                    src = open(os.path.join(dirpath, f)).read()
                    assert not re.search(r"^\s*(import oracle|from oracle)", src, flags=re.M), os.path.join(dirpath, f)
