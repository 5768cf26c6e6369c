"""Host-side checks of the C-ABI boundary (no GPU needed): the library loads and exports every
function include/gsw.h declares, and the binding declares exactly those."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "gsw.h")


def _declared():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(gsw_[a-z_0-9]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ppopp_menglts19_b200 import _lib
    if not os.path.exists(_lib.LIB_PATH):
        subprocess.check_call(["make", "-C", ROOT, "-j8", "all"])
    return ctypes.CDLL(_lib.LIB_PATH)


def test_header_declares_north_star_api():
    names = _declared()
    for must in ["gsw_graph_create", "gsw_bfs", "gsw_sssp", "gsw_cc", "gsw_pr", "gsw_dpr", "gsw_bc", "gsw_force_config"]:
        assert must in names


def test_library_exports_every_declared_symbol(lib):
    for name in _declared():
        assert hasattr(lib, name), name


def test_binding_matches_header(lib):
    from paper_conf_ppopp_menglts19_b200 import _lib
    assert sorted(_lib.SIGNATURES) == _declared()


def test_host_only_calls(lib):
    """Calls that need no device: version string, workspace sizing, argument validation."""
    from paper_conf_ppopp_menglts19_b200 import _lib
    L = _lib.load()
    assert b"sm_100a" in L.gsw_version()
    sz = ctypes.c_size_t()
    assert L.gsw_workspace_size(1000, 5000, 0, 0, ctypes.byref(sz)) == _lib.GSW_OK
    assert sz.value > 1000 * 4 + 5000 * 4
    assert L.gsw_workspace_size(0, 5, 0, 0, ctypes.byref(sz)) == _lib.GSW_EINVAL
    assert L.gsw_workspace_size(10, 1 << 32, 0, 0, ctypes.byref(sz)) == _lib.GSW_EOVERFLOW
    assert L.gsw_bfs(None, 0, None, None) == _lib.GSW_EINVAL
    assert b"null" in L.gsw_last_error()
    cfg = _lib.gsw_config(7, 0, 0, 0, 0, 0)
    assert L.gsw_force_config(None, ctypes.byref(cfg)) == _lib.GSW_EINVAL


def test_sass_is_sm100a():
    from paper_conf_ppopp_menglts19_b200 import _lib
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ppopp_menglts19_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", txt), f
