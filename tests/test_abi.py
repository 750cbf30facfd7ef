"""CPU-side checks of the C-ABI library (no compute calls need a GPU here)."""
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "ap.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ap_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    import ctypes
    import paper_conf_cluster_liulldgl22_b200 as ap
    lib = ctypes.CDLL(ap.LIB_PATH)
    decl = _declared()
    assert "ap_search_exhaustive" in decl and len(decl) >= 12
    for name in decl:
        assert hasattr(lib, name), name
    assert sorted(ap.EXPORTS) == decl


def test_no_gpu_fails_loudly():
    """With no device the product path errors (AP_ERR_CUDA); it never falls back."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_cluster_liulldgl22_b200 as ap
    with pytest.raises(ap.APError) as ei:
        ap.ap_plan_create([1, 2], [3, 4], [1, 0], 10**9)
    assert ei.value.status == 3


def test_host_only_calls():
    import paper_conf_cluster_liulldgl22_b200 as ap
    assert ap.ap_count(10, 4) == 84
    assert ap.ap_count(66, 8) == 696190560
    assert ap.ap_count(98, 16) == 154744841157936784
    with pytest.raises(ap.APError):
        ap.ap_count(5, 6)
    with pytest.raises(ap.APError) as ei:
        ap.ap_count(200, 60)
    assert ei.value.status == 2
    assert "sm_100a" in ap.ap_version()


def test_product_package_does_not_import_oracle():
    """The product path never routes through the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_cluster_liulldgl22_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", txt).lower().replace("oracle/", ""), f


def test_sass_has_no_fallback_and_uses_tma():
    """cuobjdump of the built library: sm_100a code, TMA bulk copy (UBLKCP) in the
    prologue, integer max-plus (VIMNMX / VIADD) in the sweep."""
    import shutil
    import subprocess
    import paper_conf_cluster_liulldgl22_b200 as ap
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("no cuobjdump")
    out = subprocess.run([exe, "-sass", ap.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "UBLKCP" in out
    assert "VIMNMX" in out
