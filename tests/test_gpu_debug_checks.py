"""Device-side bounds checks in place of compute-sanitizer (SURVEY §4 layer 5).

The GPU pool refuses compute-sanitizer (tests/test_gpu_sanitizer.py skips there), so this
test builds libap.so with -DAP_DEBUG_CHECKS=1 (ap_device.cuh: AP_CHECK prints and traps)
and runs tools/sanitize_run.py -- every kernel family, C1/C2 plus the p = 16, saturating,
memory and two-phase paths -- against it.  A failed check traps the kernel, the CUDA
error fails the call and the script, and this test.  Checked: candidate cut vectors in
the sweep, child indices and Algorithm-1 prefix rows of the heuristic pool, its job
rings and slot ids, best-cut output rows, and the critical-path walk's stage and column
word indices (ap_master.cuh).
"""
import os
import subprocess
import sys
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
def test_debug_checks_build_runs_every_kernel_family_clean():
    with tempfile.TemporaryDirectory() as td:
        lib = os.path.join(td, "libap_debug.so")
        env = dict(os.environ, AP_LIB_OUT=lib, AP_SPLIT_COMPILE="0", AP_OBJ_TAG=".dbg",
                   AP_NVCC_EXTRA="-DAP_DEBUG_CHECKS=1")
        b = subprocess.run([sys.executable, os.path.join(ROOT, "paper_conf_cluster_liulldgl22_b200",
                                                         "_build.py"), "--force"],
                           capture_output=True, text=True, timeout=1200, cwd=ROOT, env=env)
        assert b.returncode == 0 and os.path.exists(lib), (b.stdout + b.stderr)[-3000:]
        env = dict(os.environ, AP_LIB_PATH=lib)
        r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "sanitize_run.py")],
                           capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
        out = r.stdout + r.stderr
        assert "AP_CHECK failed" not in out, out[-3000:]
        assert r.returncode == 0 and "sanitize run ok" in out, out[-3000:]
