"""The bounds-checked library (libspgemm_b200_checked.so: kernels.cu built with -DSPGEMM_CHECKS, every
SPG_CHECK a device-side bounds check that prints its site and traps) on the small multiplies of
tools/sanitize_cases.py -- every path (in-core two-phase and fused plans, host cut, forced chunking,
the medium / CTA whole and pieced / dense tiers, column panels), each result compared with the
oracle.  This stands in for compute-sanitizer, which is closed on the GPU pool."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
def test_checked_build_all_paths():
    lib = os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200", "libspgemm_b200_checked.so")
    assert os.path.exists(lib), "build the checked library (build.py builds both)"
    env = dict(os.environ, SPGEMM_CHECKED="1")
    code = ("import sys; sys.path.insert(0, %r); "
            "from paper_conf_ipps_xia0ar21_b200 import capi; assert capi.LIB_PATH.endswith('_checked.so'); "
            "import runpy; runpy.run_path(%r, run_name='__main__')") % (ROOT, os.path.join(ROOT, "tools", "sanitize_cases.py"))
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    out = r.stdout + r.stderr
    assert "SPG_CHECK failed" not in out, out[-3000:]
    assert r.returncode == 0, out[-3000:]
    assert "sanitize cases ok" in out
