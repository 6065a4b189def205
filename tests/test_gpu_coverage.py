"""Debug coverage-counter build: every C element is stored by exactly one tile,
nothing outside the matrices is stored.  Runs tests/tools/coverage_check.py in a subprocess with the
-DVB_COVERAGE library (libvbgemm_cov.so, built by __graft_entry__.build())."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_every_c_element_written_exactly_once():
    sys.path.insert(0, os.path.join(ROOT, "paper_conf_ppopp_li0yjl19_b200"))
    import build as vbbuild
    lib = vbbuild.build_coverage()
    env = dict(os.environ, VB_LIB=lib)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "tools", "coverage_check.py")], env=env, cwd=ROOT,
                         capture_output=True, text=True, timeout=900)
    rows = [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]
    assert out.returncode == 0, out.stdout[-3000:] + out.stderr[-3000:]
    assert len(rows) == 10 and all(r["wrong_counts"] == 0 and r["max_count"] == 1 for r in rows), rows


def test_product_build_rejects_coverage():
    import paper_conf_ppopp_li0yjl19_b200 as vb
    from paper_conf_ppopp_li0yjl19_b200 import _native as nv
    if "libvbgemm_cov" in nv.LIB_PATH:
        pytest.skip("running against the coverage build")
    with pytest.raises(vb.VbError):
        nv.debug_set_coverage(0, 0, 0, 0)
