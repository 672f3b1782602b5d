"""The debug library (libphoton_debug.so: PHOTON_DEBUG=1, device-side bounds checks that print their site and
trap) under the GPU parity tests that exercise the kernels' computed addresses -- K1 cell / stage / warp-index
bounds on long, empty, ragged and tiny warps and on B above and below 4096, the match's bucket and candidate
segments, the type lists -- each still compared element by element with the CPU oracle.  compute-sanitizer is
disabled on the GPU pool (tests/test_sanitizer.py skips there); this is the check that runs instead."""
import os
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SUBSET = ("random_small or k1_fused or empty_warps or config_small or capacity_retry or match_many or "
          "k1_long_warps or chain_cuda_graph or out_reuse or group_full or stable_c6 or stable_degenerate or "
          "config_full")


def test_parity_subset_under_debug_library():
    from paper_conf_micro_liusc23_b200 import build as b
    so = b.build(debug=True)  # no-op when the prebuilt library is current
    env = dict(os.environ, PHOTON_LIB_OVERRIDE=so)
    cmd = [sys.executable, "-m", "pytest", "-q", "-m", "gpu and not slow", "-p", "no:cacheprovider",
           os.path.join(ROOT, "tests", "test_parity_gpu.py"), os.path.join(ROOT, "tests", "test_parity_gpu2.py"),
           "-k", SUBSET]
    p = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT, env=env)
    out = p.stdout + p.stderr
    assert "PHOTON_DCHECK failed" not in out, out[-4000:]
    assert p.returncode == 0, out[-4000:]
    import re
    m = re.search(r"(\d+) passed", out)
    assert m and int(m.group(1)) >= 40 and " failed" not in out, out[-4000:]  # the subset really ran


def test_debug_library_is_the_one_loaded():
    from paper_conf_micro_liusc23_b200 import build as b
    so = b.build(debug=True)
    code = ("import paper_conf_micro_liusc23_b200._lib as L; L.load(); import sys; "
            "print(open('/proc/self/maps').read().count('libphoton_debug.so') > 0)")
    p = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, cwd=ROOT,
                       env=dict(os.environ, PHOTON_LIB_OVERRIDE=so), timeout=300)
    assert p.stdout.strip().endswith("True"), p.stdout + p.stderr
