"""The C-ABI library: builds for sm_100a, loads without a GPU, exports exactly what include/photon.h declares,
and fails loudly (no CPU fallback) when no device is present.  CPU only (no compute calls)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "photon.h")


def declared():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"PHOTON_API\s+[\w\s\*]*?\b(photon_\w+)\s*\(", src)))


def test_header_declarations_are_bound_and_exported():
    from paper_conf_micro_liusc23_b200 import _lib
    names = declared()
    assert len(names) >= 20
    L = _lib.load()
    for n in names:
        assert hasattr(L, n), n
    assert sorted(_lib.EXPORTED) == names  # the binding mirrors the header exactly
    nm = subprocess.run(["nm", "-D", "--defined-only", _lib.SO_PATH], capture_output=True, text=True).stdout
    exported = sorted(set(re.findall(r"\b(photon_\w+)$", nm, re.M)))
    assert exported == names  # and the library exports nothing else under the prefix


def test_sass_is_sm100a_and_uses_bulk_copy():
    from paper_conf_micro_liusc23_b200 import _lib
    out = subprocess.run(["cuobjdump", "-lelf", _lib.SO_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", _lib.SO_PATH], capture_output=True, text=True).stdout
    assert "UBLKCP" in sass  # cp.async.bulk (TMA copy engine) in the streaming kernel


def test_abi_version_and_no_gpu_behaviour():
    import torch
    from paper_conf_micro_liusc23_b200 import Photon, PhotonUnavailable, _lib
    L = _lib.load()
    assert L.photon_abi_version() == 1
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    ctx = ctypes.c_void_p()
    assert L.photon_create(ctypes.byref(ctx), 0) == _lib.ECUDA
    with pytest.raises(PhotonUnavailable):
        Photon(0)


def test_host_argument_validation_without_gpu():
    # host-detectable errors return EINVAL before touching the device (NULL ctx / NULL trace)
    from paper_conf_micro_liusc23_b200 import _lib
    L = _lib.load()
    assert L.photon_bbv_build(None, None, None, 0, None, None, None, None) == _lib.EINVAL
    assert L.photon_check(None, None, None) == _lib.EINVAL
