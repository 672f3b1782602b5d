"""ctypes declarations of libphoton's C ABI (include/photon.h).  Argument marshalling only.

Loading fails loudly (PhotonUnavailable) when the in-tree libphoton.so is missing: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os
from ctypes import POINTER, c_double, c_int, c_int64, c_size_t, c_uint8, c_uint32, c_uint64, c_void_p, c_char_p

HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("PHOTON_LIB_OVERRIDE") or os.path.join(HERE, "libphoton.so")  # override: profiling builds

OK, EINVAL, ECUDA, ERANGE, ECAPACITY, EWORKSPACE = 0, -1, -2, -3, -4, -5
STATUS = {0: "OK", -1: "EINVAL", -2: "ECUDA", -3: "ERANGE", -4: "ECAPACITY", -5: "EWORKSPACE"}


class PhotonUnavailable(RuntimeError):
    pass


class PhotonError(RuntimeError):
    def __init__(self, code: int, msg: str = "", index: int = -1):
        super().__init__(f"photon {STATUS.get(code, code)} ({code}){': ' + msg if msg else ''}"
                         f"{f' [index {index}]' if index >= 0 else ''}")
        self.code = code
        self.index = index


class Trace(ctypes.Structure):
    _fields_ = [("n_kernels", c_uint32), ("n_bb", c_uint32), ("n_warps", c_uint64), ("n_events", c_uint64),
                ("kernel_warp_off", c_void_p), ("warp_event_off", c_void_p), ("bb", c_void_p),
                ("bb_len", c_void_p), ("bb_bin", c_void_p)]


class Types(ctypes.Structure):
    _fields_ = [("capacity", c_uint64), ("warp_type", c_void_p), ("kernel_type_off", c_void_p),
                ("type_key", c_void_p), ("type_count", c_void_p), ("type_first_warp", c_void_p),
                ("warp_sampling_ok", c_void_p)]


class MatchParams(ctypes.Structure):
    _fields_ = [("theta_num", c_uint32), ("theta_den", c_uint32), ("n_cores", c_uint64),
                ("pool_all_prior", c_uint32)]


class Timing(ctypes.Structure):
    _fields_ = [("n_kernels", c_uint32), ("n_bb", c_uint32), ("n_records", c_uint64), ("kernel_rec_off", c_void_p),
                ("bb", c_void_p), ("issue", c_void_p), ("retire", c_void_p)]


class StableParams(ctypes.Structure):
    _fields_ = [("window_n", c_uint32), ("delta_num", c_uint32), ("delta_den", c_uint32), ("rate_num", c_uint32),
                ("rate_den", c_uint32)]


class WarpStableParams(ctypes.Structure):
    _fields_ = [("window_n", c_uint32), ("delta_num", c_uint32), ("delta_den", c_uint32)]


TYPE_ROW_BYTES = 88  # photon_type_row
ROW_PAD = 0xFFFFFFFF  # PHOTON_ROW_PAD: kernel id of a padding row
PAIR_PAD = 0xFFFFFFFFFFFFFFFF  # PHOTON_PAIR_PAD: an unused pair slot
PROF_SECTIONS = ["bbv_fused", "bbv", "kbb", "group_unfused", "canon", "sig", "scan", "resolve", "stable", "prep"]

# (name, restype, argtypes) — mirrors include/photon.h
_SIGS = [
    ("photon_abi_version", c_int, []),
    ("photon_create", c_int, [POINTER(c_void_p), c_int]),
    ("photon_destroy", None, [c_void_p]),
    ("photon_last_error", c_char_p, [c_void_p]),
    ("photon_check", c_int, [c_void_p, c_void_p, POINTER(c_int64)]),
    ("photon_ws_status", c_int, [c_void_p, c_void_p, c_void_p, POINTER(c_int64)]),
    ("photon_profile", c_int, [c_void_p, c_int]),
    ("photon_profile_read", c_int, [c_void_p, c_void_p, POINTER(c_double), POINTER(c_uint64)]),
    ("photon_launch_count", c_uint64, []),
    ("photon_bbv_workspace_bytes", c_size_t, [POINTER(Trace)]),
    ("photon_bbv_build", c_int, [c_void_p, POINTER(Trace), c_void_p, c_size_t, c_void_p, c_void_p, c_void_p, c_void_p]),
    ("photon_group_workspace_bytes", c_size_t, [POINTER(Trace), c_uint64]),
    ("photon_warp_group", c_int, [c_void_p, POINTER(Trace), c_void_p, c_void_p, c_size_t, POINTER(Types), c_void_p]),
    ("photon_warp_group2", c_int, [c_void_p, POINTER(Trace), c_void_p, c_void_p, c_size_t, POINTER(Types), c_void_p,
                                   c_void_p]),
    ("photon_analyse", c_int, [c_void_p, POINTER(Trace), c_void_p, c_size_t, POINTER(Types), c_void_p, MatchParams,
                               c_void_p, c_size_t, c_void_p, c_void_p, c_void_p]),
    ("photon_types_total", c_int, [c_void_p, POINTER(Types), c_uint32, POINTER(c_uint64), c_void_p]),
    ("photon_match_workspace_bytes", c_size_t, [c_uint32, c_uint64, c_uint64]),
    ("photon_kernel_match", c_int, [c_void_p, c_uint32, POINTER(Types), c_void_p, MatchParams, c_void_p, c_size_t,
                                    c_void_p, c_void_p, c_void_p]),
    ("photon_match_stats", c_int, [c_void_p, c_uint32, c_uint64, c_void_p, c_size_t, POINTER(c_uint64), c_void_p]),
    ("photon_sig_build", c_int, [c_void_p, c_uint32, c_void_p, c_void_p, c_void_p, c_uint32, c_uint32, c_void_p,
                                 c_void_p, c_void_p, c_size_t, c_void_p]),
    ("photon_match_scan", c_int, [c_void_p, c_uint32, c_void_p, c_void_p, c_void_p, c_void_p, MatchParams, c_uint32,
                                  c_uint32, c_void_p, c_size_t, c_void_p, c_uint64, c_void_p, c_void_p]),
    ("photon_match_resolve", c_int, [c_void_p, c_uint32, c_void_p, c_void_p, c_void_p, c_void_p, MatchParams,
                                     c_void_p, c_uint64, c_void_p, c_size_t, c_void_p, c_void_p, c_void_p]),
    ("photon_stable_workspace_bytes", c_size_t, [POINTER(Timing)]),
    ("photon_bb_stable", c_int, [c_void_p, POINTER(Timing), c_void_p, StableParams, c_void_p, c_size_t, c_void_p,
                                 c_void_p, c_void_p, c_void_p]),
    ("photon_warp_stable_workspace_bytes", c_size_t, [POINTER(Timing)]),
    ("photon_warp_stable", c_int, [c_void_p, POINTER(Timing), c_void_p, WarpStableParams, c_void_p, c_size_t,
                                   c_void_p, c_void_p, c_void_p]),
    ("photon_kernel_predict", c_int, [c_void_p, c_uint32, c_void_p, c_void_p, c_void_p, c_void_p, c_void_p,
                                      c_size_t, c_void_p, c_void_p, c_void_p]),
    ("photon_bb_predict_workspace_bytes", c_size_t, [POINTER(Trace)]),
    ("photon_bb_predict", c_int, [c_void_p, POINTER(Trace), c_void_p, c_void_p, c_void_p, c_size_t, c_void_p,
                                  c_void_p, c_void_p]),
    ("photon_group_full_workspace_bytes", c_size_t, [POINTER(Trace), c_uint64]),
    ("photon_warp_group_full", c_int, [c_void_p, POINTER(Trace), c_void_p, c_void_p, c_size_t, POINTER(Types),
                                       c_void_p]),
    ("photon_ingest_workspace_bytes", c_size_t, [c_uint64, c_uint64]),
    ("photon_ingest_tagged", c_int, [c_void_p, c_uint64, c_uint64, c_void_p, c_void_p, c_void_p, c_size_t,
                                     c_void_p, c_void_p, c_void_p]),
    ("photon_pool_export_workspace_bytes", c_size_t, [c_uint32]),
    ("photon_pool_export", c_int, [c_void_p, c_uint32, POINTER(Types), c_void_p, c_void_p, c_void_p, c_size_t,
                                   POINTER(Types), c_void_p, c_void_p, c_void_p, c_void_p]),
    ("photon_pool_match_workspace_bytes", c_size_t, [c_uint32, c_uint64, c_uint32, c_uint64, c_uint64]),
    ("photon_kernel_match_pooled", c_int, [c_void_p, c_uint32, POINTER(Types), c_void_p, c_uint64, c_uint32,
                                           POINTER(Types), c_void_p, c_uint64, MatchParams, c_void_p, c_size_t,
                                           c_void_p, c_void_p, c_void_p]),
    ("photon_types_export", c_int, [c_void_p, c_uint32, POINTER(Types), c_uint32, c_uint64, c_void_p, c_uint64,
                                    c_void_p, c_void_p]),
    ("photon_merge_workspace_bytes", c_size_t, [c_uint64, c_uint32]),
    ("photon_types_merge", c_int, [c_void_p, c_void_p, c_uint64, c_uint32, c_void_p, c_void_p, c_size_t,
                                   POINTER(Types), c_void_p]),
    ("photon_types_remap", c_int, [c_void_p, c_uint32, c_uint64, c_void_p, POINTER(Types), c_uint32, c_uint64,
                                   c_uint32, c_void_p, c_size_t, c_void_p, c_void_p]),
]

EXPORTED = [n for n, _, _ in _SIGS]

_lib = None


def load(path: str = SO_PATH):
    """Loads libphoton.so (built in-tree by build.py / __graft_entry__.build()).  Raises if missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise PhotonUnavailable(f"{path} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(path)
    for name, res, args in _SIGS:
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L
