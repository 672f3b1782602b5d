"""photon-b200: the data-parallel online-analysis hot path of Photon (MICRO '23) on B200 (sm_100a).

C ABI: include/photon.h (libphoton.so, built in-tree).  Python binding: `Photon` (api.py), same call names.
Multi-GPU driver: dist.py (torch.distributed over NCCL).
"""
from ._lib import PhotonError, PhotonUnavailable, load  # noqa: F401
from .api import DeviceTiming, DeviceTrace, Photon, to_device, to_numpy  # noqa: F401

__all__ = ["Photon", "DeviceTrace", "DeviceTiming", "PhotonError", "PhotonUnavailable", "to_device", "to_numpy",
           "load"]
