"""B200-native CapGPU hot path (Ma, Subramaniyan, Wang, ICPP '25).

The method runs in hand-written sm_100a CUDA kernels behind the C ABI of
include/capgpu.h (libcapgpu.so, built in-tree by ``build.py``); ``capgpu.py`` is
a thin ctypes binding with the same names.  There is no CPU fallback.
"""
from .capgpu import CapGPU, CapGPUError, lib, workload_from  # noqa: F401

__all__ = ["CapGPU", "CapGPUError", "lib", "workload_from"]
