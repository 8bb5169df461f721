"""B200-native just-in-time checkpoint capture / restore (Gupta et al., EuroSys '24).

The product is libjitc.so (C ABI in include/jitc.h: CUDA sm_100a kernels +
NCCL); `jitc` is its thin ctypes binding.  There is no CPU fallback.
"""
from . import jitc  # noqa: F401
from .jitc import Context, JitcError  # noqa: F401

__all__ = ["jitc", "Context", "JitcError"]
