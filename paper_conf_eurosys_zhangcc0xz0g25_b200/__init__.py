"""B200-native BLESS hot path (Zhang et al., EuroSys '25).

Native library (``lib/libbless.so``, built by ``build.py``): C++ scheduler,
engine and the sm_100a tenant kernels behind the C ABI in
``include/bless/bless.h``.  ``capi`` is the ctypes binding (same names);
``models`` builds the configs' tenant kernel sequences with PyTorch-owned
device memory.
"""
from . import capi  # noqa: F401

__all__ = ["capi"]
