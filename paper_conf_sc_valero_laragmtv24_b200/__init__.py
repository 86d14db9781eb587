"""B200-native HPCCG conjugate-gradient hot path (JACC paper, SC'24 workshops).

The product is ``libhpccg.so`` (C ABI in ``include/hpccg.h``; sm_100a kernels in
``csrc/``).  ``hpccg`` is its thin ctypes binding.  There is no CPU fallback.
"""
from . import hpccg  # noqa: F401
from .hpccg import Context, Problem, HpccgError  # noqa: F401

__all__ = ["hpccg", "Context", "Problem", "HpccgError"]
