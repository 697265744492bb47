"""B200-native hot path of APT (Adaptive Parallel Training for GNNs, PPoPP'25).

The product is the sm_100a C-ABI library ``libapt.so`` (include/apt.h); ``apt``
is its thin ctypes binding.  There is no CPU fallback: importing ``apt`` and
calling into it raises if the library was not built.
"""
from . import apt  # noqa: F401
