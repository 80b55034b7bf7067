"""B200-native Harmony-DP training step (Li et al., HotOS '21) behind a C ABI.

The product is libharmony.so (csrc/, built for sm_100a by `build.py`); `harmony` is its
ctypes binding.  See include/harmony.h and DESIGN.md.
"""
from . import harmony  # noqa: F401
