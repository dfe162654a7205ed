"""B200-native Hilbert-sorted BVH Barnes-Hut step (Cassell et al., SC'24).

The product is the C-ABI library libnbody_b200.so (include/nbody.h, sources
in csrc/); this package is its thin Python binding.  Importing the package
does not touch the GPU; creating an ``NBody`` loads the library and fails
loudly if it is missing.
"""
from .nbody import NBody  # noqa: F401
from ._capi import NBodyError  # noqa: F401

__all__ = ["NBody", "NBodyError"]
__version__ = "0.1.0"
