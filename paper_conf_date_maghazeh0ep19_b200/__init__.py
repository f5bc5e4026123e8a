"""B200-native KTILER: cache-aware kernel tiling of an image-processing kernel graph.

The product is libktiler.so (C ABI in include/ktiler.h: planner + sm_100a kernels +
launcher); this package is its ctypes binding (``ktiler``) and the north star's graphs
(``pipeline``).  No CPU fallback exists.
"""
from . import ktiler  # noqa: F401
from .pipeline import Motivational, Pipeline  # noqa: F401
