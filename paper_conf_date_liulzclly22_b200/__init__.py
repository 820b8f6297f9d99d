"""B200-native batched 3-D L-shape pattern routing (FastGR pattern-routing stage).

The product is the C-ABI CUDA library ``libfastgr.so`` (include/fastgr.h);
``fastgr`` is its thin ctypes binding.
"""
from . import fastgr  # noqa: F401
from .fastgr import Router, FgrError  # noqa: F401
