"""B200-native yaSpMV: y = A·x over BCCOO / BCCOO+ (Yan, Li, Zhang, Zhou, PPoPP'14).

The product is the C-ABI library ``libyaspmv.so`` (include/yaspmv.h); this package is
its thin Python binding plus the multi-GPU power-iteration driver (``dist``).
"""
from ._lib import YaspmvError, EXPORTED  # noqa: F401  (raises ImportError if the .so is missing)
from .matrix import Comm, Matrix, l2_persist, make_params, nrm2sq, nrm2sq_scratch_bytes, scale, version  # noqa: F401

__all__ = ["Comm", "Matrix", "l2_persist", "make_params", "nrm2sq", "nrm2sq_scratch_bytes", "scale", "version", "YaspmvError"]
