"""B200-native accessibility-map (AM) engine -- AICA (Chen et al., ICPP 2019).

The compute path is the C-ABI library ``libam.so`` (CUDA, sm_100a) declared in
``include/am.h``; this package is the thin Python binding over it (argument
marshalling only -- every step of the AM runs in the library's kernels) plus
the multi-GPU drivers in :mod:`.distributed`.  Importing it without the built
library raises immediately: there is no CPU fallback.
"""
from .binding import (  # noqa: F401
    AM_EINVAL, AM_ECUDA, AM_ENOMEM, AM_ESTATE, AM_OK, AMError, Context, LIB_PATH, Stats,
    exported_symbols, lib, unpack, words_per_map,
)

__all__ = ["Context", "Stats", "AMError", "unpack", "words_per_map", "LIB_PATH", "lib",
           "exported_symbols"]
