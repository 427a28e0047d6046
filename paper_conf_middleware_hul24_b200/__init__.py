"""Menos server segment on B200 (sm_100a): Python binding of libmenos.so.

The product is the C-ABI library (include/menos.h) built from csrc/ for sm_100a; this package only
marshals arguments.  See DESIGN.md for the path, the boundary and the kernels.
"""
from .menos import (FWD_NOGRAD, FWD_SAVE, TARGET_BITS, TARGET_INDEX, Batch, MenosError, Server,  # noqa: F401
                    launch_count, lib)
