"""B200-native (sm_100a) implementation of the CRoCCo v2.0 hot path
(Davis et al., IPDPS 2023): curvilinear compressible Navier-Stokes RHS with
characteristic WENO-SYMBO inviscid fluxes, 4th-order central viscous fluxes,
Williamson low-storage RK3 and block ghost fill, as the C-ABI library
libcrocco.so (include/crocco.h).  ``crocco`` is the ctypes binding with the
C names; ``solver.Solver`` is a thin torch-memory driver over it.
"""
from . import crocco  # noqa: F401

__all__ = ["crocco"]
