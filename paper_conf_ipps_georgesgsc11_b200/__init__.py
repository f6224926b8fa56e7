"""B200-native multifrontal sparse SPD Cholesky: the factor-update hot path of
George et al., "Multifrontal Factorization of Sparse SPD Matrices on GPUs"
(IPDPS 2011), re-designed for sm_100a.

The product is the C-ABI library ``libmf.so`` (include/mf.h).  This package is
a thin ctypes binding with the same names (argument marshalling only).  There
is NO CPU fallback: importing the binding fails loudly if libmf.so is missing,
and ``mf_create`` fails without a CUDA device.
"""
from .mf import (  # noqa: F401
    MF_OK, MF_NOT_SPD, MF_ERR_ARG, MF_ERR_STATE, MF_ERR_NOMEM, MF_ERR_CUDA, MF_ERR_NCCL,
    MfError, MfNotSPD, lib, lib_path, Options, Info, Solver, EXPORTED_SYMBOLS, MF_VARIANTS, MF_VARIANT_FEATURES,
    DEV_ALLOC_FN, DEV_FREE_FN,
)
