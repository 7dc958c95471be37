"""B200-native CRSD SpMV (Sun et al., ICPP 2011): y = alpha*A*x + beta*y for
diagonal sparse matrices stored in Compressed Row Segment with
Diagonal-pattern format. The compute path is libcrsd.so (C-ABI in
include/crsd.h, sm_100a kernels in csrc/); this package is its binding.
"""
from .crsd import (  # noqa: F401
    CRSDMatrix,
    Comm,
    P2PComm,
    CRSDError,
    dist_plan,
    partition_rows,
    version,
    CRSD_SUM_DUPLICATES,
    CRSD_HOST_ONLY,
    CRSD_DROP_ZEROS,
    CRSD_PAPER_ELL,
    CGResult,
    TUNE_JIT_DESC_ISSUE,
    TUNE_JIT_ONE_LAUNCH,
    TUNE_JIT_SPLIT_ALL,
    TUNE_JIT_SEQUENTIAL,
    TUNE_DIST_BOUNDARY_SERIAL,
    TUNE_NO_JIT,
    TUNE_HALO_UNFUSED,
    TUNE_JIT_NO_PDL,
    TUNE_JIT_NO_SLAB,
    TUNE_JIT_NO_REGSTAGE,
)
