"""B200-native community-reordered CSR SpMV (Balaji et al., ISPASS'23 hot path).

    spmv      ctypes binding of include/spmv.h (libspmv.so, sm_100a)
    dist      row-block power iteration over torch.distributed (NCCL all-gather)
    build     in-tree nvcc build of libspmv.so
"""
from . import spmv  # noqa: F401
from .spmv import Plan, SpmvError, reorder, scale_vec  # noqa: F401
