"""B200-native (sm_100a) hash-based two-phase CSR SpGEMM (Nagasaka, Nukada, Matsuoka, ICPP 2017).

C = A * B with A, B, C in CSR (int64 rpt, int32 col, fp32/fp64 values):
  phase 1 (symbolic): n_prod per row -> grouping -> per-group hash counting -> prefix sum,
  phase 2 (numeric):  grouping by nnz -> per-group hash accumulation -> gather -> sort -> write.
The kernels live in libspgemm.so (csrc/, C ABI in include/spgemm.h); this package only
marshals arguments.  See DESIGN.md.
"""
from ._lib import NUM_RANGE_GROUP, SYM_RANGE_GROUP, SpgemmError, group_bounds, load  # noqa: F401
from .spgemm import CsrMatrix, Handle, spgemm  # noqa: F401

__all__ = ["CsrMatrix", "Handle", "spgemm", "group_bounds", "load", "SpgemmError"]
