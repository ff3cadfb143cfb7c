"""CPU ORACLE for the two-phase hash SpGEMM — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference) may
import this package.  The product path (paper_conf_icpp_nagasakanm17_b200) never imports
it and shares no code with it.  Arithmetic lives in oracle/gustavson.c (plain C,
row-wise Gustavson, Alg. 1 and PAPER.md:90-96 Alg. 2) and
oracle/binning.py (Table-I style grouping).

Row-parallel variants (symbolic_omp, spgemm(parallel=True)): SURVEY.md §8(c) step 6, each row
still summed in Algorithm 1 order; pinned to the single-thread functions bit for bit.

Pins: tests/test_oracle_pins.py (closed forms, paper-printed Table II QCD count,
identities, brute force, column unions, scipy cross-check).  "parity unpinned": none of
the functions below.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Tuple

import numpy as np

from .binning import bin_of  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gustavson.c")
_SO = os.path.join(_HERE, "liboracle.so")
_LIB = None

CC_FLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    """Compile oracle/gustavson.c -> oracle/liboracle.so with gcc (no GPU needed)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CC_FLAGS, "-o", _SO, _SRC, "-lm"])
    return _SO


def _lib():
    global _LIB
    if _LIB is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        lib.oracle_nprod.restype = I64
        lib.oracle_nprod.argtypes = [I64, P, P, P, P]
        lib.oracle_symbolic.restype = ctypes.c_int
        lib.oracle_symbolic.argtypes = [I64, I64, I64, P, P, P, P, P]
        lib.oracle_symbolic_omp.restype = ctypes.c_int
        lib.oracle_symbolic_omp.argtypes = [I64, I64, I64, P, P, P, P, P]
        for f in (lib.oracle_numeric_f64, lib.oracle_numeric_f32, lib.oracle_numeric_omp_f64,
                  lib.oracle_numeric_omp_f32):
            f.restype = ctypes.c_int
            f.argtypes = [I64, I64, I64, P, P, P, P, P, P, P, P, P, P]
        lib.oracle_threads.restype = ctypes.c_int
        _LIB = lib
    return _LIB


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _csr_arrays(M):
    rpt = np.ascontiguousarray(M.rpt, dtype=np.int64)
    col = np.ascontiguousarray(M.col, dtype=np.int32)
    return rpt, col


def nprod(A, B) -> Tuple[np.ndarray, int]:
    """Per-row intermediate-product counts (Alg. 2) and their int64 total."""
    a_rpt, a_col = _csr_arrays(A)
    b_rpt, _ = _csr_arrays(B)
    out = np.empty(A.m, dtype=np.int64)
    total = _lib().oracle_nprod(A.m, _p(a_rpt), _p(a_col), _p(b_rpt), _p(out))
    return out, int(total)


def symbolic(A, B) -> np.ndarray:
    """rpt of C = A*B (int64, m+1), counting stored (not value-nonzero) entries."""
    a_rpt, a_col = _csr_arrays(A)
    b_rpt, b_col = _csr_arrays(B)
    c_rpt = np.empty(A.m + 1, dtype=np.int64)
    rc = _lib().oracle_symbolic(A.m, B.m, B.n, _p(a_rpt), _p(a_col), _p(b_rpt), _p(b_col), _p(c_rpt))
    if rc != 0:
        raise ValueError(f"oracle_symbolic failed: {rc}")
    return c_rpt


def symbolic_omp(A, B) -> np.ndarray:
    """symbolic() on all host cores (row-parallel; identical result)."""
    a_rpt, a_col = _csr_arrays(A)
    b_rpt, b_col = _csr_arrays(B)
    c_rpt = np.empty(A.m + 1, dtype=np.int64)
    rc = _lib().oracle_symbolic_omp(A.m, B.m, B.n, _p(a_rpt), _p(a_col), _p(b_rpt), _p(b_col), _p(c_rpt))
    if rc != 0:
        raise ValueError(f"oracle_symbolic_omp failed: {rc}")
    return c_rpt


def threads() -> int:
    """Threads the row-parallel functions use (OMP_NUM_THREADS, else all cores of the process)."""
    return int(_lib().oracle_threads())


def cores() -> int:
    """Host cores available to this process."""
    return len(os.sched_getaffinity(0))


def spgemm(A, B, dtype=np.float64, parallel: bool = False, with_abs: bool = True):
    """C = A*B in working precision `dtype` (np.float32 or np.float64).

    Returns (rpt int64[m+1], col int32[nnz], val dtype[nnz], absval float64[nnz] or None) where
    absval = (|A|*|B|)_ij is the scale of the comparison tolerance.  parallel=True runs the
    row-parallel functions (same result, all host cores)."""
    dtype = np.dtype(dtype)
    a_rpt, a_col = _csr_arrays(A)
    b_rpt, b_col = _csr_arrays(B)
    a_val = np.ascontiguousarray(A.val, dtype=dtype)
    b_val = np.ascontiguousarray(B.val, dtype=dtype)
    c_rpt = symbolic_omp(A, B) if parallel else symbolic(A, B)
    nnz = int(c_rpt[-1])
    c_col = np.empty(nnz, dtype=np.int32)
    c_val = np.empty(nnz, dtype=dtype)
    c_abs = np.empty(nnz, dtype=np.float64) if (with_abs or not parallel) else None
    if parallel:
        fn = _lib().oracle_numeric_omp_f64 if dtype == np.float64 else _lib().oracle_numeric_omp_f32
    else:
        fn = _lib().oracle_numeric_f64 if dtype == np.float64 else _lib().oracle_numeric_f32
    if dtype not in (np.float64, np.float32):
        raise TypeError(dtype)
    rc = fn(A.m, B.m, B.n, _p(a_rpt), _p(a_col), _p(a_val), _p(b_rpt), _p(b_col), _p(b_val),
            _p(c_rpt), _p(c_col), _p(c_val), _p(c_abs))
    if rc != 0:
        raise ValueError(f"oracle numeric failed: {rc}")
    return c_rpt, c_col, c_val, c_abs


def row_slice(A, r0: int, r1: int):
    """Rows [r0, r1) of A as a CSR view (used to check row-block sharding)."""
    from synth import Csr
    s, e = int(A.rpt[r0]), int(A.rpt[r1])
    return Csr(r1 - r0, A.n, A.rpt[r0:r1 + 1] - s, A.col[s:e],
               None if A.val is None else A.val[s:e], A.name + f"[{r0}:{r1}]")
