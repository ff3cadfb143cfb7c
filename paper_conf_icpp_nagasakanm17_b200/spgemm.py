"""Python API over libspgemm.so: CSR tensors on a CUDA device, C = A * B.

PyTorch is used only for device memory and streams; every step of the two-phase hash
SpGEMM (Figure 1 (1)-(7)) runs in the library's sm_100a kernels.  There is no
CPU fallback: without the built library or a B200 the calls raise.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from typing import Optional

import numpy as np
import torch

from . import _lib
from ._lib import SPGEMM_F32, SPGEMM_F64, Allocator, Stats, check, load


@dataclass
class CsrMatrix:
    """CSR on a device: rpt int64 [m+1], col int32 [nnz], val float32/float64 [nnz] or None."""
    m: int
    n: int
    rpt: torch.Tensor
    col: torch.Tensor
    val: Optional[torch.Tensor] = None

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @classmethod
    def from_host(cls, A, device="cuda", dtype=torch.float32, pin: bool = False) -> "CsrMatrix":
        """From any object with m, n, rpt, col, val numpy arrays (e.g. synth.Csr)."""
        def t(x, dt):
            x = torch.from_numpy(np.ascontiguousarray(x)).to(dt)
            return x.pin_memory() if pin else (x.to(device) if device is not None else x)
        val = None if A.val is None else t(A.val, dtype)
        return cls(int(A.m), int(A.n), t(A.rpt, torch.int64), t(A.col, torch.int32), val)

    def to(self, device, non_blocking: bool = False) -> "CsrMatrix":
        return CsrMatrix(self.m, self.n, self.rpt.to(device, non_blocking=non_blocking),
                         self.col.to(device, non_blocking=non_blocking),
                         None if self.val is None else self.val.to(device, non_blocking=non_blocking))

    def numpy(self):
        return (self.rpt.cpu().numpy(), self.col.cpu().numpy(),
                None if self.val is None else self.val.cpu().numpy())


def _ptr(t: Optional[torch.Tensor]) -> Optional[int]:
    if t is None or t.numel() == 0:
        return None
    if not t.is_contiguous():
        raise ValueError("tensors must be contiguous")
    return t.data_ptr()


def _check_csr(M: CsrMatrix, device: torch.device, name: str) -> None:
    if M.rpt.dtype != torch.int64 or M.col.dtype != torch.int32:
        raise TypeError(f"{name}: rpt must be int64 and col int32")
    if M.rpt.device != device or M.col.device != device:
        raise ValueError(f"{name}: tensors must live on {device}")
    if M.rpt.numel() != M.m + 1:
        raise ValueError(f"{name}: rpt has {M.rpt.numel()} entries, expected m+1 = {M.m + 1}")


class Handle:
    """One spgemm_handle_t bound to a device and a stream (include/spgemm.h)."""

    def __init__(self, device=None, stream: Optional[torch.cuda.Stream] = None, torch_allocator: bool = False):
        lib = load()
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else
                                   torch.device(device).index or 0)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        self._alloc_keep = None
        alloc_ptr = None
        if torch_allocator:
            dev = self.device.index

            def _alloc(nbytes, stream, ctx):
                try:
                    return torch.cuda.caching_allocator_alloc(int(nbytes), dev, int(stream or 0))
                except RuntimeError:
                    return None

            def _free(ptr, nbytes, stream, ctx):
                torch.cuda.caching_allocator_delete(ptr)

            a = Allocator(_lib.ALLOC_FN(_alloc), _lib.FREE_FN(_free), None)
            self._alloc_keep = a
            alloc_ptr = ctypes.byref(a)
        h = ctypes.c_void_p()
        st = lib.spgemm_create(ctypes.byref(h), self.device.index, ctypes.c_void_p(self.stream.cuda_stream), alloc_ptr)
        self._h = h
        if st != 0:
            msg = (lib.spgemm_last_error(h) or b"").decode() if h.value else ""
            if h.value:
                lib.spgemm_destroy(h)
            self._h = None
            raise _lib.SpgemmError(st, f"spgemm_create: {msg}")
        self._A = self._B = None
        self.c_rpt = None
        self.nnz_c = 0
        self.nprod = 0
        # per-call ctypes objects and entry points, made once (host latency of small multiplies)
        self._nnz_out, self._nprod_out = ctypes.c_int64(), ctypes.c_int64()
        self._nnz_ref, self._nprod_ref = ctypes.byref(self._nnz_out), ctypes.byref(self._nprod_out)
        self._f_sym, self._f_num = lib.spgemm_symbolic, lib.spgemm_numeric

    # ----------------------------------------------------------------- options / info
    def set_option(self, name: str, value: int) -> "Handle":
        check(load().spgemm_set_option(self._h, _lib.OPTIONS[name], int(value)), self._h, f"set_option({name})")
        return self

    def stats(self) -> dict:
        s = Stats()
        check(load().spgemm_get_stats(self._h, ctypes.byref(s)), self._h, "spgemm_get_stats")
        return s.to_dict()

    def grouping(self, phase: int):
        """(n_prod int64[m], perm int32[m], offsets int64[ngroups+1]) of the last symbolic call."""
        m = self._A.m
        ng = 13 if phase == 1 else 21  # groups incl. cluster, global, range and batched ESC (numeric)
        nprod = np.empty(m, dtype=np.int64)
        perm = np.empty(m, dtype=np.int32)
        off = np.zeros(ng + 1, dtype=np.int64)
        check(load().spgemm_get_grouping(self._h, phase, nprod.ctypes.data_as(ctypes.c_void_p),
                                         perm.ctypes.data_as(ctypes.c_void_p),
                                         off.ctypes.data_as(ctypes.c_void_p)), self._h, "spgemm_get_grouping")
        return nprod, perm, off

    def _empty(self, n: int, dtype) -> torch.Tensor:
        """Device buffer from torch's caching allocator, associated with the handle's stream
        (no stream switch when that is already the current stream)."""
        if torch.cuda.current_stream(self.device) == self.stream:
            return torch.empty(n, dtype=dtype, device=self.device)
        with torch.cuda.stream(self.stream):
            return torch.empty(n, dtype=dtype, device=self.device)

    # ----------------------------------------------------------------- the two phases
    def symbolic(self, A: CsrMatrix, B: CsrMatrix, c_rpt: Optional[torch.Tensor] = None):
        """Phase 1 (PAPER.md:80 steps (1)-(4)): returns (c_rpt, nnz(C), sum n_prod)."""
        _check_csr(A, self.device, "A")
        _check_csr(B, self.device, "B")
        if A.n != B.m:
            raise ValueError(f"shape mismatch: A is {A.m}x{A.n}, B is {B.m}x{B.n}")
        if c_rpt is None:
            c_rpt = self._empty(A.m + 1, torch.int64)
        st = self._f_sym(self._h, A.m, B.m, B.n, _ptr(A.rpt), _ptr(A.col), _ptr(B.rpt), _ptr(B.col), _ptr(c_rpt),
                         self._nnz_ref, self._nprod_ref)
        check(st, self._h, "spgemm_symbolic")
        self._A, self._B, self.c_rpt = A, B, c_rpt
        self.nnz_c, self.nprod = self._nnz_out.value, self._nprod_out.value
        return c_rpt, self.nnz_c, self.nprod

    def numeric(self, a_val: torch.Tensor, b_val: torch.Tensor, c_col: torch.Tensor, c_val: torch.Tensor) -> None:
        """Phase 2 (PAPER.md:80 steps (6)-(7)), asynchronous on the handle's stream."""
        if a_val.dtype != b_val.dtype or c_val.dtype != a_val.dtype:
            raise TypeError("A, B and C values must share one dtype")
        dt = {torch.float32: SPGEMM_F32, torch.float64: SPGEMM_F64}.get(a_val.dtype)
        if dt is None:
            raise TypeError(f"unsupported dtype {a_val.dtype}")
        if c_col.dtype != torch.int32 or c_col.numel() != self.nnz_c or c_val.numel() != self.nnz_c:
            raise ValueError("c_col/c_val must hold exactly nnz(C) entries (int32 / value dtype)")
        st = self._f_num(self._h, dt, _ptr(a_val), _ptr(b_val), _ptr(c_col), _ptr(c_val))
        check(st, self._h, "spgemm_numeric")

    def multiply(self, A: CsrMatrix, B: CsrMatrix) -> CsrMatrix:
        """C = A * B with C allocated to its exact nnz."""
        c_rpt, nnz, _ = self.symbolic(A, B)
        # col and val of C in one allocation of exactly nnz(C) entries each
        vs = A.val.element_size()
        off = (4 * nnz + 15) // 16 * 16
        buf = self._empty(off + vs * nnz, torch.uint8)
        c_col = buf[:4 * nnz].view(torch.int32)
        c_val = buf[off:off + vs * nnz].view(A.val.dtype)
        self.numeric(A.val, B.val, c_col, c_val)
        return CsrMatrix(A.m, B.n, c_rpt, c_col, c_val)

    def row_partition(self, A: CsrMatrix, B: CsrMatrix, nparts: int) -> np.ndarray:
        """n_prod-balanced contiguous row blocks of A (multi-GPU sharding)."""
        splits = np.zeros(nparts + 1, dtype=np.int64)
        st = load().spgemm_row_partition(self._h, A.m, B.m, _ptr(A.rpt), _ptr(A.col), _ptr(B.rpt), nparts,
                                         splits.ctypes.data_as(ctypes.c_void_p))
        check(st, self._h, "spgemm_row_partition")
        return splits

    def close(self) -> None:
        if getattr(self, "_h", None) is not None and self._h.value:
            load().spgemm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def spgemm(A: CsrMatrix, B: CsrMatrix, handle: Optional[Handle] = None) -> CsrMatrix:
    """C = A * B on A's device (two-phase hash SpGEMM, sm_100a)."""
    if handle is None:
        with Handle(A.rpt.device) as h:
            return h.multiply(A, B)
    return handle.multiply(A, B)
