"""Seeded synthetic CSR inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NO arithmetic of the SpGEMM method: no products, no hashing, no
intermediate-product counts, no binning.  It only builds matrix *structure* and
*values* with the shapes of the paper's workloads (Table II),
following the recipes of SURVEY.md §8(d) restated in DESIGN.md "Input recipe".

All generators use NumPy PCG64 (`np.random.default_rng(seed)`) except R-MAT (synth/rmat.c,
a counter-based splitmix64 draw, compiled on first use) and return a `Csr`
with int64 row pointers, int32 column indices (sorted, de-duplicated unless a
generator says otherwise) and float64 values (callers cast to float32 for SP runs;
both sides then see the identical rounded values).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Optional

import numpy as np


@dataclass
class Csr:
    m: int
    n: int
    rpt: np.ndarray  # int64 [m+1]
    col: np.ndarray  # int32 [nnz]
    val: Optional[np.ndarray] = None  # float64/float32 [nnz]
    name: str = ""
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.rpt[-1] - self.rpt[0])

    def row_lengths(self) -> np.ndarray:
        return np.diff(self.rpt)

    def with_values(self, kind: str = "uniform", seed: int = 0) -> "Csr":
        return Csr(self.m, self.n, self.rpt, self.col, values(self.nnz, kind, seed),
                   self.name, dict(self.meta, values=kind))

    def astype(self, dtype) -> "Csr":
        return Csr(self.m, self.n, self.rpt, self.col,
                   None if self.val is None else self.val.astype(dtype), self.name, self.meta)

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.m, self.n), dtype=np.float64)
        rows = np.repeat(np.arange(self.m), np.diff(self.rpt))
        np.add.at(d, (rows, self.col[: len(rows)]), self.val if self.val is not None else 1.0)
        return d


# --------------------------------------------------------------------------- values

def values(nnz: int, kind: str = "uniform", seed: int = 0) -> np.ndarray:
    """Value recipes: uniform U(-1,1); int {-3..3}; positive U(0.5,1.5); ones."""
    rng = np.random.default_rng(seed + 7919)
    if kind == "uniform":
        return rng.uniform(-1.0, 1.0, size=nnz)
    if kind == "int":
        return rng.integers(-3, 4, size=nnz).astype(np.float64)
    if kind == "positive":
        return rng.uniform(0.5, 1.5, size=nnz)
    if kind == "ones":
        return np.ones(nnz, dtype=np.float64)
    raise ValueError(f"unknown value kind {kind!r}")


# --------------------------------------------------------------------------- assembly

def from_coo(m: int, n: int, rows: np.ndarray, cols: np.ndarray,
             vals: Optional[np.ndarray] = None, dedup: bool = True, name: str = "") -> Csr:
    """Sort (row, col) pairs into CSR; with dedup=True repeated pairs are merged (values summed)."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    key = rows * np.int64(n) + cols
    if dedup:
        if vals is None:
            key = np.unique(key)
            v = None
        else:
            key, inv = np.unique(key, return_inverse=True)
            v = np.zeros(len(key), dtype=np.float64)
            np.add.at(v, inv, vals)
    else:
        order = np.argsort(key, kind="stable")
        key = key[order]
        v = None if vals is None else np.asarray(vals, dtype=np.float64)[order]
    r = key // n
    c = (key - r * n).astype(np.int32)
    rpt = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rpt[1:])
    return Csr(m, n, rpt, c, v, name)


# --------------------------------------------------------------------------- structures

def poisson2d(n: int) -> Csr:
    """Config 1: 2-D 5-point Laplacian on an n x n grid, 4 on the diagonal, -1 on neighbours."""
    idx = np.arange(n * n, dtype=np.int64)
    x, y = idx // n, idx % n
    R, C, V = [idx], [idx], [np.full(n * n, 4.0)]
    for mask, off in ((x > 0, -n), (x < n - 1, n), (y > 0, -1), (y < n - 1, 1)):
        R.append(idx[mask]); C.append(idx[mask] + off); V.append(np.full(int(mask.sum()), -1.0))
    A = from_coo(n * n, n * n, np.concatenate(R), np.concatenate(C), np.concatenate(V),
                 name=f"poisson{n}")
    A.meta["values"] = "poisson"
    return A


def banded(M: int, lo: int, hi: int, w: int, seed: int, name: str = "banded") -> Csr:
    """FEM-like band (cant-like recipe): L_i ~ U{lo..hi}; columns drawn without replacement
    from [i-w, i+w] ∩ [0, M); the diagonal is always present."""
    rng = np.random.default_rng(seed)
    L = rng.integers(lo, hi + 1, size=M)
    width = 2 * w + 1
    offs = np.arange(-w, w + 1, dtype=np.int64)
    rpt = np.zeros(M + 1, dtype=np.int64)
    cols_out = []
    chunk = max(1, (1 << 22) // width)
    for s in range(0, M, chunk):
        e = min(M, s + chunk)
        rows = np.arange(s, e, dtype=np.int64)
        cols = rows[:, None] + offs[None, :]
        valid = (cols >= 0) & (cols < M)
        keys = rng.random((e - s, width))
        keys[:, w] = -1.0  # force the diagonal
        keys[~valid] = 2.0
        srt = np.sort(keys, axis=1)
        k = np.minimum(L[s:e], valid.sum(axis=1))
        kth = np.take_along_axis(srt, (k - 1)[:, None], axis=1)
        sel = (keys <= kth) & valid
        rpt[s + 1:e + 1] = sel.sum(axis=1)
        cols_out.append(cols[sel])
    np.cumsum(rpt, out=rpt)
    col = np.concatenate(cols_out).astype(np.int32)
    return Csr(M, M, rpt, col, None, name)


def _powerlaw_lengths(rng, M: int, alpha: float, lmax: int) -> np.ndarray:
    lv = np.arange(1, lmax + 1, dtype=np.float64)
    p = lv ** (-alpha)
    p /= p.sum()
    return rng.choice(np.arange(1, lmax + 1), size=M, p=p)


def webbase_like(M: int = 1_000_005, seed: int = 7, lmax: int = 4700, alpha: float = 2.15) -> Csr:
    """Config 3: power-law web graph (webbase-1M shape)."""
    rng = np.random.default_rng(seed)
    L = _powerlaw_lengths(rng, M, alpha, lmax)
    L[M // 2] = lmax
    for s in range(0, M, 4096):  # rows sorted by length (descending) inside 4096-row host blocks
        L[s:s + 4096] = np.sort(L[s:s + 4096])[::-1]
    rows = np.repeat(np.arange(M, dtype=np.int64), L)
    h = np.repeat(np.maximum(8, 2 * L), L)
    local = rng.random(len(rows)) < 0.95
    cols = np.clip(rows + rng.integers(-h, h + 1), 0, M - 1)
    cdf = np.cumsum(L.astype(np.float64)); cdf /= cdf[-1]
    ng = int((~local).sum())
    cols[~local] = np.minimum(np.searchsorted(cdf, rng.random(ng), side="right"), M - 1)
    return from_coo(M, M, rows, cols, name="webbase_like")


def _powerlaw_window(M, alpha, lmax, window, frac_global, seed, name, symmetrise=False) -> Csr:
    rng = np.random.default_rng(seed)
    L = _powerlaw_lengths(rng, M, alpha, lmax)
    rows = np.repeat(np.arange(M, dtype=np.int64), L)
    glob = rng.random(len(rows)) < frac_global
    cols = np.clip(rows + rng.integers(-window, window + 1, size=len(rows)), 0, M - 1)
    cols[glob] = rng.integers(0, M, size=int(glob.sum()))
    d = np.arange(M, dtype=np.int64)
    rows = np.concatenate([rows, d]); cols = np.concatenate([cols, d])
    if symmetrise:
        rows, cols = np.concatenate([rows, cols]), np.concatenate([cols, rows])
    return from_coo(M, M, rows, cols, name=name)


def economics_like(seed: int = 19) -> Csr:
    return _powerlaw_window(206_500, 1.6, 43, 2000, 0.30, seed, "economics_like")


def circuit_like(seed: int = 20) -> Csr:
    return _powerlaw_window(170_998, 2.2, 176, 50, 0.02, seed, "circuit_like", symmetrise=True)


def qcd_like(L: int = 8) -> Csr:
    """QCD-like: L^4 periodic lattice x 12 dof (3 colours x 4 spins), 39 nnz per row
    (SURVEY.md §8(d)); index = site*12 + s*3 + c, site = C-order ravel of (x0,x1,x2,x3)."""
    nsite = L ** 4
    M = nsite * 12
    site = np.arange(nsite, dtype=np.int64)
    coords = np.stack(np.unravel_index(site, (L, L, L, L)), axis=1)
    R, C = [], []
    for s in range(4):
        for c in range(3):
            row = site * 12 + s * 3 + c
            for c2 in range(3):  # on-site colour mixing
                R.append(row); C.append(site * 12 + s * 3 + c2)
            for mu in range(4):
                for sign in (+1, -1):
                    nc = coords.copy()
                    nc[:, mu] = (nc[:, mu] + sign) % L
                    nsite_idx = np.ravel_multi_index(tuple(nc.T), (L, L, L, L)).astype(np.int64)
                    spins = (s, (s + 2) % 4) if sign > 0 else (((s + mu) % 4),)
                    for s2 in spins:
                        for c2 in range(3):
                            R.append(row); C.append(nsite_idx * 12 + s2 * 3 + c2)
    return from_coo(M, M, np.concatenate(R), np.concatenate(C), name="qcd_like")


def epidemiology_like(n: int = 725) -> Csr:
    """Epidemiology-like: n x n torus, moves {(1,0),(-1,0),(0,1),(1,1)}; 4 nnz per row."""
    idx = np.arange(n * n, dtype=np.int64)
    x, y = idx // n, idx % n
    R, C = [], []
    for dx, dy in ((1, 0), (-1, 0), (0, 1), (1, 1)):
        R.append(idx); C.append(((x + dx) % n) * n + (y + dy) % n)
    return from_coo(n * n, n * n, np.concatenate(R), np.concatenate(C), name="epidemiology_like")


_RMAT_SO = None


def _rmat_lib():
    """Compile synth/rmat.c (gcc -O3 -fopenmp) on first use and load it (ctypes)."""
    global _RMAT_SO
    if _RMAT_SO is None:
        import ctypes
        import os
        import subprocess
        here = os.path.dirname(os.path.abspath(__file__))
        src, so = os.path.join(here, "rmat.c"), os.path.join(here, "librmat.so")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-o", so, src])
        lib = ctypes.CDLL(so)
        lib.rmat_csr.restype = ctypes.c_int64
        lib.rmat_csr.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_double, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
        _RMAT_SO = lib
    return _RMAT_SO


def rmat(scale: int, edge_factor: int = 16, a: float = 0.45, b: float = 0.15, c: float = 0.15,
         seed: int = 1) -> Csr:
    """Config 5: R-MAT (a,b,c,d) directed graph, duplicates merged, no relabelling
    (synth/rmat.c: counter-based draws, OpenMP; s22 in ~1 s on 8 cores)."""
    N = 1 << scale
    rpt = np.empty(N + 1, dtype=np.int64)
    col = np.empty(edge_factor * N, dtype=np.int32)
    nnz = _rmat_lib().rmat_csr(scale, edge_factor, a, b, c, seed, rpt.ctypes.data, col.ctypes.data)
    if nnz < 0:
        raise MemoryError("rmat_csr: out of host memory")
    return Csr(N, N, rpt, col[:nnz].copy(), None, f"rmat{scale}")


_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _mix64(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic), as in synth/rmat.c."""
    z = z + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def _rmat_numpy(scale: int, edge_factor: int = 16, a: float = 0.45, b: float = 0.15, c: float = 0.15,
                seed: int = 1) -> Csr:
    """The same generator as synth/rmat.c in NumPy (small scales; cross-check of the C build)."""
    N = 1 << scale
    E = edge_factor * N
    s0 = _mix64(np.array([seed], dtype=np.uint64))[0]
    e = np.arange(E, dtype=np.uint64)
    r = np.zeros(E, dtype=np.int64)
    q = np.zeros(E, dtype=np.int64)
    ab, abc = a + b, a + b + c
    for lvl in range(scale):
        x = _mix64(s0 ^ (e * np.uint64(64) + np.uint64(lvl)))
        u = (x >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
        r |= (u >= ab).astype(np.int64) << lvl
        q |= (((u >= a) & (u < ab)) | (u >= abc)).astype(np.int64) << lvl
    key = np.unique(r * N + q)
    rr = key // N
    col = (key - rr * N).astype(np.int32)
    rpt = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(np.bincount(rr, minlength=N), out=rpt[1:])
    return Csr(N, N, rpt, col, None, f"rmat{scale}")


def aggregation_prolongator(n: int, agg: int = 2, smoothed: bool = True, seed: int = 0) -> Csr:
    """AMG prolongator of the n x n 5-point grid (the Galerkin product R A P of
    algebraic multigrid is a chained SpGEMM).  Aggregates are agg x agg blocks of grid points;
    coarse point c = (x // agg) * ceil(n / agg) + y // agg.  Tentative prolongator: one entry per
    fine point (its aggregate).  smoothed=True gives the STRUCTURE of the smoothed-aggregation
    prolongator (I - w D^-1 A) P_tent — row i holds the aggregates of i and of its grid neighbours —
    built combinatorially (no product is formed here); values are seeded U(0.5, 1.5)."""
    nc = -(-n // agg)
    idx = np.arange(n * n, dtype=np.int64)
    x, y = idx // n, idx % n
    R, C = [idx], [(x // agg) * nc + y // agg]
    if smoothed:
        for dx, dy in ((1, 0), (-1, 0), (0, 1), (0, -1)):
            ok = (x + dx >= 0) & (x + dx < n) & (y + dy >= 0) & (y + dy < n)
            R.append(idx[ok]); C.append(((x[ok] + dx) // agg) * nc + (y[ok] + dy) // agg)
    Pm = from_coo(n * n, nc * nc, np.concatenate(R), np.concatenate(C), name=f"prolongator{n}")
    return Pm.with_values("positive", seed)


def transpose(M: Csr) -> Csr:
    """CSR of M^T (a format conversion: the same entries, rows and columns swapped)."""
    rows = np.repeat(np.arange(M.m, dtype=np.int64), np.diff(M.rpt))
    T = from_coo(M.n, M.m, M.col.astype(np.int64), rows, M.val, dedup=False, name=M.name + "^T")
    T.meta = dict(M.meta)
    return T


def random_sparse(m: int, n: int, density: float, seed: int, dup: bool = False,
                  unsorted: bool = False) -> Csr:
    """Small random pattern for brute-force pins; optional duplicate/unsorted columns."""
    rng = np.random.default_rng(seed)
    nnz = int(round(m * n * density))
    rows = rng.integers(0, m, size=nnz)
    cols = rng.integers(0, n, size=nnz)
    if not dup:
        A = from_coo(m, n, rows, cols, name="random")
    else:
        A = from_coo(m, n, rows, cols, dedup=False, name="random_dup")
    if unsorted:
        col = A.col.copy()
        for i in range(m):
            s, e = A.rpt[i], A.rpt[i + 1]
            col[s:e] = rng.permutation(col[s:e])
        A = Csr(A.m, A.n, A.rpt, col, A.val, A.name + "_unsorted")
    return A


# --------------------------------------------------------------------------- named configs

MIXED = {
    # name: (builder, value kind) — SURVEY.md §8(d) config-4 families
    "protein": lambda: banded(36_417, 34, 204, 134, 11, "protein_like"),
    "spheres": lambda: banded(83_334, 63, 81, 80, 12, "spheres_like"),
    "cantilever": lambda: banded(62_451, 50, 78, 70, 1, "cant_like"),
    "ship": lambda: banded(140_874, 9, 102, 43, 14, "ship_like"),
    "windtunnel": lambda: banded(217_918, 2, 105, 38, 15, "windtunnel_like"),
    "harbor": lambda: banded(46_835, 2, 100, 42, 16, "harbor_like"),
    "qcd": qcd_like,
    "accelerator": lambda: banded(121_192, 2, 41, 40, 18, "accelerator_like"),
    "economics": economics_like,
    "circuit": circuit_like,
    "epidemiology": epidemiology_like,
    "webbase": webbase_like,
}


def config(name: str, value_kind: str = "uniform", seed: int = 0) -> Csr:
    """BASELINE.json configs: 'poisson64' (1), 'cant' (2), 'webbase' (3), 'mixed:<family>' (4),
    'rmat<scale>' (5).  Poisson keeps its own stencil values."""
    if name.startswith("poisson"):
        return poisson2d(int(name[len("poisson"):] or 64))
    if name == "cant":
        A = MIXED["cantilever"]()
    elif name == "webbase":
        A = webbase_like()
    elif name.startswith("mixed:"):
        A = MIXED[name.split(":", 1)[1]]()
    elif name.startswith("rmat"):
        A = rmat(int(name[4:]))
    else:
        raise ValueError(f"unknown config {name!r}")
    return A.with_values(value_kind, seed)
