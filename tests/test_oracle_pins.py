"""Pins of the CPU oracle against what the paper and the mathematics fix (-m "not gpu").

Each pin is chosen so a plausible oracle mistake (dropped term, wrong sign, wrong index,
transposed operand, dropped structural zero, unsorted output) fails at least one test:
  * closed forms of the 5-point Poisson square (SURVEY.md §8(c) pins; verified by hand for n=2),
  * Table II's printed QCD intermediate-product count,
  * Table I's printed group bounds for the grouping oracle,
  * identities A*I = A, I*B = B, P*B, D*A (one product per entry => bit-exact),
  * dense brute force on tiny non-square inputs (pattern = boolean matmul of patterns),
  * column unions computed with Python sets, row sums C*1 = A*(B*1), transposes,
  * scipy.sparse cross-check with strictly positive values.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from synth import Csr, from_coo

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _dense_pattern(M: Csr) -> np.ndarray:
    d = np.zeros((M.m, M.n), dtype=bool)
    rows = np.repeat(np.arange(M.m), np.diff(M.rpt))
    d[rows, M.col] = True
    return d


def _rows_of(rpt, col):
    return [col[rpt[i]:rpt[i + 1]] for i in range(len(rpt) - 1)]


def _assert_sorted_rows(rpt, col):
    for i in range(len(rpt) - 1):
        r = col[rpt[i]:rpt[i + 1]]
        assert np.all(np.diff(r) > 0), f"row {i} not strictly increasing"


# ----------------------------------------------------------------- Poisson closed forms

def _poisson_nnz(n):
    return 5 * n * n - 4 * n


def _poisson_nprod(n):
    # interior rows: 5 entries x 5 = 25; edge (non-corner) rows: 4 entries, sum of degrees...
    return 25 * (n - 2) ** 2 + 16 * 4 * (n - 2) + 9 * 4


def _poisson_nnzc(n):
    return n * n + 4 * n * (n - 1) + 4 * n * (n - 2) + 4 * (n - 1) ** 2


@pytest.mark.parametrize("n", [2, 3, 4, 5, 7, 10, 33, 64])
def test_poisson_closed_forms(n):
    A = synth.poisson2d(n)
    assert A.nnz == _poisson_nnz(n)
    nprod, total = oracle.nprod(A, A)
    assert total == _poisson_nprod(n)
    rpt = oracle.symbolic(A, A)
    assert rpt[-1] == _poisson_nnzc(n)


def test_poisson64_histogram_and_values():
    A = synth.poisson2d(64)
    rpt, col, val, _ = oracle.spgemm(A, A, np.float64)
    hist = dict(zip(*np.unique(np.diff(rpt), return_counts=True)))
    assert hist == {13: 3600, 12: 240, 9: 240, 11: 4, 8: 8, 6: 4}
    _assert_sorted_rows(rpt, col)
    n = 64
    deg = np.diff(A.rpt) - 1
    for i in range(A.m):
        xi, yi = divmod(i, n)
        for c, v in zip(col[rpt[i]:rpt[i + 1]], val[rpt[i]:rpt[i + 1]]):
            xj, yj = divmod(int(c), n)
            dx, dy = abs(xi - xj), abs(yi - yj)
            if dx == dy == 0:
                assert v == 16 + deg[i]          # 4*4 + sum over neighbours (-1)(-1)
            elif dx + dy == 1:
                assert v == -8                   # a_ii a_ij + a_ij a_jj
            elif (dx, dy) in ((2, 0), (0, 2)):
                assert v == 1                    # one path through the middle node
            elif (dx, dy) == (1, 1):
                assert v == 2                    # two paths around the corner
            else:
                pytest.fail(f"unexpected entry ({i},{c})")
    # fp32 run is bit-identical (small integers)
    r32, c32, v32, _ = oracle.spgemm(A, A, np.float32)
    assert np.array_equal(r32, rpt) and np.array_equal(c32, col) and np.array_equal(v32, val)


# ----------------------------------------------------------------- lattice shapes

def test_epidemiology_torus():
    A = synth.epidemiology_like(37).with_values("ones")
    nprod, total = oracle.nprod(A, A)
    assert np.all(nprod == 16) and total == 16 * 37 * 37
    rpt, col, val, _ = oracle.spgemm(A, A, np.float64)
    assert np.all(np.diff(rpt) == 10)            # 10 distinct sums of two moves
    assert set(np.unique(val).tolist()) == {1.0, 2.0}
    assert np.all(np.add.reduceat(val, rpt[:-1]) == 16)
    big = synth.epidemiology_like(725)
    assert oracle.symbolic(big, big)[-1] == 10 * 725 * 725


def test_qcd_table2_paper_count():
    g = json.load(open(os.path.join(GOLDEN, "table2_qcd.json")))
    A = synth.qcd_like()
    assert A.m == g["rows"] and A.nnz == g["nnz"]
    assert np.diff(A.rpt).max() == g["max_nnz_per_row"]
    _, total = oracle.nprod(A, A)
    assert total == g["nprod_A2"]                # PAPER.md:205, printed
    rpt = oracle.symbolic(A, A)
    rows = _rows_of(A.rpt, A.col)
    for i in [0, 1, 11, 12345, A.m - 1]:         # set-union pin of the symbolic count
        u = set()
        for k in rows[i]:
            u.update(rows[k].tolist())
        assert rpt[i + 1] - rpt[i] == len(u) == 210
    Q = A.with_values("ones")
    rpt2, col2, val2, _ = oracle.spgemm(Q, Q, np.float64)
    assert np.all(np.add.reduceat(val2, rpt2[:-1]) == 39 * 39)


# ----------------------------------------------------------------- identities

def _eye(n):
    idx = np.arange(n)
    return from_coo(n, n, idx, idx, np.ones(n))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_identities(dtype):
    A = synth.random_sparse(53, 41, 0.15, seed=3).with_values("uniform", 1)
    A_d = A.astype(dtype)
    I_left, I_right = _eye(53).astype(dtype), _eye(41).astype(dtype)
    for L, R in ((A_d, I_right), (I_left, A_d)):
        rpt, col, val, _ = oracle.spgemm(L, R, dtype)
        assert np.array_equal(rpt, A.rpt) and np.array_equal(col, A.col)
        assert np.array_equal(val, A_d.val)
    # permutation P*A moves rows; D*A scales rows (one product per entry)
    rng = np.random.default_rng(5)
    perm = rng.permutation(53)
    P = from_coo(53, 53, np.arange(53), perm, np.ones(53)).astype(dtype)
    rpt, col, val, _ = oracle.spgemm(P, A_d, dtype)
    for i in range(53):
        s, e = A.rpt[perm[i]], A.rpt[perm[i] + 1]
        assert np.array_equal(col[rpt[i]:rpt[i + 1]], A.col[s:e])
        assert np.array_equal(val[rpt[i]:rpt[i + 1]], A_d.val[s:e])
    dvals = rng.uniform(-2, 2, 53)
    D = from_coo(53, 53, np.arange(53), np.arange(53), dvals).astype(dtype)
    rpt, col, val, _ = oracle.spgemm(D, A_d, dtype)
    rows = np.repeat(np.arange(53), np.diff(A.rpt))
    assert np.array_equal(val, (D.val[rows] * A_d.val).astype(dtype))


# ----------------------------------------------------------------- brute force

@pytest.mark.parametrize("seed", range(6))
def test_bruteforce_dense(seed):
    rng = np.random.default_rng(100 + seed)
    m, k, n = (int(x) for x in rng.integers(1, 65, size=3))
    dens = float(rng.uniform(0.02, 0.4))
    A = synth.random_sparse(m, k, dens, seed=seed).with_values("uniform", seed)
    B = synth.random_sparse(k, n, dens, seed=seed + 50).with_values("uniform", seed + 50)
    rpt, col, val, absv = oracle.spgemm(A, B, np.float64)
    pat = (_dense_pattern(A).astype(np.int64) @ _dense_pattern(B).astype(np.int64)) > 0
    got = np.zeros((m, n), dtype=bool)
    rows = np.repeat(np.arange(m), np.diff(rpt))
    got[rows, col] = True
    assert np.array_equal(got, pat)
    _assert_sorted_rows(rpt, col)
    D = A.to_dense() @ B.to_dense()
    assert np.all(np.abs(val - D[rows, col]) <= 1e-12 * absv + 1e-300)
    absD = np.abs(A.to_dense()) @ np.abs(B.to_dense())
    assert np.allclose(absv, absD[rows, col], rtol=1e-12, atol=0)
    # integer values: exact in both precisions
    Ai = A.with_values("int", seed); Bi = B.with_values("int", seed + 1)
    Di = Ai.to_dense() @ Bi.to_dense()
    for dt in (np.float64, np.float32):
        r2, c2, v2, _ = oracle.spgemm(Ai.astype(dt), Bi.astype(dt), dt)
        assert np.array_equal(r2, rpt) and np.array_equal(c2, col)
        assert np.array_equal(v2.astype(np.float64), Di[rows, col])


def test_column_union_sets_and_row_sums():
    A = synth.random_sparse(300, 200, 0.03, seed=9).with_values("int", 2)
    B = synth.random_sparse(200, 500, 0.02, seed=10).with_values("int", 3)
    rpt, col, val, _ = oracle.spgemm(A, B, np.float64)
    ra, rb = _rows_of(A.rpt, A.col), _rows_of(B.rpt, B.col)
    for i in range(A.m):
        u = set()
        for kk in ra[i]:
            u.update(rb[kk].tolist())
        assert sorted(u) == col[rpt[i]:rpt[i + 1]].tolist()
    ones = np.ones(B.n)
    rs_B = np.array([B.val[B.rpt[q]:B.rpt[q + 1]].sum() for q in range(B.m)])
    rs_AB = np.array([(A.val[A.rpt[i]:A.rpt[i + 1]] * rs_B[A.col[A.rpt[i]:A.rpt[i + 1]]]).sum()
                      for i in range(A.m)])
    rs_C = np.array([val[rpt[i]:rpt[i + 1]].sum() for i in range(A.m)])
    assert np.array_equal(rs_C, rs_AB) and ones.shape == (B.n,)


def test_nprod_column_count_identity():
    # sum_i nprod_i = sum_k nnz(A[:,k]) * nnz(B[k,:])  (a different route to Alg. 2's total)
    for seed in range(3):
        A = synth.random_sparse(120, 90, 0.05, seed=seed)
        B = synth.random_sparse(90, 70, 0.08, seed=seed + 7)
        _, total = oracle.nprod(A, B)
        colcount = np.bincount(A.col, minlength=A.n)
        assert total == int((colcount * np.diff(B.rpt)).sum())


# ----------------------------------------------------------------- structural zeros, transpose

def test_structural_zero_golden():
    g = json.load(open(os.path.join(GOLDEN, "structural_zero_2x2.json")))
    a = g["A"]
    A = Csr(a["m"], a["n"], np.array(a["rpt"], np.int64), np.array(a["col"], np.int32),
            np.array(a["val"]))
    for dt in (np.float64, np.float32):
        rpt, col, val, _ = oracle.spgemm(A.astype(dt), A.astype(dt), dt)
        assert rpt.tolist() == g["C"]["rpt"] and col.tolist() == g["C"]["col"]
        assert val.tolist() == g["C"]["val"]


def _transpose(M: Csr) -> Csr:
    rows = np.repeat(np.arange(M.m), np.diff(M.rpt))
    return from_coo(M.n, M.m, M.col, rows, M.val)


def test_transpose_identity():
    A = synth.random_sparse(70, 40, 0.08, seed=21).with_values("int", 1)
    B = synth.random_sparse(40, 90, 0.06, seed=22).with_values("int", 2)
    rpt, col, val, _ = oracle.spgemm(A, B, np.float64)
    C = Csr(A.m, B.n, rpt, col, val)
    rt, ct, vt, _ = oracle.spgemm(_transpose(B), _transpose(A), np.float64)
    Ct = _transpose(C)
    assert np.array_equal(Ct.rpt, rt) and np.array_equal(Ct.col, ct) and np.array_equal(Ct.val, vt)


def test_scipy_crosscheck_positive():
    sp = pytest.importorskip("scipy.sparse")
    A = synth.banded(3000, 5, 20, 15, seed=4).with_values("positive", 1)
    B = synth.random_sparse(3000, 2500, 0.002, seed=5).with_values("positive", 2)
    rpt, col, val, absv = oracle.spgemm(A, B, np.float64)
    SA = sp.csr_matrix((A.val, A.col, A.rpt), shape=(A.m, A.n))
    SB = sp.csr_matrix((B.val, B.col, B.rpt), shape=(B.m, B.n))
    SC = (SA @ SB).tocsr()
    SC.sort_indices()
    assert np.array_equal(SC.indptr, rpt) and np.array_equal(SC.indices, col)
    assert np.all(np.abs(SC.data - val) <= 1e-12 * absv)


# ----------------------------------------------------------------- input conventions

def test_duplicates_and_unsorted_inputs():
    base = synth.random_sparse(80, 60, 0.1, seed=31, dup=True)
    A = base.with_values("int", 4)
    B = synth.random_sparse(60, 75, 0.1, seed=32, unsorted=True).with_values("int", 5)
    rpt, col, val, _ = oracle.spgemm(A, B, np.float64)
    # reference: merge duplicates / sort first, then multiply
    rows = np.repeat(np.arange(A.m), np.diff(A.rpt))
    A2 = from_coo(A.m, A.n, rows, A.col, A.val)
    rowsb = np.repeat(np.arange(B.m), np.diff(B.rpt))
    B2 = from_coo(B.m, B.n, rowsb, B.col, B.val)
    r2, c2, v2, _ = oracle.spgemm(A2, B2, np.float64)
    assert np.array_equal(rpt, r2) and np.array_equal(col, c2) and np.array_equal(val, v2)
    assert A.nnz > A2.nnz  # the input really had duplicates


def test_empty_and_degenerate():
    E = Csr(0, 5, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0))
    B = synth.random_sparse(5, 4, 0.5, seed=1).with_values("uniform", 1)
    rpt, col, val, _ = oracle.spgemm(E, B, np.float64)
    assert rpt.tolist() == [0] and len(col) == 0
    Z = Csr(3, 5, np.zeros(4, np.int64), np.zeros(0, np.int32), np.zeros(0))
    rpt, col, val, _ = oracle.spgemm(Z, B, np.float64)
    assert rpt.tolist() == [0, 0, 0, 0]
    nprod, total = oracle.nprod(Z, B)
    assert total == 0 and np.all(nprod == 0)


def test_row_slice_offset():
    A = synth.random_sparse(100, 100, 0.05, seed=41).with_values("int", 1)
    rpt, col, val, _ = oracle.spgemm(A, A, np.float64)
    S = oracle.row_slice(A, 37, 81)
    # a_rpt[0] != 0 convention: pass the un-rebased pointers
    S_off = Csr(S.m, S.n, A.rpt[37:82].copy(), A.col, A.val)
    for X in (S, S_off):
        r2, c2, v2, _ = oracle.spgemm(X, A, np.float64)
        assert np.array_equal(r2, rpt[37:82] - rpt[37])
        assert np.array_equal(c2, col[rpt[37]:rpt[81]]) and np.array_equal(v2, val[rpt[37]:rpt[81]])


def test_oracle_rejects_bad_index():
    A = Csr(1, 3, np.array([0, 1], np.int64), np.array([5], np.int32), np.ones(1))
    B = synth.random_sparse(3, 3, 0.5, seed=1).with_values()
    with pytest.raises(ValueError):
        oracle.symbolic(A, B)


# ----------------------------------------------------------------- grouping oracle

def test_bin_of_table1_p100():
    g = json.load(open(os.path.join(GOLDEN, "table1_groups_p100.json")))
    groups = sorted(g["groups"], key=lambda x: -x["id"])   # ascending key ranges: 6,5,...,1
    for col_name in ("nprod", "nnz"):
        upper = [grp[col_name][1] for grp in groups if grp[col_name][1] is not None]
        paper_id = [grp["id"] for grp in groups]
        for grp in groups:
            lo, hi = grp[col_name]
            probes = [max(lo, 1), (hi if hi is not None else lo * 4)]
            for key in probes:
                b = int(oracle.bin_of([key], upper)[0])
                assert paper_id[b] == grp["id"], (col_name, key, b)
    assert oracle.bin_of([0], [32, 512])[0] == -1
    keys = np.random.default_rng(0).integers(0, 20000, size=10000)
    h = oracle.binning.group_histogram(keys, [32, 512, 1024, 2048, 4096, 8192])
    assert h.sum() == (keys > 0).sum()


# ----------------------------------------------------------------- working precision (R10)

@pytest.mark.parametrize("parallel", [False, True])
def test_fp32_working_precision(parallel):
    """Reading R10 (value tables of 4 B for SP): products and sums are rounded to
    fp32 in Algorithm 1's order.  Row 0: products 2^24, 1, -2^24 (in that order) sum to 0 in fp32
    (2^24 + 1 rounds to 2^24, ties-to-even) and to 1 in fp64.  Row 1: one product
    (1 + 2^-12)^2 = 1 + 2^-11 + 2^-24 rounds to 1 + 2^-11 in fp32 (tie, even mantissa) and is
    exact in fp64.  An oracle accumulating or multiplying in double fails the fp32 half."""
    x = 1.0 + 2.0 ** -12
    # A row 0 = [1, 1, 1] at cols 0..2, row 1 = [x] at col 0; B rows 0..2 = 2^24, 1, -2^24 at col 0
    B = Csr(3, 1, np.array([0, 1, 2, 3], dtype=np.int64), np.array([0, 0, 0], dtype=np.int32),
            np.array([2.0 ** 24, 1.0, -2.0 ** 24]))
    A2 = Csr(2, 3, np.array([0, 3, 4], dtype=np.int64), np.array([0, 1, 2, 0], dtype=np.int32),
             np.array([1.0, 1.0, 1.0, x]))
    rpt, col, v32, _ = oracle.spgemm(A2.astype(np.float32), B.astype(np.float32), np.float32, parallel=parallel)
    assert rpt.tolist() == [0, 1, 2] and col.tolist() == [0, 0]
    assert v32[0] == np.float32(0.0)
    assert v32[1] == np.float32(x * 2.0 ** 24)  # row 1 = x * b_00 = x * 2^24: exact in fp32
    rpt, col, v64, _ = oracle.spgemm(A2, B, np.float64, parallel=parallel)
    assert v64[0] == 1.0
    # the product rounding itself: (1 + 2^-12) * (1 + 2^-12) with both factors fp32
    P = Csr(1, 1, np.array([0, 1], dtype=np.int64), np.array([0], dtype=np.int32), np.array([x]))
    _, _, p32, _ = oracle.spgemm(P.astype(np.float32), P.astype(np.float32), np.float32, parallel=parallel)
    _, _, p64, _ = oracle.spgemm(P, P, np.float64, parallel=parallel)
    assert p32[0] == np.float32(1.0 + 2.0 ** -11)
    assert p64[0] == 1.0 + 2.0 ** -11 + 2.0 ** -24


@pytest.mark.parametrize("name,dtype", [("rmat12", np.float32), ("mixed:economics", np.float64),
                                        ("poisson64", np.float64)])
def test_parallel_oracle_identical(name, dtype):
    """the row-parallel oracle equals the single-thread one bit for bit
    (every row is still summed in Algorithm 1 order)."""
    A = synth.config(name).astype(dtype)
    s = oracle.spgemm(A, A, dtype)
    p = oracle.spgemm(A, A, dtype, parallel=True)
    for x, y in zip(s, p):
        assert np.array_equal(x, y)
    assert np.array_equal(oracle.symbolic_omp(A, A), s[0])
    assert oracle.threads() >= 1 and oracle.cores() >= 1


# ----------------------------------------------------------------- Galerkin product (chained, rectangular)

def test_galerkin_rap_closed_form():
    """PAPER.md:14, 302 (AMG's Galerkin product): with the tentative aggregation prolongator of 2x2
    aggregates (one 1 per fine row) on the n x n 5-point Laplacian, R A P (R = P^T) sums A over
    pairs of aggregates: an interior coarse row is again a 5-point stencil, 8 on the diagonal
    (4 points x 4 minus their 8 internal links) and -2 to each edge neighbour (2 crossing links)."""
    n = 8
    A = synth.poisson2d(n)
    P = synth.aggregation_prolongator(n, smoothed=False)
    P = Csr(P.m, P.n, P.rpt, P.col, np.ones(P.nnz), P.name)
    R = synth.transpose(P)
    rpt, col, val, _ = oracle.spgemm(A, P, np.float64)
    AP = Csr(A.m, P.n, rpt, col, val)
    assert (AP.m, AP.n) == (64, 16)
    rpt2, col2, val2, _ = oracle.spgemm(R, AP, np.float64)
    nc = n // 2
    for I in range(nc * nc):
        cx, cy = I // nc, I % nc
        row = dict(zip(col2[rpt2[I]:rpt2[I + 1]].tolist(), val2[rpt2[I]:rpt2[I + 1]].tolist()))
        want = {I: 8.0}  # 4 diagonals of 4 minus 4 internal links counted both ways (A's diagonal is 4 everywhere)
        for dx, dy in ((1, 0), (-1, 0), (0, 1), (0, -1)):
            if 0 <= cx + dx < nc and 0 <= cy + dy < nc:
                want[(cx + dx) * nc + cy + dy] = -2.0
        assert row == want, (I, row, want)
    # R A P of a symmetric A is symmetric
    D = np.zeros((nc * nc, nc * nc))
    for I in range(nc * nc):
        D[I, col2[rpt2[I]:rpt2[I + 1]]] = val2[rpt2[I]:rpt2[I + 1]]
    assert np.array_equal(D, D.T)
