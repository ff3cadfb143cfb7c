"""Generator statistics (-m "not gpu"): each config within tolerance of the recipe numbers
of SURVEY.md §8(d) / DESIGN.md "Input recipe" (exact for the deterministic lattices)."""
import numpy as np
import pytest

import oracle
import synth


def _check_csr(A):
    assert A.rpt.dtype == np.int64 and A.col.dtype == np.int32
    assert A.rpt[0] == 0 and np.all(np.diff(A.rpt) >= 0) and A.rpt[-1] == len(A.col)
    assert A.col.min() >= 0 and A.col.max() < A.n
    for i in range(0, A.m, max(1, A.m // 200)):
        r = A.col[A.rpt[i]:A.rpt[i + 1]]
        assert np.all(np.diff(r) > 0)


def test_poisson_config1():
    A = synth.config("poisson64")
    _check_csr(A)
    assert (A.m, A.nnz) == (4096, 20224)
    assert set(np.unique(A.val).tolist()) == {4.0, -1.0}


def test_cant_like_config2():
    A = synth.config("cant")
    _check_csr(A)
    assert A.m == 62451
    assert abs(A.nnz - 3_993_794) / 3_993_794 < 0.02
    L = A.row_lengths()
    assert L.max() <= 78 and L.min() >= 50
    assert np.all(np.abs(A.val) <= 1.0)


@pytest.mark.slow
def test_webbase_like_config3():
    A = synth.webbase_like()
    _check_csr(A)
    assert A.m == 1_000_005
    assert abs(A.nnz - 3_253_450) / 3_253_450 < 0.05
    assert 3000 < A.row_lengths().max() <= 4700
    _, total = oracle.nprod(A, A)
    assert 0.7 < total / 77_629_587 < 1.3


def test_lattices_exact():
    Q = synth.qcd_like()
    _check_csr(Q)
    assert np.all(Q.row_lengths() == 39) and Q.m == 49152
    E = synth.epidemiology_like()
    _check_csr(E)
    assert np.all(E.row_lengths() == 4) and E.m == 725 * 725


@pytest.mark.parametrize("fam,rows,per_row", [
    ("protein", 36417, 119.1), ("spheres", 83334, 72.0), ("ship", 140874, 54.2),
    ("windtunnel", 217918, 49.5), ("harbor", 46835, 50.0), ("accelerator", 121192, 21.5),
    ("economics", 206500, 5.4), ("circuit", 170998, 5.7)])
def test_mixed_families(fam, rows, per_row):
    A = synth.MIXED[fam]()
    _check_csr(A)
    assert A.m == rows
    assert abs(A.nnz / A.m - per_row) / per_row < 0.05


def test_rmat_small():
    A = synth.rmat(12)
    _check_csr(A)
    assert A.m == 4096 and 0.5 * 16 * 4096 < A.nnz <= 16 * 4096
    L = A.row_lengths()
    assert L[:16].mean() > 3 * L.mean()  # hubs at low indices (no relabelling)


def test_values_recipes():
    assert set(np.unique(synth.values(10000, "int", 1)).tolist()) == set(range(-3, 4))
    v = synth.values(10000, "positive", 1)
    assert v.min() >= 0.5 and v.max() <= 1.5
    v = synth.values(10000, "uniform", 1)
    assert v.min() >= -1 and v.max() <= 1
    assert np.array_equal(synth.values(100, "uniform", 3), synth.values(100, "uniform", 3))


@pytest.mark.parametrize("scale,seed", [(6, 1), (10, 1), (12, 5)])
def test_rmat_c_matches_numpy_twin(scale, seed):
    """synth/rmat.c (OpenMP, counter-based draws) equals its NumPy twin exactly."""
    from synth.matrices import _rmat_numpy
    A, B = synth.rmat(scale, seed=seed), _rmat_numpy(scale, seed=seed)
    assert np.array_equal(A.rpt, B.rpt) and np.array_equal(A.col, B.col)


def test_aggregation_prolongator_structure():
    """Tentative: one entry per fine row (its 2x2 aggregate); smoothed: the aggregates of the row's
    point and of its grid neighbours; transpose is an involution."""
    n = 10
    T = synth.aggregation_prolongator(n, smoothed=False)
    assert (T.m, T.n) == (100, 25) and np.all(np.diff(T.rpt) == 1)
    assert T.col[3 * n + 7] == (3 // 2) * 5 + 7 // 2
    S = synth.aggregation_prolongator(n)
    _check_csr(S)
    i = 4 * n + 5  # (4, 5): its aggregate (2, 2) and the neighbours' (1|2, 2) and (2, 2|3)
    assert S.col[S.rpt[i]:S.rpt[i + 1]].tolist() == sorted({2 * 5 + 2, 1 * 5 + 2, 2 * 5 + 3})
    TT = synth.transpose(synth.transpose(S))
    assert np.array_equal(TT.rpt, S.rpt) and np.array_equal(TT.col, S.col) and np.array_equal(TT.val, S.val)
