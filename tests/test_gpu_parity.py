"""Parity of the CUDA path (through the C ABI) with the CPU oracle (-m gpu).

Comparison rule: rpt and col bit-exact; values within
rtol * (|A||B|)_ij with rtol 1e-5 (fp32) / 1e-12 (fp64); integer-valued inputs bit-exact.
Inputs are the seeded synthetic configs of BASELINE.json (synth/), same arrays on both sides.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from synth import Csr, from_coo

pytestmark = pytest.mark.gpu

RTOL = {np.float32: 1e-5, np.float64: 1e-12}


@pytest.fixture(scope="module")
def spg():
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import paper_conf_icpp_nagasakanm17_b200 as P
    P.load()
    return P


def _dev(spg, M: Csr, dtype):
    return spg.CsrMatrix.from_host(M, "cuda", {np.float32: torch.float32, np.float64: torch.float64}[dtype])


def run_gpu(spg, A: Csr, B: Csr, dtype, opts=None, handle=None):
    own = handle is None
    h = handle or spg.Handle()
    try:
        h.set_option("timing", 2)
        for k, v in (opts or {}).items():
            h.set_option(k, v)
        C = h.multiply(_dev(spg, A.astype(dtype), dtype), _dev(spg, B.astype(dtype), dtype))
        torch.cuda.synchronize()
        st = h.stats()
        rpt, col, val = C.numpy()
        return rpt, col, val, st, h.nprod
    finally:
        if own:
            h.close()


def assert_parity(got, ref, dtype, exact=False, what=""):
    rpt, col, val = got[:3]
    r_rpt, r_col, r_val, r_abs = ref
    assert np.array_equal(rpt, r_rpt), f"{what}: rpt differs"
    assert np.array_equal(col, r_col), f"{what}: col differs"
    if exact:
        assert np.array_equal(val, r_val), f"{what}: values not bit-exact"
    else:
        err = np.abs(val.astype(np.float64) - r_val.astype(np.float64))
        bad = err > RTOL[dtype] * r_abs
        assert not bad.any(), f"{what}: {bad.sum()} values out of tolerance, max err/S " \
                              f"{(err / np.maximum(r_abs, 1e-300)).max():.3g}"


def check(spg, A, B, dtype, exact=False, opts=None, what=""):
    A = A.astype(dtype)
    B = B.astype(dtype)
    ref = oracle.spgemm(A, B, dtype)
    got = run_gpu(spg, A, B, dtype, opts)
    assert_parity(got, ref, dtype, exact, what)
    _, total = oracle.nprod(A, B)
    assert got[4] == total, f"{what}: nprod {got[4]} != {total}"
    return got


# ------------------------------------------------------------------ BASELINE configs

@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_config1_poisson(spg, dtype):
    A = synth.config("poisson64")
    got = check(spg, A, A, dtype, exact=True, what="poisson64")
    assert got[3]["nnz_c"] == 51972 and got[4] == 100104


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_config2_cant(spg, dtype):
    A = synth.config("cant")
    check(spg, A, A, dtype, what="cant")


def test_config2_cant_int_exact(spg):
    A = synth.config("cant", "int")
    check(spg, A, A, np.float32, exact=True, what="cant int")


def test_config3_webbase(spg):
    A = synth.config("webbase")
    got = check(spg, A, A, np.float32, what="webbase")
    assert got[3]["sym_rows"][10] > 0  # heavy rows exercise the optimistic/global path


def test_config3_webbase_int_exact(spg):
    A = synth.config("webbase", "int")
    check(spg, A, A, np.float32, exact=True, what="webbase int")


@pytest.mark.parametrize("family", list(synth.MIXED))
def test_config4_mixed(spg, family):
    A = synth.config(f"mixed:{family}")
    check(spg, A, A, np.float64, what=family)


def test_rmat_s16(spg):
    A = synth.rmat(16).with_values("uniform", 3)
    check(spg, A, A, np.float32, what="rmat16")


# ------------------------------------------------------------------ forced paths

def _mixed_small():
    A = synth.webbase_like(M=30000, seed=3, lmax=900, alpha=1.7)
    return A.with_values("uniform", 4)


def _banded_small():
    return synth.banded(20000, 2, 90, 60, seed=5, name="banded_small").with_values("uniform", 6)


@pytest.mark.parametrize("range_hash", [0, 1])
@pytest.mark.parametrize("group", list(range(0, 12)))
def test_forced_symbolic_group(spg, group, range_hash):
    for A in (_mixed_small(), _banded_small()):
        ref = oracle.spgemm(A, A, np.float64)
        got = run_gpu(spg, A, A, np.float64, {"sym_min_group": group, "range_hash": range_hash})
        assert_parity(got, ref, np.float64, what=f"{A.name} sym group>={group} range_hash={range_hash}")


@pytest.mark.parametrize("range_hash", [0, 1])
@pytest.mark.parametrize("group", list(range(0, 14)))
@pytest.mark.parametrize("bitmap_rank", [2, 0])  # CTA groups: two-level bitmap rank / bucket sort
def test_forced_numeric_group(spg, group, range_hash, bitmap_rank):
    if bitmap_rank == 0 and not 4 <= group <= 9:
        pytest.skip("bucket sort ablation only differs in the CTA-per-row groups")
    for A in (_mixed_small(), _banded_small()):
        ref = oracle.spgemm(A, A, np.float32)
        got = run_gpu(spg, A, A, np.float32, {"num_min_group": group, "range_hash": range_hash,
                                              "bitmap_rank": bitmap_rank})
        assert_parity(got, ref, np.float32, what=f"{A.name} num group>={group} range_hash={range_hash}")


@pytest.mark.parametrize("group", [4, 6, 8, 9])
def test_bitmap_rank_dense_clusters_f64(spg, group):
    """Two-level bitmap rank on rows whose keys form dense clusters plus far outliers (webbase
    shape), fp64 (group 9 fp64 exceeds shared memory with the rank scratch: bucket sort)."""
    A = synth.config("webbase", "int")
    A = oracle.row_slice(A, 0, 60000)
    B = synth.config("webbase", "int")
    got = check(spg, A, B, np.float64, exact=True, opts={"num_min_group": group}, what=f"dense clusters g{group}")


@pytest.mark.parametrize("config", ["cant", "webbase", "mixed:protein", "mixed:economics"])
def test_paper_hash_only(spg, config):
    """The paper's multiplicative hash everywhere (range-offset hash disabled)."""
    A = synth.config(config, "int")
    check(spg, A, A, np.float32, exact=True, opts={"range_hash": 0}, what=f"{config} paper hash")


def test_overflow_retry_in_global_memory(spg):
    """Optimistic one-CTA table -> cluster DSMEM table -> global table (PAPER.md:155 chain)."""
    A = _mixed_small()
    ref = oracle.spgemm(A, A, np.float64)
    got = run_gpu(spg, A, A, np.float64, {"sym_min_group": 10, "sym_fill_limit": 16, "range_hash": 0})
    assert got[3]["sym_overflow_rows"] > 0 and got[3]["sym_overflow2_rows"] == 0
    assert_parity(got, ref, np.float64, what="overflow -> cluster")
    got = run_gpu(spg, A, A, np.float64, {"sym_min_group": 10, "sym_fill_limit": 16, "range_hash": 0,
                                          "cluster_fill_limit": 40})
    assert got[3]["sym_overflow2_rows"] > 0
    assert_parity(got, ref, np.float64, what="overflow -> cluster -> global")
    got = run_gpu(spg, A, A, np.float64, {"sym_min_group": 10, "sym_fill_limit": 16, "range_hash": 0, "cluster": 0})
    assert_parity(got, ref, np.float64, what="overflow -> global (cluster off)")


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("group", [10, 11, 12])
def test_cluster_numeric_rows(spg, dtype, group):
    """Every row through a cluster-per-row numeric kernel (DSMEM table over 2/4/8 CTAs)."""
    for A in (_mixed_small(), _banded_small(), synth.config("poisson64")):
        ref = oracle.spgemm(A.astype(dtype), A.astype(dtype), dtype)
        got = run_gpu(spg, A, A, dtype, {"num_min_group": group})
        assert got[3]["num_rows"][group] == (np.diff(ref[0]) > 0).sum()
        assert_parity(got, ref, dtype, what=f"{A.name} cluster-{2 << (group - 10)} numeric")


@pytest.mark.parametrize("flat", [0, 1])
@pytest.mark.parametrize("group", [0, 3, 5, 8, 10, 13])
def test_flat_and_vw_loops(spg, flat, group):
    """Both product loops (load-balanced flattened / VW lanes per A entry) in every kernel family."""
    for A in (_mixed_small(), _banded_small()):
        ref = oracle.spgemm(A, A, np.float32)
        for opts in ({"num_min_group": group}, {"sym_min_group": min(group, 11), "range_hash": 0},
                     {"sym_min_group": 10, "sym_fill_limit": 16, "range_hash": 0}):
            got = run_gpu(spg, A, A, np.float32, dict(opts, flat=flat))
            assert_parity(got, ref, np.float32, what=f"{A.name} {opts} flat={flat}")


@pytest.mark.parametrize("lanes", [1, 2, 4, 8, 16, 32])
def test_lanes_per_b_row(spg, lanes):
    A = synth.MIXED["harbor"]().with_values("int", 1)
    ref = oracle.spgemm(A, A, np.float64)
    got = run_gpu(spg, A, A, np.float64, {"lanes": lanes})
    assert_parity(got, ref, np.float64, exact=True, what=f"lanes={lanes}")


@pytest.mark.parametrize("long_row", [-1, 1, 16])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_long_row_cta_pass(spg, long_row, dtype):
    """B rows longer than long_row are walked by the whole CTA (second pass); 1 = every row."""
    A = _mixed_small()
    ref = oracle.spgemm(A.astype(dtype), A.astype(dtype), dtype)
    for opts in ({"long_row": long_row}, {"long_row": long_row, "range_hash": 0},
                 {"long_row": long_row, "sym_min_group": 10, "sym_fill_limit": 64, "range_hash": 0},
                 {"long_row": long_row, "sym_min_group": 11, "num_min_group": 10}):
        got = run_gpu(spg, A, A, dtype, opts)
        assert_parity(got, ref, dtype, what=f"{opts}")


@pytest.mark.parametrize("graphs", [0, 1])
def test_graph_replay(spg, graphs):
    """Repeated multiplies on one handle replay the captured phase-1/phase-2 segments."""
    A = synth.config("mixed:economics", "int")
    ref = oracle.spgemm(A.astype(np.float32), A.astype(np.float32), np.float32)
    with spg.Handle() as h:
        h.set_option("graphs", graphs)
        dA = _dev(spg, A, np.float32)
        replays = 0
        for it in range(4):
            C = h.multiply(dA, dA)
            torch.cuda.synchronize()
            st = h.stats()
            assert_parity(C.numpy() + (None,), ref, np.float32, exact=True, what=f"iter {it}")
            replays += st["graph_replays"]
            if graphs and it == 3:  # (the caching allocator's output addresses repeat by now)
                assert replays >= 1
            if graphs:
                assert st["symbolic_ms"] > 0 and st["numeric_ms"] > 0
            else:
                assert max(st["num_group_ms"]) > 0 and max(st["sym_group_ms"]) > 0
            del C


def test_serial_streams(spg):
    A = _mixed_small()
    ref = oracle.spgemm(A, A, np.float64)
    got = run_gpu(spg, A, A, np.float64, {"streams": 0})
    assert_parity(got, ref, np.float64, what="no streams")


# ------------------------------------------------------------------ edge cases

def test_rectangular_and_identities(spg):
    A = synth.random_sparse(700, 300, 0.02, seed=1).with_values("uniform", 1)
    B = synth.random_sparse(300, 1100, 0.01, seed=2).with_values("uniform", 2)
    check(spg, A, B, np.float64, what="rect")
    idx = np.arange(300)
    I = from_coo(300, 300, idx, idx, np.ones(300))
    got = run_gpu(spg, A.astype(np.float32), I.astype(np.float32), np.float32)
    assert np.array_equal(got[0], A.rpt) and np.array_equal(got[1], A.col)
    assert np.array_equal(got[2], A.val.astype(np.float32))


def test_structural_zero_and_degenerate(spg):
    A = Csr(2, 2, np.array([0, 2, 4], np.int64), np.array([0, 1, 0, 1], np.int32),
            np.array([1.0, 1.0, 1.0, -1.0]))
    got = run_gpu(spg, A, A, np.float64)
    assert got[0].tolist() == [0, 2, 4] and got[1].tolist() == [0, 1, 0, 1]
    assert got[2].tolist() == [2.0, 0.0, 0.0, 2.0]
    # m = 0
    E = Csr(0, 5, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0))
    B = synth.random_sparse(5, 4, 0.5, seed=1).with_values()
    got = run_gpu(spg, E, B, np.float64)
    assert got[0].tolist() == [0] and len(got[1]) == 0
    # A with no entries / empty rows
    Z = Csr(3, 5, np.zeros(4, np.int64), np.zeros(0, np.int32), np.zeros(0))
    got = run_gpu(spg, Z, B, np.float32)
    assert got[0].tolist() == [0, 0, 0, 0]
    # empty rows interleaved
    A2 = synth.random_sparse(500, 500, 0.003, seed=9).with_values("int", 2)
    assert (np.diff(A2.rpt) == 0).any()
    check(spg, A2, A2, np.float64, exact=True, what="sparse empty rows")


def test_duplicates_unsorted(spg):
    A = synth.random_sparse(400, 300, 0.05, seed=31, dup=True).with_values("int", 4)
    B = synth.random_sparse(300, 350, 0.05, seed=32, unsorted=True).with_values("int", 5)
    check(spg, A, B, np.float64, exact=True, what="dup/unsorted")


def test_duplicate_columns_in_b_rows(spg):
    """Repeated columns inside B rows (legal input) must not race in any accumulation path."""
    base = synth.banded(3000, 4, 30, 20, seed=8)
    rng = np.random.default_rng(3)
    rows = np.repeat(np.arange(base.m), np.diff(base.rpt))
    extra = rng.integers(0, len(rows), size=len(rows) // 3)
    B = from_coo(base.m, base.n, np.concatenate([rows, rows[extra]]), np.concatenate([base.col, base.col[extra]]),
                 dedup=False).with_values("int", 2)
    A = synth.banded(3000, 4, 30, 20, seed=9).with_values("int", 1)
    for rh in (0, 1):
        check(spg, A, B, np.float64, exact=True, opts={"range_hash": rh}, what=f"dup B rows rh={rh}")
        check(spg, A, B, np.float32, exact=True, opts={"range_hash": rh, "lanes": 4}, what=f"dup B rows vw4 rh={rh}")


def test_large_column_indices(spg):
    n = 2**31 - 2
    rng = np.random.default_rng(0)
    B = from_coo(64, n, rng.integers(0, 64, 500), rng.integers(0, n, 500), rng.uniform(-1, 1, 500))
    A = synth.random_sparse(50, 64, 0.2, seed=4).with_values("uniform", 5)
    check(spg, A, B, np.float64, what="huge n")


def test_row_slice_offset_pointer(spg):
    A = synth.MIXED["accelerator"]().with_values("uniform", 2)
    ref = oracle.spgemm(A, A, np.float64)
    r0, r1 = 1000, 50000
    dA = _dev(spg, A, np.float64)
    sl = spg.CsrMatrix(r1 - r0, A.n, dA.rpt[r0:r1 + 1].contiguous(), dA.col, dA.val)  # a_rpt[0] != 0
    with spg.Handle() as h:
        C = h.multiply(sl, dA)
        rpt, col, val = C.numpy()
    s, e = ref[0][r0], ref[0][r1]
    assert np.array_equal(rpt, ref[0][r0:r1 + 1] - s)
    assert np.array_equal(col, ref[1][s:e])
    assert np.all(np.abs(val - ref[2][s:e]) <= 1e-12 * ref[3][s:e])


def test_structure_reuse_and_torch_allocator(spg):
    A = synth.MIXED["ship"]()
    A1 = A.with_values("int", 1)
    A2 = A.with_values("int", 2)
    r1 = oracle.spgemm(A1, A1, np.float64)
    r2 = oracle.spgemm(A2, A2, np.float64)
    with spg.Handle(torch_allocator=True) as h:
        d1 = _dev(spg, A1, np.float64)
        C = h.multiply(d1, d1)
        assert_parity(C.numpy() + (None,), r1, np.float64, exact=True, what="first")
        d2 = _dev(spg, A2, np.float64)
        h.numeric(d2.val, d2.val, C.col, C.val)   # same structure, new values
        assert_parity(C.numpy() + (None,), r2, np.float64, exact=True, what="reuse")
        st = h.stats()
        assert st["workspace_peak_bytes"] > 0


# ------------------------------------------------------------------ range rows (warp-per-row)

RANGE_CASES = ["cant", "mixed:protein", "mixed:accelerator", "mixed:circuit"]


@pytest.mark.parametrize("name", RANGE_CASES)
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("mode", [1, 2])  # 1: bitmap-union count, 2: per-product flags
def test_range_rows(spg, name, dtype, mode):
    """Every row that qualifies (min n_prod lowered to 1) through the warp-per-row kernels."""
    A = synth.config(name)
    got = check(spg, A, A, dtype, opts={"range_min_nprod": 1, "range_warp": mode}, what=f"{name} range rows")
    st = got[3]
    assert st["sym_rows"][spg.SYM_RANGE_GROUP] > 0
    assert st["num_rows"][spg.NUM_RANGE_GROUP] == st["sym_rows"][spg.SYM_RANGE_GROUP]


def test_range_rows_int_exact_and_deterministic(spg):
    A = synth.config("cant", "int")
    got = check(spg, A, A, np.float32, exact=True, what="cant int range")
    assert got[3]["num_rows"][spg.NUM_RANGE_GROUP] == A.m  # every cant row is a range row
    U = synth.config("cant")
    a = run_gpu(spg, U, U, np.float32)
    b = run_gpu(spg, U, U, np.float32)
    assert np.array_equal(a[2], b[2])  # plain read-modify-write accumulation: same bits every run


def test_range_rows_off_matches(spg):
    A = _banded_small()
    ref = oracle.spgemm(A, A, np.float64)
    on = run_gpu(spg, A, A, np.float64)
    off = run_gpu(spg, A, A, np.float64, {"range_warp": 0})
    assert on[3]["sym_rows"][spg.SYM_RANGE_GROUP] > 0 and off[3]["sym_rows"][spg.SYM_RANGE_GROUP] == 0
    assert_parity(on, ref, np.float64, what="range on")
    assert_parity(off, ref, np.float64, what="range off")


def test_range_rows_unsorted_b(spg):
    """B rows not strictly increasing: symbolic range rows stay, numeric takes the hash groups."""
    A = _banded_small()
    rng = np.random.default_rng(3)
    col = A.col.copy()
    for i in range(0, A.m, 7):  # reverse some rows
        s, e = A.rpt[i], A.rpt[i + 1]
        col[s:e] = col[s:e][::-1]
    B = Csr(A.m, A.n, A.rpt.copy(), col, A.val.copy(), name="banded_unsorted")
    got = check(spg, A, B, np.float64, what="unsorted B")
    assert got[3]["sym_rows"][spg.SYM_RANGE_GROUP] > 0 and got[3]["num_rows"][spg.NUM_RANGE_GROUP] == 0


@pytest.mark.parametrize("wmax", [40, 700])
def test_range_rows_ragged(spg, wmax):
    """Spans that are not multiples of 16/32, rows with a single A entry, empty rows, R = 1;
    wmax 700: spans beyond 1024 (flag-store count) and beyond 2048 (not range rows)."""
    rng = np.random.default_rng(11)
    m = 3000
    rows, cols = [], []
    for i in range(m):
        if i % 97 == 0:
            continue  # empty row
        w = int(rng.integers(0, wmax))
        L = int(rng.integers(1, 2 * w + 2))
        c = np.unique(np.clip(i + rng.integers(-w, w + 1, L), 0, m - 1))
        rows += [i] * len(c)
        cols += c.tolist()
    A = from_coo(m, m, np.array(rows), np.array(cols), name="ragged").with_values("uniform", 12)
    for dtype in (np.float32, np.float64):
        for mode in (1, 2):
            got = check(spg, A, A, dtype, opts={"range_min_nprod": 1, "range_warp": mode}, what="ragged range")
            assert got[3]["sym_rows"][spg.SYM_RANGE_GROUP] > 0


# ------------------------------------------------------------------ intermediate steps

def _block_diag(X: Csr, Y: Csr, name: str) -> Csr:
    rpt = np.concatenate([X.rpt[:-1] - X.rpt[0], Y.rpt - Y.rpt[0] + X.nnz]).astype(np.int64)
    col = np.concatenate([X.col, Y.col + X.n]).astype(np.int32)
    val = np.concatenate([X.val, Y.val])
    return Csr(X.m + Y.m, X.n + Y.n, rpt, col, val, name=name)


def test_nprod_and_grouping(spg):
    A = _block_diag(_mixed_small(), _banded_small(), "graph+banded")  # hash-group and range rows
    nprod_ref, total = oracle.nprod(A, A)
    ref_rpt = oracle.symbolic(A, A)
    with spg.Handle() as h:
        dA = _dev(spg, A, np.float32)
        h.symbolic(dA, dA)
        nprod, perm, off = h.grouping(1)
        nprod2, perm2, off2 = h.grouping(2)
    assert np.array_equal(nprod, nprod_ref) and h.nprod == total
    # range rows (kernels_range.cu): exact column span R_i of row i of C, from the oracle's C
    r_rpt, r_col, _, _ = oracle.spgemm(A, A, np.float32)
    lens = np.diff(r_rpt)
    span = np.zeros(A.m, dtype=np.int64)
    nz = lens > 0
    span[nz] = r_col[r_rpt[1:][nz] - 1].astype(np.int64) - r_col[r_rpt[:-1][nz]] + 1
    is_range = (nprod_ref >= 256) & (nprod_ref <= 65536) & (span <= 2048) & (span <= 4 * nprod_ref)
    assert is_range.any() and (~is_range & (nprod_ref > 0)).any()  # both kinds present
    for ph, (p, o, keys) in ((1, (perm, off, nprod_ref)), (2, (perm2, off2, np.diff(ref_rpt)))):
        upper = spg.group_bounds(ph)
        want = oracle.bin_of(keys, upper)
        want[is_range] = spg.SYM_RANGE_GROUP if ph == 1 else spg.NUM_RANGE_GROUP
        nonempty = np.flatnonzero(want >= 0)
        assert o[-1] == len(nonempty)
        assert np.array_equal(np.sort(p[:o[-1]]), nonempty)       # a permutation of grouped rows
        for g in range(len(o) - 1):
            rows = p[o[g]:o[g + 1]]
            assert np.all(want[rows] == g), f"phase {ph} group {g}"


def test_row_partition(spg):
    A = synth.config("webbase")
    nprod_ref, total = oracle.nprod(A, A)
    excl = np.concatenate([[0], np.cumsum(nprod_ref)])
    with spg.Handle() as h:
        dA = _dev(spg, A, np.float32)
        for P in (1, 2, 3, 8):
            s = h.row_partition(dA, dA, P)
            want = [int(np.searchsorted(excl, (total * p) // P, side="left")) for p in range(P)] + [A.m]
            assert s.tolist() == want


# ------------------------------------------------------------------ config 5 at full size

@pytest.mark.slow
def test_rmat_s20_full(spg):
    """R-MAT s20 (config 5's shape at 1/4 size): full rpt and every row against the oracle."""
    A = synth.rmat(20).with_values("uniform", 7)
    A32 = A.astype(np.float32)
    with spg.Handle() as h:
        dA = _dev(spg, A32, np.float32)
        C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        rpt = C.rpt.cpu().numpy()
        assert np.array_equal(rpt, oracle.symbolic_omp(A32, A32))
        _chunked_full_parity(C, A32, rpt, 1e-5)


def _sampled_rows_parity(C, A32, rows, rtol):
    """Compare the listed rows of a device C with the oracle, one row at a time, copying only
    those rows to the host (C may be tens of GB)."""
    rpt = C.rpt.cpu().numpy()
    for r in rows:
        r = int(r)
        S = oracle.row_slice(A32, r, r + 1)
        r_rpt, r_col, r_val, r_abs = oracle.spgemm(S, A32, np.float32)
        s, e = int(rpt[r]), int(rpt[r + 1])
        assert e - s == r_rpt[1], f"row {r}: nnz {e - s} != {r_rpt[1]}"
        assert np.array_equal(C.col[s:e].cpu().numpy(), r_col), f"row {r}: col differs"
        v = C.val[s:e].cpu().numpy()
        assert np.all(np.abs(v.astype(np.float64) - r_val) <= rtol * r_abs), f"row {r}: values"
    return rpt


def _chunked_full_parity(C, A32, rpt, rtol, max_entries=200_000_000):
    """Every row of a device C against the row-parallel oracle, in row blocks of at most
    `max_entries` output entries (C may be tens of GB): col bit-exact, values within rtol * S."""
    r0 = 0
    while r0 < A32.m:
        r1 = int(np.searchsorted(rpt, rpt[r0] + max_entries, side="right")) - 1
        r1 = min(A32.m, max(r1, r0 + 1))
        S = oracle.row_slice(A32, r0, r1)
        c_rpt, c_col, c_val, c_abs = oracle.spgemm(S, A32, np.float32, parallel=True)
        s, e = int(rpt[r0]), int(rpt[r1])
        assert np.array_equal(c_rpt + s, rpt[r0:r1 + 1]), f"rows [{r0}, {r1}): rpt"
        col = C.col[s:e].cpu().numpy()
        assert np.array_equal(col, c_col), f"rows [{r0}, {r1}): col differs"
        val = C.val[s:e].cpu().numpy().astype(np.float64)
        bad = np.abs(val - c_val.astype(np.float64)) > rtol * c_abs
        assert not bad.any(), f"rows [{r0}, {r1}): {int(bad.sum())} values out of tolerance"
        del col, val, c_col, c_val, c_abs
        r0 = r1


@pytest.mark.slow
def test_rmat_s22_full_parity(spg):
    """Config 5 at full single-GPU size, EVERY row: R-MAT(0.45,0.15,0.15,0.25) s22 ef16, nnz(C) >
    2^31 (int64 rpt path).  Full rpt against the row-parallel oracle's symbolic pass (Alg. 2 n_prod
    total too), then every row's columns bit-exact and values within 1e-5 * S in row blocks; the
    heaviest C rows (by C-row length) are in the blocks like every other row."""
    A = synth.rmat(22).with_values("uniform", 7)
    A32 = A.astype(np.float32)
    with spg.Handle() as h:
        dA = _dev(spg, A32, np.float32)
        C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        st = h.stats()
        _, total = oracle.nprod(A32, A32)
        assert h.nprod == total
        assert C.nnz > 2**31 - 1  # exercises 64-bit row pointers / output offsets
        rpt = C.rpt.cpu().numpy()
        assert np.array_equal(rpt, oracle.symbolic_omp(A32, A32)), "rpt differs from the oracle"
        assert st["nnz_c"] == C.nnz == rpt[-1]
        assert any(st["num_kernel"][g] == 9 for g in range(15, 22) if st["num_rows"][g]), "ESC rows expected at s22"
        heavy = np.argsort(np.diff(rpt))[-8:]  # C-row length
        assert np.diff(rpt)[heavy].min() > 8192  # rows beyond the CTA groups are part of the check
        _chunked_full_parity(C, A32, rpt, 1e-5)


@pytest.mark.slow
def test_rmat_s23_rpt_and_heavy_rows(spg):
    """Config 5 at its largest size (s23: nnz(C) 5.3e9, C 42 GB): full rpt against the oracle,
    the 16 heaviest C rows and 48 random rows value-checked."""
    A = synth.rmat(23).with_values("uniform", 7)
    A32 = A.astype(np.float32)
    with spg.Handle() as h:
        dA = _dev(spg, A32, np.float32)
        C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        rpt = C.rpt.cpu().numpy()
        assert np.array_equal(rpt, oracle.symbolic_omp(A32, A32)), "rpt differs from the oracle"
        _, total = oracle.nprod(A32, A32)
        assert h.nprod == total
        rng = np.random.default_rng(3)
        rows = np.concatenate([np.argsort(np.diff(rpt))[-16:], rng.integers(0, A.m, 48)])
        _sampled_rows_parity(C, A32, rows, 1e-5)


# ------------------------------------------------------------------ rank-indexed accumulation
# CTA-per-row numeric groups 4-9 accumulate at the rank of the column from a two-level bitmap of
# the row's span (kernels_rankacc.cu).  Fast path: <= TPR A non-zeros and
# <= 8*TPR products held in registers; slow path: chunked re-walks (QCD-like rows: 1521 products,
# 210 outputs, so products > 8*TPR in group 4).

def _rank_rows(st):
    return sum(st["num_rows"][g] for g in range(4, 10))


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("name", ["rmat14", "webbase_small", "mixed:qcd", "mixed:circuit"])
def test_rank_acc_vs_paper_hash(spg, name, dtype):
    A = _mixed_small() if name == "webbase_small" else (
        synth.rmat(14).with_values("uniform", 9) if name == "rmat14" else synth.config(name))
    got = check(spg, A, A, dtype, what=f"{name} rank_acc")
    st = got[3]
    if name != "mixed:circuit":
        assert _rank_rows(st) > 0, "no rows in the rank-accumulate groups"
    # kernel family per group (spgemm_kernel_t): rank for low-compression inputs, the paper hash
    # for the QCD-like rows (n_prod/nnz = 7.2), rank counts for symbolic groups 5-9 either way
    want = 1 if name == "mixed:qcd" else 2
    for g in range(3, 10):
        if st["num_rows"][g]:
            assert st["num_kernel"][g] == want, (g, st["num_kernel"])
    for g in range(5, 10):
        if st["sym_rows"][g]:
            assert st["sym_kernel"][g] == 2, (g, st["sym_kernel"])
    got = check(spg, A, A, dtype, opts={"rank_acc": 0}, what=f"{name} paper hash")
    assert all(k in (0, 1, 3, 4, 5, 7) for k in got[3]["num_kernel"][:13]), got[3]["num_kernel"]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rank_l1_pct_splits_groups(spg, dtype):
    """RANK_L1_PCT: the rank kernels run only for groups whose key bound B has 100*W <= v*B
    (W = n/1024 + 1 level-1 words); the groups below keep the paper hash, results unchanged."""
    A = synth.rmat(14).with_values("uniform", 9)
    w = A.n // 1024 + 1
    got = check(spg, A, A, dtype, opts={"rank_l1_pct": 1, "rank_l1_pct_sym": 1}, what="rank_l1_pct=1")
    st = got[3]
    num_bounds = [8, 16, 64, 128, 256, 512, 1024, 2048, 4096, 8192]
    sym_bounds = [16, 32, 128, 256, 512, 1024, 2048, 4096, 8192, 16384]
    seen = set()
    for g in range(3, 10):
        if st["num_rows"][g]:
            want = 2 if 100 * w <= num_bounds[g] else 1
            seen.add(want)
            assert st["num_kernel"][g] == want, (g, st["num_kernel"])
    for g in range(5, 10):
        if st["sym_rows"][g]:
            assert st["sym_kernel"][g] == (2 if 100 * w <= sym_bounds[g] else 1), (g, st["sym_kernel"])
    assert 1 in seen, "no CTA group fell back to the paper hash"


@pytest.mark.parametrize("name", ["rmat14", "mixed:qcd"])
def test_rank_acc_int_exact(spg, name):
    A = synth.rmat(14).with_values("int", 2) if name == "rmat14" else synth.config(name, "int")
    check(spg, A, A, np.float32, exact=True, what=f"{name} int")


def test_rank_acc_duplicates_and_unsorted(spg):
    # duplicate and unsorted columns inside B rows: equal keys share one rank (summed)
    rng = np.random.default_rng(21)
    m = 1500
    rows = np.repeat(np.arange(m), 200)
    cols = rng.integers(0, 200000, size=rows.size)
    dup = rng.random(rows.size) < 0.2
    cols[dup] = cols[np.maximum(np.arange(rows.size) - 1, 0)][dup]
    A = from_coo(m, 200000, rows, cols, rng.uniform(-1, 1, rows.size), dedup=False)
    B = from_coo(200000, 200000, rng.integers(0, 200000, 800000), rng.integers(0, 200000, 800000),
                 rng.uniform(-1, 1, 800000), dedup=False)
    for M in (A, B):  # shuffle the entries inside every row
        r = np.repeat(np.arange(M.m), np.diff(M.rpt))
        o = np.lexsort((rng.random(r.size), r))
        M.col[:] = M.col[o]
        M.val[:] = M.val[o]
    got = check(spg, A, B, np.float64, what="dup/unsorted rank_acc")
    assert _rank_rows(got[3]) > 0


def _big_rows(seed, m=240, k=1 << 17, n=1 << 21):
    """Rows of C with 9K-60K entries over a ~2M-column span (numeric groups 10-12)."""
    rng = np.random.default_rng(seed)
    la = rng.integers(400, 2500, size=m)
    rows = np.repeat(np.arange(m), la)
    A = from_coo(m, k, rows, rng.integers(0, k, size=rows.size))
    br = np.repeat(np.arange(k), 24)
    B = from_coo(k, n, br, rng.integers(0, n, size=br.size))
    return A, B


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rank_acc_big_rows(spg, dtype):
    A, B = _big_rows(31)
    A, B = A.with_values("uniform", 1), B.with_values("uniform", 2)
    got = check(spg, A, B, dtype, what="big rows rank")
    assert got[3]["num_rows"][10] > 0 and sum(got[3]["num_rows"][11:13]) > 0, "no rows above the CTA groups"
    check(spg, A, B, dtype, opts={"rank_big_shared": 0}, what="big rows rank, level 2 in global memory")
    check(spg, A, B, dtype, opts={"rank_big_shared": 2}, what="big rows rank, group 10 in registers, output in C")
    check(spg, A, B, dtype, opts={"rank_mid": 0}, what="big rows rank, group 9 one CTA per row")
    for mx in (0, 1, 2):  # groups >= 10 + mx on the DSMEM cluster tables, the rest rank-big (one slab)
        got = check(spg, A, B, dtype, opts={"rank_big_max": mx}, what=f"big rows rank_big_max={mx}")
        assert all(got[3]["num_kernel"][10 + c] in (0, 4 if c >= mx else 6) for c in range(3)), got[3]["num_kernel"]
    check(spg, A, B, dtype, opts={"rank_acc": 0}, what="big rows cluster")


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rank_count_big_rows_chunked(spg, dtype):
    """Symbolic rows above the last n_prod bound (group 10) counted exactly by the rank-count
    kernel: rows with more than 32768 non-empty 32-column blocks take level 2 in chunks; with
    RANK_BIG_SYM 0 the same rows go through the paper's optimistic -> cluster -> global chain."""
    A, B = _big_rows(33)
    A, B = A.with_values("uniform", 1), B.with_values("uniform", 2)
    # non-empty 32-column blocks per row of C (the chunking must be exercised)
    blocks = [np.unique(B.col[np.concatenate([np.arange(B.rpt[k], B.rpt[k + 1])
                                              for k in A.col[A.rpt[i]:A.rpt[i + 1]]])] >> 5).size
              for i in range(A.m)]
    assert max(blocks) > 32768, max(blocks)
    got = check(spg, A, B, dtype, opts={"rank_big_sym": 2}, what="big rows exact count")
    st = got[3]
    assert st["sym_rows"][10] > 0 and st["sym_kernel"][10] == 2, (st["sym_rows"][10], st["sym_kernel"])
    assert st["sym_overflow_rows"] == 0
    got = check(spg, A, B, dtype, opts={"rank_big_sym": 0}, what="big rows optimistic chain")
    assert got[3]["sym_kernel"][10] == 1 and got[3]["sym_overflow_rows"] > 0


def test_rank_count_rows_above_65535_blocks(spg):
    """Chunked big-row count on rows with more than 65535 non-empty 32-column blocks (n = 2^23:
    the level-1 prefix needs 32 bits; R-MAT s23's heaviest rows)."""
    rng = np.random.default_rng(34)
    m, k, n = 6, 1 << 17, 1 << 23
    la = rng.integers(4500, 5500, size=m)
    rows = np.repeat(np.arange(m), la)
    A = from_coo(m, k, rows, rng.integers(0, k, size=rows.size)).with_values("uniform", 1)
    br = np.repeat(np.arange(k), 24)
    B = from_coo(k, n, br, rng.integers(0, n, size=br.size)).with_values("uniform", 2)
    blocks = [np.unique(B.col[np.concatenate([np.arange(B.rpt[q], B.rpt[q + 1])
                                              for q in A.col[A.rpt[i]:A.rpt[i + 1]]])] >> 5).size
              for i in range(A.m)]
    assert min(blocks) > 65535, blocks
    got = check(spg, A, B, np.float32, opts={"rank_big_sym": 2}, what="rows above 65535 blocks")
    assert got[3]["sym_kernel"][10] == 2


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rank_mid_group9_rows(spg, dtype):
    """Numeric group 9 (4096 < nnz_i <= 8192): products in registers, output reduced into C,
    two CTAs per SM (RANK_MID 2, default); the persistent rank-big variant (1) and one CTA per row
    with the row in shared memory (0); all against the oracle."""
    rng = np.random.default_rng(35)
    m, k, n = 500, 1 << 17, 1 << 21
    la = rng.integers(180, 340, size=m)
    rows = np.repeat(np.arange(m), la)
    A = from_coo(m, k, rows, rng.integers(0, k, size=rows.size)).with_values("uniform", 1)
    br = np.repeat(np.arange(k), 24)
    B = from_coo(k, n, br, rng.integers(0, n, size=br.size)).with_values("uniform", 2)
    got = check(spg, A, B, dtype, what="group 9 registers, output reduced into C")
    assert got[3]["num_rows"][9] > 0 and got[3]["num_kernel"][9] == 2, (got[3]["num_rows"][9], got[3]["num_kernel"])
    got = check(spg, A, B, dtype, opts={"rank_mid": 1}, what="group 9 persistent rank-big")
    assert got[3]["num_kernel"][9] == 6
    got = check(spg, A, B, dtype, opts={"rank_mid": 0}, what="group 9 one CTA per row")
    assert got[3]["num_kernel"][9] == 2


@pytest.mark.parametrize("name", ["rmat14", "webbase_small"])
def test_rank_gout_groups(spg, name):
    """RANK_GOUT: rank groups 3-8 reduce into the row of C instead of a shared-memory row."""
    A = _mixed_small() if name == "webbase_small" else synth.rmat(14).with_values("uniform", 9)
    got = check(spg, A, A, np.float32, opts={"rank_gout": 1}, what=f"{name} rank_gout")
    assert _rank_rows(got[3]) > 0


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rank_big_groups_duplicates_unsorted(spg, dtype):
    """Numeric groups 9-10 (output reduced into C; level 2 in shared memory) and the chunked symbolic
    count on B rows with duplicate and unsorted columns: equal keys share one rank and are summed
    (reading R7); integer values, bit-exact."""
    rng = np.random.default_rng(36)
    m, k, n = 360, 1 << 16, 1 << 21
    la = np.where(np.arange(m) % 2 == 0, rng.integers(190, 330, size=m), rng.integers(450, 900, size=m))
    rows = np.repeat(np.arange(m), la)
    A = from_coo(m, k, rows, rng.integers(0, k, size=rows.size), rng.integers(-3, 4, rows.size).astype(float),
                 dedup=False)
    br = np.repeat(np.arange(k), 24)
    bc = rng.integers(0, n, size=br.size)
    dup = rng.random(br.size) < 0.2
    bc[dup] = bc[np.maximum(np.arange(br.size) - 1, 0)][dup]
    B = from_coo(k, n, br, bc, rng.integers(-3, 4, br.size).astype(float), dedup=False)
    r = np.repeat(np.arange(B.m), np.diff(B.rpt))
    o = np.lexsort((rng.random(r.size), r))
    B.col[:] = B.col[o]
    B.val[:] = B.val[o]
    for opts in ({}, {"rank_big_sym": 2, "rank_big_shared": 2}, {"rank_mid": 1}):
        got = check(spg, A, B, dtype, exact=True, opts=opts, what=f"dup/unsorted big groups {opts}")
        assert got[3]["num_rows"][9] > 0 and got[3]["num_rows"][10] > 0, got[3]["num_rows"]


def test_rank_acc_big_rows_int_exact(spg):
    A, B = _big_rows(32)
    check(spg, A.with_values("int", 3), B.with_values("int", 4), np.float32, exact=True, what="big rows int")


# ------------------------------------------------------------------ thread-per-row tiny rows
# symbolic groups 0-1 and numeric groups 0-1 (kernels_tiny.cu): sorted register tables

@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("name", ["mixed:epidemiology", "mixed:economics", "webbase_small", "poisson64"])
def test_tiny_rows_vs_paper_hash(spg, name, dtype):
    A = _mixed_small() if name == "webbase_small" else synth.config(name)
    got = check(spg, A, A, dtype, exact=(name == "poisson64"), what=f"{name} tiny")
    st = got[3]
    assert any(st["num_kernel"][g] == 7 for g in (0, 1) if st["num_rows"][g]) or name == "poisson64"
    for g in (0, 1):
        if st["num_rows"][g]:
            assert st["num_kernel"][g] == 7, st["num_kernel"]
    got = check(spg, A, A, dtype, opts={"tiny": 2}, what=f"{name} tiny symbolic too")
    for g in (0, 1):
        if got[3]["sym_rows"][g]:
            assert got[3]["sym_kernel"][g] == 7, got[3]["sym_kernel"]
    check(spg, A, A, dtype, opts={"tiny": 0}, what=f"{name} partial-warp hash")


def test_tiny_rows_int_exact_and_duplicates(spg):
    # duplicate columns inside A and B rows, unsorted: equal keys accumulate in one register slot
    rng = np.random.default_rng(41)
    m, n = 20000, 60000
    rows = rng.integers(0, m, 50000)
    A = from_coo(m, n, rows, rng.integers(0, n, rows.size), dedup=False).with_values("int", 5)
    B = from_coo(n, n, rng.integers(0, n, 90000), rng.integers(0, n, 90000), dedup=False).with_values("int", 6)
    for M in (A, B):
        r = np.repeat(np.arange(M.m), np.diff(M.rpt))
        o = np.lexsort((rng.random(r.size), r))
        M.col[:] = M.col[o]
        M.val[:] = M.val[o]
    got = check(spg, A, B, np.float32, exact=True, opts={"tiny": 2}, what="tiny dup int")
    assert got[3]["num_kernel"][0] == 7 and got[3]["sym_kernel"][0] == 7


# ------------------------------------------------------------------ batched kernels (kernels_esc.cu)
# Numeric ESC rows (expand, bucket, in-bucket rank, compress; one CTA per batch of rows of one
# symbolic group) and the batched paper-hash symbolic kernels.  ESC_GROUPS forces every symbolic
# group 2-8 onto ESC whatever the library's rule (which only picks them at R-MAT s22 scale).

ESC_ALL = sum(1 << g for g in range(2, 9))


def _esc_kernels(st):
    return [g for g in range(15, 22) if st["num_rows"][g]]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("name", ["rmat14", "rmat16", "webbase_small", "mixed:circuit", "mixed:economics"])
def test_esc_numeric(spg, name, dtype):
    A = _mixed_small() if name == "webbase_small" else (
        synth.rmat(int(name[4:])).with_values("uniform", 9) if name.startswith("rmat") else synth.config(name))
    got = check(spg, A, A, dtype, opts={"esc_groups": ESC_ALL}, what=f"{name} esc")
    st = got[3]
    groups = _esc_kernels(st)
    assert groups, "no rows took the ESC kernels"
    assert all(st["num_kernel"][g] == 9 for g in groups), st["num_kernel"]


@pytest.mark.parametrize("name", ["rmat14", "webbase_small"])
def test_esc_int_exact(spg, name):
    A = _mixed_small() if name == "webbase_small" else synth.rmat(14)
    A = A.with_values("int", 3)
    check(spg, A, A, np.float32, exact=True, opts={"esc_groups": ESC_ALL}, what=f"{name} esc int")


def test_esc_duplicates_unsorted_and_compression(spg):
    """Duplicate and unsorted columns inside A and B rows (equal keys: one entry, summed in the
    run), and ESC_PCT large enough to send compressing rows through ESC as well."""
    rng = np.random.default_rng(23)
    m, n = 3000, 50000
    rows = np.repeat(np.arange(m), 120)
    cols = rng.integers(0, n, size=rows.size)
    dup = rng.random(rows.size) < 0.3
    cols[dup] = cols[np.maximum(np.arange(rows.size) - 1, 0)][dup]
    A = from_coo(m, n, rows, cols, rng.uniform(-1, 1, rows.size), dedup=False)
    B = from_coo(n, n, rng.integers(0, n, 400000), rng.integers(0, 12000, 400000),  # column band wider
                 rng.uniform(-1, 1, 400000), dedup=False)                            # than range rows
    for M in (A, B):
        r = np.repeat(np.arange(M.m), np.diff(M.rpt))
        o = np.lexsort((rng.random(r.size), r))
        M.col[:] = M.col[o]
        M.val[:] = M.val[o]
    got = check(spg, A, B, np.float64, opts={"esc_groups": ESC_ALL, "esc_pct": 100000}, what="esc dup/unsorted")
    assert _esc_kernels(got[3])


@pytest.mark.parametrize("name", ["rmat16", "webbase_small", "mixed:qcd"])
def test_batched_symbolic(spg, name):
    """BATCH bit 1: symbolic groups 2-9 by the batched paper hash (Alg. 5 per row, rows of one
    group flattened over a CTA)."""
    A = _mixed_small() if name == "webbase_small" else (
        synth.rmat(16).with_values("uniform", 5) if name == "rmat16" else synth.config(name))
    got = check(spg, A, A, np.float32, opts={"batch": 3, "esc_groups": ESC_ALL}, what=f"{name} batched")
    st = got[3]
    assert any(st["sym_kernel"][g] == 8 for g in range(2, 10) if st["sym_rows"][g]), st["sym_kernel"]


def test_esc_auto_rule_off_below_scale(spg):
    """The library picks ESC only for wide matrices (n/1024 + 1 > 1024 level-1 words)."""
    A = synth.rmat(16).with_values("uniform", 4)
    got = check(spg, A, A, np.float32, what="rmat16 default")
    assert not _esc_kernels(got[3])


# ------------------------------------------------------------------ validation and graph keys

def test_validate_rejects_bad_input(spg):
    """SPGEMM_OPT_VALIDATE: an out-of-range column and a non-monotone rpt are reported as
    SPGEMM_ERR_INVALID_INPUT before any kernel reads through them (and the handle stays usable)."""
    A = synth.config("mixed:economics")
    good = _dev(spg, A, np.float32)
    with spg.Handle() as h:
        h.set_option("validate", 1)
        bad_col = spg.CsrMatrix(good.m, good.n, good.rpt.clone(), good.col.clone(), good.val)
        bad_col.col[5] = good.n + 1000
        with pytest.raises(spg.SpgemmError, match="INVALID_INPUT"):
            h.multiply(bad_col, good)
        bad_rpt = spg.CsrMatrix(good.m, good.n, good.rpt.clone(), good.col, good.val)
        bad_rpt.rpt[10] = bad_rpt.rpt[12] + 1
        with pytest.raises(spg.SpgemmError, match="INVALID_INPUT"):
            h.multiply(bad_rpt, good)
        torch.cuda.synchronize()
        C = h.multiply(good, good)
        ref = oracle.spgemm(A.astype(np.float32), A.astype(np.float32), np.float32)
        assert_parity(C.numpy() + (None,), ref, np.float32, what="after rejected inputs")


def test_graph_replay_new_structure_same_shape(spg):
    """Two different structures with the same m, n, nnz(C)-independent pointers through one handle
    (the numeric graph key includes max nnz_i and the global-table shape: ADVICE r1)."""
    A1 = _mixed_small()
    rng = np.random.default_rng(5)
    A2 = synth.webbase_like(M=30000, seed=9, lmax=2500, alpha=1.5).with_values("uniform", 2)
    with spg.Handle() as h:
        for it, A in enumerate((A1, A2, A1, A2)):
            h.set_option("num_min_group", 13 if it % 2 else -1)  # global group on odd calls
            ref = oracle.spgemm(A.astype(np.float32), A.astype(np.float32), np.float32)
            C = h.multiply(_dev(spg, A, np.float32), _dev(spg, A, np.float32))
            torch.cuda.synchronize()
            assert_parity(C.numpy() + (None,), ref, np.float32, what=f"call {it}")
            del C


@pytest.mark.parametrize("name", ["mixed:economics", "poisson64"])
def test_graph_cache_rotating_buffers(spg, name):
    """Several cached graphs per segment: five output-buffer sets (and two inputs) used in turn
    through one handle; the four most recent calls replay their own instantiated graphs, an older
    one is recycled (poisson64: the small-matrix path; economics: the grouped path)."""
    A = synth.config(name, "int").astype(np.float32)
    A2 = A.with_values("int", 11).astype(np.float32)
    refs = [oracle.spgemm(M, M, np.float32) for M in (A, A2)]
    with spg.Handle() as h:
        ins = [(_dev(spg, M, np.float32)) for M in (A, A2)]
        c_rpts = [torch.empty(A.m + 1, dtype=torch.int64, device="cuda") for _ in range(5)]
        outs = {}
        replays = 0
        for it in range(15):
            j = it % 5
            dA = ins[it % 2]
            c_rpt, nnz, _ = h.symbolic(dA, dA, c_rpt=c_rpts[j])
            if (j, it % 2) not in outs:
                outs[(j, it % 2)] = (torch.empty(nnz, dtype=torch.int32, device="cuda"),
                                     torch.empty(nnz, dtype=torch.float32, device="cuda"))
            c_col, c_val = outs[(j, it % 2)]
            h.numeric(dA.val, dA.val, c_col, c_val)
            torch.cuda.synchronize()
            got = (c_rpt.cpu().numpy(), c_col.cpu().numpy(), c_val.cpu().numpy(), None)
            assert_parity(got, refs[it % 2], np.float32, exact=True, what=f"call {it}")
            replays = h.stats()["graph_replays"]
        assert replays >= 1


# ------------------------------------------------------------------ Galerkin product R A P (f3)

def _galerkin_inputs(n):
    A = synth.poisson2d(n)
    P = synth.aggregation_prolongator(n, agg=2, smoothed=True, seed=3)
    return A, P, synth.transpose(P)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_galerkin_rap_chained(spg, dtype):
    """AMG's R A P as two chained rectangular multiplies through the ABI, the
    second reading the first's device output; both against the oracle."""
    A, Pm, R = _galerkin_inputs(96)
    AP_ref = oracle.spgemm(A.astype(dtype), Pm.astype(dtype), dtype)
    AP_h = Csr(A.m, Pm.n, AP_ref[0], AP_ref[1], AP_ref[2].astype(np.float64))
    RAP_ref = oracle.spgemm(R.astype(dtype), AP_h.astype(dtype), dtype)
    with spg.Handle() as h:
        AP = h.multiply(_dev(spg, A, dtype), _dev(spg, Pm, dtype))
        torch.cuda.synchronize()
        assert_parity(AP.numpy() + (None,), AP_ref, dtype, what="A P")
        # the oracle's second product starts from its own A P; compare structure exactly and
        # values within the tolerance of that product
        RAP = h.multiply(_dev(spg, R, dtype), AP)
        torch.cuda.synchronize()
        assert_parity(RAP.numpy() + (None,), RAP_ref, dtype, what="R (A P)")
        assert (RAP.m, RAP.n) == (Pm.n, Pm.n)


def test_numeric_rerun_new_values(spg):
    """Structure reuse: one symbolic phase, then numeric re-runs with new values
    of A and B (same structures) into the same C buffers; every run against the oracle."""
    A, Pm, _ = _galerkin_inputs(64)
    with spg.Handle() as h:
        dA, dP = _dev(spg, A, np.float64), _dev(spg, Pm, np.float64)
        c_rpt, nnz, _ = h.symbolic(dA, dP)
        c_col = torch.empty(nnz, dtype=torch.int32, device="cuda")
        c_val = torch.empty(nnz, dtype=torch.float64, device="cuda")
        for seed in range(3):
            A2 = A.with_values("int", 10 + seed)
            P2 = Pm.with_values("int", 20 + seed)
            h.numeric(torch.from_numpy(A2.val).cuda(), torch.from_numpy(P2.val).cuda(), c_col, c_val)
            torch.cuda.synchronize()
            ref = oracle.spgemm(A2, P2, np.float64)
            got = (c_rpt.cpu().numpy(), c_col.cpu().numpy(), c_val.cpu().numpy())
            assert_parity(got + (None,), ref, np.float64, exact=True, what=f"re-run {seed}")


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("name", ["rmat14", "webbase_small", "mixed:circuit"])
def test_warp_sorted_rows(spg, name, dtype):
    """WSORT ablation (kernels_wsort.cu): symbolic groups 2-5 count the distinct columns of a
    bitonic-sorted register row; numeric rows of those groups are sorted, summed and compacted in
    registers / warp-private shared memory."""
    A = _mixed_small() if name == "webbase_small" else (
        synth.rmat(14).with_values("uniform", 9) if name == "rmat14" else synth.config(name))
    got = check(spg, A, A, dtype, opts={"wsort": 3}, what=f"{name} wsort")
    st = got[3]
    assert any(st["sym_kernel"][g] == 10 for g in range(2, 6) if st["sym_rows"][g]), st["sym_kernel"]
    assert any(st["num_kernel"][g] == 10 for g in range(15, 19) if st["num_rows"][g]), st["num_kernel"]
