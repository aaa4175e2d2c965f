"""Pins for the fp64 oracle (-m "not gpu").

Every check ties the oracle to something other than itself: the hand-derived
4x2 closed form, the paper's printed Table 4, Random123's Philox vectors,
closed forms (eq 5 flops, n = 1, orthonormal and Q0*D inputs), LAPACK via
numpy (an independent implementation), mathematical identities, and brute
force agreement between independently written algorithms.
"""
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden_rows(name):
    rows = []
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def _ls_fixture():
    d = {r[0]: np.array([float(v) for v in r[1:]]) for r in _golden_rows("ls_4x2.txt")}
    A = d["A"].reshape(4, 2)  # listed row by row
    return A, d


ALL_QR = [oracle.cgs, oracle.mgs, oracle.householder,
          lambda A: oracle.tsqr(A, tile=8), lambda A: oracle.rgsqr(A, nb=1, tile=4)]


# ---------------------------------------------------------------- closed forms

@pytest.mark.parametrize("qr", ALL_QR)
def test_4x2_closed_form(qr):
    A, d = _ls_fixture()
    Q, R, s = qr(A)
    assert s == 0
    np.testing.assert_allclose(R, np.array([[d["R"][0], d["R"][1]], [d["R"][2], d["R"][3]]]), atol=1e-14)
    np.testing.assert_allclose(Q[:, 0], d["Q1"], atol=1e-14)
    np.testing.assert_allclose(Q[:, 1], d["Q2"], atol=1e-14)


def test_4x2_least_squares():
    A, d = _ls_fixture()
    for solver in (oracle.ls_normal, oracle.ls_qr):
        x, s = solver(A, d["b"])
        assert s == 0
        np.testing.assert_allclose(x, d["x"], atol=1e-13)
        r = d["b"] - A @ x
        np.testing.assert_allclose(r, d["r"], atol=1e-13)
        assert abs(r @ r - d["rr"][0]) < 1e-12
    # CGLS preconditioned by the exact R converges in one iteration
    _, R, _ = oracle.householder(A)
    x, it, _ = oracle.cgls(A, d["b"], R, tol=1e-12, maxit=10)
    np.testing.assert_allclose(x, d["x"], atol=1e-12)
    assert it <= 2


@pytest.mark.parametrize("qr", ALL_QR)
def test_single_column(qr):
    a = synth.gaussian(37, 1, seed=3)
    Q, R, s = qr(a)
    assert s == 0
    nrm = np.sqrt(np.sum(a[:, 0] ** 2))
    assert abs(R[0, 0] - nrm) <= 1e-14 * nrm
    np.testing.assert_allclose(Q[:, 0], a[:, 0] / nrm, atol=1e-15)


@pytest.mark.parametrize("qr", ALL_QR)
def test_orthonormal_times_diagonal(qr):
    """A = Q0 D with D > 0 diagonal has the QR factors Q0, D (uniqueness)."""
    g = synth.rng(11)
    Q0 = synth.haar(50, 7, g)
    D = np.diag(2.0 ** g.integers(-6, 7, size=7).astype(float))
    Q, R, s = qr(Q0 @ D)
    assert s == 0
    np.testing.assert_allclose(R, D, atol=1e-12 * D.max())
    np.testing.assert_allclose(Q, Q0, atol=1e-12)
    Q, R, _ = qr(Q0)
    np.testing.assert_allclose(R, np.eye(7), atol=1e-13)


# ------------------------------------------------------- brute force / identities

@pytest.mark.parametrize("m,n", [(5, 1), (6, 3), (17, 5), (33, 16), (64, 16), (40, 13), (9, 9)])
def test_qr_identities_and_agreement(m, n):
    A = synth.gaussian(m, n, seed=m * 100 + n)
    ref_Q, ref_R = np.linalg.qr(A)  # LAPACK, an independent implementation
    d = np.sign(np.diag(ref_R))
    ref_Q, ref_R = ref_Q * d, (ref_R.T * d).T
    kappa = np.linalg.cond(A)
    for qr in ALL_QR + [lambda A: oracle.tsqr(A, tile=max(n, 4)), lambda A: oracle.rgsqr(A, nb=2, tile=n)]:
        Q, R, s = qr(A)
        assert s == 0
        assert np.all(np.tril(R, -1) == 0.0)
        assert np.all(np.diag(R) > 0)
        assert oracle.backward_error(A, Q, R) < 1e-14
        tol = 1e-13 * kappa ** 2
        assert oracle.orthogonality(Q) < tol
        np.testing.assert_allclose(R, ref_R, atol=tol * np.abs(ref_R).max())
        np.testing.assert_allclose(Q, ref_Q, atol=tol)


@pytest.mark.parametrize("m,n,nb,tile", [(300, 40, 8, 32), (1000, 64, 32, 256), (257, 33, 32, 64),
                                         (129, 96, 16, 100)])
def test_rgsqr_and_tsqr_match_householder(m, n, nb, tile):
    """Alg 1 with the eq-8 panel reaches the unique QR (same as Householder)."""
    A = synth.svd_matrix(m, n, "geometric", 1e3, seed=5 + m)
    Qh, Rh, _ = oracle.householder(A)
    Q, R, s = oracle.rgsqr(A, nb=nb, tile=tile)
    assert s == 0
    np.testing.assert_allclose(R, Rh, atol=1e-11)
    np.testing.assert_allclose(Q, Qh, atol=1e-10)
    Q, R, s = oracle.tsqr(A, tile=tile)
    np.testing.assert_allclose(R, Rh, atol=1e-11)
    np.testing.assert_allclose(Q, Qh, atol=1e-10)


def test_cgs_loses_more_orthogonality_than_mgs():
    """Known behaviour: CGS ~ kappa^2 u, MGS ~ kappa u, Householder ~ u."""
    A = synth.svd_matrix(400, 30, "geometric", 1e6, seed=9)
    o_c = oracle.orthogonality(oracle.cgs(A)[0])
    o_m = oracle.orthogonality(oracle.mgs(A)[0])
    o_h = oracle.orthogonality(oracle.householder(A)[0])
    assert o_h < 1e-13
    assert o_h < o_m < o_c
    assert o_m < 1e-6  # ~ kappa * u
    for qr in (oracle.cgs, oracle.mgs, oracle.householder):
        Q, R, _ = qr(A)
        assert oracle.backward_error(A, Q, R) < 1e-14  # independent of kappa


# ----------------------------------------------------------------- flop count

@pytest.mark.parametrize("m,n,nb", [(32768, 16384, 128), (65536, 4096, 32), (1000, 256, 32), (77, 128, 128)])
def test_eq5_flops_closed_form(m, n, nb):
    """eq 5 solves to exactly 2 m n^2 when n = nb * 2^k."""
    assert oracle.rgsqr_flops(m, n, nb) == 2.0 * m * n * n


def test_split_rule():
    for n in range(2, 700):
        h = oracle.rgsqr_split(n)
        assert 1 <= h < n
        if n >= 64:
            assert h % 32 == 0 and abs(h - n / 2) < 32


# -------------------------------------------------------------- least squares

@pytest.mark.parametrize("kappa", [1e1, 1e3, 1e4])
def test_ls_solvers_agree(kappa):
    A = synth.svd_matrix(600, 40, "geometric", kappa, seed=21)
    b = synth.rhs(A, seed=21, consistent=False)
    x_np = np.linalg.lstsq(A, b, rcond=None)[0]
    x_qr, _ = oracle.ls_qr(A, b)
    x_ne, _ = oracle.ls_normal(A, b)
    assert np.linalg.norm(x_qr - x_np) / np.linalg.norm(x_np) < 1e-15 * kappa * 100
    assert np.linalg.norm(x_ne - x_np) / np.linalg.norm(x_np) < 1e-15 * kappa ** 2 * 100
    _, R, _ = oracle.householder(A)
    x_cg, it, rel = oracle.cgls(A, b, R, tol=1e-12, maxit=50)
    assert it <= 3  # exact R: kappa(A R^-1) = 1
    assert np.linalg.norm(x_cg - x_np) / np.linalg.norm(x_np) < 1e-15 * kappa * 100


def test_cgls_rate_with_perturbed_preconditioner():
    """Imperfect R -> more iterations, bounded by the linear rate of P:L310."""
    A = synth.svd_matrix(500, 30, "geometric", 1e3, seed=4)
    b = synth.rhs(A, seed=4, consistent=True)
    x_star = np.linalg.lstsq(A, b, rcond=None)[0]
    _, R, _ = oracle.householder(A)
    g = synth.rng(8)
    Rp = R * (1 + 0.05 * np.triu(g.standard_normal(R.shape)))
    k = np.linalg.cond(A @ np.linalg.inv(Rp))
    x, it, rel = oracle.cgls(A, b, Rp, tol=1e-13, maxit=200)
    assert 2 < it <= 200
    assert np.linalg.norm(x - x_star) / np.linalg.norm(x_star) < 1e-9
    # CG bound on the energy norm: iterations to reduce by 1e-13 <= ln(2/1e-13) * sqrt(k)/2 + 1
    assert it <= np.log(2 / 1e-13) * np.sqrt(k) / 2 + 2
    # no preconditioner (R = I) is plain CGLS and needs many more iterations
    _, it_plain, _ = oracle.cgls(A, b, np.eye(30), tol=1e-13, maxit=500)
    assert it_plain > it


# ----------------------------------------------------------------- metrics

def test_metrics_closed_forms():
    g = synth.rng(2)
    Q0 = synth.haar(80, 6, g)
    eps = 1e-3
    Q = Q0.copy()
    Q[:, 2] *= 1 + eps
    # I - Q^T Q has the single nonzero entry 1 - (1+eps)^2
    assert abs(oracle.orthogonality(Q) - abs(1 - (1 + eps) ** 2)) < 1e-15
    R = np.triu(g.standard_normal((6, 6)))
    A = Q0 @ R
    # A - Q R = -eps * q_2 r_2^T  -> ||.||_F = eps * ||r_2|| (row 2 of R)
    be = oracle.backward_error(A, Q, R)
    assert abs(be - eps * np.linalg.norm(R[2]) / np.linalg.norm(A)) < 1e-14
    G = synth.probes(6, 400, seed=1)
    assert abs(oracle.backward_error_probe(A, Q, R, G) / be - 1) < 0.15
    assert abs(oracle.orthogonality_probe(Q, G) / oracle.orthogonality(Q) - 1) < 0.15


# -------------------------------------------------------------- SVD / low rank

def test_jacobi_svd_against_lapack():
    A = synth.gaussian(40, 25, seed=77)
    U, S, V, sweeps = oracle.svd_jacobi(A)
    np.testing.assert_allclose(S, np.linalg.svd(A, compute_uv=False), rtol=1e-13)
    np.testing.assert_allclose(U @ np.diag(S) @ V.T, A, atol=1e-13)
    np.testing.assert_allclose(V.T @ V, np.eye(25), atol=1e-13)
    D = np.diag([3.0, 1.0, 2.0])
    _, S, _, _ = oracle.svd_jacobi(D)
    np.testing.assert_allclose(S, [3.0, 2.0, 1.0])


def test_table4_closed_form_reproduces_paper():
    """Table 4's printed errors are the Eckart-Young optimum for the
    arithmetic spectrum with cond 1e6 and n = 1024 -- pins synth.sigma('arithmetic')
    and the Frobenius reading of the metric (reading #12)."""
    s = synth.sigma(1024, "arithmetic", 1e6)
    for r, printed, _ in _golden_rows("table4_lowrank.txt"):
        r = int(r)
        opt = np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2))
        assert f"{opt:.2e}" == printed


def test_qr_svd_lowrank_is_optimal_small():
    """QR-SVD (section 3.4) on a scaled Table-4 workload reaches the closed-form optimum."""
    m, n = 2048, 128
    A = synth.svd_matrix(m, n, "arithmetic", 1e6, seed=31)
    s = synth.sigma(n, "arithmetic", 1e6)
    Q, R, _ = oracle.householder(A)
    Ub, S, Vb, _ = oracle.svd_jacobi(R)
    np.testing.assert_allclose(S, s, rtol=1e-10)
    for r in (2, 8, 16, 32, 64):
        U = Q @ Ub[:, :r]
        err = oracle.lowrank_error(A, U, S[:r], Vb[:, :r])
        opt = np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2))
        assert abs(err - opt) < 1e-10


def test_randomized_lowrank_full_sketch_is_exact_optimum():
    m, n, r = 300, 60, 10
    A = synth.svd_matrix(m, n, "geometric", 1e4, seed=12)
    s = synth.sigma(n, "geometric", 1e4)
    Om = oracle.gaussian_philox(n, n, seed=99)
    U, S, V, st = oracle.lowrank(A, r, n - r, 0, Om)
    assert st == 0
    opt = np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2))
    assert abs(oracle.lowrank_error(A, U, S, V) - opt) < 1e-10
    np.testing.assert_allclose(S, s[:r], rtol=1e-9)
    # small oversampling + one power iteration is near-optimal (reading #17)
    Om = oracle.gaussian_philox(n, r + 8, seed=5)
    U, S, V, _ = oracle.lowrank(A, r, 8, 1, Om)
    assert oracle.lowrank_error(A, U, S, V) / opt < 1.1


# ----------------------------------------------------------------- generators

def test_philox_known_answers():
    for row in _golden_rows("philox_kat.txt"):
        v = [int(x, 16) for x in row]
        assert oracle.philox4x32_10(v[0:4], v[4:6]) == v[6:10]


def test_gaussian_philox_moments_and_determinism():
    Z = oracle.gaussian_philox(500, 40, seed=123)
    assert abs(Z.mean()) < 0.02 and abs(Z.var() - 1) < 0.03
    np.testing.assert_array_equal(Z, oracle.gaussian_philox(500, 40, seed=123))
    assert not np.array_equal(Z, oracle.gaussian_philox(500, 40, seed=124))


def test_generator_spectra():
    for kind in ("geometric", "arithmetic", "cluster"):
        A = synth.svd_matrix(200, 20, kind, 1e4, seed=1)
        np.testing.assert_allclose(np.linalg.svd(A, compute_uv=False), synth.sigma(20, kind, 1e4), rtol=1e-12)


def test_gaussian_philox_box_muller_mapping():
    """The word -> Gaussian mapping of the sketch stream (reading #17) pinned
    against the KAT-pinned Philox words: element e takes call e >> 1 with counter
    {e >> 1, 0, 0, 0} and key {seed lo, seed hi}; even e uses words (0, 1), odd e words (2, 3);
    u1 = (w_a + 1) 2^-32 in (0, 1], u2 = w_b 2^-32, z = sqrt(-2 ln u1) cos(2 pi u2).  A swapped
    word pair, a dropped +1 (ln 0 at w_a = 0), a column-major / row-major mix-up of the (rows x
    cols) fill or a 2^-31 scale all fail here."""
    seed = 0x1234_5678_9ABC_DEF0
    rows, cols = 37, 3
    Z = oracle.gaussian_philox(rows, cols, seed)
    flat = Z.reshape(-1, order="F")
    for e in range(rows * cols):
        w = oracle.philox4x32_10([e >> 1, 0, 0, 0], [seed & 0xFFFFFFFF, seed >> 32])
        a, b = (w[0], w[1]) if e % 2 == 0 else (w[2], w[3])
        u1 = (a + 1.0) * 2.0 ** -32
        u2 = b * 2.0 ** -32
        z = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
        assert abs(flat[e] - z) <= 4e-16 * max(1.0, abs(z)), (e, flat[e], z)
    # the stream does not depend on the shape it is read into (element index = e)
    np.testing.assert_array_equal(oracle.gaussian_philox(rows * cols, 1, seed)[:, 0], flat)
