"""GPU parity of ls_solve_refined and orthogonalize (C-ABI) against the fp64 oracle (-m gpu).

Tolerances (north_star): refined LS ||x - x*||/||x*|| <= 1e-5 for cond <= 1e4 (x* = the
oracle's solution of the fp32-rounded problem); orthogonality <= 1e-5 after
reorthogonalisation.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rg():
    import paper_conf_hpdc_zhangbw20_b200 as rg
    return rg


def _dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()


@pytest.mark.parametrize("kind,kappa", [("geometric", 1e2), ("geometric", 1e4), ("arithmetic", 1e4),
                                        ("cluster", 1e4)])
@pytest.mark.parametrize("consistent", [False, True])
def test_ls_refined_parity(rg, kind, kappa, consistent):
    m, n = 8192, 256
    A = synth.svd_matrix(m, n, kind, kappa, seed=31).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=31, consistent=consistent).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    x = torch.zeros(n, dtype=torch.float64, device="cuda")
    x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), x, tol=1e-10, maxit=200)
    xe = x.cpu().numpy()
    fe = np.linalg.norm(xe - x_star) / np.linalg.norm(x_star)
    assert st == rg.RG_OK, (st, it, rel)
    assert fe <= 1e-5, (fe, it)
    assert it <= 60   # reortho'd R: kappa(A R^-1) ~ 1 (reading #8; SURVEY [EMU] ~10-18)


def test_ls_refined_4x2_closed_form(rg):
    A = np.array([[1, 1], [1, 2], [1, 3], [1, 4]], dtype=np.float32)
    b = np.array([1, 3, 2, 5], dtype=np.float32)
    x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), tol=1e-13)
    np.testing.assert_allclose(x.cpu().numpy(), [0.0, 1.1], atol=1e-9)


def test_ls_host_pointers(rg):
    A = np.asfortranarray(synth.svd_matrix(4096, 64, "geometric", 1e3, seed=2).astype(np.float32))
    b = synth.rhs(A.astype(np.float64), seed=2, consistent=False).astype(np.float32)
    x = np.zeros(64)
    x, it, rel, st = rg.ls_solve_refined(A, b, x)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    assert np.linalg.norm(x - x_star) / np.linalg.norm(x_star) <= 1e-5


def test_ls_paper_faithful_mode_converges(rg):
    """Paper-faithful preconditioner (reortho = 0 and the paper's fp32 TSQR/MGS panel, eq 8 +
    Alg 2; reading #26) against a reortho pass (CholQR2 panels) and the default (one split-precision
    pass, reading #8): all reach the
    LS solution (Alg 3), and the reorthogonalised R needs no more CGLS iterations than the
    one-pass R (the one-pass preconditioner is what makes the paper's kappa = 1e4
    geometric case slow)."""
    A = synth.svd_matrix(8192, 128, "geometric", 1e4, seed=5).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=5, consistent=True).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    iters = {}
    for name, o in (("faithful", rg.make_opts(reortho=0, panel="mgs")), ("one-pass", rg.make_opts(reortho=0)),
                    ("reortho", rg.make_opts(reortho=1)), ("default", rg.make_opts())):
        x, it, _, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), opts=o, maxit=400)
        assert st == rg.RG_OK, (name, it, st)
        xv = x.cpu().numpy()
        assert np.linalg.norm(xv - x_star) / np.linalg.norm(x_star) <= 1e-5, name
        iters[name] = it
    # measured (B200, round 2): faithful 48, one-pass 8, reortho 15.  The one-pass R of the
    # default panels is not the paper's: at n = 128 the whole factorization is two 64-column
    # CholQR2 leaves with fp64 Grams and one 16-bit level, so it is nearly fp32-accurate and can
    # beat R2 R1 (whose R2 carries a full 16-bit pass); only the paper's configuration is compared.
    assert iters["reortho"] <= iters["faithful"], iters
    assert iters["reortho"] <= 30, iters
    # the default preconditioner (one split-precision pass, reading #8) is at least as good as the
    # 16-bit pass + reortho pass (config 3: 8 vs 19 iterations)
    assert iters["default"] <= iters["reortho"], iters


@pytest.mark.parametrize("kappa", [1.0, 1e3, 1e4])
def test_orthogonalize_parity(rg, kappa):
    m, n = 16384, 256
    A = (synth.gaussian(m, n, seed=7) if kappa == 1.0 else
         synth.svd_matrix(m, n, "geometric", kappa, seed=7)).astype(np.float32)
    Ad = _dev(A)
    R = torch.zeros(n, n, device="cuda").t()
    Q, R, passes, est = rg.orthogonalize(Ad, R, orth_tol=1e-5, max_passes=3)
    Qn = Q.cpu().numpy().astype(np.float64)
    orth = oracle.orthogonality(Qn)
    assert orth <= 1e-5, (orth, passes, est)
    be = oracle.backward_error(A.astype(np.float64), Qn, R.cpu().numpy().astype(np.float64))
    assert be <= 5e-3
    assert 1 <= passes <= 3
    assert abs(est - orth) <= 0.5 * orth + 1e-7   # Hutchinson estimate is close


def test_orthogonalize_fixed_two_passes(rg):
    A = synth.gaussian(2 ** 16, 256, seed=8).astype(np.float32)
    Ad = _dev(A)
    Q, _, passes, est = rg.orthogonalize(Ad, None, orth_tol=0.0, max_passes=2)
    assert passes == 2
    assert oracle.orthogonality(Q.cpu().numpy().astype(np.float64)) <= 1e-5


@pytest.mark.parametrize("solver", ["cgls", "lsqr"])
@pytest.mark.parametrize("m,n,kappa", [(16384, 512, 1e2), (16384, 512, 1e4), (12300, 1000, 1e4)])
def test_ls_one_pass_cgls_matches_two_pass(rg, monkeypatch, m, n, kappa, solver):
    """The one-pass product (q = A t and A^T q in one sweep of A; A^T r, for LSQR A^T u, by
    recurrence) and the two-pass form (recomputed from r / u, RGSQR_CGLS_TWO_PASS=1) reach the same
    solution (reading #24).  12300 x 1000: a ragged 64-row tail block."""
    A = synth.svd_matrix(m, n, "geometric", kappa, seed=61).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=61, consistent=False).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    out = []
    for two in (False, True):
        if two:
            monkeypatch.setenv("RGSQR_CGLS_TWO_PASS", "1")
        else:
            monkeypatch.delenv("RGSQR_CGLS_TWO_PASS", raising=False)
        h = rg.Handle(0)   # fresh handle: its captured CGLS graph follows the current mode
        x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), tol=1e-10, maxit=200, handle=h,
                                             opts=rg.make_opts(solver=solver))
        torch.cuda.synchronize()
        out.append((x.cpu().numpy(), it, rel, st))
        h.close()
    (x1, it1, _, st1), (x2, it2, _, st2) = out
    assert st1 == rg.RG_OK and st2 == rg.RG_OK
    assert abs(it1 - it2) <= 2, (it1, it2)
    assert np.linalg.norm(x1 - x2) / np.linalg.norm(x2) <= 1e-8
    assert np.linalg.norm(x1 - x_star) / np.linalg.norm(x_star) <= 1e-5


@pytest.mark.parametrize("m,n", [(60, 13), (64, 1), (100, 7), (1028, 64), (4100, 1000)])
def test_ls_one_pass_cgls_edges(rg, m, n):
    """Edge shapes of the one-pass product's 64-row blocks (reading #24): a single partial block,
    one column, exact and ragged block counts, n near the kernel's 1024-column limit; every lda
    a multiple of 4 so the one-pass form is the one taken."""
    A = synth.svd_matrix(m, n, "geometric", 1e3, seed=71 + n).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=71 + n, consistent=False).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), tol=1e-12, maxit=200)
    assert st == rg.RG_OK, (st, it, rel)
    xe = x.cpu().numpy()
    assert np.linalg.norm(xe - x_star) / np.linalg.norm(x_star) <= 1e-5, it


@pytest.mark.parametrize("kind,kappa", [("geometric", 1e2), ("geometric", 1e4), ("arithmetic", 1e4)])
@pytest.mark.parametrize("consistent", [False, True])
def test_ls_lsqr_parity(rg, kind, kappa, consistent):
    """NEXT-4: LSQR (opts.solver = 1) on the same R-preconditioned operator reaches the oracle's LS
    solution to the north_star tolerance, in about as many iterations as CGLS (the two are
    mathematically equivalent Krylov methods on M = A R^-1)."""
    m, n = 8192, 256
    A = synth.svd_matrix(m, n, kind, kappa, seed=37).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=37, consistent=consistent).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    out = {}
    for solver in ("cgls", "lsqr"):
        x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), tol=1e-10, maxit=200,
                                             opts=rg.make_opts(solver=solver))
        assert st == rg.RG_OK, (solver, it, rel, st)
        xe = x.cpu().numpy()
        fe = np.linalg.norm(xe - x_star) / np.linalg.norm(x_star)
        assert fe <= 1e-5, (solver, fe, it)
        out[solver] = (it, xe)
    assert abs(out["lsqr"][0] - out["cgls"][0]) <= 3, out
    assert np.linalg.norm(out["lsqr"][1] - out["cgls"][1]) / np.linalg.norm(x_star) <= 1e-7


def test_ls_lsqr_4x2_closed_form(rg):
    A = np.array([[1, 1], [1, 2], [1, 3], [1, 4]], dtype=np.float32)
    b = np.array([1, 3, 2, 5], dtype=np.float32)
    x, it, rel, st = rg.ls_solve_refined(_dev(A), torch.from_numpy(b).cuda(), tol=1e-13,
                                         opts=rg.make_opts(solver="lsqr"))
    np.testing.assert_allclose(x.cpu().numpy(), [0.0, 1.1], atol=1e-9)
