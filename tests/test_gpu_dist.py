"""The library's OWN row-sharded code path (the row split of eq 8) run on
one GPU with in-process virtual ranks (rg_vgroup_create / rg_set_vcomm), against the fp64 oracle
(-m gpu).

Every rank is a separate rg_handle on its own CUDA stream, called from its own host thread; the
collectives (column-norm allreduce, K1 block allreduce + finish, CholQR Gram allreduce, TSQR
allgather + stack, CGLS scalar / vector allreduces, low-rank projection allreduce) go through
librgsqr's `dist` branches exactly as with NCCL, with a deterministic fixed-rank-order reduction
on the device.  Checks: the north_star tolerances against the oracle on the gathered result, R /
x / S replicated bit-identically on every rank, and P-invariance against the single-GPU call
(SURVEY 8(c) "Multi-GPU: P-invariance").
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


def _cuts(m, P):
    """Uneven contiguous row blocks (the ABI allows any split with sum m_local = m)."""
    w = np.linspace(1.0, 1.6, P)
    c = np.concatenate([[0], np.cumsum(w / w.sum() * m)]).round().astype(int)
    c[-1] = m
    return c


class Ranks:
    """P handles on cuda:0, each with its own non-blocking stream, attached to one virtual group."""

    def __init__(self, rg, P):
        self.rg = rg
        self.P = P
        self.group = rg.VGroup(P)
        self.streams = [torch.cuda.Stream() for _ in range(P)]
        self.h = [rg.Handle(0, stream=s.cuda_stream) for s in self.streams]
        for r, h in enumerate(self.h):
            h.set_vcomm(self.group, r)

    def run(self, fns):
        torch.cuda.synchronize()
        out = self.rg.run_ranks(fns)
        torch.cuda.synchronize()
        return out

    def close(self):
        for h in self.h:
            h.close()
        self.group.close()


@pytest.fixture(params=[2, 4], ids=["P2", "P4"])
def ranks(rg, request):
    R = Ranks(rg, request.param)
    yield R
    R.close()


def _dist_factor(rg, ranks, A, **kw):
    P = ranks.P
    m, n = A.shape
    c = _cuts(m, P)
    blocks = [_dev(A[c[r]:c[r + 1]]) for r in range(P)]
    Qs = [torch.zeros(n, c[r + 1] - c[r], device="cuda").t() for r in range(P)]
    Rs = [torch.zeros(n, n, device="cuda").t() for r in range(P)]
    o = rg.make_opts(**kw)
    ranks.run([lambda r=r: rg.rgsqr_factor(blocks[r], Q=Qs[r], R=Rs[r], handle=ranks.h[r], opts=o)
               for r in range(P)])
    Q = np.vstack([q.cpu().numpy() for q in Qs]).astype(np.float64)
    Rl = [x.cpu().numpy() for x in Rs]
    for r in range(1, P):   # replicated, bit for bit (fixed-order reductions on every rank)
        np.testing.assert_array_equal(Rl[r], Rl[0])
    return Q, Rl[0].astype(np.float64)


def _check_against_oracle(A, Q, R, kappa, orth_scale=1e-2):
    A64 = A.astype(np.float64)
    n = A.shape[1]
    assert np.all(np.tril(R, -1) == 0) and np.all(np.diag(R) > 0)
    be = oracle.backward_error(A64, Q, R)
    orth = oracle.orthogonality(Q)
    assert be <= 5e-3, be
    assert orth <= orth_scale * np.sqrt(n), orth
    Qo, Ro, _ = oracle.householder(A64)
    dr = np.linalg.norm(R - Ro) / np.linalg.norm(Ro)
    dq = np.linalg.norm(Q - Qo) / np.linalg.norm(Qo)
    # first-order perturbation of the unique factors (DESIGN reading #25)
    bound = max(10 * kappa * (be + orth / np.sqrt(n)), 1e-5)
    assert dr <= bound and dq <= bound, (dr, dq, be, orth)
    return be, orth


@pytest.mark.parametrize("panel", ["auto", "mgs"])
@pytest.mark.parametrize("m,n,kappa", [(6000, 160, None), (9000, 96, 1e2), (3000, 33, None)])
def test_dist_rgsqr_factor(rg, ranks, panel, m, n, kappa):
    """rgsqr_factor through the row-sharded branches: column-norm allreduce, K1 allreduce +
    proj_finish, and per panel either the streaming CholQR2 with the Gram allreduce (auto) or the
    local TSQR + allgather + stacked MGS + apply (mgs, eq 8 at GPU granularity)."""
    A = (synth.gaussian(m, n, seed=101 + n) if kappa is None else
         synth.svd_matrix(m, n, "geometric", kappa, seed=101 + n)).astype(np.float32)
    k = np.linalg.cond(A.astype(np.float64)) if kappa is None else kappa
    Q, R = _dist_factor(rg, ranks, A, panel=panel)
    _check_against_oracle(A, Q, R, k)
    # P-invariance: the single-GPU call (its own kernels: leaf / fused panels) gives the same
    # unique factors to the first-order bound
    Q1, R1 = rg.rgsqr_factor(_dev(A), opts=rg.make_opts(panel=panel))
    torch.cuda.synchronize()
    R1 = R1.cpu().numpy().astype(np.float64)
    Q1 = Q1.cpu().numpy().astype(np.float64)
    be = oracle.backward_error(A.astype(np.float64), Q1, R1)
    assert np.linalg.norm(R - R1) / np.linalg.norm(R1) <= max(20 * k * (be + 1e-3), 1e-4)


def test_dist_rgsqr_split_precision(rg, ranks):
    """split = 1 (3 x 16-bit K1 / K2, reading #9) through the sharded K1 allreduce of the lo
    and hi products: the factorization is fp32-accurate."""
    A = synth.gaussian(5000, 128, seed=7).astype(np.float32)
    Q, R = _dist_factor(rg, ranks, A, split=True)
    be, orth = _check_against_oracle(A, Q, R, np.linalg.cond(A.astype(np.float64)))
    assert be <= 1e-5 and orth <= 1e-4, (be, orth)


def test_dist_breakdown_reported_on_every_rank(rg, ranks):
    """A zero column fails the CholQR pivot on every rank (the reduced Gram is replicated); the
    guarded TSQR fallback runs its allgather on every rank and reports RG_BREAKDOWN everywhere."""
    A = synth.gaussian(4000, 70, seed=9).astype(np.float32)
    A[:, 45] = 0.0
    P = ranks.P
    c = _cuts(4000, P)
    blocks = [_dev(A[c[r]:c[r + 1]]) for r in range(P)]

    def call(r):
        try:
            rg.rgsqr_factor(blocks[r], handle=ranks.h[r])
        except rg.RGError as e:
            return e.status, e.info
        return 0, -1

    out = ranks.run([lambda r=r: call(r) for r in range(P)])
    assert all(st == rg.RG_BREAKDOWN for st, _ in out), out
    assert len({info for _, info in out}) == 1


@pytest.mark.parametrize("kappa", [1.0, 1e3])
def test_dist_orthogonalize(rg, ranks, kappa):
    """orthogonalize: split-precision reortho passes and the Hutchinson probe allreduce; the
    gathered Q is orthonormal to 1e-5 (north_star) and every rank sees the same estimate."""
    m, n = 20000, 128
    A = (synth.gaussian(m, n, seed=17) if kappa == 1.0 else
         synth.svd_matrix(m, n, "geometric", kappa, seed=17)).astype(np.float32)
    P = ranks.P
    c = _cuts(m, P)
    blocks = [_dev(A[c[r]:c[r + 1]]) for r in range(P)]
    Rs = [torch.zeros(n, n, device="cuda").t() for _ in range(P)]
    out = ranks.run([lambda r=r: rg.orthogonalize(blocks[r], Rs[r], orth_tol=1e-5, max_passes=3,
                                                  handle=ranks.h[r]) for r in range(P)])
    ests = {o[3] for o in out}
    passes = {o[2] for o in out}
    assert len(ests) == 1 and len(passes) == 1
    Q = np.vstack([b.cpu().numpy() for b in blocks]).astype(np.float64)
    orth = oracle.orthogonality(Q)
    assert orth <= 1e-5, (orth, passes, ests)
    R = Rs[0].cpu().numpy().astype(np.float64)
    for r in range(1, P):
        np.testing.assert_array_equal(Rs[r].cpu().numpy(), Rs[0].cpu().numpy())
    assert oracle.backward_error(A.astype(np.float64), Q, R) <= 5e-3
    est = ests.pop()
    assert abs(est - orth) <= 0.5 * orth + 1e-7


@pytest.mark.parametrize("solver", ["cgls", "lsqr"])
@pytest.mark.parametrize("consistent", [False, True])
def test_dist_ls_solve_refined(rg, ranks, consistent, solver):
    """ls_solve_refined: the sharded QR preconditioner + CGLS with the ||q||^2 and A^T r
    allreduces; fe <= 1e-5 at kappa = 1e4 (north_star), x replicated."""
    m, n = 12000, 128
    A = synth.svd_matrix(m, n, "geometric", 1e4, seed=23).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=23, consistent=consistent).astype(np.float32)
    x_star, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    P = ranks.P
    c = _cuts(m, P)
    blocks = [_dev(A[c[r]:c[r + 1]]) for r in range(P)]
    bs = [torch.from_numpy(b[c[r]:c[r + 1]].copy()).cuda() for r in range(P)]
    xs = [torch.zeros(n, dtype=torch.float64, device="cuda") for _ in range(P)]
    o = rg.make_opts(solver=solver)
    out = ranks.run([lambda r=r: rg.ls_solve_refined(blocks[r], bs[r], xs[r], tol=1e-10, maxit=200,
                                                     handle=ranks.h[r], opts=o) for r in range(P)])
    assert all(o[3] == rg.RG_OK for o in out), [o[1:] for o in out]
    assert len({o[1] for o in out}) == 1
    for r in range(1, P):
        np.testing.assert_array_equal(xs[r].cpu().numpy(), xs[0].cpu().numpy())
    x = xs[0].cpu().numpy()
    fe = np.linalg.norm(x - x_star) / np.linalg.norm(x_star)
    assert fe <= 1e-5, (fe, out[0][1])


def test_dist_lowrank(rg, ranks):
    """lowrank_approx row-sharded: local Y = A_p Omega, sharded RGSQR of Y, the B^T = A^T Q
    allreduce, replicated small QR + Jacobi SVD; the error matches the oracle's run of the same
    algorithm on the same Philox sketch, S replicated."""
    m, n, k, rank, p, q = 4096, 768, 256, 48, 16, 1
    A, s = synth.lowrank_matrix(m, n, k, "geometric", 1e6, seed=61)
    A64 = A.astype(np.float64)
    P = ranks.P
    c = _cuts(m, P)
    blocks = [_dev(A[c[r]:c[r + 1]]) for r in range(P)]
    out = ranks.run([lambda r=r: rg.lowrank_approx(blocks[r], rank, oversample=p, power_iters=q, seed=99,
                                                   handle=ranks.h[r]) for r in range(P)])
    U = np.vstack([o[0].cpu().numpy() for o in out]).astype(np.float64)
    S = out[0][1].cpu().numpy().astype(np.float64)
    V = out[0][2].cpu().numpy().astype(np.float64)
    for r in range(1, P):
        np.testing.assert_array_equal(out[r][1].cpu().numpy(), out[0][1].cpu().numpy())
        np.testing.assert_array_equal(out[r][2].cpu().numpy(), out[0][2].cpu().numpy())
    err = oracle.lowrank_error(A64, U, S, V)
    Om = oracle.gaussian_philox(n, rank + p, 99)
    Uo, So, Vo, _ = oracle.lowrank(A64, rank, p, q, Om)
    err_o = oracle.lowrank_error(A64, Uo, So, Vo)
    assert abs(err - err_o) <= 1e-3 * err_o + 1e-5, (err, err_o)
    np.testing.assert_allclose(S, So, rtol=2e-3)


def test_vgroup_argument_checks(rg):
    import ctypes
    L = rg.lib()
    g = ctypes.c_void_p()
    assert L.rg_vgroup_create(ctypes.byref(g), 0) == -2
    assert L.rg_vgroup_create(ctypes.byref(g), rg.RG_MAX_RANKS + 1) == -2
    grp = rg.VGroup(2)
    h = rg.Handle(0)
    assert L.rg_set_vcomm(h.ptr, grp.ptr, 2) == -3
    h.set_vcomm(grp, 1)
    assert L.rg_vgroup_destroy(grp.ptr) == -1        # a handle is still attached
    h.set_vcomm(None, 0)
    assert L.rg_set_comm(h.ptr, None, 0, 1) == 0      # NULL communicator = single-GPU mode
    assert L.rg_set_comm(h.ptr, ctypes.c_void_p(1), 0, rg.RG_MAX_RANKS + 1) == -4
    grp.close()
    h.close()
