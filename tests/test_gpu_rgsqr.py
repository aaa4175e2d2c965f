"""GPU parity of rgsqr_factor (C-ABI) against the fp64 oracle (-m gpu).

Tolerances (BASELINE north_star, restated in DESIGN.md "Tolerances"):
  backward error ||A - QR||_F / ||A||_F <= 5e-3, orthogonality ||I - Q^T Q||_F <= 1e-2 sqrt(n)
  before reorthogonalisation on well-conditioned inputs (reading #11).  Distance to the
  unique QR (oracle Householder, positive diagonal): ||R - R*||_F/||R*||_F <= 10 kappa * be.
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
    """numpy (m, n) -> column-major CUDA fp32 tensor (strides (1, m))."""
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()


def _run(rg, A32, **kw):
    Ad = _dev(A32)
    Q, R = rg.rgsqr_factor(Ad, opts=rg.make_opts(**kw))
    torch.cuda.synchronize()
    return Q.cpu().numpy().astype(np.float64), R.cpu().numpy().astype(np.float64)


def _check_qr(A32, Q, R, kappa=10.0, orth_scale=1e-2):
    """Identities and distance to the UNIQUE factors Q*, R* of the oracle's Householder QR
    (positive diagonal).  Tolerance (reading #25): the computed pair is the exact QR
    U (T R) of A - dA with Q = U T, T^T T = Q^T Q = I - E, so to first order
        ||R - R*||_F / ||R*||_F <= sqrt(2) kappa be + ||E||_F / sqrt(2),
        ||Q - Q*||_F / ||Q*||_F <= (1 + sqrt(2)) kappa be + ||E||_F / sqrt(2 n)
    (Sun's perturbation bounds of the QR factors; be = ||dA||_F / ||A||_F); the tests use
    10 kappa be + orth and 10 kappa be + orth / sqrt(n)."""
    A = np.asarray(A32, dtype=np.float64)
    m, n = A.shape
    assert np.all(np.isfinite(Q)) and np.all(np.isfinite(R))
    assert np.all(np.tril(R, -1) == 0)
    assert np.all(np.diag(R) > 0)
    be = oracle.backward_error(A, Q, R)
    orth = oracle.orthogonality(Q)
    assert be <= 5e-3, be
    assert orth <= orth_scale * np.sqrt(n), orth
    Qo, Ro, _ = oracle.householder(A)
    dr = np.linalg.norm(R - Ro) / np.linalg.norm(Ro)
    dq = np.linalg.norm(Q - Qo) / np.linalg.norm(Qo)
    assert dr <= 10 * kappa * be + orth + 1e-6, (dr, be, orth, kappa)
    assert dq <= 10 * kappa * be + orth / np.sqrt(n) + 1e-6, (dq, be, orth, kappa)
    return be, orth, dr


@pytest.mark.parametrize("panel", ["auto", "mgs"])
@pytest.mark.parametrize("m,n", [(64, 1), (100, 7), (256, 32), (1000, 32), (1024, 64), (1025, 96), (4099, 64),
                                 (3000, 200), (8192, 256), (777, 333), (70000, 40)])
def test_rgsqr_gaussian_parity(rg, m, n, panel):
    A = synth.gaussian(m, n, seed=synth.SEED_BASE + m + n).astype(np.float32)
    Q, R = _run(rg, A, panel=panel)
    _check_qr(A, Q, R, kappa=np.linalg.cond(A))


@pytest.mark.parametrize("kappa", [1e2, 1e4, 1e6])
def test_rgsqr_ill_conditioned_backward_error(rg, kappa):
    """Backward error independent of cond(A) (Fig 3); orthogonality grows ~kappa u_h.
    The distance to the unique factors is checked where its first-order bound (reading #25) is
    informative (kappa be < 0.05, i.e. kappa = 1e2 here); beyond that the QR factors of A are
    not determined to working accuracy by any 16-bit-update method and only be is meaningful."""
    A = synth.svd_matrix(4096, 128, "geometric", kappa, seed=21).astype(np.float32)
    Q, R = _run(rg, A)
    A64 = A.astype(np.float64)
    be = oracle.backward_error(A64, Q, R)
    assert be < 5e-3
    assert np.all(np.diag(R) > 0) and np.all(np.tril(R, -1) == 0)
    if kappa * be < 0.05:
        _check_qr(A, Q, R, kappa=kappa, orth_scale=1.0)
    else:
        # the leading columns are well conditioned: their block of R is still pinned
        k = 16
        Ak = A64[:, :k]
        _, Rk, _ = oracle.householder(Ak)
        kk = np.linalg.cond(Ak)
        assert np.linalg.norm(R[:k, :k] - Rk) / np.linalg.norm(Rk) <= 10 * kk * be + 1e-2


@pytest.mark.parametrize("kappa", [10.0, 1e5])
@pytest.mark.parametrize("n", [32, 96])
def test_rgsqr_streaming_cholqr_panel(rg, monkeypatch, kappa, n):
    """The three-launch streaming CholQR2 panel (used when a panel's rows do not fit in the
    fused kernel's shared memory) forced on a small case; kappa = 1e5 makes the panels take
    the second CholQR pass, whose R = R2 R1 product reads R2 back from the elimination scratch."""
    monkeypatch.setenv("RGSQR_CQ_STREAM", "1")
    h = rg.Handle(0)
    A = synth.svd_matrix(3000, n, "geometric", kappa, seed=31).astype(np.float32)
    Q, R = rg.rgsqr_factor(_dev(A), handle=h)
    torch.cuda.synchronize()
    Q = Q.cpu().numpy().astype(np.float64)
    R = R.cpu().numpy().astype(np.float64)
    A64 = A.astype(np.float64)
    be = oracle.backward_error(A64, Q, R)
    assert be < (1e-6 if n == 32 else 5e-3)
    Qo, Ro, _ = oracle.householder(A64)
    # forward error of R ~ kappa * backward error (as in _check_qr)
    assert np.linalg.norm(R - Ro) / np.linalg.norm(Ro) <= max(10 * kappa * be, 1e-5)
    if n == 32:
        assert oracle.orthogonality(Q) < 1e-5


@pytest.mark.parametrize("kappa", [10.0, 1e4, 1e6])
def test_rgsqr_wide_leaf_level(rg, monkeypatch, kappa):
    """RGSQR_WIDE=1: the last recursion level as one 64-column CholQR2 kernel (same unique QR)."""
    monkeypatch.setenv("RGSQR_WIDE", "1")
    h = rg.Handle(0)
    A = synth.svd_matrix(8192, 160, "geometric", kappa, seed=51).astype(np.float32)
    Q, R = rg.rgsqr_factor(_dev(A), handle=h)
    torch.cuda.synchronize()
    Q = Q.cpu().numpy().astype(np.float64)
    R = R.cpu().numpy().astype(np.float64)
    _check_qr(A, Q, R, kappa=kappa, orth_scale=(1e-2 if kappa < 1e3 else 1.0))


def test_rgsqr_wide_breakdown_status(rg, monkeypatch):
    monkeypatch.setenv("RGSQR_WIDE", "1")
    h = rg.Handle(0)
    A = synth.gaussian(4096, 64, seed=52).astype(np.float32)
    A[:, 40] = 0.0
    with pytest.raises(rg.RGError) as e:
        rg.rgsqr_factor(_dev(A), handle=h)
    assert e.value.status == rg.RG_BREAKDOWN


def test_rgsqr_tall_panel_streaming_path(rg):
    """m = 200000: more rows per CTA than the fused panel holds -> streaming passes by design."""
    A = synth.gaussian(200000, 40, seed=41).astype(np.float32)
    Q, R = _run(rg, A)
    _check_qr(A, Q, R, kappa=np.linalg.cond(A))


@pytest.mark.parametrize("pad", [0, 3])
def test_rgsqr_tall_streaming_aligned_and_unaligned(rg, pad):
    """Streaming passes (m = 200000) through both load paths: lda = m (16-byte aligned columns:
    cp.async ring, vector stores) and lda = m + 3 (register prefetch, scalar stores); the two
    must agree to rounding and meet the factorization bounds."""
    m, n = 200000, 64
    A = synth.gaussian(m, n, seed=43).astype(np.float32)
    big = np.zeros((n, m + pad), dtype=np.float32)
    big[:, :m] = A.T
    Ad = torch.from_numpy(big).cuda().t()[:m]          # column-major view, lda = m + pad
    Q = torch.zeros(n, m + pad, device="cuda").t()[:m]
    Q, R = rg.rgsqr_factor(Ad, Q=Q)
    torch.cuda.synchronize()
    Qn = Q.cpu().numpy().astype(np.float64)
    Rn = R.cpu().numpy().astype(np.float64)
    _check_qr(A, Qn, Rn, kappa=np.linalg.cond(A))
    Q0, R0 = _run(rg, A)
    assert np.linalg.norm(Rn - R0) / np.linalg.norm(R0) < 1e-5


def test_rgsqr_tall_streaming_breakdown(rg):
    """Streaming panels (m = 200000): an exactly zero column in the second 32-column panel fails
    the CholQR pivot test there, the guarded MGS/TSQR fallback reports the breakdown, and an
    ill-conditioned tall matrix (kappa 1e3) factors to the usual bounds."""
    m = 200000
    A = synth.gaussian(m, 64, seed=47).astype(np.float32)
    A[:, 40] = 0.0
    with pytest.raises(rg.RGError) as e:
        _run(rg, A)
    assert e.value.status == rg.RG_BREAKDOWN
    B = synth.svd_matrix(m, 64, "geometric", 1e3, seed=48).astype(np.float32)
    Q, R = _run(rg, B)
    _check_qr(B, Q, R, kappa=1e3, orth_scale=1.0)


def test_rgsqr_config1(rg):
    """BASELINE config 1: 1024 x 64, cond ~ 10 (geometric spectrum), vs the fp64 oracle."""
    A = synth.svd_matrix(1024, 64, "geometric", 10.0, seed=synth.SEED_BASE + 0).astype(np.float32)
    Q, R = _run(rg, A)
    be, orth, dr = _check_qr(A, Q, R, kappa=10.0)
    assert be < 2e-4  # fp16 updates, fp32 panel: SURVEY [EMU] ~4e-5


@pytest.mark.parametrize("panel", ["auto", "mgs"])
def test_rgsqr_single_panel_is_fp32_accurate(rg, panel):
    """n <= 32: the whole call is one fp32 panel (no tensor cores)."""
    A = synth.gaussian(5000, 32, seed=3).astype(np.float32)
    Q, R = _run(rg, A, panel=panel)
    A64 = A.astype(np.float64)
    assert oracle.backward_error(A64, Q, R) < 1e-6
    assert oracle.orthogonality(Q) < 1e-5


def test_rgsqr_bf16(rg):
    A = synth.gaussian(2048, 128, seed=4).astype(np.float32)
    Q, R = _run(rg, A, precision="bf16")
    _check_qr(A, Q, R, kappa=np.linalg.cond(A), orth_scale=5e-2)


def test_rgsqr_scaling_invariance(rg):
    """AP = Q (R P) for power-of-two P (section 3.5): Q identical, R column-scaled."""
    A = synth.gaussian(2048, 96, seed=5).astype(np.float32)
    g = synth.rng(6)
    p = (2.0 ** g.integers(-20, 21, size=96)).astype(np.float32)
    Q1, R1 = _run(rg, A)
    Q2, R2 = _run(rg, A * p)
    np.testing.assert_array_equal(Q1, Q2)
    np.testing.assert_allclose(R2, R1 * p, rtol=1e-6, atol=0)


def test_rgsqr_badly_scaled_columns(rg):
    """Columns far outside the fp16 range factor correctly thanks to scaling."""
    A = synth.gaussian(4096, 64, seed=7).astype(np.float32)
    A[:, ::3] *= 1e6
    A[:, 1::3] *= 1e-6
    Q, R = _run(rg, A)
    Ar = A.astype(np.float64)
    assert oracle.backward_error(Ar, Q, R) < 5e-3
    assert oracle.orthogonality(Q) < 1e-2 * 8


def test_rgsqr_deterministic(rg):
    A = synth.gaussian(4096, 128, seed=8).astype(np.float32)
    Q1, R1 = _run(rg, A)
    Q2, R2 = _run(rg, A)
    np.testing.assert_array_equal(Q1, Q2)
    np.testing.assert_array_equal(R1, R2)


def test_rgsqr_inplace_and_lda(rg):
    A = synth.gaussian(1000, 64, seed=9).astype(np.float32)
    big = np.zeros((1024 + 13, 64), dtype=np.float32)
    big[:1000] = A
    Bd = _dev(big)
    view = Bd[:1000]
    Q, R = rg.rgsqr_factor(view, Q=view)
    torch.cuda.synchronize()
    Qn = Bd.cpu().numpy()[:1000].astype(np.float64)
    _check_qr(A, Qn, R.cpu().numpy().astype(np.float64), kappa=np.linalg.cond(A))
    np.testing.assert_array_equal(Bd.cpu().numpy()[1000:], 0)


def test_rgsqr_host_pointers(rg):
    A = np.asfortranarray(synth.gaussian(3000, 96, seed=10).astype(np.float32))
    Q, R = rg.rgsqr_factor(A)
    _check_qr(A, Q.astype(np.float64), R.astype(np.float64), kappa=np.linalg.cond(A))


def test_rgsqr_breakdown_status(rg):
    A = synth.gaussian(512, 40, seed=11).astype(np.float32)
    A[:, 17] = 0.0
    with pytest.raises(rg.RGError) as e:
        _run(rg, A)
    assert e.value.status == rg.RG_BREAKDOWN
    A = synth.gaussian(512, 40, seed=11).astype(np.float32)
    A[3, 5] = np.nan
    with pytest.raises(rg.RGError) as e:
        _run(rg, A)
    assert e.value.status == rg.RG_NONFINITE and e.value.info == 5


def test_rgsqr_after_breakdown_is_clean(rg):
    """A failed panel (CholQR pivot) must not leak its fallback flag into later calls."""
    A = synth.gaussian(512, 40, seed=11).astype(np.float32)
    A[:, 3] = 0.0
    with pytest.raises(rg.RGError):
        _run(rg, A)
    B = synth.svd_matrix(4096, 96, "geometric", 1e2, seed=12).astype(np.float32)
    Q, R = _run(rg, B)
    _check_qr(B, Q, R, kappa=1e2, orth_scale=1.0)


def test_rgsqr_invalid_arguments(rg):
    import ctypes
    h = rg.default_handle()
    L = rg.lib()
    o = rg.make_opts()
    A = torch.zeros(10, 20, device="cuda")
    p = ctypes.c_void_p(A.data_ptr())
    assert L.rgsqr_factor(h.ptr, 10, 20, p, 10, p, 10, p, 20, ctypes.byref(o)) == -2   # m < n
    assert L.rgsqr_factor(h.ptr, 20, 0, p, 20, p, 20, p, 20, ctypes.byref(o)) == -3
    assert L.rgsqr_factor(h.ptr, 20, 10, None, 20, p, 20, p, 20, ctypes.byref(o)) == -4
    assert L.rgsqr_factor(h.ptr, 20, 10, p, 19, p, 20, p, 20, ctypes.byref(o)) == -5
    assert L.rgsqr_factor(h.ptr, 20, 10, p, 20, p, 20, p, 9, ctypes.byref(o)) == -9


@pytest.mark.parametrize("m,n,pad", [(3000, 96, 0), (5000, 300, 7), (20000, 1000, 0), (4099, 640, 3),
                                     (6000, 1536, 0), (8192, 2048, 5)])
def test_rgsqr_pinned_host_pipeline(rg, m, n, pad):
    """Pinned host A/Q/R take the pipelined path (column-chunked H2D, chunked scaling, Q columns
    D2H as their panels finish, and the column-lazy schedule: levels wider than 256 columns apply
    their K1 / K2 in 256-column chunks as the columns arrive -- n >= 640 here); per-column
    scaling, per-column norms and the chunk's unchanged split-K decomposition make it the same
    arithmetic as the device path, so Q and R must be bit-identical to it."""
    A = synth.gaussian(m, n, seed=synth.SEED_BASE + 31 + n).astype(np.float32)
    Ah = torch.zeros(n, m + pad, dtype=torch.float32, pin_memory=True)
    Ah[:, :m].copy_(torch.from_numpy(np.ascontiguousarray(A.T)))
    Ah = Ah.t()[:m]
    Qh = torch.full((n, m + pad), -1.0, dtype=torch.float32, pin_memory=True).t()[:m]
    Rh = torch.full((n, n), -1.0, dtype=torch.float32, pin_memory=True).t()
    for _ in range(2):   # second call reuses the staging buffers and copy streams
        rg.rgsqr_factor(Ah, Q=Qh, R=Rh)
        Qd, Rd = rg.rgsqr_factor(_dev(A))
        torch.cuda.synchronize()
        np.testing.assert_array_equal(Qh.numpy(), Qd.cpu().numpy())
        np.testing.assert_array_equal(Rh.numpy(), Rd.cpu().numpy())
    _check_qr(A, Qh.numpy().astype(np.float64), Rh.numpy().astype(np.float64), kappa=np.linalg.cond(A))


def test_rgsqr_pinned_host_pipeline_breakdown(rg):
    A = synth.gaussian(2048, 300, seed=13).astype(np.float32)
    A[:, 257] = 0.0   # a zero column in the third H2D chunk
    Ah = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    Qh = torch.empty(300, 2048, dtype=torch.float32, pin_memory=True).t()
    Rh = torch.empty(300, 300, dtype=torch.float32, pin_memory=True).t()
    with pytest.raises(rg.RGError) as e:
        rg.rgsqr_factor(Ah, Q=Qh, R=Rh)
    with pytest.raises(rg.RGError) as ed:
        _run(rg, A)
    assert e.value.status == ed.value.status == rg.RG_BREAKDOWN
    assert e.value.info == ed.value.info
    B = synth.gaussian(2048, 300, seed=14).astype(np.float32)
    Bh = torch.from_numpy(np.ascontiguousarray(B.T)).pin_memory().t()
    rg.rgsqr_factor(Bh, Q=Qh, R=Rh)
    _check_qr(B, Qh.numpy().astype(np.float64), Rh.numpy().astype(np.float64), kappa=np.linalg.cond(B))


@pytest.mark.parametrize("kw", [dict(precision="bf16"), dict(split=True), dict(panel="mgs"), dict(scale=False),
                                dict(reortho=1), dict(nb=16)])
def test_rgsqr_pinned_host_options(rg, kw):
    """Every option through pinned host buffers (pipelined when reortho = 0, staged otherwise)
    gives the device-pointer call's Q and R bit for bit."""
    m, n = 6000, 200
    A = synth.gaussian(m, n, seed=synth.SEED_BASE + 77).astype(np.float32) * np.float32(3e-3)
    Ah = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    Qh = torch.empty(n, m, dtype=torch.float32, pin_memory=True).t()
    Rh = torch.empty(n, n, dtype=torch.float32, pin_memory=True).t()
    o = rg.make_opts(**kw)
    rg.rgsqr_factor(Ah, Q=Qh, R=Rh, opts=o)
    Qd, Rd = rg.rgsqr_factor(_dev(A), opts=o)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(Qh.numpy(), Qd.cpu().numpy())
    np.testing.assert_array_equal(Rh.numpy(), Rd.cpu().numpy())
    _check_qr(A, Qh.numpy().astype(np.float64), Rh.numpy().astype(np.float64), kappa=np.linalg.cond(A),
              orth_scale=5e-2 if kw.get("precision") == "bf16" or kw.get("scale") is False else 1e-2)


def test_rgsqr_k2_cluster_pair_bit_identical(rg, monkeypatch):
    """The cluster-pair K2 (two CTAs share the multicast B tile; levels with >= 9 k-blocks, i.e.
    h >= 576) runs the same MMAs in the same order per tile as the single-CTA K2: Q and R are
    bit-identical with it on (default) and off (RGSQR_K2_PAIR=0)."""
    A = synth.gaussian(8192, 1536, seed=51).astype(np.float32)
    out = {}
    for pair in ("1", "0"):
        monkeypatch.setenv("RGSQR_K2_PAIR", pair)
        h = rg.Handle(0)
        try:
            Ad = _dev(A)
            Q, R = rg.rgsqr_factor(Ad, handle=h)
            torch.cuda.synchronize()
            out[pair] = (Q.cpu().numpy(), R.cpu().numpy())
        finally:
            h.close()
    np.testing.assert_array_equal(out["1"][0], out["0"][0])
    np.testing.assert_array_equal(out["1"][1], out["0"][1])
    Q, R = (x.astype(np.float64) for x in out["1"])
    _check_qr(A, Q, R, kappa=np.linalg.cond(A))
