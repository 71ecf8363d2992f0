"""K7/K8 norm kernels through the C-ABI (mario_k_norm_fwd / mario_k_norm_bwd) against plain
PyTorch fp32/fp64 math on the same bf16 inputs (readings A1/A2: LayerNorm / RMSNorm over the
hidden dimension, biased variance, eps inside the square root).

Variants: 3 = warp-per-row v2 forward (persistent, shifted one-pass stats) + the row-pipelined backward,
2 = row-pipelined persistent kernels (every width n % 8 == 0 up to 8192 forward, 5120 backward),
1 = block-per-row-tile backward, 0 = warp-per-row. Widths cover the block-per-row-tile kernels (n = 2048, 2560, 4096: one 16-byte chunk per thread;
5120: two) and the warp-per-row fallback (n = 64, 776); row counts are ragged against the R-row
tile and the CTA row ranges."""
import pytest
import torch

from paper_conf_ppopp_liultj25_b200 import _lib

pytestmark = pytest.mark.gpu

EPS = 1e-5


def _inputs(rows, n, seed):
    g = torch.Generator(device="cuda").manual_seed(seed)
    x = (torch.randn(rows, n, device="cuda", generator=g) * 1.5 + 0.3).bfloat16()
    gam = torch.randn(n, device="cuda", generator=g)
    bet = torch.randn(n, device="cuda", generator=g)
    dy = torch.randn(rows, n, device="cuda", generator=g).bfloat16()
    dres = torch.randn(rows, n, device="cuda", generator=g).bfloat16()
    return x, gam, bet, dy, dres


def _ref_fwd(x, gam, bet, rms):
    xf = x.double()
    if rms:
        mean = torch.zeros(xf.shape[0], 1, dtype=torch.float64, device=x.device)
        rstd = torch.rsqrt((xf * xf).mean(1, keepdim=True) + EPS)
        y = xf * rstd * gam.double()
    else:
        mean = xf.mean(1, keepdim=True)
        rstd = torch.rsqrt(((xf - mean) ** 2).mean(1, keepdim=True) + EPS)
        y = (xf - mean) * rstd * gam.double() + bet.double()
    return y, mean.squeeze(1), rstd.squeeze(1)


def _ref_bwd(dy, x, gam, dres, rms):
    """dx of y = xhat * g (+ b): dx = rstd * (dy g - mean(dy g) - xhat mean(dy g xhat)) (+ dres)."""
    xf, d = x.double(), dy.double()
    _, mean, rstd = _ref_fwd(x, gam, gam, rms)
    xh = (xf - mean[:, None]) * rstd[:, None]
    gp = d * gam.double()
    sg = torch.zeros_like(rstd)[:, None] if rms else gp.mean(1, keepdim=True)
    sgx = (gp * xh).mean(1, keepdim=True)
    dx = (gp - sg - xh * sgx) * rstd[:, None]
    if dres is not None:
        dx = dx + dres.double()
    return dx, (d * xh).sum(0), d.sum(0), (d.abs() * xh.abs()).sum(0), d.abs().sum(0)


CASES = [(1, 2048), (37, 2048), (8195, 2048), (517, 2560), (300, 4096), (129, 5120), (33, 64), (70, 776),
         (2000, 192), (5, 8192)]


@pytest.fixture(params=[3, 2, 1, 0], ids=["warp2", "pipe", "tile", "row"])
def variant(request):
    L = _lib.lib()
    assert L.mario_k_norm_set_variant(request.param) == 0
    yield request.param
    L.mario_k_norm_set_variant(3)


@pytest.mark.parametrize("rms", [0, 1], ids=["ln", "rms"])
@pytest.mark.parametrize("rows,n", CASES)
def test_norm_fwd(variant, rows, n, rms):
    L = _lib.lib()
    x, gam, bet, _, _ = _inputs(rows, n, rows * 31 + n + rms)
    y = torch.empty_like(x)
    stats = torch.empty(rows, 2, device="cuda")
    assert L.mario_k_norm_fwd(x.data_ptr(), gam.data_ptr(), bet.data_ptr(), y.data_ptr(), stats.data_ptr(), rows, n,
                              EPS, rms, 1, None) == 0
    torch.cuda.synchronize()
    yr, mean, rstd = _ref_fwd(x, gam, bet, rms)
    # one bf16 rounding of the output (2^-9 relative) plus fp32 statistics
    err = (y.double() - yr).abs()
    assert (err <= yr.abs() * 2.0 ** -8 + 2e-3).all(), err.max().item()
    assert torch.allclose(stats[:, 0].double(), mean, rtol=1e-5, atol=1e-5)
    assert torch.allclose(stats[:, 1].double(), rstd, rtol=1e-5, atol=1e-6)


@pytest.mark.parametrize("rms", [0, 1], ids=["ln", "rms"])
@pytest.mark.parametrize("with_res", [True, False], ids=["dres", "nodres"])
@pytest.mark.parametrize("rows,n", CASES)
def test_norm_bwd_fused(variant, rows, n, rms, with_res):
    L = _lib.lib()
    x, gam, bet, dy, dres = _inputs(rows, n, rows * 17 + n + 2 * rms)
    if not with_res:
        dres = None
    stats = torch.empty(rows, 2, device="cuda")
    y = torch.empty_like(x)
    assert L.mario_k_norm_fwd(x.data_ptr(), gam.data_ptr(), bet.data_ptr(), y.data_ptr(), stats.data_ptr(), rows, n,
                              EPS, rms, 1, None) == 0
    dx = torch.empty_like(x)
    dg0 = torch.randn(n, device="cuda")     # accumulation: += into existing gradients
    db0 = torch.randn(n, device="cuda")
    ds0 = torch.randn(n, device="cuda")
    dg, db, ds = dg0.clone(), db0.clone(), ds0.clone()
    part = torch.empty(3 * n * 148 * 8, device="cuda")
    assert L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), gam.data_ptr(),
                              dres.data_ptr() if dres is not None else None, dx.data_ptr(), dg.data_ptr(),
                              db.data_ptr(), ds.data_ptr(), part.data_ptr(), part.numel(), rows, n, rms, 1,
                              None) == 0
    torch.cuda.synchronize()
    dxr, dgr, dbr, dga, dba = _ref_bwd(dy, x, gam, dres, rms)
    err = (dx.double() - dxr).abs()
    scale = dxr.abs().max().item()
    assert err.max().item() <= 1e-2 * scale, (err.max().item(), scale)
    assert (err <= dxr.abs() * 2.0 ** -7 + 1e-3 * scale).float().mean().item() > 0.999
    # column sums: fp32 accumulation of bf16 products, bounded by 1e-5 of the absolute sum
    assert ((dg.double() - dg0.double() - dgr).abs() <= 1e-5 * dga + 1e-5).all()
    if not rms:
        assert ((db.double() - db0.double() - dbr).abs() <= 1e-5 * dba + 1e-5).all()
    else:
        assert torch.equal(db, db0)
    # dsum: column sums of the written (rounded) dx
    dsr = dx.double().sum(0)
    assert ((ds.double() - ds0.double() - dsr).abs() <= 1e-5 * dx.double().abs().sum(0) + 1e-5).all()


def test_norm_bwd_is_deterministic():
    L = _lib.lib()
    rows, n = 8192, 2048
    x, gam, bet, dy, dres = _inputs(rows, n, 5)
    stats = torch.empty(rows, 2, device="cuda")
    y = torch.empty_like(x)
    L.mario_k_norm_fwd(x.data_ptr(), gam.data_ptr(), bet.data_ptr(), y.data_ptr(), stats.data_ptr(), rows, n, EPS,
                       0, 1, None)
    part = torch.empty(3 * n * 148 * 8, device="cuda")
    outs = []
    for _ in range(2):
        dx = torch.empty_like(x)
        dg, db, ds = (torch.zeros(n, device="cuda") for _ in range(3))
        L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), gam.data_ptr(), dres.data_ptr(),
                           dx.data_ptr(), dg.data_ptr(), db.data_ptr(), ds.data_ptr(), part.data_ptr(), part.numel(),
                           rows, n, 0, 1, None)
        torch.cuda.synchronize()
        outs.append((dx, dg, db, ds))
    for a, b in zip(*outs):
        assert torch.equal(a, b)
