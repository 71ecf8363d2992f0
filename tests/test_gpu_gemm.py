"""K1-K4 GEMM unit tests through the C-ABI (mario_k_gemm_*) against fp32 torch math on the
same bf16-rounded inputs."""
import pytest
import torch

from paper_conf_ppopp_liultj25_b200 import _lib

pytestmark = pytest.mark.gpu

SHAPES = [(128, 256, 64), (296, 200, 72), (256, 512, 1024), (1000, 384, 136), (64, 64, 64),
          (2048, 2048, 512)]


def _ptr(t):
    return t.data_ptr() if t is not None else None


def _run(a_mn, b_mn, M, N, K, out_f32, bias=False, resid=False, gelu2=False, aux=False, beta=0.0):
    dev = "cuda"
    g = torch.Generator(device=dev).manual_seed(M * 7 + N * 3 + K)
    A = torch.randn(M, K, device=dev, generator=g).bfloat16()
    B = torch.randn(N, K, device=dev, generator=g).bfloat16()
    Ast = A.t().contiguous() if a_mn else A
    Bst = B.t().contiguous() if b_mn else B
    ref = A.float() @ B.float().t()
    b = torch.randn(N, device=dev, generator=g) if bias else None
    if b is not None:
        ref = ref + b
    z = torch.randn(M, N, device=dev, generator=g).bfloat16() if aux else None
    if z is not None:
        zf = z.float()
        t = torch.tanh(0.7978845608028654 * (zf + 0.044715 * zf ** 3))
        ref = ref * (0.5 * (1 + t) + 0.5 * zf * (1 - t * t) * 0.7978845608028654 * (1 + 3 * 0.044715 * zf * zf))
    r = torch.randn(M, N, device=dev, generator=g).bfloat16() if resid else None
    if r is not None:
        ref = ref + r.float()
    if out_f32:
        D = torch.randn(M, N, device=dev, generator=g)
        ref = ref + beta * D
    else:
        D = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
    D2 = torch.empty(M, N, device=dev, dtype=torch.bfloat16) if gelu2 else None
    err = _lib.lib().mario_k_gemm_bf16(
        _ptr(Ast), Ast.shape[1], a_mn, _ptr(Bst), Bst.shape[1], b_mn, M, N, K, _ptr(D), N, int(out_f32),
        beta, _ptr(b), _ptr(r), N, _ptr(D2), _ptr(z), N, None)
    assert err == 0
    torch.cuda.synchronize()
    scale = ref.abs().max().item()
    tol = 2e-3 if out_f32 else 1e-2
    assert (D.float() - ref).abs().max().item() <= tol * scale
    if gelu2:
        gref = torch.nn.functional.gelu((z if aux else D).float(), approximate="tanh")
        assert (D2.float() - gref).abs().max().item() <= 2e-2 * gref.abs().max().item() + 1e-2


@pytest.fixture(params=[0, 2, 3], ids=["single_cta", "cta_pair_n128", "cta_pair_n256"])
def variant(request):
    L = _lib.lib()
    assert L.mario_k_gemm_set_variant(request.param) == 0
    yield request.param
    L.mario_k_gemm_set_variant(-1)


@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 1), (1, 0)])
@pytest.mark.parametrize("M,N,K", SHAPES + [(768, 1280, 320), (520, 264, 200)])
def test_gemm_bf16_majors(a_mn, b_mn, M, N, K, variant):
    _run(a_mn, b_mn, M, N, K, out_f32=False)


@pytest.mark.parametrize("M,N,K", SHAPES[:4] + [(768, 1280, 320)])
def test_gemm_bf16_wgrad_accumulate(M, N, K, variant):
    _run(1, 1, M, N, K, out_f32=True, beta=1.0)


def test_gemm_bf16_epilogues(variant):
    _run(0, 0, 384, 640, 256, out_f32=False, bias=True, resid=True)
    _run(0, 0, 384, 640, 256, out_f32=False, bias=True, gelu2=True)
    _run(0, 1, 384, 640, 256, out_f32=False, aux=True)
    _run(0, 1, 384, 640, 256, out_f32=False, aux=True, gelu2=True)     # D2 = gelu(aux): fc2 dgrad


def test_gemm_bf16_deterministic():
    M, N, K = 1024, 768, 2048
    A = torch.randn(K, M, device="cuda").bfloat16()
    B = torch.randn(K, N, device="cuda").bfloat16()
    outs = []
    for _ in range(2):
        D = torch.zeros(M, N, device="cuda")
        assert _lib.lib().mario_k_gemm_bf16(A.data_ptr(), M, 1, B.data_ptr(), N, 1, M, N, K, D.data_ptr(), N,
                                            1, 0.0, None, None, 0, None, None, 0, None) == 0
        outs.append(D)
    torch.cuda.synchronize()
    assert torch.equal(outs[0], outs[1])


@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 1)])
def test_gemm_f32(a_mn, b_mn):
    M, N, K = 200, 130, 70
    A = torch.randn(M, K, device="cuda", dtype=torch.float64)
    B = torch.randn(N, K, device="cuda", dtype=torch.float64)
    ref = A @ B.t()
    Ast = (A.t() if a_mn else A).float().contiguous()
    Bst = (B.t() if b_mn else B).float().contiguous()
    D = torch.empty(M, N, device="cuda")
    assert _lib.lib().mario_k_gemm_f32(Ast.data_ptr(), Ast.shape[1], a_mn, Bst.data_ptr(), Bst.shape[1], b_mn,
                                       M, N, K, D.data_ptr(), N, 0.0, None, None, 0, None, None, 0, None) == 0
    torch.cuda.synchronize()
    assert (D.double() - ref).abs().max().item() < 1e-4 * ref.abs().max().item()


@pytest.mark.parametrize("sk", [1, 0], ids=["streamk", "tiles"])
@pytest.mark.parametrize("a_mn,b_mn,out_f32", [(0, 0, 0), (0, 1, 0), (1, 1, 1)])
def test_gemm_streamk(sk, a_mn, b_mn, out_f32):
    """Auto kernel selection at a shape whose 45 pair tiles fill 61% of a wave (stream-K splits the
    k-blocks evenly over all pairs, partial tiles finished in pair order) plus ragged M/N/K."""
    L = _lib.lib()
    assert L.mario_k_gemm_set_streamk(sk) == 0
    try:
        _run(a_mn, b_mn, 2184, 1280, 2112, out_f32=bool(out_f32), beta=1.0 if out_f32 else 0.0,
             bias=not out_f32, resid=not out_f32)
        _run(a_mn, b_mn, 2000, 1000, 3000, out_f32=bool(out_f32), beta=1.0 if out_f32 else 0.0)
        if not out_f32:
            _run(a_mn, b_mn, 2184, 1280, 2112, out_f32=False, aux=True)
            _run(a_mn, b_mn, 2184, 1280, 2112, out_f32=False, bias=True, gelu2=True)
    finally:
        L.mario_k_gemm_set_streamk(0)


@pytest.mark.parametrize("sk", [1, 0], ids=["streamk", "tiles"])
def test_gemm_streamk_deterministic(sk):
    L = _lib.lib()
    assert L.mario_k_gemm_set_streamk(sk) == 0
    g = torch.Generator(device="cuda").manual_seed(3)
    M, N, K = 8192, 2048, 8192
    A = torch.randn(M, K, device="cuda", generator=g).bfloat16()
    B = torch.randn(N, K, device="cuda", generator=g).bfloat16()
    outs = []
    for _ in range(3):
        D = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
        assert L.mario_k_gemm_bf16(A.data_ptr(), K, 0, B.data_ptr(), K, 0, M, N, K, D.data_ptr(), N, 0, 0.0, None,
                                   None, N, None, None, N, None) == 0
        outs.append(D)
    torch.cuda.synchronize()
    L.mario_k_gemm_set_streamk(0)
    assert torch.equal(outs[0], outs[1]) and torch.equal(outs[0], outs[2])
    ref = A.float() @ B.float().t()
    assert (outs[0].float() - ref).abs().max().item() <= 1e-2 * ref.abs().max().item()
