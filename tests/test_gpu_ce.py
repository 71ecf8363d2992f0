"""K13 softmax cross-entropy through the C-ABI (mario_k_softmax_ce) against plain PyTorch fp64 on
the same fp32 logits (l[t] = logsumexp(z_t) - z_t[y_t], dlogits = (softmax - onehot)
/ Ntok, readings A4/A21). Vocabularies: the tiny 256, a ragged 1000, LLaMA's 32000 and GPT's padded
50304 (the register-resident one-read kernel), 50 (not a multiple of 4: the generic kernel)."""
import pytest
import torch

from paper_conf_ppopp_liultj25_b200 import _lib

pytestmark = pytest.mark.gpu


def _run(B, s, V, bf16, seed, scale=3.0):
    L = _lib.lib()
    g = torch.Generator(device="cuda").manual_seed(seed)
    rows = B * s
    logits = torch.randn(rows, V, device="cuda", generator=g) * scale
    tok = torch.randint(0, V, (B, s + 1), device="cuda", generator=g, dtype=torch.int32)
    dl = torch.empty(rows, V, device="cuda", dtype=torch.bfloat16 if bf16 else torch.float32)
    rl = torch.empty(rows, device="cuda")
    inv = 1.0 / (rows * 3)
    assert L.mario_k_softmax_ce(logits.data_ptr(), tok.data_ptr(), s + 1, s, rows, V, inv, dl.data_ptr(),
                                rl.data_ptr(), int(bf16), None) == 0
    torch.cuda.synchronize()
    return logits, tok, dl, rl, inv


@pytest.mark.parametrize("bf16", [1, 0], ids=["bf16", "f32"])
@pytest.mark.parametrize("B,s,V", [(2, 32, 256), (3, 37, 1000), (1, 64, 32000), (2, 40, 50304), (2, 9, 50)])
def test_softmax_ce_matches_fp64(B, s, V, bf16):
    logits, tok, dl, rl, inv = _run(B, s, V, bf16, seed=V + B)
    z = logits.double()
    y = tok[:, 1:].reshape(-1).long()
    lse = torch.logsumexp(z, 1)
    ref_loss = lse - z[torch.arange(z.shape[0], device="cuda"), y]
    assert torch.allclose(rl.double(), ref_loss, rtol=1e-5, atol=1e-5)
    p = torch.softmax(z, 1)
    ref = p.clone()
    ref[torch.arange(z.shape[0], device="cuda"), y] -= 1.0
    ref *= inv
    err = (dl.double() - ref).abs()
    tol = (ref.abs() * (2.0 ** -8 if bf16 else 1e-5)) + 1e-7 * inv
    assert (err <= tol).all(), err.max().item()
    # rows of dlogits sum to 0 (up to storage rounding)
    assert (dl.double().sum(1).abs() <= 2e-2 * inv).all()


def test_softmax_ce_deterministic():
    a = _run(2, 64, 50304, 1, seed=7)
    b = _run(2, 64, 50304, 1, seed=7)
    assert torch.equal(a[2], b[2]) and torch.equal(a[3], b[3])
