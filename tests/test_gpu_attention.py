"""K5/K6 attention through the C-ABI (mario_k_attn_*) vs torch SDPA in fp32 on the same inputs,
at sizes spanning many 64-row tiles with a ragged tail; deterministic backward."""
import math

import pytest
import torch
import torch.nn.functional as F

from paper_conf_ppopp_liultj25_b200 import _lib, api  # noqa: F401  (api registers signatures)

pytestmark = pytest.mark.gpu


def _ref(qkv, B, s, nh, dh, dO):
    h = nh * dh
    x = qkv.float().view(B, s, 3, nh, dh).permute(2, 0, 3, 1, 4)
    q, k, v = (t.detach().clone().requires_grad_(True) for t in x)
    o = F.scaled_dot_product_attention(q, k, v, is_causal=True)
    lse = torch.logsumexp((q @ k.transpose(-1, -2)) / math.sqrt(dh) +
                          torch.triu(torch.full((s, s), float("-inf"), device="cuda"), 1), dim=-1)
    o.backward(dO.float().view(B, s, nh, dh).permute(0, 2, 1, 3))
    dqkv = torch.stack([q.grad, k.grad, v.grad]).permute(1, 3, 0, 2, 4).reshape(B * s, 3 * h)
    return o.permute(0, 2, 1, 3).reshape(B * s, h), lse.permute(1, 0, 2).reshape(nh, B * s), dqkv


@pytest.fixture(params=[-1, 2, 3, 0], ids=["auto_tcgen05", "tcgen05_1q", "tcgen05_2q", "mma_sync"])
def attn_variant(request):
    L = _lib.lib()
    assert L.mario_k_attn_set_variant(request.param) == 0
    yield request.param
    L.mario_k_attn_set_variant(-1)


@pytest.mark.parametrize("B,s,nh,dh", [(2, 200, 3, 128), (1, 1024, 2, 80), (2, 130, 4, 64), (3, 64, 2, 16),
                                       (1, 2048, 2, 128), (2, 300, 2, 64), (1, 128, 1, 128)])
@pytest.mark.parametrize("bf16", [1, 0])
def test_attention_vs_sdpa(B, s, nh, dh, bf16, attn_variant):
    if not bf16 and s > 1024:
        pytest.skip("fp32 SIMT path checked at smaller s")
    g = torch.Generator(device="cuda").manual_seed(s * nh + dh)
    dt = torch.bfloat16 if bf16 else torch.float32
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda", generator=g).to(dt)
    dO = torch.randn(B * s, h, device="cuda", generator=g).to(dt)
    O = torch.empty(B * s, h, device="cuda", dtype=dt)
    lse = torch.empty(nh, B * s, device="cuda")
    L = _lib.lib()
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, bf16, None) == 0
    dqkv = torch.empty(B * s, 3 * h, device="cuda", dtype=dt)
    scr = torch.empty(nh, B * s, device="cuda")
    assert L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dqkv.data_ptr(),
                              scr.data_ptr(), B, s, nh, dh, bf16, None) == 0
    torch.cuda.synchronize()
    o_ref, lse_ref, d_ref = _ref(qkv, B, s, nh, dh, dO)
    tol = 2e-2 if bf16 else 1e-4
    assert (O.float() - o_ref).abs().max().item() <= tol * o_ref.abs().max().item()
    assert (lse - lse_ref).abs().max().item() <= 1e-3
    for part in range(3):
        a = dqkv.float()[:, part * h:(part + 1) * h]
        r = d_ref[:, part * h:(part + 1) * h]
        assert (a - r).abs().max().item() <= tol * r.abs().max().item(), part
    # determinism: a second backward is bitwise identical
    d2 = torch.empty_like(dqkv)
    assert L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d2.data_ptr(),
                              scr.data_ptr(), B, s, nh, dh, bf16, None) == 0
    torch.cuda.synchronize()
    assert torch.equal(d2, dqkv)


@pytest.mark.parametrize("B,s,nh,dh", [(2, 256, 3, 128), (1, 2048, 2, 128), (2, 384, 2, 64), (4, 2048, 16, 128)])
def test_attention_bwd_ds_workspace(B, s, nh, dh):
    """dQ from the stored dS (mario_k_attn_bwd_ws) vs SDPA, bitwise deterministic, and within bf16
    rounding of the recomputing path (both are the c1 attention backward)."""
    L = _lib.lib()
    ws_bytes = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
    nt = s // 128
    assert ws_bytes == B * nh * nt * (nt + 1) * 16384
    g = torch.Generator(device="cuda").manual_seed(7 * s + nh)
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda", generator=g).bfloat16()
    dO = torch.randn(B * s, h, device="cuda", generator=g).bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
    scr = torch.empty(nh, B * s, device="cuda")
    ws = torch.full((ws_bytes,), 0x7f, device="cuda", dtype=torch.uint8)   # garbage: must be fully overwritten
    outs = []
    for _ in range(2):
        d = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
        assert L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d.data_ptr(),
                                     scr.data_ptr(), ws.data_ptr(), ws_bytes, B, s, nh, dh, None) == 0
        outs.append(d)
    d_rc = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
    assert L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d_rc.data_ptr(),
                              scr.data_ptr(), B, s, nh, dh, 1, None) == 0
    torch.cuda.synchronize()
    assert torch.equal(outs[0], outs[1])
    # dK, dV come from the same kernel either way
    assert torch.equal(outs[0][:, h:], d_rc[:, h:])
    if s <= 2048 and B * nh <= 4:
        _, _, d_ref = _ref(qkv, B, s, nh, dh, dO)
        for part in range(3):
            a = outs[0].float()[:, part * h:(part + 1) * h]
            r = d_ref[:, part * h:(part + 1) * h]
            assert (a - r).abs().max().item() <= 2e-2 * r.abs().max().item(), part
    dq, dq_rc = outs[0].float()[:, :h], d_rc.float()[:, :h]
    assert (dq - dq_rc).abs().max().item() <= 1e-2 * dq_rc.abs().max().item()


@pytest.mark.parametrize("B,s,nh,dh", [(1, 16384, 2, 128), (1, 8192, 2, 64)])
def test_attention_long_sequence(B, s, nh, dh):
    """cfg 5's sequence length (LLaMA2-13B at s = 16384): the tcgen05 forward and the
    recomputing backward (fa_bwd_dq_pers: the dS image would exceed its 1 GiB bound there) vs SDPA on
    reduced heads; bitwise-deterministic backward."""
    g = torch.Generator(device="cuda").manual_seed(s + nh)
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda", generator=g).bfloat16()
    dO = torch.randn(B * s, h, device="cuda", generator=g).bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    L = _lib.lib()
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
    scr = torch.empty(nh, B * s, device="cuda")
    outs = []
    for _ in range(2):
        d = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
        assert L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d.data_ptr(),
                                  scr.data_ptr(), B, s, nh, dh, 1, None) == 0
        outs.append(d)
    torch.cuda.synchronize()
    assert torch.equal(outs[0], outs[1])
    o_ref, lse_ref, d_ref = _ref(qkv, B, s, nh, dh, dO)
    assert (O.float() - o_ref).abs().max().item() <= 2e-2 * o_ref.abs().max().item()
    assert (lse - lse_ref).abs().max().item() <= 1e-3
    for part in range(3):
        a = outs[0].float()[:, part * h:(part + 1) * h]
        r = d_ref[:, part * h:(part + 1) * h]
        assert (a - r).abs().max().item() <= 2e-2 * r.abs().max().item(), part
