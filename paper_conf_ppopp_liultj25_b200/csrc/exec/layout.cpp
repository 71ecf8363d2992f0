#include "layout.h"

#include <algorithm>

#include "../plan/model.h"

namespace mario {
size_t flash_attn_bwd_ds_bytes(int dh, int B, int s, int nh);           // kernels/attn_tc.cu
size_t flash_attn_pad_bytes(int dh, int B, int s, int nh, int bwd);      // kernels/attn_mma.cu
}

namespace mario {

size_t elt_size(const mario_model& m) { return m.dtype == MARIO_BF16 ? 2 : 4; }
size_t tokens_per_micro(const mario_model& m) { return static_cast<size_t>(m.micro_batch) * m.seq_len; }

LayerAct layer_act_layout(const mario_model& m, bool store_act) {
  const size_t T = tokens_per_micro(m), E = elt_size(m), h = m.hidden, f = m.ffn_hidden;
  const size_t nh = m.n_heads;
  LayerAct L{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
  L.H_in = take(T * h * E);
  L.st1 = take(T * 2 * 4);          // mean, rstd (fp32)
  L.QKV = take(T * 3 * h * E);
  L.O = take(T * h * E);
  L.LSE = take(nh * T * 4);
  L.H1 = take(T * h * E);
  L.st2 = take(T * 2 * 4);
  L.Z = take(T * (m.family == MARIO_GPT ? f : 2 * f) * E);   // GPT: Z; LLaMA: GU = [gate | up]
  L.A = take(store_act ? T * h * E : 0);
  L.A2 = take(store_act ? T * h * E : 0);
  L.G = take(store_act ? T * f * E : 0);
  L.bytes = o;
  return L;
}

LayerTrans layer_trans_layout(const mario_model& m, bool store_act) {
  const size_t T = tokens_per_micro(m), E = elt_size(m), h = m.hidden, f = m.ffn_hidden;
  LayerTrans L{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
  L.A = take(store_act ? 0 : T * h * E);
  L.A2 = take(store_act ? 0 : T * h * E);
  L.G = take(store_act ? 0 : T * f * E);
  L.attn_pad_bytes = m.dtype == MARIO_BF16 ? flash_attn_pad_bytes(h / m.n_heads, m.micro_batch, m.seq_len, m.n_heads, 0) : 0;
  L.attn_pad = take(L.attn_pad_bytes);
  L.bytes = o;
  return L;
}

HeadAct head_act_layout(const mario_model& m) {
  const size_t T = tokens_per_micro(m), E = elt_size(m), h = m.hidden, V = m.vocab;
  HeadAct H{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
  (void)V;
  H.H_last = take(T * h * E);
  H.stf = take(T * 2 * 4);
  H.dHf = take(T * h * E);
  H.bytes = o;
  return H;
}

HeadScratch head_scratch_layout(const mario_model& m) {
  const size_t T = tokens_per_micro(m), E = elt_size(m), h = m.hidden, V = m.vocab;
  const size_t budget = static_cast<size_t>(640) << 20;   // logits + dlogits of one chunk
  size_t n = 1, rows = T;
  while (rows * V * (4 + E) > budget && rows > 128) {
    n *= 2;
    rows = (T + n - 1) / n;
    rows = (rows + 127) / 128 * 128;
  }
  HeadScratch H{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
  H.rows = static_cast<int>(rows);
  H.Hf = take(T * h * E);
  H.logits = take(rows * V * 4);
  H.dlog = take(rows * V * E);
  H.bytes = o;
  return H;
}

size_t stage_input_bytes(const mario_model& m) { return align_up(tokens_per_micro(m) * m.hidden * elt_size(m)); }

size_t act_set_bytes(const mario_model& m, int k, int K, bool store_act) {
  const int lps = m.n_layers / K;
  size_t b = layer_act_layout(m, store_act).bytes * lps;
  if (k == K - 1) b += head_act_layout(m).bytes;
  return b;
}

size_t cfw_work_bytes(const mario_model& m, int k, int K, bool store_act) {
  // one layer's stored + transient tensors + the two running residual buffers (+ head)
  size_t b = layer_act_layout(m, store_act).bytes + layer_trans_layout(m, store_act).bytes + 2 * stage_input_bytes(m);
  if (k == K - 1) b += head_act_layout(m).bytes;
  return b;
}

BwScratch bw_scratch_layout(const mario_model& m, bool store_act) {
  const size_t T = tokens_per_micro(m), E = elt_size(m), h = m.hidden, f = m.ffn_hidden;
  BwScratch b{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
  for (int i = 0; i < 3; ++i) b.dH[i] = take(T * h * E);
  b.dA = take(T * h * E);
  b.dQKV = take(T * 3 * h * E);
  b.dO = take(T * h * E);
  b.dZ = take(T * 2 * f * E);
  b.dM = take(T * f * E);
  b.Dsc = take(static_cast<size_t>(m.n_heads) * T * 4);
  b.sort = take(T * 8 * 2);
  b.Arec = take(store_act ? 0 : T * h * E);
  for (int i = 0; i < 2; ++i) b.dH32[i] = take(m.dtype == MARIO_BF16 ? T * h * 4 : 0);
  b.attn_pad_bytes = m.dtype == MARIO_BF16 ? flash_attn_pad_bytes(h / m.n_heads, m.micro_batch, m.seq_len, m.n_heads, 1) : 0;
  b.attn_pad = take(b.attn_pad_bytes);
  // the attention backward's dS image (fa_bwd_dq_img: dQ from the stored dS, no S/dP recompute);
  // only where it stays small next to the rest of the scratch (not at s = 16384)
  b.dS_bytes = 0;
  if (m.dtype == MARIO_BF16) {
    const size_t ds = flash_attn_bwd_ds_bytes(h / m.n_heads, m.micro_batch, m.seq_len, m.n_heads);
    if (ds > 0 && ds <= (static_cast<size_t>(1) << 30)) b.dS_bytes = ds;
  }
  b.dS = take(b.dS_bytes);
  b.bytes = o;
  return b;
}

size_t bw_scratch_bytes(const mario_model& m, bool store_act) { return bw_scratch_layout(m, store_act).bytes; }

size_t logits_bytes(const mario_model& m) { return head_scratch_layout(m).bytes; }

size_t weight_copy_bytes(const mario_model& m, const std::vector<int32_t>& idx) {
  if (m.dtype != MARIO_BF16) return 0;
  auto ps = model_params(m);
  size_t b = 0;
  for (int32_t i : idx) if (ps[i].is_matrix()) b += align_up(ps[i].numel() * 2);
  return b;
}

}  // namespace mario
