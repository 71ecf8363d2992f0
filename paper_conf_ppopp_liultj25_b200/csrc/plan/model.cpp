#include "model.h"

namespace mario {

std::vector<ParamSpec> model_params(const mario_model& m) {
  std::vector<ParamSpec> out;
  const int64_t h = m.hidden, f = m.ffn_hidden, V = m.vocab;
  if (m.family == MARIO_GPT) {
    out.push_back({"wte", {V, h}});
    out.push_back({"wpe", {m.seq_len, h}});
  } else {
    out.push_back({"emb", {V, h}});
  }
  for (int l = 0; l < m.n_layers; ++l) {
    const std::string p = "h" + std::to_string(l) + ".";
    if (m.family == MARIO_GPT) {
      out.push_back({p + "ln1.g", {h}}); out.push_back({p + "ln1.b", {h}});
      out.push_back({p + "qkv.w", {3 * h, h}}); out.push_back({p + "qkv.b", {3 * h}});
      out.push_back({p + "proj.w", {h, h}}); out.push_back({p + "proj.b", {h}});
      out.push_back({p + "ln2.g", {h}}); out.push_back({p + "ln2.b", {h}});
      out.push_back({p + "fc1.w", {f, h}}); out.push_back({p + "fc1.b", {f}});
      out.push_back({p + "fc2.w", {h, f}}); out.push_back({p + "fc2.b", {h}});
    } else {
      out.push_back({p + "n1.g", {h}});
      out.push_back({p + "qkv.w", {3 * h, h}});
      out.push_back({p + "o.w", {h, h}});
      out.push_back({p + "n2.g", {h}});
      out.push_back({p + "gu.w", {2 * f, h}});
      out.push_back({p + "down.w", {h, f}});
    }
  }
  if (m.family == MARIO_GPT) {
    out.push_back({"lnf.g", {h}}); out.push_back({"lnf.b", {h}});
    if (!m.tie_embeddings) out.push_back({"head.w", {V, h}});
  } else {
    out.push_back({"nf.g", {h}});
    out.push_back({"out.w", {V, h}});
  }
  return out;
}

static int params_per_layer(const mario_model& m) { return m.family == MARIO_GPT ? 12 : 6; }

std::vector<int32_t> stage_param_indices(const mario_model& m, int k, int K) {
  std::vector<int32_t> idx;
  const int n_embed = m.family == MARIO_GPT ? 2 : 1;
  const int ppl = params_per_layer(m);
  const int lps = m.n_layers / K;
  if (k == 0) for (int i = 0; i < n_embed; ++i) idx.push_back(i);
  for (int l = k * lps; l < (k + 1) * lps; ++l)
    for (int j = 0; j < ppl; ++j) idx.push_back(n_embed + l * ppl + j);
  if (k == K - 1) {
    const int base = n_embed + m.n_layers * ppl;
    if (m.family == MARIO_GPT) {
      idx.push_back(base); idx.push_back(base + 1);
      if (!m.tie_embeddings) idx.push_back(base + 2);
      else if (K > 1) idx.push_back(0);  // own copy of the tied wte for the LM head
    } else {
      idx.push_back(base); idx.push_back(base + 1);
    }
  }
  return idx;
}

static double layer_fwd_flops(const mario_model& m) {
  const double T = static_cast<double>(m.micro_batch) * m.seq_len;
  const double h = m.hidden, f = m.ffn_hidden, s = m.seq_len;
  const double lin = m.family == MARIO_GPT ? (4 * h * h + 2 * h * f) : (4 * h * h + 3 * h * f);
  // causal attention: QK^T and PV over half the s x s scores each: 2 * (2*s*s*h/2) per sample
  return 2.0 * T * lin + 2.0 * m.micro_batch * s * s * h;
}

double stage_fwd_flops(const mario_model& m, int k, int K) {
  const double T = static_cast<double>(m.micro_batch) * m.seq_len;
  double fl = layer_fwd_flops(m) * (m.n_layers / K);
  if (k == K - 1) fl += 2.0 * T * m.hidden * m.vocab;
  return fl;
}

double model_flops_per_sample(const mario_model& m) {
  const double s = m.seq_len, h = m.hidden, f = m.ffn_hidden, L = m.n_layers;
  const double P = m.family == MARIO_GPT ? (4 * h * h + 2 * h * f) : (4 * h * h + 3 * h * f);
  return 3.0 * (L * (2 * s * P + 4 * s * s * h) + 2 * s * h * m.vocab);
}

const char* validate_model(const mario_model& m) {
  if (m.family != MARIO_GPT && m.family != MARIO_LLAMA) return "unknown family";
  if (m.n_layers <= 0 || m.hidden <= 0 || m.n_heads <= 0 || m.ffn_hidden <= 0 || m.vocab <= 0 ||
      m.seq_len <= 0 || m.micro_batch <= 0) return "non-positive model dimension";
  if (m.hidden % m.n_heads) return "hidden % n_heads != 0";
  const int dh = m.hidden / m.n_heads;
  if (dh != 16 && dh != 32 && dh != 64 && dh != 80 && dh != 128) return "head_dim must be 16/32/64/80/128";
  if (m.dtype != MARIO_F32 && m.dtype != MARIO_BF16) return "unknown dtype";
  if (m.hidden % 8 || m.ffn_hidden % 8 || m.vocab % 8) return "hidden, ffn_hidden, vocab must be multiples of 8";
  return nullptr;
}

}  // namespace mario
