#include "arena.h"

#include <algorithm>
#include <cstdint>

namespace mario {

size_t red_width(const mario_model& m) {
  return std::max<size_t>({static_cast<size_t>(3) * m.hidden, static_cast<size_t>(2) * m.ffn_hidden,
                           static_cast<size_t>(m.hidden)});
}

Arena make_arena(const PlanObj& P, int dev, const PlanObj::Pools& pools) {
  const mario_model& m = P.model;
  const int K = P.pp.K();
  Arena a;
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes, 1024); return r; };
  const auto& rp = P.rank_params[dev];
  a.wcopy.assign(rp.idx.size(), SIZE_MAX);
  if (m.dtype == MARIO_BF16)
    for (size_t j = 0; j < rp.idx.size(); ++j)
      if (P.params[rp.idx[j]].is_matrix()) a.wcopy[j] = take(P.params[rp.idx[j]].numel() * 2);
  size_t act_max = 0, cfw_max = 0;
  bool has_last = false;
  for (int p = 0; p < P.pp.parts(); ++p) {
    int k = P.pp.vstage(dev, p);
    act_max = std::max(act_max, act_set_bytes(m, k, K, P.store_act));
    cfw_max = std::max(cfw_max, cfw_work_bytes(m, k, K, P.store_act));
    has_last = has_last || k == K - 1;
  }
  a.ckpt_stride = stage_input_bytes(m);
  a.n_ckpt = pools.ckpt;
  a.ckpt = take(a.ckpt_stride * std::max(1, a.n_ckpt));
  a.act_stride = align_up(act_max, 1024);
  a.n_act = pools.act;
  a.act = take(a.act_stride * std::max(1, a.n_act));
  a.cfw = take(cfw_max);
  a.bw = take(bw_scratch_bytes(m, P.store_act));
  if (has_last) a.logits = take(logits_bytes(m));
  a.msg_stride = stage_input_bytes(m);
  a.n_sa = pools.send_act; a.n_sg = pools.send_grad; a.n_rg = pools.recv_grad;
  a.sa = take(a.msg_stride * std::max(1, a.n_sa));
  a.sg = take(a.msg_stride * std::max(1, a.n_sg));
  a.rg = take(a.msg_stride * std::max(1, a.n_rg));
  a.tokens = take(static_cast<size_t>(P.pp.N) * m.micro_batch * (m.seq_len + 1) * 4);
  a.loss = take(static_cast<size_t>(P.pp.N) * P.pp.parts() * 8 + tokens_per_micro(m) * 4);
  a.red_bytes = static_cast<size_t>(kRedBlocks) * red_width(m) * 4 * 2;
  a.red = take(a.red_bytes);
  if (m.family == MARIO_LLAMA && m.dtype == MARIO_BF16)
    a.rope = take(static_cast<size_t>(m.seq_len) * (m.hidden / m.n_heads / 2) * 8);
  a.total = o;
  return a;
}

}  // namespace mario
