// Byte offsets of every executor buffer inside one rank's caller-provided workspace.
#pragma once
#include <cstddef>
#include <vector>

#include "../plan/plan_obj.h"
#include "layout.h"

namespace mario {

constexpr int kRedBlocks = 128;   // row blocks of the deterministic two-pass column reductions

struct Arena {
  std::vector<size_t> wcopy;      // per packed tensor: offset of its bf16 copy (SIZE_MAX = none)
  size_t ckpt = 0, ckpt_stride = 0; int n_ckpt = 0;
  size_t act = 0, act_stride = 0; int n_act = 0;
  size_t cfw = 0, bw = 0, logits = SIZE_MAX;
  size_t sa = 0, sg = 0, rg = 0, msg_stride = 0; int n_sa = 0, n_sg = 0, n_rg = 0;
  size_t tokens = 0, loss = 0, red = 0, red_bytes = 0;
  size_t rope = SIZE_MAX;         // LLaMA bf16: RoPE (cos, sin) table [s][dh/2], rebuilt each iteration
  size_t total = 0;
};

Arena make_arena(const PlanObj& P, int dev, const PlanObj::Pools& pools);
size_t red_width(const mario_model& m);

}  // namespace mario
