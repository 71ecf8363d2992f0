// Static arena layout of one rank: every buffer the executor uses has a
// fixed offset computed once from the plan, so the planner's memory model is exact
// (reading A13) and nothing is allocated inside the iteration.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>

#include "../../../include/mario.h"

namespace mario {

inline size_t align_up(size_t x, size_t a = 256) { return (x + a - 1) / a * a; }

// Offsets (bytes) of the tensors one decoder layer saves for its backward, inside an
// activation set. T = mbs * s tokens, E = element size of the compute dtype.
struct LayerAct {
  size_t H_in, st1, A, QKV, O, LSE, H1, st2, A2, Z, G;   // GPT: Z,G = [T,f]; LLaMA: Z = GU [T,2f], G = M [T,f]
  size_t bytes;
};
LayerAct layer_act_layout(const mario_model& m);

// Head (last virtual stage): final-norm stats and output, dlogits.
struct HeadAct {
  size_t H_last, stf, Hf, dlogits;
  size_t bytes;
};
HeadAct head_act_layout(const mario_model& m);

size_t elt_size(const mario_model& m);
size_t tokens_per_micro(const mario_model& m);
size_t stage_input_bytes(const mario_model& m);                  // [T, h]
size_t act_set_bytes(const mario_model& m, int k, int K);        // lps layers (+ head)
size_t cfw_work_bytes(const mario_model& m, int k, int K);       // transient CFW scratch
// Backward scratch (shared by every BW of the rank): rotating dH buffers and per-layer grads.
struct BwScratch {
  size_t dH[3], dA, dQKV, dO, dZ, dM, Dsc, sort;
  size_t bytes;
};
BwScratch bw_scratch_layout(const mario_model& m);
size_t bw_scratch_bytes(const mario_model& m);
size_t logits_bytes(const mario_model& m);                      // fp32 [T, V]
size_t weight_copy_bytes(const mario_model& m, const std::vector<int32_t>& param_idx);

}  // namespace mario
