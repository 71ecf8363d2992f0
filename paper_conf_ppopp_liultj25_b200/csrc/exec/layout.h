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
// Norm outputs (A, A2) and the MLP activation (G = gelu(Z) / M = swiglu(GU)) are NOT stored:
// the backward recomputes them from H_in/H1 (+ stats) and Z/GU (cheap, bandwidth-bound).
struct LayerAct {
  size_t H_in, st1, QKV, O, LSE, H1, st2, Z;   // GPT: Z = [T,f]; LLaMA: Z = GU [T,2f]
  size_t bytes;
};
LayerAct layer_act_layout(const mario_model& m);
// Per-layer transients of the forward (reused layer after layer): A, A2 [T,h], G|M [T,f].
struct LayerTrans {
  size_t A, A2, G;
  size_t bytes;
};
LayerTrans layer_trans_layout(const mario_model& m);

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
  size_t dH[3], dA, dQKV, dO, dZ, dM, Dsc, sort, Arec;   // dM doubles as the G/M recompute buffer
  size_t dS, dS_bytes;   // attention dS image (bf16, when the shape allows it and it is <= 1 GiB; else 0 bytes)
  size_t bytes;
};
BwScratch bw_scratch_layout(const mario_model& m);
size_t bw_scratch_bytes(const mario_model& m);
size_t logits_bytes(const mario_model& m);                      // fp32 [T, V]
size_t weight_copy_bytes(const mario_model& m, const std::vector<int32_t>& param_idx);

}  // namespace mario
