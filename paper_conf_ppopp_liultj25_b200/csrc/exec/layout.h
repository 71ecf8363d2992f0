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
// With the plan's `store_act` set (the default when the memory budget allows it) the activation set
// also keeps what the backward would otherwise recompute: the norm outputs A, A2 [T,h] (the QKV /
// MLP-input GEMM operands) and the MLP activation G = gelu(Z) (GPT, as the forward's fc1 epilogue
// computed it from the fp32 pre-activation) / M = swiglu(GU) (LLaMA) [T,f]: +(2h + f) per token and
// layer, and the backward drops two norm_apply passes, the G output of the fc2-dgrad epilogue (GPT) or
// the swiglu recompute (LLaMA). Otherwise (lean set) they are transients and the backward recomputes
// them from H_in/H1 with the stored (mean, rstd), and from Z/GU.
struct LayerAct {
  size_t H_in, st1, QKV, O, LSE, H1, st2, Z;   // GPT: Z = [T,f]; LLaMA: Z = GU [T,2f]
  size_t A, A2, G;                             // store_act only (else 0 bytes, offset unused)
  size_t bytes;
};
LayerAct layer_act_layout(const mario_model& m, bool store_act);
// Per-layer transients of the forward (reused layer after layer): A, A2 [T,h], G|M [T,f] (lean set
// only).
struct LayerTrans {
  size_t A, A2, G;
  size_t attn_pad, attn_pad_bytes;   // padded-head-dim attention workspace (bf16, dh not 64 / 128), else 0 bytes
                                     // (test the size: with store_act the offset itself can be 0)
  size_t bytes;
};
LayerTrans layer_trans_layout(const mario_model& m, bool store_act);

// Head (last virtual stage), what its BW needs: the last layer's output, the final-norm stats and
// dHf = dloss/dHf. The logits never outlive the FW / RC that computes them (K13, fused head): the
// head runs over token chunks (logits chunk -> softmax-CE -> dlogits chunk -> head dgrad rows of dHf
// and head wgrad) inside the forward, since the loss ends the graph (BW needs only the
// gradient of the stage output).
struct HeadAct {
  size_t H_last, stf, dHf;
  size_t bytes;
};
HeadAct head_act_layout(const mario_model& m);
// Scratch of the fused head (per device with the last virtual stage): Hf [T, h], and a chunk of
// `rows` tokens of fp32 logits [rows, V] and dlogits [rows, V] (compute dtype).
struct HeadScratch {
  size_t Hf, logits, dlog;
  int rows;      // token rows per chunk (a power-of-2 split of T, multiple of 128 where T allows)
  size_t bytes;
};
HeadScratch head_scratch_layout(const mario_model& m);

size_t elt_size(const mario_model& m);
size_t tokens_per_micro(const mario_model& m);
size_t stage_input_bytes(const mario_model& m);                  // [T, h]
size_t act_set_bytes(const mario_model& m, int k, int K, bool store_act);    // lps layers (+ head)
size_t cfw_work_bytes(const mario_model& m, int k, int K, bool store_act);   // transient CFW scratch
// Backward scratch (shared by every BW of the rank): rotating dH buffers and per-layer grads.
struct BwScratch {
  size_t dH[3], dA, dQKV, dO, dZ, dM, Dsc, sort;   // dM doubles as the G/M recompute buffer
  size_t Arec;      // lean set: the recomputed norm output (0 bytes with store_act)
  size_t dH32[2];   // bf16 mode: the fp32 residual-gradient stream (reading A30); 0 bytes in fp32 mode
  size_t attn_pad, attn_pad_bytes;  // padded-head-dim attention backward workspace (bf16, dh not 64 / 128), else 0 bytes
  size_t dS, dS_bytes;   // attention dS image (bf16, when the shape allows it and it is <= 1 GiB; else 0 bytes)
  size_t bytes;
};
BwScratch bw_scratch_layout(const mario_model& m, bool store_act);
size_t bw_scratch_bytes(const mario_model& m, bool store_act);
size_t logits_bytes(const mario_model& m);                      // head_scratch_layout(m).bytes
size_t weight_copy_bytes(const mario_model& m, const std::vector<int32_t>& param_idx);

}  // namespace mario
