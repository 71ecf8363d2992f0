// Model description, partition into virtual stages and the packed parameter layout.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../../include/mario.h"

namespace mario {

struct ParamSpec {
  std::string name;
  std::vector<int64_t> shape;
  int64_t numel() const { int64_t n = 1; for (auto s : shape) n *= s; return n; }
  bool is_matrix() const { return shape.size() == 2; }
};

// Global parameters in canonical order (synth.param_shapes mirrors it).
std::vector<ParamSpec> model_params(const mario_model& m);

// Indices (into model_params) held by virtual stage k of K (reading A8: even layers,
// embedding on stage 0, final norm + head on stage K-1; a tied GPT head keeps its own wte
// copy on the last stage when K > 1).
std::vector<int32_t> stage_param_indices(const mario_model& m, int k, int K);

// Algorithmic forward FLOPs (causal attention) of one micro-batch on virtual stage k.
double stage_fwd_flops(const mario_model& m, int k, int K);
// Megatron/PaLM model FLOPs per sample (non-causal attention, no recompute), SURVEY §8(d) d3.
double model_flops_per_sample(const mario_model& m);

const char* validate_model(const mario_model& m);

}  // namespace mario
