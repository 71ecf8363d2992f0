// Planner internals: IR, virtual pipeline, base schedules, the four graph passes and the
// dynamic-programming simulator (§5.1-§5.2). Host-only C++17.
#pragma once
#include <cstdint>
#include <string>
#include <utility>
#include <vector>

#include "../../../include/mario.h"

namespace mario {
namespace plan {

enum Op : int32_t { FW = MARIO_OP_FW, CFW = MARIO_OP_CFW, RC = MARIO_OP_RC, BW = MARIO_OP_BW,
                    SA = MARIO_OP_SA, RA = MARIO_OP_RA, SG = MARIO_OP_SG, RG = MARIO_OP_RG };

inline bool is_compute(int op) { return op == FW || op == CFW || op == RC || op == BW; }
inline bool is_recv(int op) { return op == RA || op == RG; }
inline bool is_send(int op) { return op == SA || op == SG; }
const char* op_name(int op);

struct Instr {
  int32_t op, m, p;
  bool operator==(const Instr& o) const { return op == o.op && m == o.m && p == o.p; }
  bool operator!=(const Instr& o) const { return !(*this == o); }
};
using List = std::vector<Instr>;
using Lists = std::vector<List>;

// Virtual pipeline geometry.
struct Pipe {
  int scheme = MARIO_1F1B, S = 1, N = 1, v = 1;
  int K() const { return scheme == MARIO_INTERLEAVE ? S * v : S; }
  int parts() const { return scheme == MARIO_INTERLEAVE ? v : scheme == MARIO_CHIMERA ? 2 : 1; }
  int part_of_micro(int m) const {
    if (scheme != MARIO_CHIMERA) return 0;
    return (m % S) < S / 2 ? 0 : 1;
  }
  int vstage(int d, int p) const {
    if (scheme == MARIO_1F1B) return d;
    if (scheme == MARIO_INTERLEAVE) return p * S + d;
    return p == 0 ? d : S - 1 - d;
  }
  std::pair<int, int> device_part(int k, int pipeline) const {
    if (scheme == MARIO_1F1B) return {k, 0};
    if (scheme == MARIO_INTERLEAVE) return {k % S, k / S};
    return pipeline == 0 ? std::make_pair(k, 0) : std::make_pair(S - 1 - k, 1);
  }
};

// Algorithm 1: returns false if the target lies outside the pipeline.
bool find_inst(const Pipe& pp, int d, int m, int p, int t, bool nxt, int* d_o, int* p_o);

Lists build_base(const Pipe& pp);
// keep: devices left un-checkpointed in their base order (budget extension, reading A28)
Lists pass1_apply_checkpoint(const Lists& in, const std::vector<bool>& keep = {});
Lists pass2_overlap_recompute(const Lists& in);
Lists pass3_remove_redundancy(const Lists& in);

struct SimCosts {
  std::vector<double> fw, bw, rc;         // per virtual stage (ms)
  double comm_act = 0, comm_grad = 0;     // per message (ms), per virtual-stage boundary
  std::vector<double> act, ckpt, work;    // per virtual stage (bytes), memory walk
  std::vector<double> static_bytes;       // per device
};

struct SimResult {
  bool ok = false;
  double makespan = 0;
  std::vector<double> busy;
  std::vector<std::vector<double>> start, finish;  // per device, per compute instr in list order
};
SimResult simulate(const Pipe& pp, const Lists& L, const SimCosts& c);

struct MemResult {
  std::vector<double> peak;     // static + dynamic
  std::vector<int> max_live_act, max_live_ckpt;
};
MemResult memory_walk(const Pipe& pp, const Lists& L, const SimCosts& c);

Lists pass4_prepose_forward(const Pipe& pp, const Lists& in, const SimCosts& c, double budget, int max_rounds = 8);

}  // namespace plan
}  // namespace mario
