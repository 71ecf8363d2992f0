// The opaque mario_plan object (immutable after mario_plan returns).
#pragma once
#include <atomic>
#include <cstdint>
#include <string>
#include <map>
#include <vector>

#include "model.h"
#include "plan.h"

inline uint64_t mario_next_plan_serial() {
  static std::atomic<uint64_t> next{1};
  return next.fetch_add(1);
}

struct mario_plan {
  // never reused (unlike the object's address): keys the executor's CUDA-graph cache
  const uint64_t serial = mario_next_plan_serial();
  mario_model model{};
  mario::plan::Pipe pp;
  int level = MARIO_LEVEL_MARIO;
  uint64_t budget = 0;
  int unckpt_tail = 0;   // MARIO_LEVEL_BUDGET: devices S-k .. S-1 left un-checkpointed (A28)
  bool store_act = true;   // activation sets keep the norm outputs A, A2 (exec/layout.h); lean if the budget needs it
  int lps = 1;                       // layers per virtual stage
  mario::plan::Lists lists;
  std::vector<std::vector<mario_instr>> instrs;   // per device, exported IR
  mario::plan::SimCosts costs;
  mario::plan::SimResult sim;
  mario::plan::MemResult mem;
  // exported simulator arrays
  std::vector<double> busy;
  std::vector<uint64_t> peak;
  std::vector<int32_t> live_act, live_ckpt;
  // parameters
  std::vector<mario::ParamSpec> params;
  std::vector<std::string> param_names;
  std::map<std::string, int> param_index;   // name -> global index (executor weight lookups)
  struct RankParams {
    std::vector<int32_t> idx;        // global param index per packed tensor
    std::vector<uint64_t> off, cnt;  // element offset / count in the packed buffer
    std::vector<int32_t> part;       // part (virtual stage slot) owning the tensor
    uint64_t total = 0;
  };
  std::vector<RankParams> rank_params;
  // executor pools per device (slot counts) for multi-process and loopback execution
  struct Pools { int ckpt = 0, act = 0, send_act = 0, send_grad = 0, recv_grad = 0; };
  std::vector<Pools> pools_mp, pools_lb;
  // send slot of every message, per device: (micro, part) -> slot, held from its FW/CFW (BW) until
  // the receiver's RA (RG). Assigned once along a valid execution order of the plan's DAG, so an
  // executor that reuses a slot only after its previous message was consumed adds no cycle:
  //  - sa_slot / sg_slot (pools_mp): along peer_order, the simulator's timeline (instructions in
  //    order of their simulated times), used by the per-rank executors (peer transport, NCCL);
  //  - sa_slot_lb / sg_slot_lb (pools_lb): along loopback_order, used by the loopback executor,
  //    which copies a message out at the receiver's RA in that order.
  std::vector<std::map<std::pair<int, int>, int>> sa_slot, sg_slot, sa_slot_lb, sg_slot_lb;
  std::vector<std::pair<int, int>> peer_order;   // (device, list index) in simulated-time order
  std::vector<uint64_t> workspace_mp, workspace_lb;  // bytes per device
  // global execution order used by loopback (device, list index), round-robin like the simulator
  std::vector<std::pair<int, int>> loopback_order;
  std::string serialized;
  std::vector<std::vector<mario_commop>> comm_ops;   // per rank, issue order
  // world-rank programs for PP x DP (key: (dp, world rank)), built on first use
  mutable std::map<std::pair<int, int>, std::vector<mario_commop>> comm_ops_dp;
};
typedef struct mario_plan PlanObj;
const std::vector<mario_commop>& comm_program_dp(const PlanObj& P, int dp, int rank);   // plan_api.cpp
namespace mario { void exec_forget_plan(uint64_t serial); }   // executor.cu: drop cached graphs
