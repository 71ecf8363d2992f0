// mario_tune: the schedule tuner of PAPER.md §5.3 (Eq. 1), a grid search that scores
// every configuration with the planner's simulator (F = 0 if the simulated peak > budget).
#include <algorithm>
#include <vector>

#include "../plan/model.h"
#include "../plan/plan_obj.h"
#include "status.h"

using namespace mario;

extern "C" mario_status mario_tune(const mario_model* model, int32_t devices, int32_t global_batch,
                                   uint64_t mem_budget_bytes, const mario_tune_costs* costs,
                                   mario_tune_result* results, int32_t cap, int32_t* n, int32_t* best) {
  return guard([&]() -> mario_status {
    if (!model || !n || !best || devices < 1 || global_batch < 1) return set_error(MARIO_EINVAL, "bad argument");
    std::vector<int> mbs_list = {1, 2, 4, 8};
    if (costs && costs->n_mbs > 0) mbs_list.assign(costs->mbs, costs->mbs + costs->n_mbs);
    std::vector<mario_tune_result> out;
    const int schemes[3] = {MARIO_1F1B, MARIO_INTERLEAVE, MARIO_CHIMERA};
    const int pp_min = std::min(4, devices);
    for (int sch : schemes) {
      const int v = sch == MARIO_INTERLEAVE ? 2 : 1;
      for (int pp = pp_min; pp <= devices; ++pp) {
        if (devices % pp) continue;
        const int dp = devices / pp;
        if (model->n_layers % (pp * v)) continue;
        if (sch == MARIO_CHIMERA && pp % 2) continue;
        if (sch == MARIO_INTERLEAVE && pp < 2) continue;
        for (size_t mi = 0; mi < mbs_list.size(); ++mi) {
          const int mbs = mbs_list[mi];
          if (global_batch % (dp * mbs)) continue;
          const int N = global_batch / (dp * mbs);
          if ((sch == MARIO_INTERLEAVE || sch == MARIO_CHIMERA) && N % pp) continue;
          mario_model m = *model;
          m.micro_batch = mbs;
          if (validate_model(m)) continue;
          const int K = pp * v, lps = m.n_layers / K;
          std::vector<double> fw(K), bw(K), rc(K);
          for (int k = 0; k < K; ++k) {
            double lf, lb, hf = 0, hb = 0;
            if (costs && costs->layer_fw_ms && costs->layer_bw_ms) {
              lf = costs->layer_fw_ms[mi];
              lb = costs->layer_bw_ms[mi];
              if (k == K - 1 && costs->head_fw_ms) hf = costs->head_fw_ms[mi];
              if (k == K - 1 && costs->head_bw_ms) hb = costs->head_bw_ms[mi];
            } else {
              const double f = stage_fwd_flops(m, k, K) / 1e12;   // ms at 1 PFLOP/s
              lf = f / lps;
              lb = 2 * lf;
              hf = hb = 0;   // already included in stage_fwd_flops for the last stage
            }
            fw[k] = lps * lf + hf;
            bw[k] = lps * lb + hb;
            rc[k] = fw[k];
          }
          mario_costs mc{fw.data(), bw.data(), rc.data(), costs ? costs->p2p_alpha_ms : 0.01,
                         costs ? costs->p2p_GBps : 700.0, nullptr, nullptr, nullptr, -1.0};
          // the budget-driven level (A28) joins the grid when there is a budget to drive it
          std::vector<int> levels{MARIO_LEVEL_BASE, MARIO_LEVEL_MARIO};
          if (mem_budget_bytes > 0) levels.push_back(MARIO_LEVEL_BUDGET);
          for (int level : levels) {
            PlanObj* P = nullptr;
            mario_tune_result r{sch, pp, v, dp, mbs, N, level, 0, 0.0, 0.0, 0.0, 0};
            const uint64_t plan_budget = level == MARIO_LEVEL_BUDGET ? mem_budget_bytes : 0;
            if (mario_plan(&m, pp, N, sch, v, plan_budget, level, &mc, &P) == MARIO_OK) {
              mario_sim sim;
              mario_plan_simulate(P, &sim);
              r.makespan_ms = sim.makespan_ms;
              r.bubble_ratio = sim.bubble_ratio;
              r.peak_bytes = *std::max_element(sim.peak_bytes, sim.peak_bytes + sim.n_dev);
              r.feasible = (mem_budget_bytes == 0 || r.peak_bytes <= mem_budget_bytes) ? 1 : 0;
              const double eff = dp > 1 ? (costs && costs->dp_efficiency > 0 ? costs->dp_efficiency : 0.95) : 1.0;
              r.samples_per_s = r.feasible ? global_batch / (sim.makespan_ms / 1e3) * eff : 0.0;   // F = 0 if OOM
              mario_plan_destroy(P);
            }
            out.push_back(r);
          }
        }
      }
    }
    *n = static_cast<int32_t>(out.size());
    *best = -1;
    double bv = 0;
    for (size_t i = 0; i < out.size(); ++i)
      if (out[i].samples_per_s > bv) { bv = out[i].samples_per_s; *best = static_cast<int32_t>(i); }
    if (results)
      for (int i = 0; i < std::min<int>(cap, static_cast<int>(out.size())); ++i) results[i] = out[i];
    return MARIO_OK;
  });
}
