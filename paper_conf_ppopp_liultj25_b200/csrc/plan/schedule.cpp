// Base schedules, graph passes 1-4 and the DP timeline simulator (§5.1-§5.2).
// The readings of the paper's open points are DESIGN.md A9-A17 (same as SURVEY §8(c) c3);
// tests/test_planner.py checks these lists byte-for-byte against oracle/schedule.py.
#include "plan.h"

#include <algorithm>
#include <cmath>
#include <limits>
#include <map>
#include <set>
#include <stdexcept>
#include <tuple>

namespace mario {
namespace plan {

const char* op_name(int op) {
  switch (op) {
    case FW: return "FW"; case CFW: return "CFW"; case RC: return "RC"; case BW: return "BW";
    case SA: return "SA"; case RA: return "RA"; case SG: return "SG"; case RG: return "RG";
  }
  return "??";
}

// Algorithm 1 — step = -1 (prev) / +1 (next) in the FW direction; opposite for BW.
bool find_inst(const Pipe& pp, int d, int m, int p, int t, bool nxt, int* d_o, int* p_o) {
  (void)m;
  int step = nxt ? 1 : -1;
  if (t == BW) step = -step;
  int dd = d, po = p;
  if (pp.scheme == MARIO_1F1B) {
    dd = d + step;
    if (dd < 0 || dd >= pp.S) return false;
  } else if (pp.scheme == MARIO_CHIMERA) {
    dd = p == 0 ? d + step : d - step;
    if (dd < 0 || dd >= pp.S) return false;
  } else {  // Interleave: modular wrap, part_id changes when crossing (reading A9: p + step)
    dd = (d + step + pp.S) % pp.S;
    if (dd != d + step) po = p + step;
    if (po < 0 || po >= pp.v) return false;
  }
  *d_o = dd;
  *p_o = po;
  return true;
}

namespace {

void fw_group(const Pipe& pp, int d, int m, int p, List& L) {
  int k = pp.vstage(d, p);
  if (k > 0) L.push_back({RA, m, p});
  L.push_back({FW, m, p});
  if (k < pp.K() - 1) L.push_back({SA, m, p});
}
void bw_group(const Pipe& pp, int d, int m, int p, List& L) {
  int k = pp.vstage(d, p);
  if (k < pp.K() - 1) L.push_back({RG, m, p});
  L.push_back({BW, m, p});
  if (k > 0) L.push_back({SG, m, p});
}

Lists build_1f1b(const Pipe& pp) {
  Lists out(pp.S);
  for (int d = 0; d < pp.S; ++d) {
    int warm = std::min(pp.S - d - 1, pp.N);
    List& L = out[d];
    for (int i = 0; i < warm; ++i) fw_group(pp, d, i, 0, L);
    for (int i = 0; i < pp.N - warm; ++i) {
      fw_group(pp, d, warm + i, 0, L);
      bw_group(pp, d, i, 0, L);
    }
    for (int i = pp.N - warm; i < pp.N; ++i) bw_group(pp, d, i, 0, L);
  }
  return out;
}

Lists build_interleave(const Pipe& pp) {
  const int S = pp.S, N = pp.N, v = pp.v, total = N * v;
  auto chunk = [&](int k, bool fwd) { int c = (k % (S * v)) / S; return fwd ? c : v - 1 - c; };
  auto micro = [&](int k) { return (k / (S * v)) * S + k % S; };
  Lists out(S);
  for (int d = 0; d < S; ++d) {
    int warm = (N == S) ? total : std::min((S - d - 1) * 2 + (v - 1) * S, total);
    List& L = out[d];
    for (int k = 0; k < warm; ++k) fw_group(pp, d, micro(k), chunk(k, true), L);
    for (int i = 0; i < total - warm; ++i) {
      int kf = warm + i;
      fw_group(pp, d, micro(kf), chunk(kf, true), L);
      bw_group(pp, d, micro(i), chunk(i, false), L);
    }
    for (int kb = total - warm; kb < total; ++kb) bw_group(pp, d, micro(kb), chunk(kb, false), L);
  }
  return out;
}

// Chimera basic unit by greedy list scheduling at F=1, B=2 (reading A10): BW first, then the deeper
// virtual stage, then the micro-batch; identical to oracle/schedule.py::build_chimera.
Lists build_chimera(const Pipe& pp) {
  const int D = pp.S;
  Pipe unit{MARIO_CHIMERA, D, D, 1};
  const double F = 1.0, B = 2.0, EPS = 1e-12;
  using Key = std::tuple<int, int, int>;  // (op, m, k)
  std::map<Key, double> fin;
  std::set<Key> remaining;
  for (int m = 0; m < D; ++m)
    for (int k = 0; k < D; ++k) { remaining.insert({FW, m, k}); remaining.insert({BW, m, k}); }
  auto owner = [&](int m, int k) { return unit.device_part(k, unit.part_of_micro(m)).first; };
  auto done_by = [&](const Key& key, double t) {
    auto it = fin.find(key);
    return it != fin.end() && it->second <= t + EPS;
  };
  std::vector<std::vector<Instr>> order(D);
  std::vector<double> busy_until(D, 0.0);
  double t = 0.0;
  while (!remaining.empty()) {
    bool progressed = false;
    for (int d = 0; d < D; ++d) {
      if (busy_until[d] > t + EPS) continue;
      // ready tuples sorted by (BW first, deeper stage first, m)
      std::vector<std::tuple<int, int, int, int>> ready;
      for (const Key& key : remaining) {
        int op = std::get<0>(key), m = std::get<1>(key), k = std::get<2>(key);
        if (owner(m, k) != d) continue;
        if (op == FW) {
          if (k > 0 && !done_by({FW, m, k - 1}, t)) continue;
        } else {
          if (!done_by({FW, m, k}, t)) continue;
          Key dep = (k == D - 1) ? Key{FW, m, k} : Key{BW, m, k + 1};
          if (!done_by(dep, t)) continue;
        }
        ready.push_back({op == BW ? 0 : 1, -k, m, op});
      }
      if (ready.empty()) continue;
      std::sort(ready.begin(), ready.end());
      int k = -std::get<1>(ready[0]), m = std::get<2>(ready[0]), op = std::get<3>(ready[0]);
      remaining.erase({op, m, k});
      double dur = op == FW ? F : B;
      fin[{op, m, k}] = t + dur;
      busy_until[d] = t + dur;
      order[d].push_back({op, m, unit.part_of_micro(m)});
      progressed = true;
    }
    double nxt = INFINITY;
    for (double b : busy_until) if (b > t + EPS) nxt = std::min(nxt, b);
    for (auto& kv : fin) if (kv.second > t + EPS) nxt = std::min(nxt, kv.second);
    if (std::isinf(nxt)) {
      if (!progressed && !remaining.empty()) throw std::runtime_error("chimera greedy stalled");
      continue;
    }
    t = nxt;
  }
  Lists out(D);
  for (int d = 0; d < D; ++d)
    for (int u = 0; u < pp.N / D; ++u)
      for (const Instr& x : order[d]) {
        int mm = u * D + x.m;
        if (x.op == FW) fw_group(pp, d, mm, x.p, out[d]); else bw_group(pp, d, mm, x.p, out[d]);
      }
  return out;
}

int index_of(const List& L, const Instr& x) {
  for (size_t i = 0; i < L.size(); ++i) if (L[i] == x) return static_cast<int>(i);
  return -1;
}

}  // namespace

Lists build_base(const Pipe& pp) {
  if (pp.scheme == MARIO_1F1B) return build_1f1b(pp);
  if (pp.scheme == MARIO_INTERLEAVE) return build_interleave(pp);
  return build_chimera(pp);
}

// Pass 1: FW -> CFW; RC inserted right before BW (after RG), reading A14.
Lists pass1_apply_checkpoint(const Lists& in, const std::vector<bool>& keep) {
  Lists out;
  for (size_t d = 0; d < in.size(); ++d) {
    const List& L = in[d];
    if (d < keep.size() && keep[d]) { out.push_back(L); continue; }
    List N;
    for (const Instr& x : L) {
      if (x.op == FW) N.push_back({CFW, x.m, x.p});
      else if (x.op == BW) { N.push_back({RC, x.m, x.p}); N.push_back(x); }
      else N.push_back(x);
    }
    out.push_back(std::move(N));
  }
  return out;
}

// Pass 2: RC_i immediately before RG_i (reading A15).
Lists pass2_overlap_recompute(const Lists& in) {
  Lists out;
  for (const List& L : in) {
    List N, rcs;
    for (const Instr& x : L) (x.op == RC ? rcs : N).push_back(x);
    for (const Instr& r : rcs) {
      int a = index_of(N, {RG, r.m, r.p});
      if (a < 0) a = index_of(N, {BW, r.m, r.p});
      N.insert(N.begin() + a, r);
    }
    out.push_back(std::move(N));
  }
  return out;
}

// Pass 3: CFW_i and BW_i adjacent ignoring comm and RC_i -> un-checkpoint (A16).
Lists pass3_remove_redundancy(const Lists& in) {
  Lists out;
  for (const List& L : in) {
    List N = L;
    for (const Instr& x : L) {
      if (x.op != CFW) continue;
      int i = index_of(N, x), j = index_of(N, {BW, x.m, x.p});
      bool between = false;
      for (int q = i + 1; q < j; ++q)
        if (is_compute(N[q].op) && !(N[q] == Instr{RC, x.m, x.p})) { between = true; break; }
      if (!between) {
        N[i] = {FW, x.m, x.p};
        N.erase(N.begin() + index_of(N, {RC, x.m, x.p}));
      }
    }
    out.push_back(std::move(N));
  }
  return out;
}

// DP timeline, reading A12: serial compute per device in list order; receives
// block the device until the data arrives; sends are buffered and posted when everything
// before them in the list has completed.
SimResult simulate(const Pipe& pp, const Lists& L, const SimCosts& c) {
  const int S = pp.S, P = pp.parts();
  SimResult r;
  r.busy.assign(S, 0.0);
  r.start.assign(S, {});
  r.finish.assign(S, {});
  // post time of sends, flat index ((device * N + micro) * parts + part) * 2 + (SG ? 1 : 0); NaN = not posted
  std::vector<double> post(static_cast<size_t>(S) * pp.N * P * 2, std::numeric_limits<double>::quiet_NaN());
  auto key = [&](int d, int m, int p, bool grad) { return ((static_cast<size_t>(d) * pp.N + m) * P + p) * 2 + (grad ? 1 : 0); };
  std::vector<size_t> ptr(S, 0);
  std::vector<double> dev_t(S, 0.0);
  size_t total = 0, done = 0;
  for (const List& l : L) total += l.size();
  double makespan = 0;
  bool any = false;
  while (done < total) {
    bool progressed = false;
    for (int d = 0; d < S; ++d) {
      const List& l = L[d];
      while (ptr[d] < l.size()) {
        const Instr& x = l[ptr[d]];
        const int k = pp.vstage(d, x.p);
        if (is_send(x.op)) {
          post[key(d, x.m, x.p, x.op == SG)] = dev_t[d];
        } else if (is_recv(x.op)) {
          int sd, sp;
          if (!find_inst(pp, d, x.m, x.p, x.op == RA ? FW : BW, false, &sd, &sp)) return r;  // malformed
          const double t = post[key(sd, x.m, sp, x.op == RG)];
          if (std::isnan(t)) break;
          dev_t[d] = std::max(dev_t[d], t + (x.op == RA ? c.comm_act : c.comm_grad));
        } else {
          double dur = (x.op == FW || x.op == CFW) ? c.fw[k] : x.op == RC ? c.rc[k] : c.bw[k];
          r.start[d].push_back(dev_t[d]);
          r.finish[d].push_back(dev_t[d] + dur);
          dev_t[d] += dur;
          r.busy[d] += dur;
          if (!any || dev_t[d] > makespan) makespan = dev_t[d];
          any = true;
        }
        ++ptr[d];
        ++done;
        progressed = true;
      }
    }
    if (!progressed) return r;  // cycle -> ok = false
  }
  r.ok = true;
  r.makespan = makespan;
  return r;
}

// P:254, reading A13: list-order accounting; FW keeps its activation set until BW; a CFW's
// dynamic memory is transient; RC materialises the set again until BW.
MemResult memory_walk(const Pipe& pp, const Lists& L, const SimCosts& c) {
  MemResult out;
  for (int d = 0; d < pp.S; ++d) {
    double cur = 0, peak = 0;
    int la = 0, lc = 0, ma = 0, mc = 0;
    for (const Instr& x : L[d]) {
      const int k = pp.vstage(d, x.p);
      if (x.op == FW) { ++lc; ++la; cur += c.act[k] + c.ckpt[k]; peak = std::max(peak, cur); }
      else if (x.op == CFW) { ++lc; cur += c.ckpt[k]; peak = std::max(peak, cur + c.work[k]); }
      else if (x.op == RC) { ++la; cur += c.act[k]; peak = std::max(peak, cur); }
      else if (x.op == BW) { --la; --lc; cur -= c.act[k] + c.ckpt[k]; }
      ma = std::max(ma, la);
      mc = std::max(mc, lc);
    }
    double st = d < static_cast<int>(c.static_bytes.size()) ? c.static_bytes[d] : 0.0;
    out.peak.push_back(st + peak);
    out.max_live_act.push_back(ma);
    out.max_live_ckpt.push_back(mc);
  }
  return out;
}

namespace {
std::vector<int> group_starts(const List& L) {
  std::vector<int> out;
  for (size_t j = 0; j < L.size(); ++j) {
    if (is_compute(L[j].op) || is_recv(L[j].op)) {
      if (j > 0 && is_recv(L[j - 1].op)) continue;
      out.push_back(static_cast<int>(j));
    }
  }
  out.push_back(static_cast<int>(L.size()));
  return out;
}
}  // namespace

// Pass 4, reading A17: devices ascending, CFWs in list order; move [RA_i CFW_i]
// to the earliest group boundary after the previous forward that keeps the graph acyclic,
// does not raise the simulated makespan and keeps the peak within budget. The sender's SA_i
// follows its CFW_i only if that CFW was preposed (the receiver moved too); otherwise SA_i
// stays in place and the output is buffered. Iterated to a fixpoint.
Lists pass4_prepose_forward(const Pipe& pp, const Lists& in, const SimCosts& c, double budget, int max_rounds) {
  Lists lists = in;
  std::set<std::tuple<int, int, int>> preposed;
  SimResult cur = simulate(pp, lists, c);
  if (!cur.ok) throw std::runtime_error("pass4: input lists deadlock");
  double best = cur.makespan;
  for (int round = 0; round < max_rounds; ++round) {
    bool changed = false;
    for (int d = 0; d < pp.S; ++d) {
      std::vector<Instr> cfws;
      for (const Instr& y : lists[d]) if (y.op == CFW) cfws.push_back(y);
      for (const Instr& x : cfws) {
        const List& L = lists[d];
        int i = index_of(L, x);
        int prev_f = -1;
        for (int j = 0; j < i; ++j) if (L[j].op == FW || L[j].op == CFW) prev_f = j;
        int lo = prev_f + 1;
        int gstart = (i > 0 && L[i - 1] == Instr{RA, x.m, x.p}) ? i - 1 : i;
        std::vector<int> cands;
        for (int j : group_starts(L)) if (j >= lo && j < gstart) cands.push_back(j);
        for (int j : cands) {
          Lists trial = lists;
          List grp(L.begin() + gstart, L.begin() + i + 1);
          List rest(L.begin(), L.begin() + gstart);
          rest.insert(rest.end(), L.begin() + i + 1, L.end());
          List nl(rest.begin(), rest.begin() + j);
          nl.insert(nl.end(), grp.begin(), grp.end());
          nl.insert(nl.end(), rest.begin() + j, rest.end());
          trial[d] = std::move(nl);
          int sd, sp;
          if (find_inst(pp, d, x.m, x.p, FW, false, &sd, &sp) && preposed.count({sd, x.m, sp})) {
            List& SL = trial[sd];
            SL.erase(SL.begin() + index_of(SL, {SA, x.m, sp}));
            SL.insert(SL.begin() + index_of(SL, {CFW, x.m, sp}) + 1, Instr{SA, x.m, sp});
          }
          SimResult r = simulate(pp, trial, c);
          if (!r.ok || r.makespan > best + 1e-9) continue;
          if (budget > 0) {
            MemResult mr = memory_walk(pp, trial, c);
            if (*std::max_element(mr.peak.begin(), mr.peak.end()) > budget) continue;
          }
          lists = std::move(trial);
          best = r.makespan;
          preposed.insert({d, x.m, x.p});
          changed = true;
          break;
        }
      }
    }
    if (!changed) break;
  }
  return lists;
}

}  // namespace plan
}  // namespace mario
