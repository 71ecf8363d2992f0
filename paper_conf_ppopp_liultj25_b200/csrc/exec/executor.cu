// Per-rank executor of a Mario plan (Table 3).
//
// Each rank walks its instruction list once per iteration and enqueues, asynchronously:
//   FW / CFW / RC / BW  -> layer kernels on the compute stream (list order = the plan's
//                          horizontal dependencies, so RC lands exactly where the plan put
//                          it: before the RG wait, inside the bubble)
//   RA / RG             -> ncclRecv on the channel's stream into a static slot; the compute
//                          stream waits on it at the RA/RG position (blocking receive)
//   SA / SG             -> ncclSend on the channel's stream after everything before it in the
//                          list (buffered send; a preposed CFW's output stays in its send slot
//                          until its SA)
// One NCCL communicator + stream per channel (ordered pair x {activation, gradient}) keeps
// every channel a FIFO, so any acyclic plan is deadlock-free.
// Loopback (world == 1, multi-stage plan): every rank's list runs in this process on one GPU
// in the simulator's round-robin order; RA/RG become device-to-device copies.
// Peer transport (mario_init_emulated: S virtual ranks in one process, each on its own streams and,
// optionally, its own SM partition of the GPU): the per-rank code path of the multi-process
// executor (slot-reuse guards, blocking receives, pair gradient reductions) with the channel
// implemented in peer memory instead of NCCL: a send is a flag the sender's stream writes after the
// message is complete (P:222 buffered send); a receive is a stream wait on that flag, a copy out of
// the sender's send slot and a "consumed" flag the sender's next use of the slot waits on.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <array>
#include <initializer_list>
#include <map>
#include <set>
#include <memory>
#include <mutex>
#include <stdexcept>
#include <string>
#include <tuple>
#include <vector>

#include "../capi/status.h"
#include "../kernels/kernels.h"
#include "../kernels/layers.h"
#include "../kernels/kstats.h"
#include "arena.h"
#include "drv.h"

extern "C" long long mario_kernel_launches(void);

namespace mario {
namespace {

using plan::Instr;

#define CU(x)                                                                       \
  do {                                                                              \
    cudaError_t e_ = (x);                                                           \
    if (e_ != cudaSuccess) throw CudaErr(std::string(#x) + ": " + cudaGetErrorString(e_)); \
  } while (0)
#define NC(x)                                                                       \
  do {                                                                              \
    ncclResult_t r_ = (x);                                                          \
    if (r_ != ncclSuccess) throw NcclErr(std::string(#x) + ": " + ncclGetErrorString(r_)); \
  } while (0)

#define DRV(x)                                                                      \
  do {                                                                              \
    cudaError_t e_ = (x);                                                           \
    if (e_ != cudaSuccess) throw CudaErr(std::string(#x) + ": stream memory operation failed"); \
  } while (0)

struct CudaErr : std::runtime_error { using std::runtime_error::runtime_error; };
struct NcclErr : std::runtime_error { using std::runtime_error::runtime_error; };

// ------------------------------------------------------------------ context
struct Channel {
  ncclComm_t comm = nullptr;
  cudaStream_t stream = nullptr;
};

struct Context {
  int rank = 0, world = 1, device = 0;
  int dp = 1;                         // data-parallel replicas: world = stages * dp (reading A29)
  bool inited = false;
  ncclComm_t world_comm = nullptr;
  ncclComm_t dp_comm = nullptr;       // this stage's replicas (kind 6 split)
  std::map<std::tuple<int, int, int>, Channel> channels;   // (src, dst, kind)
  std::map<std::pair<int, int>, ncclComm_t> pair_comms;      // (lo, hi) 2-rank comms
  std::set<std::tuple<int, int, int>> created_channels;       // split already done (all ranks)
  std::set<std::pair<int, int>> created_pairs;
  cudaStream_t loss_stream = nullptr;
  bool timing = false;
  std::vector<std::vector<double>> t_start, t_finish;
  // CUDA-graph replay of whole iterations (single-process: S = 1 or loopback)
  bool graphs = false;
  cudaStream_t cap_stream = nullptr;
  // key: (plan serial, weights, grads, workspace, kstats generation) — event-timed launches captured
  // in a graph re-record their events on every replay, so a new timing set needs a new capture.
  // The serial is never reused (a freed plan's address can be), and mario_plan_destroy evicts.
  using GKey = std::tuple<uint64_t, const void*, const void*, const void*, long long>;
  std::map<GKey, cudaGraphExec_t> graph_cache;
  std::map<GKey, long long> graph_kernels;
  std::set<GKey> graph_seen;
  bool sticky = false;
  // peer transport, emulated pipeline (mario_init_emulated): `world` virtual ranks in this process
  bool emulated = false;
  int emu_sms = 0;                              // SMs of each rank's partition (0: unpartitioned)
  std::vector<cudaStream_t> emu_st;             // per rank: compute stream
  std::vector<cudaStream_t> emu_side;           // per rank: side stream (independent wgrads)
  cudaStream_t side_st = nullptr;               // loopback / NCCL: side stream of the caller's work
  std::vector<std::array<cudaStream_t, 2>> emu_rx;   // per rank: receive streams (activation, gradient)
  bool emu_green = false;                       // streams live in green contexts
  uint32_t* flags = nullptr;                    // device flag block (reset every iteration)
  size_t flags_cap = 0;
  // peer transport across processes (mario_init_peer: one process per rank, CUDA IPC): every rank
  // maps the other ranks' workspace and grads and rank 0's flag block; flags carry the iteration
  // number (epoch) instead of being reset
  bool ipc = false;
  uint32_t epoch = 0;
  struct PeerPtrs { uint8_t* ws = nullptr; float* gr = nullptr; uint32_t* flags = nullptr; };
  std::vector<PeerPtrs> peers;
  std::vector<void*> ipc_opened;
  uint32_t* ipc_flags_own = nullptr;            // this rank's flag block (rank 0's is the shared one)
  size_t ipc_flag_words = 0;
  cudaStream_t ipc_st = nullptr, ipc_rx[2] = {nullptr, nullptr}, ipc_side = nullptr;
  const void* bound_ws = nullptr;               // the buffers the imported records describe
  const void* bound_gr = nullptr;
};
Context g;

// ------------------------------------------------------------- per-device state
// Ordering events outlive one mario_run_iter call in a per-device cache: a call takes what it
// needs and hands them back at the end instead of creating and destroying every slot / dependency
// event per iteration (re-recording an event whose earlier record is still pending is legal; the
// waits enqueued before already refer to that earlier record).
std::mutex g_ev_mu;
std::map<int, std::vector<cudaEvent_t>> g_ev_cache;
cudaEvent_t ev_get() {
  int dev = 0;
  cudaGetDevice(&dev);
  {
    std::lock_guard<std::mutex> lk(g_ev_mu);
    auto& v = g_ev_cache[dev];
    if (!v.empty()) {
      cudaEvent_t e = v.back();
      v.pop_back();
      return e;
    }
  }
  cudaEvent_t e;
  CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  return e;
}
void ev_put(cudaEvent_t e) {
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_ev_mu);
  g_ev_cache[dev].push_back(e);
}

template <class T>
struct Dev {
  const PlanObj* P = nullptr;
  int d = 0;
  Arena a;
  uint8_t* ws = nullptr;
  const float* w = nullptr;   // packed fp32 master weights of this rank
  float* gr = nullptr;        // packed fp32 grads of this rank
  std::map<std::pair<int, int>, int> tensor;   // (part, global param idx) -> packed index j
  // host-side slot pools for send / recv-grad buffers
  std::vector<bool> sa_used, sg_used, rg_used;
  std::map<std::pair<int, int>, int> sa_of, sg_of, rg_of;
  std::vector<cudaEvent_t> sa_free, sg_free, rg_free, ck_free;   // event guarding slot reuse
  std::vector<bool> sa_free_set, sg_free_set, rg_free_set, ck_free_set;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_next = 0;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> timed;   // per compute instr
  // peer transport: this rank's streams and the consumption flag guarding each send slot's reuse
  cudaStream_t st = nullptr;
  cudaStream_t rx[2] = {nullptr, nullptr};
  cudaStream_t side = nullptr;   // independent backward GEMMs (MARIO_GEMM_OVERLAP)
  int sms = 0;
  std::vector<const uint32_t*> sa_guard, sg_guard;
  std::vector<std::tuple<int, int, int>> sa_guard_key, sg_guard_key;   // the guarding message

  const mario_model& M() const { return P->model; }
  template <class U = uint8_t> U* at(size_t off) const { return reinterpret_cast<U*>(ws + off); }
  cudaEvent_t event() {
    if (ev_next == ev_pool.size()) ev_pool.push_back(ev_get());
    return ev_pool[ev_next++];
  }
};

int acquire(std::vector<bool>& used) {
  for (size_t i = 0; i < used.size(); ++i) if (!used[i]) { used[i] = true; return static_cast<int>(i); }
  throw std::runtime_error("executor slot pool exhausted (planner/executor mismatch)");
}

template <class T>
struct Exec {
  cudaStream_t st;
  int gemm_persistent = 1;   // the next GEMMs' grid mode (see GemmArgs::persistent)
  bool loopback;
  bool peer = false;                           // peer transport (emulated ranks, one per stream set)
  std::vector<std::unique_ptr<Dev<T>>> devs;   // loopback / peer: all ranks; NCCL: one (this rank)
  // peer: the flag block [ready | done][kind][receiving vstage][micro] + reduction flags, and
  // where each message sits: (kind, receiving vstage, micro) -> (sender rank, send slot)
  uint32_t* flags = nullptr;
  int fK = 0, fN = 0;
  uint32_t fv = 1;                             // value a flag is raised to: 1 (reset per call) or the epoch
  int me = -1;                                 // multi-process peer transport: this rank (else -1: all local)
  bool mine(int d) const { return me < 0 || d == me; }
  // host walk state (peer): messages whose "ready" / "consumed" flag write is already enqueued. A
  // flag wait is only ever enqueued after the write it waits for (like an event record before its
  // wait): a wait enqueued first could sit in front of its own write if the driver maps the two
  // streams onto one hardware queue, and deadlock.
  std::set<std::tuple<int, int, int>> ready_walked, consumed_walked;

  Dev<T>& dev(int d) { return (loopback || peer) ? *devs[d] : *devs[0]; }
  uint32_t* flag_ready(int kind, int k, int m) { return flags + (static_cast<size_t>(kind) * fK + k) * fN + m; }
  uint32_t* flag_done(int kind, int k, int m) { return flags + (static_cast<size_t>(2 + kind) * fK + k) * fN + m; }
  uint32_t* flag_misc(size_t i) { return flags + static_cast<size_t>(4) * fK * fN + i; }

  // ---- weights --------------------------------------------------------------
  int tidx(Dev<T>& D, int p, const std::string& name) {
    const auto g = D.P->param_index.find(name);
    if (g != D.P->param_index.end()) {
      auto it = D.tensor.find({p, g->second});
      if (it != D.tensor.end()) return it->second;
    }
    throw std::runtime_error("parameter " + name + " not held by part " + std::to_string(p));
  }
  const T* Wm(Dev<T>& D, int p, const std::string& name) {   // compute-dtype matrix
    int j = tidx(D, p, name);
    if (sizeof(T) == 2) return D.template at<T>(D.a.wcopy[j]);
    return reinterpret_cast<const T*>(D.w + D.P->rank_params[D.d].off[j]);
  }
  const float* Wf(Dev<T>& D, int p, const std::string& name) {
    return D.w + D.P->rank_params[D.d].off[tidx(D, p, name)];
  }
  float* G(Dev<T>& D, int p, const std::string& name) {
    return D.gr + D.P->rank_params[D.d].off[tidx(D, p, name)];
  }

  const float2* rope_tab(Dev<T>& D) const {
    return D.a.rope == SIZE_MAX ? nullptr : reinterpret_cast<const float2*>(D.ws + D.a.rope);
  }

  // ---- GEMM dispatch --------------------------------------------------------
  // D[M,N] = A[M,K] . B[N,K]^T  (see kernels.h); bf16 tcgen05 or fp32 SIMT by dtype.
  void gemm(const T* A, int lda, int a_mn, const T* B, int ldb, int b_mn, int M, int N, int K, void* Dp, int ldd,
            bool out_f32, float beta, const float* bias = nullptr, const T* resid = nullptr, T* D2 = nullptr,
            const T* aux = nullptr, bool d2_from_aux = false, float* colsum_part = nullptr, const T* dot = nullptr,
            float* dot_out = nullptr, int dot_seg = 0) {
    if constexpr (sizeof(T) == 2) {
      GemmArgs g;
      g.A = A; g.lda = lda; g.a_mn = a_mn; g.B = B; g.ldb = ldb; g.b_mn = b_mn; g.M = M; g.N = N; g.K = K;
      g.ep.out_f32 = out_f32;
      if (out_f32) g.ep.d_f32 = static_cast<float*>(Dp); else g.ep.d_bf16 = static_cast<__nv_bfloat16*>(Dp);
      g.ep.ldd = ldd; g.ep.beta = beta; g.ep.bias = bias;
      g.ep.residual = resid; g.ep.ld_res = ldd; g.ep.d2_bf16 = D2; g.ep.aux = aux; g.ep.ld_aux = ldd;
      g.ep.d2_from_aux = d2_from_aux ? 1 : 0;
      g.ep.colsum_part = colsum_part;
      g.ep.dot = dot; g.ep.ld_dot = ldd; g.ep.dot_out = dot_out; g.ep.dot_seg = dot_seg; g.ep.dot_stride = M;
      g.persistent = gemm_persistent;
      CU(gemm_bf16(g, st));
    } else {
      GemmF32Args g;
      g.A = A; g.lda = lda; g.a_mn = a_mn; g.B = B; g.ldb = ldb; g.b_mn = b_mn; g.M = M; g.N = N; g.K = K;
      g.D = static_cast<float*>(Dp); g.ldd = ldd; g.beta = beta; g.bias = bias; g.residual = resid;
      g.ld_res = ldd; g.D2 = D2; g.aux = aux; g.ld_aux = ldd; g.d2_from_aux = d2_from_aux ? 1 : 0;
      CU(gemm_f32(g, st));
    }
  }
  // dX[T,in] = dY W with, per head of `seg` columns, Dd[head][t] = sum bf16(dX[t, head]) * X[t, head]
  // fused into the epilogue (bf16: the attention backward's D = rowsum(dO o O))
  void lin_dgrad_dot(const T* dY, const T* W, int Tn, int out, int in, T* dX, const T* X, float* Dd, int seg) {
    gemm(dY, out, 0, W, in, 1, Tn, in, out, dX, in, false, 0.f, nullptr, nullptr, nullptr, nullptr, false, nullptr, X,
         Dd, seg);
  }
  // Y[T,out] = X W^T (+bias, +resid, D2 = gelu)
  void lin_fwd(const T* X, const T* W, int Tn, int out, int in, T* Y, const float* bias, const T* resid = nullptr,
               T* Y2 = nullptr) {
    gemm(X, in, 0, W, in, 0, Tn, out, in, Y, out, false, 0.f, bias, resid, Y2);
  }
  // dX[T,in] = dY W (optionally * gelu'(aux); G = gelu(aux) as a second output when G != NULL)
  // colsum_part (bf16 only): the epilogue also writes column partial sums of dX ([Tn/32][in] fp32)
  void lin_dgrad(const T* dY, const T* W, int Tn, int out, int in, T* dX, const T* aux = nullptr, T* G = nullptr,
                 float* colsum_part = nullptr) {
    gemm(dY, out, 0, W, in, 1, Tn, in, out, dX, in, false, 0.f, nullptr, nullptr, G, aux, G != nullptr, colsum_part);
  }
  // dW[out,in] += dY^T X (fp32)
  void lin_wgrad(const T* dY, const T* X, int Tn, int out, int in, float* dW) {
    gemm(dY, out, 1, X, in, 1, out, in, Tn, dW, in, true, 1.f);
  }

  // ---- overlap of independent backward GEMMs (MARIO_GEMM_OVERLAP=1) ------------------------
  // A wgrad that does not depend on the dgrad next to it runs on the rank's side stream as a
  // non-persistent grid, launched after the persistent dgrad: its CTA pairs take the SMs the
  // dgrad's last, partly empty wave frees (256 pair tiles on 74 pairs = 3.46 waves at cfg 2). Tiles
  // are still computed whole by one pair each, so the results are bitwise unchanged.
  static bool overlap_on() {
    static const bool on = getenv("MARIO_GEMM_OVERLAP") && atoi(getenv("MARIO_GEMM_OVERLAP")) != 0;
    return on;
  }
  bool side_open = false;
  template <class F>
  void on_side(Dev<T>& D, F&& f) {
    if (!(sizeof(T) == 2 && overlap_on() && D.side)) { f(); return; }
    cudaEvent_t e = D.event();
    CU(cudaEventRecord(e, st));
    CU(cudaStreamWaitEvent(D.side, e, 0));
    cudaStream_t keep = st;
    st = D.side;
    gemm_persistent = 0;
    f();
    gemm_persistent = 1;
    st = keep;
    side_open = true;
  }
  void join_side(Dev<T>& D) {
    if (!side_open) return;
    cudaEvent_t e = D.event();
    CU(cudaEventRecord(e, D.side));
    CU(cudaStreamWaitEvent(st, e, 0));
    side_open = false;
  }

  // ---- forward of one virtual stage -------------------------------------------
  // mode: 0 = FW (keep activations in act set), 1 = CFW (scratch), 2 = RC (act set, no loss)
  void stage_forward(Dev<T>& D, const mario_instr& x, int mode, T* out) {
    const mario_model& m = D.M();
    const int K = D.P->pp.K(), k = x.vstage, p = x.part, lps = D.P->lps;
    const int Tn = static_cast<int>(tokens_per_micro(m)), h = m.hidden, f = m.ffn_hidden, nh = m.n_heads;
    const int dh = h / nh, s = m.seq_len, mbs = m.micro_batch;
    const bool gpt = m.family == MARIO_GPT;
    const bool sn = D.P->store_act;
    const LayerAct LA = layer_act_layout(m, sn);
    const LayerTrans LT = layer_trans_layout(m, sn);
    const HeadAct HA = head_act_layout(m);
    // cfw scratch: [one layer's stored tensors][transients A, A2, G][run0][run1][head]
    uint8_t* cfw = D.template at<uint8_t>(D.a.cfw);
    uint8_t* trans = cfw + LA.bytes;
    uint8_t* base;
    size_t lstride;
    if (mode == 1) { base = cfw; lstride = 0; }
    else { base = D.template at<uint8_t>(D.a.act + static_cast<size_t>(x.aslot) * D.a.act_stride); lstride = LA.bytes; }
    uint8_t* run_base = trans + LT.bytes;
    uint8_t* head_base = (mode == 1) ? run_base + 2 * stage_input_bytes(m) : base + LA.bytes * lps;
    T* run[2] = {reinterpret_cast<T*>(run_base), reinterpret_cast<T*>(run_base + stage_input_bytes(m))};
    const int32_t* tok = D.template at<int32_t>(D.a.tokens) + static_cast<size_t>(x.micro) * mbs * (s + 1);
    // stage input
    const T* Hin;
    if (k == 0) {
      T* H0 = (mode == 1) ? run[0] : reinterpret_cast<T*>(base + LA.H_in);
      const T* wte = Wm(D, p, gpt ? "wte" : "emb");
      const T* wpe = gpt ? Wm(D, p, "wpe") : nullptr;
      embed_fwd<T>(tok, s + 1, mbs, s, wte, wpe, H0, h, st);
      Hin = H0;
    } else {
      Hin = D.template at<T>(D.a.ckpt + static_cast<size_t>(x.slot) * D.a.ckpt_stride);
    }
    for (int li = 0; li < lps; ++li) {
      const int l = k * lps + li;
      const std::string pre = "h" + std::to_string(l) + ".";
      uint8_t* L = base + li * lstride;
      T* A = reinterpret_cast<T*>(sn ? L + LA.A : trans + LT.A);
      T* QKV = reinterpret_cast<T*>(L + LA.QKV);
      T* O = reinterpret_cast<T*>(L + LA.O);
      float* LSE = reinterpret_cast<float*>(L + LA.LSE);
      T* H1 = reinterpret_cast<T*>(L + LA.H1);
      T* A2 = reinterpret_cast<T*>(sn ? L + LA.A2 : trans + LT.A2);
      T* Z = reinterpret_cast<T*>(L + LA.Z);
      T* Gt = reinterpret_cast<T*>(sn ? L + LA.G : trans + LT.G);
      float* st1 = reinterpret_cast<float*>(L + LA.st1);
      float* st2 = reinterpret_cast<float*>(L + LA.st2);
      // output of this layer
      T* Hout;
      if (li + 1 < lps) Hout = (mode == 1) ? run[(li + 1) & 1] : reinterpret_cast<T*>(base + (li + 1) * lstride + LA.H_in);
      else if (k == K - 1) Hout = reinterpret_cast<T*>(head_base + HA.H_last);
      else Hout = out;
      if (gpt) {
        layernorm_fwd<T>(Hin, Wf(D, p, pre + "ln1.g"), Wf(D, p, pre + "ln1.b"), A, st1, Tn, h, m.norm_eps, st);
        lin_fwd(A, Wm(D, p, pre + "qkv.w"), Tn, 3 * h, h, QKV, Wf(D, p, pre + "qkv.b"));
      } else {
        rmsnorm_fwd<T>(Hin, Wf(D, p, pre + "n1.g"), A, st1, Tn, h, m.norm_eps, st);
        lin_fwd(A, Wm(D, p, pre + "qkv.w"), Tn, 3 * h, h, QKV, nullptr);
        rope<T>(QKV, mbs, s, nh, dh, m.rope_base, 0, st, rope_tab(D));
      }
      attn_fwd<T>(QKV, O, LSE, mbs, s, nh, dh, st, LT.attn_pad_bytes ? trans + LT.attn_pad : nullptr);
      if (gpt) {
        lin_fwd(O, Wm(D, p, pre + "proj.w"), Tn, h, h, H1, Wf(D, p, pre + "proj.b"), Hin);
        layernorm_fwd<T>(H1, Wf(D, p, pre + "ln2.g"), Wf(D, p, pre + "ln2.b"), A2, st2, Tn, h, m.norm_eps, st);
        lin_fwd(A2, Wm(D, p, pre + "fc1.w"), Tn, f, h, Z, Wf(D, p, pre + "fc1.b"), nullptr, Gt);
        lin_fwd(Gt, Wm(D, p, pre + "fc2.w"), Tn, h, f, Hout, Wf(D, p, pre + "fc2.b"), H1);
      } else {
        lin_fwd(O, Wm(D, p, pre + "o.w"), Tn, h, h, H1, nullptr, Hin);
        rmsnorm_fwd<T>(H1, Wf(D, p, pre + "n2.g"), A2, st2, Tn, h, m.norm_eps, st);
        lin_fwd(A2, Wm(D, p, pre + "gu.w"), Tn, 2 * f, h, Z, nullptr);
        swiglu_fwd<T>(Z, Gt, Tn, f, st);
        lin_fwd(Gt, Wm(D, p, pre + "down.w"), Tn, h, f, Hout, nullptr, H1);
      }
      Hin = Hout;
    }
    if (k == K - 1) {
      // fused head (K13): final norm, then per token chunk logits -> softmax-CE -> dlogits -> the
      // head's dgrad rows (dHf, kept for BW) and wgrad. The loss ends the graph, so the head's
      // backward needs nothing a later instruction produces; running it here keeps only dHf [T, h]
      // instead of dlogits [T, V] alive until BW. CFW (mode 1) records the loss only; RC (mode 2)
      // replays the gradients without the loss; FW does both: each head contribution is added once.
      const HeadScratch HS = head_scratch_layout(m);
      uint8_t* hs = D.template at<uint8_t>(D.a.logits);
      T* Hl = reinterpret_cast<T*>(head_base + HA.H_last);
      float* stf = reinterpret_cast<float*>(head_base + HA.stf);
      T* dHf = reinterpret_cast<T*>(head_base + HA.dHf);
      T* Hf = reinterpret_cast<T*>(hs + HS.Hf);
      float* logits = reinterpret_cast<float*>(hs + HS.logits);
      T* dlog = reinterpret_cast<T*>(hs + HS.dlog);
      const int V = m.vocab;
      if (gpt) layernorm_fwd<T>(Hl, Wf(D, p, "lnf.g"), Wf(D, p, "lnf.b"), Hf, stf, Tn, h, m.norm_eps, st);
      else rmsnorm_fwd<T>(Hl, Wf(D, p, "nf.g"), Hf, stf, Tn, h, m.norm_eps, st);
      const std::string hw = gpt ? (m.tie_embeddings ? "wte" : "head.w") : "out.w";
      const T* Wh = Wm(D, p, hw);
      float* row_loss = reinterpret_cast<float*>(D.template at<uint8_t>(D.a.loss) +
                                                 static_cast<size_t>(D.P->pp.N) * D.P->pp.parts() * 8);
      const float inv_ntok = 1.0f / static_cast<float>(static_cast<double>(D.P->pp.N) * Tn);
      for (int r0 = 0; r0 < Tn; r0 += HS.rows) {
        const int rows = std::min(HS.rows, Tn - r0);
        const T* Hfc = Hf + static_cast<size_t>(r0) * h;
        gemm(Hfc, h, 0, Wh, h, 0, rows, V, h, logits, V, true, 0.f);
        softmax_ce<T>(logits, tok, s + 1, s, rows, V, inv_ntok, dlog, row_loss + r0, st, r0);
        if (mode != 1) {
          lin_dgrad(dlog, Wh, rows, V, h, dHf + static_cast<size_t>(r0) * h);   // dHf rows
          lin_wgrad(dlog, Hfc, rows, V, h, G(D, p, hw));                        // dW_head += dlog^T Hf
        }
      }
      if (mode != 2) loss_reduce(row_loss, Tn, D.template at<double>(D.a.loss) + x.micro, st);
    }
  }

  // ---- backward of one virtual stage ------------------------------------------
  void stage_backward(Dev<T>& D, const mario_instr& x, const T* dout, T* dstage_in) {
    const mario_model& m = D.M();
    const int K = D.P->pp.K(), k = x.vstage, p = x.part, lps = D.P->lps;
    const int Tn = static_cast<int>(tokens_per_micro(m)), h = m.hidden, f = m.ffn_hidden, nh = m.n_heads;
    const int dh = h / nh, s = m.seq_len, mbs = m.micro_batch;
    const bool gpt = m.family == MARIO_GPT;
    const bool sn = D.P->store_act;
    const LayerAct LA = layer_act_layout(m, sn);
    const HeadAct HA = head_act_layout(m);
    const BwScratch BS = bw_scratch_layout(m, sn);
    uint8_t* base = D.template at<uint8_t>(D.a.act + static_cast<size_t>(x.aslot) * D.a.act_stride);
    uint8_t* head_base = base + LA.bytes * lps;
    uint8_t* sc = D.template at<uint8_t>(D.a.bw);
    T* dHbuf[3] = {reinterpret_cast<T*>(sc + BS.dH[0]), reinterpret_cast<T*>(sc + BS.dH[1]),
                   reinterpret_cast<T*>(sc + BS.dH[2])};
    T* dA = reinterpret_cast<T*>(sc + BS.dA);
    T* dQKV = reinterpret_cast<T*>(sc + BS.dQKV);
    T* dO = reinterpret_cast<T*>(sc + BS.dO);
    T* dZ = reinterpret_cast<T*>(sc + BS.dZ);
    T* dM = reinterpret_cast<T*>(sc + BS.dM);
    float* Dsc = reinterpret_cast<float*>(sc + BS.Dsc);
    // the attention backward's D = rowsum(dO o O) per head from the dO GEMM's epilogue (bf16, head dims
    // the unpadded tcgen05 backward takes: the padded path computes D on the unpadded heads itself)
    static const bool fuse_D_env = getenv("MARIO_FUSE_D") ? atoi(getenv("MARIO_FUSE_D")) != 0 : true;
    const bool fuse_D = fuse_D_env && sizeof(T) == 2 && (dh == 64 || dh == 128);
    // bf16 mode (reading A30): the residual-stream gradient dH is carried in fp32 between layers
    // (dH32, two buffers: LN2 reads [0] writes [1], LN1 reads [1] writes [0]); the bf16 dH buffers
    // are the operand copies of the GEMMs. nullptr = the bf16 dH is exact (a received message).
    constexpr bool r32 = sizeof(T) == 2;
    float* dH32buf[2] = {reinterpret_cast<float*>(sc + BS.dH32[0]), reinterpret_cast<float*>(sc + BS.dH32[1])};
    const float* dH32 = nullptr;
    float* red = D.template at<float>(D.a.red);
    const size_t red_floats = D.a.red_bytes / sizeof(float);
    const int32_t* tok = D.template at<int32_t>(D.a.tokens) + static_cast<size_t>(x.micro) * mbs * (s + 1);
    int cur = 0;
    const T* dH;   // gradient of the current layer's output
    if (k == K - 1) {
      // the head's gradients were produced by the fused head of the FW / RC (stage_forward)
      T* Hl = reinterpret_cast<T*>(head_base + HA.H_last);
      float* stf = reinterpret_cast<float*>(head_base + HA.stf);
      const T* dHf = reinterpret_cast<const T*>(head_base + HA.dHf);
      T* dHl = dHbuf[cur];
      if constexpr (r32) {
        norm_bwd_mixed(dHf, Hl, stf, Wf(D, p, gpt ? "lnf.g" : "nf.g"), nullptr, nullptr, dHl, dH32buf[0], Tn, h,
                       gpt ? 0 : 1, G(D, p, gpt ? "lnf.g" : "nf.g"), gpt ? G(D, p, "lnf.b") : nullptr,
                       gpt ? G(D, p, "h" + std::to_string(k * lps + lps - 1) + ".fc2.b") : nullptr, red, red_floats,
                       st);
        dH32 = dH32buf[0];
      } else if (gpt) {
        // + the fc2 bias gradient of this stage's last layer (column sums of dHl)
        norm_bwd<T>(dHf, Hl, stf, Wf(D, p, "lnf.g"), nullptr, dHl, Tn, h, 0, G(D, p, "lnf.g"), G(D, p, "lnf.b"),
                    G(D, p, "h" + std::to_string(k * lps + lps - 1) + ".fc2.b"), red, red_floats, st);
      } else {
        norm_bwd<T>(dHf, Hl, stf, Wf(D, p, "nf.g"), nullptr, dHl, Tn, h, 1, G(D, p, "nf.g"), nullptr, nullptr, red,
                    red_floats, st);
      }
      dH = dHl;
    } else {
      dH = dout;
      cur = 2;   // first written buffer rotates from 0
    }
    for (int li = lps - 1; li >= 0; --li) {
      const int l = k * lps + li;
      const std::string pre = "h" + std::to_string(l) + ".";
      uint8_t* L = base + li * LA.bytes;
      const T* Hin = (li == 0 && k > 0) ? D.template at<T>(D.a.ckpt + static_cast<size_t>(x.slot) * D.a.ckpt_stride)
                                        : reinterpret_cast<T*>(L + LA.H_in);
      // norm outputs A / A2 and the MLP activation G / M: stored in the activation set (store_act),
      // else recomputed (A / A2 into the shared Arec, G / M into the dM buffer)
      T* A = reinterpret_cast<T*>(sn ? L + LA.A : sc + BS.Arec);
      T* A2 = reinterpret_cast<T*>(sn ? L + LA.A2 : sc + BS.Arec);
      T* Gt = sn ? reinterpret_cast<T*>(L + LA.G) : dM;
      T* QKV = reinterpret_cast<T*>(L + LA.QKV);
      T* O = reinterpret_cast<T*>(L + LA.O);
      float* LSE = reinterpret_cast<float*>(L + LA.LSE);
      T* H1 = reinterpret_cast<T*>(L + LA.H1);
      T* Z = reinterpret_cast<T*>(L + LA.Z);
      float* st1 = reinterpret_cast<float*>(L + LA.st1);
      float* st2 = reinterpret_cast<float*>(L + LA.st2);
      T* dH1 = dHbuf[(cur + 1) % 3];
      T* dHin = (li == 0) ? (k == 0 ? dHbuf[(cur + 2) % 3] : dstage_in) : dHbuf[(cur + 2) % 3];
      if (gpt) {
        // dZ = (dH W2) * gelu'(Z); in the lean set the epilogue also recomputes G = gelu(Z) for the fc2
        // wgrad; fc1.b = column sums of dZ: fused into that epilogue (bf16), finished before `red` is reused
        const bool fuse_b1 = sizeof(T) == 2 && Tn % 32 == 0 && f % 32 == 0 &&
                             static_cast<size_t>(Tn / 32) * f <= red_floats;
        lin_dgrad(dH, Wm(D, p, pre + "fc2.w"), Tn, h, f, dZ, Z, sn ? nullptr : Gt, fuse_b1 ? red : nullptr);
        if (fuse_b1) colsum_finish(red, Tn / 32, f, G(D, p, pre + "fc1.b"), st);
        lin_wgrad(dH, Gt, Tn, h, f, G(D, p, pre + "fc2.w"));
        // fc2.b: fused into the norm backward that wrote dH (this stage), else a column sum here
        if (li == lps - 1 && k != K - 1) colsum<T>(dH, nullptr, nullptr, Tn, h, h, 0, G(D, p, pre + "fc2.b"), nullptr, red, st);
        if (!sn) norm_recompute<T>(H1, Wf(D, p, pre + "ln2.g"), Wf(D, p, pre + "ln2.b"), A2, st2, Tn, h, m.norm_eps, 0, st);
        if (!fuse_b1) colsum<T>(dZ, nullptr, nullptr, Tn, f, f, 0, G(D, p, pre + "fc1.b"), nullptr, red, st);
        lin_dgrad(dZ, Wm(D, p, pre + "fc1.w"), Tn, f, h, dA);               // dA2
        on_side(D, [&] { lin_wgrad(dZ, A2, Tn, f, h, G(D, p, pre + "fc1.w")); });
        if constexpr (r32)
          norm_bwd_mixed(dA, H1, st2, Wf(D, p, pre + "ln2.g"), dH32 ? nullptr : dH, dH32, dH1, dH32buf[1], Tn, h, 0,
                         G(D, p, pre + "ln2.g"), G(D, p, pre + "ln2.b"), G(D, p, pre + "proj.b"), red, red_floats, st);
        else
          norm_bwd<T>(dA, H1, st2, Wf(D, p, pre + "ln2.g"), dH, dH1, Tn, h, 0, G(D, p, pre + "ln2.g"),
                      G(D, p, pre + "ln2.b"), G(D, p, pre + "proj.b"), red, red_floats, st);
        if (fuse_D) lin_dgrad_dot(dH1, Wm(D, p, pre + "proj.w"), Tn, h, h, dO, O, Dsc, dh);
        else lin_dgrad(dH1, Wm(D, p, pre + "proj.w"), Tn, h, h, dO);
        on_side(D, [&] { lin_wgrad(dH1, O, Tn, h, h, G(D, p, pre + "proj.w")); });
      } else {
        if (!sn) swiglu_fwd<T>(Z, Gt, Tn, f, st);                             // recompute M (into dM)
        lin_wgrad(dH, Gt, Tn, h, f, G(D, p, pre + "down.w"));
        lin_dgrad(dH, Wm(D, p, pre + "down.w"), Tn, h, f, dM);              // overwrites M (consumed)
        swiglu_bwd<T>(Z, dM, dZ, Tn, f, st);
        if (!sn) norm_recompute<T>(H1, Wf(D, p, pre + "n2.g"), nullptr, A2, st2, Tn, h, m.norm_eps, 1, st);
        lin_dgrad(dZ, Wm(D, p, pre + "gu.w"), Tn, 2 * f, h, dA);
        on_side(D, [&] { lin_wgrad(dZ, A2, Tn, 2 * f, h, G(D, p, pre + "gu.w")); });
        if constexpr (r32)
          norm_bwd_mixed(dA, H1, st2, Wf(D, p, pre + "n2.g"), dH32 ? nullptr : dH, dH32, dH1, dH32buf[1], Tn, h, 1,
                         G(D, p, pre + "n2.g"), nullptr, nullptr, red, red_floats, st);
        else
          norm_bwd<T>(dA, H1, st2, Wf(D, p, pre + "n2.g"), dH, dH1, Tn, h, 1, G(D, p, pre + "n2.g"), nullptr, nullptr,
                      red, red_floats, st);
        if (fuse_D) lin_dgrad_dot(dH1, Wm(D, p, pre + "o.w"), Tn, h, h, dO, O, Dsc, dh);
        else lin_dgrad(dH1, Wm(D, p, pre + "o.w"), Tn, h, h, dO);
        on_side(D, [&] { lin_wgrad(dH1, O, Tn, h, h, G(D, p, pre + "o.w")); });
      }
      // O = nullptr: D = rowsum(dO o O) is already in Dsc (fused into the dO GEMM above). GPT: the
      // attention kernels may also leave the qkv-bias column partials per 32 tokens in `red`
      static const bool fuse_qkvb = getenv("MARIO_FUSE_QKVB") ? atoi(getenv("MARIO_FUSE_QKVB")) != 0 : true;
      const bool bp_fit = fuse_qkvb && gpt && Tn % 32 == 0 && static_cast<size_t>(Tn / 32) * 3 * h <= red_floats;
      bool qkvb_part = false;
      attn_bwd<T>(QKV, fuse_D ? nullptr : O, dO, LSE, dQKV, Dsc, mbs, s, nh, dh, st, BS.dS_bytes ? sc + BS.dS : nullptr,
                  BS.dS_bytes, BS.attn_pad_bytes ? sc + BS.attn_pad : nullptr, bp_fit ? red : nullptr, &qkvb_part);
      if (!gpt) rope<T>(dQKV, mbs, s, nh, dh, m.rope_base, 1, st, rope_tab(D));
      if (!sn) {
        join_side(D);   // the fc1 / MLP-input wgrad read A2 (Arec), which the recompute below overwrites
        if (gpt) norm_recompute<T>(Hin, Wf(D, p, pre + "ln1.g"), Wf(D, p, pre + "ln1.b"), A, st1, Tn, h, m.norm_eps, 0, st);
        else norm_recompute<T>(Hin, Wf(D, p, pre + "n1.g"), nullptr, A, st1, Tn, h, m.norm_eps, 1, st);
      }
      if (gpt && qkvb_part) colsum_finish(red, Tn / 32, 3 * h, G(D, p, pre + "qkv.b"), st);
      else if (gpt) colsum<T>(dQKV, nullptr, nullptr, Tn, 3 * h, 3 * h, 0, G(D, p, pre + "qkv.b"), nullptr, red, st);
      lin_dgrad(dQKV, Wm(D, p, pre + "qkv.w"), Tn, 3 * h, h, dA);
      on_side(D, [&] { lin_wgrad(dQKV, A, Tn, 3 * h, h, G(D, p, pre + "qkv.w")); });
      if constexpr (r32) {
        // the stage input's gradient leaves as a bf16 message (SG): no fp32 copy needed there
        float* out32 = (li == 0 && k > 0) ? nullptr : dH32buf[0];
        norm_bwd_mixed(dA, Hin, st1, Wf(D, p, pre + (gpt ? "ln1.g" : "n1.g")), nullptr, dH32buf[1], dHin, out32, Tn,
                       h, gpt ? 0 : 1, G(D, p, pre + (gpt ? "ln1.g" : "n1.g")), gpt ? G(D, p, pre + "ln1.b") : nullptr,
                       (gpt && li > 0) ? G(D, p, "h" + std::to_string(l - 1) + ".fc2.b") : nullptr, red, red_floats,
                       st);
        dH32 = out32;
      } else if (gpt) {
        // + the previous layer's fc2 bias gradient (column sums of dHin) when it is on this stage
        norm_bwd<T>(dA, Hin, st1, Wf(D, p, pre + "ln1.g"), dH1, dHin, Tn, h, 0, G(D, p, pre + "ln1.g"),
                    G(D, p, pre + "ln1.b"), li > 0 ? G(D, p, "h" + std::to_string(l - 1) + ".fc2.b") : nullptr, red,
                    red_floats, st);
      } else {
        norm_bwd<T>(dA, Hin, st1, Wf(D, p, pre + "n1.g"), dH1, dHin, Tn, h, 1, G(D, p, pre + "n1.g"), nullptr, nullptr,
                    red, red_floats, st);
      }
      join_side(D);   // this layer's wgrads read buffers the next layer overwrites
      dH = dHin;
      cur = (cur + 2) % 3;
    }
    if (k == 0) {
      if (r32 && dH32)
        embed_bwd<float>(tok, s + 1, mbs, s, dH32, h, G(D, p, gpt ? "wte" : "emb"), gpt ? G(D, p, "wpe") : nullptr,
                         sc + BS.sort, st);
      else
        embed_bwd<T>(tok, s + 1, mbs, s, dH, h, G(D, p, gpt ? "wte" : "emb"), gpt ? G(D, p, "wpe") : nullptr,
                     sc + BS.sort, st);
    }
  }

  // ---- one instruction ----------------------------------------------------------
  T* send_slot(Dev<T>& D, bool grad, int idx) {
    return D.template at<T>((grad ? D.a.sg : D.a.sa) + static_cast<size_t>(idx) * D.a.msg_stride);
  }

  void run_instr(int d, const mario_instr& x) {
    Dev<T>& D = dev(d);
    if (peer) { st = D.st; set_sm_budget(D.sms); }
    const mario_model& m = D.M();
    const int K = D.P->pp.K();
    const auto key = std::make_pair(x.micro, x.part);
    const size_t msg_bytes = tokens_per_micro(m) * m.hidden * sizeof(T);
    switch (x.op) {
      case MARIO_OP_FW:
      case MARIO_OP_CFW:
      case MARIO_OP_RC: {
        T* out = nullptr;
        if (x.op != MARIO_OP_RC && x.vstage < K - 1) {
          const int i = (loopback ? D.P->sa_slot_lb : D.P->sa_slot)[d].at(key);   // the plan's slot
          if (D.sa_used.at(i)) throw std::runtime_error("send slot still held (planner/executor mismatch)");
          D.sa_used[i] = true;
          D.sa_of[key] = i;
          if (peer) {
            if (D.sa_guard[i]) DRV(drv::wait_flag(st, D.sa_guard[i], fv));   // previous message consumed
          } else if (!loopback && D.sa_free_set[i]) {
            CU(cudaStreamWaitEvent(st, D.sa_free[i], 0));
          }
          out = send_slot(D, false, i);
        } else if (x.op == MARIO_OP_RC && x.vstage < K - 1) {
          out = D.template at<T>(D.a.cfw);   // RC's stage output is not needed: scratch
        }
        timed_begin(D);
        stage_forward(D, x, x.op == MARIO_OP_FW ? 0 : x.op == MARIO_OP_CFW ? 1 : 2, out);
        timed_end(D);
        break;
      }
      case MARIO_OP_BW: {
        const T* dout = nullptr;
        if (x.vstage < K - 1) dout = D.template at<T>(D.a.rg + static_cast<size_t>(D.rg_of[key]) * D.a.msg_stride);
        T* din = nullptr;
        if (x.vstage > 0) {
          const int i = (loopback ? D.P->sg_slot_lb : D.P->sg_slot)[d].at(key);
          if (D.sg_used.at(i)) throw std::runtime_error("send slot still held (planner/executor mismatch)");
          D.sg_used[i] = true;
          D.sg_of[key] = i;
          if (peer) {
            if (D.sg_guard[i]) DRV(drv::wait_flag(st, D.sg_guard[i], fv));
          } else if (!loopback && D.sg_free_set[i]) {
            CU(cudaStreamWaitEvent(st, D.sg_free[i], 0));
          }
          din = send_slot(D, true, i);
        }
        timed_begin(D);
        stage_backward(D, x, dout, din);
        timed_end(D);
        // release stage-input slot, recv-grad slot (activation slots are list-order, planner-assigned)
        if (x.slot >= 0 && !loopback) { CU(cudaEventRecord(D.ck_free[x.slot], st)); D.ck_free_set[x.slot] = true; }
        if (x.vstage < K - 1) {
          int i = D.rg_of[key];
          if (!loopback) { CU(cudaEventRecord(D.rg_free[i], st)); D.rg_free_set[i] = true; }
          D.rg_used[i] = false;
          D.rg_of.erase(key);
        }
        break;
      }
      case MARIO_OP_SA:
      case MARIO_OP_SG:
        // loopback: the receiver copies out of the held slot; NCCL: the send is issued by
        // issue_send() from the rank's comm program, in the receiver's order
        if (peer) {
          // buffered send at its list position: mark the message complete; the slot is
          // free for this rank's next message once the receiver's "consumed" flag is up
          const bool grad = x.op == MARIO_OP_SG;
          auto& of = grad ? D.sg_of : D.sa_of;
          const int i = of.at(key);
          const int kd = grad ? x.vstage - 1 : x.vstage + 1;
          DRV(drv::write_flag(st, flag_ready(grad, kd, x.micro), fv));
          (grad ? D.sg_guard : D.sa_guard)[i] = flag_done(grad, kd, x.micro);
          (grad ? D.sg_guard_key : D.sa_guard_key)[i] = std::make_tuple(grad ? 1 : 0, kd, x.micro);
          (grad ? D.sg_used : D.sa_used)[i] = false;
          of.erase(key);
          ready_walked.insert(std::make_tuple(grad ? 1 : 0, kd, x.micro));
        }
        break;
      case MARIO_OP_RA:
      case MARIO_OP_RG: {
        const bool grad = x.op == MARIO_OP_RG;
        T* dst;
        if (!grad) {
          dst = D.template at<T>(D.a.ckpt + static_cast<size_t>(x.slot) * D.a.ckpt_stride);
        } else {
          int i = acquire(D.rg_used);
          D.rg_of[key] = i;
          dst = D.template at<T>(D.a.rg + static_cast<size_t>(i) * D.a.msg_stride);
        }
        if (peer) {
          // blocking receive: wait for the sender's flag, pull the message out of the
          // sender's slot on this rank's receive stream, flag it consumed, then the compute stream
          // waits for the copy at this list position
          const int kind = grad ? 1 : 0;
          // the sender (Alg. 1 find_prev) and the slot the plan gave its message
          int sd = -1, sp = -1;
          plan::find_inst(D.P->pp, d, x.micro, x.part, grad ? MARIO_OP_BW : MARIO_OP_FW, false, &sd, &sp);
          const std::pair<int, int> src{sd, (grad ? D.P->sg_slot : D.P->sa_slot)[sd].at({x.micro, sp})};
          Dev<T>& Sd = dev(src.first);
          // MARIO_PEER_RX=0: receive on the compute stream itself (no prefetch, fewer streams)
          static const bool rx_streams = !getenv("MARIO_PEER_RX") || atoi(getenv("MARIO_PEER_RX")) != 0;
          cudaStream_t rs = rx_streams ? D.rx[kind] : st;
          if (!grad && D.ck_free_set[x.slot]) CU(cudaStreamWaitEvent(rs, D.ck_free[x.slot], 0));
          if (grad) {
            const int i = D.rg_of[key];
            if (D.rg_free_set[i]) CU(cudaStreamWaitEvent(rs, D.rg_free[i], 0));
          }
          DRV(drv::wait_flag(rs, flag_ready(kind, x.vstage, x.micro), fv));
          CU(cudaMemcpyAsync(dst, send_slot(Sd, grad, src.second), msg_bytes, cudaMemcpyDeviceToDevice, rs));
          DRV(drv::write_flag(rs, flag_done(kind, x.vstage, x.micro), fv));
          consumed_walked.insert(std::make_tuple(kind, x.vstage, x.micro));
          if (rs != st) {
            cudaEvent_t e = D.event();
            CU(cudaEventRecord(e, rs));
            CU(cudaStreamWaitEvent(st, e, 0));
          }
        } else if (loopback) {
          Dev<T>& Sd = dev(x.peer);
          // the sender's part for this micro-batch: find via its held slots
          int sp = -1;
          auto& sof = grad ? Sd.sg_of : Sd.sa_of;
          for (auto& kv : sof) if (kv.first.first == x.micro && sender_part_ok(Sd, kv.first.second, x, grad)) { sp = kv.first.second; break; }
          if (sp < 0) throw std::runtime_error("loopback: no held send slot for receive");
          const int i = sof[{x.micro, sp}];
          CU(cudaMemcpyAsync(dst, send_slot(Sd, grad, i), msg_bytes, cudaMemcpyDeviceToDevice, st));
          (grad ? Sd.sg_used : Sd.sa_used)[i] = false;
          sof.erase({x.micro, sp});
        } else {
          Channel& ch = channel(x.peer, D.d, grad ? 1 : 0);
          if (!grad && D.ck_free_set[x.slot]) CU(cudaStreamWaitEvent(ch.stream, D.ck_free[x.slot], 0));
          if (grad) {
            int i = D.rg_of[key];
            if (D.rg_free_set[i]) CU(cudaStreamWaitEvent(ch.stream, D.rg_free[i], 0));
          }
          NC(ncclRecv(dst, msg_bytes, ncclUint8, peer_in_channel(D.d, x.peer), ch.comm, ch.stream));
          cudaEvent_t e = D.event();
          CU(cudaEventRecord(e, ch.stream));
          CU(cudaStreamWaitEvent(st, e, 0));   // blocking receive at this list position
        }
        break;
      }
    }
  }

  // peer: may instruction x of rank d be enqueued now, i.e. is every flag it will wait on already
  // written by enqueued work? (receives: the sender's "ready"; a send slot's reuse: the previous
  // message's "consumed")
  bool can_walk(int d, const mario_instr& x) {
    Dev<T>& D = dev(d);
    const int K = D.P->pp.K();
    const auto key = std::make_pair(x.micro, x.part);
    auto slot_ok = [&](int i, const std::vector<const uint32_t*>& guard,
                       const std::vector<std::tuple<int, int, int>>& gkey) {
      return !guard[i] || consumed_walked.count(gkey[i]) > 0;
    };
    switch (x.op) {
      case MARIO_OP_RA: return ready_walked.count(std::make_tuple(0, x.vstage, x.micro)) > 0;
      case MARIO_OP_RG: return ready_walked.count(std::make_tuple(1, x.vstage, x.micro)) > 0;
      case MARIO_OP_FW:
      case MARIO_OP_CFW: return x.vstage >= K - 1 || slot_ok(D.P->sa_slot[d].at(key), D.sa_guard, D.sa_guard_key);
      case MARIO_OP_BW: return x.vstage == 0 || slot_ok(D.P->sg_slot[d].at(key), D.sg_guard, D.sg_guard_key);
      default: return true;
    }
  }

  void issue_send(Dev<T>& D, const mario_commop& op) {
    const bool grad = op.c == 1;
    auto& of = grad ? D.sg_of : D.sa_of;
    const auto key = std::make_pair(op.micro, op.part);
    auto it = of.find(key);
    if (it == of.end()) throw std::runtime_error("send: message not produced");
    const int i = it->second;
    Channel& ch = channel(D.d, op.b, op.c);
    cudaEvent_t e = D.event();
    CU(cudaEventRecord(e, st));
    CU(cudaStreamWaitEvent(ch.stream, e, 0));
    NC(ncclSend(send_slot(D, grad, i), static_cast<size_t>(op.count), ncclUint8, peer_in_channel(D.d, op.b), ch.comm,
                ch.stream));
    auto& fr = grad ? D.sg_free : D.sa_free;
    auto& fs = grad ? D.sg_free_set : D.sa_free_set;
    CU(cudaEventRecord(fr[i], ch.stream));
    fs[i] = true;
    (grad ? D.sg_used : D.sa_used)[i] = false;
    of.erase(it);
  }

  bool sender_part_ok(Dev<T>& Sd, int sp, const mario_instr& x, bool grad) {
    // the sender's virtual stage must be adjacent to ours in the right direction
    const int ks = Sd.P->pp.vstage(Sd.d, sp);
    return grad ? ks == x.vstage + 1 : ks == x.vstage - 1;
  }

  void timed_begin(Dev<T>& D) {
    if (!g.timing) return;
    cudaEvent_t a, b;
    CU(cudaEventCreate(&a));
    CU(cudaEventCreate(&b));
    CU(cudaEventRecord(a, st));
    D.timed.push_back({a, b});
  }
  void timed_end(Dev<T>& D) {
    if (!g.timing) return;
    CU(cudaEventRecord(D.timed.back().second, st));
  }

  Channel& channel(int src, int dst, int kind) {
    auto it = g.channels.find({src, dst, kind});
    if (it == g.channels.end()) throw std::runtime_error("missing NCCL channel");
    return it->second;
  }
  static int peer_in_channel(int me, int other) { return me < other ? 1 : 0; }   // 2-rank comm: lo=0, hi=1
};

// Create per-channel 2-rank communicators for every (src, dst, kind) the plan uses, plus the
// pair communicators for gradient synchronisation. Collective over all ranks: every rank
// iterates the same sorted set.
// With PP x DP every split op is issued by all ranks of all replicas; each replica's members pass
// their replica as the colour, so one call creates one communicator per replica. Channels and
// pairs are stored in stage space (the replica offset removed).
void ensure_channels(const PlanObj& P) {
  const int S = P.pp.S, off = (g.rank / S) * S, color = 1 + g.rank / S;
  for (const mario_commop& op : comm_program_dp(P, g.dp, g.rank)) {
    if (op.kind == 0) {
      const auto c = std::make_tuple(op.a - off, op.b - off, op.c);
      if (g.created_channels.count(c)) continue;
      g.created_channels.insert(c);
      const int lo = std::min(op.a, op.b), hi = std::max(op.a, op.b);
      const bool member = g.rank == lo || g.rank == hi;
      ncclComm_t comm = nullptr;
      NC(ncclCommSplit(g.world_comm, member ? color : NCCL_SPLIT_NOCOLOR, g.rank == lo ? 0 : 1, &comm, nullptr));
      if (member) {
        Channel ch;
        ch.comm = comm;
        CU(cudaStreamCreateWithFlags(&ch.stream, cudaStreamNonBlocking));
        g.channels[c] = ch;
      }
    } else if (op.kind == 1) {
      const auto pr = std::make_pair(op.a - off, op.b - off);
      if (g.created_pairs.count(pr)) continue;
      g.created_pairs.insert(pr);
      const bool member = g.rank == op.a || g.rank == op.b;
      ncclComm_t comm = nullptr;
      NC(ncclCommSplit(g.world_comm, member ? color : NCCL_SPLIT_NOCOLOR, g.rank == op.a ? 0 : 1, &comm, nullptr));
      if (member) g.pair_comms[pr] = comm;
    } else if (op.kind == 6 && !g.dp_comm) {
      NC(ncclCommSplit(g.world_comm, op.a, op.b, &g.dp_comm, nullptr));   // colour = stage, key = replica
    }
  }
}

template <class T>
mario_status run_iter_t(const PlanObj& P, const void* weights, const int32_t* tokens, float* loss, void* grads,
                        void* workspace, cudaStream_t st) {
  const bool peer = g.emulated || g.ipc;
  const bool loopback = !peer && g.world == 1 && P.pp.S > 1;
  if (g.emulated && P.pp.S != static_cast<int>(g.emu_st.size()))
    return set_error(MARIO_ESTATE, "plan stages != emulated world size");
  if (g.ipc) {
    if (P.pp.S != g.world) return set_error(MARIO_ESTATE, "plan stages != peer world size");
    if (static_cast<int>(g.peers.size()) != g.world || workspace != g.bound_ws || grads != g.bound_gr)
      return set_error(MARIO_ESTATE, "buffers not bound: mario_peer_export / mario_peer_import first");
  }
  if (!loopback && !peer && P.pp.S * g.dp != g.world) return set_error(MARIO_ESTATE, "plan stages * dp != world size");
  const int me = g.rank % P.pp.S, off = g.rank - me;   // stage and the replica's rank offset
  const auto& prog = comm_program_dp(P, g.dp, g.rank);
  Exec<T> E;
  E.st = st;
  E.loopback = loopback;
  E.peer = peer;
  if (g.ipc) {
    E.me = g.rank;
    E.fv = ++g.epoch;
  }
  const mario_model& m = P.model;
  const int S = P.pp.S;
  std::vector<int> my_devs;
  if (loopback || peer) for (int d = 0; d < S; ++d) my_devs.push_back(d);
  else my_devs.push_back(me);
  // peer: flag block = [ready | done][activation | gradient][K][N] + per-rank "backward done" + one
  // "chunk summed" flag per (multi-copy parameter, copy)
  std::map<int, std::vector<std::pair<int, int>>> copies;   // global param idx -> (dev, packed j)
  for (int d = 0; d < S; ++d) {
    const auto& rp = P.rank_params[d];
    for (size_t j = 0; j < rp.idx.size(); ++j) copies[rp.idx[j]].push_back({d, static_cast<int>(j)});
  }
  size_t n_multi_flags = 0;
  for (auto& kv : copies) if (kv.second.size() > 1) n_multi_flags += kv.second.size();
  size_t flag_words = 0;
  if (peer) {
    E.fK = P.pp.K();
    E.fN = P.pp.N;
    // + per rank: backward done, (ipc) gathered, (ipc) loss ready
    flag_words = static_cast<size_t>(4) * E.fK * E.fN + 3 * S + n_multi_flags;
    if (g.ipc) {
      if (flag_words > g.ipc_flag_words) return set_error(MARIO_EINVAL, "plan needs more peer flags than allocated");
      E.flags = g.peers[0].flags;
    } else if (g.flags_cap < flag_words) {
      if (g.flags) CU(cudaFree(g.flags));
      g.flags = nullptr;
      CU(cudaMalloc(&g.flags, flag_words * 4));
      g.flags_cap = flag_words;
    }
    if (!g.ipc) E.flags = g.flags;
  }
  size_t wofs = 0, wsofs = 0;
  for (int d : my_devs) {
    auto D = std::make_unique<Dev<T>>();
    D->P = &P;
    D->d = d;
    const auto& pools = loopback ? P.pools_lb[d] : P.pools_mp[d];
    if (g.emulated) {
      D->st = g.emu_st[d];
      D->rx[0] = g.emu_rx[d][0];
      D->rx[1] = g.emu_rx[d][1];
      D->side = g.emu_side[d];
      D->sms = g.emu_sms;
    } else if (g.ipc && d == E.me) {
      D->st = g.ipc_st;
      D->rx[0] = g.ipc_rx[0];
      D->rx[1] = g.ipc_rx[1];
      D->side = g.ipc_side;
    } else {
      if (!g.side_st) CU(cudaStreamCreateWithFlags(&g.side_st, cudaStreamNonBlocking));
      D->side = g.side_st;
    }
    D->a = make_arena(P, d, pools);
    D->ws = static_cast<uint8_t*>(workspace) + wsofs;
    D->w = static_cast<const float*>(weights) + wofs;
    D->gr = static_cast<float*>(grads) + wofs;
    if (g.ipc && d != E.me) {   // another process's rank: its mapped workspace and grads
      D->ws = g.peers[d].ws;
      D->gr = g.peers[d].gr;
      D->w = nullptr;
    }
    const auto& rp = P.rank_params[d];
    for (size_t j = 0; j < rp.idx.size(); ++j) D->tensor[{rp.part[j], rp.idx[j]}] = static_cast<int>(j);
    D->sa_used.assign(std::max(1, pools.send_act), false);
    D->sg_used.assign(std::max(1, pools.send_grad), false);
    D->rg_used.assign(std::max(1, pools.recv_grad), false);
    auto mk = [&](std::vector<cudaEvent_t>& v, std::vector<bool>& set, size_t n) {
      v.resize(n);
      set.assign(n, false);
      for (auto& e : v) e = ev_get();
    };
    mk(D->sa_free, D->sa_free_set, D->sa_used.size());
    mk(D->sg_free, D->sg_free_set, D->sg_used.size());
    mk(D->rg_free, D->rg_free_set, D->rg_used.size());
    mk(D->ck_free, D->ck_free_set, std::max(1, pools.ckpt));
    D->sa_guard.assign(D->sa_used.size(), nullptr);
    D->sg_guard.assign(D->sg_used.size(), nullptr);
    D->sa_guard_key.assign(D->sa_used.size(), {});
    D->sg_guard_key.assign(D->sg_used.size(), {});
    if (loopback) {
      wofs += rp.total;
      wsofs += align_up(P.workspace_lb[d], 1 << 20);
    } else if (g.emulated) {
      wofs += rp.total;
      wsofs += align_up(P.workspace_mp[d], 1 << 20);
    }
    // tokens H2D (outside any captured graph: the host buffer changes every call)
    const size_t tok_bytes = static_cast<size_t>(P.pp.N) * m.micro_batch * (m.seq_len + 1) * 4;
    if (E.mine(d))
      CU(cudaMemcpyAsync(D->ws + D->a.tokens, tokens, tok_bytes, cudaMemcpyDefault, st));   // host or device tokens
    E.devs.push_back(std::move(D));
  }
  if (!loopback && !peer && g.world > 1) ensure_channels(P);

  // Single-process iterations are a fixed launch sequence over fixed buffers: the second call
  // with the same (plan, weights, grads, workspace) is captured into a CUDA graph, later calls
  // replay it (no per-kernel launch cost). Disabled while timing/kstats instrumentation is on.
  const bool graphable = g.graphs && g.world == 1 && !g.timing && !g.ipc;
  const auto gkey = std::make_tuple(P.serial, weights, static_cast<const void*>(grads),
                                    static_cast<const void*>(workspace), kstats_generation());
  bool replayed = false, capturing = false;
  if (graphable) {
    if (!g.cap_stream) CU(cudaStreamCreateWithFlags(&g.cap_stream, cudaStreamNonBlocking));
    cudaEvent_t e0 = E.devs[0]->event();
    CU(cudaEventRecord(e0, st));
    CU(cudaStreamWaitEvent(g.cap_stream, e0, 0));
    auto it = g.graph_cache.find(gkey);
    if (it != g.graph_cache.end()) {
      CU(cudaGraphLaunch(it->second, g.cap_stream));
      note_launch(static_cast<int>(g.graph_kernels[gkey]));   // kernels executed by the replay
      replayed = true;
    } else if (g.graph_seen.count(gkey)) {
      CU(cudaStreamBeginCapture(g.cap_stream, cudaStreamCaptureModeThreadLocal));
      E.st = g.cap_stream;
      capturing = true;
      g.graph_kernels[gkey] = -mario_kernel_launches();
    } else {
      g.graph_seen.insert(gkey);
    }
  }
  cudaStream_t body = E.st;
  cudaEvent_t t0_peer = nullptr;
  if (!replayed) {
  if (peer) {
    // reset the flags (ipc: epochs instead), then fork every rank's streams off the caller's stream
    if (!g.ipc) CU(cudaMemsetAsync(E.flags, 0, flag_words * 4, body));
    if (g.timing) {
      CU(cudaEventCreate(&t0_peer));
      CU(cudaEventRecord(t0_peer, body));
    }
    cudaEvent_t fork = E.devs[0]->event();
    CU(cudaEventRecord(fork, body));
    for (auto& Dp : E.devs) {
      if (!E.mine(Dp->d)) continue;
      CU(cudaStreamWaitEvent(Dp->st, fork, 0));
      CU(cudaStreamWaitEvent(Dp->rx[0], fork, 0));
      CU(cudaStreamWaitEvent(Dp->rx[1], fork, 0));
    }
  }
  for (auto& Dp : E.devs) {
    Dev<T>& D = *Dp;
    if (!E.mine(D.d)) continue;
    const auto& rp = P.rank_params[D.d];
    cudaStream_t s0 = peer ? D.st : body;
    if (peer) set_sm_budget(D.sms);
    CU(cudaMemsetAsync(D.gr, 0, rp.total * 4, s0));
    CU(cudaMemsetAsync(D.ws + D.a.loss, 0, static_cast<size_t>(P.pp.N) * P.pp.parts() * 8, s0));
    if (sizeof(T) == 2)
      for (size_t j = 0; j < rp.idx.size(); ++j)
        if (D.a.wcopy[j] != SIZE_MAX)
          cast_f32_bf16(D.w + rp.off[j], reinterpret_cast<__nv_bfloat16*>(D.ws + D.a.wcopy[j]), rp.cnt[j], s0);
    if (D.a.rope != SIZE_MAX)
      rope_table(reinterpret_cast<float2*>(D.ws + D.a.rope), m.seq_len, m.hidden / m.n_heads, m.rope_base, s0);
  }

  // walk the plan
  if (loopback) {
    for (auto [d, i] : P.loopback_order) E.run_instr(d, P.instrs[d][i]);
  } else if (g.ipc) {
    // one rank per process: walk this rank's list; every flag it waits on is raised by another
    // process (own context, own hardware queues), so no cross-rank enqueue order is needed
    for (const mario_instr& x : P.instrs[E.me]) E.run_instr(E.me, x);
    E.st = body;
  } else if (peer) {
    // every rank runs on its own streams and waits only on flags, so the device executes the
    // plan's DAG concurrently. The host enqueues in peer_order (the simulated timeline, the order in
    // which the send slots were assigned), so every flag wait follows the write it waits for
    for (auto [d, i] : P.peer_order) {
      if (!E.can_walk(d, P.instrs[d][i])) throw std::runtime_error("peer walk: a flag wait precedes its write");
      E.run_instr(d, P.instrs[d][i]);
    }
    E.st = body;
    set_sm_budget(0);
  } else {
    const auto& L = P.instrs[me];
    std::vector<std::vector<mario_commop>> sends_after(L.size());
    for (mario_commop op : prog)
      if (op.kind == 2) { op.a -= off; op.b -= off; sends_after[op.list_index].push_back(op); }   // stage space
    for (size_t i = 0; i < L.size(); ++i) {
      E.run_instr(me, L[i]);
      for (const mario_commop& op : sends_after[i]) E.issue_send(*E.devs[0], op);
    }
    // the iteration ends when every channel stream has drained (its last sends complete)
    for (auto& kv : g.channels) {
      cudaEvent_t e = E.devs[0]->event();
      CU(cudaEventRecord(e, kv.second.stream));
      CU(cudaStreamWaitEvent(st, e, 0));
    }
  }

  // gradient finalization (reading A7): sum every copy of each parameter (tied embeddings,
  // Chimera replicas) and write the sum back to every copy.
  if (peer) {
    // Every copy of a multi-copy parameter (tied wte, Chimera replicas) is summed in copy order,
    // one element chunk per copy, by the chunk's owner rank reading the other copies in peer memory
    // (a reduce-scatter); the owners flag their chunks done and every other holder pulls them back
    // (an all-gather). Flags: per-rank "all BW done" before any chunk is read, per-chunk "summed"
    // before it is copied back, so no copy is overwritten while another rank still reads it.
    const uint32_t fv = E.fv;
    for (auto& Dp : E.devs) if (E.mine(Dp->d)) DRV(drv::write_flag(Dp->st, E.flag_misc(Dp->d), fv));
    size_t fi = static_cast<size_t>(S);
    for (auto& kv : copies) {
      const auto& cp = kv.second;
      if (cp.size() < 2) continue;
      if (cp.size() > 8) throw std::runtime_error("more than 8 copies of a parameter");
      const size_t n = P.rank_params[cp[0].first].cnt[cp[0].second];
      auto ptr = [&](std::pair<int, int> c) { return E.dev(c.first).gr + P.rank_params[c.first].off[c.second]; };
      const size_t nc = cp.size(), chunk = (n + nc - 1) / nc;
      for (size_t c = 0; c < nc; ++c) {                       // reduce-scatter: owner of chunk c = copy c
        if (!E.mine(cp[c].first)) continue;
        Dev<T>& O = E.dev(cp[c].first);
        const size_t lo = std::min(n, c * chunk), hi = std::min(n, lo + chunk);
        for (auto& h : cp) DRV(drv::wait_flag(O.st, E.flag_misc(h.first), fv));
        CopySrcs src{};
        src.n = static_cast<int>(nc);
        for (size_t j = 0; j < nc; ++j) src.p[j] = ptr(cp[j]) + lo;
        if (hi > lo) sum_copies_f32(ptr(cp[c]) + lo, src, hi - lo, O.st);
        DRV(drv::write_flag(O.st, E.flag_misc(fi + c), fv));
      }
      for (size_t c = 0; c < nc; ++c) {                       // all-gather
        const size_t lo = std::min(n, c * chunk), hi = std::min(n, lo + chunk);
        for (size_t j = 0; j < nc; ++j) {
          if (j == c || !E.mine(cp[j].first)) continue;
          Dev<T>& H = E.dev(cp[j].first);
          DRV(drv::wait_flag(H.st, E.flag_misc(fi + c), fv));
          if (hi > lo) CU(cudaMemcpyAsync(ptr(cp[j]) + lo, ptr(cp[c]) + lo, (hi - lo) * 4, cudaMemcpyDeviceToDevice, H.st));
        }
      }
      fi += nc;
    }
    if (g.ipc) {
      // no rank may start its next iteration (zeroing grads, overwriting slots) while another still
      // reads its memory: all-gathered barrier; then the last stage(s)' loss partials are readable
      Dev<T>& D = E.dev(E.me);
      const size_t gath = fi, lossf = fi + S;
      DRV(drv::write_flag(D.st, E.flag_misc(gath + E.me), fv));
      for (int r = 0; r < S; ++r) DRV(drv::wait_flag(D.st, E.flag_misc(gath + r), fv));
      DRV(drv::write_flag(D.st, E.flag_misc(lossf + E.me), fv));
      for (int r = 0; r < S; ++r) DRV(drv::wait_flag(D.st, E.flag_misc(lossf + r), fv));
    }
    // join every rank's stream back into the caller's (or capture) stream
    for (auto& Dp : E.devs) {
      if (!E.mine(Dp->d)) continue;
      cudaEvent_t e = Dp->event();
      CU(cudaEventRecord(e, Dp->st));
      CU(cudaStreamWaitEvent(body, e, 0));
    }
  } else if (loopback) {
    for (auto& kv : copies) {
      if (kv.second.size() < 2) continue;
      auto ptr = [&](std::pair<int, int> c) { return E.dev(c.first).gr + P.rank_params[c.first].off[c.second]; };
      const size_t n = P.rank_params[kv.second[0].first].cnt[kv.second[0].second];
      float* acc = ptr(kv.second[0]);
      for (size_t c = 1; c < kv.second.size(); ++c) add_f32(acc, ptr(kv.second[c]), n, E.st);
      for (size_t c = 1; c < kv.second.size(); ++c) copy_f32(ptr(kv.second[c]), acc, n, E.st);
    }
  } else if (S > 1 || g.dp > 1) {
    Dev<T>& D = *E.devs[0];
    // local duplicates first (e.g. Chimera rank 0 holds the tied wte twice)
    for (auto& kv : copies) {
      std::vector<int> mine;
      for (auto& c : kv.second) if (c.first == me) mine.push_back(c.second);
      for (size_t c = 1; c < mine.size(); ++c)
        add_f32(D.gr + P.rank_params[me].off[mine[0]], D.gr + P.rank_params[me].off[mine[c]],
                P.rank_params[me].cnt[mine[0]], st);
    }
    // then pairwise all-reduce with the other holder, in the comm program's (global) order
    NC(ncclGroupStart());
    for (const mario_commop& op : prog) {
      if (op.kind != 4) continue;
      int j0 = -1;
      for (auto& c : copies[op.a]) if (c.first == me) { j0 = c.second; break; }
      float* buf = D.gr + P.rank_params[me].off[j0];
      NC(ncclAllReduce(buf, buf, static_cast<size_t>(op.count), ncclFloat32, ncclSum,
                       g.pair_comms[{op.b - off, op.c - off}], st));
    }
    NC(ncclGroupEnd());
    for (auto& kv : copies) {
      std::vector<int> mine;
      for (auto& c : kv.second) if (c.first == me) mine.push_back(c.second);
      for (size_t c = 1; c < mine.size(); ++c)
        copy_f32(D.gr + P.rank_params[me].off[mine[c]], D.gr + P.rank_params[me].off[mine[0]],
                 P.rank_params[me].cnt[mine[0]], st);
    }
    // AR (Table 3; reading A29): average the whole gradient buffer over the stage's replicas
    for (const mario_commop& op : prog)
      if (op.kind == 7) NC(ncclAllReduce(D.gr, D.gr, static_cast<size_t>(op.count), ncclFloat32, ncclAvg, g.dp_comm, st));
  }

  }   // !replayed
  if (capturing) {
    cudaGraph_t graph;
    CU(cudaStreamEndCapture(g.cap_stream, &graph));
    g.graph_kernels[gkey] += mario_kernel_launches();
    cudaGraphExec_t exec;
    CU(cudaGraphInstantiate(&exec, graph, 0));
    CU(cudaGraphDestroy(graph));
    g.graph_cache[gkey] = exec;
    CU(cudaGraphLaunch(exec, g.cap_stream));
    E.st = st;
  }
  if (replayed || capturing) {
    cudaEvent_t e1 = E.devs[0]->event();
    CU(cudaEventRecord(e1, g.cap_stream));
    CU(cudaStreamWaitEvent(st, e1, 0));
  }

  // loss (reading A21): per-micro-batch fp64 sums, combined on the host in micro-batch order
  const int K = P.pp.K();
  std::vector<double> sums(P.pp.N, 0.0);
  for (auto& Dp : E.devs) {
    Dev<T>& D = *Dp;
    bool has_last = false;
    for (int p = 0; p < P.pp.parts(); ++p) has_last = has_last || P.pp.vstage(D.d, p) == K - 1;
    if (!has_last) continue;
    std::vector<double> h(static_cast<size_t>(P.pp.N));
    CU(cudaMemcpyAsync(h.data(), D.ws + D.a.loss, P.pp.N * 8, cudaMemcpyDeviceToHost, st));
    CU(cudaStreamSynchronize(st));
    for (int i = 0; i < P.pp.N; ++i) sums[i] += h[i];
  }
  if (!loopback && !peer && g.world > 1) {
    // share the last stage(s)' per-micro-batch sums with every rank (summed over replicas too)
    double* dbuf = reinterpret_cast<double*>(E.devs[0]->ws + E.devs[0]->a.loss);
    CU(cudaMemcpyAsync(dbuf, sums.data(), P.pp.N * 8, cudaMemcpyHostToDevice, st));
    NC(ncclAllReduce(dbuf, dbuf, P.pp.N, ncclFloat64, ncclSum, g.world_comm, st));
    CU(cudaMemcpyAsync(sums.data(), dbuf, P.pp.N * 8, cudaMemcpyDeviceToHost, st));
  }
  CU(cudaStreamSynchronize(st));
  double total = 0.0;
  for (int i = 0; i < P.pp.N; ++i) total += sums[i];
  const double ntok = static_cast<double>(P.pp.N) * tokens_per_micro(m) * (loopback ? 1 : g.dp);
  if (loss) *loss = static_cast<float>(total / ntok);

  // timeline export
  if (g.timing) {
    g.t_start.assign(S, {});
    g.t_finish.assign(S, {});
    cudaEvent_t t0 = t0_peer;   // peer: the fork point every rank's stream starts from
    for (auto& Dp : E.devs) if (!Dp->timed.empty() && !t0) t0 = Dp->timed[0].first;
    for (auto& Dp : E.devs) {
      for (auto& pr : Dp->timed) {
        float a = 0.f, b = 0.f;
        CU(cudaEventElapsedTime(&a, t0, pr.first));
        CU(cudaEventElapsedTime(&b, t0, pr.second));
        g.t_start[Dp->d].push_back(a);
        g.t_finish[Dp->d].push_back(b);
      }
    }
    for (auto& Dp : E.devs)
      for (auto& pr : Dp->timed) { cudaEventDestroy(pr.first); cudaEventDestroy(pr.second); }
    if (t0_peer) cudaEventDestroy(t0_peer);
  }
  for (auto& Dp : E.devs) {
    for (auto v : {&Dp->sa_free, &Dp->sg_free, &Dp->rg_free, &Dp->ck_free, &Dp->ev_pool})
      for (auto e : *v) ev_put(e);
  }
  return MARIO_OK;
}

}  // namespace

void exec_forget_plan(uint64_t serial) {
  for (auto it = g.graph_cache.begin(); it != g.graph_cache.end();) {
    if (std::get<0>(it->first) == serial) { cudaGraphExecDestroy(it->second); it = g.graph_cache.erase(it); }
    else ++it;
  }
  for (auto it = g.graph_kernels.begin(); it != g.graph_kernels.end();)
    it = std::get<0>(it->first) == serial ? g.graph_kernels.erase(it) : std::next(it);
  for (auto it = g.graph_seen.begin(); it != g.graph_seen.end();)
    it = std::get<0>(*it) == serial ? g.graph_seen.erase(it) : std::next(it);
}

}  // namespace mario

using namespace mario;

extern "C" mario_status mario_nccl_unique_id(void* out128) {
  if (!out128) return set_error(MARIO_EINVAL, "NULL out");
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return set_error(MARIO_ENCCL, "ncclGetUniqueId failed");
  static_assert(sizeof(ncclUniqueId) == 128, "nccl id size");
  memcpy(out128, &id, 128);
  return MARIO_OK;
}

extern "C" mario_status mario_init_dp(int32_t rank, int32_t world, int32_t device, int32_t dp,
                                      const void* nccl_unique_id) {
  try {
    if (world < 1 || rank < 0 || rank >= world) return set_error(MARIO_EINVAL, "bad rank/world");
    if (dp < 1 || world % dp) return set_error(MARIO_EINVAL, "world % dp != 0");
    if (g.inited) return set_error(MARIO_ESTATE, "already initialised");
    CU(cudaSetDevice(device));
    g.rank = rank; g.world = world; g.device = device; g.dp = dp;
    if (world > 1) {
      if (!nccl_unique_id) return set_error(MARIO_EINVAL, "NULL nccl id");
      ncclUniqueId id;
      memcpy(&id, nccl_unique_id, 128);
      NC(ncclCommInitRank(&g.world_comm, world, id, rank));
    }
    g.inited = true;
    g.sticky = false;
    return MARIO_OK;
  } catch (const CudaErr& e) {
    return set_error(MARIO_ECUDA, e.what());
  } catch (const NcclErr& e) {
    return set_error(MARIO_ENCCL, e.what());
  }
}

extern "C" mario_status mario_init_emulated(int32_t world, int32_t device, int32_t sms_per_rank) {
  try {
    if (world < 1) return set_error(MARIO_EINVAL, "world < 1");
    if (sms_per_rank < 0) return set_error(MARIO_EINVAL, "sms_per_rank < 0");
    if (g.inited) return set_error(MARIO_ESTATE, "already initialised");
    CU(cudaSetDevice(device));
    CU(cudaFree(nullptr));   // primary context up before any green context retains it
    g.rank = 0; g.world = 1; g.device = device; g.dp = 1;
    g.emu_st.assign(world, nullptr);
    g.emu_rx.assign(world, {nullptr, nullptr});
    g.emu_side.assign(world, nullptr);
    g.emu_sms = 0;
    g.emu_green = false;
    if (sms_per_rank > 0) {
      std::vector<std::vector<cudaStream_t>> ps;
      int got = 0;
      const std::string err = drv::make_partitions(device, world, sms_per_rank, 4, ps, &got);
      if (!err.empty()) {
        drv::destroy_partitions();
        return set_error(MARIO_EINVAL, "SM partitions: " + err);
      }
      for (int r = 0; r < world; ++r) g.emu_st[r] = ps[r][0], g.emu_rx[r] = {ps[r][1], ps[r][2]}, g.emu_side[r] = ps[r][3];
      g.emu_sms = got;
      g.emu_green = true;
    } else {
      for (int r = 0; r < world; ++r) {
        CU(cudaStreamCreateWithFlags(&g.emu_st[r], cudaStreamNonBlocking));
        for (auto& x : g.emu_rx[r]) CU(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
        CU(cudaStreamCreateWithFlags(&g.emu_side[r], cudaStreamNonBlocking));
      }
    }
    g.emulated = true;
    g.inited = true;
    g.sticky = false;
    return MARIO_OK;
  } catch (const CudaErr& e) {
    return set_error(MARIO_ECUDA, e.what());
  }
}

extern "C" int32_t mario_emulated_sms(void) { return g.emulated ? g.emu_sms : -1; }

// ------------------------------------------------------------- multi-process peer transport
namespace {
constexpr size_t kPeerFlagWords = static_cast<size_t>(1) << 20;   // 4 MiB of flags per rank
struct PeerRecord {            // what one rank publishes (mario_peer_export), 256 bytes
  cudaIpcMemHandle_t ws, gr, flags;
  uint64_t ws_off, gr_off, flags_off;
  int32_t rank, world;
  uint8_t pad[256 - 3 * sizeof(cudaIpcMemHandle_t) - 3 * 8 - 8];
};
static_assert(sizeof(PeerRecord) == 256, "peer record size");

// IPC handle of the allocation containing p, and p's offset in it
mario_status ipc_handle(const void* p, cudaIpcMemHandle_t* h, uint64_t* off) {
  using PFN = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
  static PFN range = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPointByVersion("cuMemGetAddressRange", &f, 12000, cudaEnableDefault, &q);
    return reinterpret_cast<PFN>(f);
  }();
  if (!range) return set_error(MARIO_ECUDA, "cuMemGetAddressRange unavailable");
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, reinterpret_cast<CUdeviceptr>(p)) != 0) return set_error(MARIO_EINVAL, "not device memory");
  if (cudaIpcGetMemHandle(h, reinterpret_cast<void*>(base)) != cudaSuccess)
    return set_error(MARIO_ECUDA, "cudaIpcGetMemHandle failed (memory not from cudaMalloc?)");
  *off = reinterpret_cast<uint64_t>(p) - static_cast<uint64_t>(base);
  return MARIO_OK;
}
}  // namespace

extern "C" mario_status mario_init_peer(int32_t rank, int32_t world, int32_t device) {
  try {
    if (world < 1 || rank < 0 || rank >= world) return set_error(MARIO_EINVAL, "bad rank/world");
    if (g.inited) return set_error(MARIO_ESTATE, "already initialised");
    CU(cudaSetDevice(device));
    g.rank = rank; g.world = world; g.device = device; g.dp = 1;
    CU(cudaMalloc(&g.ipc_flags_own, kPeerFlagWords * 4));
    CU(cudaMemset(g.ipc_flags_own, 0, kPeerFlagWords * 4));
    g.ipc_flag_words = kPeerFlagWords;
    CU(cudaStreamCreateWithFlags(&g.ipc_st, cudaStreamNonBlocking));
    for (auto& x : g.ipc_rx) CU(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&g.ipc_side, cudaStreamNonBlocking));
    CU(cudaDeviceSynchronize());
    g.epoch = 0;
    g.ipc = true;
    g.inited = true;
    g.sticky = false;
    return MARIO_OK;
  } catch (const CudaErr& e) {
    return set_error(MARIO_ECUDA, e.what());
  }
}

extern "C" mario_status mario_peer_export(const void* workspace, const void* grads, void* record) {
  if (!g.ipc) return set_error(MARIO_ESTATE, "mario_init_peer not called");
  if (!workspace || !grads || !record) return set_error(MARIO_EINVAL, "NULL argument");
  PeerRecord r{};
  if (mario_status e = ipc_handle(workspace, &r.ws, &r.ws_off)) return e;
  if (mario_status e = ipc_handle(grads, &r.gr, &r.gr_off)) return e;
  if (mario_status e = ipc_handle(g.ipc_flags_own, &r.flags, &r.flags_off)) return e;
  r.rank = g.rank;
  r.world = g.world;
  memcpy(record, &r, sizeof r);
  g.bound_ws = workspace;
  g.bound_gr = grads;
  return MARIO_OK;
}

extern "C" mario_status mario_peer_import(const void* records) {
  if (!g.ipc) return set_error(MARIO_ESTATE, "mario_init_peer not called");
  if (!records || !g.bound_ws) return set_error(MARIO_EINVAL, "export this rank's buffers first");
  for (void* p : g.ipc_opened) cudaIpcCloseMemHandle(p);
  g.ipc_opened.clear();
  g.peers.assign(g.world, {});
  const PeerRecord* rec = static_cast<const PeerRecord*>(records);
  for (int r = 0; r < g.world; ++r) {
    if (rec[r].rank != r || rec[r].world != g.world) return set_error(MARIO_EINVAL, "records out of rank order");
    if (r == g.rank) {
      g.peers[r] = {static_cast<uint8_t*>(const_cast<void*>(g.bound_ws)),
                    static_cast<float*>(const_cast<void*>(g.bound_gr)), g.ipc_flags_own};
      continue;
    }
    void* base[3];
    const cudaIpcMemHandle_t* hs[3] = {&rec[r].ws, &rec[r].gr, &rec[r].flags};
    for (int i = 0; i < 3; ++i) {
      if (cudaIpcOpenMemHandle(&base[i], *hs[i], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
        return set_error(MARIO_ECUDA, "cudaIpcOpenMemHandle failed for rank " + std::to_string(r));
      g.ipc_opened.push_back(base[i]);
    }
    g.peers[r] = {static_cast<uint8_t*>(base[0]) + rec[r].ws_off,
                  reinterpret_cast<float*>(static_cast<uint8_t*>(base[1]) + rec[r].gr_off),
                  reinterpret_cast<uint32_t*>(static_cast<uint8_t*>(base[2]) + rec[r].flags_off)};
  }
  return MARIO_OK;
}

extern "C" mario_status mario_init(int32_t rank, int32_t world, int32_t device, const void* nccl_unique_id) {
  return mario_init_dp(rank, world, device, 1, nccl_unique_id);
}

extern "C" mario_status mario_run_iter(const struct mario_plan* plan, const void* weights, const int32_t* tokens,
                                       float* loss, void* grads, void* workspace, void* stream) {
  if (!g.inited) return set_error(MARIO_ESTATE, "mario_init not called");
  if (g.sticky) return set_error(MARIO_ECUDA, "context has a sticky error; call mario_finalize");
  if (!plan || !weights || !tokens || !grads || !workspace) return set_error(MARIO_EINVAL, "NULL argument");
  try {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    mario_status r = plan->model.dtype == MARIO_BF16
                         ? run_iter_t<__nv_bfloat16>(*plan, weights, tokens, loss, grads, workspace, st)
                         : run_iter_t<float>(*plan, weights, tokens, loss, grads, workspace, st);
    if (r == MARIO_OK) {
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) { g.sticky = true; return set_error(MARIO_ECUDA, cudaGetErrorString(e)); }
    }
    return r;
  } catch (const CudaErr& e) {
    g.sticky = true;
    return set_error(MARIO_ECUDA, e.what());
  } catch (const NcclErr& e) {
    g.sticky = true;
    return set_error(MARIO_ENCCL, e.what());
  } catch (const std::exception& e) {
    return set_error(MARIO_EINVAL, e.what());
  }
}

namespace mario {
void adamw_step(float* p, const float* g, float* m, float* v, size_t n, float lr, float b1, float b2, float eps,
                float wd, int step, cudaStream_t st);
}

extern "C" mario_status mario_adamw_step(void* params, const void* grads, void* m, void* v, uint64_t n, float lr,
                                         float beta1, float beta2, float eps, float weight_decay, int32_t step,
                                         void* stream) {
  if (!params || !grads || !m || !v || step < 1) return set_error(MARIO_EINVAL, "bad argument");
  mario::adamw_step(static_cast<float*>(params), static_cast<const float*>(grads), static_cast<float*>(m),
                    static_cast<float*>(v), static_cast<size_t>(n), lr, beta1, beta2, eps, weight_decay, step,
                    static_cast<cudaStream_t>(stream));
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_error(MARIO_ECUDA, cudaGetErrorString(e));
  return MARIO_OK;
}

extern "C" mario_status mario_set_graphs(int32_t enable) {
  g.graphs = enable != 0;
  if (!g.graphs) {
    for (auto& kv : g.graph_cache) cudaGraphExecDestroy(kv.second);
    g.graph_cache.clear();
    g.graph_seen.clear();
  }
  return MARIO_OK;
}

extern "C" mario_status mario_set_timing(int32_t enable) {
  g.timing = enable != 0;
  return MARIO_OK;
}

extern "C" mario_status mario_last_timeline(int32_t device, const double** start_ms, const double** finish_ms,
                                            int32_t* n) {
  if (device < 0 || device >= static_cast<int32_t>(g.t_start.size()) || !start_ms || !finish_ms || !n)
    return set_error(MARIO_EINVAL, "no timeline for device");
  *start_ms = g.t_start[device].data();
  *finish_ms = g.t_finish[device].data();
  *n = static_cast<int32_t>(g.t_start[device].size());
  return MARIO_OK;
}

// The paper's profiled estimators: per-virtual-stage mean durations of FW/CFW, BW and RC
// in the last timed iteration of `plan` on this rank (every rank's in loopback / emulated mode),
// in the layout mario_costs expects ([K] arrays). A stage with no RC gets its forward time.
extern "C" mario_status mario_last_costs(const struct mario_plan* plan, double* fw_ms, double* bw_ms, double* rc_ms) {
  if (!plan || !fw_ms || !bw_ms || !rc_ms) return set_error(MARIO_EINVAL, "NULL argument");
  const int K = plan->pp.K();
  std::vector<double> sum[3];
  std::vector<int> cnt[3];
  for (int c = 0; c < 3; ++c) { sum[c].assign(K, 0.0); cnt[c].assign(K, 0); }
  bool any = false;
  for (int d = 0; d < plan->pp.S && d < static_cast<int>(g.t_start.size()); ++d) {
    size_t j = 0;
    for (const mario_instr& x : plan->instrs[d]) {
      if (x.op != MARIO_OP_FW && x.op != MARIO_OP_CFW && x.op != MARIO_OP_RC && x.op != MARIO_OP_BW) continue;
      if (j >= g.t_start[d].size()) break;
      const int c = (x.op == MARIO_OP_BW) ? 1 : (x.op == MARIO_OP_RC ? 2 : 0);
      sum[c][x.vstage] += g.t_finish[d][j] - g.t_start[d][j];
      ++cnt[c][x.vstage];
      ++j;
      any = true;
    }
  }
  if (!any) return set_error(MARIO_ESTATE, "no timed iteration of this plan (mario_set_timing(1) first)");
  for (int k = 0; k < K; ++k) {
    fw_ms[k] = cnt[0][k] ? sum[0][k] / cnt[0][k] : 0.0;
    bw_ms[k] = cnt[1][k] ? sum[1][k] / cnt[1][k] : 0.0;
    rc_ms[k] = cnt[2][k] ? sum[2][k] / cnt[2][k] : fw_ms[k];
  }
  return MARIO_OK;
}

extern "C" mario_status mario_finalize(void) {
  for (auto& kv : g.channels) {
    if (kv.second.comm) ncclCommDestroy(kv.second.comm);
    if (kv.second.stream) cudaStreamDestroy(kv.second.stream);
  }
  g.channels.clear();
  for (auto& kv : g.pair_comms) if (kv.second) ncclCommDestroy(kv.second);
  g.pair_comms.clear();
  g.created_channels.clear();
  g.created_pairs.clear();
  for (auto& kv : g.graph_cache) cudaGraphExecDestroy(kv.second);
  g.graph_cache.clear();
  g.graph_seen.clear();
  {
    std::lock_guard<std::mutex> lk(g_ev_mu);
    int cur = 0;
    cudaGetDevice(&cur);
    for (auto& kv : g_ev_cache) {
      cudaSetDevice(kv.first);
      for (auto e : kv.second) cudaEventDestroy(e);
    }
    g_ev_cache.clear();
    cudaSetDevice(cur);
  }
  if (g.emulated) {
    cudaDeviceSynchronize();
    for (size_t r = 0; r < g.emu_st.size(); ++r) {
      cudaStreamDestroy(g.emu_st[r]);
      for (auto x : g.emu_rx[r]) cudaStreamDestroy(x);
      if (r < g.emu_side.size()) cudaStreamDestroy(g.emu_side[r]);
    }
    g.emu_st.clear();
    g.emu_rx.clear();
    g.emu_side.clear();
    if (g.emu_green) drv::destroy_partitions();
    g.emu_green = false;
    g.emulated = false;
    g.emu_sms = 0;
  }
  if (g.flags) cudaFree(g.flags);
  g.flags = nullptr;
  g.flags_cap = 0;
  if (g.side_st) cudaStreamDestroy(g.side_st);
  g.side_st = nullptr;
  if (g.ipc) {
    cudaDeviceSynchronize();
    for (void* p : g.ipc_opened) cudaIpcCloseMemHandle(p);
    g.ipc_opened.clear();
    g.peers.clear();
    if (g.ipc_flags_own) cudaFree(g.ipc_flags_own);
    g.ipc_flags_own = nullptr;
    if (g.ipc_st) cudaStreamDestroy(g.ipc_st);
    for (auto& x : g.ipc_rx) { if (x) cudaStreamDestroy(x); x = nullptr; }
    if (g.ipc_side) cudaStreamDestroy(g.ipc_side);
    g.ipc_st = nullptr;
    g.ipc_side = nullptr;
    g.ipc = false;
    g.bound_ws = g.bound_gr = nullptr;
    g.world = 1;
  }
  if (g.dp_comm) ncclCommDestroy(g.dp_comm);
  g.dp_comm = nullptr;
  if (g.world_comm) ncclCommDestroy(g.world_comm);
  g.world_comm = nullptr;
  g.dp = 1;
  g.inited = false;
  g.sticky = false;
  return MARIO_OK;
}
