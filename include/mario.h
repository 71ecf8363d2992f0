/* mario.h — C-ABI of libmario.so: a B200-native Mario-scheduled pipeline iteration.
 *
 * The library follows the paper's statement of the problem (Listing 1):
 *   schedule = mario.optimize(mario_conf, model_conf, global_bs);  mario.run(schedule)
 * as north_star fixes it:  mario_plan(model, stages, microbatches, scheme, mem_budget)
 * returns per-device instruction lists (IR: Table 3) produced by the four graph
 * passes (§5.1) and checked by the simulator (§5.2);
 * mario_run_iter(plan, weights, batch) executes one rank's list and returns loss and grads.
 *
 * Conventions
 *  - Every call returns mario_status (0 = OK, < 0 = error); no C++ exception crosses the
 *    ABI. mario_last_error() gives a thread-local message valid until the next call.
 *  - Ownership: plans are owned by the library (opaque, immutable, safe to read from
 *    several threads) and freed by mario_plan_destroy. Weights, grads, tokens, loss and
 *    workspace are owned by the caller; the library never frees caller memory.
 *  - Sizes are in elements unless named *_bytes.
 */
#ifndef MARIO_H
#define MARIO_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  MARIO_OK = 0,
  MARIO_EINVAL = -1,     /* bad argument, unsupported shape, NULL pointer            */
  MARIO_EBUDGET = -2,    /* simulated peak memory > mem_budget ("F = 0 if OOM") */
  MARIO_EDEADLOCK = -3,  /* the instruction graph has a cycle                         */
  MARIO_ECUDA = -4,      /* CUDA error (sticky: finalize the context)                 */
  MARIO_ENCCL = -5,      /* NCCL error (sticky)                                       */
  MARIO_ESTATE = -6      /* wrong call order / plan and context disagree              */
} mario_status;

typedef enum { MARIO_GPT = 0, MARIO_LLAMA = 1 } mario_family;
/* Pipeline schemes: "V" 1F1B, "W" Interleave, "X" Chimera. */
typedef enum { MARIO_1F1B = 0, MARIO_INTERLEAVE = 1, MARIO_CHIMERA = 2 } mario_scheme;
/* Evaluation configurations: base, ckpt (pass 1 only), ovlp (= passes 1-4). */
/* MARIO_LEVEL_BUDGET (extension, DESIGN reading A28): passes 1-4 on devices
 * 0 .. S-k-1 while the tail devices S-k .. S-1 keep their full activations in base order; k is the
 * feasible choice (every device's simulated peak <= mem_budget) with the smallest simulated
 * makespan, ties to the smaller k. Needs mem_budget_bytes > 0. */
typedef enum { MARIO_LEVEL_BASE = 0, MARIO_LEVEL_CKPT = 1, MARIO_LEVEL_MARIO = 2, MARIO_LEVEL_BUDGET = 3 } mario_level;
typedef enum { MARIO_F32 = 0, MARIO_BF16 = 1 } mario_dtype;
/* Instruction types (Table 3). */
typedef enum {
  MARIO_OP_FW = 0, MARIO_OP_CFW = 1, MARIO_OP_RC = 2, MARIO_OP_BW = 3,
  MARIO_OP_SA = 4, MARIO_OP_RA = 5, MARIO_OP_SG = 6, MARIO_OP_RG = 7
} mario_op;

/* model_conf (Table 4; details per DESIGN.md readings A1/A2). */
typedef struct {
  int32_t family;          /* mario_family                                   */
  int32_t n_layers, hidden, n_heads, ffn_hidden, vocab, seq_len;
  int32_t micro_batch;     /* samples per micro-batch (mbs)                  */
  int32_t tie_embeddings;  /* GPT: LM head tied to wte                       */
  int32_t dtype;           /* mario_dtype: compute/storage precision         */
  float norm_eps, rope_base;
} mario_model;

/* One IR record (micro_id m, part_id p). vstage = virtual stage;
 * peer = device of the matching SA/RA or SG/RG (-1 otherwise); slot = stage-input
 * (checkpoint) slot on this device; aslot = activation-set slot (-1 for CFW). */
typedef struct { int32_t op, micro, part, vstage, peer, slot, aslot; } mario_instr;

/* Optional cost table for the simulator (the paper's profiled estimators).
 * Arrays are indexed by virtual stage [0, K); NULL arrays fall back to analytic costs
 * (FLOPs / 1e15 FLOP/s, comm = alpha + bytes / GBps). act/ckpt/work override the
 * per-virtual-stage dynamic memory model (bytes). */
typedef struct {
  const double *fw_ms, *bw_ms, *rc_ms;
  double p2p_alpha_ms, p2p_GBps;         /* <= 0 GBps: bytes ignored */
  const double *act_bytes, *ckpt_bytes, *work_bytes;
  double static_bytes;                   /* < 0: use the analytic static model */
} mario_costs;

typedef struct {
  double makespan_ms, bubble_ratio;
  int32_t n_dev;
  const double* busy_ms;        /* [n_dev]                          */
  const uint64_t* peak_bytes;   /* [n_dev] static + peak dynamic    */
  const int32_t* max_live_act;  /* [n_dev] live activation sets      */
  const int32_t* max_live_ckpt; /* [n_dev] live stage-input checkpoints */
} mario_sim;

/* One communication operation of a rank's NCCL program, in issue order (see
 * mario_plan_comm_ops). kind: 0 = split a 2-rank channel communicator (a = src, b = dst,
 * c = 0 activation / 1 gradient; collective over ALL ranks), 1 = split a replica-pair
 * communicator (a < b), 2 = send on channel (a -> b, c) the message of (micro, part = sender
 * part), issued right after list instruction list_index, 3 = receive on channel (a -> b, c) at
 * list instruction list_index (part = receiver part), 4 = all-reduce of parameter a (count
 * floats) on pair (b, c), 5 = all-reduce of count fp64 loss partials on the world,
 * 6 = split the data-parallel communicator of stage a (b = replica, c = dp; collective over ALL
 * ranks), 7 = average the rank's whole fp32 gradient buffer (count floats) over that
 * communicator (the AR phase of Table 3; reading A29). Kinds 6/7 appear only for dp > 1. */
typedef struct { int32_t kind, a, b, c, micro, part, list_index; int64_t count; } mario_commop;

struct mario_plan;

/* Build a plan: partition (even layers, embedding on virtual stage 0, final norm + head on
 * the last, reading A8), expand the scheme into per-device lists, apply the passes
 * for `level`, simulate. chunks = Interleave v (1 otherwise).
 * Errors: EINVAL (L % (S*v) != 0, h % heads != 0, head_dim not in {16,32,64,80,128},
 * Interleave with N % S != 0, Chimera with odd S or N % S != 0, NULL out);
 * EBUDGET if the simulated per-device peak exceeds mem_budget_bytes (0 = no budget). */
mario_status mario_plan(const mario_model* model, int32_t stages, int32_t microbatches,
                        int32_t scheme, int32_t chunks, uint64_t mem_budget_bytes, int32_t level,
                        const mario_costs* costs, struct mario_plan** out);
/* Borrowed view of device `device`'s ordered list, valid until mario_plan_destroy. */
mario_status mario_plan_instrs(const struct mario_plan* plan, int32_t device,
                               const mario_instr** instrs, int32_t* n);
/* Simulator results (borrowed arrays, valid until destroy). */
mario_status mario_plan_simulate(const struct mario_plan* plan, mario_sim* out);
/* Simulated start/finish (ms) of every compute instruction of `device`, in list order of its
 * compute instructions; arrays of length *n owned by the plan. */
mario_status mario_plan_timeline(const struct mario_plan* plan, int32_t device,
                                 const double** start_ms, const double** finish_ms, int32_t* n);
/* The ordered communication program of `rank` under world = stages (multi-process mode).
 * Sends on each channel are issued in the receiver's receive order (sends are buffered, so
 * this adds no dependency) — required because pass 4 may move an SA ahead of an earlier
 * micro-batch's SA while NCCL channels are FIFO. Array owned by the plan. */
mario_status mario_plan_comm_ops(const struct mario_plan* plan, int32_t rank, const mario_commop** ops, int32_t* n);
/* PP x DP (reading A29): the program of world rank `rank` when world =
 * stages * dp and rank = replica * stages + stage. Same as mario_plan_comm_ops(rank % stages) with
 * every rank field offset into the replica's range, preceded by a kind-6 split and with a kind-7
 * gradient average before the loss all-reduce. EINVAL unless 0 <= rank < stages * dp. */
mario_status mario_plan_comm_ops_dp(const struct mario_plan* plan, int32_t dp, int32_t rank, const mario_commop** ops,
                                    int32_t* n);
/* Canonical text serialization (deterministic). If buf is NULL or cap too small, *needed
 * receives the size including the terminating NUL and MARIO_EINVAL is returned for cap>0. */
mario_status mario_plan_serialize(const struct mario_plan* plan, char* buf, size_t cap, size_t* needed);
/* Byte sizes of rank `rank`'s packed fp32 parameters (= grads) and required workspace.
 * rank -1: loopback totals (all ranks concatenated); -2: emulated peer-transport totals. */
mario_status mario_plan_rank_layout(const struct mario_plan* plan, int32_t rank, uint64_t* param_count,
                                    uint64_t* workspace_bytes);
/* Packed parameter layout of `rank`: for each tensor j, its global name index (see
 * mario_param_name), element offset and element count. Arrays owned by the plan. */
mario_status mario_plan_rank_params(const struct mario_plan* plan, int32_t rank, const int32_t** name_idx,
                                    const uint64_t** offset, const uint64_t** count, int32_t* n);
/* Name of the global parameter `idx` (canonical order), e.g. "h3.qkv.w". */
const char* mario_param_name(const struct mario_plan* plan, int32_t idx);
int32_t mario_param_count(const struct mario_plan* plan);
/* Shape of global parameter `idx`: *ndim (1 or 2) dims written to dims[4] (row-major, e.g.
 * qkv.w = [3h, h]). EINVAL on a bad index or NULL pointers. */
mario_status mario_param_shape(const struct mario_plan* plan, int32_t idx, int64_t* dims, int32_t* ndim);
/* k of MARIO_LEVEL_BUDGET (0 for the other levels); -1 on NULL. */
int32_t mario_plan_unckpt_tail(const struct mario_plan* plan);
/* 1 if the plan's activation sets keep the layers' norm outputs and MLP activation (the backward
 * reads them instead of recomputing them; chosen unless it would exceed mem_budget_bytes, where the
 * lean set is planned instead; env MARIO_STORE_ACT=0/1 forces either), 0 for the lean set, -1 on NULL. */
int32_t mario_plan_store_act(const struct mario_plan* plan);
void mario_plan_destroy(struct mario_plan* plan);

/* Schedule tuner (§5.3, Eq. 1): grid search
 *   max F(b, E(a, b, pp, mbs), dmem, dp)  over  a in {no ckpt (BASE), Mario (passes 1-4)},
 *   b in {1F1B, Interleave (v = 2), Chimera}, pp in [min(4, D), D] with dp * pp = D,
 *   mbs in {1, 2, 4, 8, ...} with global_batch = dp * mbs * N,
 * where F = global_batch / simulated makespan, times dp_efficiency if dp > 1, and F = 0 when the
 * simulated per-device peak exceeds mem_budget_bytes. Per-layer costs per micro-batch
 * size (the profiled estimators E) may be supplied; NULL arrays = analytic (FLOPs at
 * 1 PFLOP/s, linear in mbs). Writes up to cap results (every evaluated configuration) and the
 * index of the best one (-1 if none is feasible). The "Auto" scheme of P:167 is the best row. */
typedef struct {
  int32_t n_mbs;              /* number of micro-batch sizes in mbs[] (0 = {1,2,4,8})        */
  const int32_t* mbs;
  const double *layer_fw_ms, *layer_bw_ms, *head_fw_ms, *head_bw_ms;   /* [n_mbs] or NULL */
  double p2p_alpha_ms, p2p_GBps, dp_efficiency;
} mario_tune_costs;
typedef struct {
  int32_t scheme, pp, chunks, dp, micro_batch, microbatches, level, feasible;
  double makespan_ms, samples_per_s, bubble_ratio;
  uint64_t peak_bytes;
} mario_tune_result;
mario_status mario_tune(const mario_model* model, int32_t devices, int32_t global_batch, uint64_t mem_budget_bytes,
                        const mario_tune_costs* costs, mario_tune_result* results, int32_t cap, int32_t* n,
                        int32_t* best);

/* Executor context. world == 1 with a multi-stage plan runs every rank's list in this
 * process on one GPU ("loopback": device-to-device copies instead of NCCL). world > 1:
 * one process per GPU, nccl_unique_id = 128 bytes from mario_nccl_unique_id() on rank 0. */
mario_status mario_nccl_unique_id(void* out128);
mario_status mario_init(int32_t rank, int32_t world, int32_t device, const void* nccl_unique_id);
/* PP x DP: world = stages * dp processes, rank = replica * stages + stage; every replica runs the
 * same plan on its own micro-batches, gradients are averaged over the replicas of each stage
 * (ncclAvg) after the pipeline flush and the loss is the mean over all replicas' tokens.
 * mario_init(...) == mario_init_dp(..., dp = 1, ...). EINVAL if world % dp != 0. */
mario_status mario_init_dp(int32_t rank, int32_t world, int32_t device, int32_t dp, const void* nccl_unique_id);
/* Emulated pipeline over the PEER TRANSPORT: `world` pipeline ranks hosted by this process on one
 * GPU, each with its own compute and receive streams; with sms_per_rank > 0 every rank's streams
 * live in a green context owning a disjoint partition of that many SMs (the driver rounds to
 * its granularity: multiples of 8 on sm_100), so the S stages run concurrently the way S GPUs do.
 * The executor then follows the per-rank code path of the multi-process executor: each rank walks
 * its own list; RA/RG are blocking receives implemented as a device-side wait on the
 * sender's "ready" flag, a copy out of the sender's send slot and a "consumed" flag; SA/SG are
 * buffered sends that raise the "ready" flag; a send slot is reused only after the
 * receiver's "consumed" flag; tied-embedding / Chimera replica copies are summed by a
 * reduce-scatter + all-gather over peer memory (reading A7). Buffers: mario_plan_rank_layout(-2)
 * (all ranks' packed parameters / multi-process workspaces concatenated). Results are bitwise
 * identical to loopback. EINVAL if the partitions do not fit or green contexts are unavailable;
 * ESTATE if a context is already initialised. mario_run_iter then requires plan stages == world.
 * mario_emulated_sms: SMs per rank partition (0 = unpartitioned), -1 if not emulated. */
mario_status mario_init_emulated(int32_t world, int32_t device, int32_t sms_per_rank);
int32_t mario_emulated_sms(void);
/* Multi-process PEER TRANSPORT (CUDA IPC): one process per pipeline rank, on one GPU or on GPUs
 * with peer access; the same per-rank executor path and flags as mario_init_emulated, with every
 * other rank's workspace, grads and rank 0's flag block mapped through CUDA IPC. Flags carry the
 * iteration number (each rank must call mario_run_iter the same number of times); an
 * end-of-iteration barrier keeps a rank from overwriting memory another rank still reads.
 *  mario_init_peer(rank, world, device)                     ESTATE if already initialised
 *  mario_peer_export(workspace, grads, record)              record: 256 bytes out (IPC handles +
 *                     offsets of this rank's caller-owned workspace / grads and its flag block);
 *                     the buffers must come from cudaMalloc (any offset inside an allocation)
 *  mario_peer_import(records)                               records: world x 256 bytes, rank order,
 *                     gathered by the caller over any out-of-band channel
 * mario_run_iter then requires exactly the exported workspace and grads (ESTATE otherwise) and
 * plan stages == world. Tensors on a rank stay rank-local: weights/grads/workspace as
 * mario_plan_rank_layout(rank). */
mario_status mario_init_peer(int32_t rank, int32_t world, int32_t device);
mario_status mario_peer_export(const void* workspace, const void* grads, void* record);
mario_status mario_peer_import(const void* records);
/* One training iteration of `plan` on this rank (all ranks in loopback).
 *  weights : device, this rank's packed fp32 parameters (loopback: all ranks concatenated)
 *  tokens  : HOST int32 [N*mbs][s+1]; x = tokens[:, :s], y = tokens[:, 1:] (reading A4)
 *  loss    : host, receives the global-batch mean loss (identical on all ranks)
 *  grads   : device fp32, same layout as weights, OVERWRITTEN (not accumulated) with
 *            dloss/dtheta; Chimera replicas and tied embeddings are summed (reading A7)
 *  workspace: device, >= workspace_bytes of mario_plan_rank_layout (loopback: sum)
 *  stream  : caller's cudaStream_t; the call synchronizes it before returning. */
mario_status mario_run_iter(const struct mario_plan* plan, const void* weights, const int32_t* tokens,
                            float* loss, void* grads, void* workspace, void* stream);
/* Replay single-process iterations (world = 1: S = 1 or loopback) from a CUDA graph captured on
 * the second call with the same (plan, weights, grads, workspace) pointers; the graph is reused
 * while those pointers are unchanged (weights may change in place, e.g. by mario_adamw_step).
 * Disabled automatically while timing or kernel statistics are enabled. 0 disables and frees. */
mario_status mario_set_graphs(int32_t enable);
/* Per-instruction measured timeline of the last mario_run_iter on this rank (ms from the
 * iteration start, CUDA events) when timing was enabled with mario_set_timing(1). */
mario_status mario_set_timing(int32_t enable);
mario_status mario_last_timeline(int32_t device, const double** start_ms, const double** finish_ms, int32_t* n);
/* The paper's profile step: per-virtual-stage mean FW/CFW, BW and RC durations (ms) of the
 * last timed mario_run_iter of `plan` (timing on), written to three caller arrays of K = stages x
 * chunks entries -- the mario_costs arrays, so mario_plan can re-plan and simulate with measured costs.
 * A stage without RC reports its forward time. ESTATE if no timed iteration is recorded. */
mario_status mario_last_costs(const struct mario_plan* plan, double* fw_ms, double* bw_ms, double* rc_ms);
/* OS (Table 3): AdamW (reading A27: decoupled weight decay, bias correction; step >= 1)
 * applied in place to n packed fp32 parameters with fp32 moments m, v (device pointers, caller
 * owned, zero-initialised before step 1); grads as returned by mario_run_iter. Asynchronous on
 * `stream`. EINVAL on NULL pointers or step < 1. */
mario_status mario_adamw_step(void* params, const void* grads, void* m, void* v, uint64_t n, float lr, float beta1,
                              float beta2, float eps, float weight_decay, int32_t step, void* stream);
mario_status mario_finalize(void);
const char* mario_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
