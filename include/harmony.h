/*
 * harmony.h — C ABI of the B200-native Harmony-DP training step.
 *
 * Method: Li, Phanishayee, Murray, Kim, "Doing more with less: Training large
 * DNN models on commodity servers for the masses", HotOS '21.
 * Citations "P:a-b" are PAPER.md lines.  The interface follows the paper's
 * problem statement: the user targets "a single virtual accelerator device with
 * practically unbounded memory", supplies a model "as if running
 * sequentially on a single device", a parallelization scheme,
 * the hardware configuration and a mini-batch size.
 * Behind these calls the library decomposes the step into per-layer x
 * per-microbatch forward / backward / update tasks,
 * late-binds them to streams and HBM slots under a per-GPU memory cap, swaps
 * state and activations to pinned host RAM, groups
 * microbatches, runs each layer's update just in time,
 * and inserts collectives to keep the result that of the plain single-device
 * step.
 *
 * Process models (both run the same planner and executor):
 *  - ONE process per GPU (harmony_init; rank r of world_size).  Every rank calls
 *    the same functions in the same order; collectives (NCCL, loaded with dlopen)
 *    run inside harmony_step / harmony_read_state.
 *  - ONE process, N ranks: "a single virtual accelerator device" (
 *    harmony_init_group).  The caller holds one context and passes the global
 *    batch; the library drives the N rank programs itself and runs the collectives
 *    (reduce-scatter of dW, all-gather of weight shards and loss partials) as its own
 *    pulls from the peers' HBM — over NVLink between GPUs, or inside one GPU when
 *    ranks share it (a loopback that runs the N > 1 data path on a single B200).
 *
 * Conventions for every call:
 *  - Status codes only; no exception or abort crosses the ABI.  On failure
 *    harmony_last_error(ctx) returns a NUL-terminated message.  A CUDA or NCCL
 *    error is sticky: afterwards only harmony_finalize is valid.
 *  - Pointer arguments are caller-owned and only read/written during the call
 *    (the library copies what it keeps into its own pinned host store).
 *  - Buffers may be HOST or DEVICE pointers wherever "host or device" is said;
 *    the library detects which with cudaPointerGetAttributes.
 *  - A context is not thread-safe.
 *  - Row-major everywhere.  Linear weights are W[d_in][d_out], Y = X.W + b.
 *
 * Parameter packing (per layer, fp32, canonical order):
 *  HARMONY_LAYER_MLP:          W[d_in][d_out], b[d_out]
 *  HARMONY_LAYER_TRANSFORMER:  ln1_g[d], ln1_b[d], W_qkv[d][3d], b_qkv[3d],
 *     W_o[d][d], b_o[d], ln2_g[d], ln2_b[d], W_fc1[d][4d], b_fc1[4d],
 *     W_fc2[4d][d], b_fc2[d]            (12 d^2 + 13 d floats; QKV columns are
 *     [Q | K | V], head h owning columns h*dh .. h*dh+dh-1 of each third).
 *  The transformer layer is a pre-LN block (reading c1):
 *     U=LN1(X); QKV=U W_qkv+b_qkv; C=MHA(QKV) (causal optional);
 *     X2=X+C W_o+b_o; U2=LN2(X2); H=U2 W_fc1+b_fc1; Y=X2+GeLU_tanh(H) W_fc2+b_fc2.
 *  Loss (reading c2): L = (1/B) sum_b 1/2 ||Y_b - T_b||^2 over the GLOBAL batch B.
 *  Optimizer (reading c3): Adam [30] with bias correction, t from 1.
 */
#ifndef HARMONY_H_
#define HARMONY_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HARMONY_ABI_VERSION 1

typedef struct harmony_ctx harmony_ctx; /* opaque; owns all device and pinned memory */

typedef enum {
  HARMONY_OK = 0,
  HARMONY_E_INVALID_ARG = 1,   /* bad sizes, NULL where required, batch != m*b          */
  HARMONY_E_BAD_STATE = 2,     /* calls out of order (e.g. step before register_layers)  */
  HARMONY_E_CAP_TOO_SMALL = 3, /* minimum working set exceeds hbm_cap_bytes               */
  HARMONY_E_HOST_OOM = 4,      /* pinned host allocation failed                           */
  HARMONY_E_CUDA = 5,          /* CUDA runtime / driver error (sticky)                    */
  HARMONY_E_NCCL = 6,          /* NCCL missing or failed (sticky)                         */
  HARMONY_E_UNSUPPORTED = 7    /* valid request the build does not support (e.g. d%8!=0 on bf16) */
} harmony_status;

typedef enum { HARMONY_FP32 = 0, HARMONY_BF16_FP32MASTER = 1 } harmony_precision;
typedef enum { HARMONY_LAYER_MLP = 0, HARMONY_LAYER_TRANSFORMER = 1 } harmony_layer_kind;
typedef enum { HARMONY_ACT_NONE = 0, HARMONY_ACT_RELU = 1, HARMONY_ACT_GELU_TANH = 2 } harmony_act;
typedef enum { HARMONY_PARAM = 0, HARMONY_GRAD = 1, HARMONY_ADAM_M = 2, HARMONY_ADAM_V = 3 } harmony_state_kind;

/* Schedules.  HARMONY_SCHED_HARMONY_DP is the paper's Harmony-DP (input-batch
 * grouping P:537-548 + JIT update P:549-553 + p2p weight shards P:738-748).
 * HARMONY_SCHED_PER_GPU_VIRT is the baseline the paper compares against
 * (per-GPU memory virtualization, Fig. 5(b)): each microbatch swaps
 * the weights in and out for its own forward and backward, and the update runs
 * after the whole backward.  Both compute the identical result. */
typedef enum { HARMONY_SCHED_HARMONY_DP = 0, HARMONY_SCHED_PER_GPU_VIRT = 1, HARMONY_SCHED_HARMONY_PP = 2 } harmony_schedule;
/* HARMONY_SCHED_HARMONY_PP (groups only, num_ranks >= 2, layers >= ranks): the paper's virtualized
 * pipeline (Fig. 4; DESIGN reading c27).  Layer l runs on rank
 * l % num_ranks; every layer-level task runs its group of m microbatches back to back (input-batch
 * grouping); activations and gradients go to the next / previous layer's rank peer to peer; each
 * layer's weights are swapped in once for its forward group, once for its backward group and out
 * once after its just-in-time update — 3|W| per iteration for the whole box.  The batch is ONE
 * minibatch of m*b samples (not num_ranks*m*b); the result is bit-identical to the single-rank
 * Harmony-DP step with the same m and b (same kernels, same accumulation order). */

typedef struct {
  uint32_t struct_size;      /* = sizeof(harmony_config) (ABI versioning)                   */
  int32_t rank;              /* this process's rank in the data-parallel group, 0..world-1   */
  int32_t world_size;        /* N GPUs (one process each); 1 = no collectives                */
  int32_t device;            /* CUDA device ordinal used by this process                     */
  uint64_t hbm_cap_bytes;    /* per-GPU arena budget in bytes; 0 = uncapped (all resident)   */
  void* arena;               /* optional caller-owned DEVICE buffer of hbm_cap_bytes (e.g. a
                                torch tensor); NULL = the library allocates the arena itself */
  int32_t microbatches;      /* m microbatches per rank per step (the input-batch group)     */
  int32_t microbatch_size;   /* b samples per microbatch; local batch = m*b, global = N*m*b  */
  int32_t precision;         /* harmony_precision                                            */
  int32_t schedule;          /* harmony_schedule                                             */
  int32_t retain_grads;      /* 1 = keep the last reduced gradients readable (HARMONY_GRAD)  */
  int32_t stash_policy;      /* 0 = stash every op input (36d+2hS+16 B/token/block);
                                1 = recompute elementwise outputs (LN outputs, GeLU) in the
                                backward (24d+2hS+16 B/token/block);
                                2 = block recompute: stash only the fp32 block
                                input (4d B/token/block), the backward re-runs the block's
                                forward first (4/3 of the GEMM FLOPs, far fewer swap bytes);
                                3 = as 2, plus the fused attention's output C (bf16) and row
                                log-sum-exp (6d+4h B/token/block): the recompute skips the
                                attention forward (falls back to 2 when attention is unfused).
                                All four give bit-identical results (reading c13).           */
  double lr, beta1, beta2, eps, weight_decay; /* Adam; weight_decay must be 0 (reading c3).  Doubles:
                                the kernel uses fp32 b and (1-b) each rounded once from these */
  uint8_t nccl_id[128];      /* ncclUniqueId from harmony_get_unique_id() on rank 0, broadcast
                                to all ranks by the caller (ignored when world_size == 1)    */
  int32_t groups;            /* G microbatch groups (0 or 1 = one group; m % G == 0; Harmony-DP):
                                group 0's forward, then each group's backward interleaved layer by
                                layer with the next group's forward, so stash swap-ins and spills
                                use both directions of the host link (SURVEY §8(d) direction
                                balance).  Every layer's fp32 dW stays in HBM across the groups.
                                The microbatches keep their canonical order in every accumulation:
                                results are bit-identical for every G (reading c21).             */
  int32_t fwd_pack;          /* forward pack size ("pack size per pass", P:749-757,
                                783-801): 0 or 1 = one forward task per microbatch; 2 = the forward
                                pass runs each layer on two consecutive microbatches at once (GEMMs
                                of 2*b*S rows), while the backward stays per microbatch (its working
                                set is the larger one).  Harmony-DP, block recompute (stash_policy
                                2), transformer layers of one width, m % (2*G) == 0; anything else
                                is HARMONY_E_UNSUPPORTED.  Every per-row and per-element result is
                                computed in the same order, so the step is bit-identical.        */
} harmony_config;

typedef struct {
  int32_t kind;      /* harmony_layer_kind                                            */
  int32_t d_in;      /* input width (transformer: d)                                  */
  int32_t d_out;     /* output width (transformer: must equal d_in)                   */
  int32_t n_heads;   /* transformer heads h (d % h == 0)                              */
  int32_t seq_len;   /* transformer sequence length S (MLP: 1)                        */
  int32_t causal;    /* transformer: 1 = causal mask                                  */
  int32_t act;       /* MLP activation (harmony_act)                                  */
} harmony_layer_desc;

/* Per-step statistics of THIS rank (the copy ledger).  Bytes are what
 * was actually issued to the copy engines / NCCL during the last step. */
typedef struct {
  uint64_t h2d_bytes, d2h_bytes;               /* all host<->device copies            */
  uint64_t h2d_weight_bytes, d2h_weight_bytes; /* compute-copy weights W (Fig. 5)     */
  uint64_t h2d_state_bytes, d2h_state_bytes;   /* fp32 master W, Adam m, v (K) */
  uint64_t h2d_stash_bytes, d2h_stash_bytes;   /* stashed activations    */
  uint64_t h2d_input_bytes, d2h_output_bytes;  /* X, T in; loss out                   */
  uint64_t h2d_grad_bytes, d2h_grad_bytes;     /* dW crossing PCIe (Harmony-DP: 0)     */
  uint64_t nvlink_bytes;                        /* bytes this rank sent through NCCL   */
  uint64_t peak_arena_bytes;                    /* arena bytes the plan uses           */
  uint64_t kernel_launches;                     /* kernels launched in the step        */
  uint64_t n_ops;                               /* ops in the static program           */
  double step_seconds;                          /* device time of the step (CUDA events)*/
  uint64_t graph;                               /* 1 = the step replayed its captured CUDA graph
                                                   (pinned/device inputs, profiling off; disable
                                                   with HARMONY_NO_GRAPH=1)                  */
} harmony_step_stats;

/* Static plan summary (host-only; also available without a GPU via harmony_plan_dry). */
typedef struct {
  uint64_t arena_bytes;            /* bytes of arena the plan lays out                   */
  uint64_t min_working_set_bytes;  /* smallest cap this model/batch can run under        */
  uint64_t resident_weight_bytes, total_weight_bytes;  /* compute copies                 */
  uint64_t resident_state_bytes, total_state_bytes;    /* master+m+v shards of this rank */
  uint64_t resident_stash_bytes, total_stash_bytes;    /* per step                       */
  uint64_t pred_h2d_bytes, pred_d2h_bytes;             /* per step, this rank            */
  uint64_t pred_h2d_weight_bytes, pred_d2h_weight_bytes;
  uint64_t flops_per_step;         /* algorithmic GEMM FLOPs of this rank's step         */
  int64_t n_params;                /* model parameters                                   */
  int32_t n_ops, n_compute_ops, n_copy_ops, n_comm_ops;
  int32_t weight_slots, stash_slots, state_slots;
  int32_t hazards;                 /* conflicting accesses the independent byte-range validator
                                      found in the program (must be 0; register refuses otherwise) */
} harmony_plan_summary;

/* sizeof of the ABI structs as the library was compiled: harmony_config, harmony_layer_desc,
 * harmony_step_stats, harmony_plan_summary, hk_gemm_args, harmony_kernel_profile (bindings
 * check their mirrors). */
void harmony_abi_sizes(uint64_t out[6]);

/* Per-kernel-class timing (CUDA events recorded on the launching stream around every launch
 * while profiling is on).  Classes: 0 GEMM (work = algorithmic FLOPs 2MNK), 1 Adam (work =
 * algorithmic HBM bytes, 30 B/param bf16 / 32 fp32), 2 LayerNorm fwd+bwd (bytes), 3 softmax
 * fwd+bwd (bytes), 4 other, 5 fused attention fwd/bwd (work = algorithmic FLOPs of its QK^T, PV
 * (and backward) contractions).  Totals accumulate over steps since harmony_set_profiling(ctx, 1). */
typedef struct {
  uint64_t launches[6];
  double seconds[6];
  double work[6];
  double busy_seconds[6];  /* union of the class's launch intervals on all streams: launches of one
                              class that overlap (e.g. a dgrad GEMM on the compute stream beside a
                              wgrad GEMM on the side stream) count once, so work / busy_seconds is the
                              class's throughput while it runs, not each launch's stretched share */
} harmony_kernel_profile;

/* The step timeline of the last profiled step (profiling on): one record per op of the static
 * program, in issue order — kind (OP_INPUT 0, H2D 1, D2H 2, FWD 3, LOSS 4, BWD 5, UPD 6,
 * ALLGATHER 7, REDUCESCATTER 8, LOSS_GATHER 9, LOSS_OUT 10), stream (0 compute, 1 h2d, 2 d2h,
 * 3 comm), tensor class of a copy (0 weight, 1 state, 2 stash, 3 input, 4 output, 5 grad, 6 none),
 * layer, microbatch, bytes moved, and [t0, t1] in seconds from the step's start: CUDA events
 * recorded on the op's stream around it (after its cross-stream waits), so the span is the op's
 * own time on its stream.  The evidence for swap/compute overlap and achieved host-link GB/s.
 * Writes min(n, cap) records to out (nullable) and the count to *n_out. */
typedef struct {
  int32_t op, kind, stream, cat, layer, micro;
  uint64_t bytes;
  double t0, t1;
} harmony_timeline_rec;
harmony_status harmony_read_timeline(const harmony_ctx* ctx, harmony_timeline_rec* out, int32_t cap, int32_t* n_out);

/* The kernel launches of the last profiled step: class (as harmony_kernel_profile), stream (0-3 as
 * above, 4 = the weight-gradient side stream, -1 other), algorithmic work, [t0, t1] seconds from the
 * step's start (events on the launching stream around the launch). */
typedef struct {
  int32_t cat, stream;
  double work, t0, t1;
} harmony_kernel_rec;
harmony_status harmony_read_kernel_timeline(const harmony_ctx* ctx, harmony_kernel_rec* out, int32_t cap,
                                           int32_t* n_out);

harmony_status harmony_set_profiling(harmony_ctx* ctx, int32_t on);
harmony_status harmony_read_profile(const harmony_ctx* ctx, harmony_kernel_profile* out);

/* Writes an ncclUniqueId (128 bytes) into out.  Call on rank 0 only, then broadcast. */
harmony_status harmony_get_unique_id(uint8_t out[128]);

/* Validates cfg, selects cfg->device, creates streams/events, allocates (or adopts)
 * the arena and, for world_size > 1, the NCCL communicator.  *out owns everything. */
harmony_status harmony_init(const harmony_config* cfg, harmony_ctx** out);

/* Single-process group: one context driving num_ranks data-parallel ranks (1..16), rank r on
 * CUDA device devices[r] (NULL = all on device 0; repeated ordinals = ranks sharing a GPU, each
 * with its own arena of cfg->hbm_cap_bytes).  cfg->rank, cfg->world_size, cfg->device and
 * cfg->nccl_id are ignored; cfg->arena must be NULL.  Ranks on different GPUs need peer access
 * (HARMONY_E_UNSUPPORTED otherwise).  Afterwards the context is used like a rank context:
 * harmony_register_layers, harmony_step with the GLOBAL batch (x, target: num_ranks*m*b rows;
 * rank r takes rows r*m*b .. (r+1)*m*b-1, reading c14), harmony_read_state (no collective),
 * harmony_finalize.  harmony_step's stats are box totals (bytes summed over ranks); per-rank
 * ledgers via harmony_read_rank_stats.  Collectives: rank r's reduced-gradient shard is the sum
 * of the N ranks' fp32 partials in rank order 0..N-1 (deterministic, the same on one GPU or many);
 * all-gathers are copies.  Per-kernel profiling is not available for num_ranks > 1. */
harmony_status harmony_init_group(const harmony_config* cfg, int32_t num_ranks, const int32_t* devices,
                                  harmony_ctx** out);
harmony_status harmony_read_rank_stats(const harmony_ctx* ctx, int32_t rank, harmony_step_stats* out);
/* Host-only planning of a group of num_ranks ranks (no CUDA call): for HARMONY_SCHED_HARMONY_PP the
 * group's one program (each op tagged rank=r), else rank 0's data-parallel program. */
harmony_status harmony_plan_dry_group(const harmony_config* cfg, int32_t num_ranks, int32_t n_layers,
                                      const harmony_layer_desc* descs, harmony_plan_summary* out, char* program_text,
                                      uint64_t text_len);

/* Registers the layer stack and its initial fp32 parameters (canonical packing, one
 * host array per layer, identical on every rank).  Decomposes the step into tasks,
 * plans residency / slots / swap sets / the per-stream program, and fills the pinned
 * host store (this rank's shard of master W, m = v = 0, and of the compute copy).
 * Returns HARMONY_E_CAP_TOO_SMALL when the minimum working set exceeds the cap.
 * Weight tying is impossible by construction (each layer owns its parameters;
 * reading c4: no weight is read after its own backward, so JIT updates are exact). */
harmony_status harmony_register_layers(harmony_ctx* ctx, int32_t n_layers, const harmony_layer_desc* descs,
                                       const float* const* init_params);

/* One training step on this rank's local batch of m*b samples.
 *  x:      host or device fp32 [m*b, S, d_in] (MLP: [m*b, d_in]), this rank's rows of
 *          the global batch (rank r holds global rows r*m*b .. (r+1)*m*b-1, reading c14)
 *  target: host or device fp32, the output shape
 *  batch:  must equal m*b
 *  loss_out (nullable): the GLOBAL loss (rank partials summed in rank order, c22)
 *  stats (nullable): this rank's ledger for the step
 * Synchronous: returns when the update of every layer has finished on this GPU.
 * Ordering: the step's first copy waits for work the caller queued on the legacy default stream
 * (e.g. torch ops on its default stream writing x / target); work on other caller streams must be
 * synchronised by the caller before the call.  On any failure after work was issued the context
 * is marked broken (only harmony_finalize is valid) and Adam's t is not advanced. */
harmony_status harmony_step(harmony_ctx* ctx, const float* x, const float* target, int64_t batch, double* loss_out,
                            harmony_step_stats* stats);

/* Reads one fp32 state tensor of `layer` (n_floats = the layer's parameter count) into
 * the host buffer dst.  HARMONY_GRAD needs retain_grads.  For world_size > 1 this is a
 * collective (all ranks must call it with the same arguments). */
harmony_status harmony_read_state(harmony_ctx* ctx, int32_t layer, int32_t which, float* dst, uint64_t n_floats);

harmony_status harmony_read_stats(const harmony_ctx* ctx, harmony_step_stats* out);
harmony_status harmony_plan_info(const harmony_ctx* ctx, harmony_plan_summary* out);

/* Host-only planning (no CUDA call): what register_layers would plan for this
 * config.  program_text (nullable) receives a textual dump of the per-stream program
 * (truncated to text_len bytes).  Used by the CPU tests of the scheduler. */
harmony_status harmony_plan_dry(const harmony_config* cfg, int32_t n_layers, const harmony_layer_desc* descs,
                                harmony_plan_summary* out, char* program_text, uint64_t text_len);

/* ---- Operator decomposition of one GEMM fwd+bwd across the DP group.
 * Y = X.W with X [M,K], W [K,N] (bf16, row-major), K split across the world_size ranks: rank r passes
 * its K-slice X[:, r*K/N' .. ] as a [M][K/N'] array and W[r*K/N' .., :] as [K/N'][N] (N' = world).
 * The forward runs as `chunks` row-chunk tile subtasks whose fp32 partials are reduce-scattered
 * (NCCL) while the next chunk computes; rank r receives Y_shard = rows [r*M/N', (r+1)*M/N') of Y
 * (fp32).  Backward: dY_shard (bf16, the same rows) is all-gathered, then dX_slice = dY.W_slice^T
 * (bf16 [M][K/N']) and dW_slice = X_slice^T.dY (fp32 [K/N'][N]) are computed locally.  All pointers are
 * DEVICE pointers owned by the caller; run() is synchronous and collective (every rank calls it).
 * Requirements: K % (8*world) == 0, M % (world*chunks) == 0, M and N multiples of 8. */
typedef struct harmony_split_gemm harmony_split_gemm;
harmony_status harmony_split_gemm_init(const harmony_config* cfg, int64_t M, int64_t N, int64_t K, int32_t chunks,
                                       harmony_split_gemm** out);
harmony_status harmony_split_gemm_run(harmony_split_gemm* g, const void* X_slice, const void* W_slice,
                                      const void* dY_shard, float* Y_shard, void* dX_slice, float* dW_slice,
                                      double* seconds);
/* The same decomposition with all ranks in one process (rank r on devices[r]; NULL = device 0;
 * repeated ordinals = ranks sharing a GPU).  run_group takes per-rank pointer arrays (num_ranks
 * entries each, rank r's slices/shards as above, DEVICE pointers on rank r's GPU).  The chunk
 * reduce-scatter is the library's own: rank i's rows of chunk c are the sum of every rank's fp32
 * partial in rank order 0..N-1 (pulled from the peers' buffers); the dY all-gather is a copy. */
harmony_status harmony_split_gemm_init_group(int32_t num_ranks, const int32_t* devices, int64_t M, int64_t N,
                                             int64_t K, int32_t chunks, harmony_split_gemm** out);
harmony_status harmony_split_gemm_run_group(harmony_split_gemm* g, const void* const* X_slice,
                                            const void* const* W_slice, const void* const* dY_shard,
                                            float* const* Y_shard, void* const* dX_slice, float* const* dW_slice,
                                            double* seconds);
harmony_status harmony_split_gemm_finalize(harmony_split_gemm* g);

/* Frees every device and pinned allocation and the communicator; ctx is invalid after. */
harmony_status harmony_finalize(harmony_ctx* ctx);

/* Last error message of ctx (or of the last failed context-less call when ctx is NULL). */
const char* harmony_last_error(const harmony_ctx* ctx);

int32_t harmony_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* HARMONY_H_ */
