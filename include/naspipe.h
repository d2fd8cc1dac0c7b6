/*
 * naspipe.h — C ABI of the B200-native NASPipe hot path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, cited P:L<line>):
 *   Causal-synchronous-parallel (CSP) pipelined training of sampled subnets over a
 *   supernet partitioned into stages (Def.2; Alg.1/Alg.2).
 *   A supernet is a sequence of m choice blocks with n candidates each; a subnet
 *   y picks one candidate per block; subnets are trained in the chronological order of
 *   their submission.  The result (every candidate's parameters and every subnet's loss)
 *   equals training the subnets one at a time in that order (Def.1), with
 *   plain SGD on the active candidates (reading A3).
 *
 * Conventions
 *   - Every function returns naspipe_status (0 = OK, < 0 = error) unless stated otherwise.
 *     naspipe_last_error() returns a thread-local message for the last error.
 *   - Invalid arguments -> NASPIPE_EINVAL with no state change (a rejected submit does not
 *     consume a sequence id).  CUDA / NCCL faults are sticky: every later call on the
 *     handle returns the same code.
 *   - Pointers are host pointers unless a field says "device".  No torch types.
 *   - Handles are not thread-safe; one handle per process (multi-process mode: one per rank).
 *   - Parameters are exchanged as float32 "packed candidate vectors" in the canonical
 *     order of the family (weights row-major [out,in], then biases, then norm gamma/beta):
 *       MLP:          W[d,d], b[d]
 *       TRANSFORMER:  Wqkv[3d,d], bqkv[3d], Wo[d,d], bo[d], ln1.g[d], ln1.b[d],
 *                     W1[f,d], b1[f], W2[d,f], b2[d], ln2.g[d], ln2.b[d]
 *       SPOS_CNN:     for each conv of the candidate in order (stride-2 blocks: the proj
 *                     branch's dw, pw first; then the main branch's convs), the conv weight
 *                     (pw [out,in]; dw [C,k,k]) followed by its BatchNorm gamma[out], beta[out].
 *                     Main branch, choices with kernel k (SURVEY §8c "C2 SPOS candidate",
 *                     DESIGN.md A16/A27): Shuffle = pw in->mid, dw k (stride s), pw mid->out;
 *                     Xception = dw3 (s), pw in->mid, dw3, pw mid->mid, dw3, pw mid->out.
 */
#ifndef NASPIPE_H_
#define NASPIPE_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default) /* the library builds with -fvisibility=hidden */
#endif

#define NASPIPE_ABI_VERSION 4

typedef enum {
  NASPIPE_OK = 0,
  NASPIPE_EINVAL = -1,   /* invalid argument / inconsistent spec                        */
  NASPIPE_ESTATE = -2,   /* call not valid in the current state (e.g. get before drain) */
  NASPIPE_ENOMEM = -3,   /* host or device allocation failed                            */
  NASPIPE_ECUDA = -4,    /* CUDA runtime / driver error (sticky)                        */
  NASPIPE_ENCCL = -5,    /* NCCL error (sticky)                                         */
  NASPIPE_EBUDGET = -6,  /* HBM weight budget cannot hold one task's candidates         */
  NASPIPE_EINTERNAL = -7 /* internal invariant violated (e.g. version check) (sticky)   */
} naspipe_status;

typedef enum { NASPIPE_MLP = 0, NASPIPE_TRANSFORMER = 1, NASPIPE_SPOS_CNN = 2 } naspipe_family;

/* spec.sync_policy: how stages admit queued forwards (Fig.1).
 *   CSP      causal synchronous parallel (Def.2): admit the lowest-id queued forward
 *            whose dependencies are finished on the stage (Alg.1/Alg.2) — the method.
 *   INORDER  "NASPipe w/o scheduler" (Fig.6 ablation): queued forwards are taken
 *            strictly in id order; a blocked head blocks the stage.  Numerics = CSP.
 *   ASP      asynchronous (PipeDream-style): dependencies ignored; a forward
 *            reads the weights current on its stage, a backward's input gradient uses the
 *            weights current at its start (no weight stashing).  Executable; results
 *            depend on the stage count (Table 3).
 *   BSP      bulk synchronous (GPipe / Retiarii): bulks of `bulk_size`
 *            consecutive subnets; within a bulk dependencies are ignored, forwards run
 *            before backwards on every stage, and the next bulk starts after the flush
 *            (every subnet of the bulk finished on every stage).  Numerics: every task of a
 *            bulk reads the bulk-start weights, the SGD WRITEs accumulate into a per-
 *            candidate fp32 copy, copied back into the masters at the flush (= the bulk's
 *            gradients, summed, applied once).  Executable with every candidate resident
 *            (naspipe_create: EINVAL with hbm_weight_budget_bytes > 0).
 *   SERIAL   "NASPipe w/o scheduler" as P:L454 words it: it "had to finish the execution of a
 *            pipeline before injecting the next pipeline" -- one subnet in flight at a time
 *            (the window forced to W = 1; reading A32).  Numerics = CSP. */
typedef enum { NASPIPE_SYNC_CSP = 0, NASPIPE_SYNC_INORDER = 1, NASPIPE_SYNC_ASP = 2, NASPIPE_SYNC_BSP = 3,
               NASPIPE_SYNC_SERIAL = 4 } naspipe_sync;
typedef enum { NASPIPE_FP32 = 0, NASPIPE_BF16 = 1 } naspipe_dtype; /* compute dtype; masters fp32 */

/* spec.flags */
#define NASPIPE_FLAG_TRACE 1         /* keep the executed task trace (naspipe_get_trace)      */
#define NASPIPE_FLAG_VERSION_CHECK 2 /* assert candidate versions at every task start        */
#define NASPIPE_FLAG_NULL_KERNELS 4  /* run planner/transport only; kernels become no-ops     */
#define NASPIPE_FLAG_TIMING 8        /* CUDA-event timing of the dominant kernel (GEMM)      */
/* Activation recomputation ("NASPIPE adopts activation recomputing techniques";
 * reading A13): the forward keeps only each block's input; the backward recomputes the
 * block's forward before its gradient.  The kernels are deterministic and CSP/BSP never
 * update a candidate between F(y) and B(y), so results are bitwise those without it.
 * TRANSFORMER family only, not with ASP (EINVAL otherwise). */
#define NASPIPE_FLAG_RECOMPUTE 16
/* Executed layer mirroring (P:L166 per-subnet balanced partitions, P:L298
 * "Layer Mirroring ... the new parameters are actively pushed to all the other mirrored
 * ones"; reading A31): subnet y runs its blocks on the stages of ITS OWN balanced
 * partition (naspipe_plan_mirrored's schedule, mirror latency = link_latency), every stage
 * holds a mirror copy of every candidate, and after each backward's SGD WRITE the updated
 * fp32 master and bf16 shadow are pushed to the other stages' copies on a push stream; a task
 * that reads a candidate last written on another stage waits for that push.  Numerics are the
 * sequential result (CSP).  naspipe_create only (single process), CSP with strict
 * backward-first, every candidate resident, no recompute (EINVAL otherwise).  Tasks are
 * planned and issued at naspipe_drain (the mirrored plan is computed over the submitted
 * stream). */
#define NASPIPE_FLAG_MIRROR 32
/* Timing-driven execution (Alg.1 P:L170-197 run on OBSERVED completions,
 * Alg.3's predictor P:L239-273 evaluated online; reading A39): instead of walking
 * the logical-time plan, the host polls each stage's running task (a CUDA event) and, the
 * moment a stage is free, picks its next task by Alg.1 + Alg.2 with the state it observes:
 * the lowest-id backward whose output gradient has arrived, else the lowest-id queued forward
 * whose input has arrived and whose candidates' previous users have finished their backward
 * on this stage (Def.2), stage 0 admitting y < (lowest unfinished id) + W.  At every backward
 * start the stage runs Alg.3's prediction of its next forward (Alg.2 on its queue with the
 * starting backward counted finished); naspipe_get_timed_stats reports how often it was right.
 * The schedule depends on kernel timing (it is not unique); the numerics do not (CSP): results
 * are bitwise those of the planned executor.  naspipe_create only, CSP with strict
 * backward-first, every candidate resident, no mirroring (EINVAL otherwise).  Tasks run at
 * naspipe_drain over the submitted stream; the trace's t is microseconds since that drain. */
#define NASPIPE_FLAG_TIMED 64

/*
 * Supernet specification.  naspipe_create deep-copies it and every array it points to.
 *   family, n_blocks (m), n_choices (n), batch (B), compute_dtype   — all families
 *   width                                                          — MLP (d)
 *   d_model, seq_len, choice_heads[n], choice_ffn[n]               — TRANSFORMER
 *   lr            plain SGD learning rate (reading A3)
 *   init_seed     counter-hash initialisation (reading A21): w = bound*(2u-1),
 *                 u = (splitmix64(seed ^ (uid*0x9E3779B97F4A7C15 + i)) >> 40) * 2^-24,
 *                 uid = b*n + c, i = index in the packed vector, bound = 1/sqrt(fan_in);
 *                 LayerNorm gamma = 1, beta = 0.
 *   stage_of_block [m] optional, non-decreasing, 0..n_stages-1 each used; NULL = balanced
 *                 partition (reading A12) of the cost table.
 *   cost_fwd, cost_bwd [m*n] optional integer ticks >= 0 per (block, choice); NULL =
 *                 naspipe_default_costs.  A stage task costs max(1, sum over its blocks).
 *   window        W: stage 0 starts F(y,0) only for y < (lowest unfinished id) + W
 *                 (reading A7); 0 = 4 * n_stages.
 *   lookahead     residency prefetch depth L in tasks ("2"); 0 = 2.
 *   residency_horizon  H: Belady's "next use" looks at the stage's next H tasks only
 *                 (reading A26); 0 = 64, < 0 = unbounded (decisions wait for the final plan).
 *   hbm_weight_budget_bytes  per-stage device budget for candidate fp32 masters; 0 = all
 *                 candidates resident (no context switching).
 *   bwd_policy    0 = strict backward-first (reading A5); 1 = Alg.1 alternation.
 *   link_latency  lambda ticks for stage-boundary deliveries in the planner (reading A8).
 *   SPOS_CNN only (SPOS [9] search space; op types of Table 5):
 *   image_hw      input resolution (square), divisible by 2^(1 + n_cnn_stages)
 *   num_classes   classes of the frozen FC head
 *   stem_channels frozen stem conv3x3 s2 3->stem_channels (+BN(1,0)+ReLU), % 16 == 0
 *   head_channels frozen head pw Clast->head_channels, BN(1,0), ReLU, GAP, FC (no bias)
 *   n_cnn_stages, stage_repeats[n_cnn_stages] (sum = n_blocks), stage_channels[..] (% 32,
 *                 strictly increasing, first > stem_channels): the first block of each
 *                 stage has stride 2, inp = C_prev, mid = C/2, out = C - C_prev; the
 *                 others stride 1 with inp = mid = out = C/2 (channel split).
 *   choice_kernel[n] (3, 5 or 7): the k of every depthwise conv of choice n;
 *   choice_xception[n] (0 = Shuffle, 1 = Xception, 2 = Table 5's dense "Conv 3x3", P:L447:
 *                 the Shuffle block with its depthwise conv replaced by a dense 3x3 conv over
 *                 the mid channels, weights [mid][3][3][mid], k 3 and dilation 1 only;
 *                 DESIGN.md A40); choice_dilation[n] (ABI 4; 1 or 2,
 *                 NULL = all 1): dilation of choice n's depthwise convs, pad dilation*(k/2)
 *                 (Table 5's "Dil Conv 3x3"; A36)
 *   Frozen stem/head/FC weights use the counter hash with uids m*n + {0, 1, 2}, fan_in
 *   27 / C_last / head_channels; they are never updated (reading A2).
 */
typedef struct {
  int32_t abi_version; /* = NASPIPE_ABI_VERSION */
  int32_t family;
  int32_t n_blocks;
  int32_t n_choices;
  int32_t batch;
  int32_t compute_dtype;
  int32_t width;
  int32_t d_model;
  int32_t seq_len;
  const int32_t* choice_heads;
  const int32_t* choice_ffn;
  float lr;
  uint64_t init_seed;
  const int32_t* stage_of_block;
  const int32_t* cost_fwd;
  const int32_t* cost_bwd;
  int32_t window;
  int32_t lookahead;
  int32_t residency_horizon;
  int64_t hbm_weight_budget_bytes;
  int32_t bwd_policy;
  int32_t link_latency;
  int32_t flags;
  /* SPOS_CNN (ignored otherwise) */
  int32_t image_hw;
  int32_t num_classes;
  int32_t stem_channels;
  int32_t head_channels;
  int32_t n_cnn_stages;
  const int32_t* stage_repeats;
  const int32_t* stage_channels;
  const int32_t* choice_kernel;
  const int32_t* choice_xception;
  /* ABI 3: synchronisation policy (naspipe_sync; 0 = CSP) and BSP bulk size (0 = 4 * n_stages) */
  int32_t sync_policy;
  int32_t bulk_size;
  /* ABI 4: per-choice depthwise dilation (SPOS_CNN; NULL = 1) */
  const int32_t* choice_dilation;
  /* ABI 4: per-choice token mixer (TRANSFORMER; NULL = all attention): 0 multi-head attention,
   * 1 Conv 3x1, 2 Sep Conv 7x1, 3 Light Conv 5x1 (heads = its weight-sharing heads H) --
   * Table 5's NLP ops; internals: DESIGN.md A38, oracle/transformer.py */
  const int32_t* choice_op;
} naspipe_supernet_spec;

/* naspipe_batch.where */
#define NASPIPE_BATCH_HOST 0      /* input/target are host float32 buffers; read
                                     asynchronously, must stay valid until naspipe_drain */
#define NASPIPE_BATCH_DEVICE 1    /* device float32 buffers on the stage-0 / last-stage
                                     device; borrowed until naspipe_drain                */
#define NASPIPE_BATCH_SYNTHETIC 2 /* generated on the device from synth_seed (perf only)  */

/* One subnet's batch: input [batch x sample] and target [batch x sample] float32, where
 * sample = width (MLP) or seq_len*d_model (TRANSFORMER), row-major.  SPOS_CNN: input is
 * float32 NHWC [batch, image_hw, image_hw, 3], target is int32 labels [batch] in
 * [0, num_classes) (loss = mean cross-entropy of the frozen head, reading A18). */
typedef struct {
  const void* input;
  const void* target;
  int32_t where;
  uint64_t synth_seed;
} naspipe_batch;

typedef struct naspipe_handle naspipe_t;

/* ---------------------------------------------------------------------------------------
 * Engine (the hot path)
 * ------------------------------------------------------------------------------------- */

/* Single-process engine: all n_stages stages live in this process; stage K runs on CUDA
 * device (current_device + K) % device_count.  Allocates all device memory, initialises
 * every candidate from init_seed.  EBUDGET if the budget cannot hold one task's need. */
int naspipe_create(const naspipe_supernet_spec* spec, int32_t n_stages, naspipe_t** out);

/* Multi-process engine (one process per GPU): this process runs stage `stage_rank` on CUDA
 * device `device`.  nccl_ids points to 2*(n_stages-1) ncclUniqueId blobs (128 bytes each):
 * [2k] = activation channel k -> k+1, [2k+1] = gradient channel k+1 -> k, identical on every
 * rank.  Every rank must make the same sequence of naspipe_submit / naspipe_drain calls. */
int naspipe_create_rank(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t stage_rank,
                        int32_t device, const void* nccl_ids, naspipe_t** out);

/* Multi-process engine with the PEER-MEMORY transport (the paper's
 * inter-stage send/recv, re-designed for NVLink/NVSwitch): this process runs stage
 * `stage_rank` on CUDA device `device` and allocates its receive rings (stage-input
 * activations and output gradients, `window` slots each) plus a flag page.  The producing
 * kernels of the neighbouring ranks store boundary tensors straight into these rings over
 * CUDA IPC mappings (NVLink peer stores; plain HBM stores when two ranks share one GPU) and
 * publish each slot with a stream memory write; consumers wait on it with a stream memory
 * wait.  Protocol: create on every rank -> naspipe_peer_export -> exchange the blobs out of
 * band (e.g. torch.distributed all_gather_object over gloo) -> naspipe_peer_connect with the
 * blob of rank-1 (NULL on rank 0) and of rank+1 (NULL on the last rank) -> identical
 * submit / drain sequences on every rank.  ESTATE if submit comes before connect (D > 1);
 * EINVAL for a blob of the wrong rank, stage count, window or slot size.  The engine owns
 * the rings; blobs are plain bytes, valid while the exporting engine lives. */
int naspipe_create_rank_peer(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t stage_rank,
                             int32_t device, naspipe_t** out);
/* Write this rank's blob (CUDA IPC handles of its rings and flag page, sizes, rank) into dst;
 * *n = its size (dst NULL: size query only).  EINVAL if cap < size or not a peer engine. */
int naspipe_peer_export(naspipe_t* h, void* dst, size_t cap, size_t* n);
/* Map the neighbours' rings (see naspipe_create_rank_peer).  Once per engine. */
int naspipe_peer_connect(naspipe_t* h, const void* prev_blob, size_t prev_n, const void* next_blob,
                         size_t next_n);

/* Submit the next subnet in chronological order.  subnet_choice_vec [m] with entries in
 * [0, n).  Assigns and returns its sequence id (0, 1, 2, ...).  Plans as far as the
 * streaming rule allows and issues the planned tasks asynchronously. */
int naspipe_submit(naspipe_t* h, const int32_t* subnet_choice_vec, const naspipe_batch* batch,
                   int64_t* seq_id_out);

/* Fix N = number of submitted subnets, plan and run everything, wait for the devices. */
int naspipe_drain(naspipe_t* h);

/* Copy candidate (block, choice)'s fp32 master parameters (packed order above) into dst.
 * Only on the rank that owns the block.  ESTATE before naspipe_drain. */
int naspipe_get_params(naspipe_t* h, int32_t block, int32_t choice, float* dst, size_t n_floats);
int naspipe_set_params(naspipe_t* h, int32_t block, int32_t choice, const float* src,
                       size_t n_floats);

/* Per-subnet losses (last stage's rank), seq ids [0, n). ESTATE before drain. */
int naspipe_get_losses(naspipe_t* h, float* dst, int64_t n);

/* Executed tasks in issue order: 4 int64 per task (tick, stage, kind 0=F/1=B, seq id). */
int naspipe_get_trace(naspipe_t* h, int64_t* dst, size_t cap_tasks, size_t* n_tasks);

/* Statistics, 16 doubles: [0] tasks, [1] kernel launches, [2] h2d bytes, [3] d2h bytes,
 * [4] p2p bytes, [5] makespan ticks, [6] dominant-kernel launches, [7] dominant-kernel
 * algorithmic work (flops of the transformer GEMMs / HBM bytes of the SPOS BatchNorm
 * kernels; both counted whether or not TIMING is on), [8] dominant-kernel ms (TIMING flag
 * only), [9] residency loads, [10] residency evicts, [11] writebacks, [12] version checks
 * passed, [13] algorithmic flops of every tcgen05 GEMM launched by this process,
 * [14] tcgen05 GEMM launches of this process, [15] algorithmic HBM bytes of every kernel
 * the families launched (SPOS: each tensor read / written once per launch at its stored
 * width; 0 for the other families). */
int naspipe_get_stats(naspipe_t* h, double* dst16);

/* Turn the dominant-kernel CUDA-event timing (stats [6..8]) on or off for the work submitted
 * from now on (bench.py measures throughput with it off and the roofline with it on: the
 * events between kernels cost PDL overlap).  Only between a drain and the next submit:
 * ESTATE otherwise.  The initial state is the spec's NASPIPE_FLAG_TIMING. */
int naspipe_set_timing(naspipe_t* h, int on);

/* Residency trace: 4 int64 per event (stage, task index, op 0=LOAD/1=EVICT, uid=b*n+c). */
int naspipe_get_residency_trace(naspipe_t* h, int64_t* dst, size_t cap, size_t* n);

/* NASPIPE_FLAG_TIMED engines: dst[0] tasks issued by the timing-driven executor, [1] backward
 * starts, [2] Alg.3 predictions made at those starts (a queued forward was admissible), [3]
 * predictions equal to the forward the stage actually ran next, [4] host decision-loop
 * wall time (ms), [5] reserved.  Zeros for other engines. */
int naspipe_get_timed_stats(naspipe_t* h, double* dst6);

void naspipe_destroy(naspipe_t* h); /* implies drain; NULL is a no-op */

/* ---------------------------------------------------------------------------------------
 * Host-only helpers (no device needed): spec queries and the deterministic CSP planner.
 * ------------------------------------------------------------------------------------- */
int naspipe_param_count(const naspipe_supernet_spec* spec, int32_t block, int32_t choice,
                        size_t* n_floats);
/* Analytic integer tick table (1 tick = 1 us): cost_fwd/cost_bwd [m*n]. */
int naspipe_default_costs(const naspipe_supernet_spec* spec, int32_t* cost_fwd, int32_t* cost_bwd);
/* Stage of each block for n_stages (the spec's or the balanced partition). */
int naspipe_partition(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t* stage_of_block);
/* Per-subnet balanced partitions with layer mirroring ("a D-partition
 * ... of a subnet's sequential list of layers, with each partition having roughly the same
 * execution time"; "Layer Mirroring ... the new parameters are actively pushed to all
 * the other mirrored ones"; reading A31).  PLANNING ONLY (the executor runs the
 * supernet partition of naspipe_partition).
 *   Subnet y's stage of block b = the balanced partition (A12's DP and tie rule) of y's own
 *   per-block costs cost_fwd + cost_bwd of (b, c_y[b]); stage_of_block [N*m] receives it.
 *   Schedule: the O2 event model (spec window, link_latency, strict backward-first, lowest id)
 *   with CSP read across stages: F(y, K) starts at t only if for each of y's blocks b on K
 *   the previous user x of (b, c_y[b]) finished B(x, stage_x(b)) (its WRITE) by t, plus
 *   mirror_latency ticks (>= 0) when stage_x(b) != K.
 *   trace: 4 int64 per task start (tick, stage, kind 0=F/1=B, y), *n_tasks = 2*N*n_stages
 *   (entries beyond cap_tasks are not written); stall/bubble [n_stages] or NULL.
 *   Errors: EINVAL for a choice out of range, n_stages outside 1..m, a sync_policy other
 *   than CSP or bwd_policy != 0, mirror_latency < 0, NULL n_tasks/makespan. */
int naspipe_plan_mirrored(const naspipe_supernet_spec* spec, int32_t n_stages, const int32_t* choices,
                          int64_t n_subnets, int32_t mirror_latency, int32_t* stage_of_block, int64_t* trace,
                          size_t cap_tasks, size_t* n_tasks, int64_t* makespan, int64_t* stall,
                          int64_t* bubble);

/* Initial packed parameters of one candidate (same generator the engine uses). */
int naspipe_init_params(const naspipe_supernet_spec* spec, int32_t block, int32_t choice,
                        float* dst, size_t n_floats);

/* SPOS_CNN frozen (never-updated, reading A2) weights: part 0 = stem [C0,3,3,3] ([out, kh,
 * kw, in]), 1 = head 1x1 conv [head_channels, C_last], 2 = FC [num_classes, head_channels];
 * the counter hash of init_seed with uid = n_blocks*n_choices + part.  EINVAL for other
 * families or a size mismatch. */
int naspipe_init_frozen(const naspipe_supernet_spec* spec, int32_t part, float* dst, size_t n_floats);

typedef struct naspipe_plan_handle naspipe_plan_t;
/* Plan N subnets (choices [N*m]) on n_stages stages: the logical-time CSP schedule
 * using the spec's window, costs, policy and latency. */
int naspipe_plan_create(const naspipe_supernet_spec* spec, int32_t n_stages,
                        const int32_t* choices, int64_t n_subnets, naspipe_plan_t** out);
int naspipe_plan_trace(const naspipe_plan_t* p, int64_t* dst, size_t cap_tasks, size_t* n_tasks);
int naspipe_plan_makespan(const naspipe_plan_t* p, int64_t* makespan);
/* deps(y, K): ids of the latest earlier users of y's stage-K candidates (dependency table). */
int naspipe_plan_deps(const naspipe_plan_t* p, int64_t y, int32_t stage, int64_t* dst, size_t cap,
                      size_t* n);
/* Belady residency of stage K under budget bytes of fp32 masters (0 = all resident), depth
 * L (0 = spec's), next-use horizon H (0 = spec's, < 0 = unbounded); 4 int64 per event
 * (stage, task index, op 0=LOAD/1=EVICT, uid); writebacks counted in *n_writebacks. */
int naspipe_plan_residency(const naspipe_plan_t* p, int32_t stage, int64_t budget_bytes,
                           int32_t depth, int32_t horizon, int64_t* dst, size_t cap, size_t* n,
                           int64_t* n_writebacks);
/* Idle ticks per stage [n_stages]: stalled (a queued forward is blocked by a dependency)
 * and bubble (nothing queued).  busy + stall + bubble = makespan on every stage. */
int naspipe_plan_idle(const naspipe_plan_t* p, int64_t* stall, int64_t* bubble);
/* Multi-process point-to-point schedule of one rank (= stage) in the order the executor
 * issues it: 3 int64 per operation (op 0=SEND_ACT to rank+1, 1=RECV_ACT from rank-1,
 * 2=SEND_GRAD to rank-1, 3=RECV_GRAD from rank+1; peer rank; subnet id). */
int naspipe_plan_comm_schedule(const naspipe_plan_t* p, int32_t rank, int64_t* dst, size_t cap, size_t* n);
void naspipe_plan_destroy(naspipe_plan_t* p);

/* Fill 128 bytes with a fresh ncclUniqueId (for naspipe_create_rank's nccl_ids). */
int naspipe_nccl_unique_id(void* out128);

/* Process-wide PDL switch (programmatic dependent launch between consecutive kernels of a
 * stream; default on where the engine allows it).  bench.py turns it off for its CUPTI
 * kernel-time run so that every kernel's recorded interval is its own execution, not the
 * wait for its predecessor.  Results are bitwise the same either way. */
int naspipe_set_pdl(int enabled);

const char* naspipe_last_error(void);
int naspipe_abi_version(void);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif /* NASPIPE_H_ */
