/*
 * hogbatch.h — C ABI of libhogbatch.so, the B200 (sm_100a) hot path of
 * Adaptive Hogbatch (Ma, Rusu, Wu, Sim, IPDPSW/MARWS 2021; /root/reference/PAPER.md).
 *
 * Every entry point returns an int status: HB_OK (0) or a negative HB_E* code;
 * hb_last_error() returns a thread-local human-readable message for the last
 * failure on the calling thread.  No C++ exception crosses this boundary.
 * No torch types appear here: device memory is passed as raw pointers (the
 * Python binding allocates it with torch), streams as cudaStream_t cast to void*.
 *
 * Notation (§III): an MLP with L weight layers and widths
 * n_0 = d_in, n_1..n_{L-1} hidden, n_L = C classes.  Layer l (1-based) holds
 * W_l in R^{n_l x n_{l-1}} (the paper's W^l in R^{d_{l+1} x d_l}, row-major
 * [out, in]) and a bias b_l in R^{n_l}.  Hidden activation: sigmoid; output:
 * softmax with cross-entropy loss (L258).  The batch loss is the mean over
 * the batch (R10).
 */
#ifndef HOGBATCH_H
#define HOGBATCH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HB_ABI_VERSION 2

/* status codes */
enum {
  HB_OK = 0,
  HB_EINVAL = -1,       /* bad argument (size, pointer, dtype, state)          */
  HB_ENOMEM = -2,       /* device or host allocation failed                    */
  HB_ECUDA = -3,        /* a CUDA runtime/driver call failed (message captured) */
  HB_ENCCL = -4,        /* an NCCL call failed                                 */
  HB_ESTATE = -5,       /* call not valid in the object's current state        */
  HB_EUNSUPPORTED = -6  /* valid request this build does not implement         */
};

/* hidden activation F_l (sigmoid) */
enum { HB_SIGMOID = 0 };

/* arithmetic of a model (fixed at creation) */
enum {
  HB_PREC_BF16 = 0,      /* tcgen05 tensor cores: bf16 operands, fp32 accumulate, fp32 master */
  HB_PREC_FP32_CHECK = 1 /* fp32 CUDA-core check mode (SIMT GEMMs, fp32 activations)          */
};

/* dtype of the input matrix X */
enum { HB_BF16 = 0, HB_F32 = 1 };

/* scheduling policies (§VI) */
enum {
  HB_MINIBATCH = 0, /* one worker, fixed b: mini-batch SGD (L55–L56, L262)            */
  HB_HOGBATCH = 1,  /* Algorithm 1: every worker gets the same b (L147–L170)          */
  HB_STATIC = 2,    /* CPU+GPU Hogbatch: fixed per-worker b (L172–L179)               */
  HB_ADAPTIVE = 3   /* Algorithm 2: adaptive per-worker b (L181–L238)                 */
};

/* Algorithm 2 readings (R3, R21) */
enum { HB_RESET_FASTEST = 0, HB_RESET_NONE = 1 };          /* u^E <- min_u in the "fastest" branch, or never */
enum { HB_CREDIT_DISPATCH = 0, HB_CREDIT_COMPLETION = 1 }; /* when u^E += incr is counted                    */

/* trace actions */
enum { HB_ACT_NONE = 0, HB_ACT_HALVE = 1, HB_ACT_DOUBLE = 2, HB_ACT_CLAMP_LO = 3, HB_ACT_CLAMP_HI = 4 };

typedef struct hb_model hb_model;
typedef struct hb_worker hb_worker;
typedef struct hb_comm hb_comm;
typedef struct hb_coord hb_coord;

/* Per-worker policy (Algorithm 2 inputs min_b^E, max_b^E [L194]; initial size [L236]). */
typedef struct hb_worker_policy {
  int32_t min_b;  /* lower threshold (never crossed, L236)                                */
  int32_t max_b;  /* upper threshold                                                        */
  int32_t init_b; /* initial batch size                                                     */
  float incr;     /* updates credited per served batch: 1 (Alg. 1 worker) or t*beta (L234)  */
  double c0, c1;  /* deterministic mode: virtual cost T(b) = c0 + c1*b                      */
} hb_worker_policy;

typedef struct hb_policy {
  int32_t kind;          /* HB_MINIBATCH .. HB_ADAPTIVE                                      */
  int32_t alpha;         /* batch scale factor, default 2 (L236)                              */
  double eta0;           /* learning rate at batch b0; lr = eta0 * b / b0 (L179)              */
  int32_t b0;
  int32_t reset;         /* HB_RESET_*                                                        */
  int32_t credit;        /* HB_CREDIT_*                                                       */
  int32_t deterministic; /* 1: virtual clock + SERIAL execution in trace order (L125–L128)   */
  int32_t eval_loss;     /* 1: full-data loss at every epoch end (excluded from timing, L258) */
  int64_t max_steps;     /* stop after this many served batches in total (0 = no limit)      */
  int32_t merges_per_epoch; /* multi-GPU: replica merges per epoch (needs comm; 0 = none)     */
  float merge_gamma;     /* W <- W_base + gamma * sum(W_E - W_base); 1 = delta sum (R18)     */
  hb_comm* comm;         /* nullable; NCCL communicator for the merge                         */
  int32_t n_workers;     /* entries in workers[] (with a shared coordinator: ALL processes' workers) */
  const hb_worker_policy* workers;
  int32_t update;        /* -1: each model's HB_OPT_UPDATE; HB_UPDATE_HOGWILD / HB_UPDATE_ATOMIC for
                            this run (concurrent in-place updates of the shared model [L128])   */
  int32_t epoch_barrier; /* 1 (default): an epoch ends when no worker can be served and all are idle
                            [L170]; 0: as soon as a worker cannot be served, the next epoch starts
                            without waiting for the others' in-flight batches (no idle bubble;
                            not with merges)                                                    */
  int32_t check_labels;  /* 1: verify every label is in [0, C) before training (HB_EINVAL)      */
  struct hb_coord* coord;/* nullable: cross-process coordinator (hb_coord_create): one 𝔹 and one
                            Algorithm 2 state for the workers of every process of the node     */
  int32_t first_worker;  /* with coord: global id of this process's workers[0]                 */
} hb_policy;

/* Training data (borrowed; caller-owned).  X and y are both device pointers (used in place) or
 * both host pointers (pinned for overlap; pageable works but copies synchronously): host data
 * is staged by hogbatch_run into a device copy owned by the model, in chunks (HB_STAGE_ROWS;
 * default 32768 rows, at most 32 MB) on a copy stream, and a batch waits only for the chunk
 * holding its last row — the host->device transfer of the data set overlaps training on its
 * first rows ("the coordinator owns the data" [L123]; batches are row ranges [L141]). */
typedef struct hb_dataset {
  const void* X;  /* [n x ldx] row-major, dtype x_dtype; ldx*elemsize must be a multiple of 16 */
  int64_t ldx;    /* row stride in elements (>= n_0)                                           */
  int32_t x_dtype;/* HB_BF16 (required for HB_PREC_BF16) or HB_F32                             */
  const int32_t* y; /* [n] labels in [0, C)                                                    */
  int64_t n;      /* number of examples N                                                      */
  /* format HB_DATA_CSR: X is unused and the rows are given sparse (the paper's data sets are sparse
   * LIBSVM files "processed in dense format" [L255]): hogbatch_run copies the CSR arrays to the
   * device (when host pointers; all host or all device) and densifies them into a dense
   * [n x ldx] copy of dtype x_dtype owned by the model, chunk by chunk on its copy stream (a memset
   * and a warp-per-row scatter kernel per chunk); batches wait only for their chunk, as for dense
   * host data.  Column indices must lie in [0, n_cols) with n_cols <= ldx; values are x_dtype. */
  int32_t format;          /* HB_DATA_DENSE (0, default) or HB_DATA_CSR (1)                    */
  int64_t n_cols;          /* CSR: number of features (the model's n_0)                        */
  const int64_t* indptr;   /* CSR: [n + 1] row offsets into indices / values                   */
  const int32_t* indices;  /* CSR: [nnz] column indices                                        */
  const void* values;      /* CSR: [nnz] values of dtype x_dtype                               */
} hb_dataset;
enum { HB_DATA_DENSE = 0, HB_DATA_CSR = 1 };

/* One record per ScheduleWork message (O5). */
typedef struct hb_trace_rec {
  int64_t seq;
  int32_t epoch, worker;
  double vtime, u_before;
  int32_t b_before, action, b_after, served;
  double u_after;
  int64_t offset; /* first row of the served batch, -1 if not served */
  double lr;      /* 0 if not served                                 */
} hb_trace_rec;

/* Output statistics of hogbatch_run.  All pointers are caller-owned and nullable. */
typedef struct hb_stats {
  int32_t max_epochs;     /* capacity of the per-epoch arrays                                 */
  int32_t epochs_done;
  double* epoch_loss;     /* [max_epochs] full-data loss at epoch end (NaN if not evaluated) */
  double* epoch_train_s;  /* [max_epochs] training seconds of the epoch (loss eval excluded) */
  int64_t* updates;       /* [max_epochs * n_workers] served batches per worker per epoch    */
  int64_t* samples;       /* [max_epochs * n_workers] examples per worker per epoch          */
  hb_trace_rec* trace;    /* [trace_cap] schedule trace (all modes)                          */
  int64_t trace_cap, trace_len;
  float* step_loss;       /* [step_loss_cap] per-step batch loss, deterministic mode only    */
  int64_t step_loss_cap, n_steps;
  double total_train_s;   /* training seconds, loss evaluation excluded                     */
  int64_t total_samples;
  int32_t n_merges;
  int32_t want_train_loss;/* input: 1 = accumulate the training loss on the device (one small
                             reduction kernel per step)                                       */
  double train_loss;      /* mean per-example cross-entropy of the forward passes of every batch
                             this process served (before each update) — the run's training
                             metric, read back with 8 bytes; NaN unless want_train_loss         */
} hb_stats;

/* ---- library ---------------------------------------------------------------- */
const char* hb_last_error(void);
int hb_abi_version(void);
/* 1 if a CUDA device of compute capability 10.x is visible, else 0 */
int hb_device_ok(int32_t device);

/* ---- model (§V.B: "The global model is allocated and initialized") ----
 * dims[0..n_dims-1] = n_0 .. n_L; n_dims >= 2, all > 0, n_L >= 2 -> else HB_EINVAL.
 * activation must be HB_SIGMOID.  precision HB_PREC_*.  Weights are initialised
 * W ~ N(0, 1/fan_in), b = 0 from `seed` (R11).  The model owns its device
 * memory: fp32 master weights+biases, bf16 shadow weights (bf16 mode). */
int mlp_create(const int32_t* dims, int32_t n_dims, int32_t activation, int32_t precision,
               uint64_t seed, int32_t device, hb_model** out);
int mlp_destroy(hb_model* m);
/* number of parameters P + sum n_l (weights + biases) */
int mlp_num_params(const hb_model* m, int64_t* n_out);
/* Which step implementation the model's workers use at `batch` rows (<= 0: 8192)
 * (introspection for tests / benches):
 * returns 1 and sets *cluster_size (1, 2, 4 or 8 CTAs per 128-row block) if SGD steps take the fused
 * row-block chain (one kernel for forward, softmax-xent head and the whole dX chain, then the dW
 * GEMMs; eligible: bf16 model, uniform hidden width n <= 512, n_0 <= 512, C <= 16, 2..12 layers,
 * HB_OPT_ROWCHAIN = 1, batch >= HB_OPT_FUSED_MIN_BATCH), 0 if they take the per-layer GEMM chain,
 * < 0 on error. */
int mlp_fused_path(const hb_model* m, int32_t batch, int32_t* cluster_size);
/* Per-model settings (defaults = the measured B200 choices; none is read from the environment):
 *   HB_OPT_FUSED_MIN_BATCH  steps of >= value rows take the fused row-block chain when the shape is
 *                           eligible (0 = never; default 4096, the measured crossover).  Set before
 *                           creating workers (they allocate what the fused path needs).
 *   HB_OPT_ROWCHAIN         1 = fused row-block chain allowed (default), 0 = per-layer GEMM chain
 *   HB_OPT_RC_CLUSTER       CTAs per 128-row block of the fused chain: 1, 2, 4, 8 or 0 = auto
 *   HB_OPT_BWD_OVERLAP      1 = dW_l runs on a second stream overlapping dX_{l-1} (default)
 *   HB_OPT_HEAD_FUSE        1 = the output layer's dX runs in the head GEMM's epilogue (C <= 16;
 *                           default 0, measured slower at b = 8192)
 *   HB_OPT_DW_PAIR          1 = split-K dW GEMMs with 256-wide tiles run on CTA pairs
 *                           (tcgen05 cta_group::2; default 0, measured not faster)
 *   HB_OPT_PDL              1 = programmatic dependent launch between the step's kernels (default)
 *   HB_OPT_GRAPHS           1 = hogbatch_run replays one CUDA graph per (batch size, lr) (default)
 *   HB_OPT_INFLIGHT         steps a worker may have enqueued before the oldest completes in
 *                           hogbatch_run (1..4; 0 = auto: 2 for a single worker, else 1, R23)
 *   HB_OPT_STAGE_ROWS       rows per H2D staging chunk of a host dataset (0 = auto: chunks growing
 *                           from 4096 rows by doubling, each <= 32768 rows and <= 32 MB)
 *   HB_OPT_UPDATE           HB_UPDATE_HOGWILD (plain read-modify-write of the shared model, Hogwild
 *                           [L128, L170]; default) or HB_UPDATE_ATOMIC (the dW epilogue adds -lr*dW
 *                           with atomic adds: no concurrent update is lost)
 *   HB_OPT_STEP_KERNEL_MAX_B steps of at most this many rows (and below the fused chain's threshold)
 *                           run as ONE persistent launch: the step's 3L - 1 GEMMs as stages
 *                           separated by grid barriers (narrow nets: widths <= 1024, C <= 16,
 *                           L <= 8; plain workers); 0 = per-layer launches (default: measured
 *                           slower on B200 — 86 vs 58 us per C2 step at b = 32)
 *   HB_OPT_GEMM_PAIR        1 = forward, dX and unsplit dW GEMMs with >= 256 output columns, an
 *                           even number of 128-row tiles and >= 74 tile pairs (one wave) run as
 *                           persistent CTA pairs (tcgen05 cta_group::2, 256 x 256 tiles; default);
 *                           0 = one CTA per 128-row tile
 *   HB_OPT_HEAD_KERNEL      1 = the output layer of a net with C <= 8 classes (and at least one
 *                           hidden layer) runs on the per-layer path as ONE streaming CUDA-core pass
 *                           over H_{L-1} / sigma'_{L-1}: logits, softmax cross-entropy, dZ_{L-1}
 *                           (Eq. (2)) and dW_L / db_L from fp32 dZ_L, then a small reduction kernel
 *                           applies Eq. (3) to W_L, b_L (default); 0 = tensor-core head GEMM,
 *                           output-layer dX GEMM and dW GEMM (R24 split-precision dZ_L)
 * Unknown key or out-of-range value -> HB_EINVAL. */
enum {
  HB_OPT_FUSED_MIN_BATCH = 0, HB_OPT_ROWCHAIN = 1, HB_OPT_RC_CLUSTER = 2, HB_OPT_BWD_OVERLAP = 3,
  HB_OPT_HEAD_FUSE = 4, HB_OPT_DW_PAIR = 5, HB_OPT_PDL = 6, HB_OPT_GRAPHS = 7, HB_OPT_INFLIGHT = 8,
  HB_OPT_STAGE_ROWS = 9, HB_OPT_UPDATE = 10, HB_OPT_STEP_KERNEL_MAX_B = 11,
  HB_OPT_GEMM_PAIR = 12, HB_OPT_HEAD_KERNEL = 13
};
enum { HB_UPDATE_HOGWILD = 0, HB_UPDATE_ATOMIC = 1 };
int mlp_set_option(hb_model* m, int32_t key, int64_t value);
int mlp_get_option(const hb_model* m, int32_t key, int64_t* value);
/* host flat fp32 layout: [W_1 (n_1 x n_0 row-major, unpadded), b_1, W_2, b_2, ...]; n must equal
 * mlp_num_params.  Blocking.  set also refreshes the bf16 shadow. */
int mlp_get_params(const hb_model* m, float* host_dst, int64_t n);
int mlp_set_params(hb_model* m, const float* host_src, int64_t n);

/* ---- worker (§V.A: GPU worker, exclusive device interface) ----------
 * device: the model's device (or -1 for it; any other device -> HB_EUNSUPPORTED: one model per GPU,
 * several GPUs = one process per GPU sharing a coordinator, hb_coord_create).  max_batch >= 1 sizes
 * the worker's activation scratch.
 * replica 0 = reference replica: the worker updates the shared (global) model in place (Hogbatch
 *   [L170]; concurrent workers race, Hogwild [L128]).
 * replica 1 = deep replica [L134, L174]: the worker owns a private copy of the global model's
 *   parameters (taken at creation) and its steps update that copy; hb_merge_replicas (called by
 *   hogbatch_run at its merge points) integrates it into the global model ("push", [L141, L175]).
 *   Several deep replicas on one GPU emulate a multi-GPU replica run with the same merge arithmetic.
 * cuda_stream may be NULL (the worker creates its own stream — a BLOCKING stream, so its work is
 * ordered after the caller's legacy-default-stream work such as torch copies) or a borrowed
 * cudaStream_t.  Destroy workers before their model. */
int mlp_worker_create(hb_model* m, int32_t device, int32_t max_batch, int32_t replica, void* cuda_stream,
                      hb_worker** out);
/* the worker's current parameters (a deep replica's private copy; the global model's for a
 * reference replica) in the mlp_get_params layout (blocking) */
int mlp_worker_params(hb_worker* w, float* host_dst, int64_t n);
/* Nested worker: the GPU form of Algorithm 2's CPU worker [L224-L235].  Each ExecuteWork(B) is
 * split into t contiguous sub-batches (the first b mod t get ceil(b/t) rows) run concurrently on
 * t internal streams, each updating the shared model in place (Hogwild [L229-L232]) with
 * lr * size/b; credit it with incr = t*beta in hb_worker_policy [L234, L238].  t >= 1,
 * max_batch >= t.  In deterministic mode the sub-batches run in order. */
int mlp_worker_create_nested(hb_model* m, int32_t max_batch, int32_t t, void* cuda_stream, hb_worker** out);
int mlp_worker_destroy(hb_worker* w);
/* cudaStream_t of the worker (borrowed) */
void* mlp_worker_stream(hb_worker* w);

/* ---- one SGD step (Alg. 1 ExecuteWork lines 2–3, Eq. (1)–(3)) ----------------------
 * X: device pointer to the first row of the batch, [batch x ldx] of x_dtype (bf16 mode needs
 * HB_BF16 and (ldx*2) % 16 == 0 and X 16-byte aligned); y: device int32 [batch] labels in
 * [0, C) (out-of-range labels are undefined behaviour).  1 <= batch <= max_batch.
 * Enqueued asynchronously on the worker's stream; if loss_out != NULL the call blocks and
 * writes the batch-mean loss of the forward pass (before the update). */
int mlp_step(hb_worker* w, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y,
             int32_t batch, float lr, float* loss_out);
/* test-only: same forward/backward as mlp_step but no update; copies the gradients to
 * host_grads in the mlp_get_params flat layout (blocking). */
int mlp_step_grads(hb_worker* w, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y,
                   int32_t batch, float* host_grads, int64_t n, float* loss_out);
/* test-only: the per-example cross-entropy  -log softmax(z_i)[y_i]  [L258] of the first n rows of
 * the worker's last step (forward pass before the update), copied to host_dst[n] (blocking).
 * 1 <= n <= max_batch, plain workers only (HB_EUNSUPPORTED for nested workers). */
int mlp_row_losses(hb_worker* w, float* host_dst, int32_t n);

/* ---- epoch-end loss (L273: "The loss computation is always performed on the GPU") ---
 * mean cross-entropy over n examples, reduced deterministically in fp64.  Blocking. */
int mlp_loss(hb_model* m, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y,
             int64_t n, double* loss_out);

/* ---- coordinator (Algorithms 1 and 2) ------------------------------------------------
 * Runs the policy's coordinator on the deterministic virtual clock (hb_worker_policy c0/c1)
 * over N examples for `epochs` epochs, without touching any GPU; writes up to cap records. */
int hb_schedule_trace(const hb_policy* p, int64_t N, int32_t epochs, hb_trace_rec* out,
                      int64_t cap, int64_t* n_out);
/* ---- shared coordinator (multi-GPU: one process per GPU, one coordinator for the node) ----
 * PAPER.md L123 (one coordinator owns the data), L218–L220 (one set 𝔹 of remaining examples),
 * L130/L185 (the batch sizes adapt to the relative speed of ALL workers).  The Algorithm 2 state,
 * the epoch cursor over 𝔹 and the run control live in POSIX shared memory `name` ("/..."): rank 0
 * creates and initialises it from p (the global worker specs; N examples), the other ranks attach
 * (waiting up to 60 s for rank 0).  Pass it as hb_policy.coord (with first_worker = the global id of
 * the process's first worker) to hogbatch_run on every rank: the processes join each run before
 * any schedules, the epoch ends when every worker of every process is idle, and each process
 * performs every issued merge (its NCCL collective) in order.  Destroy after the last run
 * (rank 0 unlinks the segment).  A peer that stops responding surfaces as HB_ESTATE after 30 min. */
int hb_coord_create(const char* name, const hb_policy* p, int64_t N, int32_t nranks, int32_t rank, hb_coord** out);
int hb_coord_destroy(hb_coord* c);
/* test / custom-driver entry points on the shared state (no GPU, no run in progress):
 * reset to a fresh run of policy p over N examples; one ScheduleWork(worker) at time `now`; the
 * worker idles because it could not be served (*epoch_ended = 1 if every worker now idles: the
 * cursor returns to row 0 and the epoch advances, Alg. 1 [L170]) */
int hb_coord_reset(hb_coord* c, const hb_policy* p, int64_t N);
int hb_coord_schedule(hb_coord* c, int32_t worker, double now, hb_trace_rec* out);
int hb_coord_idle(hb_coord* c, int32_t worker, int32_t* epoch_ended);

/* Trains with n_workers workers (one host thread each, concurrent Hogbatch updates of the
 * shared model, L170) under policy p for `epochs` epochs over data (device or host, see
 * hb_dataset).  Blocking.  All workers belong to one global model (reference or deep replicas;
 * deep replicas need merges_per_epoch >= 1 and are merged with hb_merge_replicas, reference
 * workers of different processes with hb_merge over p->comm).
 * p->deterministic = 1 executes the virtual-clock trace serially (SERIAL policy, L125).
 * Stats arrays indexed by worker are indexed by the GLOBAL worker id (p->n_workers entries per
 * epoch); with a shared coordinator each process fills its own workers' entries and trace. */
int hogbatch_run(hb_worker** workers, int32_t n_workers, const hb_policy* p,
                 const hb_dataset* data, int32_t epochs, hb_stats* stats_out);

/* ---- instrumentation ----------------------------------------------------------------
 * hb_kernel_launches: number of CUDA kernels this library launched in this process.
 * hb_prof_enable(1): every kernel launch of the hot path is bracketed by CUDA events on its
 * own stream; hb_prof_read (blocking: synchronises the device) accumulates per class the
 * launch count, device milliseconds and the ALGORITHMIC flops / bytes of those launches
 * (DESIGN.md §Roofline), writes the first n of: HB_PROF_N class totals, then the per-layer entries
 * (n <= HB_PROF_N * (1 + HB_PROF_LAYERS)), and optionally resets. */
enum {
  HB_PROF_FWD_GEMM = 0,   /* hidden-layer forward GEMM + bias + sigmoid/sigma' epilogue */
  HB_PROF_HEAD_GEMM = 1,  /* output-layer forward GEMM (logits)                         */
  HB_PROF_SOFTMAX = 2,    /* softmax cross-entropy + dZ_L                               */
  HB_PROF_DGRAD_GEMM = 3, /* dX GEMM + sigma' epilogue                                  */
  HB_PROF_WGRAD_GEMM = 4, /* dW GEMM + fused in-place SGD epilogue                      */
  HB_PROF_BIAS = 5,       /* bias gradient + bias SGD                                   */
  HB_PROF_OTHER = 6,      /* loss reduction, shadow refresh, merge kernels              */
  HB_PROF_ROWCHAIN = 7,   /* fused per-row-block forward + softmax-xent + dX chain (narrow nets) */
  HB_PROF_STEPK = 8,      /* persistent small-batch step kernel (all GEMMs of a step in one launch) */
  HB_PROF_HEAD = 9,       /* small-C output layer in one CUDA-core pass: logits + softmax-CE + dX + dW partials */
  HB_PROF_N = 10,
  HB_PROF_LAYERS = 16     /* per-layer breakdown: entry HB_PROF_N + cls * HB_PROF_LAYERS + layer (0-based) */
};
typedef struct hb_prof_entry {
  int64_t launches;
  double ms, flops, bytes;
} hb_prof_entry;
int64_t hb_kernel_launches(void);
int hb_prof_enable(int32_t on);
int hb_prof_read(hb_prof_entry* out, int32_t n, int32_t reset);

/* Local replica merge (deep replicas of this process): with B the merge base
 * (hb_merge_begin / the previous merge), G <- G + gamma * sum_E (R_E - B) over the deep-replica
 * workers among workers[0..n) (fixed order; reference replicas contribute through G itself), then
 * B <- G and every replica R_E <- G (bf16 shadows rewritten).  Blocking; at most 8 deep replicas. */
int hb_merge_replicas(hb_model* m, hb_worker* const* workers, int32_t n, float gamma);

/* Merge points of one epoch of served batch sizes batches[0..n) over N examples:
 * mid_epoch_out = merges due while serving, total_out = merges performed in the epoch (always
 * merges_per_epoch: the rest is issued at the epoch end). */
int hb_merge_schedule(int64_t N, int32_t merges_per_epoch, const int32_t* batches, int64_t n_batches,
                      int32_t* mid_epoch_out, int32_t* total_out);

/* ---- asynchronous cross-replica Hogbatch (NEXT f2; "reference replicas",
 * L175 "the learning rate can be decreased" for stale replicas) ---------------------------
 * After mlp_attach_peers / mlp_attach_ipc_peers, every SGD update this model applies (the dW
 * epilogue's W -= lr * dW and the bias update) is ALSO added, scaled by `scale` (stale-gradient
 * damping, 0 <= scale; 1 = none), to each peer replica's fp32 master with an atomic add —
 * peer-to-peer over NVLink, no round barrier — and the peer's bf16 shadow element is rewritten
 * from the value that add produced.  Peers are models of identical shape: in this process
 * (mlp_attach_peers: another model on this GPU, or on a peer-accessible GPU) or in another
 * process (mlp_ipc_handle exports a model's 128-byte handle pair; mlp_attach_ipc_peers maps up to
 * 7 of them).  Updates made while the peers are detached are not propagated; n = 0 detaches.
 * bf16 models only.  Concurrent updates of one replica race as in Hogwild [L128, L170]; under
 * HB_UPDATE_ATOMIC only the shadow refresh is racy.  (NVLink multicast — one multimem.red per
 * update for all replicas — is the intended transport; it needs a multicast domain, which the
 * development pool's one-GPU leases do not have.) */
int mlp_attach_peers(hb_model* m, hb_model* const* peers, int32_t n, float scale);
int mlp_ipc_handle(const hb_model* m, uint8_t out[128]);
int mlp_attach_ipc_peers(hb_model* m, const uint8_t* handles, int32_t n, float scale);

/* ---- multi-GPU replica merge over NCCL (future work L277) -------- */
int hb_nccl_unique_id(uint8_t out[128]);
int hb_comm_create(const uint8_t id[128], int32_t nranks, int32_t rank, int32_t device,
                   hb_comm** out);
int hb_comm_destroy(hb_comm* c);
/* snapshot the current model as the merge base W_base (call when all ranks agree) */
int hb_merge_begin(hb_model* m);
/* W <- W_base + gamma * allreduce_sum(W - W_base); W_base <- W; bf16 shadow refreshed.
 * Collective: every rank must call it.  stream may be NULL (model's internal stream).
 * Blocking. */
int hb_merge(hb_model* m, hb_comm* c, float gamma, void* cuda_stream);

#ifdef __cplusplus
}
#endif
#endif /* HOGBATCH_H */
