// model.h — internal definitions of hb_model / hb_worker (not part of the ABI).
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <map>
#include <tuple>
#include <mutex>
#include <vector>

#include "../../include/hogbatch.h"

namespace hb {

// graph replays of one worker that may be enqueued before the oldest completes (hogbatch_run)
constexpr int HB_MAX_INFLIGHT = 4;

// One fully-connected layer W_l [n_out x n_in] (row stride ldw, padded to 8 elements so every
// bf16 row is 16-byte aligned for TMA) and bias b_l [n_out]; offsets index the flat parameter
// buffers (fp32 master, bf16 shadow share the indexing).
struct Layer {
  int n_in = 0, n_out = 0;
  int ldw = 0;  // row stride of W (elements)
  int ldo = 0;  // row stride of this layer's activations / gradients (elements)
  size_t w_off = 0, b_off = 0;
};

int choose_bn(int M, int N, int K = 0);

extern thread_local int g_prof_layer;
// Tags the Prof records of the launches issued while it lives with weight layer l (0-based).
struct ProfLayer {
  int prev;
  explicit ProfLayer(int l) : prev(g_prof_layer) { g_prof_layer = l; }
  ~ProfLayer() { g_prof_layer = prev; }
};

// Brackets the kernel launches of one hot-path operation: counts launches and, when profiling
// is enabled (hb_prof_enable), records CUDA events on the launch stream.
struct Prof {
  int cls;
  cudaStream_t s;
  int layer;
  cudaEvent_t e0 = nullptr;
  Prof(int cls, cudaStream_t s);
  void done(int nlaunch, double flops, double bytes);
};

}  // namespace hb

struct hb_model {
  int device = 0;
  int prec = HB_PREC_BF16;
  std::vector<int> dims;
  // per-model settings (mlp_set_option, HB_OPT_*); defaults are the measured B200 choices
  int rc_min_b = 4096;              // HB_OPT_FUSED_MIN_BATCH: fused row-block step from this b up (0 = never)
  int opt_rowchain = 1;             // HB_OPT_ROWCHAIN
  int opt_rc_cluster = 0;           // HB_OPT_RC_CLUSTER: CTAs per row block of the fused chain (0 = auto)
  int opt_bwd_overlap = 1;          // HB_OPT_BWD_OVERLAP: dW_l on a second stream, overlapping dX_{l-1}
  int opt_head_fuse = 0;            // HB_OPT_HEAD_FUSE: output layer's dX in the head epilogue
  int opt_dw_pair = 0;              // HB_OPT_DW_PAIR: split-K dW GEMMs on CTA pairs (cta_group::2)
  int opt_gemm_pair = 1;            // HB_OPT_GEMM_PAIR: forward / dX / unsplit dW GEMMs on persistent CTA pairs
  int opt_head_kernel = 1;          // HB_OPT_HEAD_KERNEL: small-C output layer as one CUDA-core pass (head.cuh)
  int opt_pdl = 1;                  // HB_OPT_PDL: programmatic dependent launch
  int opt_graphs = 1;               // HB_OPT_GRAPHS: hogbatch_run replays one CUDA graph per (b, lr)
  int opt_inflight = 0;             // HB_OPT_INFLIGHT: steps a worker may enqueue ahead (0 = auto)
  int64_t opt_stage_rows = 0;       // HB_OPT_STAGE_ROWS: host-dataset staging chunk rows (0 = auto)
  int opt_update = 0;               // HB_OPT_UPDATE: HB_UPDATE_HOGWILD or HB_UPDATE_ATOMIC
  int opt_step_kernel_max_b = 0;    // HB_OPT_STEP_KERNEL_MAX_B: persistent one-launch step up to this b
                                    // (off by default: measured slower than the per-layer launches)
  std::vector<hb::Layer> layers;
  size_t total = 0;                 // floats in the flat parameter buffer (incl. padding)
  float* master = nullptr;          // fp32 master weights + biases (the shared global model)
  __nv_bfloat16* shadow = nullptr;  // bf16 copy read by the tensor cores
  float* base = nullptr;            // merge base W_base (hb_merge_begin)
  float* delta = nullptr;           // merge send/recv buffer
  cudaStream_t stream = nullptr;    // internal stream (loss evaluation, merges)
  hb_worker* eval = nullptr;        // scratch for mlp_loss
  std::mutex eval_mu;
  double* chunk_sums = nullptr;
  int64_t chunk_cap = 0;
  // hogbatch_run over a HOST dataset: device staging copy (reused across calls), the copy
  // stream and one event per staged chunk of rows
  void* stage_x = nullptr;
  size_t stage_x_cap = 0;
  // stage_x holds exactly the densification (zeros elsewhere) of the host CSR dataset whose
  // structure is still in csr_ptr / csr_idx: the next CSR staging of the same shape zeroes only
  // those nonzeros instead of the whole dense buffer
  struct {
    bool valid = false;
    int64_t n = 0, ldx = 0, n_cols = 0;
    int xdt = 0;
  } csr_dense;
  int32_t* stage_y = nullptr;
  size_t stage_y_cap = 0;
  cudaStream_t copy_stream = nullptr;
  std::vector<cudaEvent_t> stage_ev;
  // asynchronous cross-replica updates (NEXT f2): peer replicas' fp32 master / bf16 shadow
  // (identical layout) that every update of this model is also added to, scaled by peer_scale
  std::vector<std::pair<float*, __nv_bfloat16*>> peers;
  std::vector<void*> ipc_opened;  // cudaIpcOpenMemHandle mappings to close
  float peer_scale = 1.f;
  // CSR datasets: device copies of the sparse arrays (reused across calls)
  int64_t* csr_ptr = nullptr;
  int32_t* csr_idx = nullptr;
  void* csr_val = nullptr;
  size_t csr_ptr_cap = 0, csr_nnz_cap = 0;
};

struct hb_worker {
  hb_model* m = nullptr;        // the model this worker's steps update: the global model (reference
                                // replica) or, for a deep replica, the worker's private copy
  hb_model* global = nullptr;   // the global model the worker belongs to (== m for reference replicas)
  int max_b = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  std::vector<void*> H, S, dZ;  // per-layer activations, sigma' stash, output gradients
  int ld_dzL = 0;               // row stride of dZ_L (32 with the split-precision head, R24)
  unsigned* sk_bar = nullptr;   // persistent small-batch step: stage arrival counters + generation
  int sk_grid = 0;              // its fixed grid size
  bool hilo = false;            // dZ_L stored as bf16 hi / lo planes (C <= 16, bf16 model)
  float* logits = nullptr;      // [max_b x ldc] fp32
  int ldc = 0;
  float* row_loss = nullptr;    // [max_b]
  std::vector<float*> bpart;    // per layer [ceil(max_b/128) x n_out] bias-gradient partial sums
  int* d_off = nullptr;         // device row offset of the current batch (graph replay)
  int* h_off = nullptr;         // pinned host sources of d_off, one per in-flight slot
  int slot = 0;                 // next slot (graph replays of a worker may be queued HB_MAX_INFLIGHT deep)
  // CUDA graphs of one SGD step, per (batch size, lr), for the dataset they were captured on
  struct Graph {
    cudaGraphExec_t exec = nullptr;
    int launches = 0;
  };
  std::map<std::tuple<int, uint32_t, int, const double*>, Graph> graphs;  // (b, lr bits, slot, loss accumulator)
  const void* g_X = nullptr;
  const void* g_y = nullptr;
  int64_t g_ldx = 0, g_rows = 0;
  double* dsum = nullptr;
  double* h_dsum = nullptr;     // pinned
  float* grads = nullptr;       // mlp_step_grads output (flat padded layout)
  float* ws = nullptr;          // split-K partial tiles of the dW GEMMs (148 x 128 x 256 fp32)
  float* hws = nullptr;         // head kernel: per-CTA partial dW_L [grid x C x n] and db_L [grid x C]
  cudaStream_t s2 = nullptr;    // dW GEMMs overlap the next dX GEMM on this stream
  std::vector<cudaEvent_t> ev_bwd;  // per layer: "dX_l issued" (W_l no longer read)
  cudaEvent_t ev_join2 = nullptr;
  // fused row-block path (rowchain.cuh): the dW GEMMs of all layers run concurrently after the
  // chain kernel, one stream and one split-K workspace per layer
  std::vector<cudaStream_t> sdw;
  std::vector<cudaEvent_t> ev_dw;
  cudaEvent_t ev_chain = nullptr;
  std::vector<float*> ws_l;
  // nested worker (Alg. 2 "CPU worker", L224-L235): t sub-workers run the sub-batches of one
  // ExecuteWork concurrently, each updating the shared model in place
  std::vector<hb_worker*> subs;
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;
};

namespace hb {
int clone_model(hb_model* m, hb_model** out);
// zero rows [r0, r1) of the dense X [.. x ldx] (dtype xdt) and scatter the CSR rows into them on s;
// *bad (device int) is set if a column index is outside [0, n_cols)
int densify_csr_rows(const int64_t* indptr, const int32_t* indices, const void* vals, int xdt, int64_t r0, int64_t r1,
                     int64_t n_cols, void* X, int64_t ldx, cudaStream_t s, int* bad, bool zero_first = true);
// One SGD step.  X / y: the batch's first row, or (d_off != nullptr, tensor-core path) the
// dataset base with the batch's first row read from *d_off on the device.  x_rows = rows of X.
int run_step(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, int64_t x_rows, const int32_t* y,
             const int* d_off, int b, float lr, bool grads_only, cudaStream_t s);
// One SGD step replayed from a CUDA graph captured for (b, lr) on the dataset (X, y): the
// batch's row offset is copied from pinned host memory by the graph's first node.
int step_graph(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, int64_t off, int b,
               float lr, double* loss_acc = nullptr);
void clear_graphs(hb_worker* w);
// One ExecuteWork(B) of a worker on rows [off, off + b) of the dataset (X, y with x_rows rows):
// a plain worker runs one SGD step; a nested worker splits B into its t sub-batches (the first
// b mod t get ceil(b/t) rows, R6) with lr scaled to each sub-batch (lr * size / b),
// concurrently on the sub-workers' streams (serial = in order on w->stream, deterministic).
// If loss_dst != nullptr the summed per-row losses of the batch are written to (accumulate: added
// to) *loss_dst (device).
int worker_execute(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, int64_t x_rows, const int32_t* y,
                   int64_t off, int b, float lr, bool graphs, bool serial, double* loss_dst, bool accumulate = false);
bool prof_enabled();
int finish_loss(hb_worker* w, int b, float* loss_out, cudaStream_t s);
// enqueue sum of the last step's per-row losses into *dst (device double)
void sum_rows_into(hb_worker* w, int b, double* dst, cudaStream_t s, bool accumulate = false);
}  // namespace hb
