// model.cu — C ABI of the MLP-SGD hot path: model and worker objects, one SGD step
// (forward GEMM chain, softmax-xent head, dX/dW GEMMs, fused in-place SGD), epilogue-free loss
// evaluation, parameter I/O and the NCCL replica merge.
//
// Paper: Ma, Rusu, Wu, Sim (IPDPSW/MARWS 2021), §III (Eq. (1)–(3),
// L41–L56), §V.A (workers, L132–L134), §VI (Hogbatch, L147–L170), §VII.A (sigmoid hidden layers,
// softmax cross-entropy, L258).
#include <cudaTypedefs.h>

#include <atomic>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <random>
#include <set>
#include <string>
#include <vector>

#include "kernels.cuh"
#include "model.h"
#include "tc_gemm.cuh"
#include "rowchain.cuh"
#include "step_kernel.cuh"
#include "head.cuh"

namespace hb {

// ----------------------------------------------------------------------------------------
// errors
// ----------------------------------------------------------------------------------------
static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }
int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

// ----------------------------------------------------------------------------------------
// instrumentation: launch counter + optional per-launch CUDA-event timing per kernel class
// ----------------------------------------------------------------------------------------
std::atomic<int64_t> g_launches{0};
static std::atomic<bool> g_prof_on{false};
struct PendRec {
  cudaEvent_t e0, e1;
  int cls;
  double flops, bytes;
  int nl;
  int layer;
};
thread_local int g_prof_layer = -1;  // layer of the launches being bracketed (ProfLayer), -1 = none
static std::mutex g_prof_mu;
static std::vector<PendRec> g_pend;
static std::vector<cudaEvent_t> g_evpool;
static hb_prof_entry g_agg[HB_PROF_N];
static hb_prof_entry g_agg_l[HB_PROF_N][HB_PROF_LAYERS];

static cudaEvent_t ev_get() {
  {
    std::lock_guard<std::mutex> g(g_prof_mu);
    if (!g_evpool.empty()) {
      cudaEvent_t e = g_evpool.back();
      g_evpool.pop_back();
      return e;
    }
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

bool prof_enabled() { return g_prof_on.load(); }

Prof::Prof(int cls_, cudaStream_t s_) : cls(cls_), s(s_), layer(g_prof_layer) {
  if (g_prof_on.load(std::memory_order_relaxed)) {
    e0 = ev_get();
    cudaEventRecord(e0, s);
  }
}

void Prof::done(int nlaunch, double flops, double bytes) {
  g_launches.fetch_add(nlaunch, std::memory_order_relaxed);
  if (!e0) return;
  cudaEvent_t e1 = ev_get();
  cudaEventRecord(e1, s);
  std::lock_guard<std::mutex> g(g_prof_mu);
  g_pend.push_back({e0, e1, cls, flops, bytes, nlaunch, layer});
  e0 = nullptr;
}

// ----------------------------------------------------------------------------------------
// TMA tensor maps (driver entry point; no link-time dependency on libcuda)
// ----------------------------------------------------------------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

static int ensure_encode() {
  static std::once_flag once;
  static cudaError_t err = cudaSuccess;
  std::call_once(once, [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    err = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (err == cudaSuccess && q == cudaDriverEntryPointSuccess)
      g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  });
  if (!g_encode) return fail(HB_ECUDA, std::string("cuTensorMapEncodeTiled unavailable: ") + cudaGetErrorString(err));
  return HB_OK;
}

// bf16 2-D map: dims {inner, outer}, row stride in bytes, box {box_inner, box_outer}, 128B swizzle,
// out-of-bounds elements read as zero (this is how ragged M/N/K tails are handled).
static int make_map(CUtensorMap* out, const void* base, uint64_t inner, uint64_t outer,
                    uint64_t stride_bytes, uint32_t box_inner, uint32_t box_outer) {
  int rc = ensure_encode();
  if (rc) return rc;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {stride_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = g_encode(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides,
                        box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    return fail(HB_ECUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ") inner=" +
                              std::to_string(inner) + " outer=" + std::to_string(outer) +
                              " stride=" + std::to_string(stride_bytes));
  return HB_OK;
}

// ----------------------------------------------------------------------------------------
// GEMM dispatch
// ----------------------------------------------------------------------------------------
static std::mutex g_attr_mu;
static std::set<std::pair<const void*, int>> g_attr_done;

// bf16 output map for the TMA-store epilogue: [rows x cols] row stride ld elements, box 64 x 128
static int make_out_map(CUtensorMap* out, const void* base, int64_t cols, int64_t rows, int64_t ld) {
  return make_map(out, base, cols, rows, ld * 2, 64, TC_BM);
}

template <int BN, bool A_MN, bool B_MN, int EPI, bool PAIR = false>
static int launch_tc(const CUtensorMap& ma, const CUtensorMap& mb, int M, int N, int K, const int* offA,
                     const int* offB, const EpiArgs& ep, cudaStream_t s, int splits = 1) {
  using Cfg = TcCfg<BN, B_MN, EPI, PAIR>;
  CUtensorMap mo0 = ma, mo1 = ma;  // unused unless the epilogue stages its outputs for TMA stores
  if (TmaOut<BN, EPI, PAIR>::on) {
    int rc = make_out_map(&mo0, ep.out0, N, M, ep.ld0 > 0 ? ep.ld0 : round_up(N, 8));
    if (!rc && EPI == EPI_FWD_SIG && ep.out1) rc = make_out_map(&mo1, ep.out1, N, M, ep.ld1);
    if (rc) return rc;
  }
  auto kern = tc_gemm_kernel<BN, A_MN, B_MN, EPI, PAIR>;
  int dev = 0;
  cudaGetDevice(&dev);
  {
    std::lock_guard<std::mutex> g(g_attr_mu);
    auto key = std::make_pair((const void*)kern, dev);
    if (!g_attr_done.count(key)) {
      HB_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM_BYTES));
      g_attr_done.insert(key);
    }
  }
  // persistent: one CTA per SM (at most one per tile) walking the tiles; split-K: one CTA per
  // (tile, split) with the splits of a tile in one cluster
  const int tiles = ((N + BN - 1) / BN) * ((M + TC_BM - 1) / TC_BM);
  static int nsm = 0;
  if (!nsm) {
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm <= 0) nsm = 148;
  }
  const int pair_tiles = ((N + BN - 1) / BN) * ((M + 2 * TC_BM - 1) / (2 * TC_BM));
  dim3 grid = splits == 1 ? (PAIR ? dim3(2 * std::min(pair_tiles, nsm / 2), 1, 1) : dim3(std::min(tiles, nsm), 1, 1))
              : PAIR      ? dim3((M + TC_BM - 1) / TC_BM, (N + BN - 1) / BN, splits)
                          : dim3((N + BN - 1) / BN, (M + TC_BM - 1) / TC_BM, splits);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = dim3(TC_THREADS);
  cfg.dynamicSmemBytes = Cfg::SMEM_BYTES;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (!ep.no_pdl) {  // programmatic dependent launch: prologue overlaps the previous kernel's tail
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  if (splits > 1 || PAIR) {  // the splits of a tile and / or the two M tiles of a CTA pair form a cluster
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = PAIR ? 2 : 1;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = splits;
    ++na;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  HB_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, ma, mb, mo0, mo1, K, offA, offB, ep));
  HB_CUDA_TRY(cudaGetLastError());
  return HB_OK;
}

template <bool A_MN, bool B_MN, int EPI>
static int launch_tc_bn(int bn, const CUtensorMap& ma, const CUtensorMap& mb, int M, int N, int K,
                        const int* offA, const int* offB, const EpiArgs& ep, cudaStream_t s, int splits = 1) {
  switch (bn) {
    case 16: return launch_tc<16, A_MN, B_MN, EPI>(ma, mb, M, N, K, offA, offB, ep, s, splits);
    case 32: return launch_tc<32, A_MN, B_MN, EPI>(ma, mb, M, N, K, offA, offB, ep, s, splits);
    case 64: return launch_tc<64, A_MN, B_MN, EPI>(ma, mb, M, N, K, offA, offB, ep, s, splits);
    case 128: return launch_tc<128, A_MN, B_MN, EPI>(ma, mb, M, N, K, offA, offB, ep, s, splits);
    default: return launch_tc<256, A_MN, B_MN, EPI>(ma, mb, M, N, K, offA, offB, ep, s, splits);
  }
}

// split-K factor of a dW GEMM (K = batch): enough CTAs to cover the 148 SMs, power of two
// <= 8 (portable cluster size), at least one k-block per split
static int choose_bn_base(int M, int N);

// Launch-choice overrides from the environment exist only in the tuning build (-DHB_TUNING);
// the product library uses the measured defaults and the per-model options (mlp_set_option).
#ifdef HB_TUNING
static int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return v && *v ? atoi(v) : dflt;
}
#define HB_TUNE(name, dflt) env_int(name, dflt)
#else
#define HB_TUNE(name, dflt) (dflt)
#endif

int choose_splits(int M, int N, int K, int bn) {
  static const int max_s = HB_TUNE("HB_MAX_SPLITS", 4);  // 8-CTA clusters of 200 KB CTAs do not all co-reside
  const long tiles = (long)((M + TC_BM - 1) / TC_BM) * ((N + bn - 1) / bn);
  const int nkb = (K + TC_BK - 1) / TC_BK;
  int S = 1;
  while (S * 2 <= max_s && tiles * S * 2 <= 148 && S * 2 <= nkb) S *= 2;
  if (S == 4 && tiles * 8 <= 64 && 8 <= nkb) S = 8;  // a few 8-CTA clusters still co-reside
  return S;
}

// tile width of a dW GEMM: narrow enough that tiles x splits fill the SMs
static int choose_bn_wgrad(int M, int N, int K) {
  static const int forced = HB_TUNE("HB_WGRAD_BN", 0);
  if (forced) return forced;
  if (K < 2048) return choose_bn(M, N, K);  // short K: no split-K, spread tiles over the SMs
  int bn = choose_bn_base(M, N);          // long K: split-K supplies the parallelism
  const long mt = (M + TC_BM - 1) / TC_BM;
  // 256-wide tiles x 4 splits filling >= 96 SMs beat narrower tiles on more SMs (operand bytes per
  // MMA through shared memory; measured on B200, 1024 x 1024 x 8192 dW: BN 256 x 4 splits 21.6 us,
  // BN 128 x 2 splits 26.5 us, BN 64 x 1 38.7 us — scripts/gpu_dw_sweep.sh)
  if (N >= 256 && mt * ((N + 255) / 256) * 4 >= 96) return 256;
  while (bn > 64 && mt * ((N + bn - 1) / bn) * 4 < 148) bn /= 2;
  return bn;
}

static int choose_bn_base(int M, int N) {
  if (N <= 16) return 16;
  if (N <= 32) return 32;
  if (N <= 64) return 64;
  if (N <= 128) return 128;
  const long mt = (M + TC_BM - 1) / TC_BM;
  if (mt * ((N + 255) / 256) >= 148) return 256;
  return 128;
}

// Tile width: the base rule, narrowed while the grid would leave most SMs idle (small batches:
// M = b <= a few hundred rows gives 1-2 row tiles; narrower tiles spread the epilogue)
int choose_bn(int M, int N, int K) {
  static const int forced = HB_TUNE("HB_FWD_BN", 0);  // tuning only: forward / dX tile width
  if (forced && N > 16) return forced;
  int bn = choose_bn_base(M, N);
  const long mt = (M + TC_BM - 1) / TC_BM;
  // fewer than ~4 waves of 256-wide tiles and a short K: 128-wide tiles balance the persistent
  // CTAs better (measured on B200: C3 8192 x 1024 x 1024 layers 30.8 vs 28.9 M samples/s); long-K
  // tiles keep 256 (width 4096-8192 at b = 2048, K = 4096: 55 vs 49% of peak with 256)
  if (bn == 256 && K > 0 && K <= 2048 && mt * ((N + 255) / 256) < 4 * 148) bn = 128;
  while (bn > 32 && mt * ((N + bn - 1) / bn) < 64) bn /= 2;
  return bn;
}

// GEMMs on persistent CTA pairs (HB_OPT_GEMM_PAIR): 256 x 256 tiles, an even number of 128-row
// tiles (no pair half entirely outside M) and at least a full wave of pair tiles (74 pairs on 148
// SMs; measured on B200: 8192 x 512 x 512 with 64 pair tiles 13.2 vs 10.3 us for one-CTA tiles,
// 8192 x 1024 x 1024 with 128 pair tiles 24.7 vs 26.4 us, C4 layers 15-29 % faster)
static bool pair_shape_ok(int M, int N) {
  const int mt = (M + TC_BM - 1) / TC_BM;
  return N >= 256 && mt % 2 == 0 && (long)(mt / 2) * ((N + 255) / 256) >= 74;
}
static bool fwd_pair_ok(int epi, bool a_mn, int M, int N, const EpiArgs& ep) {
  return ep.fwd_pair && !a_mn && (epi == EPI_FWD_SIG || epi == EPI_DGRAD_SIG) && pair_shape_ok(M, N);
}

// One tcgen05 GEMM launch.  A is [M x K] (K-major) or stored [K x M] (MN-major); B is [N x K]
// (K-major) or stored [K x N] (MN-major).  a_rows / b_rows = number of stored rows covered by
// the tensor map (0: exactly the GEMM extent); offA / offB = device row offsets (nullable).
struct TcOp {
  const void* p;
  int64_t ld;
  int64_t rows;
  const int* off;
};

static int gemm_tc(int epi, bool a_mn, bool b_mn, int M, int N, int K, TcOp A, TcOp B, const EpiArgs& ep,
                   cudaStream_t s) {
  const int bn = epi == EPI_HEAD_XENT                          ? 16
                 : (epi == EPI_WGRAD_SGD || epi == EPI_WGRAD_STORE) ? (ep.force_bn ? ep.force_bn : choose_bn_wgrad(M, N, K))
                                                                    : choose_bn(M, N, K);
  CUtensorMap ma, mb;
  const int64_t ar = A.rows ? A.rows : (a_mn ? K : M);
  const int64_t br = B.rows ? B.rows : (b_mn ? K : N);
  int rc = a_mn ? make_map(&ma, A.p, M, ar, A.ld * 2, 64, 64) : make_map(&ma, A.p, K, ar, A.ld * 2, 64, TC_BM);
  if (rc) return rc;
  // persistent CTA-pair forward / dX GEMM (256 x 256 tiles, each CTA loads 128 rows of B)
  const bool fpair = fwd_pair_ok(epi, a_mn, M, N, ep);
  rc = b_mn ? make_map(&mb, B.p, N, br, B.ld * 2, 64, 64) : make_map(&mb, B.p, K, br, B.ld * 2, 64, fpair ? 128 : bn);
  if (rc) return rc;
  if (fpair) {
    if (epi == EPI_FWD_SIG) return launch_tc<256, false, false, EPI_FWD_SIG, true>(ma, mb, M, N, K, A.off, B.off, ep, s);
    if (epi == EPI_DGRAD_SIG) return launch_tc<256, false, true, EPI_DGRAD_SIG, true>(ma, mb, M, N, K, A.off, B.off, ep, s);
  }
  if (!a_mn && !b_mn) {
    if (epi == EPI_FWD_SIG) return launch_tc_bn<false, false, EPI_FWD_SIG>(bn, ma, mb, M, N, K, A.off, B.off, ep, s);
    if (epi == EPI_FWD_LOGITS)
      return launch_tc_bn<false, false, EPI_FWD_LOGITS>(bn, ma, mb, M, N, K, A.off, B.off, ep, s);
    if (epi == EPI_HEAD_XENT) return launch_tc<16, false, false, EPI_HEAD_XENT>(ma, mb, M, N, K, A.off, B.off, ep, s);
  } else if (!a_mn && b_mn) {
    if (epi == EPI_DGRAD_SIG) return launch_tc_bn<false, true, EPI_DGRAD_SIG>(bn, ma, mb, M, N, K, A.off, B.off, ep, s);
  } else if (a_mn && b_mn) {
    const int S = !ep.ws ? 1 : ep.force_splits ? ep.force_splits : choose_splits(M, N, K, bn);
    // unsplit dW GEMMs with 256-wide tiles (C4) on persistent CTA pairs as well
    if (S == 1 && ep.fwd_pair && bn == 256 && pair_shape_ok(M, N)) {
      if (epi == EPI_WGRAD_SGD) return launch_tc<256, true, true, EPI_WGRAD_SGD, true>(ma, mb, M, N, K, A.off, B.off, ep, s);
      if (epi == EPI_WGRAD_STORE) return launch_tc<256, true, true, EPI_WGRAD_STORE, true>(ma, mb, M, N, K, A.off, B.off, ep, s);
    }
    // CTA pairs (256-row tiles over two SMs sharing the B tile): BN 256, >= 2 splits, even M tiles
    if (ep.pair && bn == 256 && S >= 2 && S <= 4 && ((M + TC_BM - 1) / TC_BM) % 2 == 0) {
      if (epi == EPI_WGRAD_SGD) return launch_tc<256, true, true, EPI_WGRAD_SGD, true>(ma, mb, M, N, K, A.off, B.off, ep, s, S);
      if (epi == EPI_WGRAD_STORE)
        return launch_tc<256, true, true, EPI_WGRAD_STORE, true>(ma, mb, M, N, K, A.off, B.off, ep, s, S);
    }
    if (epi == EPI_WGRAD_SGD)
      return launch_tc_bn<true, true, EPI_WGRAD_SGD>(bn, ma, mb, M, N, K, A.off, B.off, ep, s, S);
    if (epi == EPI_WGRAD_STORE)
      return launch_tc_bn<true, true, EPI_WGRAD_STORE>(bn, ma, mb, M, N, K, A.off, B.off, ep, s, S);
  }
  return fail(HB_EUNSUPPORTED, "gemm_tc: unsupported epilogue/major combination");
}

template <int EPI, typename TA, typename TB>
static int launch_simt_t(const void* A, int64_t sam, int64_t sak, const void* B, int64_t sbn, int64_t sbk,
                         int M, int N, int K, const EpiArgs& ep, cudaStream_t s) {
  dim3 grid((N + 63) / 64, (M + 63) / 64);
  simt_gemm_kernel<EPI, TA, TB><<<grid, 256, 0, s>>>(static_cast<const TA*>(A), sam, sak,
                                                     static_cast<const TB*>(B), sbn, sbk, M, N, K, ep);
  HB_CUDA_TRY(cudaGetLastError());
  return HB_OK;
}

template <int EPI>
static int launch_simt(const void* A, int adt, int64_t sam, int64_t sak, const void* B, int bdt, int64_t sbn,
                       int64_t sbk, int M, int N, int K, const EpiArgs& ep, cudaStream_t s) {
  if (adt == HB_F32 && bdt == HB_F32) return launch_simt_t<EPI, float, float>(A, sam, sak, B, sbn, sbk, M, N, K, ep, s);
  if (adt == HB_BF16 && bdt == HB_F32)
    return launch_simt_t<EPI, __nv_bfloat16, float>(A, sam, sak, B, sbn, sbk, M, N, K, ep, s);
  if (adt == HB_F32 && bdt == HB_BF16)
    return launch_simt_t<EPI, float, __nv_bfloat16>(A, sam, sak, B, sbn, sbk, M, N, K, ep, s);
  return launch_simt_t<EPI, __nv_bfloat16, __nv_bfloat16>(A, sam, sak, B, sbn, sbk, M, N, K, ep, s);
}

// fp32 check-mode GEMM with the same operand conventions as gemm_tc
static int gemm_simt(int epi, bool a_mn, bool b_mn, int M, int N, int K, const void* A, int64_t lda, int adt,
                     const void* B, int64_t ldb, int bdt, const EpiArgs& ep, cudaStream_t s) {
  const int64_t sam = a_mn ? 1 : lda, sak = a_mn ? lda : 1;
  const int64_t sbn = b_mn ? 1 : ldb, sbk = b_mn ? ldb : 1;
  switch (epi) {
    case EPI_FWD_SIG: return launch_simt<EPI_FWD_SIG>(A, adt, sam, sak, B, bdt, sbn, sbk, M, N, K, ep, s);
    case EPI_FWD_LOGITS: return launch_simt<EPI_FWD_LOGITS>(A, adt, sam, sak, B, bdt, sbn, sbk, M, N, K, ep, s);
    case EPI_DGRAD_SIG: return launch_simt<EPI_DGRAD_SIG>(A, adt, sam, sak, B, bdt, sbn, sbk, M, N, K, ep, s);
    case EPI_WGRAD_SGD: return launch_simt<EPI_WGRAD_SGD>(A, adt, sam, sak, B, bdt, sbn, sbk, M, N, K, ep, s);
    default: return launch_simt<EPI_WGRAD_STORE>(A, adt, sam, sak, B, bdt, sbn, sbk, M, N, K, ep, s);
  }
}

// algorithmic bytes of one GEMM launch (operands once, epilogue reads/writes once)
static double gemm_bytes(int epi, int M, int N, int K, double es, bool shadow) {
  const double mn = (double)M * N, io = ((double)M * K + (double)N * K) * es;
  switch (epi) {
    case EPI_FWD_SIG: return io + 2.0 * mn * es + 4.0 * N;
    case EPI_FWD_LOGITS: return io + 4.0 * mn + 4.0 * N;
    case EPI_HEAD_XENT: return io + mn * es + 8.0 * M + 4.0 * N;
    case EPI_DGRAD_SIG: return io + 2.0 * mn * es;
    case EPI_WGRAD_SGD: return io + 8.0 * mn + (shadow ? 2.0 * mn : 0.0);
    default: return io + 4.0 * mn;
  }
}

static int prof_class(int epi) {
  return epi == EPI_FWD_SIG ? HB_PROF_FWD_GEMM
         : (epi == EPI_FWD_LOGITS || epi == EPI_HEAD_XENT) ? HB_PROF_HEAD_GEMM
         : epi == EPI_DGRAD_SIG ? HB_PROF_DGRAD_GEMM
                                : HB_PROF_WGRAD_GEMM;
}

// Planning mode of the persistent small-batch step (step_kernel.cuh): while g_plan is set, the
// step's GEMMs are RECORDED (arguments + the layer they belong to) instead of launched, so the
// persistent kernel runs exactly the GEMMs, operands and fused epilogues of the per-layer path.
struct SkPlanEntry {
  int epi;
  bool a_mn, b_mn;
  int M, N, K;
  TcOp A, B;
  EpiArgs ep;
  int layer;
};
static thread_local std::vector<SkPlanEntry>* g_plan = nullptr;
// Set while a step graph is captured with a training-loss accumulator: the step adds the sum of its
// row losses into *g_loss_acc on a side stream (off the step's critical path, before its join)
static thread_local double* g_loss_acc = nullptr;

static int gemm_tc_p(int epi, bool a_mn, bool b_mn, int M, int N, int K, TcOp A, TcOp B, const EpiArgs& ep,
                     cudaStream_t s) {
  if (M <= 0 || N <= 0 || K <= 0) return HB_OK;
  if (g_plan) {
    g_plan->push_back(SkPlanEntry{epi, a_mn, b_mn, M, N, K, A, B, ep, g_prof_layer});
    return HB_OK;
  }
  Prof pr(prof_class(epi), s);
  int rc = gemm_tc(epi, a_mn, b_mn, M, N, K, A, B, ep, s);
  if (!rc) pr.done(1, 2.0 * M * N * (double)K, gemm_bytes(epi, M, N, K, 2.0, true));
  return rc;
}

static int gemm_simt_p(int epi, bool a_mn, bool b_mn, int M, int N, int K, const void* A, int64_t lda, int adt,
                       const void* B, int64_t ldb, int bdt, const EpiArgs& ep, cudaStream_t s) {
  if (M <= 0 || N <= 0 || K <= 0) return HB_OK;
  Prof pr(prof_class(epi), s);
  int rc = gemm_simt(epi, a_mn, b_mn, M, N, K, A, lda, adt, B, ldb, bdt, ep, s);
  if (!rc) pr.done(1, 2.0 * M * N * (double)K, gemm_bytes(epi, M, N, K, 4.0, false));
  return rc;
}

// ----------------------------------------------------------------------------------------
// fused row-block chain (rowchain.cuh): eligibility and launch
// ----------------------------------------------------------------------------------------
struct RcCfg {
  bool ok = false;
  int CS = 1, NH = 64, NCA = 1, NS = 2, tmem = 128, smem = 0, s_tma = 0;
};

#ifdef HB_TUNING
static unsigned long long* g_rc_trace = nullptr;  // tuning only: hb_rc_trace
static int g_bench_part = 0;                      // tuning only: hb_bench_step part
static int64_t g_rc_trace_cap = 0;
#else
static constexpr unsigned long long* g_rc_trace = nullptr;
static constexpr int g_bench_part = 0;
#endif
static constexpr int RC_SMEM_CAP = 232448;  // 227 KB opt-in dynamic shared memory per CTA

// n_0 - n x (L-1) - C with uniform hidden width n <= 512, n_0 <= 512, C <= 16, 2 <= L <= 12
// (HB_ROWCHAIN=0 disables).  Cluster size for a batch of b rows: the widest CS in {1,2,4,8} with
// at least 64 output columns per CTA whose CS x ceil(b/128) CTAs still fit the SMs in one wave
// (every doubling halves the W bytes each SM streams per layer); HB_RC_CS forces it.
static RcCfg rowchain_cfg(const hb_model* m, int b = 8192) {
  RcCfg c;
  if (!m->opt_rowchain || m->prec != HB_PREC_BF16) return c;
  const int L = (int)m->layers.size();
  if (L < 2 || L > RC_MAX_L) return c;
  const int n0 = m->dims[0], n = m->dims[1], C = m->dims[L];
  for (int l = 1; l < L; ++l)
    if (m->dims[l] != n) return c;
  if (n0 > 512 || n > 512 || C > 16) return c;
  // measured on B200 (scripts/rc_probe.py, C2 shape): the fused chain is latency-bound at
  // ~65-90 us whatever the batch, the per-layer chain is cheaper below b = 8192
  if (m->rc_min_b <= 0 || b < m->rc_min_b) return c;
  const int cs_env = m->opt_rc_cluster;
  static int nsm = 0;
  if (!nsm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm <= 0) nsm = 148;
  }
  const int rbs = std::max(1, (b + 127) / 128);
  auto nh_of = [&](int cs) { return (int)round_up((n + cs - 1) / cs, 64); };
  int cs = 1;
  if (cs_env == 1 || cs_env == 2 || cs_env == 4 || cs_env == 8) {
    cs = cs_env;
  } else {
    while (cs < RC_MAX_CS && nh_of(cs * 2) >= 64 && (n + cs * 2 * 64 - 1) / (cs * 2 * 64) >= 1 &&
           nh_of(cs * 2) * (cs * 2 - 1) < n && (long)cs * 2 * rbs <= nsm)
      cs *= 2;
  }
  while (nh_of(cs) > 256 && cs < RC_MAX_CS) cs *= 2;  // TMEM: two NH-column accumulators
  c.CS = cs;
  c.NH = nh_of(cs);
  if (c.NH > 256) return c;
  c.NCA = std::max((n0 + 63) / 64, c.CS * c.NH / 64);
  const int stb = c.NH * 128;
  // 1 KB alignment slack + abuf + W ring + staged bias (1 KB) + mbarriers
  // sigma' staging for TMA stores (2 chunk buffers) when the W ring keeps >= 2 stages: the
  // per-thread-row global stores it replaces cost ~0.45 us per chunk (B200, C2 b = 8192) and a
  // 2-stage ring measured as fast as 3 (scripts/gpu_refresh.sh)
  static const int s_tma_env = HB_TUNE("HB_RC_S_TMA", 1);
  c.s_tma = s_tma_env && (RC_SMEM_CAP - (1024 + c.NCA * RC_CHUNK + 2 * RC_CHUNK + 1024 + 8 * (2 * 2 + c.NCA + 8) + 16)) /
                             (c.NH * 128) >= 2;
  const int fixed = 1024 + c.NCA * RC_CHUNK + (c.s_tma ? 2 * RC_CHUNK : 0) + 1024 + 8 * (2 * RC_MAX_STAGES + c.NCA + 8) + 16;
  static const int ns_env = HB_TUNE("HB_RC_NS", 0);  // tuning only: force the W ring depth
  c.NS = std::min(RC_MAX_STAGES, (RC_SMEM_CAP - fixed) / stb);
  if (ns_env >= 2 && ns_env < c.NS) c.NS = ns_env;
  if (c.NS < 2) return c;
  c.smem = 1024 + c.NCA * RC_CHUNK + c.NS * stb + (c.s_tma ? 2 * RC_CHUNK : 0) + 1024 + 8 * (2 * c.NS + c.NCA + 8) + 16;
  c.tmem = 64;
  while (c.tmem < 2 * c.NH) c.tmem *= 2;
  c.ok = true;
  return c;
}

// One launch of the fused chain for batch rows [0, b) of X (row offset *d_off when non-null).
static int launch_rowchain(hb_worker* w, const RcCfg& c, const void* X, int64_t ldx, int64_t x_rows,
                           const int32_t* y, const int* d_off, int b, cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  const int n = m->dims[1];
  RcParams P;
  std::memset(&P, 0, sizeof(P));
  int rc = make_map(&P.mX, X, m->dims[0], x_rows, ldx * 2, 64, 128);
  for (int l = 0; l < L && !rc; ++l) {
    const Layer& Ly = m->layers[l];
    const __nv_bfloat16* W = m->shadow + Ly.w_off;
    rc = make_map(&P.mW[l], W, Ly.n_in, Ly.n_out, (int64_t)Ly.ldw * 2, 64, l == L - 1 ? 16 : c.NH);
    if (!rc && l >= 1) rc = make_map(&P.mWt[l], W, Ly.n_in, Ly.n_out, (int64_t)Ly.ldw * 2, 64, 64);
    if (!rc && l <= L - 2) {
      rc = make_map(&P.mH[l], w->H[l], n, b, (int64_t)Ly.ldo * 2, 64, 32);
      if (!rc) rc = make_map(&P.mDZ[l], w->dZ[l], n, b, (int64_t)Ly.ldo * 2, 64, 32);
      if (!rc) rc = make_map(&P.mS[l], w->S[l], n, b, (int64_t)Ly.ldo * 2, 64, 32);
      P.S[l] = static_cast<__nv_bfloat16*>(w->S[l]);
    }
    P.bias[l] = m->master + Ly.b_off;
    P.bpart[l] = w->bpart[l];
  }
  if (rc) return rc;
  P.d_off = d_off;
  P.y = y;
  P.dz_head = static_cast<__nv_bfloat16*>(w->dZ[L - 1]);
  P.row_loss = w->row_loss;
  P.ldo = m->layers[0].ldo;
  P.ldo_head = w->ld_dzL;
  P.L = L;
  P.n0 = m->dims[0];
  P.n = n;
  P.C = m->dims[L];
  P.b = b;
  P.CS = c.CS;
  P.NH = c.NH;
  P.nstages = c.NS;
  P.abuf_chunks = c.NCA;
  P.tmem_cols = c.tmem;
  static const int korder = HB_TUNE("HB_RC_KORDER", 0);  // 1 measured slower (B200, C2 b = 8192: 103 vs 88 us)
  P.korder = korder;
  P.s_tma = c.s_tma;
  P.inv_b = 1.0f / (float)b;
  P.dbg = g_rc_trace;
  int dev = 0;
  cudaGetDevice(&dev);
  {
    std::lock_guard<std::mutex> g(g_attr_mu);
    auto key = std::make_pair((const void*)rowchain_kernel, dev);
    if (!g_attr_done.count(key)) {
      HB_CUDA_TRY(cudaFuncSetAttribute(rowchain_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, RC_SMEM_CAP));
      g_attr_done.insert(key);
    }
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(c.CS * ((b + 127) / 128), 1, 1);
  cfg.blockDim = dim3(RC_THREADS);
  cfg.dynamicSmemBytes = c.smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (m->opt_pdl) {
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  if (c.CS > 1) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = c.CS;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  HB_CUDA_TRY(cudaLaunchKernelEx(&cfg, rowchain_kernel, P));
  HB_CUDA_TRY(cudaGetLastError());
  return HB_OK;
}

// algorithmic FLOPs / bytes of one chain launch: forward + dX contractions; X, W (read by the
// forward and the dX GEMMs), y, and the H/S/dZ/row-loss traffic the dW GEMMs need
static void rowchain_cost(const hb_model* m, int b, double* flops, double* bytes) {
  const int L = (int)m->layers.size();
  double P = 0, hid = 0;
  for (int l = 0; l < L; ++l) P += (double)m->layers[l].n_in * m->layers[l].n_out;
  for (int l = 0; l + 1 < L; ++l) hid += m->layers[l].n_out;
  const double p1 = (double)m->layers[0].n_in * m->layers[0].n_out;
  *flops = 2.0 * b * P + 2.0 * b * (P - p1);
  *bytes = 2.0 * b * m->dims[0] + 4.0 * P + 4.0 * b + 2.0 * b * hid * 4.0 + 2.0 * b * m->dims[L] + 4.0 * b;
}

// ----------------------------------------------------------------------------------------
// model / worker
// ----------------------------------------------------------------------------------------
// the output layer's dW GEMM runs transposed (M = n_in, N = C) and, with C <= 16, on the
// split-precision dZ_L (R24)
static bool head_transposed(const Layer& Ly) { return Ly.n_out < 128 && Ly.n_out < Ly.n_in; }
static bool head_hilo(const Layer& Ly) { return Ly.n_out <= 16 && head_transposed(Ly); }
static int64_t ld_dz(const hb_worker* w, int l) {
  return l == (int)w->m->layers.size() - 1 ? w->ld_dzL : w->m->layers[l].ldo;
}

// ---- small-C output layer as one CUDA-core pass (head.cuh) ---------------------------------
// Shape of the launch for a batch of b rows: CMAX classes (2/4/8), CPT 8-column chunks per
// thread, T threads, RB rows per round; a contiguous range of `rows` rows per CTA, grid CTAs
// (at most the resident capacity: one 256-thread CTA per SM, more for narrower rows).
struct HeadCfg {
  bool ok = false;
  int cmax = 0, cw = 0, cpt = 0, T = 0, rb = 0, rows = 0, grid = 0;
  int grid_max = 0;  // upper bound of grid over every batch size (sizes the worker's partial buffers)
};
static HeadCfg head_shape(const hb_model* m, int b) {
  HeadCfg h;
  const int L = (int)m->layers.size();
  if (m->prec != HB_PREC_BF16 || L < 2 || b <= 0) return h;
  const Layer& Ly = m->layers[L - 1];
  const int C = Ly.n_out, n = Ly.n_in;
  if (C > HEAD_MAX_C) return h;
  h.cmax = C <= 2 ? 2 : C <= 4 ? 4 : 8;
  const bool narrow = n <= 1024;  // HeadShape: 8-byte chunks, 16 / CMAX rows per round, two CTAs per SM
  h.cw = narrow ? 4 : 8;
  const int maxt = narrow ? 256 : h.cmax <= 4 ? 512 : 256;  // HeadShape::MAXT
  const int nc = (n + h.cw - 1) / h.cw;
  h.T = std::min(maxt, (nc + 31) / 32 * 32);
  h.cpt = (nc + h.T - 1) / h.T;
  if (h.cmax * h.cpt > (h.cmax <= 4 ? 4 : 8)) return h;  // register budget (wider rows: tensor-core head)
  h.rb = narrow ? (h.cmax == 8 ? 4 : 16 / h.cmax) : std::max(1, std::min(16 / h.cmax, 4 / h.cpt));
  static int nsm = 0;
  if (!nsm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm <= 0) nsm = 148;
  }
  const int rounds = (b + h.rb - 1) / h.rb;
  const int cap = narrow ? 2 * nsm : nsm * std::max(1, maxt / h.T);
  // every CTA's dW_L / bias partials (C x n floats) are re-read by the update kernel and its
  // prologue (first bulk copies, W_L columns) is a fixed cost: at most ~2 MB of partials (but a CTA
  // per SM), and at least 4 rounds per CTA once the batch exceeds one round per resident CTA
  h.grid_max = std::min(cap, std::max(nsm, (int)((2 << 20) / (4L * C * n))));
  int g = std::min(rounds, h.grid_max);
  if (rounds > cap) g = std::max(1, std::min(g, rounds / 4));
  h.rows = (rounds + g - 1) / g * h.rb;
  h.grid = (b + h.rows - 1) / h.rows;
  h.ok = true;
  return h;
}
// the per-layer step uses it unless disabled, the model is recorded for the persistent step
// kernel (g_plan) or the worker has no partial buffer
static HeadCfg head_cfg(const hb_worker* w, int b) {
  if (!w->m->opt_head_kernel || !w->hws || g_plan) return HeadCfg{};
  return head_shape(w->m, b);
}

static int act_dt(const hb_model* m) { return m->prec == HB_PREC_BF16 ? HB_BF16 : HB_F32; }
static size_t act_size(const hb_model* m) { return m->prec == HB_PREC_BF16 ? 2 : 4; }

// grid of a worker's persistent step kernel: fixed per worker (the stage barriers count launches of
// one grid size), enough CTAs for the widest stage at max_batch, at most one per SM
static int step_kernel_grid(const hb_model* m, int max_b) {
  int mx = 1;
  for (const Layer& Ly : m->layers) mx = std::max(mx, std::max(Ly.n_out, Ly.n_in));
  const long t = (long)((max_b + TC_BM - 1) / TC_BM) * ((mx + 31) / 32) + (long)((mx + TC_BM - 1) / TC_BM) * ((mx + 31) / 32);
  int nsm = 148, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  return (int)std::max<long>(1, std::min<long>(t, nsm > 0 ? nsm : 148));
}

static void free_worker_buffers(hb_worker* w) {
  for (void* p : w->H) cudaFree(p);
  for (void* p : w->S) cudaFree(p);
  for (void* p : w->dZ) cudaFree(p);
  w->H.clear();
  w->S.clear();
  w->dZ.clear();
  clear_graphs(w);
  for (float* p : w->bpart) cudaFree(p);
  w->bpart.clear();
  cudaFree(w->d_off);
  if (w->h_off) cudaFreeHost(w->h_off);
  w->d_off = nullptr;
  w->h_off = nullptr;
  cudaFree(w->ws);
  w->ws = nullptr;
  cudaFree(w->hws);
  w->hws = nullptr;
  for (cudaEvent_t e : w->ev_bwd) cudaEventDestroy(e);
  w->ev_bwd.clear();
  if (w->ev_join2) cudaEventDestroy(w->ev_join2);
  w->ev_join2 = nullptr;
  for (cudaStream_t x : w->sdw) cudaStreamDestroy(x);
  w->sdw.clear();
  for (cudaEvent_t e : w->ev_dw) cudaEventDestroy(e);
  w->ev_dw.clear();
  if (w->ev_chain) cudaEventDestroy(w->ev_chain);
  w->ev_chain = nullptr;
  for (float* p : w->ws_l) cudaFree(p);
  w->ws_l.clear();
  if (w->s2) cudaStreamDestroy(w->s2);
  w->s2 = nullptr;
  cudaFree(w->sk_bar);
  w->sk_bar = nullptr;
  cudaFree(w->logits);
  cudaFree(w->row_loss);
  cudaFree(w->dsum);
  cudaFree(w->grads);
  if (w->h_dsum) cudaFreeHost(w->h_dsum);
  w->logits = w->row_loss = w->grads = nullptr;
  w->dsum = nullptr;
  w->h_dsum = nullptr;
}

static int alloc_worker(hb_model* m, int max_b, cudaStream_t stream, bool own, hb_worker** out, bool train = true) {
  hb_worker* w = new hb_worker();
  w->m = m;
  w->global = m;
  w->max_b = max_b;
  w->stream = stream;
  w->own_stream = own;
  const int L = (int)m->layers.size();
  const size_t es = act_size(m);
  auto fail_free = [&](int rc) {
    free_worker_buffers(w);
    if (w->own_stream && w->stream) cudaStreamDestroy(w->stream);
    delete w;
    return rc;
  };
  int max_w = 1;
  for (int l = 0; l < L; ++l) {
    const Layer& Ly = m->layers[l];
    max_w = std::max(max_w, Ly.n_out);
    void* p = nullptr;
    if (l < L - 1) {
      if (cudaMalloc(&p, (size_t)max_b * Ly.ldo * es) != cudaSuccess) return fail_free(fail(HB_ENOMEM, "H alloc"));
      w->H.push_back(p);
      if (cudaMalloc(&p, (size_t)max_b * Ly.ldo * es) != cudaSuccess) return fail_free(fail(HB_ENOMEM, "S alloc"));
      w->S.push_back(p);
    }
    // the head's dZ_L of a bf16 model with C <= 16 and a transposed head dW GEMM holds two bf16
    // planes (hi in columns [0, 16), lo in [16, 32), R24)
    const bool hl = l == L - 1 && m->prec == HB_PREC_BF16 && head_hilo(Ly);
    const int64_t ldz = hl ? 32 : Ly.ldo;
    if (l == L - 1) {
      w->hilo = hl;
      w->ld_dzL = (int)ldz;
    }
    if (cudaMalloc(&p, (size_t)max_b * ldz * es) != cudaSuccess) return fail_free(fail(HB_ENOMEM, "dZ alloc"));
    cudaMemset(p, 0, (size_t)max_b * ldz * es);
    w->dZ.push_back(p);
  }
  const int C = m->layers.back().n_out;
  w->ldc = (int)round_up(C, 4);
  const int mt = (max_b + 127) / 128;
  const HeadCfg hc = head_shape(m, max_b);  // hc.grid_max bounds the head kernel's grid at every b
  for (int l = 0; l < L; ++l) {
    float* p = nullptr;
    const size_t rows = std::max<size_t>((size_t)4 * mt, hc.ok ? (size_t)hc.grid_max : 0);  // x4: per-quadrant (fused path)
    if (cudaMalloc(&p, rows * m->layers[l].n_out * 4) != cudaSuccess)
      return fail_free(fail(HB_ENOMEM, "bias partial alloc"));
    w->bpart.push_back(p);
  }
  if (hc.ok && cudaMalloc(&w->hws, (size_t)hc.grid_max * C * (m->layers.back().n_in + 1) * 4) != cudaSuccess)
    return fail_free(fail(HB_ENOMEM, "head partial alloc"));
  if (m->prec == HB_PREC_BF16 && cudaMalloc(&w->ws, (size_t)148 * TC_BM * 256 * 4) != cudaSuccess)
    return fail_free(fail(HB_ENOMEM, "split-K workspace alloc"));
  if (m->prec == HB_PREC_BF16) {  // second stream for the dW GEMMs (backward overlap)
    if (cudaStreamCreateWithFlags(&w->s2, cudaStreamNonBlocking) != cudaSuccess)
      return fail_free(fail(HB_ECUDA, "stream create"));
    for (int l = 0; l < L; ++l) {
      cudaEvent_t e;
      cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
      w->ev_bwd.push_back(e);
    }
    cudaEventCreateWithFlags(&w->ev_join2, cudaEventDisableTiming);
  }
  if (train && rowchain_cfg(m, max_b).ok) {  // fused path possible: per-layer dW streams + workspaces
    for (int l = 0; l < L; ++l) {
      cudaStream_t x;
      cudaEvent_t e;
      float* p = nullptr;
      if (cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking) != cudaSuccess)
        return fail_free(fail(HB_ECUDA, "stream create"));
      w->sdw.push_back(x);
      cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
      w->ev_dw.push_back(e);
      if (cudaMalloc(&p, (size_t)148 * TC_BM * 256 * 4) != cudaSuccess)
        return fail_free(fail(HB_ENOMEM, "split-K workspace alloc"));
      w->ws_l.push_back(p);
    }
    cudaEventCreateWithFlags(&w->ev_chain, cudaEventDisableTiming);
  }
  if (train && m->prec == HB_PREC_BF16) {  // persistent small-batch step: stage barriers + generation word
    if (cudaMalloc(&w->sk_bar, (SK_MAX_S + 1) * sizeof(unsigned)) != cudaSuccess)
      return fail_free(fail(HB_ENOMEM, "step-kernel barrier alloc"));
    cudaMemset(w->sk_bar, 0, (SK_MAX_S + 1) * sizeof(unsigned));
    w->sk_grid = step_kernel_grid(m, max_b);
  }
  if (cudaMalloc(&w->logits, (size_t)max_b * w->ldc * 4) != cudaSuccess ||
      cudaMalloc(&w->row_loss, (size_t)max_b * 4) != cudaSuccess ||
      cudaMalloc(&w->d_off, sizeof(int)) != cudaSuccess || cudaMallocHost(&w->h_off, HB_MAX_INFLIGHT * sizeof(int)) != cudaSuccess ||
      cudaMalloc(&w->dsum, 64 * sizeof(double)) != cudaSuccess ||
      cudaMallocHost(&w->h_dsum, 64 * sizeof(double)) != cudaSuccess)
    return fail_free(fail(HB_ENOMEM, "worker scratch alloc"));
  *out = w;
  return HB_OK;
}

}  // namespace hb

using namespace hb;

// ----------------------------------------------------------------------------------------
// one SGD step: Eq. (1) forward, softmax-xent head, Eq. (2) backward, Eq. (3) in-place update
// ----------------------------------------------------------------------------------------
namespace hb {

// fp32 check mode: SIMT GEMMs, fp32 activations, standalone softmax / bias kernels.
static int run_step_simt(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, const int32_t* y, int b, float lr,
                         bool grads_only, cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  int rc;
  const void* Ain = X;
  int64_t lda = ldx;
  int ain_dt = xdt;
  for (int l = 0; l < L; ++l) {
    const Layer& Ly = m->layers[l];
    EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
    ep.M = b;
    ep.N = Ly.n_out;
    ep.bias = m->master + Ly.b_off;
    int epi;
    if (l < L - 1) {
      epi = EPI_FWD_SIG;
      ep.out0 = w->H[l];
      ep.ld0 = Ly.ldo;
      ep.out1 = w->S[l];
      ep.ld1 = Ly.ldo;
    } else {
      epi = EPI_FWD_LOGITS;
      ep.out0 = w->logits;
      ep.ld0 = w->ldc;
    }
    rc = gemm_simt_p(epi, false, false, b, Ly.n_out, Ly.n_in, Ain, lda, ain_dt, m->master + Ly.w_off, Ly.ldw, HB_F32,
                     ep, s);
    if (rc) return rc;
    if (l < L - 1) {
      Ain = w->H[l];
      lda = Ly.ldo;
      ain_dt = HB_F32;
    }
  }
  {
    const Layer& Ly = m->layers[L - 1];
    Prof pr(HB_PROF_SOFTMAX, s);
    softmax_xent_kernel<float><<<(b * 32 + 255) / 256, 256, 0, s>>>(
        w->logits, w->ldc, y, nullptr, b, Ly.n_out, static_cast<float*>(w->dZ[L - 1]), Ly.ldo, w->row_loss,
        1.0f / (float)b);
    HB_CUDA_TRY(cudaGetLastError());
    pr.done(1, 0.0, (double)b * Ly.n_out * 8.0 + 8.0 * b);
  }
  for (int l = L - 1; l >= 0; --l) {
    const Layer& Ly = m->layers[l];
    const void* dZl = w->dZ[l];
    const void* Al = l == 0 ? X : w->H[l - 1];
    const int64_t ldal = l == 0 ? ldx : m->layers[l - 1].ldo;
    const int al_dt = l == 0 ? xdt : HB_F32;
    if (l > 0) {
      const Layer& Lp = m->layers[l - 1];
      EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
      ep.M = b;
      ep.N = Ly.n_in;
      ep.out0 = w->dZ[l - 1];
      ep.ld0 = Lp.ldo;
      ep.aux = w->S[l - 1];
      ep.ldaux = Lp.ldo;
      rc = gemm_simt_p(EPI_DGRAD_SIG, false, true, b, Ly.n_in, Ly.n_out, dZl, Ly.ldo, HB_F32, m->master + Ly.w_off,
                       Ly.ldw, HB_F32, ep, s);
      if (rc) return rc;
    }
    {
      EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
      const int epi = grads_only ? EPI_WGRAD_STORE : EPI_WGRAD_SGD;
      ep.master = m->master + Ly.w_off;
      ep.ldw = Ly.ldw;
      ep.lr = lr;
      if (grads_only) ep.out0 = w->grads + Ly.w_off;
      const bool tr = Ly.n_out < 128 && Ly.n_out < Ly.n_in;
      ep.transposed = tr ? 1 : 0;
      if (!tr) {
        ep.M = Ly.n_out;
        ep.N = Ly.n_in;
        rc = gemm_simt_p(epi, true, true, Ly.n_out, Ly.n_in, b, dZl, Ly.ldo, HB_F32, Al, ldal, al_dt, ep, s);
      } else {
        ep.M = Ly.n_in;
        ep.N = Ly.n_out;
        rc = gemm_simt_p(epi, true, true, Ly.n_in, Ly.n_out, b, Al, ldal, al_dt, dZl, Ly.ldo, HB_F32, ep, s);
      }
      if (rc) return rc;
    }
    {
      const int splits = (b + 127) / 128;
      Prof pr(HB_PROF_BIAS, s);
      colsum_partial_kernel<float><<<dim3((Ly.n_out + 63) / 64, splits), dim3(64, 4), 0, s>>>(
          static_cast<const float*>(dZl), Ly.ldo, b, Ly.n_out, 128, w->bpart[l]);
      bias_apply_kernel<<<(Ly.n_out + 255) / 256, 256, 0, s>>>(w->bpart[l], splits, Ly.n_out, lr,
                                                               m->master + Ly.b_off,
                                                               grads_only ? w->grads + Ly.b_off : nullptr);
      HB_CUDA_TRY(cudaGetLastError());
      pr.done(2, (double)b * Ly.n_out, (double)b * Ly.n_out * 4.0 + 8.0 * Ly.n_out);
    }
  }
  return HB_OK;
}

// Optionally (HB_HEAD_FUSE=1) the output layer's dX runs in the head kernel's epilogue when C <= 16.
// Off by default: measured slower on B200 at b = 8192 (37.5 M vs 42.5 M samples/s on C2) because
// the head grid has only b/128 CTAs while the separate dX GEMM fills all 148 SMs.
static bool head_dx_fused(const hb_model* m) {
  return m->opt_head_fuse && m->layers.size() >= 2 && m->layers.back().n_out <= 16;
}

// The output layer in one pass (head.cuh): logits, softmax-CE row losses and, when training, dZ_{L-1}
// with its bias partials (one row per CTA) and the per-CTA dW_L / db_L partials.
template <int CMAX, int CPT, int RB, int CW>
static int launch_head_t(const HeadCfg& hc, HeadArgs a, bool pdl, cudaStream_t s) {
  auto kern = head_fused_kernel<CMAX, CPT, RB, CW>;
  // wide rows: one CTA per SM with the deepest ring that fits; narrow rows (CW = 4): two CTAs per SM
  constexpr int kMaxSmem = CW == 4 ? 100 * 1024 : 200 * 1024;
  {
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> g(g_attr_mu);
    auto key = std::make_pair((const void*)kern, dev);
    if (!g_attr_done.count(key)) {
      HB_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmem));
      g_attr_done.insert(key);
    }
  }
  // ring of RB-row stages of H (and S): as deep as fits, at most HEAD_MAX_STAGES
  const size_t stage = (size_t)RB * a.ld * 2 * (a.dz ? 2 : 1);
  a.stages = (int)std::min<size_t>(HEAD_MAX_STAGES, kMaxSmem / stage);
  if (a.stages < 2) return fail(HB_EUNSUPPORTED, "head kernel: rows too wide for the shared-memory ring");
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(hc.grid);
  cfg.blockDim = dim3(hc.T);
  cfg.dynamicSmemBytes = stage * a.stages;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  HB_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, a));
  HB_CUDA_TRY(cudaGetLastError());
  return HB_OK;
}

static int launch_head(hb_worker* w, const HeadCfg& hc, const int32_t* y, const int* d_off, int b, bool train,
                       cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  const Layer& Ly = m->layers[L - 1];
  const Layer& Lp = m->layers[L - 2];
  HeadArgs a{};
  a.H = static_cast<const __nv_bfloat16*>(w->H[L - 2]);
  a.S = train ? static_cast<const __nv_bfloat16*>(w->S[L - 2]) : nullptr;
  a.ld = Lp.ldo;
  a.W = m->shadow + Ly.w_off;
  a.ldw = Ly.ldw;
  a.bias = m->master + Ly.b_off;
  a.y = y;
  a.yoff = d_off;
  a.b = b;
  a.n = Ly.n_in;
  a.C = Ly.n_out;
  a.rows_per_cta = hc.rows;
  a.inv_b = 1.0f / (float)b;
  a.row_loss = w->row_loss;
  a.dz = train ? static_cast<__nv_bfloat16*>(w->dZ[L - 2]) : nullptr;
  a.bpart = w->bpart[L - 2];
  a.dwp = w->hws;
  a.dbp = w->hws + (size_t)hc.grid * a.C * a.n;
  ProfLayer pl(L - 1);
  Prof pr(HB_PROF_HEAD, s);
  const bool pdl = m->opt_pdl != 0;
  int rc;
  switch (hc.cw * 10000 + hc.cmax * 1000 + hc.cpt * 100 + hc.rb) {
    case 82104: rc = launch_head_t<2, 1, 4, 8>(hc, a, pdl, s); break;
    case 82202: rc = launch_head_t<2, 2, 2, 8>(hc, a, pdl, s); break;
    case 84104: rc = launch_head_t<4, 1, 4, 8>(hc, a, pdl, s); break;
    case 88102: rc = launch_head_t<8, 1, 2, 8>(hc, a, pdl, s); break;
    case 42108: rc = launch_head_t<2, 1, 8, 4>(hc, a, pdl, s); break;
    case 44104: rc = launch_head_t<4, 1, 4, 4>(hc, a, pdl, s); break;
    case 48104: rc = launch_head_t<8, 1, 4, 4>(hc, a, pdl, s); break;
    default: return fail(HB_EUNSUPPORTED, "head kernel shape");
  }
  if (rc) return rc;
  // algorithmic: H read (+ S read, dZ_{L-1} written when training), labels, row losses
  const double bn = (double)b * a.n;
  pr.done(1, (train ? 6.0 : 2.0) * bn * a.C, bn * (train ? 6.0 : 2.0) + 8.0 * b);
  return HB_OK;
}

// Eq. (3) for the output layer from the head kernel's partials: W_L -= lr dW_L, b_L -= lr db_L (or,
// grads_only, the gradients stored), the same element update as the dW GEMM epilogue.
static int launch_head_update(hb_worker* w, const HeadCfg& hc, float lr, bool grads_only, cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  const Layer& Ly = m->layers[L - 1];
  const int C = Ly.n_out, n = Ly.n_in;
  EpiArgs ep{};
  ep.master = m->master + Ly.w_off;
  ep.shadow = m->shadow + Ly.w_off;
  ep.ldw = Ly.ldw;
  ep.lr = lr;
  ep.transposed = 1;
  ep.atomic = m->opt_update == HB_UPDATE_ATOMIC;
  if (grads_only) ep.out0 = w->grads + Ly.w_off;
  if (!grads_only && !m->peers.empty()) {  // f2: the update also goes to every peer replica
    ep.npeer = (int)m->peers.size();
    ep.pscale = m->peer_scale;
    for (int p = 0; p < ep.npeer; ++p) {
      ep.pm_off[p] = m->peers[p].first - m->master;
      ep.ps_off[p] = m->peers[p].second - m->shadow;
    }
  }
  ep.bias_upd = m->master + Ly.b_off;
  ep.bias_grad = grads_only ? w->grads + Ly.b_off : nullptr;
  const float* dwp = w->hws;
  const float* dbp = w->hws + (size_t)hc.grid * C * n;
  const int blocks = (int)(((int64_t)C * n + HU_X - 1) / HU_X);
  ProfLayer pl(L - 1);
  Prof pr(HB_PROF_WGRAD_GEMM, s);
  if (grads_only)
    head_update_kernel<EPI_WGRAD_STORE><<<blocks, dim3(HU_X, HU_Y), 0, s>>>(ep, dwp, dbp, hc.grid, C, n);
  else
    head_update_kernel<EPI_WGRAD_SGD><<<blocks, dim3(HU_X, HU_Y), 0, s>>>(ep, dwp, dbp, hc.grid, C, n);
  HB_CUDA_TRY(cudaGetLastError());
  pr.done(1, (double)hc.grid * C * n, (double)hc.grid * C * (n + 1) * 4.0 + (double)C * n * 10.0);
  return HB_OK;
}

// Forward chain (Eq. (1)) of the bf16 tensor-core path.  X holds x_rows rows; the batch starts
// at row *d_off (graph replay) or at row 0 (d_off == nullptr).  With want_grad the head writes
// dZ_L and its bias partials; otherwise only the per-row losses (mlp_loss).
static int forward_tc(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, const int* d_off,
                      int b, bool want_grad, cudaStream_t s, const HeadCfg& hc) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  int rc;
  TcOp A{X, ldx, x_rows, d_off};
  for (int l = 0; l < L; ++l) {
    const Layer& Ly = m->layers[l];
    ProfLayer pl(l);
    TcOp B{m->shadow + Ly.w_off, Ly.ldw, 0, nullptr};
    EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
    ep.M = b;
    ep.N = Ly.n_out;
    ep.bias = m->master + Ly.b_off;
    if (l < L - 1) {
      ep.out0 = w->H[l];
      ep.ld0 = Ly.ldo;
      ep.out1 = want_grad ? w->S[l] : nullptr;
      ep.ld1 = Ly.ldo;
      ep.fwd_pair = m->opt_gemm_pair;
      rc = gemm_tc_p(EPI_FWD_SIG, false, false, b, Ly.n_out, Ly.n_in, A, B, ep, s);
      if (rc) return rc;
      A = TcOp{w->H[l], Ly.ldo, b, nullptr};
      continue;
    }
    // output layer + softmax cross-entropy: dZ_L = (softmax(z) - onehot(y)) / b, per-row loss
    if (hc.ok) {  // small C: one CUDA-core pass, also the output layer's dX and dW partials (head.cuh)
      rc = launch_head(w, hc, y, d_off, b, want_grad, s);
      if (rc) return rc;
    } else if (Ly.n_out <= 16) {
      ep.out0 = want_grad ? w->dZ[l] : nullptr;
      ep.ld0 = w->ld_dzL;
      ep.hilo = w->hilo ? 16 : 0;
      ep.y = y;
      ep.yoff = d_off;
      ep.row_loss = w->row_loss;
      ep.inv_b = 1.0f / (float)b;
      ep.bpart_out = want_grad ? w->bpart[l] : nullptr;
      ep.ldp = Ly.n_out;
      if (want_grad && head_dx_fused(m)) {  // the output layer's dX runs in this kernel's epilogue
        const Layer& Lp = m->layers[l - 1];
        ep.w_head = m->master + Ly.w_off;
        ep.ldw_head = Ly.ldw;
        ep.n_prev = Lp.n_out;
        ep.s_prev = static_cast<const __nv_bfloat16*>(w->S[l - 1]);
        ep.dz_prev = static_cast<__nv_bfloat16*>(w->dZ[l - 1]);
        ep.ld_prev = Lp.ldo;
        ep.bpart_prev = w->bpart[l - 1];
      }
      rc = gemm_tc_p(EPI_HEAD_XENT, false, false, b, Ly.n_out, Ly.n_in, A, B, ep, s);
      if (rc) return rc;
    } else {
      ep.out0 = w->logits;
      ep.ld0 = w->ldc;
      rc = gemm_tc_p(EPI_FWD_LOGITS, false, false, b, Ly.n_out, Ly.n_in, A, B, ep, s);
      if (rc) return rc;
      {
        // algorithmic bytes: fp32 logits read once, bf16 dZ written once, labels and row losses
        Prof pr(HB_PROF_SOFTMAX, s);
        softmax_xent_kernel<__nv_bfloat16><<<(b * 32 + 255) / 256, 256, 0, s>>>(
            w->logits, w->ldc, y, d_off, b, Ly.n_out, want_grad ? static_cast<__nv_bfloat16*>(w->dZ[l]) : nullptr,
            w->ld_dzL, w->row_loss, 1.0f / (float)b);
        HB_CUDA_TRY(cudaGetLastError());
        pr.done(1, 0.0, (double)b * Ly.n_out * (want_grad ? 6.0 : 4.0) + 8.0 * b);
      }
      if (want_grad) {  // bias-gradient partials of dZ_L (reduced by the head's dW GEMM)
        Prof pr(HB_PROF_BIAS, s);
        colsum_partial_kernel<__nv_bfloat16><<<dim3((Ly.n_out + 63) / 64, (b + 127) / 128), dim3(64, 4), 0, s>>>(
            static_cast<const __nv_bfloat16*>(w->dZ[l]), w->ld_dzL, b, Ly.n_out, 128, w->bpart[l]);
        HB_CUDA_TRY(cudaGetLastError());
        pr.done(1, 0.0, (double)b * Ly.n_out * 2.0 + 4.0 * ((b + 127) / 128) * Ly.n_out);
      }
    }
  }
  return HB_OK;
}

// dW_l = dZ_l^T A_{l-1} with the fused in-place SGD of W_l and b_l (b_l from the partials of the
// dZ producer) on stream s, split-K workspace ws
static int launch_wgrad(hb_worker* w, int l, const void* X, int64_t ldx, int64_t x_rows, const int* d_off, int b,
                        float lr, bool grads_only, cudaStream_t s, float* ws, int part_rows, int force_bn = 0,
                        int force_splits = 0) {
  hb_model* m = w->m;
  const Layer& Ly = m->layers[l];
  ProfLayer pl(l);
  TcOp dZl{w->dZ[l], ld_dz(w, l), b, nullptr};
  TcOp Al = l == 0 ? TcOp{X, ldx, x_rows, d_off} : TcOp{w->H[l - 1], m->layers[l - 1].ldo, b, nullptr};
  EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
  const int epi = grads_only ? EPI_WGRAD_STORE : EPI_WGRAD_SGD;
  ep.master = m->master + Ly.w_off;
  ep.shadow = m->shadow + Ly.w_off;
  ep.ldw = Ly.ldw;
  ep.lr = lr;
  if (grads_only) ep.out0 = w->grads + Ly.w_off;
  ep.bpart_in = w->bpart[l];
  ep.ldp = Ly.n_out;
  ep.n_mtiles = part_rows;
  ep.force_bn = force_bn;
  ep.force_splits = force_splits;
  ep.pair = m->opt_dw_pair;
  ep.fwd_pair = m->opt_gemm_pair;
  ep.no_pdl = !m->opt_pdl;
  ep.atomic = m->opt_update == HB_UPDATE_ATOMIC;
  if (!grads_only && !m->peers.empty()) {  // f2: the update also goes to every peer replica
    ep.npeer = (int)m->peers.size();
    ep.pscale = m->peer_scale;
    for (int p = 0; p < ep.npeer; ++p) {
      ep.pm_off[p] = m->peers[p].first - m->master;
      ep.ps_off[p] = m->peers[p].second - m->shadow;
    }
  }
  ep.bias_upd = m->master + Ly.b_off;
  ep.bias_grad = grads_only ? w->grads + Ly.b_off : nullptr;
  ep.ws = ws;
  const bool tr = head_transposed(Ly);  // small head: M = n_in instead of n_out
  ep.transposed = tr ? 1 : 0;
  if (!tr) {
    ep.M = Ly.n_out;
    ep.N = Ly.n_in;
    return gemm_tc_p(epi, true, true, Ly.n_out, Ly.n_in, b, dZl, Al, ep, s);
  }
  ep.M = Ly.n_in;
  ep.N = Ly.n_out;
  if (l == (int)m->layers.size() - 1 && w->hilo) {  // both dZ_L planes: N = 32, halves summed (R24)
    ep.N = 32;
    ep.hilo = 16;
    ep.n_real = Ly.n_out;
    ep.force_bn = 32;
  }
  return gemm_tc_p(epi, true, true, Ly.n_in, ep.N, b, Al, dZl, ep, s);
}

// Fused path: one rowchain launch (forward, head, dX chain for every 128-row block), then the dW
// GEMMs of all layers concurrently on the worker's per-layer streams (they only read H/dZ and each
// updates a different W_l; every dX read of W happened inside the chain), joined on s.
static int run_step_rowchain(hb_worker* w, const RcCfg& c, const void* X, int64_t ldx, int64_t x_rows,
                             const int32_t* y, const int* d_off, int b, float lr, bool grads_only, cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  if (g_bench_part != 2) {
    Prof pr(HB_PROF_ROWCHAIN, s);
    int rc = launch_rowchain(w, c, X, ldx, x_rows, y, d_off, b, s);
    if (rc) return rc;
    double fl, by;
    rowchain_cost(m, b, &fl, &by);
    pr.done(1, fl, by);
  }
  if (g_bench_part == 1) return HB_OK;
  static const bool conc = HB_TUNE("HB_RC_DW_SERIAL", 0) == 0;
  if (!conc) {
    for (int l = L - 1; l >= 0; --l) {
      int rc = launch_wgrad(w, l, X, ldx, x_rows, d_off, b, lr, grads_only, s, w->ws_l[l], 4 * ((b + 127) / 128));
      if (rc) return rc;
    }
    if (g_loss_acc) sum_rows_into(w, b, g_loss_acc, s, true);
    return HB_OK;
  }
  HB_CUDA_TRY(cudaEventRecord(w->ev_chain, s));
  for (int l = L - 1; l >= 0; --l) {
    HB_CUDA_TRY(cudaStreamWaitEvent(w->sdw[l], w->ev_chain, 0));
    static const int fbn = HB_TUNE("HB_RC_WGRAD_BN", 0), fs = HB_TUNE("HB_RC_WGRAD_S", 0);
    const Layer& Ly = m->layers[l];
    const bool wide = Ly.n_out >= 128 || Ly.n_out >= Ly.n_in;  // not the transposed small head
    // the L GEMMs share the SMs, so each takes wide tiles (fewer L2 re-reads of dZ / H) and a
    // short split: measured on B200 (scripts/gpu_dw_sweep.sh, C2 b = 8192) BN 256 x 4 splits
    // 32 us vs 59 us for the standalone choice (BN 64 x 4).  Every GEMM uses clusters of <= 4 so
    // that all of them are co-resident (B200: 33 clusters of 4 x 200 KB CTAs at once)
    const int bn = fbn ? fbn : Ly.n_in <= 64 ? 64 : Ly.n_in <= 128 ? 128 : 256;
    int sp = fs ? fs : b >= 1024 ? 4 : 2;
    while (sp > 1 && sp > (b + TC_BK - 1) / TC_BK) sp /= 2;  // at least one k-block per split
    int rc = launch_wgrad(w, l, X, ldx, x_rows, d_off, b, lr, grads_only, w->sdw[l], w->ws_l[l],
                          4 * ((b + 127) / 128),  // per-quadrant bias partials of the chain
                          wide ? bn : 0, sp);  // the small head keeps its BN 16 tiles, 4 splits
    if (rc) return rc;
    if (l == L - 1 && g_loss_acc) sum_rows_into(w, b, g_loss_acc, w->sdw[l], true);  // row losses of the chain
    HB_CUDA_TRY(cudaEventRecord(w->ev_dw[l], w->sdw[l]));
  }
  for (int l = L - 1; l >= 0; --l) HB_CUDA_TRY(cudaStreamWaitEvent(s, w->ev_dw[l], 0));
  return HB_OK;
}

static int step_gemms(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, const int* d_off,
                      int b, float lr, bool grads_only, cudaStream_t s, bool overlap);

// ---- persistent small-batch step (step_kernel.cuh) -------------------------------------------
// Eligible: bf16 plain worker with its stage-barrier buffer, b <= HB_OPT_STEP_KERNEL_MAX_B, a
// fused softmax-xent head (C <= 16, not fused with its dX), every width <= 1024, L <= 8 layers.
static bool step_kernel_ok(const hb_worker* w, int b) {
  const hb_model* m = w->m;
  if (!w->sk_bar || m->opt_step_kernel_max_b <= 0 || b > m->opt_step_kernel_max_b) return false;
  const int L = (int)m->layers.size();
  if (L > SK_MAX_S / 2 || 3 * L - 1 > SK_MAX_G || m->layers.back().n_out > 16 || head_dx_fused(m)) return false;
  for (const Layer& Ly : m->layers)
    if (Ly.n_out > 1024 || Ly.n_in > 1024) return false;
  return true;
}

static int run_step_persistent(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y,
                               const int* d_off, int b, float lr, bool grads_only, cudaStream_t s) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  std::vector<SkPlanEntry> plan;
  g_plan = &plan;
  int rc = step_gemms(w, X, ldx, x_rows, y, d_off, b, lr, grads_only, s, false);
  g_plan = nullptr;
  if (rc) return rc;
  if ((int)plan.size() > SK_MAX_G) return fail(HB_EUNSUPPORTED, "persistent step: too many GEMMs");
  static SkParams P;  // ~15 KB: built on the host thread, copied into the launch's parameters
  static std::mutex pmu;
  std::lock_guard<std::mutex> g(pmu);
  std::memset(&P, 0, sizeof(P));
  double flops = 0.0, bytes = 0.0;
  int nst = 0;
  for (size_t k = 0; k < plan.size(); ++k) {
    const SkPlanEntry& e = plan[k];
    SkGemm& Q = P.g[k];
    const int l = e.layer;
    switch (e.epi) {
      case EPI_FWD_SIG: Q.kind = SK_FWD; Q.stage = l; break;
      case EPI_HEAD_XENT: Q.kind = SK_HEAD; Q.stage = L - 1; break;
      case EPI_DGRAD_SIG: Q.kind = SK_DGRAD; Q.stage = 2 * L - 1 - l; break;
      case EPI_WGRAD_SGD:
      case EPI_WGRAD_STORE:
        Q.kind = e.epi == EPI_WGRAD_SGD ? SK_WGRAD : SK_WGRAD_STORE;
        Q.stage = std::min(2 * L - l, 2 * L - 1);
        break;
      default: return fail(HB_EUNSUPPORTED, "persistent step: unsupported epilogue");
    }
    const int bn = Q.kind == SK_HEAD ? 16 : 32;
    const int64_t ar = e.A.rows ? e.A.rows : (e.a_mn ? e.K : e.M);
    const int64_t br = e.B.rows ? e.B.rows : (e.b_mn ? e.K : e.N);
    rc = e.a_mn ? make_map(&Q.ma, e.A.p, e.M, ar, e.A.ld * 2, 64, 64) : make_map(&Q.ma, e.A.p, e.K, ar, e.A.ld * 2, 64, TC_BM);
    if (!rc) rc = e.b_mn ? make_map(&Q.mb, e.B.p, e.N, br, e.B.ld * 2, 64, 64) : make_map(&Q.mb, e.B.p, e.K, br, e.B.ld * 2, 64, bn);
    if (rc) return rc;
    Q.ep = e.ep;
    Q.offA = e.A.off;
    Q.offB = e.B.off;
    Q.M = e.M;
    Q.N = e.N;
    Q.K = e.K;
    Q.tiles_m = (e.M + TC_BM - 1) / TC_BM;
    Q.tiles_n = (e.N + bn - 1) / bn;
    nst = std::max(nst, Q.stage + 1);
    flops += 2.0 * e.M * e.N * (double)e.K;
    bytes += gemm_bytes(e.epi, e.M, e.N, e.K, 2.0, true);
  }
  P.ng = (int)plan.size();
  P.nstages = nst;
  P.bar = w->sk_bar;
  P.dbg = g_rc_trace;
  int dev = 0;
  cudaGetDevice(&dev);
  {
    std::lock_guard<std::mutex> ga(g_attr_mu);
    auto key = std::make_pair((const void*)step_kernel, dev);
    if (!g_attr_done.count(key)) {
      HB_CUDA_TRY(cudaFuncSetAttribute(step_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SK_SMEM_BYTES));
      g_attr_done.insert(key);
    }
  }
  Prof pr(HB_PROF_STEPK, s);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(w->sk_grid, 1, 1);
  cfg.blockDim = dim3(TC_THREADS);
  cfg.dynamicSmemBytes = SK_SMEM_BYTES;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident (grid barriers)
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  HB_CUDA_TRY(cudaLaunchKernelEx(&cfg, step_kernel, P));
  HB_CUDA_TRY(cudaGetLastError());
  pr.done(1, flops, bytes);
  return HB_OK;
}

// One SGD step of the bf16 tensor-core path: forward + fused head, then for l = L..1
// dgrad (reads W_l before it is updated) and wgrad with the fused in-place SGD of W_l and b_l.
// 3L - 1 kernel launches for C <= 16 (L fwd incl. head, L-1 dgrad, L wgrad).  Narrow nets take
// the fused row-block path (L + 1 launches).
static int run_step_tc(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, const int* d_off,
                       int b, float lr, bool grads_only, cudaStream_t s) {
  hb_model* m = w->m;
  {
    const RcCfg c = rowchain_cfg(m, b);
    if (c.ok && !w->sdw.empty()) return run_step_rowchain(w, c, X, ldx, x_rows, y, d_off, b, lr, grads_only, s);
  }
  if (step_kernel_ok(w, b)) {
    int rc = run_step_persistent(w, X, ldx, x_rows, y, d_off, b, lr, grads_only, s);
    if (!rc && g_loss_acc) sum_rows_into(w, b, g_loss_acc, s, true);
    return rc;
  }
  return step_gemms(w, X, ldx, x_rows, y, d_off, b, lr, grads_only, s, m->opt_bwd_overlap && w->s2);
}

// The 3L - 1 tcgen05 GEMMs of one step in dependency order: forward + fused head, then for
// l = L..1 the dX GEMM (reads W_l) and the dW GEMM with the fused SGD of W_l.
static int step_gemms(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, const int* d_off,
                      int b, float lr, bool grads_only, cudaStream_t s, bool overlap) {
  hb_model* m = w->m;
  const int L = (int)m->layers.size();
  const HeadCfg hc = head_cfg(w, b);
  int rc = forward_tc(w, X, ldx, x_rows, y, d_off, b, true, s, hc);
  if (rc) return rc;
  // dW_l only has to follow dX_l (the last reader of W_l): it runs on the worker's second stream,
  // overlapping dX_{l-1} (HB_OPT_BWD_OVERLAP = 0 keeps everything on one stream)
  cudaStream_t s2 = overlap ? w->s2 : s;
  if (g_loss_acc && !g_plan) {  // the step's row losses into the training-loss accumulator, on s2
    if (s2 != s) {
      HB_CUDA_TRY(cudaEventRecord(w->ev_join2, s));
      HB_CUDA_TRY(cudaStreamWaitEvent(s2, w->ev_join2, 0));
    }
    sum_rows_into(w, b, g_loss_acc, s2, true);
  }
  for (int l = L - 1; l >= 0; --l) {
    const Layer& Ly = m->layers[l];
    TcOp dZl{w->dZ[l], ld_dz(w, l), b, nullptr};
    TcOp Wl{m->shadow + Ly.w_off, Ly.ldw, 0, nullptr};
    if (l > 0 && !(l == L - 1 && (hc.ok || head_dx_fused(m)))) {  // dZ_{l-1} = (dZ_l W_l) * sigma'(Z_{l-1}) + bias partials
      const Layer& Lp = m->layers[l - 1];
      EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
      ep.M = b;
      ep.N = Ly.n_in;
      ep.out0 = w->dZ[l - 1];
      ep.ld0 = Lp.ldo;
      ep.aux = w->S[l - 1];
      ep.ldaux = Lp.ldo;
      ep.bpart_out = w->bpart[l - 1];
      ep.ldp = Lp.n_out;
      ep.fwd_pair = m->opt_gemm_pair;
      ProfLayer pl(l);
      rc = gemm_tc_p(EPI_DGRAD_SIG, false, true, b, Ly.n_in, Ly.n_out, dZl, Wl, ep, s);
      if (rc) return rc;
    }
    if (s2 != s) {
      HB_CUDA_TRY(cudaEventRecord(w->ev_bwd[l], s));
      HB_CUDA_TRY(cudaStreamWaitEvent(s2, w->ev_bwd[l], 0));
    }
    if (l == L - 1 && hc.ok)  // the head kernel's dW_L / db_L partials, reduced and applied
      rc = launch_head_update(w, hc, lr, grads_only, s2);
    else  // the partials of dZ_l: per 128-row tile of its dX GEMM, or per CTA of the head kernel
      rc = launch_wgrad(w, l, X, ldx, x_rows, d_off, b, lr, grads_only, s2, w->ws,
                        l == L - 2 && hc.ok ? hc.grid : (b + TC_BM - 1) / TC_BM);
    if (rc) return rc;
  }
  if (s2 != s) {  // join: the step completes on the worker's stream
    HB_CUDA_TRY(cudaEventRecord(w->ev_join2, s2));
    HB_CUDA_TRY(cudaStreamWaitEvent(s, w->ev_join2, 0));
  }
  return HB_OK;
}

int run_step(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, int64_t x_rows, const int32_t* y,
             const int* d_off, int b, float lr, bool grads_only, cudaStream_t s) {
  if (w->m->prec == HB_PREC_BF16) return run_step_tc(w, X, ldx, x_rows, y, d_off, b, lr, grads_only, s);
  if (d_off) return fail(HB_EUNSUPPORTED, "device row offsets are a tensor-core-path feature");
  return run_step_simt(w, X, ldx, xdt, y, b, lr, grads_only, s);
}

void clear_graphs(hb_worker* w) {
  for (auto& kv : w->graphs)
    if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
  w->graphs.clear();
}

int step_graph(hb_worker* w, const void* X, int64_t ldx, int64_t x_rows, const int32_t* y, int64_t off, int b,
               float lr, double* loss_acc) {
  if (w->g_X != X || w->g_y != y || w->g_ldx != ldx || w->g_rows != x_rows) {
    clear_graphs(w);
    w->g_X = X;
    w->g_y = y;
    w->g_ldx = ldx;
    w->g_rows = x_rows;
  }
  uint32_t lrbits;
  std::memcpy(&lrbits, &lr, 4);
  // one graph per in-flight slot: a queued replay reads its batch offset from its own pinned
  // word when it starts, so up to HB_MAX_INFLIGHT replays of this worker may be enqueued
  const int slot = w->slot;
  w->slot = (w->slot + 1) % HB_MAX_INFLIGHT;
  auto key = std::make_tuple(b, lrbits, slot, (const double*)loss_acc);
  auto it = w->graphs.find(key);
  if (it == w->graphs.end()) {
    cudaStream_t s = w->stream;
    const int64_t l0 = g_launches.load();
    HB_CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    cudaMemcpyAsync(w->d_off, w->h_off + slot, sizeof(int), cudaMemcpyHostToDevice, s);
    g_loss_acc = loss_acc;
    int rc = run_step(w, X, ldx, HB_BF16, x_rows, y, w->d_off, b, lr, false, s);
    g_loss_acc = nullptr;
    cudaGraph_t graph = nullptr;
    cudaError_t ce = cudaStreamEndCapture(s, &graph);
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone) {
      cudaGraph_t g2 = nullptr;  // an invalidated capture: end it so the stream is usable again
      cudaStreamEndCapture(s, &g2);
      if (g2) cudaGraphDestroy(g2);
    }
    if (rc) {
      if (graph) cudaGraphDestroy(graph);
      cudaGetLastError();
      return rc;
    }
    if (ce != cudaSuccess) return fail(HB_ECUDA, std::string("graph capture: ") + cudaGetErrorString(ce));
    hb_worker::Graph gr;
    ce = cudaGraphInstantiate(&gr.exec, graph, 0);
    cudaGraphDestroy(graph);
    if (ce != cudaSuccess) return fail(HB_ECUDA, std::string("graph instantiate: ") + cudaGetErrorString(ce));
    gr.launches = (int)(g_launches.load() - l0);
    g_launches.fetch_sub(gr.launches);  // counted when replayed
    it = w->graphs.emplace(key, gr).first;
  }
  w->h_off[slot] = (int)off;  // the replay that last used this slot has completed (caller's in-flight bound)
  HB_CUDA_TRY(cudaGraphLaunch(it->second.exec, w->stream));
  g_launches.fetch_add(it->second.launches);
  return HB_OK;
}

int worker_execute(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, int64_t x_rows, const int32_t* y,
                   int64_t off, int b, float lr, bool graphs, bool serial, double* loss_dst, bool accumulate) {
  const size_t xes = xdt == HB_BF16 ? 2 : 4;
  auto xrow = [&](int64_t o) { return static_cast<const char*>(X) + o * ldx * xes; };
  if (w->subs.empty()) {
    if (graphs && loss_dst && accumulate)  // the step graph accumulates its own row losses (side stream)
      return step_graph(w, X, ldx, x_rows, y, off, b, lr, loss_dst);
    int rc = graphs ? step_graph(w, X, ldx, x_rows, y, off, b, lr)
                    : run_step(w, xrow(off), ldx, xdt, b, y + off, nullptr, b, lr, false, w->stream);
    if (!rc && loss_dst) sum_rows_into(w, b, loss_dst, w->stream, accumulate);
    return rc;
  }
  const int t = (int)w->subs.size();
  const int base = b / t, extra = b % t;
  if (!serial) HB_CUDA_TRY(cudaEventRecord(w->ev_fork, w->stream));
  int64_t o = off;
  for (int i = 0; i < t; ++i) {
    const int sz = base + (i < extra ? 1 : 0);
    if (sz == 0) continue;
    hb_worker* sw = w->subs[i];
    const float lr_i = lr * (float)sz / (float)b;  // eta proportional to the (sub-)batch size (L179)
    int rc;
    if (serial) {
      rc = run_step(sw, xrow(o), ldx, xdt, sz, y + o, nullptr, sz, lr_i, false, w->stream);
      if (!rc && loss_dst) sum_rows_into(sw, sz, loss_dst, w->stream, accumulate || i > 0);
    } else {
      HB_CUDA_TRY(cudaStreamWaitEvent(sw->stream, w->ev_fork, 0));
      rc = graphs ? step_graph(sw, X, ldx, x_rows, y, o, sz, lr_i)
                  : run_step(sw, xrow(o), ldx, xdt, sz, y + o, nullptr, sz, lr_i, false, sw->stream);
      HB_CUDA_TRY(cudaEventRecord(w->ev_join[i], sw->stream));
      HB_CUDA_TRY(cudaStreamWaitEvent(w->stream, w->ev_join[i], 0));
    }
    if (rc) return rc;
    o += sz;
  }
  if (!serial && loss_dst) {  // after the join: the sub-batch losses in sub-worker order
    o = off;
    bool first = true;
    for (int i = 0; i < t; ++i) {
      const int sz = base + (i < extra ? 1 : 0);
      if (sz == 0) continue;
      sum_rows_into(w->subs[i], sz, loss_dst, w->stream, accumulate || !first);
      first = false;
    }
  }
  return HB_OK;
}

static int check_step_args(hb_worker* w, const void* X, int64_t ldx, int32_t xdt, const int32_t* y, int32_t batch) {
  if (!w) return fail(HB_EINVAL, "null worker");
  hb_model* m = w->m;
  HB_CHECK_ARG(X && y, "null X or y");
  HB_CHECK_ARG(batch >= 1 && batch <= w->max_b, "batch must be in [1, max_batch]");
  HB_CHECK_ARG(xdt == HB_BF16 || xdt == HB_F32, "x_dtype must be HB_BF16 or HB_F32");
  HB_CHECK_ARG(ldx >= m->dims[0], "ldx < n_0");
  if (m->prec == HB_PREC_BF16) {
    HB_CHECK_ARG(xdt == HB_BF16, "bf16 model needs HB_BF16 input");
    HB_CHECK_ARG((ldx * 2) % 16 == 0, "ldx*2 must be a multiple of 16 bytes (pad n_0 to a multiple of 8)");
    HB_CHECK_ARG((reinterpret_cast<uintptr_t>(X) & 15) == 0, "X must be 16-byte aligned");
  }
  return HB_OK;
}

void sum_rows_into(hb_worker* w, int b, double* dst, cudaStream_t s, bool accumulate) {
  Prof pr(HB_PROF_OTHER, s);
  sum_rows_kernel<<<1, 1024, 0, s>>>(w->row_loss, b, dst, 0, accumulate ? 1 : 0);
  pr.done(1, 0.0, 4.0 * b);
}

int finish_loss(hb_worker* w, int b, float* loss_out, cudaStream_t s) {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  sum_rows_kernel<<<1, 1024, 0, s>>>(w->row_loss, b, w->dsum, 0);
  HB_CUDA_TRY(cudaGetLastError());
  HB_CUDA_TRY(cudaMemcpyAsync(w->h_dsum, w->dsum, sizeof(double), cudaMemcpyDeviceToHost, s));
  HB_CUDA_TRY(cudaStreamSynchronize(s));
  *loss_out = (float)(w->h_dsum[0] / (double)b);
  return HB_OK;
}

}  // namespace hb

extern "C" {

const char* hb_last_error(void) { return hb::g_err.c_str(); }

int64_t hb_kernel_launches(void) { return hb::g_launches.load(); }

int hb_prof_enable(int32_t on) {
  hb::g_prof_on.store(on != 0);
  return HB_OK;
}

int hb_prof_read(hb_prof_entry* out, int32_t n, int32_t reset) {
  HB_CHECK_ARG(out || n == 0, "null out");
  HB_CUDA_TRY(cudaDeviceSynchronize());
  std::lock_guard<std::mutex> g(hb::g_prof_mu);
  for (auto& r : hb::g_pend) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, r.e0, r.e1) == cudaSuccess) {
      for (int k = 0; k < 2; ++k) {
        if (k == 1 && (r.layer < 0 || r.layer >= HB_PROF_LAYERS)) break;
        hb_prof_entry& a = k == 0 ? hb::g_agg[r.cls] : hb::g_agg_l[r.cls][r.layer];
        a.launches += r.nl;
        a.ms += ms;
        a.flops += r.flops;
        a.bytes += r.bytes;
      }
    }
    hb::g_evpool.push_back(r.e0);
    hb::g_evpool.push_back(r.e1);
  }
  hb::g_pend.clear();
  for (int i = 0; i < n && i < HB_PROF_N; ++i) out[i] = hb::g_agg[i];
  for (int i = HB_PROF_N; i < n && i < HB_PROF_N * (1 + HB_PROF_LAYERS); ++i) {
    const int j = i - HB_PROF_N;
    out[i] = hb::g_agg_l[j / HB_PROF_LAYERS][j % HB_PROF_LAYERS];
  }
  if (reset) {
    for (auto& a : hb::g_agg) a = hb_prof_entry{};
    for (auto& row : hb::g_agg_l)
      for (auto& a : row) a = hb_prof_entry{};
  }
  return HB_OK;
}
int hb_abi_version(void) { return HB_ABI_VERSION; }

int hb_device_ok(int32_t device) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || device < 0 || device >= n) return 0;
  cudaDeviceProp p;
  if (cudaGetDeviceProperties(&p, device) != cudaSuccess) return 0;
  return p.major == 10 ? 1 : 0;
}

int mlp_create(const int32_t* dims, int32_t n_dims, int32_t activation, int32_t precision, uint64_t seed,
               int32_t device, hb_model** out) {
  HB_CHECK_ARG(out, "null out");
  *out = nullptr;
  HB_CHECK_ARG(dims && n_dims >= 2, "need n_dims >= 2");
  for (int i = 0; i < n_dims; ++i) HB_CHECK_ARG(dims[i] > 0, "all dims must be > 0");
  HB_CHECK_ARG(dims[n_dims - 1] >= 2, "need at least 2 classes");
  if (activation != HB_SIGMOID) return fail(HB_EUNSUPPORTED, "only HB_SIGMOID hidden activation (PAPER.md L258)");
  HB_CHECK_ARG(precision == HB_PREC_BF16 || precision == HB_PREC_FP32_CHECK, "bad precision");
  HB_CUDA_TRY(cudaSetDevice(device));
  if (precision == HB_PREC_BF16 && !hb_device_ok(device))
    return fail(HB_EUNSUPPORTED, "bf16 tensor-core path needs an sm_100 (B200) device");
  hb_model* m = new hb_model();
  m->device = device;
  m->prec = precision;
  m->dims.assign(dims, dims + n_dims);
  // fused row-block path from this batch size up (measured crossover on B200, DESIGN.md §5:
  // C2 fused 104.5 vs 109.1 us at 4096, 173 vs 88 at 2048); other options: model.h defaults
  size_t off = 0;
  for (int l = 1; l < n_dims; ++l) {
    Layer Ly;
    Ly.n_in = dims[l - 1];
    Ly.n_out = dims[l];
    Ly.ldw = (int)round_up(Ly.n_in, 8);
    Ly.ldo = (int)round_up(Ly.n_out, 8);
    Ly.w_off = round_up(off, 16);
    Ly.b_off = round_up(Ly.w_off + (size_t)Ly.n_out * Ly.ldw, 16);
    off = Ly.b_off + Ly.n_out;
    m->layers.push_back(Ly);
  }
  m->total = round_up(off, 16);
  if (cudaMalloc(&m->master, m->total * 4) != cudaSuccess ||
      (precision == HB_PREC_BF16 && cudaMalloc(&m->shadow, m->total * 2) != cudaSuccess)) {
    cudaFree(m->master);
    delete m;
    return fail(HB_ENOMEM, "model alloc");
  }
  // blocking stream: ordered after the caller's legacy-stream work (e.g. torch copies)
  if (cudaStreamCreate(&m->stream) != cudaSuccess) {
    cudaFree(m->master);
    cudaFree(m->shadow);
    delete m;
    return fail(HB_ECUDA, "stream create");
  }
  // W ~ N(0, 1/fan_in), b = 0 (R11)
  std::vector<float> h(m->total, 0.f);
  std::mt19937_64 gen(seed);
  std::normal_distribution<double> nd(0.0, 1.0);
  for (const Layer& Ly : m->layers) {
    const double sd = 1.0 / std::sqrt((double)Ly.n_in);
    for (int i = 0; i < Ly.n_out; ++i)
      for (int j = 0; j < Ly.n_in; ++j) h[Ly.w_off + (size_t)i * Ly.ldw + j] = (float)(nd(gen) * sd);
  }
  int rc = [&]() -> int {
    // copy and shadow refresh on the same stream: a pageable cudaMemcpy may return before its
    // DMA lands, so the refresh must be stream-ordered after it
    HB_CUDA_TRY(cudaMemcpyAsync(m->master, h.data(), m->total * 4, cudaMemcpyHostToDevice, m->stream));
    if (m->shadow) {
      refresh_shadow_kernel<<<256, 256, 0, m->stream>>>(m->master, m->shadow, (int64_t)m->total);
      HB_CUDA_TRY(cudaGetLastError());
    }
    HB_CUDA_TRY(cudaStreamSynchronize(m->stream));
    return HB_OK;
  }();
  if (rc) {
    mlp_destroy(m);
    return rc;
  }
  *out = m;
  return HB_OK;
}

int mlp_destroy(hb_model* m) {
  if (!m) return HB_OK;
  cudaSetDevice(m->device);
  cudaDeviceSynchronize();
  for (void* p : m->ipc_opened) cudaIpcCloseMemHandle(p);
  if (m->eval) mlp_worker_destroy(m->eval);
  cudaFree(m->master);
  cudaFree(m->shadow);
  cudaFree(m->base);
  cudaFree(m->delta);
  cudaFree(m->chunk_sums);
  cudaFree(m->stage_x);
  cudaFree(m->stage_y);
  cudaFree(m->csr_ptr);
  cudaFree(m->csr_idx);
  cudaFree(m->csr_val);
  for (cudaEvent_t e : m->stage_ev) cudaEventDestroy(e);
  if (m->copy_stream) cudaStreamDestroy(m->copy_stream);
  if (m->stream) cudaStreamDestroy(m->stream);
  delete m;
  return HB_OK;
}

}  // extern "C"

namespace hb {
int densify_csr_rows(const int64_t* indptr, const int32_t* indices, const void* vals, int xdt, int64_t r0, int64_t r1,
                     int64_t n_cols, void* X, int64_t ldx, cudaStream_t s, int* bad, bool zero_first) {
  const size_t es = xdt == HB_BF16 ? 2 : 4;
  if (zero_first)
    HB_CUDA_TRY(cudaMemsetAsync(static_cast<char*>(X) + (size_t)r0 * ldx * es, 0, (size_t)(r1 - r0) * ldx * es, s));
  if (!vals) {  // zero the nonzeros of rows [r0, r1) only (the rest of the rows is already zero)
    const unsigned blocks0 = (unsigned)(((r1 - r0) * 32 + 255) / 256);
    if (xdt == HB_BF16)
      zero_csr_kernel<__nv_bfloat16><<<blocks0, 256, 0, s>>>(indptr, indices, r0, r1, n_cols, static_cast<__nv_bfloat16*>(X), ldx);
    else
      zero_csr_kernel<float><<<blocks0, 256, 0, s>>>(indptr, indices, r0, r1, n_cols, static_cast<float*>(X), ldx);
    HB_CUDA_TRY(cudaGetLastError());
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return HB_OK;
  }
  const int64_t warps = r1 - r0;
  const unsigned blocks = (unsigned)((warps * 32 + 255) / 256);
  if (xdt == HB_BF16)
    densify_csr_kernel<__nv_bfloat16><<<blocks, 256, 0, s>>>(indptr, indices, static_cast<const __nv_bfloat16*>(vals),
                                                             r0, r1, n_cols, static_cast<__nv_bfloat16*>(X), ldx, bad);
  else
    densify_csr_kernel<float><<<blocks, 256, 0, s>>>(indptr, indices, static_cast<const float*>(vals), r0, r1, n_cols,
                                                     static_cast<float*>(X), ldx, bad);
  HB_CUDA_TRY(cudaGetLastError());
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return HB_OK;
}

int check_labels_dev(const int32_t* y, int64_t n, int C, int device, bool* ok) {
  HB_CUDA_TRY(cudaSetDevice(device));
  int* d = nullptr;
  HB_CUDA_TRY(cudaMalloc(&d, sizeof(int)));
  int h = 0;
  cudaMemset(d, 0, sizeof(int));
  check_labels_kernel<<<592, 256>>>(y, n, C, d);
  cudaError_t e = cudaMemcpy(&h, d, sizeof(int), cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return fail(HB_ECUDA, std::string("label check: ") + cudaGetErrorString(e));
  *ok = h == 0;
  return HB_OK;
}

// A deep replica of m (same shape, options and device): private fp32 master + bf16 shadow holding
// a copy of m's current parameters.
int clone_model(hb_model* m, hb_model** out) {
  hb_model* r = nullptr;
  int rc = mlp_create(m->dims.data(), (int32_t)m->dims.size(), HB_SIGMOID, m->prec, 0, m->device, &r);
  if (rc) return rc;
  r->rc_min_b = m->rc_min_b;
  r->opt_rowchain = m->opt_rowchain;
  r->opt_rc_cluster = m->opt_rc_cluster;
  r->opt_bwd_overlap = m->opt_bwd_overlap;
  r->opt_head_fuse = m->opt_head_fuse;
  r->opt_dw_pair = m->opt_dw_pair;
  r->opt_gemm_pair = m->opt_gemm_pair;
  r->opt_head_kernel = m->opt_head_kernel;
  r->opt_pdl = m->opt_pdl;
  r->opt_graphs = m->opt_graphs;
  r->opt_inflight = m->opt_inflight;
  r->opt_stage_rows = m->opt_stage_rows;
  r->opt_update = m->opt_update;
  r->opt_step_kernel_max_b = m->opt_step_kernel_max_b;
  if (cudaDeviceSynchronize() != cudaSuccess ||
      cudaMemcpy(r->master, m->master, m->total * 4, cudaMemcpyDeviceToDevice) != cudaSuccess ||
      (m->shadow && cudaMemcpy(r->shadow, m->shadow, m->total * 2, cudaMemcpyDeviceToDevice) != cudaSuccess)) {
    mlp_destroy(r);
    return fail(HB_ECUDA, "replica copy");
  }
  *out = r;
  return HB_OK;
}
}  // namespace hb

extern "C" {

int mlp_num_params(const hb_model* m, int64_t* n_out) {
  HB_CHECK_ARG(m && n_out, "null arg");
  int64_t n = 0;
  for (const Layer& Ly : m->layers) n += (int64_t)Ly.n_out * Ly.n_in + Ly.n_out;
  *n_out = n;
  return HB_OK;
}

#ifdef HB_TUNING
// Tuning only: cap > 0 arms per-step phase stamps in every later rowchain launch (the buffer is
// overwritten by each launch); cap == 0 copies the last launch's stamps to host and disarms.
int hb_rc_trace(unsigned long long* host, int64_t cap) {
  if (cap > 0 && !host) {
    cudaFree(g_rc_trace);
    g_rc_trace = nullptr;
    HB_CUDA_TRY(cudaMalloc(&g_rc_trace, cap * sizeof(unsigned long long)));
    HB_CUDA_TRY(cudaMemset(g_rc_trace, 0, cap * sizeof(unsigned long long)));
    g_rc_trace_cap = cap;
    return HB_OK;
  }
  HB_CHECK_ARG(host && cap > 0, "bad args");
  HB_CUDA_TRY(cudaDeviceSynchronize());
  HB_CUDA_TRY(cudaMemcpy(host, g_rc_trace, std::min(cap, g_rc_trace_cap) * sizeof(unsigned long long),
                         cudaMemcpyDeviceToHost));
  HB_CUDA_TRY(cudaMemset(g_rc_trace, 0, g_rc_trace_cap * sizeof(unsigned long long)));
  return HB_OK;
}

// Tuning only: mean device microseconds of one SGD step of worker w on rows [0, batch) of (X, y),
// captured once into a CUDA graph and replayed `iters` times back to back (lr = 0: the model
// is unchanged).  part = 0 whole step, 1 fused chain only (dW GEMMs skipped), 2 dW GEMMs only.
int hb_bench_step(hb_worker* w, const void* X, int64_t ldx, const int32_t* y, int32_t batch, int32_t iters,
                  int32_t part, float* us_out) {
  int rc = check_step_args(w, X, ldx, HB_BF16, y, batch);
  if (rc) return rc;
  HB_CHECK_ARG(us_out && iters > 0 && part >= 0 && part <= 2, "bad args");
  HB_CHECK_ARG(w->m->prec == HB_PREC_BF16 && w->subs.empty(), "bf16 plain worker only");
  HB_CUDA_TRY(cudaSetDevice(w->m->device));
  cudaStream_t s = w->stream;
  g_bench_part = part;
  rc = run_step(w, X, ldx, HB_BF16, batch, y, nullptr, batch, 0.f, false, s);  // warm-up, attributes
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  if (!rc) {
    HB_CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    for (int i = 0; i < iters && !rc; ++i) rc = run_step(w, X, ldx, HB_BF16, batch, y, nullptr, batch, 0.f, false, s);
    cudaError_t ce = cudaStreamEndCapture(s, &g);
    if (!rc && ce != cudaSuccess) rc = fail(HB_ECUDA, std::string("capture: ") + cudaGetErrorString(ce));
  }
  g_bench_part = 0;
  if (rc) {
    if (g) cudaGraphDestroy(g);
    return rc;
  }
  HB_CUDA_TRY(cudaGraphInstantiate(&ge, g, 0));
  cudaGraphDestroy(g);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaGraphLaunch(ge, s);  // warm
  cudaEventRecord(e0, s);
  cudaGraphLaunch(ge, s);
  cudaEventRecord(e1, s);
  cudaError_t ce = cudaStreamSynchronize(s);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  *us_out = ms * 1000.f / iters;
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaGraphExecDestroy(ge);
  if (ce != cudaSuccess) return fail(HB_ECUDA, std::string("bench step: ") + cudaGetErrorString(ce));
  return HB_OK;
}

#endif  // HB_TUNING

int mlp_set_option(hb_model* m, int32_t key, int64_t v) {
  HB_CHECK_ARG(m, "null model");
  auto flag = [&](int* dst) -> int {
    HB_CHECK_ARG(v == 0 || v == 1, "option value must be 0 or 1");
    *dst = (int)v;
    return HB_OK;
  };
  switch (key) {
    case HB_OPT_FUSED_MIN_BATCH:
      HB_CHECK_ARG(v >= 0 && v <= (1 << 30), "fused min batch must be >= 0");
      m->rc_min_b = (int)v;
      return HB_OK;
    case HB_OPT_ROWCHAIN: return flag(&m->opt_rowchain);
    case HB_OPT_RC_CLUSTER:
      HB_CHECK_ARG(v == 0 || v == 1 || v == 2 || v == 4 || v == 8, "cluster size must be 0, 1, 2, 4 or 8");
      m->opt_rc_cluster = (int)v;
      return HB_OK;
    case HB_OPT_BWD_OVERLAP: return flag(&m->opt_bwd_overlap);
    case HB_OPT_HEAD_FUSE: return flag(&m->opt_head_fuse);
    case HB_OPT_DW_PAIR: return flag(&m->opt_dw_pair);
    case HB_OPT_GEMM_PAIR: return flag(&m->opt_gemm_pair);
    case HB_OPT_HEAD_KERNEL: return flag(&m->opt_head_kernel);
    case HB_OPT_PDL: return flag(&m->opt_pdl);
    case HB_OPT_GRAPHS: return flag(&m->opt_graphs);
    case HB_OPT_INFLIGHT:
      HB_CHECK_ARG(v >= 0 && v <= HB_MAX_INFLIGHT, "in-flight depth must be 0 (auto) .. 4");
      m->opt_inflight = (int)v;
      return HB_OK;
    case HB_OPT_STAGE_ROWS:
      HB_CHECK_ARG(v >= 0, "staging rows must be >= 0");
      m->opt_stage_rows = v;
      return HB_OK;
    case HB_OPT_UPDATE:
      HB_CHECK_ARG(v == HB_UPDATE_HOGWILD || v == HB_UPDATE_ATOMIC, "update must be HB_UPDATE_HOGWILD or _ATOMIC");
      m->opt_update = (int)v;
      return HB_OK;
    case HB_OPT_STEP_KERNEL_MAX_B:
      HB_CHECK_ARG(v >= 0 && v <= (1 << 20), "step-kernel max batch must be >= 0");
      m->opt_step_kernel_max_b = (int)v;
      return HB_OK;
    default: return fail(HB_EINVAL, "unknown option key");
  }
}

int mlp_get_option(const hb_model* m, int32_t key, int64_t* v) {
  HB_CHECK_ARG(m && v, "null arg");
  switch (key) {
    case HB_OPT_FUSED_MIN_BATCH: *v = m->rc_min_b; return HB_OK;
    case HB_OPT_ROWCHAIN: *v = m->opt_rowchain; return HB_OK;
    case HB_OPT_RC_CLUSTER: *v = m->opt_rc_cluster; return HB_OK;
    case HB_OPT_BWD_OVERLAP: *v = m->opt_bwd_overlap; return HB_OK;
    case HB_OPT_HEAD_FUSE: *v = m->opt_head_fuse; return HB_OK;
    case HB_OPT_DW_PAIR: *v = m->opt_dw_pair; return HB_OK;
    case HB_OPT_GEMM_PAIR: *v = m->opt_gemm_pair; return HB_OK;
    case HB_OPT_HEAD_KERNEL: *v = m->opt_head_kernel; return HB_OK;
    case HB_OPT_PDL: *v = m->opt_pdl; return HB_OK;
    case HB_OPT_GRAPHS: *v = m->opt_graphs; return HB_OK;
    case HB_OPT_INFLIGHT: *v = m->opt_inflight; return HB_OK;
    case HB_OPT_STAGE_ROWS: *v = m->opt_stage_rows; return HB_OK;
    case HB_OPT_UPDATE: *v = m->opt_update; return HB_OK;
    case HB_OPT_STEP_KERNEL_MAX_B: *v = m->opt_step_kernel_max_b; return HB_OK;
    default: return fail(HB_EINVAL, "unknown option key");
  }
}

int mlp_fused_path(const hb_model* m, int32_t batch, int32_t* cluster_size) {
  HB_CHECK_ARG(m && cluster_size, "null arg");
  const RcCfg c = rowchain_cfg(m, batch > 0 ? batch : 8192);
  *cluster_size = c.ok ? c.CS : 0;
  return c.ok ? 1 : 0;
}

int mlp_get_params(const hb_model* m, float* host_dst, int64_t n) {
  int64_t need;
  int rc = mlp_num_params(m, &need);
  if (rc) return rc;
  HB_CHECK_ARG(host_dst && n == need, "n must equal mlp_num_params");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  HB_CUDA_TRY(cudaDeviceSynchronize());  // every worker's in-place updates are visible
  // the copy engine drops the row padding (pitched copies straight into the caller's buffer)
  int64_t o = 0;
  for (const Layer& Ly : m->layers) {
    HB_CUDA_TRY(cudaMemcpy2DAsync(host_dst + o, (size_t)Ly.n_in * 4, m->master + Ly.w_off, (size_t)Ly.ldw * 4,
                                  (size_t)Ly.n_in * 4, (size_t)Ly.n_out, cudaMemcpyDeviceToHost, m->stream));
    o += (int64_t)Ly.n_out * Ly.n_in;
    HB_CUDA_TRY(cudaMemcpyAsync(host_dst + o, m->master + Ly.b_off, (size_t)Ly.n_out * 4, cudaMemcpyDeviceToHost,
                                m->stream));
    o += Ly.n_out;
  }
  HB_CUDA_TRY(cudaStreamSynchronize(m->stream));
  return HB_OK;
}

int mlp_set_params(hb_model* m, const float* host_src, int64_t n) {
  int64_t need;
  int rc = mlp_num_params(m, &need);
  if (rc) return rc;
  HB_CHECK_ARG(host_src && n == need, "n must equal mlp_num_params");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  std::vector<float> h(m->total, 0.f);
  int64_t o = 0;
  for (const Layer& Ly : m->layers) {
    for (int i = 0; i < Ly.n_out; ++i)
      for (int j = 0; j < Ly.n_in; ++j) h[Ly.w_off + (size_t)i * Ly.ldw + j] = host_src[o++];
    for (int i = 0; i < Ly.n_out; ++i) h[Ly.b_off + i] = host_src[o++];
  }
  HB_CUDA_TRY(cudaDeviceSynchronize());
  HB_CUDA_TRY(cudaMemcpyAsync(m->master, h.data(), m->total * 4, cudaMemcpyHostToDevice, m->stream));
  if (m->shadow) {
    refresh_shadow_kernel<<<256, 256, 0, m->stream>>>(m->master, m->shadow, (int64_t)m->total);
    HB_CUDA_TRY(cudaGetLastError());
  }
  HB_CUDA_TRY(cudaStreamSynchronize(m->stream));
  return HB_OK;
}

static void detach_peers(hb_model* m) {
  for (void* p : m->ipc_opened) cudaIpcCloseMemHandle(p);
  m->ipc_opened.clear();
  m->peers.clear();
}

int mlp_attach_peers(hb_model* m, hb_model* const* peers, int32_t n, float scale) {
  HB_CHECK_ARG(m && n >= 0 && n <= HB_MAX_PEERS && (n == 0 || peers), "0 <= n <= 7 peers");
  HB_CHECK_ARG(scale >= 0.f, "scale must be >= 0");
  if (m->prec != HB_PREC_BF16) return fail(HB_EUNSUPPORTED, "peer replicas: bf16 models only");
  for (int i = 0; i < n; ++i) {
    HB_CHECK_ARG(peers[i] && peers[i] != m && peers[i]->dims == m->dims && peers[i]->prec == m->prec,
                 "peers must be other models of identical shape");
    if (peers[i]->device != m->device) {  // another GPU of this process: peer-to-peer access
      int can = 0;
      cudaDeviceCanAccessPeer(&can, m->device, peers[i]->device);
      if (!can) return fail(HB_EUNSUPPORTED, "no peer-to-peer access between the models' devices");
      HB_CUDA_TRY(cudaSetDevice(m->device));
      cudaError_t e = cudaDeviceEnablePeerAccess(peers[i]->device, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return fail(HB_ECUDA, "enable peer access");
      cudaGetLastError();
    }
  }
  detach_peers(m);
  for (int i = 0; i < n; ++i) m->peers.push_back({peers[i]->master, peers[i]->shadow});
  m->peer_scale = scale;
  return HB_OK;
}

int mlp_ipc_handle(const hb_model* m, uint8_t out[128]) {
  HB_CHECK_ARG(m && out, "null arg");
  if (m->prec != HB_PREC_BF16) return fail(HB_EUNSUPPORTED, "peer replicas: bf16 models only");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  cudaIpcMemHandle_t hm, hs;
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "ipc handle size");
  HB_CUDA_TRY(cudaIpcGetMemHandle(&hm, m->master));
  HB_CUDA_TRY(cudaIpcGetMemHandle(&hs, m->shadow));
  std::memcpy(out, &hm, 64);
  std::memcpy(out + 64, &hs, 64);
  return HB_OK;
}

int mlp_attach_ipc_peers(hb_model* m, const uint8_t* handles, int32_t n, float scale) {
  HB_CHECK_ARG(m && n >= 0 && n <= HB_MAX_PEERS && (n == 0 || handles), "0 <= n <= 7 peers");
  HB_CHECK_ARG(scale >= 0.f, "scale must be >= 0");
  if (m->prec != HB_PREC_BF16) return fail(HB_EUNSUPPORTED, "peer replicas: bf16 models only");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  HB_CUDA_TRY(cudaDeviceSynchronize());
  detach_peers(m);
  for (int i = 0; i < n; ++i) {
    cudaIpcMemHandle_t hm, hs;
    std::memcpy(&hm, handles + 128 * i, 64);
    std::memcpy(&hs, handles + 128 * i + 64, 64);
    void *pm = nullptr, *ps = nullptr;
    if (cudaIpcOpenMemHandle(&pm, hm, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess ||
        cudaIpcOpenMemHandle(&ps, hs, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      cudaGetLastError();
      if (pm) cudaIpcCloseMemHandle(pm);
      detach_peers(m);
      return fail(HB_ECUDA, "cudaIpcOpenMemHandle of a peer replica failed");
    }
    m->ipc_opened.push_back(pm);
    m->ipc_opened.push_back(ps);
    m->peers.push_back({static_cast<float*>(pm), static_cast<__nv_bfloat16*>(ps)});
  }
  m->peer_scale = scale;
  return HB_OK;
}

int mlp_worker_create(hb_model* m, int32_t device, int32_t max_batch, int32_t replica, void* cuda_stream,
                      hb_worker** out) {
  HB_CHECK_ARG(m && out, "null arg");
  *out = nullptr;
  HB_CHECK_ARG(max_batch >= 1, "max_batch must be >= 1");
  HB_CHECK_ARG(replica == 0 || replica == 1, "replica must be 0 (reference) or 1 (deep)");
  if (device >= 0 && device != m->device)
    return fail(HB_EUNSUPPORTED, "a worker runs on its model's device (one model per GPU; multi-GPU = one "
                                 "process per GPU with a shared coordinator, hb_coord_create)");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  hb_model* target = m;
  if (replica == 1) {  // deep replica [L134, L174]: a private copy of the global model's parameters
    int rc = clone_model(m, &target);
    if (rc) return rc;
  }
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  bool own = false;
  if (!s) {
    // a blocking stream: ordered after work on the legacy default stream (e.g. the caller's
    // torch copies of X/y), concurrent with the other workers' streams (Hogbatch, L170)
    if (cudaStreamCreate(&s) != cudaSuccess) {
      if (target != m) mlp_destroy(target);
      return fail(HB_ECUDA, "stream create");
    }
    own = true;
  }
  int rc = alloc_worker(target, max_batch, s, own, out);  // frees its own stream on failure
  if (rc) {
    if (target != m) mlp_destroy(target);
    return rc;
  }
  (*out)->global = m;
  return HB_OK;
}

int mlp_worker_params(hb_worker* w, float* host_dst, int64_t n) {
  HB_CHECK_ARG(w, "null worker");
  return mlp_get_params(w->m, host_dst, n);
}

int mlp_worker_destroy(hb_worker* w) {
  if (!w) return HB_OK;
  cudaSetDevice(w->m->device);
  cudaStreamSynchronize(w->stream);
  hb_model* replica = w->global && w->global != w->m ? w->m : nullptr;
  for (hb_worker* sw : w->subs) mlp_worker_destroy(sw);
  w->subs.clear();
  if (w->ev_fork) cudaEventDestroy(w->ev_fork);
  for (cudaEvent_t e : w->ev_join) cudaEventDestroy(e);
  w->ev_join.clear();
  free_worker_buffers(w);
  if (w->own_stream) cudaStreamDestroy(w->stream);
  delete w;
  if (replica) mlp_destroy(replica);
  return HB_OK;
}

void* mlp_worker_stream(hb_worker* w) { return w ? (void*)w->stream : nullptr; }

int mlp_worker_create_nested(hb_model* m, int32_t max_batch, int32_t t, void* cuda_stream, hb_worker** out) {
  HB_CHECK_ARG(m && out, "null arg");
  *out = nullptr;
  HB_CHECK_ARG(t >= 1 && max_batch >= t, "need 1 <= t <= max_batch");
  hb_worker* w = nullptr;
  int rc = mlp_worker_create(m, -1, 1, 0, cuda_stream, &w);  // parent: stream + events only
  if (rc) return rc;
  w->max_b = max_batch;
  const int sub_max = (max_batch + t - 1) / t;
  for (int i = 0; i < t; ++i) {
    hb_worker* sw = nullptr;
    rc = mlp_worker_create(m, -1, sub_max, 0, nullptr, &sw);
    if (rc) {
      mlp_worker_destroy(w);
      return rc;
    }
    cudaFree(sw->sk_bar);  // t concurrent sub-steps: per-layer launches, no cooperative grids
    sw->sk_bar = nullptr;
    w->subs.push_back(sw);
    cudaEvent_t e;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    w->ev_join.push_back(e);
  }
  cudaEventCreateWithFlags(&w->ev_fork, cudaEventDisableTiming);
  *out = w;
  return HB_OK;
}

int mlp_step(hb_worker* w, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y, int32_t batch, float lr,
             float* loss_out) {
  int rc = check_step_args(w, X, ldx, x_dtype, y, batch);
  if (rc) return rc;
  HB_CUDA_TRY(cudaSetDevice(w->m->device));
  if (!w->subs.empty()) {  // nested worker: t concurrent sub-batches
    rc = worker_execute(w, X, ldx, x_dtype, batch, y, 0, batch, lr, false, false, loss_out ? w->dsum : nullptr);
    if (rc || !loss_out) return rc;
    HB_CUDA_TRY(cudaMemcpyAsync(w->h_dsum, w->dsum, sizeof(double), cudaMemcpyDeviceToHost, w->stream));
    HB_CUDA_TRY(cudaStreamSynchronize(w->stream));
    *loss_out = (float)(w->h_dsum[0] / (double)batch);
    return HB_OK;
  }
  rc = run_step(w, X, ldx, x_dtype, batch, y, nullptr, batch, lr, false, w->stream);
  if (rc) return rc;
  if (loss_out) return finish_loss(w, batch, loss_out, w->stream);
  return HB_OK;
}

int mlp_step_grads(hb_worker* w, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y, int32_t batch,
                   float* host_grads, int64_t n, float* loss_out) {
  int rc = check_step_args(w, X, ldx, x_dtype, y, batch);
  if (rc) return rc;
  hb_model* m = w->m;
  if (!w->subs.empty()) return fail(HB_EUNSUPPORTED, "mlp_step_grads on a nested worker");
  int64_t need;
  mlp_num_params(m, &need);
  HB_CHECK_ARG(host_grads && n == need, "n must equal mlp_num_params");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  if (!w->grads) HB_CUDA_TRY(cudaMalloc(&w->grads, m->total * 4));
  HB_CUDA_TRY(cudaMemsetAsync(w->grads, 0, m->total * 4, w->stream));
  rc = run_step(w, X, ldx, x_dtype, batch, y, nullptr, batch, 0.f, true, w->stream);
  if (rc) return rc;
  std::vector<float> h(m->total);
  HB_CUDA_TRY(cudaMemcpyAsync(h.data(), w->grads, m->total * 4, cudaMemcpyDeviceToHost, w->stream));
  HB_CUDA_TRY(cudaStreamSynchronize(w->stream));
  int64_t o = 0;
  for (const Layer& Ly : m->layers) {
    for (int i = 0; i < Ly.n_out; ++i)
      for (int j = 0; j < Ly.n_in; ++j) host_grads[o++] = h[Ly.w_off + (size_t)i * Ly.ldw + j];
    for (int i = 0; i < Ly.n_out; ++i) host_grads[o++] = h[Ly.b_off + i];
  }
  if (loss_out) return finish_loss(w, batch, loss_out, w->stream);
  return HB_OK;
}

int mlp_row_losses(hb_worker* w, float* host_dst, int32_t n) {
  HB_CHECK_ARG(w && host_dst && n >= 1 && n <= w->max_b, "n must be in [1, max_batch]");
  if (!w->subs.empty()) return fail(HB_EUNSUPPORTED, "mlp_row_losses on a nested worker");
  HB_CUDA_TRY(cudaSetDevice(w->m->device));
  HB_CUDA_TRY(cudaMemcpyAsync(host_dst, w->row_loss, (size_t)n * 4, cudaMemcpyDeviceToHost, w->stream));
  HB_CUDA_TRY(cudaStreamSynchronize(w->stream));
  return HB_OK;
}

#ifdef HB_TUNING
// Test/tuning only: times `iters` launches of one tensor-core GEMM configuration on scratch
// buffers (bf16 operands filled with zeros, fp32 master); kind 0 = forward (bias+sigmoid),
// 1 = dgrad (sigma'), 2 = wgrad + SGD.  Reports the mean device microseconds per launch.
static int bench_gemm_impl(int32_t kind, int32_t M, int32_t N, int32_t K, int32_t iters, float* us_out,
                           unsigned long long* host_ts, int64_t cap);
int hb_bench_gemm(int32_t kind, int32_t M, int32_t N, int32_t K, int32_t iters, float* us_out) {
  return bench_gemm_impl(kind, M, N, K, iters, us_out, nullptr, 0);
}

// Unfused SGD baseline: W -= lr * G over n fp32 weights with the bf16 shadow rewritten,
// G read from HBM — 14 bytes per weight (W and G read, W and shadow written)
static __global__ void sgd_apply_kernel(float* __restrict__ W, const float* __restrict__ G, __nv_bfloat16* __restrict__ Sh,
                                        int64_t n4, float lr) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    float4 w = reinterpret_cast<float4*>(W)[i];
    const float4 g = __ldcs(reinterpret_cast<const float4*>(G) + i);
    w.x += __fmul_rn(-lr, g.x);
    w.y += __fmul_rn(-lr, g.y);
    w.z += __fmul_rn(-lr, g.z);
    w.w += __fmul_rn(-lr, g.w);
    reinterpret_cast<float4*>(W)[i] = w;
    reinterpret_cast<uint2*>(Sh)[i] = make_uint2(pack_bf16x2(w.x, w.y), pack_bf16x2(w.z, w.w));
  }
}
// tuning only: mean device microseconds of sgd_apply_kernel over n weights (graph of iters launches)
int hb_bench_sgd_apply(int64_t n, int32_t iters, float* us_out) {
  HB_CHECK_ARG(us_out && n > 0 && n % 4 == 0 && iters > 0, "bad args");
  float *W = nullptr, *G = nullptr;
  __nv_bfloat16* Sh = nullptr;
  if (cudaMalloc(&W, n * 4) || cudaMalloc(&G, n * 4) || cudaMalloc(&Sh, n * 2)) return fail(HB_ENOMEM, "bench alloc");
  cudaMemset(W, 0, n * 4);
  cudaMemset(G, 0, n * 4);
  cudaStream_t s;
  cudaStreamCreate(&s);
  int nsm = 148;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int grid = nsm * 8;
  sgd_apply_kernel<<<grid, 256, 0, s>>>(W, G, Sh, n / 4, 0.f);
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  for (int i = 0; i < iters; ++i) sgd_apply_kernel<<<grid, 256, 0, s>>>(W, G, Sh, n / 4, 0.f);
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaGraphLaunch(ge, s);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, s);
  cudaGraphLaunch(ge, s);
  cudaEventRecord(e1, s);
  cudaError_t ce = cudaStreamSynchronize(s);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  *us_out = ms * 1000.f / iters;
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  cudaStreamDestroy(s);
  cudaFree(W);
  cudaFree(G);
  cudaFree(Sh);
  if (ce != cudaSuccess) return fail(HB_ECUDA, std::string("bench sgd apply: ") + cudaGetErrorString(ce));
  return HB_OK;
}
// tuning only: per-CTA phase timestamps of one launch (8 globaltimer values per CTA)
int hb_bench_gemm_phases(int32_t kind, int32_t M, int32_t N, int32_t K, unsigned long long* host_ts, int64_t cap) {
  float us = 0.f;
  return bench_gemm_impl(kind, M, N, K, 1, &us, host_ts, cap);
}
static int bench_gemm_impl(int32_t kind, int32_t M, int32_t N, int32_t K, int32_t iters, float* us_out,
                           unsigned long long* host_ts, int64_t cap) {
  HB_CHECK_ARG(us_out && M > 0 && N > 0 && K > 0 && iters > 0 && kind >= 0 && kind <= 3, "bad args");
  // kind 0 forward, 1 dX, 2 dW + fused SGD, 3 dW storing the fp32 gradient (the unfused baseline)
  const bool dw = kind >= 2;
  const int64_t lda = round_up(dw ? M : K, 8), ldb = round_up(kind == 0 ? K : N, 8);
  const int64_t ldo = round_up(N, 8);
  const int64_t arows = dw ? K : M, brows = kind == 0 ? N : K;
  void *A = nullptr, *B = nullptr, *O = nullptr, *S = nullptr;
  float *W = nullptr, *bias = nullptr, *ws = nullptr, *bp = nullptr;
  __nv_bfloat16* Wsh = nullptr;
  size_t out_elems = (size_t)std::max<int64_t>(M, 1) * ldo;
  if (cudaMalloc(&A, arows * lda * 2) || cudaMalloc(&B, brows * ldb * 2) || cudaMalloc(&O, out_elems * 2) ||
      cudaMalloc(&S, out_elems * 2) || cudaMalloc(&W, out_elems * 4) || cudaMalloc(&Wsh, out_elems * 2) ||
      cudaMalloc(&bias, ldo * 4 + 64) || cudaMalloc(&ws, (size_t)148 * TC_BM * 256 * 4) ||
      cudaMalloc(&bp, (size_t)((std::max(M, K) + 127) / 128) * std::max<int64_t>(ldo, M) * 4 + 4096))
    return fail(HB_ENOMEM, "bench alloc");
  cudaMemset(A, 0, arows * lda * 2);
  cudaMemset(B, 0, brows * ldb * 2);
  cudaMemset(W, 0, out_elems * 4);
  cudaMemset(bias, 0, ldo * 4 + 64);
  cudaMemset(S, 0, out_elems * 2);
  cudaMemset(bp, 0, (size_t)((std::max(M, K) + 127) / 128) * std::max<int64_t>(ldo, M) * 4 + 4096);  // wgrad: ldp = M
  cudaStream_t s;
  cudaStreamCreate(&s);
  EpiArgs ep{};
    ep.no_pdl = 0;
  ep.M = M;
  ep.N = N;
  int epi;
  bool a_mn = false, b_mn = false;
  if (kind == 0) {
    epi = EPI_FWD_SIG;
    ep.bias = bias;
    ep.out0 = O;
    ep.out1 = S;
    ep.ld0 = ep.ld1 = ldo;
  } else if (kind == 1) {
    epi = EPI_DGRAD_SIG;
    b_mn = true;
    ep.out0 = O;
    ep.ld0 = ldo;
    ep.aux = S;
    ep.ldaux = ldo;
    ep.bpart_out = bp;
    ep.ldp = N;
  } else {
    epi = kind == 3 ? EPI_WGRAD_STORE : EPI_WGRAD_SGD;
    a_mn = b_mn = true;
    ep.master = W;
    ep.shadow = Wsh;
    if (kind == 3) {
      ep.out0 = W;  // dW [M x ldo] fp32
      ep.bias_grad = bias;
    }
    ep.ldw = ldo;
    ep.lr = 0.f;
    ep.ws = ws;
    ep.bpart_in = bp;
    ep.ldp = M;
    ep.n_mtiles = (K + 127) / 128;
    ep.pair = HB_TUNE("HB_DW_PAIR", 0);           // tuning: CTA-pair dW
    ep.force_splits = HB_TUNE("HB_FORCE_SPLITS", 0);
    ep.bias_upd = bias;
  }
  ep.fwd_pair = HB_TUNE("HB_GEMM_PAIR", 0);  // tuning: CTA-pair forward / dX
  TcOp a{A, lda, arows, nullptr}, b{B, ldb, brows, nullptr};
  int rc = gemm_tc(epi, a_mn, b_mn, M, N, K, a, b, ep, s);  // warm-up (sets kernel attributes)
  if (host_ts && !rc) {
    unsigned long long* d = nullptr;
    cudaMalloc(&d, cap * sizeof(unsigned long long));
    cudaMemsetAsync(d, 0, cap * sizeof(unsigned long long), s);
    EpiArgs e2 = ep;
    e2.dbg = d;
    rc = gemm_tc(epi, a_mn, b_mn, M, N, K, a, b, e2, s);
    cudaMemcpyAsync(host_ts, d, cap * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    cudaFree(d);
  }
  // capture the launches in a graph so the timing is device time, not host launch cost
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  for (int i = 0; i < iters && !rc; ++i) rc = gemm_tc(epi, a_mn, b_mn, M, N, K, a, b, ep, s);
  cudaStreamEndCapture(s, &g);
  if (!rc && g) cudaGraphInstantiate(&ge, g, 0);
  if (ge) cudaGraphLaunch(ge, s);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, s);
  if (ge) cudaGraphLaunch(ge, s);
  cudaEventRecord(e1, s);
  cudaStreamSynchronize(s);
  if (ge) cudaGraphExecDestroy(ge);
  if (g) cudaGraphDestroy(g);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  *us_out = ms * 1000.f / iters;
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaStreamDestroy(s);
  cudaFree(A); cudaFree(B); cudaFree(O); cudaFree(S); cudaFree(W); cudaFree(Wsh); cudaFree(bias); cudaFree(ws);
  cudaFree(bp);
  const cudaError_t err = cudaGetLastError();
  if (!rc && err != cudaSuccess) return fail(HB_ECUDA, cudaGetErrorString(err));
  return rc;
}

#endif  // HB_TUNING

int mlp_loss(hb_model* m, const void* X, int64_t ldx, int32_t x_dtype, const int32_t* y, int64_t n,
             double* loss_out) {
  HB_CHECK_ARG(m && loss_out, "null arg");
  HB_CHECK_ARG(n >= 1, "n must be >= 1");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  HB_CUDA_TRY(cudaDeviceSynchronize());  // see every update enqueued before this call
  const int chunk = 8192;
  std::lock_guard<std::mutex> g(m->eval_mu);
  if (!m->eval) {
    int rc = alloc_worker(m, chunk, m->stream, false, &m->eval, false);
    if (rc) return rc;
  }
  hb_worker* w = m->eval;
  int rc = check_step_args(w, X, ldx, x_dtype, y, (int)std::min<int64_t>(n, chunk));
  if (rc) return rc;
  const int64_t nchunks = (n + chunk - 1) / chunk;
  if (m->chunk_cap < nchunks) {
    cudaFree(m->chunk_sums);
    m->chunk_sums = nullptr;
    HB_CUDA_TRY(cudaMalloc(&m->chunk_sums, nchunks * sizeof(double)));
    m->chunk_cap = nchunks;
  }
  const int L = (int)m->layers.size();
  const bool bf = m->prec == HB_PREC_BF16;
  const size_t xes = x_dtype == HB_BF16 ? 2 : 4;
  cudaStream_t s = w->stream;
  for (int64_t c = 0; c < nchunks; ++c) {
    const int64_t r0 = c * chunk;
    const int b = (int)std::min<int64_t>(chunk, n - r0);
    const void* Xc = static_cast<const char*>(X) + r0 * ldx * xes;
    if (bf) {
      rc = forward_tc(w, Xc, ldx, b, y + r0, nullptr, b, false, s, head_cfg(w, b));
      if (rc) return rc;
    } else {
      const void* Ain = Xc;
      int64_t lda = ldx;
      int adt = x_dtype;
      for (int l = 0; l < L; ++l) {
        const Layer& Ly = m->layers[l];
        EpiArgs ep{};
    ep.no_pdl = !m->opt_pdl;
        ep.M = b;
        ep.N = Ly.n_out;
        ep.bias = m->master + Ly.b_off;
        int epi = EPI_FWD_SIG;
        if (l < L - 1) {
          ep.out0 = w->H[l];
          ep.ld0 = Ly.ldo;
        } else {
          epi = EPI_FWD_LOGITS;
          ep.out0 = w->logits;
          ep.ld0 = w->ldc;
        }
        rc = gemm_simt_p(epi, false, false, b, Ly.n_out, Ly.n_in, Ain, lda, adt, m->master + Ly.w_off, Ly.ldw,
                         HB_F32, ep, s);
        if (rc) return rc;
        if (l < L - 1) {
          Ain = w->H[l];
          lda = Ly.ldo;
          adt = HB_F32;
        }
      }
      softmax_xent_kernel<float><<<(b * 32 + 255) / 256, 256, 0, s>>>(
          w->logits, w->ldc, y + r0, nullptr, b, m->layers.back().n_out, (float*)nullptr, 0, w->row_loss, 1.0f);
      g_launches.fetch_add(1, std::memory_order_relaxed);
    }
    sum_rows_kernel<<<1, 1024, 0, s>>>(w->row_loss, b, m->chunk_sums, (int)c);
    g_launches.fetch_add(1, std::memory_order_relaxed);
    HB_CUDA_TRY(cudaGetLastError());
  }
  std::vector<double> h(nchunks);
  HB_CUDA_TRY(cudaMemcpyAsync(h.data(), m->chunk_sums, nchunks * sizeof(double), cudaMemcpyDeviceToHost, s));
  HB_CUDA_TRY(cudaStreamSynchronize(s));
  double tot = 0.0;
  for (double v : h) tot += v;
  *loss_out = tot / (double)n;
  return HB_OK;
}

}  // extern "C"
