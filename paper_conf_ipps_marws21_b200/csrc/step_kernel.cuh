// step_kernel.cuh — the whole SGD step of a small batch in ONE persistent launch.
//
// Below the fused chain's batch sizes (b < HB_OPT_FUSED_MIN_BATCH) a step is 3L - 1 dependent
// GEMMs (forward, softmax-xent head, dX, dW + fused SGD; Eq. (1)-(3), L43-L53) whose
// tiles are few: each launch costs ~4 us of launch, prologue and tail for ~1 us of work
// (scripts/small_batch_probe.py: 58 us per C2 step at b = 32).  This kernel runs the same GEMMs
// with the same tcgen05/TMA mainloop and the same fused epilogues (tc_epilogue_tile), as a list of
// STAGES separated by grid-wide barriers: every CTA (one per SM, cooperative launch, all
// co-resident) processes its share of each stage's output tiles, then the CTAs meet before the
// next stage reads what this one wrote.  Stage order (L weight layers, 0-based l):
//   stage l        forward l                  l = 0..L-2
//   stage L-1      head (softmax-xent, hi/lo dZ_L)
//   stage 2L-1-l   dX of layer l              l = L-1..1
//   stage 2L-l     dW + SGD of layer l        l = L-1..2   (after dX_l, the last reader of W_l)
//   stage 2L-1     dW + SGD of layers 1 and 0
// so every dX read of W_l precedes the W_l update (Eq. (3) order) and no W_l is updated while a
// stage could still read it.  Tiles are 128 x 32 (head 128 x 16), never split-K (K = b is small).
//
// Barriers: per stage an arrival counter in global memory; the epilogue warps of a CTA arrive
// after their last tile of the stage (bar.sync + __threadfence + atomicAdd); the TMA producer and
// the epilogue warps of every CTA wait (acquire) for gridDim.x arrivals before touching the next
// stage's inputs (the producer also fences the async proxy: the next TMA loads read data that
// other CTAs wrote with generic stores).  The counters only grow (a launch generation word, bumped
// by CTA 0 after the last stage, sets each launch's targets), so no waiter can miss a completion.
#pragma once

#include "tc_gemm.cuh"

namespace hb {

constexpr int SK_MAX_G = 24;   // GEMMs per step: 3L - 1 <= 23 (L <= 8 weight layers)
constexpr int SK_MAX_S = 16;   // stages: 2L <= 16
constexpr int SK_STAGES = 8;   // smem ring depth (24 KB per stage: A 128x64 + B 64x64 bf16)
constexpr int SK_A_BYTES = TC_BM * TC_BK * 2;
constexpr int SK_B_BYTES = 64 * TC_BK * 2;
constexpr int SK_STAGE_BYTES = SK_A_BYTES + SK_B_BYTES;
constexpr int SK_SMEM_BYTES = SK_STAGES * SK_STAGE_BYTES + 1024 + 256;

enum { SK_FWD = 0, SK_HEAD = 1, SK_DGRAD = 2, SK_WGRAD = 3, SK_WGRAD_STORE = 4 };

struct SkGemm {
  CUtensorMap ma, mb;  // A [K-major box {64,128} or MN-major box {64,64}], B likewise ({64,BN} / {64,64})
  EpiArgs ep;
  const int* offA;     // device row offsets of A's / B's stored rows (the batch inside the data set:
  const int* offB;     // X of the layer-0 forward (A) and dW (B) GEMMs), nullable
  int kind, stage;
  int M, N, K;
  int tiles_m, tiles_n;
};

struct SkParams {
  SkGemm g[SK_MAX_G];
  int ng, nstages;
  // [SK_MAX_S] arrival counters + [SK_MAX_S] launch generation: counters only grow — stage s of
  // this launch is complete when bar[s] reaches (gen + 1) * gridDim.x, gen = the number of earlier
  // launches on this buffer (bumped by CTA 0 after the last stage, when every CTA has read it)
  unsigned* bar;
  unsigned long long* dbg;  // tuning build: per CTA, per stage SK_DBG_W globaltimer stamps (nullable)
};
constexpr int SK_DBG_W = 8;

__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void sk_wait_stage(const unsigned* bar, unsigned n) {
  while (ld_acquire_gpu(bar) < n) {
  }
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

__device__ __forceinline__ int sk_bn(int kind) { return kind == SK_HEAD ? 16 : 32; }
__device__ __forceinline__ bool sk_a_mn(int kind) { return kind == SK_WGRAD || kind == SK_WGRAD_STORE; }
__device__ __forceinline__ bool sk_b_mn(int kind) { return kind != SK_FWD && kind != SK_HEAD; }

// the u-th output tile of stage s over its GEMMs in order: (gemm, m_tile, n_tile); false if none
__device__ __forceinline__ bool sk_tile(const SkParams& P, int s, int u, int& g, int& mt, int& nt) {
  for (int k = 0; k < P.ng; ++k) {
    const SkGemm& G = P.g[k];
    if (G.stage != s) continue;
    const int t = G.tiles_m * G.tiles_n;
    if (u < t) {
      g = k;
      mt = u % G.tiles_m;  // consecutive CTAs take consecutive row tiles of one column panel
      nt = u / G.tiles_m;
      return true;
    }
    u -= t;
  }
  return false;
}

__global__ void __launch_bounds__(TC_THREADS, 1) step_kernel(const __grid_constant__ SkParams P) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + SK_STAGES * SK_STAGE_BYTES);
  uint64_t* empty_bar = full_bar + SK_STAGES;
  uint64_t* tmem_full_bar = empty_bar + SK_STAGES;
  uint64_t* tmem_empty_bar = tmem_full_bar + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_empty_bar + 2);
  __shared__ float red[4 * 32];
  __shared__ float sbias[2][32];
  __shared__ __align__(16) float dzs[TC_BM * 16];

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < SK_STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tmem_full_bar[a], 1);
      mbar_init(&tmem_empty_bar[a], TC_EPI_WARPS);
    }
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc<64>(tmem_slot);  // two 32-column accumulators
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const unsigned G = gridDim.x;
  const unsigned gen = *reinterpret_cast<volatile unsigned*>(P.bar + SK_MAX_S);
  const unsigned target = (gen + 1u) * G;

  if (warp == 0 && lane == 0) {
    // ===== TMA producer =====
    int it = 0;
    for (int s = 0; s < P.nstages; ++s) {
      unsigned long long* dbg = P.dbg ? P.dbg + ((size_t)blockIdx.x * SK_MAX_S + s) * SK_DBG_W : nullptr;
      (void)dbg;
      HB_STAMP(dbg, dbg[0]);
      if (s > 0) {
        sk_wait_stage(P.bar + s - 1, target);
        fence_proxy_async_global();
      }
      HB_STAMP(dbg, dbg[1]);
      int g, mt, nt;
      for (int u = blockIdx.x; sk_tile(P, s, u, g, mt, nt); u += G) {
        const SkGemm& Q = P.g[g];
        const int bn = sk_bn(Q.kind);
        const bool amn = sk_a_mn(Q.kind), bmn = sk_b_mn(Q.kind);
        const int oa = Q.offA ? __ldg(Q.offA) : 0;
        const int ob = Q.offB ? __ldg(Q.offB) : 0;
        const int nkb = (Q.K + TC_BK - 1) / TC_BK;
        const int m0 = mt * TC_BM, n0 = nt * bn;
        const uint32_t bytes = SK_A_BYTES + (bmn ? SK_B_BYTES : (uint32_t)bn * TC_BK * 2);
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int st = it % SK_STAGES;
          mbar_wait(&empty_bar[st], ((it / SK_STAGES) & 1) ^ 1);
          uint8_t* sA = smem + st * SK_STAGE_BYTES;
          uint8_t* sB = sA + SK_A_BYTES;
          const int k0 = kb * TC_BK;
          mbar_arrive_expect_tx(&full_bar[st], bytes);
          if (!amn) {
            tma_load_2d(sA, &Q.ma, &full_bar[st], k0, m0 + oa);
          } else {
            tma_load_2d(sA, &Q.ma, &full_bar[st], m0, k0 + oa);
            tma_load_2d(sA + 8192, &Q.ma, &full_bar[st], m0 + 64, k0 + oa);
          }
          // B: K-major rows n0.. (box {64, bn}); MN-major one 64-wide box of the K rows
          if (!bmn)
            tma_load_2d(sB, &Q.mb, &full_bar[st], k0, n0 + ob);
          else
            tma_load_2d(sB, &Q.mb, &full_bar[st], n0, k0 + ob);
        }
      }
    }
  } else if (warp == 1 && lane == 0) {
    // ===== MMA issuer =====
    int it = 0, i = 0;
    for (int s = 0; s < P.nstages; ++s) {
      unsigned long long* dbg = P.dbg ? P.dbg + ((size_t)blockIdx.x * SK_MAX_S + s) * SK_DBG_W : nullptr;
      (void)dbg;
      bool first = true;
      int g, mt, nt;
      for (int u = blockIdx.x; sk_tile(P, s, u, g, mt, nt); u += G, ++i) {
        const SkGemm& Q = P.g[g];
        const int bn = sk_bn(Q.kind);
        const bool amn = sk_a_mn(Q.kind), bmn = sk_b_mn(Q.kind);
        const uint32_t idesc = bn == 16 ? make_idesc_bf16(TC_BM, 16, amn, bmn) : make_idesc_bf16(TC_BM, 32, amn, bmn);
        const int acc = i & 1;
        mbar_wait(&tmem_empty_bar[acc], ((i >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t tacc = tmem_base + (uint32_t)(acc * 32);
        const int nkb = (Q.K + TC_BK - 1) / TC_BK;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int st = it % SK_STAGES;
          mbar_wait(&full_bar[st], (it / SK_STAGES) & 1);
          tc_fence_after();
          HB_STAMP(dbg && first && kb == 0, dbg[2]);
          const uint32_t a_base = smem_u32(smem + st * SK_STAGE_BYTES);
          const uint32_t b_base = a_base + SK_A_BYTES;
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk) {
            const uint64_t ad = amn ? make_sw128_desc(a_base + kk * 2048, 8192, 1024) : make_sw128_desc(a_base + kk * 32, 16, 1024);
            const uint64_t bd = bmn ? make_sw128_desc(b_base + kk * 2048, 8192, 1024) : make_sw128_desc(b_base + kk * 32, 16, 1024);
            umma_bf16(tacc, ad, bd, idesc, (kb | kk) != 0);
          }
          umma_commit(&empty_bar[st]);
        }
        umma_commit(&tmem_full_bar[acc]);
        HB_STAMP(dbg && first, dbg[3]);
        first = false;
      }
    }
  } else if (warp >= 4) {
    // ===== epilogue warps =====
    const EpiTileCtx ectx{tmem_base, tmem_full_bar, tmem_empty_bar, &sbias[0][0], red, dzs, nullptr, smem, nullptr,
                          nullptr, 1, 1, warp, lane, nullptr};
    int i = 0;
    for (int s = 0; s < P.nstages; ++s) {
      unsigned long long* dbg = P.dbg && threadIdx.x == 128 ? P.dbg + ((size_t)blockIdx.x * SK_MAX_S + s) * SK_DBG_W : nullptr;
      (void)dbg;
      HB_STAMP(dbg, dbg[4]);
      if (s > 0) {  // this stage's epilogues read what other CTAs wrote in earlier stages (bias partials)
        if (threadIdx.x == 128) sk_wait_stage(P.bar + s - 1, target);
        epi_bar_sync();
      }
      HB_STAMP(dbg, dbg[5]);
      int g, mt, nt;
      for (int u = blockIdx.x; sk_tile(P, s, u, g, mt, nt); u += G, ++i) {
        const SkGemm& Q = P.g[g];
        switch (Q.kind) {
          case SK_FWD: tc_epilogue_tile<32, EPI_FWD_SIG>(Q.ep, ectx, mt, nt, i & 1, i, 32); break;
          case SK_HEAD: tc_epilogue_tile<16, EPI_HEAD_XENT>(Q.ep, ectx, mt, nt, i & 1, i, 32); break;
          case SK_DGRAD: tc_epilogue_tile<32, EPI_DGRAD_SIG>(Q.ep, ectx, mt, nt, i & 1, i, 32); break;
          case SK_WGRAD: tc_epilogue_tile<32, EPI_WGRAD_SGD>(Q.ep, ectx, mt, nt, i & 1, i, 32); break;
          default: tc_epilogue_tile<32, EPI_WGRAD_STORE>(Q.ep, ectx, mt, nt, i & 1, i, 32); break;
        }
      }
      // every output of this CTA for stage s is written: arrive
      epi_bar_sync();
      HB_STAMP(dbg, dbg[6]);
      if (threadIdx.x == 128) {
        __threadfence();
        atomicAdd(P.bar + s, 1u);
      }
      HB_STAMP(dbg, dbg[7]);
    }
    if (blockIdx.x == 0 && threadIdx.x == 128) {  // every CTA read `gen` before arriving: next launch
      sk_wait_stage(P.bar + P.nstages - 1, target);
      atomicAdd(P.bar + SK_MAX_S, 1u);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc<64>(tmem_base);
  }
}

}  // namespace hb
