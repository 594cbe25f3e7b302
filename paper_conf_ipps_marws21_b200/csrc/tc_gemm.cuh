// tc_gemm.cuh — warp-specialised tcgen05 GEMM for sm_100a with TMA loads, a TMEM accumulator
// and the fused MLP-SGD epilogues of epilogue.cuh.
//
//   C[M x N] = A[M x K] * B[N x K]^T         (bf16 operands, fp32 accumulate in TMEM)
//
// The three contractions of one SGD step (Eq. (1)/(2), L43/L49) map onto it as
//   forward  H_l  = sigma(H_{l-1} W_l^T + b_l)   A = H_{l-1} (K-major), B = W_l (K-major)
//   dgrad    dZ   = (dZ_l W_l) * S               A = dZ_l   (K-major), B = W_l (MN-major)
//   wgrad    W_l -= lr * dZ_l^T H_{l-1}          A = dZ_l   (MN-major), B = H_{l-1} (MN-major)
// so the same kernel serves all of them; the operand major-ness is a template parameter and is
// handled entirely by the TMA box shape and the UMMA shared-memory descriptor, never by a copy.
//
// CTA = 256 threads: warp 0 TMA producer, warp 1 MMA issuer (one elected thread), warp 2 TMEM
// allocator, warps 4..7 epilogue (warp w reads TMEM lanes 32*(w%4)..+31 = tile rows).
// Tile: BLOCK_M = 128 (UMMA M = 128, cta_group::1), BLOCK_N = BN (16..256), BLOCK_K = 64 (one
// 128-byte swizzle atom of bf16).  smem stages form an mbarrier ring (full/empty).
#pragma once

#include "common.cuh"
#include "epilogue.cuh"

namespace hb {

constexpr int TC_BM = 128;
constexpr int TC_BK = 64;
constexpr int TC_THREADS = 256;

template <int BN, bool B_MN>
struct TcCfg {
  static constexpr int A_BYTES = TC_BM * TC_BK * 2;                     // 16 KB
  static constexpr int B_ROWS = B_MN ? (BN < 64 ? 64 : BN) : BN;        // MN-major loads 64-wide boxes
  static constexpr int B_BYTES = B_ROWS * TC_BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES_RAW = (196 * 1024) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN;                  // power of two >= 32
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
};

template <int BN, bool A_MN, bool B_MN, int EPI>
__global__ void __launch_bounds__(TC_THREADS, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   int K, EpiArgs ep) {
  using Cfg = TcCfg<BN, B_MN>;
  constexpr int STAGES = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty_bar = full_bar + STAGES;
  uint64_t* tmem_full_bar = empty_bar + STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full_bar + 1);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN;
  const int m0 = blockIdx.y * TC_BM;
  const int num_kb = (K + TC_BK - 1) / TC_BK;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(tmem_full_bar, 1);
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0 && lane == 0) {
    // ===== TMA producer =====
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % STAGES;
      const uint32_t ph = (kb / STAGES) & 1;
      mbar_wait(&empty_bar[s], ph ^ 1);
      uint8_t* sA = smem + s * Cfg::STAGE_BYTES;
      uint8_t* sB = sA + Cfg::A_BYTES;
      mbar_arrive_expect_tx(&full_bar[s], Cfg::STAGE_BYTES);
      const int k0 = kb * TC_BK;
      if (!A_MN) {
        tma_load_2d(sA, &tmA, &full_bar[s], k0, m0);
      } else {
        tma_load_2d(sA, &tmA, &full_bar[s], m0, k0);
        tma_load_2d(sA + 8192, &tmA, &full_bar[s], m0 + 64, k0);
      }
      if (!B_MN) {
        tma_load_2d(sB, &tmB, &full_bar[s], k0, n0);
      } else {
#pragma unroll
        for (int j = 0; j < Cfg::B_ROWS / 64; ++j) tma_load_2d(sB + j * 8192, &tmB, &full_bar[s], n0 + 64 * j, k0);
      }
    }
  } else if (warp == 1 && lane == 0) {
    // ===== MMA issuer (single thread) =====
    constexpr uint32_t idesc = make_idesc_bf16(TC_BM, BN, A_MN, B_MN);
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % STAGES;
      const uint32_t ph = (kb / STAGES) & 1;
      mbar_wait(&full_bar[s], ph);
      tc_fence_after();
      const uint32_t a_base = smem_u32(smem + s * Cfg::STAGE_BYTES);
      const uint32_t b_base = a_base + Cfg::A_BYTES;
#pragma unroll
      for (int kk = 0; kk < TC_BK / 16; ++kk) {
        // K-major SW128: rows of 128 B, 8-row groups 1024 B apart (SBO); +32 B per UMMA_K = 16.
        // MN-major SW128: 64-element MN chunks 8192 B apart (LBO), 8-row K groups 1024 B apart
        // (SBO); +16 rows * 128 B = 2048 B per UMMA_K.
        const uint64_t ad = A_MN ? make_sw128_desc(a_base + kk * 2048, 8192, 1024)
                                 : make_sw128_desc(a_base + kk * 32, 16, 1024);
        const uint64_t bd = B_MN ? make_sw128_desc(b_base + kk * 2048, 8192, 1024)
                                 : make_sw128_desc(b_base + kk * 32, 16, 1024);
        umma_bf16(tmem_base, ad, bd, idesc, (kb | kk) != 0);
      }
      umma_commit(&empty_bar[s]);  // frees the smem slot when these MMAs complete
    }
    umma_commit(tmem_full_bar);     // accumulator ready
  } else if (warp >= 4) {
    // ===== epilogue: TMEM -> registers -> fused epilogue -> global =====
    mbar_wait(tmem_full_bar, 0);
    tc_fence_after();
    const int q = warp & 3;
    const int r = m0 + q * 32 + lane;
    const bool row_ok = r < ep.M;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      if (n0 + c >= ep.N) break;  // warp-uniform
      uint32_t raw[16];
      tmem_ld_32x32b_x16(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)c, raw);
      tmem_ld_wait();
      float v[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = __uint_as_float(raw[j]);
      if (row_ok) {
        const int nc = n0 + c;
        const bool vec_ok = (nc + 16 <= ep.N) && !((EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) && ep.transposed) &&
                            (EPI != EPI_WGRAD_SGD || ep.shadow != nullptr) && EPI != EPI_FWD_LOGITS &&
                            EPI != EPI_WGRAD_STORE;
        if (vec_ok) {
          epi_row16_bf16<EPI>(ep, r, nc, v);
        } else {
#pragma unroll 4
          for (int j = 0; j < 16; ++j)
            if (nc + j < ep.N) epi_elem<EPI, __nv_bfloat16, false>(ep, r, nc + j, v[j]);
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
  }
}

}  // namespace hb
