// head.cuh — the output layer of a small-C net (C <= 8) as ONE pass over the batch's last hidden
// activations, on CUDA cores, HBM-bound:
//
//   Eq. (1) output layer   z_i = H_{L-1}[i] W_L^T + b_L                       [PAPER.md L43]
//   softmax cross-entropy  loss_i = lse(z_i) - z_{i,y_i},
//                          dZ_L[i] = (softmax(z_i) - onehot(y_i)) / b           [L258]
//   Eq. (2) output dX      dZ_{L-1}[i] = (dZ_L[i] W_L) * sigma'(Z_{L-1}[i])     [L49]
//   Eq. (2) output dW, db  dW_L = dZ_L^T H_{L-1}, db_L = 1^T dZ_L  (per-CTA partials here;
//                          head_update_kernel reduces them in fixed order and applies
//                          Eq. (3) W_L -= lr dW_L, b_L -= lr db_L in place [L53])
//
// Why not tensor cores: K = C <= 8 makes the dX and dW contractions of the output layer
// 2·b·C·n FLOPs against b·n·6 bytes (H, S read, dZ_{L-1} written) — arithmetic intensity
// ~C/3 FLOP/B, far below the HBM ridge — and the logits GEMM (N = C padded to 16) runs on
// b/128 CTAs.  One streaming pass reads H_{L-1} and S_{L-1} once and writes dZ_{L-1} once
// (C4: 201 MB per 8192-row batch) instead of the three GEMMs' 268 MB across three launches;
// dZ_L never leaves the chip, so dW_L is computed from fp32 dZ_L (no bf16 rounding of dZ_L,
// which DESIGN.md R24 had to split into hi/lo planes for the tensor-core head).
//
// Layout: thread t of a T-thread CTA owns the column chunks t, t + T, ... (CPT of them, CW = 8 or 4
// columns each) of every row; rows arrive in shared memory by bulk copies (a ring of stages, see
// below) and dZ_{L-1} rows leave as coalesced 16- / 8-byte-per-lane stores.  A CTA walks a
// contiguous row range RB rows at a time: partial dot products for RB rows x C classes are reduced
// across the CTA (a transposed warp reduction, then one shared-memory pass in fixed warp order),
// warp 0 finishes the softmax with one lane per (row, class), and every thread then applies dZ_L
// of those rows to its columns (dX, dW_L and bias partials).  Deterministic: every reduction has a
// fixed order independent of timing.  DESIGN.md §5.3.
#pragma once

#include "common.cuh"
#include "epilogue.cuh"

namespace hb {

constexpr int HEAD_MAX_C = 8;

struct HeadArgs {
  const __nv_bfloat16* H;  // H_{L-1} [b x ld] bf16 (row 0 = the batch's first row)
  const __nv_bfloat16* S;  // S_{L-1} = sigma'(Z_{L-1}) [b x ld] (training only)
  int64_t ld;              // row stride of H, S and dZ (elements, multiple of 8)
  const __nv_bfloat16* W;  // W_L bf16 shadow [C x ldw] (what the tensor cores would read)
  int64_t ldw;
  const float* bias;       // b_L [C] (fp32 master)
  const int32_t* y;        // labels (dataset base when yoff != nullptr)
  const int* yoff;         // device row offset of the batch (graph replay), nullable
  int b, n, C;             // rows, n_{L-1}, classes
  int rows_per_cta;        // multiple of RB
  int stages;              // shared-memory ring depth (2 .. HEAD_MAX_STAGES)
  float inv_b;
  float* row_loss;         // [b]
  __nv_bfloat16* dz;       // dZ_{L-1} [b x ld]; nullptr = loss only (mlp_loss)
  float* bpart;            // [gridDim.x x n] column sums of dZ_{L-1} per CTA (bias partials of layer L-1)
  float* dwp;              // [gridDim.x x C x n] per-CTA partial dW_L
  float* dbp;              // [gridDim.x x C]     per-CTA partial db_L
};

// CMAX: classes rounded up (2, 4, 8); CW: columns per chunk (8 = 16-byte, 4 = 8-byte accesses);
// CPT: chunks per thread (1, 2); RB rows per round, RB * CMAX <= 32 (one softmax lane per (row,
// class) in warp 0).  Wide rows (n > 1024): CW = 8, RB = min(16 / CMAX, 4 / CPT), one CTA per SM
// (up to 512 threads) with a ring of up to 4 stages; narrow rows (n <= 1024): CW = 4 (twice the
// threads of 16-byte chunks), RB = 16 / CMAX (4 for CMAX = 8) and two CTAs per SM (100 KB rings), so one CTA's
// barriers and softmax overlap the other's rounds.
template <int CMAX, int CPT, int RB_, int CW_>
struct HeadShape {
  static constexpr int RB = RB_, CW = CW_, Q = CW_ / 2;  // Q: packed bf16 pairs per chunk
  static constexpr int NV = RB * CMAX;  // values reduced across the CTA per round
  static_assert(NV <= 32 && (NV & (NV - 1)) == 0, "one softmax lane per (row, class); power of two");
  static constexpr int MAXT = CW == 4 ? 256 : CMAX <= 4 ? 512 : 256;
};
constexpr int HEAD_MAX_STAGES = 4;

// 1-D bulk copy global -> shared (async proxy), completion counted in bytes on an mbarrier
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

// Q packed bf16 pairs -> Q float2 (exact: a bf16 is the top half of its fp32); pad columns
// [n, ld) of H / S rows are never written (TMA stores clip them) and are zeroed
template <int Q>
__device__ __forceinline__ void load_chunk(const uint8_t* src, int c0, int n, float2 (&f)[Q]) {
  uint32_t w[Q];
  if (Q == 4) {
    const uint4 u = *reinterpret_cast<const uint4*>(src);
    w[0] = u.x, w[1] = u.y, w[2 % Q] = u.z, w[3 % Q] = u.w;
  } else {
    const uint2 u = *reinterpret_cast<const uint2*>(src);
    w[0] = u.x, w[1] = u.y;
  }
#pragma unroll
  for (int k = 0; k < Q; ++k) f[k] = make_float2(__uint_as_float(w[k] << 16), __uint_as_float(w[k] & 0xffff0000u));
  if (c0 + 2 * Q > n) {
#pragma unroll
    for (int k = 0; k < Q; ++k) {
      if (c0 + 2 * k >= n) f[k].x = 0.f;
      if (c0 + 2 * k + 1 >= n) f[k].y = 0.f;
    }
  }
}

// Sum NV per-lane values over the 32 lanes of a warp, transposed: after log2(NV) halving exchanges
// (each lane keeps the half of the values selected by its lane bit) and butterfly steps for the
// remaining lane bits, lane l holds the warp total of value l >> (5 - log2 NV).  NV - 1 + 5 -
// log2(NV) shuffles instead of 5 NV; fixed order (deterministic).
template <int NV>
__device__ __forceinline__ float warp_transpose_sum(float (&v)[NV], int lane) {
  int m = NV;
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) {
    if (m > 1) {
      const int half = m / 2;
      const bool up = (lane & o) != 0;
#pragma unroll
      for (int i = 0; i < NV / 2; ++i) {
        if (i < half) {
          const float send = up ? v[i] : v[i + half];
          const float keep = up ? v[i + half] : v[i];
          v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
        }
      }
      m = half;
    } else {
      v[0] += __shfl_xor_sync(0xffffffffu, v[0], o);
    }
  }
  return v[0];
}

// Rows reach shared memory by bulk copies (one per H / S row, issued by one lane of the last warp)
// into a ring of a.stages stages of RB rows, so the HBM reads of the next rounds run while the CTA
// reduces and applies the current one.  The per-element arithmetic runs on column pairs with the
// packed fp32x2 FMA / MUL / ADD (same rounding as scalar).
template <int CMAX, int CPT, int RB_, int CW_>
__global__ void __launch_bounds__(HeadShape<CMAX, CPT, RB_, CW_>::MAXT) head_fused_kernel(HeadArgs a) {
  using SH = HeadShape<CMAX, CPT, RB_, CW_>;
  constexpr int RB = SH::RB, NV = SH::NV, CW = SH::CW, Q = SH::Q;
  constexpr int LSH = NV == 32 ? 0 : NV == 16 ? 1 : NV == 8 ? 2 : NV == 4 ? 3 : NV == 2 ? 4 : 5;
  extern __shared__ __align__(128) uint8_t hsm[];
  __shared__ float red[2][SH::MAXT / 32][NV];
  __shared__ float dzs[2][RB][CMAX];
  __shared__ __align__(8) uint64_t full[HEAD_MAX_STAGES];
  const int T = blockDim.x, tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, nw = T >> 5;
  const int C = a.C, n = a.n, nst = a.stages;
  const bool train = a.dz != nullptr;
  const int r_begin = blockIdx.x * a.rows_per_cta;
  const int r_end = min(a.b, r_begin + a.rows_per_cta);
  const int nrounds = r_end > r_begin ? (r_end - r_begin + RB - 1) / RB : 0;
  const uint32_t rowb = (uint32_t)(a.ld * 2);
  const uint32_t stage_bytes = (uint32_t)RB * rowb * (train ? 2u : 1u);
  if (tid == 0) {
    for (int i = 0; i < nst; ++i) mbar_init(&full[i], 1);
    fence_barrier_init();
    fence_proxy_async();
  }
  __syncthreads();
  asm volatile("griddepcontrol.wait;" ::: "memory");  // H / S of the previous kernel (PDL)
  auto issue = [&](int k) {  // round k's rows into stage k % nst
    if (k >= nrounds) return;
    const int r0 = r_begin + k * RB, nr = min(RB, r_end - r0);
    uint64_t* bar = &full[k % nst];
    uint8_t* st = hsm + (size_t)(k % nst) * stage_bytes;
    mbar_arrive_expect_tx(bar, (uint32_t)nr * rowb * (train ? 2u : 1u));
    for (int i = 0; i < nr; ++i) {
      bulk_g2s(st + (size_t)i * rowb, a.H + (int64_t)(r0 + i) * a.ld, rowb, bar);
      if (train) bulk_g2s(st + (size_t)(RB + i) * rowb, a.S + (int64_t)(r0 + i) * a.ld, rowb, bar);
    }
  };
  if (tid == T - 32)
    for (int k = 0; k < nst; ++k) issue(k);

  // W_L columns of this thread's chunks, as fp32 column pairs in registers
  float2 w[CPT][CMAX][Q];
  bool cok[CPT];
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    const int c0 = (j * T + tid) * CW;
    cok[j] = c0 < n;
#pragma unroll
    for (int c = 0; c < CMAX; ++c) {
      if (cok[j] && c < C) {
        load_chunk<Q>(reinterpret_cast<const uint8_t*>(a.W + (int64_t)c * a.ldw + c0), c0, n, w[j][c]);
      } else {
#pragma unroll
        for (int e = 0; e < Q; ++e) w[j][c][e] = make_float2(0.f, 0.f);
      }
    }
  }
  float2 dw[CPT][CMAX][Q];  // partial dW_L of this CTA's rows
  float2 bs[CPT][Q];        // column sums of dZ_{L-1} (bias partials of layer L-1)
#pragma unroll
  for (int j = 0; j < CPT; ++j)
#pragma unroll
    for (int e = 0; e < Q; ++e) {
      bs[j][e] = make_float2(0.f, 0.f);
#pragma unroll
      for (int c = 0; c < CMAX; ++c) dw[j][c][e] = make_float2(0.f, 0.f);
    }
  float dbacc = 0.f;  // thread c < C: this CTA's db_L[c]
  const int yo = a.yoff ? __ldg(a.yoff) : 0;
  // warp 0 (softmax): lane i * CMAX + c keeps b_L[c] and the label of row i of the round, loaded
  // one round ahead so the global-load latency is off the round's critical path
  const float bias_c = (warp == 0 && lane % CMAX < C) ? __ldg(a.bias + lane % CMAX) : 0.f;
  auto label = [&](int k) -> int {
    const int r = r_begin + k * RB + lane / CMAX;
    return (warp == 0 && lane < NV && k < nrounds && r < r_end) ? __ldg(a.y + yo + r) : -1;
  };
  int ylab = label(0);

  // ---- phase 1 of round k: partial logits of its rows over this thread's columns -> red[k & 1] ----
  auto dot_phase = [&](int k) {
    const int nr = min(RB, r_end - (r_begin + k * RB));
    const uint8_t* st = hsm + (size_t)(k % nst) * stage_bytes;
    mbar_wait(&full[k % nst], (uint32_t)(k / nst) & 1u);
    float p[NV];
#pragma unroll
    for (int i = 0; i < RB; ++i) {
      float2 acc[CMAX];
#pragma unroll
      for (int c = 0; c < CMAX; ++c) acc[c] = make_float2(0.f, 0.f);
#pragma unroll
      for (int j = 0; j < CPT; ++j) {
        if (i < nr && cok[j]) {
          float2 h[Q];
          load_chunk<Q>(st + (size_t)i * rowb + (size_t)(j * T + tid) * CW * 2, (j * T + tid) * CW, n, h);
#pragma unroll
          for (int c = 0; c < CMAX; ++c)
#pragma unroll
            for (int e = 0; e < Q; ++e) acc[c] = __ffma2_rn(h[e], w[j][c][e], acc[c]);
        }
      }
#pragma unroll
      for (int c = 0; c < CMAX; ++c) p[i * CMAX + c] = acc[c].x + acc[c].y;
    }
    const float t = warp_transpose_sum<NV>(p, lane);
    if ((lane & ((1 << LSH) - 1)) == 0) red[k & 1][warp][lane >> LSH] = t;
  };
  // ---- phase 2 of round k, warp 0 only: softmax cross-entropy; lane v = i * CMAX + c owns class c
  //      of row i (the row's max / sum over its CMAX lanes by xor shuffles inside the lane group) ----
  auto softmax_phase = [&](int k) {
    const int r0 = r_begin + k * RB, nr = min(RB, r_end - r0);
    const int ycur = ylab;
    ylab = label(k + 1);  // one round ahead: the load's latency is off the critical path
    const int i = lane / CMAX, c = lane % CMAX;
    const bool cv = lane < NV && c < C;
    float t = 0.f;
    if (lane < NV)
      for (int q = 0; q < nw; ++q) t += red[k & 1][q][lane];
    const float z = cv ? t + bias_c : -INFINITY;
    float mx = z;
#pragma unroll
    for (int o = 1; o < CMAX; o <<= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    float se = cv ? expf(z - mx) : 0.f;
#pragma unroll
    for (int o = 1; o < CMAX; o <<= 1) se += __shfl_xor_sync(0xffffffffu, se, o);
    const float lse = mx + logf(se);
    const bool rok = lane < NV && i < nr;
    if (lane < NV) dzs[k & 1][i][c] = (rok && cv) ? (expf(z - lse) - (c == ycur ? 1.f : 0.f)) * a.inv_b : 0.f;
    if (rok && c == ycur) a.row_loss[r0 + i] = lse - z;
    __syncwarp();
  };

  // Software pipeline, per iteration k: phase 1 of round k + 1, then (after warp 0's softmax of round
  // k, named barrier 1) phase 3 of round k; one CTA barrier; then warp 0 runs the softmax of round
  // k + 1 while the other warps go on to phase 1 of round k + 2, and the last warp refills stage k.
  if (nrounds > 0) {
    dot_phase(0);
    __syncthreads();
    if (warp == 0) {
      softmax_phase(0);
      asm volatile("bar.arrive 1, %0;" ::"r"(T) : "memory");
    }
  }
  for (int k = 0; k < nrounds; ++k) {
    const int r0 = r_begin + k * RB, nr = min(RB, r_end - r0);
    const uint8_t* st = hsm + (size_t)(k % nst) * stage_bytes;
    if (k + 1 < nrounds) dot_phase(k + 1);
    if (warp != 0) asm volatile("bar.sync 1, %0;" ::"r"(T) : "memory");  // dZ_L of round k ready
    if (train) {
      if (tid < C) {
#pragma unroll
        for (int i = 0; i < RB; ++i) dbacc += dzs[k & 1][i][tid];
      }
      // ---- phase 3 of round k: dX of the output layer, dW_L and the bias partials of layer L-1 ----
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        if (i >= nr) break;
        float2 d[CMAX];
#pragma unroll
        for (int c = 0; c < CMAX; ++c) d[c] = make_float2(dzs[k & 1][i][c], dzs[k & 1][i][c]);
#pragma unroll
        for (int j = 0; j < CPT; ++j) {
          if (!cok[j]) continue;
          const int c0 = (j * T + tid) * CW;
          float2 hk[Q], sv[Q];  // round k's rows are still in stage k: H re-read, not kept in registers
          load_chunk<Q>(st + (size_t)i * rowb + (size_t)c0 * 2, c0, n, hk);
          load_chunk<Q>(st + (size_t)(RB + i) * rowb + (size_t)c0 * 2, c0, n, sv);
          uint32_t pk[Q];
#pragma unroll
          for (int e = 0; e < Q; ++e) {
            float2 g = make_float2(0.f, 0.f);
#pragma unroll
            for (int c = 0; c < CMAX; ++c) {
              g = __ffma2_rn(d[c], w[j][c][e], g);
              dw[j][c][e] = __ffma2_rn(d[c], hk[e], dw[j][c][e]);
            }
            const float2 o = __fmul2_rn(g, sv[e]);
            bs[j][e] = __fadd2_rn(bs[j][e], o);
            pk[e] = pack_bf16x2(o.x, o.y);
          }
          __nv_bfloat16* dst = a.dz + (int64_t)(r0 + i) * a.ld + c0;
          if (Q == 4)
            *reinterpret_cast<uint4*>(dst) = make_uint4(pk[0], pk[1], pk[2 % Q], pk[3 % Q]);
          else
            *reinterpret_cast<uint2*>(dst) = make_uint2(pk[0], pk[1]);
        }
      }
    }
    __syncthreads();  // stage k read by everyone; red[(k + 1) & 1] complete; dzs[k & 1] consumed
    if (tid == T - 32) issue(k + nst);  // refill stage k (last warp: off warp 0's softmax path)
    if (warp == 0 && k + 1 < nrounds) {
      softmax_phase(k + 1);
      asm volatile("bar.arrive 1, %0;" ::"r"(T) : "memory");
    }
  }
  if (!train) return;
  // ---- per-CTA partials: bias sums of dZ_{L-1}, dW_L, db_L (each thread's CW consecutive columns
  //      as 16-byte stores when the row is 16-byte aligned) ----
  const bool vec = (n & 3) == 0;
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    const int c0 = (j * T + tid) * CW;
    if (!cok[j]) continue;
    auto put = [&](float* dst, const float2 (&v)[Q]) {
      if (vec && c0 + CW <= n) {
#pragma unroll
        for (int e = 0; e < Q; e += 2)
          reinterpret_cast<float4*>(dst)[e / 2] = make_float4(v[e].x, v[e].y, v[e + 1].x, v[e + 1].y);
      } else {
#pragma unroll
        for (int e = 0; e < CW; ++e)
          if (c0 + e < n) dst[e] = (e & 1) ? v[e >> 1].y : v[e >> 1].x;
      }
    };
    put(a.bpart + (int64_t)blockIdx.x * n + c0, bs[j]);
#pragma unroll
    for (int c = 0; c < CMAX; ++c)
      if (c < C) put(a.dwp + ((int64_t)blockIdx.x * C + c) * n + c0, dw[j][c]);
  }
  if (tid < C) a.dbp[blockIdx.x * C + tid] = dbacc;
}

// Eq. (3) for the output layer: dW_L[c][k] = sum over the P CTA partials in a fixed order — HU_Y
// strided subsets per entry (four interleaved accumulators each, so the loads are in flight
// together), the subsets combined in order in groups of 8, then the groups in order — followed by
// the same fused update as the dW GEMM epilogue (epi_elem: Hogwild or atomic, bf16 shadow, peer
// replicas; or the gradient stored).  Block (HU_X, HU_Y): HU_X consecutive (c, k) entries, so even a
// narrow output layer (C x n = 2048 entries) spreads over 256 blocks; the last block also reduces db_L.
constexpr int HU_X = 8, HU_Y = 64;

// column e of a [P x stride] partial array summed over its P rows in the fixed order above; the
// result is valid in the ty == 0 threads (every thread of the block must call it)
__device__ __forceinline__ float hu_reduce(const float* __restrict__ src, int64_t stride, int64_t e, bool ok, int P,
                                           float (*part)[HU_X + 1], float (*part8)[HU_X + 1]) {
  const int tx = threadIdx.x, ty = threadIdx.y;
  float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
  if (ok) {
    int p = ty;
    for (; p + 3 * HU_Y < P; p += 4 * HU_Y) {
      a0 += __ldcg(src + (int64_t)p * stride + e);
      a1 += __ldcg(src + (int64_t)(p + HU_Y) * stride + e);
      a2 += __ldcg(src + (int64_t)(p + 2 * HU_Y) * stride + e);
      a3 += __ldcg(src + (int64_t)(p + 3 * HU_Y) * stride + e);
    }
    for (; p < P; p += HU_Y) a0 += __ldcg(src + (int64_t)p * stride + e);
  }
  part[ty][tx] = (a0 + a1) + (a2 + a3);
  __syncthreads();
  if (ty < HU_Y / 8) {
    float g = 0.f;
#pragma unroll
    for (int q = 0; q < 8; ++q) g += part[ty * 8 + q][tx];
    part8[ty][tx] = g;
  }
  __syncthreads();
  float g = 0.f;
  if (ty == 0) {
#pragma unroll
    for (int q = 0; q < HU_Y / 8; ++q) g += part8[q][tx];
  }
  __syncthreads();  // part / part8 reusable
  return g;
}

template <int EPI>
__global__ void __launch_bounds__(HU_X * HU_Y) head_update_kernel(EpiArgs ep, const float* __restrict__ dwp,
                                                                  const float* __restrict__ dbp, int P, int C, int n) {
  __shared__ float part[HU_Y][HU_X + 1];
  __shared__ float part8[HU_Y / 8][HU_X + 1];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t e = (int64_t)blockIdx.x * HU_X + tx;
  const int64_t CN = (int64_t)C * n;
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const float g = hu_reduce(dwp, CN, e, e < CN, P, part, part8);
  if (ty == 0 && e < CN) {
    const int c = (int)(e / n), k = (int)(e % n);
    epi_elem<EPI, __nv_bfloat16, false>(ep, k, c, g);  // transposed: element (k, c) is W_L[c][k]
  }
  if (blockIdx.x == gridDim.x - 1) {  // db_L (HU_X >= HEAD_MAX_C entries)
    const float gb = hu_reduce(dbp, C, tx, tx < C, P, part, part8);
    if (ty == 0 && tx < C) {
      if (EPI == EPI_WGRAD_SGD) {
        if (ep.atomic)
          atomicAdd(ep.bias_upd + tx, __fmul_rn(-ep.lr, gb));
        else
          ep.bias_upd[tx] += __fmul_rn(-ep.lr, gb);
        if (ep.npeer) peer_push1(ep, ep.bias_upd + tx, nullptr, gb);
      } else {
        ep.bias_grad[tx] = gb;
      }
    }
  }
}

}  // namespace hb
