// kernels.cuh — CUDA-core kernels of the hot path:
//   * softmax cross-entropy head (warp per row, shuffle reductions)     [PAPER.md L258]
//   * bias gradient + in-place bias SGD (deterministic two-pass column sum) [Eq. (3), L53]
//   * fp32 check-mode SIMT GEMM with the same fused epilogues (HB_PREC_FP32_CHECK)
//   * deterministic fp64 loss reduction, fp32->bf16 shadow refresh, replica-merge kernels
#pragma once

#include "common.cuh"
#include "epilogue.cuh"

namespace hb {

// ---------------------------------------------------------------------------------------
// softmax cross-entropy: one warp per row.
//   lse_i = m_i + log sum_c exp(z_ic - m_i),  loss_i = lse_i - z_{i,y_i}
//   dZ_ic = (exp(z_ic - lse_i) - [c == y_i]) * inv_b        (gradient of the batch MEAN loss)
// dZ may be null (loss only, mlp_loss).  C <= 1024 with 16-byte aligned rows (ldl % 4 == 0): the
// row is read ONCE into registers (float4 per lane, <= 8 per lane), so the kernel streams
// b*C*4 bytes of logits in and b*C*sizeof(TDZ) bytes of dZ out (HBM-bound); larger C loops.
// ---------------------------------------------------------------------------------------
template <typename TDZ>
__device__ __forceinline__ void store4(TDZ* d, int c, int C, float a, float b, float e, float f) {
  const float v[4] = {a, b, e, f};
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (c + j < C) d[c + j] = to_act<TDZ>(v[j]);
}
template <>
__device__ __forceinline__ void store4<__nv_bfloat16>(__nv_bfloat16* d, int c, int C, float a, float b, float e, float f) {
  if (c + 4 <= C && ((reinterpret_cast<uintptr_t>(d + c) & 7) == 0)) {
    __nv_bfloat162 lo = __floats2bfloat162_rn(a, b), hi = __floats2bfloat162_rn(e, f);
    uint2 u;
    u.x = *reinterpret_cast<uint32_t*>(&lo);
    u.y = *reinterpret_cast<uint32_t*>(&hi);
    *reinterpret_cast<uint2*>(d + c) = u;
    return;
  }
  const float v[4] = {a, b, e, f};
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (c + j < C) d[c + j] = __float2bfloat16_rn(v[j]);
}

template <typename TDZ>
__global__ void softmax_xent_kernel(const float* __restrict__ logits, int64_t ldl,
                                    const int32_t* __restrict__ y, const int* __restrict__ yoff, int b, int C, TDZ* dZ,
                                    int64_t ldz, float* __restrict__ row_loss, float inv_b) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (warp >= b) return;
  const float* z = logits + (int64_t)warp * ldl;
  const int yi = y[(yoff ? *yoff : 0) + warp];
  if (C <= 1024 && (ldl & 3) == 0) {
    // one exp per element (kept in registers: p = exp(z - m)), dZ = p / s - onehot, scaled by 1/b
    constexpr int V = 8;
    constexpr float LOG2E = 1.4426950408889634f;
    float4 v[V];
    float m = -INFINITY;
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int c = (i * 32 + lane) * 4;
      v[i] = make_float4(-INFINITY, -INFINITY, -INFINITY, -INFINITY);
      if (c < C) {
        const float4 t = __ldg(reinterpret_cast<const float4*>(z + c));
        v[i].x = t.x;
        v[i].y = c + 1 < C ? t.y : -INFINITY;
        v[i].z = c + 2 < C ? t.z : -INFINITY;
        v[i].w = c + 3 < C ? t.w : -INFINITY;
      }
      m = fmaxf(m, fmaxf(fmaxf(v[i].x, v[i].y), fmaxf(v[i].z, v[i].w)));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    const float mb = m * LOG2E;
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < V; ++i) {  // exp2(z*log2e - m*log2e); exp2(-inf) = 0 for the masked tail
      v[i].x = exp2f(fmaf(v[i].x, LOG2E, -mb));
      v[i].y = exp2f(fmaf(v[i].y, LOG2E, -mb));
      v[i].z = exp2f(fmaf(v[i].z, LOG2E, -mb));
      v[i].w = exp2f(fmaf(v[i].w, LOG2E, -mb));
      s += (v[i].x + v[i].y) + (v[i].z + v[i].w);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) row_loss[warp] = m + logf(s) - __ldg(z + yi);
    if (dZ) {
      TDZ* d = dZ + (int64_t)warp * ldz;
      const float sc = inv_b / s;
#pragma unroll
      for (int i = 0; i < V; ++i) {
        const int c = (i * 32 + lane) * 4;
        if (c < C) {
          float4 g = make_float4(v[i].x * sc, v[i].y * sc, v[i].z * sc, v[i].w * sc);
          if (yi >= c && yi < c + 4) {  // the label's column: - 1/b
            const int j = yi - c;
            if (j == 0) g.x -= inv_b;
            if (j == 1) g.y -= inv_b;
            if (j == 2) g.z -= inv_b;
            if (j == 3) g.w -= inv_b;
          }
          store4<TDZ>(d, c, C, g.x, g.y, g.z, g.w);
        }
      }
    }
    return;
  }
  float m = -INFINITY;
  for (int c = lane; c < C; c += 32) m = fmaxf(m, z[c]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  float s = 0.f;
  for (int c = lane; c < C; c += 32) s += expf(z[c] - m);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float lse = m + logf(s);
  if (lane == 0) row_loss[warp] = lse - z[yi];
  if (dZ) {
    TDZ* d = dZ + (int64_t)warp * ldz;
    for (int c = lane; c < C; c += 32) {
      float p = expf(z[c] - lse);
      d[c] = to_act<TDZ>((p - (c == yi ? 1.f : 0.f)) * inv_b);
    }
  }
}

// ---------------------------------------------------------------------------------------
// bias gradient db = 1^T dZ (column sums over the batch), two deterministic passes:
//   pass 1: block (64 cols x 4 row lanes) sums rows [split*rps, (split+1)*rps) -> partial
//   pass 2: thread per column sums the splits in order; b -= lr*db (or stores db)
// ---------------------------------------------------------------------------------------
template <typename TDZ>
__global__ void colsum_partial_kernel(const TDZ* __restrict__ dZ, int64_t ld, int b, int n,
                                      int rows_per_split, float* __restrict__ partial) {
  __shared__ float red[4][64];
  const int col = blockIdx.x * 64 + threadIdx.x;
  const int r0 = blockIdx.y * rows_per_split;
  const int r1 = min(b, r0 + rows_per_split);
  float acc = 0.f;
  if (col < n)
    for (int r = r0 + threadIdx.y; r < r1; r += 4) acc += act_to_f(dZ[(int64_t)r * ld + col]);
  red[threadIdx.y][threadIdx.x] = acc;
  __syncthreads();
  if (threadIdx.y == 0 && col < n)
    partial[(int64_t)blockIdx.y * n + col] = (red[0][threadIdx.x] + red[1][threadIdx.x]) +
                                             (red[2][threadIdx.x] + red[3][threadIdx.x]);
}

static __global__ void bias_apply_kernel(const float* __restrict__ partial, int splits, int n, float lr,
                                  float* bias, float* grad_out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  float s = 0.f;
  for (int k = 0; k < splits; ++k) s += partial[(int64_t)k * n + c];
  if (grad_out)
    grad_out[c] = s;
  else
    bias[c] -= lr * s;
}

// ---------------------------------------------------------------------------------------
// fp32 check mode: SIMT GEMM C = A * B^T with generic strides and the same epilogues.
//   A(m,k) = A[m*sam + k*sak], B(n,k) = B[n*sbn + k*sbk].  64x64 tile, BK = 16, 256 threads,
//   4x4 outputs per thread.  Two-level fp32 accumulation (per 16-wide K tile, then total)
//   keeps the rounding error ~K/16 additions deep.
// ---------------------------------------------------------------------------------------
template <int EPI, typename TA, typename TB>
__global__ void __launch_bounds__(256) simt_gemm_kernel(const TA* __restrict__ A, int64_t sam,
                                                        int64_t sak, const TB* __restrict__ B,
                                                        int64_t sbn, int64_t sbk, int M, int N,
                                                        int K, EpiArgs ep) {
  __shared__ float As[16][68];
  __shared__ float Bs[16][68];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int m0 = blockIdx.y * 64, n0 = blockIdx.x * 64;
  float tot[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
    for (int i = threadIdx.x; i < 64 * 16; i += 256) {
      int mm = i >> 4, kk = i & 15;
      int gm = m0 + mm, gk = k0 + kk;
      As[kk][mm] = (gm < M && gk < K) ? act_to_f(A[(int64_t)gm * sam + (int64_t)gk * sak]) : 0.f;
      int gn = n0 + mm;
      Bs[kk][mm] = (gn < N && gk < K) ? act_to_f(B[(int64_t)gn * sbn + (int64_t)gk * sbk]) : 0.f;
    }
    __syncthreads();
    float part[4][4] = {};
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], bb[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) bb[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) part[i][j] = fmaf(a[i], bb[j], part[i][j]);
    }
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) tot[i][j] += part[i][j];
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int r = m0 + ty * 4 + i, n = n0 + tx * 4 + j;
      if (r < M && n < N) epi_elem<EPI, float, true>(ep, r, n, tot[i][j]);
    }
}

// ---------------------------------------------------------------------------------------
// deterministic sum of per-row losses into one double (single block, fixed order)
// ---------------------------------------------------------------------------------------
static __global__ void sum_rows_kernel(const float* __restrict__ v, int n, double* out, int slot, int accumulate = 0) {
  __shared__ double red[1024];
  double s = 0.0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) s += (double)v[i];
  red[threadIdx.x] = s;
  __syncthreads();
  for (int w = blockDim.x / 2; w > 0; w >>= 1) {
    if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) out[slot] = (accumulate ? out[slot] : 0.0) + red[0];
}

// bf16 shadow := RNE(fp32 master) over the whole flat parameter buffer
static __global__ void refresh_shadow_kernel(const float* __restrict__ master, __nv_bfloat16* shadow, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    shadow[i] = __float2bfloat16_rn(master[i]);
}

// replica merge: delta = W - W_base ... allreduce ... W = W_base + g*delta
static __global__ void merge_delta_kernel(const float* __restrict__ w, const float* __restrict__ base, float* delta, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    delta[i] = w[i] - base[i];
}

static __global__ void merge_apply_kernel(float* w, float* base, const float* __restrict__ delta, float gamma,
                                   __nv_bfloat16* shadow, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    float v = base[i] + gamma * delta[i];
    w[i] = v;
    base[i] = v;
    if (shadow) shadow[i] = __float2bfloat16_rn(v);
  }
}

// CSR -> dense rows [r0, r1) of X [.. x ldx] (zeroed beforehand): one warp per row scatters its
// nonzeros (hb_dataset format HB_DATA_CSR; the paper's sparse data "processed in dense format" [L255])
template <typename T>
static __global__ void densify_csr_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                          const T* __restrict__ vals, int64_t r0, int64_t r1, int64_t n_cols, T* X,
                                          int64_t ldx, int* bad) {
  const int64_t r = r0 + ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x & 31;
  if (r >= r1) return;
  T* row = X + r * ldx;
  for (int64_t k = indptr[r] + lane; k < indptr[r + 1]; k += 32) {
    const int32_t c = indices[k];
    if (c >= 0 && c < n_cols)
      row[c] = vals[k];
    else
      atomicOr(bad, 1);
  }
}

// the inverse scatter: zeros at the nonzero positions of rows [r0, r1) of a CSR structure (the
// previous dataset staged into X), so re-densifying a same-shape dataset needs no full memset
template <typename T>
static __global__ void zero_csr_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                       int64_t r0, int64_t r1, int64_t n_cols, T* X, int64_t ldx) {
  const int64_t r = r0 + ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x & 31;
  if (r >= r1) return;
  T* row = X + r * ldx;
  for (int64_t k = indptr[r] + lane; k < indptr[r + 1]; k += 32) {
    const int32_t c = indices[k];
    if (c >= 0 && c < n_cols) row[c] = T(0.f);
  }
}

// HB_CHECK=labels (hb_policy.check_labels): flag any label outside [0, C)
static __global__ void check_labels_kernel(const int32_t* __restrict__ y, int64_t n, int C, int* bad) {
  int any = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    any |= (y[i] < 0) | (y[i] >= C);
  if (__syncthreads_or(any) && threadIdx.x == 0) atomicOr(bad, 1);
}

// Local replica merge (hb_merge_replicas, PAPER.md L141 / L175): with G the global model, B the
// merge base (G at the previous sync point) and R_0..R_{n-1} the deep replicas of this process,
//   G <- G + gamma * sum_E (R_E - B)   (fixed E order)   then B, R_E <- G and every bf16 shadow
// is rewritten — one pass over the parameters (each replica read once and written once).
struct ReplicaPtrs {
  float* w[8];
  __nv_bfloat16* sh[8];
};
static __global__ void merge_replicas_kernel(float* g, float* base, __nv_bfloat16* g_shadow, ReplicaPtrs r, int n_rep,
                                             float gamma, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const float b0 = base[i];
    float d = 0.f;
    for (int e = 0; e < n_rep; ++e) d += r.w[e][i] - b0;
    const float v = g[i] + gamma * d;
    g[i] = v;
    base[i] = v;
    const __nv_bfloat16 h = __float2bfloat16_rn(v);
    if (g_shadow) g_shadow[i] = h;
    for (int e = 0; e < n_rep; ++e) {
      r.w[e][i] = v;
      if (r.sh[e]) r.sh[e][i] = h;
    }
  }
}

}  // namespace hb
