// epilogue.cuh — the fused per-element epilogues of the MLP-SGD GEMMs.
//
//   EPI_FWD_SIG    Eq. (1) hidden layer [PAPER.md L43, L258]: z = acc + b_n; H = sigma(z);
//                  S = sigma'(z) = sigma(z)(1 - sigma(z)) stashed for the backward pass.
//   EPI_FWD_LOGITS Eq. (1) output layer: logits = acc + b_n (fp32), softmax follows.
//   EPI_DGRAD_SIG  Eq. (2) [L49]: dZ_{l-1} = (dZ_l W_l) * sigma'(Z_{l-1})  (acc * S).
//   EPI_WGRAD_SGD  Eq. (3) [L53] fused into the dW GEMM: W -= lr * dW in place on the
//                  shared fp32 master, bf16 shadow rewritten (Hogbatch update, L170).
//   EPI_WGRAD_STORE test-only: dW written out (mlp_step_grads).
#pragma once

#include "common.cuh"

namespace hb {

constexpr int HB_MAX_PEERS = 7;

enum { EPI_FWD_SIG = 0, EPI_FWD_LOGITS = 1, EPI_DGRAD_SIG = 2, EPI_WGRAD_SGD = 3, EPI_WGRAD_STORE = 4,
       EPI_HEAD_XENT = 5 };

struct EpiArgs {
  int M, N;             // valid output extent (rows, cols of the GEMM result)
  const float* bias;    // FWD: [N]
  void* out0;           // FWD_SIG: H; LOGITS: fp32 logits; DGRAD: dZ; WGRAD_STORE: fp32 grad
  int64_t ld0;
  void* out1;           // FWD_SIG: S = sigma'(z) (nullable: forward-only / loss evaluation)
  int64_t ld1;
  const void* aux;      // DGRAD: S of the layer below
  int64_t ldaux;
  float* master;        // WGRAD_SGD: fp32 master weights
  __nv_bfloat16* shadow;// WGRAD_SGD: bf16 shadow (nullable in fp32 check mode)
  int64_t ldw;
  float lr;
  int transposed;       // WGRAD: result element (m, n) belongs to W[n][m]
  // split-precision head gradient (R24): the output layer's dZ_L is stored as two bf16
  // planes, hi = bf16(dZ) in columns [0, hilo) and lo = bf16(dZ - hi) in [hilo, 2 hilo) of the same
  // rows.  HEAD_XENT writes both; the transposed head WGRAD runs with N = 2 hilo and adds the two
  // column halves of its accumulator (dW_L = hi^T H + lo^T H), so dW_L sees dZ_L to ~2^-17.
  int hilo;             // 0 = plain bf16 dZ_L; else the lo plane's column offset (16)
  int n_real;           // hilo: the real column count C of the output (ep.N = 2 hilo is the GEMM extent)
  // bias gradient fused into the GEMMs (tensor-core path):
  float* bpart_out;     // DGRAD / HEAD_XENT: column sums of the produced dZ per 128-row M tile
  const float* bpart_in;// WGRAD: those partials for dZ_l; reduced in fixed order to db_l
  int64_t ldp;          // row stride of the partial arrays (= n_out of the layer)
  int n_mtiles;         // WGRAD: number of partial rows (ceil(b / 128))
  float* bias_upd;      // WGRAD_SGD: b_l -= lr * db_l in place
  float* bias_grad;     // WGRAD_STORE: db_l written out
  float* ws;            // WGRAD split-K: fp32 partial tiles [tiles][splits][128][BN]
  unsigned long long* dbg;  // tuning only: per-CTA phase timestamps (globaltimer ns), nullable
  int force_bn, force_splits;  // host-side launch choices for dW GEMMs (0 = heuristic)
  int pair;                    // host-side: dW GEMM on CTA pairs (tcgen05 cta_group::2) when eligible
  int fwd_pair;                // host-side: forward / dX GEMM on persistent CTA pairs when eligible
  int no_pdl;                  // host-side: launch without programmatic dependent launch
  int atomic;                  // WGRAD_SGD: W -= lr * dW with atomic adds (HB_UPDATE_ATOMIC)
  // asynchronous cross-replica Hogbatch (NEXT f2, mlp_attach_peers): every update of W / b is also
  // added, scaled by pscale (stale-gradient damping [L175]), to each peer replica's fp32 master
  // with an atomic add (peer-to-peer over NVLink), and the peer's bf16 shadow element rewritten
  int npeer;
  float pscale;
  int64_t pm_off[HB_MAX_PEERS];  // peer master - this master (elements)
  int64_t ps_off[HB_MAX_PEERS];  // peer shadow - this shadow (elements)
  // softmax cross-entropy head fused into the output-layer GEMM (C <= 16):
  const int32_t* y;     // labels (dataset base when yoff != nullptr)
  const int* yoff;      // device row offset of the batch (graph replay), nullable
  float* row_loss;      // per-row cross-entropy
  float inv_b;          // 1 / b (gradient of the batch MEAN loss)
  // fused dX of the output layer (HEAD_XENT, nullable): dZ_{L-1} = (dZ_L W_L) * S_{L-1}
  const float* w_head;  // fp32 master W_L [C x ldw_head], read before the W_L update
  int64_t ldw_head;
  int n_prev;           // n_{L-1}
  const __nv_bfloat16* s_prev;  // S_{L-1} (sigma' stash) [b x ld_prev]
  __nv_bfloat16* dz_prev;       // dZ_{L-1} [b x ld_prev]
  int64_t ld_prev;
  float* bpart_prev;    // bias partials of dZ_{L-1} [m tiles x n_prev]
};

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  __nv_bfloat162 t = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&t);
}

// f2: add -lr * pscale * g to element idx of every peer replica (and rewrite its shadow element)
__device__ __forceinline__ void peer_push1(const EpiArgs& ep, float* w_local, __nv_bfloat16* sh_local, float g) {
  const float d = __fmul_rn(-ep.lr * ep.pscale, g);
  for (int p = 0; p < ep.npeer; ++p) {
    const float nv = atomicAdd(w_local + ep.pm_off[p], d) + d;
    if (sh_local) sh_local[ep.ps_off[p]] = __float2bfloat16_rn(nv);
  }
}

template <typename T>
__device__ __forceinline__ T to_act(float v);
template <>
__device__ __forceinline__ float to_act<float>(float v) { return v; }
template <>
__device__ __forceinline__ __nv_bfloat16 to_act<__nv_bfloat16>(float v) { return __float2bfloat16_rn(v); }

__device__ __forceinline__ float act_to_f(float v) { return v; }
__device__ __forceinline__ float act_to_f(__nv_bfloat16 v) { return __bfloat162float(v); }

// Scalar epilogue for one output element (r, n) with accumulator value v.
// TAct = activation storage type (bf16 in the tensor-core path, fp32 in check mode).
// PRECISE selects expf (check mode) instead of __expf.
template <int EPI, typename TAct, bool PRECISE>
__device__ __forceinline__ void epi_elem(const EpiArgs& ep, int r, int n, float v) {
  if (EPI == EPI_FWD_SIG) {
    float z = v + ep.bias[n];
    float h, d;
    if (PRECISE) {  // check mode: IEEE exp/div, same cancellation-free form
      const float e = expf(-fabsf(z)), s = 1.0f / (1.0f + e);
      h = z >= 0.f ? s : e * s;
      d = e * s * s;
    } else {
      sigmoid_d(z, h, d);
    }
    static_cast<TAct*>(ep.out0)[(int64_t)r * ep.ld0 + n] = to_act<TAct>(h);
    if (ep.out1) static_cast<TAct*>(ep.out1)[(int64_t)r * ep.ld1 + n] = to_act<TAct>(d);
  } else if (EPI == EPI_FWD_LOGITS) {
    static_cast<float*>(ep.out0)[(int64_t)r * ep.ld0 + n] = v + ep.bias[n];
  } else if (EPI == EPI_DGRAD_SIG) {
    float s = act_to_f(static_cast<const TAct*>(ep.aux)[(int64_t)r * ep.ldaux + n]);
    static_cast<TAct*>(ep.out0)[(int64_t)r * ep.ld0 + n] = to_act<TAct>(v * s);
  } else if (EPI == EPI_WGRAD_SGD) {
    int64_t idx = ep.transposed ? (int64_t)n * ep.ldw + r : (int64_t)r * ep.ldw + n;
    float w;
    if (ep.atomic) {  // HB_UPDATE_ATOMIC: concurrent workers' updates of this weight all survive
      const float d = __fmul_rn(-ep.lr, v);
      w = atomicAdd(ep.master + idx, d) + d;
    } else {          // Hogwild read-modify-write [L128, L170] (same rounding: no fused multiply-add)
      w = ep.master[idx] + __fmul_rn(-ep.lr, v);
      ep.master[idx] = w;
    }
    if (ep.shadow) ep.shadow[idx] = __float2bfloat16_rn(w);
    if (ep.npeer) peer_push1(ep, ep.master + idx, ep.shadow ? ep.shadow + idx : nullptr, v);
  } else {  // EPI_WGRAD_STORE
    int64_t idx = ep.transposed ? (int64_t)n * ep.ldw + r : (int64_t)r * ep.ldw + n;
    static_cast<float*>(ep.out0)[idx] = v;
  }
}

// -lr * g for 4 weights, rounded once per product (no fused multiply-add): the Hogwild and the
// atomic update then produce the same bits for the same accumulator values
__device__ __forceinline__ float4 sgd_delta4(float lr, float a, float b, float c, float d) {
  return make_float4(__fmul_rn(-lr, a), __fmul_rn(-lr, b), __fmul_rn(-lr, c), __fmul_rn(-lr, d));
}

// HB_UPDATE_ATOMIC: W += d with one 16-byte atomic (sm_90+ float4 atomicAdd on global memory);
// returns the new value as seen by this update (old + d) for the bf16 shadow
__device__ __forceinline__ float4 sgd_atomic4(float4* W, float4 d) {
  const float4 old = atomicAdd(W, d);
  return make_float4(old.x + d.x, old.y + d.y, old.z + d.z, old.w + d.w);
}

// 16 fp32 values -> packed bf16 hi = bf16(v) and lo = bf16(v - hi) (R24: v = hi + lo to ~2^-17 |v|)
__device__ __forceinline__ void pack_hilo16(const float (&v)[16], uint32_t (&hp)[8], uint32_t (&lp)[8]) {
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const __nv_bfloat162 h = __floats2bfloat162_rn(v[2 * k], v[2 * k + 1]);
    const float2 hf = __bfloat1622float2(h);
    hp[k] = *reinterpret_cast<const uint32_t*>(&h);
    lp[k] = pack_bf16x2(v[2 * k] - hf.x, v[2 * k + 1] - hf.y);
  }
}

// Vectorised epilogue for 16 consecutive columns n0..n0+15 of row r (all valid, 16-byte
// aligned rows).  Used by the tensor-core kernel for full column chunks.
template <int EPI>
__device__ __forceinline__ void epi_row16_bf16(const EpiArgs& ep, int r, int n0, const float* v) {
  if (EPI == EPI_FWD_SIG) {
    uint32_t hp[8], sp[8];
    const float4* b4 = reinterpret_cast<const float4*>(ep.bias + n0);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float4 bb = __ldg(b4 + q);
      float z0 = v[4 * q] + bb.x, z1 = v[4 * q + 1] + bb.y, z2 = v[4 * q + 2] + bb.z,
            z3 = v[4 * q + 3] + bb.w;
      float h0, h1, h2, h3, d0, d1, d2, d3;
      sigmoid_d(z0, h0, d0);
      sigmoid_d(z1, h1, d1);
      sigmoid_d(z2, h2, d2);
      sigmoid_d(z3, h3, d3);
      hp[2 * q] = pack_bf16x2(h0, h1);
      hp[2 * q + 1] = pack_bf16x2(h2, h3);
      sp[2 * q] = pack_bf16x2(d0, d1);
      sp[2 * q + 1] = pack_bf16x2(d2, d3);
    }
    uint4* H = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0 + n0);
    H[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
    H[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
    if (ep.out1) {
      uint4* S = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out1) + (int64_t)r * ep.ld1 + n0);
      S[0] = make_uint4(sp[0], sp[1], sp[2], sp[3]);
      S[1] = make_uint4(sp[4], sp[5], sp[6], sp[7]);
    }
  } else if (EPI == EPI_DGRAD_SIG) {
    const uint4* S = reinterpret_cast<const uint4*>(static_cast<const __nv_bfloat16*>(ep.aux) +
                                                    (int64_t)r * ep.ldaux + n0);
    uint4 s0 = S[0], s1 = S[1];
    const __nv_bfloat162* sv0 = reinterpret_cast<const __nv_bfloat162*>(&s0);
    const __nv_bfloat162* sv1 = reinterpret_cast<const __nv_bfloat162*>(&s1);
    uint32_t o[8];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float2 a = __bfloat1622float2(sv0[q]);
      o[q] = pack_bf16x2(v[2 * q] * a.x, v[2 * q + 1] * a.y);
      float2 c = __bfloat1622float2(sv1[q]);
      o[4 + q] = pack_bf16x2(v[8 + 2 * q] * c.x, v[8 + 2 * q + 1] * c.y);
    }
    uint4* D = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0 + n0);
    D[0] = make_uint4(o[0], o[1], o[2], o[3]);
    D[1] = make_uint4(o[4], o[5], o[6], o[7]);
  } else if (EPI == EPI_WGRAD_SGD && 1) {
    float4* W = reinterpret_cast<float4*>(ep.master + (int64_t)r * ep.ldw + n0);
    uint32_t sp[8];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float4 w;
      if (ep.atomic) {
        w = sgd_atomic4(W + q, sgd_delta4(ep.lr, v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]));
      } else {
        w = W[q];
        const float4 d = sgd_delta4(ep.lr, v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
        w.x += d.x;
        w.y += d.y;
        w.z += d.z;
        w.w += d.w;
        W[q] = w;
      }
      sp[2 * q] = pack_bf16x2(w.x, w.y);
      sp[2 * q + 1] = pack_bf16x2(w.z, w.w);
    }
    uint4* Sh = reinterpret_cast<uint4*>(ep.shadow + (int64_t)r * ep.ldw + n0);
    Sh[0] = make_uint4(sp[0], sp[1], sp[2], sp[3]);
    Sh[1] = make_uint4(sp[4], sp[5], sp[6], sp[7]);
    if (ep.npeer) {
#pragma unroll
      for (int k = 0; k < 16; ++k) peer_push1(ep, ep.master + (int64_t)r * ep.ldw + n0 + k, ep.shadow + (int64_t)r * ep.ldw + n0 + k, v[k]);
    }
  } else {
#pragma unroll
    for (int j = 0; j < 16; ++j) epi_elem<EPI, __nv_bfloat16, false>(ep, r, n0 + j, v[j]);
  }
}

}  // namespace hb
