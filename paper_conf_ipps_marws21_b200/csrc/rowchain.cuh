// rowchain.cuh — fused per-row-block pass of one SGD step for narrow MLPs.
//
// For a net n_0 - n x (L-1) - C (uniform hidden width n <= 512, n_0 <= 512, C <= 16) one launch
// computes, for every block of 128 batch rows, everything of the step that is row-local:
//   forward   H_l = sigma(H_{l-1} W_l^T + b_l), S_l = sigma'(z)        l = 0..L-2  [Eq. (1), L43]
//   head      dZ_{L-1} = (softmax(H_{L-2} W_{L-1}^T + b_{L-1}) - Y)/b, row losses  [L258]
//   dX chain  dZ_{l-1} = (dZ_l W_l) * S_{l-1}                          l = L-1..1  [Eq. (2), L49]
// plus per-32-row column sums of every dZ (bias-gradient partials).  Only the dW GEMMs (K =
// batch, a reduction over ALL row blocks) remain; they run afterwards with the in-place SGD
// epilogue of tc_gemm.cuh, which also keeps Eq. (3)'s order: every dX read of W_l precedes the
// W_l update.
//
// The activations of a row block never leave the SM between layers: the A operand of every GEMM
// of the chain is a 128 x n bf16 tile resident in shared memory (`abuf`, SWIZZLE_128B K-major
// chunks of 64 columns), rewritten in place by the epilogue of the previous GEMM; only W streams
// in (TMA ring) and only what the dW GEMMs need (H_l, dZ_l, S_l) streams out (TMA stores).
// A cluster of CS = 1, 2, 4 or 8 CTAs shares a row block: CTA r computes output columns
// [r*NH, (r+1)*NH) of every layer and ships its 64-column chunks of the new activation tile to
// every other CTA of the cluster (cp.async.bulk shared::cta -> shared::cluster).  Splitting the
// columns divides the W bytes each SM must stream per layer by CS — the chain is bound by the
// W bytes in flight per SM (the shared memory left next to abuf) — so small batches use wide
// clusters and b = 8192 uses CS = 2 (64 row blocks x 2 CTAs fill the 148 SMs once).
//
// Roles (RC_THREADS = 640): warp 0 TMA producer (X once, W tiles of every step in MMA order), warp 1
// MMA issuer (one thread, tcgen05.mma M=128 N=NH into one of two TMEM accumulators), warp 2 TMEM
// allocator, warps 4..19 epilogue: quadrant q = warp % 4 (TMEM lanes = tile rows 32q..32q+31),
// part h = (warp-4)/4 (columns 16h..16h+15 of every 64-column chunk; the RC_PARTS warps of a
// quadrant meet on a named barrier before the chunk's 32-row piece is shipped, and lane 0 of
// three of them issue the peer bulk copies, the H/dZ TMA store and the sigma' TMA store).
//
// Synchronisation (mbarriers):
//   w_full/w_empty[stage]   W ring (TMA complete_tx / tcgen05.commit)
//   x_full                  X row block loaded (step 0 input)
//   chunk_ready[g]          abuf chunk g holds the previous step's output: 4 arrivals (one per
//                           32-row piece; a remote piece arrives with expect_tx + bulk copy)
//   head_ready              dZ_{L-1} tile written (input of the output layer's dX)
//   acc_full/acc_empty[2]   TMEM double buffer (MMA <-> epilogue)
//   peer_free               the OTHER CTAs' MMAs of the current step have completed (multicast
//                           commits, CS-1 arrivals per step): only then may this CTA overwrite
//                           chunks in their abufs (their input) or chunks of its own abuf whose
//                           previous bulk copies they had to consume.
#pragma once

#include "common.cuh"
#include "tc_gemm.cuh"

namespace hb {

constexpr int RC_MAX_L = 12;     // weight layers supported by one launch
constexpr int RC_MAX_CS = 8;     // CTAs per row block (portable cluster size)
// Epilogue warps: 4 TMEM quadrants x RC_PARTS column parts of every 64-column chunk (RC_PARTS = 4:
// 16 warps of 16 columns — twice the latency hiding of 2 x 32 columns; the per-chunk work is
// latency-bound, not issue-bound, on B200)
#ifndef RC_EPI_PARTS
#define RC_EPI_PARTS 4
#endif
constexpr int RC_PARTS = RC_EPI_PARTS;
constexpr int RC_EPI_WARPS = 4 * RC_PARTS;
constexpr int RC_THREADS = 128 + 32 * RC_EPI_WARPS;  // 4 control warps + the epilogue warps
constexpr int RC_EPI_THREADS = 32 * RC_EPI_WARPS;
constexpr int RC_CPW = 64 / RC_PARTS;  // columns of a chunk per epilogue warp
constexpr int RC_NG = RC_CPW / 16;     // 16-column groups per warp and chunk
constexpr int RC_NSV = RC_CPW / 8;     // uint4 of sigma' per warp row and chunk
constexpr int RC_H_COPY = RC_PARTS > 1 ? 1 : 0;  // epilogue part whose lane 0 ships pieces to peers
constexpr int RC_H_S = RC_PARTS > 2 ? 2 : 0;     // ... and whose lane 0 stores the sigma' pieces
constexpr int RC_CHUNK = 16384;  // 128 rows x 64 bf16 columns (SW128 K-major)
constexpr int RC_PIECE = 4096;   // 32 rows of a chunk (one quadrant's share)
constexpr int RC_MAX_STAGES = 12;

enum { RC_FWD = 0, RC_HEAD = 1, RC_DX = 2 };

// one warp's columns of a chunk from TMEM (32 lanes x RC_CPW columns)
__device__ __forceinline__ void rc_tmem_ld(uint32_t t, uint32_t (&r)[32]) { tmem_ld_32x32b_x32(t, r); }
__device__ __forceinline__ void rc_tmem_ld(uint32_t t, uint32_t (&r)[16]) { tmem_ld_32x32b_x16(t, r); }

__device__ __forceinline__ void epi_bar_sync_n(int) { asm volatile("bar.sync 1, %0;" ::"n"(RC_EPI_THREADS) : "memory"); }
// the RC_PARTS epilogue warps of quadrant q (named barriers 2..5)
__device__ __forceinline__ void quad_bar_sync(int q) {
  asm volatile("bar.sync %0, %1;" ::"r"(2 + q), "n"(32 * RC_PARTS) : "memory");
}

struct RcParams {
  CUtensorMap mX;                // X [x_rows x n0], box {64, 128}
  CUtensorMap mW[RC_MAX_L];      // W_l K-major, box {64, NH} (output layer {64, 16})
  CUtensorMap mWt[RC_MAX_L];     // W_l as MN-major operand (l >= 1), box {64, 64}
  CUtensorMap mH[RC_MAX_L];      // H_l store [b x n], box {64, 32}          (l <= L-2)
  CUtensorMap mDZ[RC_MAX_L];     // dZ_l store [b x n], box {64, 32}         (l <= L-2)
  CUtensorMap mS[RC_MAX_L];      // S_l store [b x n], box {64, 32}          (l <= L-2)
  const float* bias[RC_MAX_L];   // fp32 master b_l
  __nv_bfloat16* S[RC_MAX_L];    // sigma' stash S_l [b x ldo]                (l <= L-2)
  float* bpart[RC_MAX_L];        // bias-gradient partials of dZ_l [4 x row blocks x n_out(l)] (per quadrant)
  const int* d_off;              // device row offset of the batch in X / y (nullable)
  const int32_t* y;
  __nv_bfloat16* dz_head;        // dZ_{L-1} [b x ldo_head]
  float* row_loss;               // [b]
  int64_t ldo, ldo_head;
  int L, n0, n, C, b;
  int CS, NH;                    // cluster size, output columns per CTA (multiple of 64)
  int nstages, abuf_chunks, tmem_cols;
  int korder;                    // k-block order of chunked steps (rc_kchunk)
  int s_tma;                     // 1: sigma' stash staged in smem (2 chunk buffers) and TMA-stored
  float inv_b;
  unsigned long long* dbg;       // tuning only: per CTA, per step RC_DBG_W globaltimer stamps (nullable)
};
constexpr int RC_DBG_STEPS = 24;
constexpr int RC_DBG_W = 14;  // stamps per step

struct RcStep {
  int kind, layer, N, nkb, kkn;
  bool bmn;
};

// Step s of the chain: s < L-1 forward layer s; s = L-1 output layer + softmax-xent;
// s >= L dX of layer 2L-1-s (s = L: the output layer, K = C <= 16 -> one UMMA_K step).
__device__ __forceinline__ RcStep rc_step(const RcParams& P, int s) {
  RcStep st;
  if (s < P.L - 1) {
    st.kind = RC_FWD;
    st.layer = s;
    st.N = P.NH;
    st.nkb = ((s == 0 ? P.n0 : P.n) + 63) / 64;
    st.kkn = 4;
    st.bmn = false;
  } else if (s == P.L - 1) {
    st.kind = RC_HEAD;
    st.layer = P.L - 1;
    st.N = 16;
    st.nkb = (P.n + 63) / 64;
    st.kkn = 4;
    st.bmn = false;
  } else {
    st.kind = RC_DX;
    st.layer = 2 * P.L - 1 - s;
    st.N = P.NH;
    const bool head = st.layer == P.L - 1;
    st.nkb = head ? 1 : (P.n + 63) / 64;
    st.kkn = head ? 1 : 4;
    st.bmn = true;
  }
  return st;
}

// k-block i of step s reads abuf chunk rc_kchunk(...).  korder 2: own chunk t, then the other
// CTAs' chunks t-1 (a remote chunk arrives about one epilogue chunk after the local one).  korder 0: this CTA's own chunks first
// (its epilogue produced them, they are ready before the others arrive), then the others in index
// order.  korder 1: round robin over the cluster starting with this CTA (own c0, next CTA's c0, ...,
// own c1, ...): every CTA's epilogue emits its chunks in the same order at about the same time, so
// the MMAs (and the W ring behind them) keep pace with the epilogues instead of leaving all remote
// k-blocks — more W stages than the ring holds — for after the last chunk.
__device__ __forceinline__ int rc_kchunk(const RcParams& P, int s, int nkb, int i, int rank) {
  if (s == 0 || s == P.L) return i;
  const int ncl = P.NH / 64;
  if (P.korder == 2) {  // own chunks first, the other CTAs' chunks one position behind
    int v = 0;
    for (int t = 0; t <= ncl; ++t) {
      if (t < ncl) {
        const int g = rank * ncl + t;
        if (g < nkb && v++ == i) return g;
      }
      if (t >= 1)
        for (int p = 1; p < P.CS; ++p) {
          const int g = ((rank + p) % P.CS) * ncl + t - 1;
          if (g < nkb && v++ == i) return g;
        }
    }
    return i;
  }
  if (P.korder == 1) {
    for (int t = 0, v = 0; t < P.CS * ncl; ++t) {
      const int g = ((rank + t % P.CS) % P.CS) * ncl + t / P.CS;
      if (g < nkb && v++ == i) return g;
    }
    return i;  // unreachable for i < nkb
  }
  const int lo = rank * ncl, hi = min(lo + ncl, nkb);
  const int nown = max(0, hi - lo);
  if (i < nown) return lo + i;
  const int j = i - nown;
  return j < lo ? j : j + nown;
}

// abuf chunk that receives the dZ_{L-1} tile (the output layer's dX operand): with a cluster, the
// first chunk OWNED BY THE NEXT CTA — only its bulk copies ever write that chunk here, so after
// this CTA's output-layer MMAs it is free (no outgoing copy or TMA store reads it), and the
// owner's next write into it waits for this CTA's output-layer dX MMAs (peer_free)
__device__ __forceinline__ int rc_head_chunk(const RcParams& P, int rank) {
  return P.CS > 1 ? ((rank + 1) % P.CS) * (P.NH / 64) : 0;
}

__global__ void __launch_bounds__(RC_THREADS, 1) rowchain_kernel(const __grid_constant__ RcParams P) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int NCA = P.abuf_chunks;
  const int STB = P.NH * 128;  // W stage bytes: NH rows x 128 B (K-major) = NH/64 boxes of 8 KB (MN-major)
  const int NS = P.nstages;
  uint8_t* abuf = smem;
  uint8_t* ring = abuf + NCA * RC_CHUNK;
  uint8_t* sstage = ring + NS * STB;  // [2][RC_CHUNK] sigma' staging (s_tma), else empty
  float* sbias = reinterpret_cast<float*>(sstage + (P.s_tma ? 2 * RC_CHUNK : 0));  // [NH] bias of the current forward step
  uint64_t* w_full = reinterpret_cast<uint64_t*>(sbias + 256);
  uint64_t* w_empty = w_full + NS;
  uint64_t* chunk_ready = w_empty + NS;
  uint64_t* head_ready = chunk_ready + NCA;
  uint64_t* x_full = head_ready + 1;
  uint64_t* acc_full = x_full + 1;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* peer_free = acc_empty + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(peer_free + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int CS = P.CS;
  const int rank = CS > 1 ? (int)cluster_ctarank() : 0;
  const int rb = blockIdx.x / CS;  // row block
  const int NSTEPS = 2 * P.L - 1;
  const int hc = rc_head_chunk(P, rank);

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&P.mX);
    for (int s = 0; s < NS; ++s) {
      mbar_init(&w_full[s], 1);
      mbar_init(&w_empty[s], 1);
    }
    // chunk g: 4 local arrivals (one per 32-row piece) if this CTA produces it, else one
    // pre-arming arrival with expect_tx(16 KB) completed by the owner's four bulk copies
    const int ncl0 = P.NH / 64;
    for (int g = 0; g < NCA; ++g) mbar_init(&chunk_ready[g], g / ncl0 == rank ? 4 : 1);
    mbar_init(head_ready, 4);
    mbar_init(x_full, 1);
    for (int a = 0; a < 2; ++a) {
      mbar_init(&acc_full[a], 1);
      mbar_init(&acc_empty[a], RC_EPI_WARPS);
    }
    mbar_init(peer_free, CS > 1 ? CS - 1 : 1);
    fence_barrier_init();
    // pre-arm phase 0 of every valid chunk another CTA produces (step 0's output)
    for (int g = 0; g < NCA && g * 64 < P.n; ++g)
      if (g / ncl0 != rank) mbar_arrive_expect_tx(&chunk_ready[g], RC_CHUNK);
  }
  if (warp == 2) {
    switch (P.tmem_cols) {
      case 64: tmem_alloc<64>(tmem_slot); break;
      case 128: tmem_alloc<128>(tmem_slot); break;
      case 256: tmem_alloc<256>(tmem_slot); break;
      default: tmem_alloc<512>(tmem_slot); break;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (CS > 1) cluster_sync_all();  // the other CTAs' barriers are initialised before any remote op
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

  if (warp == 0 && lane == 0) {
    // ===== TMA producer: X row block, then the W tiles of every step in MMA k-order =====
    const int off = P.d_off ? __ldg(P.d_off) : 0;
    const int nc0 = (P.n0 + 63) / 64;
    mbar_arrive_expect_tx(x_full, nc0 * RC_CHUNK);
    for (int j = 0; j < nc0; ++j) tma_load_2d(abuf + j * RC_CHUNK, &P.mX, x_full, j * 64, off + rb * 128);
    int it = 0;
    for (int s = 0; s < NSTEPS; ++s) {
      const RcStep st = rc_step(P, s);
      for (int i = 0; i < st.nkb; ++i, ++it) {
        const int j = rc_kchunk(P, s, st.nkb, i, rank);
        const int stg = it % NS;
        mbar_wait(&w_empty[stg], ((it / NS) & 1) ^ 1);
        uint8_t* dst = ring + stg * STB;
        if (st.kind != RC_DX) {
          const int rows = st.kind == RC_HEAD ? 16 : P.NH;
          mbar_arrive_expect_tx(&w_full[stg], rows * 128);
          tma_load_2d(dst, &P.mW[st.layer], &w_full[stg], j * 64, st.kind == RC_HEAD ? 0 : rank * P.NH);
        } else {
          const int nb = P.NH / 64;
          mbar_arrive_expect_tx(&w_full[stg], nb * 8192);
          for (int q = 0; q < nb; ++q)
            tma_load_2d(dst + q * 8192, &P.mWt[st.layer], &w_full[stg], rank * P.NH + q * 64, j * 64);
        }
      }
    }
  } else if (warp == 1 && lane == 0) {
    // ===== MMA issuer =====
    int it = 0;
    uint32_t cnt_bits = 0;  // parity of the next chunk_ready phase per chunk
    const uint16_t others = (uint16_t)(((1u << CS) - 1) & ~(1u << rank));
    for (int s = 0; s < NSTEPS; ++s) {
      const RcStep st = rc_step(P, s);
      const int buf = s & 1;
      mbar_wait(&acc_empty[buf], ((s >> 1) & 1) ^ 1);
      tc_fence_after();
      unsigned long long* dbg =
          P.dbg && s < RC_DBG_STEPS ? P.dbg + ((size_t)blockIdx.x * RC_DBG_STEPS + s) * RC_DBG_W : nullptr;
      HB_STAMP(dbg, dbg[0]);
      const uint32_t tacc = tmem_base + (uint32_t)(buf * P.NH);
      const uint32_t idesc = make_idesc_bf16(128, st.N, false, st.bmn);
      // tuning only: per-k-block stamps of step 2 (issue, chunk ready, W ready) after the step table
      unsigned long long* kdbg = P.dbg && s == 2 ? P.dbg + (size_t)gridDim.x * RC_DBG_STEPS * RC_DBG_W : nullptr;
      for (int i = 0; i < st.nkb; ++i, ++it) {
        const int j = rc_kchunk(P, s, st.nkb, i, rank);
        HB_STAMP(kdbg && i < 16, kdbg[blockIdx.x * 16 + i]);
        uint8_t* a_ptr;
        if (s == 0) {
          if (i == 0) mbar_wait(x_full, 0);
          a_ptr = abuf + j * RC_CHUNK;
        } else if (s == P.L) {
          mbar_wait(head_ready, 0);
          a_ptr = abuf + hc * RC_CHUNK;
        } else {
          // local pieces: release.cta arrivals after fence.proxy.async; remote pieces: bulk copies
          // (async proxy, complete_tx) — both are ordered for the tensor core by the wait itself
          mbar_wait(&chunk_ready[j], (cnt_bits >> j) & 1);
          cnt_bits ^= 1u << j;
          // remote chunk: pre-arm its next phase (its owner writes it again after this step's
          // MMAs have completed, i.e. strictly after this arrive)
          if (j / (P.NH / 64) != rank && s < NSTEPS - 1) mbar_arrive_expect_tx(&chunk_ready[j], RC_CHUNK);
          a_ptr = abuf + j * RC_CHUNK;
        }
        HB_STAMP(kdbg && i < 16, kdbg[(gridDim.x + blockIdx.x) * 16 + i]);
        const int stg = it % NS;
        mbar_wait(&w_full[stg], (it / NS) & 1);
        tc_fence_after();
        HB_STAMP(kdbg && i < 16, kdbg[(2 * gridDim.x + blockIdx.x) * 16 + i]);
        HB_STAMP(dbg && i == 0, dbg[1]);
        const uint32_t a_base = smem_u32(a_ptr);
        const uint32_t b_base = smem_u32(ring + stg * STB);
        for (int kk = 0; kk < st.kkn; ++kk) {
          const uint64_t ad = make_sw128_desc(a_base + kk * 32, 16, 1024);
          const uint64_t bd = st.bmn ? make_sw128_desc(b_base + kk * 2048, 8192, 1024)
                                     : make_sw128_desc(b_base + kk * 32, 16, 1024);
          umma_bf16(tacc, ad, bd, idesc, (i | kk) != 0);
        }
        umma_commit(&w_empty[stg]);
      }
      umma_commit(&acc_full[buf]);
      if (CS > 1) umma_commit_multicast(peer_free, others);
      HB_STAMP(dbg, dbg[2]);
    }
  } else if (warp >= 4) {
    // ===== epilogue =====
    const int q = warp & 3;
    const int h = (warp - 4) >> 2;  // column part of every chunk: columns [h*RC_CPW, (h+1)*RC_CPW)
    const int et = threadIdx.x - 128;
    const int rl = q * 32 + lane;
    const int grow = rb * 128 + rl;  // batch row
    const bool row_ok = grow < P.b;
    const int ncl = P.NH / 64;
    const int n = P.n;
    const int64_t prow = (int64_t)rb * 4 + q;  // bias-gradient partial row of this quadrant
    int nmy = 0;                               // this CTA's chunks that start below n
    while (nmy < ncl && (rank * ncl + nmy) * 64 < n) ++nmy;
    for (int s = 0; s < NSTEPS; ++s) {
      const RcStep st = rc_step(P, s);
      const int buf = s & 1;
      const bool fwd = st.kind == RC_FWD;
      const int lo = fwd ? st.layer : st.layer - 1;  // layer whose activation / gradient is produced
      __nv_bfloat16* Sg = st.kind == RC_HEAD ? nullptr : P.S[lo];
      if (fwd) {  // stage this CTA's bias columns of the layer (previous step's readers are done)
        epi_bar_sync_n(RC_EPI_THREADS);
        const int nn = rank * P.NH + et;
        if (et < P.NH) sbias[et] = nn < n ? __ldg(P.bias[lo] + nn) : 0.f;
        epi_bar_sync_n(RC_EPI_THREADS);
      }
      // dX: prefetch this row's sigma' (this warp's columns of the first chunk) while the MMAs run
      uint4 sv[RC_NSV];
#pragma unroll
      for (int k = 0; k < RC_NSV; ++k) sv[k] = make_uint4(0, 0, 0, 0);
      if (st.kind == RC_DX && row_ok && nmy > 0 && (rank * ncl + 1) * 64 <= n) {
        const uint4* srow = reinterpret_cast<const uint4*>(Sg + (int64_t)grow * P.ldo + rank * ncl * 64 + h * RC_CPW);
#pragma unroll
        for (int k = 0; k < RC_NSV; ++k) sv[k] = __ldg(srow + k);
      }
      mbar_wait(&acc_full[buf], (s >> 1) & 1);
      tc_fence_after();
      unsigned long long* dbg =
          P.dbg && s < RC_DBG_STEPS && et == 0 ? P.dbg + ((size_t)blockIdx.x * RC_DBG_STEPS + s) * RC_DBG_W : nullptr;
      HB_STAMP(dbg, dbg[3]);
      if (CS > 1 && st.kind != RC_HEAD) mbar_wait(peer_free, s & 1);
      HB_STAMP(dbg, dbg[4]);
      const uint32_t tq = tmem_base + (uint32_t)(buf * P.NH) + ((uint32_t)(q * 32) << 16);
      if (st.kind == RC_HEAD) {
        // ---- softmax cross-entropy on the thread's row of logits (C <= 16) ----
        if (h == 0) {
          uint32_t raw[16];
          tmem_ld_32x32b_x16(tq, raw);
          tmem_ld_wait();
          const int C = P.C;
          const float* bl = P.bias[P.L - 1];
          float z[16], dz[16];
          float mx = -INFINITY;
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            z[j] = j < C ? __uint_as_float(raw[j]) + __ldg(bl + j) : -INFINITY;
            mx = fmaxf(mx, z[j]);
          }
          float se = 0.f;
#pragma unroll
          for (int j = 0; j < 16; ++j) se += j < C ? expf(z[j] - mx) : 0.f;
          const float lse = mx + logf(se);
          const int off = P.d_off ? __ldg(P.d_off) : 0;
          const int yi = row_ok ? __ldg(P.y + off + grow) : -1;
          float zy = 0.f;
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            dz[j] = (row_ok && j < C) ? (expf(z[j] - lse) - (j == yi ? 1.f : 0.f)) * P.inv_b : 0.f;
            zy = j == yi ? z[j] : zy;
          }
          uint32_t pk[8], lk[8];
          pack_hilo16(dz, pk, lk);  // hi feeds the chain's head dX; hi + lo the head dW GEMM (R24)
          // with a cluster the head chunk is never a TMA-store or bulk-copy source of this CTA
          // (rc_head_chunk); alone, it is chunk 0, last stored by this warp
          if (CS == 1) {
            if (lane == 0) tma_store_wait_read();
            __syncwarp();
          }
          const uint32_t row = smem_u32(abuf + hc * RC_CHUNK) + rl * 128;
          sts128(row + ((0 ^ (rl & 7)) << 4), pk[0], pk[1], pk[2], pk[3]);
          sts128(row + ((1 ^ (rl & 7)) << 4), pk[4], pk[5], pk[6], pk[7]);
          fence_proxy_async();
          __syncwarp();
          if (lane == 0) mbar_arrive(head_ready);
          if (rank == 0) {
            if (row_ok) {
              P.row_loss[grow] = lse - zy;
              uint4* D = reinterpret_cast<uint4*>(P.dz_head + (int64_t)grow * P.ldo_head);
              D[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
              if (P.ldo_head >= 16) D[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
              if (P.ldo_head >= 32) {  // lo plane at columns [16, 32)
                D[2] = make_uint4(lk[0], lk[1], lk[2], lk[3]);
                D[3] = make_uint4(lk[4], lk[5], lk[6], lk[7]);
              }
            }
            const float t = warp_colsum16(dz, lane);
            const int col = colsum16_col(lane);
            if (!(lane & 1) && col < C) P.bpart[P.L - 1][prow * C + col] = t;
          }
        }
      } else {
        // this quadrant's TMA stores of the previous step (H / dZ pieces by its h = 0 warp, sigma'
        // pieces by its h = RC_H_S warp) have read their smem before any part writes it again
        if ((h == 0 || h == RC_H_S) && lane == 0) tma_store_wait_read();
        quad_bar_sync(q);
        const bool signal = fwd || st.layer >= 2;  // the output is the next step's A operand
        for (int c = 0; c < nmy; ++c) {
          const int g = rank * ncl + c;
          const int n0 = g * 64;
          if (fwd && P.s_tma && c >= 2) {  // staging buffer c % 2: chunk c-2's S store has read it
            if (h == RC_H_S && lane == 0) tma_store_wait_read_1();
            quad_bar_sync(q);
          }
          const uint32_t srow_s = smem_u32(sstage + (c & 1) * RC_CHUNK + q * RC_PIECE) + lane * 128;
          const int nh = n0 + h * RC_CPW;  // first column of this warp's part
          const bool full_chunk = n0 + 64 <= n;
          uint32_t raw[RC_CPW];
          rc_tmem_ld(tq + (uint32_t)(c * 64 + h * RC_CPW), raw);
          // sigma' of the NEXT chunk: its global load overlaps this chunk's work (chunk 0's was
          // issued before the accumulator wait)
          uint4 svn[RC_NSV];
#pragma unroll
          for (int k = 0; k < RC_NSV; ++k) svn[k] = make_uint4(0, 0, 0, 0);
          if (!fwd && c + 1 < nmy && row_ok && n0 + 128 <= n) {
            const uint4* srow = reinterpret_cast<const uint4*>(Sg + (int64_t)grow * P.ldo + nh + 64);
#pragma unroll
            for (int k = 0; k < RC_NSV; ++k) svn[k] = __ldg(srow + k);
          }
          tmem_ld_wait();
          HB_STAMP(dbg && c == 0, dbg[6]);
          uint8_t* piece = abuf + g * RC_CHUNK + q * RC_PIECE;
          const uint32_t prow_s = smem_u32(piece) + lane * 128;
          const uint32_t sb_s = smem_u32(sbias) + (uint32_t)(c * 64 + h * RC_CPW) * 4;
#pragma unroll
          for (int g2 = 0; g2 < RC_NG; ++g2) {
            const int nc = nh + g2 * 16;
            uint32_t pk[8];
            if (fwd) {
              uint32_t sp[8];
              float bb[16];
#pragma unroll
              for (int k = 0; k < 4; ++k) {
                const float4 t = lds128f(sb_s + (uint32_t)(g2 * 16 + 4 * k) * 4);
                bb[4 * k] = t.x;
                bb[4 * k + 1] = t.y;
                bb[4 * k + 2] = t.z;
                bb[4 * k + 3] = t.w;
              }
#pragma unroll
              for (int k = 0; k < 8; ++k) {
                float h0, d0, h1, d1;
#ifdef HB_RC_FAKE_SIG  // tuning only (wrong numerics): epilogue cost without the MUFU work
                h0 = __uint_as_float(raw[g2 * 16 + 2 * k]) + bb[2 * k];
                h1 = __uint_as_float(raw[g2 * 16 + 2 * k + 1]) + bb[2 * k + 1];
                d0 = h0 * 0.25f;
                d1 = h1 * 0.25f;
#else
                sigmoid_d_fast2(__uint_as_float(raw[g2 * 16 + 2 * k]), __uint_as_float(raw[g2 * 16 + 2 * k + 1]),
                                bb[2 * k], bb[2 * k + 1], h0, h1, d0, d1);
#endif
                pk[k] = pack_bf16x2(h0, h1);
                sp[k] = pack_bf16x2(d0, d1);
              }
              if (P.s_tma) {  // swizzled like the H piece; rows >= b / columns >= n clipped by the store
                const int js = h * (RC_CPW / 8) + g2 * 2;
                sts128(srow_s + ((js ^ (lane & 7)) << 4), sp[0], sp[1], sp[2], sp[3]);
                sts128(srow_s + (((js + 1) ^ (lane & 7)) << 4), sp[4], sp[5], sp[6], sp[7]);
              } else if (row_ok) {
                __nv_bfloat16* srow = Sg + (int64_t)grow * P.ldo + nc;
                if (nc + 16 <= n) {
                  reinterpret_cast<uint4*>(srow)[0] = make_uint4(sp[0], sp[1], sp[2], sp[3]);
                  reinterpret_cast<uint4*>(srow)[1] = make_uint4(sp[4], sp[5], sp[6], sp[7]);
                } else {
#pragma unroll
                  for (int k = 0; k < 16; ++k)
                    if (nc + k < n) srow[k] = __ushort_as_bfloat16((unsigned short)(sp[k >> 1] >> (16 * (k & 1))));
                }
              }
            } else {
              float v[16];
              if (full_chunk) {
                const uint32_t sw[8] = {sv[2 * g2].x,     sv[2 * g2].y,     sv[2 * g2].z,     sv[2 * g2].w,
                                        sv[2 * g2 + 1].x, sv[2 * g2 + 1].y, sv[2 * g2 + 1].z, sv[2 * g2 + 1].w};
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                  const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&sw[k]));
                  v[2 * k] = __uint_as_float(raw[g2 * 16 + 2 * k]) * a.x;
                  v[2 * k + 1] = __uint_as_float(raw[g2 * 16 + 2 * k + 1]) * a.y;
                }
              } else {  // ragged last chunk: columns >= n are zero
                const __nv_bfloat16* srow = Sg + (int64_t)grow * P.ldo + nc;
#pragma unroll
                for (int k = 0; k < 16; ++k)
                  v[k] = (row_ok && nc + k < n) ? __uint_as_float(raw[g2 * 16 + k]) * __bfloat162float(srow[k]) : 0.f;
              }
#pragma unroll
              for (int k = 0; k < 8; ++k) pk[k] = pack_bf16x2(v[2 * k], v[2 * k + 1]);
              // bias-gradient partial of this quadrant's 32 rows (deterministic, reduced by the dW GEMM)
              const float t = warp_colsum16(v, lane);
              const int col = nc + colsum16_col(lane);
              if (!(lane & 1) && col < n) P.bpart[lo][prow * n + col] = t;
            }
            const int j0 = h * (RC_CPW / 8) + g2 * 2;  // 16-byte column chunk of the 128-byte row
            sts128(prow_s + ((j0 ^ (lane & 7)) << 4), pk[0], pk[1], pk[2], pk[3]);
            sts128(prow_s + (((j0 + 1) ^ (lane & 7)) << 4), pk[4], pk[5], pk[6], pk[7]);
          }
          HB_STAMP(dbg && c == 0, dbg[7]);
          fence_proxy_async();
          HB_STAMP(dbg && c == 0, dbg[10]);
          quad_bar_sync(q);  // both halves of the piece are written
          HB_STAMP(dbg && c == 0, dbg[11]);
          // the piece's asynchronous operations are issued by lane 0 of different warps of the
          // quadrant so their issue latencies overlap (each blocks ~0.1-0.3 us on B200):
          //   RC_H_COPY: bulk copies to the peers (their MMAs wait on them) + the local arrival,
          //   0:         TMA store of the H / dZ piece (one bulk group per chunk),
          //   RC_H_S:    TMA store of the sigma' staging piece (one bulk group per chunk)
          if (lane == 0) {
            if (h == RC_H_COPY && signal) {
              // the receivers pre-armed their chunk_ready[g] with expect_tx (MMA thread), so a
              // remote piece needs nothing but the bulk copy and its complete_tx
              for (int p = 1; p < CS; ++p) {
                const int dst = (rank + p) % CS;
                bulk_copy_s2cluster(mapa_shared(smem_u32(piece), dst), piece, RC_PIECE,
                                    mapa_shared(smem_u32(&chunk_ready[g]), dst));
              }
              mbar_arrive(&chunk_ready[g]);
              HB_STAMP(dbg && c == 0, dbg[12]);
            }
            if (h == 0) {
              tma_store_2d(fwd ? &P.mH[lo] : &P.mDZ[lo], piece, n0, rb * 128 + q * 32);
              tma_store_commit();
              HB_STAMP(dbg && c == 0, dbg[13]);
            }
            if (h == RC_H_S && fwd && P.s_tma) {
              tma_store_2d(&P.mS[lo], sstage + (c & 1) * RC_CHUNK + q * RC_PIECE, n0, rb * 128 + q * 32);
              tma_store_commit();  // one group per chunk (the staging reuse waits on chunk c-2's)
            }
          }
          HB_STAMP(dbg, dbg[c == 0 ? 8 : 9]);
#pragma unroll
          for (int k = 0; k < RC_NSV; ++k) sv[k] = svn[k];
        }
      }
      // release the accumulator (all TMEM reads of this warp have completed)
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_empty[buf]);
      HB_STAMP(dbg, dbg[5]);
    }
    if (lane == 0) tma_store_wait_all();
  }

  tc_fence_before();
  __syncthreads();
  if (CS > 1) cluster_sync_all();  // no remote access to this CTA's shared memory remains
  if (warp == 2) {
    tc_fence_after();
    switch (P.tmem_cols) {
      case 64: tmem_dealloc<64>(tmem_base); break;
      case 128: tmem_dealloc<128>(tmem_base); break;
      case 256: tmem_dealloc<256>(tmem_base); break;
      default: tmem_dealloc<512>(tmem_base); break;
    }
  }
}

}  // namespace hb
