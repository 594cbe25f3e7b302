// tc_gemm.cuh — warp-specialised tcgen05 GEMM for sm_100a with TMA loads, a TMEM accumulator
// and the fused MLP-SGD epilogues of epilogue.cuh.
//
//   C[M x N] = A[M x K] * B[N x K]^T         (bf16 operands, fp32 accumulate in TMEM)
//
// The three contractions of one SGD step (Eq. (1)/(2), L43/L49) map onto it as
//   forward  H_l  = sigma(H_{l-1} W_l^T + b_l)   A = H_{l-1} (K-major), B = W_l (K-major)
//   head     dZ_L = softmax(H W_L^T + b_L) - Y    (fused cross-entropy epilogue, C <= 16)
//   dgrad    dZ   = (dZ_l W_l) * S               A = dZ_l   (K-major), B = W_l (MN-major)
//   wgrad    W_l -= lr * dZ_l^T H_{l-1}          A = dZ_l   (MN-major), B = H_{l-1} (MN-major)
// so the same kernel serves all of them; the operand major-ness is a template parameter and is
// handled entirely by the TMA box shape and the UMMA shared-memory descriptor, never by a copy.
// The bias gradient db_l = 1^T dZ_l is fused as well: the epilogue that PRODUCES dZ (dgrad /
// head) writes per-128-row column sums, and the wgrad epilogue reduces them in fixed order and
// applies b_l -= lr * db_l — no separate reduction kernel, deterministic.
//
// CTA = 384 threads: warp 0 TMA producer, warp 1 MMA issuer (one elected thread), warp 2 TMEM
// allocator, warps 4..11 epilogue (warp w reads TMEM lanes 32*(w%4)..+31 = tile rows, and one
// half of the tile's columns); the epilogue warps stage the bias and prefetch the sigma' stash
// while the mainloop runs.
// Tile: BLOCK_M = 128 (UMMA M = 128, cta_group::1), BLOCK_N = BN (16..256), BLOCK_K = 64 (one
// 128-byte swizzle atom of bf16).  smem stages form an mbarrier ring (full/empty).
// offA / offB (nullable, device) add a row offset to the stored-row coordinate of A / B: the
// batch's first row inside the HBM-resident dataset, written once per step (graph replay).
#pragma once

#include "common.cuh"
#include "epilogue.cuh"

namespace hb {

constexpr int TC_BM = 128;
constexpr int TC_BK = 64;
#ifndef HB_EPI_WARPS
#define HB_EPI_WARPS 8
#endif
constexpr int TC_EPI_WARPS = HB_EPI_WARPS;         // epilogue warps: 4 TMEM lane quadrants x column parts
constexpr int TC_EPI_THREADS = TC_EPI_WARPS * 32;
constexpr int TC_EPI_PARTS = TC_EPI_WARPS / 4;
constexpr int TC_THREADS = 128 + TC_EPI_THREADS;   // 4 control warps + the epilogue warps

// Epilogues whose bf16 outputs are staged in swizzled shared memory and written with TMA bulk
// stores (full 128-byte lines instead of one 16-byte piece of 32 different rows per warp store).
// The tile is written in 64-column chunks through TWO staging buffers: chunk j is staged while the
// bulk stores of chunk j-1 drain, so the staging costs 2 x NOUT x 16 KB whatever BN (B200, C3
// 8192x1024x1024: 256-wide tiles with a whole-tile staged epilogue were epilogue-bound).
// CTA pairs load half of B per stage, so their ring keeps 5 stages next to two H staging buffers:
// measured on B200 (scripts/gpu_ab_nbuf.sh, C4, alternating reps) 2.123 / 2.128 M samples/s against
// 2.093 / 2.106 M with one buffer and 6 stages; staging sigma' as well (HB_PAIR_NOUT = 2, 4 stages)
// measured slower (2.077 / 2.066 M)
#ifndef HB_PAIR_NBUF
#define HB_PAIR_NBUF 2
#endif
#ifndef HB_PAIR_NOUT
#define HB_PAIR_NOUT 1
#endif
template <int BN, int EPI, bool PAIR = false>
struct TmaOut {
#ifndef HB_TMA_OUT_MAX_BN
#define HB_TMA_OUT_MAX_BN 256
#endif
  static constexpr bool on = (EPI == EPI_FWD_SIG || EPI == EPI_DGRAD_SIG) && (BN == 64 || BN == 128 || BN == 256) &&
                             BN <= HB_TMA_OUT_MAX_BN;
  static constexpr int NCHUNK = BN / 64;                   // 64-column chunks per tile
  // 256-wide tiles keep a 4-deep operand ring: one staging buffer, and the forward's sigma' stash
  // is written directly (only H goes through TMA); narrower tiles double-buffer H and S
  // (CTA pairs load half of B per stage, so their ring has room for more staging)
  static constexpr int NBUF = BN == 128 || (PAIR && HB_PAIR_NBUF == 2) ? 2 : 1;
  static constexpr int NOUT = EPI == EPI_FWD_SIG && (BN <= 128 || (PAIR && HB_PAIR_NOUT == 2)) ? 2 : 1;  // staged outputs
  static constexpr int BYTES = on ? NBUF * NOUT * TC_BM * 128 : 0;
};

// PAIR: a CTA pair (cluster x = 2) computes a 256 x BN tile with tcgen05.mma.cta_group::2 — each
// CTA loads its own 128 A rows and HALF of the B tile (BN/2 rows), the leader issues the MMAs.
// Two uses: split-K dW GEMMs (one tile per pair, clusters (2, 1, S)) and persistent forward / dX
// GEMMs (clusters (2, 1, 1) walking 256 x 256 tiles): per SM the pair halves the B operand's shared-
// memory fill and tensor-core read and the L2 traffic per flop against a 128 x 256 tile.
template <int BN, bool B_MN, int EPI = EPI_WGRAD_SGD, bool PAIR = false>
struct TcCfg {
  static constexpr int A_BYTES = TC_BM * TC_BK * 2;                     // 16 KB
  static constexpr int B_TILE = PAIR ? BN / 2 : BN;                     // B rows this CTA loads
  static constexpr int B_ROWS = B_MN ? (B_TILE < 64 ? 64 : B_TILE) : B_TILE;  // MN-major loads 64-wide boxes
  static constexpr int B_BYTES = B_ROWS * TC_BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int OUT_BYTES = TmaOut<BN, EPI, PAIR>::BYTES;
#ifndef HB_RING_BYTES
#define HB_RING_BYTES (210 * 1024)
#endif
  static constexpr int STAGES_RAW = (HB_RING_BYTES - OUT_BYTES) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  // two accumulators (double buffer); TMEM is allocated in powers of two >= 32 columns
  static constexpr int TMEM_COLS = 2 * BN <= 32 ? 32 : 2 * BN <= 64 ? 64 : 2 * BN <= 128 ? 128 : 2 * BN <= 256 ? 256 : 512;
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + OUT_BYTES + 1024 /*align*/ + 256 /*barriers*/;
};

__device__ __forceinline__ void epi_bar_sync() { asm volatile("bar.sync 1, %0;" ::"n"(TC_EPI_THREADS) : "memory"); }

// Column sums of a 32-row x 16-column register tile (one row per lane) in 16 shuffles
// (reduce-scatter): afterwards lane L holds the total of column
// 8*b4(L) + 4*b3(L) + 2*b2(L) + b1(L), where bk(L) is bit k of L (pairs L, L^1 agree).
__device__ __forceinline__ float warp_colsum16(const float (&v)[16], int lane) {
  float a[8], b[4], c[2];
  bool up = lane & 16;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    float send = up ? v[j] : v[j + 8], keep = up ? v[j + 8] : v[j];
    a[j] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
  }
  up = lane & 8;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    float send = up ? a[j] : a[j + 4], keep = up ? a[j + 4] : a[j];
    b[j] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
  }
  up = lane & 4;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    float send = up ? b[j] : b[j + 2], keep = up ? b[j + 2] : b[j];
    c[j] = keep + __shfl_xor_sync(0xffffffffu, send, 4);
  }
  up = lane & 2;
  float d = (up ? c[1] : c[0]) + __shfl_xor_sync(0xffffffffu, up ? c[0] : c[1], 2);
  return d + __shfl_xor_sync(0xffffffffu, d, 1);
}

__device__ __forceinline__ int colsum16_col(int lane) {
  return ((lane >> 4) & 1) * 8 + ((lane >> 3) & 1) * 4 + ((lane >> 2) & 1) * 2 + ((lane >> 1) & 1);
}

// Bias gradient of rows [lo, hi): db[bi] = sum_t part[t * ldp + bi] over the n_mtiles partial rows
// written by the dZ producer, then b -= lr * db (SGD) or db stored (grads).  The 256 epilogue
// threads split the work: tpr adjacent lanes per bias entry, each summing every tpr-th partial
// row with 8 independent accumulators (loads in flight), combined in a fixed butterfly order —
// deterministic, and no long chain of dependent L2 loads on the tail of the dW GEMM.
template <int EPI>
__device__ __forceinline__ void bias_reduce_update(const EpiArgs& ep, int lo, int hi, int tid) {
  const int R = hi - lo;
  if (R <= 0) return;  // CTA-uniform
  int tpr = 1;
  while (tpr < 32 && tpr * 2 * R <= TC_EPI_THREADS) tpr *= 2;
  const int r = tid / tpr, k = tid % tpr;
  const int nt = ep.n_mtiles;
  float acc = 0.f;
  if (r < R) {
    const float* col = ep.bpart_in + lo + r;
    float a[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) a[u] = 0.f;
    int t = k;
    for (; t + 7 * tpr < nt; t += 8 * tpr) {
#pragma unroll
      for (int u = 0; u < 8; ++u) a[u] += __ldcg(col + (int64_t)(t + u * tpr) * ep.ldp);
    }
    for (; t < nt; t += tpr) a[0] += __ldcg(col + (int64_t)t * ep.ldp);
    acc = ((a[0] + a[1]) + (a[2] + a[3])) + ((a[4] + a[5]) + (a[6] + a[7]));
  }
  for (int o = 1; o < tpr; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (r < R && k == 0) {
    const int bi = lo + r;
    if (EPI == EPI_WGRAD_SGD) {
      if (ep.atomic)
        atomicAdd(ep.bias_upd + bi, __fmul_rn(-ep.lr, acc));
      else
        ep.bias_upd[bi] += __fmul_rn(-ep.lr, acc);
      if (ep.npeer) peer_push1(ep, ep.bias_upd + bi, nullptr, acc);  // biases have no shadow
    }
    else
      ep.bias_grad[bi] = acc;
  }
}

// Grouped tile rasterisation: consecutive tile indices walk down GROUP_M row tiles before moving
// to the next column tile, so the ~148 tiles resident at once cover a compact block of the
// output and share both their A row panels and their B column panels through L2.  With ~148
// tiles in flight a group of m row tiles spans ~148/m column tiles, so per wave the A panels are
// re-read tiles_n*m/148 times and the B panels tiles_m/m times; for the C4 layer-1 GEMMs (64 x 16
// and 32 x 82 tiles) the traffic minimum is near m = 17.  GROUP_M = 16 measured 1.60 GB of DRAM
// traffic per layer-1 wgrad+SGD launch against 2.08 GB at 8, and +1.1 % C4 samples/s
// (profiles/r02_group_m.txt).
// CTA pairs have ~74 pair tiles in flight, so the same model gives A re-reads tiles_n*m/74 and B
// re-reads tiles_mp/m per group of m PAIR rows: the minimum for both C4 layer-1 GEMMs (32 x 16 and
// 16 x 82 pair tiles) is near m = 8.6, i.e. 8 pair rows (16 row tiles, as before the pairs).
#ifndef HB_GROUP_M
#define HB_GROUP_M 16
#endif
#ifndef HB_GROUP_M_PAIR
#define HB_GROUP_M_PAIR 8
#endif
constexpr int TC_GROUP_M = HB_GROUP_M;
constexpr int TC_GROUP_M_PAIR = HB_GROUP_M_PAIR;
template <int GROUP>
__device__ __forceinline__ void tile_coords(int t, int tiles_m, int tiles_n, int& m_tile, int& n_tile) {
  const int per_group = GROUP * tiles_n;
  const int g = t / per_group;
  const int first_m = g * GROUP;
  const int gm = min(tiles_m - first_m, GROUP);
  const int r = t - g * per_group;
  m_tile = first_m + r % gm;
  n_tile = r / gm;
}

// Write 16 bf16 values (8 packed words) of tile row rl, tile columns c..c+15 into staging output o
// (boxes of 128 rows x 64 columns, 128-byte rows, 16-byte chunks XOR-swizzled by row % 8 — the
// TMA SWIZZLE_128B layout, which also makes these per-row writes bank-conflict free).
// 16 bf16 values (8 packed words) of tile row rl, chunk columns c..c+15 (c < 64) into a 128-row x
// 128-byte staging box (TMA SWIZZLE_128B layout)
__device__ __forceinline__ void stage16_box(uint8_t* box, int rl, int c, const uint32_t* p) {
  const int j0 = c >> 3;
  uint8_t* row = box + (size_t)rl * 128;
  *reinterpret_cast<uint4*>(row + ((j0 ^ (rl & 7)) << 4)) = make_uint4(p[0], p[1], p[2], p[3]);
  *reinterpret_cast<uint4*>(row + (((j0 + 1) ^ (rl & 7)) << 4)) = make_uint4(p[4], p[5], p[6], p[7]);
}

template <int NBOX>
__device__ __forceinline__ void stage16(uint8_t* sout, int o, int rl, int c, const uint32_t* p) {
  const int box = c >> 6, j0 = (c & 63) >> 3;
  uint8_t* row = sout + ((size_t)(o * NBOX + box) * TC_BM + rl) * 128;
  *reinterpret_cast<uint4*>(row + ((j0 ^ (rl & 7)) << 4)) = make_uint4(p[0], p[1], p[2], p[3]);
  *reinterpret_cast<uint4*>(row + (((j0 + 1) ^ (rl & 7)) << 4)) = make_uint4(p[4], p[5], p[6], p[7]);
}

// The fused epilogue of ONE output tile (m_tile, n_tile) whose accumulator is TMEM buffer `acc` of
// the CTA's i-th tile: bias staging / sigma' prefetch, wait for the MMAs, TMEM -> registers ->
// EPI-specific epilogue (epilogue.cuh) -> global (or the split-K park), then release the
// accumulator to the MMA warp.  Executed by the TC_EPI_WARPS epilogue warps; shared by
// tc_gemm_kernel and the persistent small-batch step kernel (step_kernel.cuh).
struct EpiTileCtx {
  uint32_t tmem_base;
  uint64_t* tmem_full_bar;
  uint64_t* tmem_empty_bar;
  float* sbias;         // [2][BN]
  float* red;           // [4 * BN]
  float* dzs;           // [TC_BM * 16] (HEAD_XENT fused dX)
  uint8_t* sout;        // TMA-store staging
  uint8_t* smem;        // stage ring base (split-K park)
  const CUtensorMap* tmO0;
  const CUtensorMap* tmO1;
  int splits, num_kb;
  int warp, lane;
  unsigned long long* dbg;
  uint32_t empty_remote;  // CTA pair: shared::cluster address of the leader's tmem_empty_bar (0: local)
};

template <int BN, int EPI, bool PAIR = false>
__device__ __forceinline__ void tc_epilogue_tile(const EpiArgs& ep, const EpiTileCtx& x, int m_tile, int n_tile,
                                                 int acc, int i, int acc_stride = BN) {
  using TO = TmaOut<BN, EPI, PAIR>;
  const int warp = x.warp, lane = x.lane;
  const int q = warp & 3;
  const int h = (warp - 4) >> 2;  // column part 0..TC_EPI_PARTS-1
  const int et = threadIdx.x - 128;  // 0..TC_EPI_THREADS-1
  const int rl = q * 32 + lane;      // row within the tile
  constexpr int NP = BN / 16 < TC_EPI_PARTS ? BN / 16 : TC_EPI_PARTS;  // parts with columns
  constexpr int HALF = BN / NP;                                        // columns per warp
  const bool active = h < NP;
  const int c_lo = active ? h * HALF : 0;
  const int splits = x.splits, num_kb = x.num_kb;
  uint8_t* sout = x.sout;
  uint8_t* smem = x.smem;
  float* red = x.red;
  float* dzs = x.dzs;
  uint64_t* tmem_full_bar = x.tmem_full_bar;
  uint64_t* tmem_empty_bar = x.tmem_empty_bar;
  const uint32_t tmem_base = x.tmem_base;
  unsigned long long* dbg = x.dbg;
  (void)dbg;
  (void)dzs;
  (void)sout;
  (void)smem;
    const int m0 = m_tile * TC_BM, n0 = n_tile * BN;
    const int r = m0 + rl;
    const bool row_ok = r < ep.M;
    const uint32_t tbase = tmem_base + (uint32_t)(acc * acc_stride) + ((uint32_t)(q * 32) << 16);
    float* sb = x.sbias + acc * BN;

    // stage the bias of the tile's columns in shared memory while the mainloop runs
    if (EPI == EPI_FWD_SIG || EPI == EPI_FWD_LOGITS || EPI == EPI_HEAD_XENT) {
      for (int c = et; c < BN; c += TC_EPI_THREADS) sb[c] = n0 + c < ep.N ? ep.bias[n0 + c] : 0.f;
    }
    // DGRAD: prefetch this thread's row of sigma'(Z) (the S stash) for all of its columns
    constexpr int NCH = (HALF + 15) / 16;
    uint4 spre[EPI == EPI_DGRAD_SIG ? NCH : 1][2];
    if (EPI == EPI_DGRAD_SIG && active && row_ok) {
#pragma unroll
      for (int i = 0; i < NCH; ++i) {
        // group i of this warp: whole-tile layout [c_lo + 16 i], or chunked (TMA store) layout
        // chunk i / (CW/16), columns h * CW + 16 (i % (CW/16)) of it
        constexpr int G16 = (64 / TC_EPI_PARTS) / 16 > 0 ? (64 / TC_EPI_PARTS) / 16 : 1;
        const int nc = TO::on ? n0 + 64 * (i / G16) + h * (64 / TC_EPI_PARTS) + 16 * (i % G16) : n0 + c_lo + 16 * i;
        if (nc + 16 <= ep.N) {
          const uint4* S = reinterpret_cast<const uint4*>(static_cast<const __nv_bfloat16*>(ep.aux) +
                                                          (int64_t)r * ep.ldaux + nc);
          spre[i][0] = __ldg(S);
          spre[i][1] = __ldg(S + 1);
        }
      }
    }
    if (TO::on && et == 0) tma_store_wait_read();  // staging buffer of the previous tile free
    epi_bar_sync();  // sbias visible; previous tile's partial sums consumed; staging free
    HB_STAMP(dbg && et == 0 && i == 0, dbg[4]);
    mbar_wait(&tmem_full_bar[acc], (i >> 1) & 1);
    tc_fence_after();
    HB_STAMP(dbg && et == 0 && i == 0, dbg[5]);

    if (EPI == EPI_HEAD_XENT) {
      // ---- softmax cross-entropy on the thread's own row of logits (N = C <= BN = 16) ----
      float dz[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) dz[j] = 0.f;
      if (h == 0) {
        uint32_t raw[16];
        tmem_ld_32x32b_x16(tbase, raw);
        tmem_ld_wait();
        const int C = ep.N;
        float z[16];
        float mx = -INFINITY;
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          z[j] = j < C ? __uint_as_float(raw[j]) + sb[j] : -INFINITY;
          mx = fmaxf(mx, z[j]);
        }
        float se = 0.f;
#pragma unroll
        for (int j = 0; j < 16; ++j) se += j < C ? expf(z[j] - mx) : 0.f;
        const float lse = mx + logf(se);
        const int yo = ep.yoff ? __ldg(ep.yoff) : 0;
        const int yi = row_ok ? __ldg(ep.y + yo + r) : -1;
#pragma unroll
        for (int j = 0; j < 16; ++j)
          dz[j] = (row_ok && j < C) ? (expf(z[j] - lse) - (j == yi ? 1.f : 0.f)) * ep.inv_b : 0.f;
        if (row_ok) {
          float zy = 0.f;
#pragma unroll
          for (int j = 0; j < 16; ++j) zy = j == yi ? z[j] : zy;
          ep.row_loss[r] = lse - zy;
          if (ep.out0) {
            uint4* D = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0);
            uint32_t hp[8], lp[8];
            pack_hilo16(dz, hp, lp);
            D[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
            if (ep.ld0 >= 16) D[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
            if (ep.hilo) {  // lo plane at columns [16, 32) (R24)
              D[2] = make_uint4(lp[0], lp[1], lp[2], lp[3]);
              D[3] = make_uint4(lp[4], lp[5], lp[6], lp[7]);
            }
          }
        }
        if (ep.bpart_out) {
          const float t = warp_colsum16(dz, lane);
          if (!(lane & 1)) red[q * BN + colsum16_col(lane)] = t;
        }
      }
      if (ep.bpart_out) {
        epi_bar_sync();
        if (et < ep.N)
          ep.bpart_out[(int64_t)m_tile * ep.ldp + et] = (red[et] + red[BN + et]) + (red[2 * BN + et] + red[3 * BN + et]);
      }
      if (ep.dz_prev) {
        // ---- fused dX of the output layer: dZ_{L-1} = (dZ_L W_L) * sigma'(Z_{L-1}) [Eq. (2), L49],
        //      column-parallel over the tile's rows (coalesced S loads / dZ stores); each thread
        //      owns whole columns, so its running sums are the bias partials of dZ_{L-1} ----
        if (h == 0) {
          float4* d4 = reinterpret_cast<float4*>(dzs + rl * 16);
#pragma unroll
          for (int qq = 0; qq < 4; ++qq) d4[qq] = make_float4(dz[4 * qq], dz[4 * qq + 1], dz[4 * qq + 2], dz[4 * qq + 3]);
        }
        epi_bar_sync();
        const int C = ep.N;
        const int rows = min(TC_BM, ep.M - m0);
        for (int pc = et; 2 * pc < ep.n_prev; pc += TC_EPI_THREADS) {
          const int n = 2 * pc;
          const bool two = n + 1 < ep.n_prev;
          float w0[16], w1[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            w0[j] = j < C ? __ldg(ep.w_head + (int64_t)j * ep.ldw_head + n) : 0.f;
            w1[j] = (j < C && two) ? __ldg(ep.w_head + (int64_t)j * ep.ldw_head + n + 1) : 0.f;
          }
          float cs0 = 0.f, cs1 = 0.f;
#pragma unroll 4
          for (int rr = 0; rr < rows; ++rr) {
            const float4* d4 = reinterpret_cast<const float4*>(dzs + rr * 16);
            float a0 = 0.f, a1 = 0.f;
#pragma unroll
            for (int qq = 0; qq < 4; ++qq) {
              const float4 d = d4[qq];
              a0 = fmaf(d.x, w0[4 * qq], fmaf(d.y, w0[4 * qq + 1], fmaf(d.z, w0[4 * qq + 2], fmaf(d.w, w0[4 * qq + 3], a0))));
              a1 = fmaf(d.x, w1[4 * qq], fmaf(d.y, w1[4 * qq + 1], fmaf(d.z, w1[4 * qq + 2], fmaf(d.w, w1[4 * qq + 3], a1))));
            }
            const int64_t gr = (int64_t)(m0 + rr);
            const float2 sf = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(ep.s_prev + gr * ep.ld_prev + n));
            const float o0 = a0 * sf.x, o1 = two ? a1 * sf.y : 0.f;
            *reinterpret_cast<__nv_bfloat162*>(ep.dz_prev + gr * ep.ld_prev + n) = __floats2bfloat162_rn(o0, o1);
            cs0 += o0;
            cs1 += o1;
          }
          ep.bpart_prev[(int64_t)m_tile * ep.n_prev + n] = cs0;
          if (two) ep.bpart_prev[(int64_t)m_tile * ep.n_prev + n + 1] = cs1;
        }
      }
    } else {
      if ((EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) && splits == 1 && ep.hilo) {
        // split-precision head dW (R24, transposed, one 32-column tile): column c of the result is
        // acc[c] + acc[hilo + c] (hi and lo planes of dZ_L); the warps of part 0 own the tile
        if (h == 0) {
          uint32_t r0[16], r1[16];
          tmem_ld_32x32b_x16(tbase, r0);
          tmem_ld_32x32b_x16(tbase + (uint32_t)ep.hilo, r1);
          tmem_ld_wait();
          if (row_ok) {
#pragma unroll
            for (int j = 0; j < 16; ++j)
              if (j < ep.n_real)
                epi_elem<EPI, __nv_bfloat16, false>(ep, r, j, __uint_as_float(r0[j]) + __uint_as_float(r1[j]));
          }
        }
      } else if (TO::on) {
        // ---- 64-column chunks through two staging buffers, one bulk-store group per chunk ----
        constexpr int CW = 64 / TC_EPI_PARTS;  // columns of a chunk per warp
        static_assert(CW % 16 == 0, "chunk columns per warp");
        int pi = 0;  // index into this warp's prefetched sigma' groups (dgrad)
#pragma unroll
        for (int j = 0; j < TO::NCHUNK; ++j) {
          uint8_t* sbuf = sout + (size_t)(j % TO::NBUF) * TO::NOUT * TC_BM * 128;
          if (j >= TO::NBUF) {  // the bulk stores of chunk j - NBUF have read this buffer
            if (et == 0) {
              if (TO::NBUF == 2)
                tma_store_wait_read_1();
              else
                tma_store_wait_read();
            }
            epi_bar_sync();
          }
          // this warp's columns of the chunk: every TMEM load in flight before the one wait
          uint32_t rawc[CW / 16][16];
#pragma unroll
          for (int g = 0; g < CW / 16; ++g)
            if (n0 + 64 * j + h * CW + 16 * g < ep.N) tmem_ld_32x32b_x16(tbase + (uint32_t)(64 * j + h * CW + 16 * g), rawc[g]);
          tmem_ld_wait();
          HB_STAMP(dbg && et == 0 && i == 1 && j == 0, dbg[31]);  // tuning: first chunk loaded (tile 1)
#pragma unroll
          for (int g = 0; g < CW / 16; ++g, ++pi) {
            const int cc = h * CW + 16 * g;  // column within the chunk
            const int c = 64 * j + cc;       // column within the tile
            const int nc = n0 + c;
            float v[16];
#pragma unroll
            for (int k = 0; k < 16; ++k) v[k] = nc < ep.N ? __uint_as_float(rawc[g][k]) : 0.f;
            if (EPI == EPI_FWD_SIG) {
              // all rows / columns staged; rows >= M and columns >= N are clipped by the TMA store
              uint32_t hp[8], sp[8];
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) {
                float h0, d0, h1, d1;
                sigmoid_d_fast2(v[2 * qq], v[2 * qq + 1], sb[c + 2 * qq], sb[c + 2 * qq + 1], h0, h1, d0, d1);
                hp[qq] = pack_bf16x2(h0, h1);
                sp[qq] = pack_bf16x2(d0, d1);
              }
              stage16_box(sbuf, rl, cc, hp);
              if (ep.out1) {
                if (TO::NOUT == 2) {
                  stage16_box(sbuf + TC_BM * 128, rl, cc, sp);
                } else if (row_ok) {  // sigma' stash written directly (256-wide tiles)
                  __nv_bfloat16* S = static_cast<__nv_bfloat16*>(ep.out1) + (int64_t)r * ep.ld1 + nc;
                  if (nc + 16 <= ep.N) {
                    reinterpret_cast<uint4*>(S)[0] = make_uint4(sp[0], sp[1], sp[2], sp[3]);
                    reinterpret_cast<uint4*>(S)[1] = make_uint4(sp[4], sp[5], sp[6], sp[7]);
                  } else {
#pragma unroll
                    for (int k = 0; k < 16; ++k)
                      if (nc + k < ep.N) S[k] = __ushort_as_bfloat16((unsigned short)(sp[k >> 1] >> (16 * (k & 1))));
                  }
                }
              }
            } else {  // DGRAD: dZ = acc * sigma'(Z) (prefetched S), fp32 values feed the bias partials
              if (row_ok && nc < ep.N) {
                if (nc + 16 <= ep.N) {
                  const uint4 s0 = spre[pi][0], s1 = spre[pi][1];
                  const __nv_bfloat162* sv0 = reinterpret_cast<const __nv_bfloat162*>(&s0);
                  const __nv_bfloat162* sv1 = reinterpret_cast<const __nv_bfloat162*>(&s1);
#pragma unroll
                  for (int qq = 0; qq < 4; ++qq) {
                    const float2 a = __bfloat1622float2(sv0[qq]);
                    v[2 * qq] *= a.x;
                    v[2 * qq + 1] *= a.y;
                    const float2 b2 = __bfloat1622float2(sv1[qq]);
                    v[8 + 2 * qq] *= b2.x;
                    v[8 + 2 * qq + 1] *= b2.y;
                  }
                } else {
                  const __nv_bfloat16* S = static_cast<const __nv_bfloat16*>(ep.aux) + (int64_t)r * ep.ldaux;
#pragma unroll
                  for (int k = 0; k < 16; ++k) v[k] = nc + k < ep.N ? v[k] * __bfloat162float(S[nc + k]) : 0.f;
                }
              } else {
#pragma unroll
                for (int k = 0; k < 16; ++k) v[k] = 0.f;
              }
              uint32_t pk[8];
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) pk[qq] = pack_bf16x2(v[2 * qq], v[2 * qq + 1]);
              stage16_box(sbuf, rl, cc, pk);
              if (ep.bpart_out) {
                const float t = warp_colsum16(v, lane);
                if (!(lane & 1)) red[q * BN + c + colsum16_col(lane)] = t;
              }
            }
          }
          HB_STAMP(dbg && et == 0 && i == 1 && j < 4, dbg[27 + j]);  // tuning: chunk j computed (tile 1)
          fence_proxy_async();
          epi_bar_sync();  // the chunk is staged
          if (et == 0) {
            if (n0 + 64 * j < ep.N) {
              tma_store_2d(x.tmO0, sbuf, n0 + 64 * j, m0);
              if (TO::NOUT == 2 && ep.out1) tma_store_2d(x.tmO1, sbuf + TC_BM * 128, n0 + 64 * j, m0);
            }
            tma_store_commit();  // one group per chunk (empty groups keep the count)
          }
        }
      } else if (active) {
#pragma unroll
        for (int cc = 0; cc < HALF; cc += 16) {
          const int c = c_lo + cc;
          if (n0 + c >= ep.N) break;  // warp-uniform
          uint32_t raw[16];
          tmem_ld_32x32b_x16(tbase + (uint32_t)c, raw);
          tmem_ld_wait();
          float v[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = __uint_as_float(raw[j]);
          const int nc = n0 + c;
          const bool full = nc + 16 <= ep.N;
          if (EPI == EPI_DGRAD_SIG) {
            // dZ = acc * sigma'(Z) (prefetched S), stored bf16; fp32 values feed the bias partials
            if (row_ok) {
              if (full) {
                const uint4 s0 = spre[0][0], s1 = spre[0][1];
                const __nv_bfloat162* sv0 = reinterpret_cast<const __nv_bfloat162*>(&s0);
                const __nv_bfloat162* sv1 = reinterpret_cast<const __nv_bfloat162*>(&s1);
#pragma unroll
                for (int qq = 0; qq < 4; ++qq) {
                  float2 a = __bfloat1622float2(sv0[qq]);
                  v[2 * qq] *= a.x;
                  v[2 * qq + 1] *= a.y;
                  float2 b2 = __bfloat1622float2(sv1[qq]);
                  v[8 + 2 * qq] *= b2.x;
                  v[8 + 2 * qq + 1] *= b2.y;
                }
                uint32_t pk[8];
#pragma unroll
                for (int qq = 0; qq < 8; ++qq) pk[qq] = pack_bf16x2(v[2 * qq], v[2 * qq + 1]);
                uint4* D = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0 + nc);
                D[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                D[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
              } else {
                const __nv_bfloat16* S = static_cast<const __nv_bfloat16*>(ep.aux) + (int64_t)r * ep.ldaux;
                __nv_bfloat16* D = static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0;
#pragma unroll
                for (int j = 0; j < 16; ++j) {
                  if (nc + j < ep.N) {
                    v[j] *= __bfloat162float(S[nc + j]);
                    D[nc + j] = __float2bfloat16_rn(v[j]);
                  } else {
                    v[j] = 0.f;
                  }
                }
              }
            } else {
#pragma unroll
              for (int j = 0; j < 16; ++j) v[j] = 0.f;
            }
            if (ep.bpart_out) {
              const float t = warp_colsum16(v, lane);
              if (!(lane & 1)) red[q * BN + c + colsum16_col(lane)] = t;
            }
            // advance the prefetched-S ring (static register indexing)
#pragma unroll
            for (int i = 0; i + 1 < NCH; ++i) {
              spre[i][0] = spre[i + 1][0];
              spre[i][1] = spre[i + 1][1];
            }
          } else if ((EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) && splits > 1) {
            // split-K: park the fp32 partial tile in this CTA's (now idle) stage ring, row stride
            // BN + 4 floats (conflict-free row-per-lane writes); the cluster reduces it over DSMEM
            if (num_kb == 0) {
#pragma unroll
              for (int j = 0; j < 16; ++j) v[j] = 0.f;
            }
            const uint32_t pa = smem_u32(smem) + (uint32_t)((rl * (BN + 4) + c) * 4);
#pragma unroll
            for (int qq = 0; qq < 4; ++qq)
              sts128(pa + qq * 16, __float_as_uint(v[4 * qq]), __float_as_uint(v[4 * qq + 1]),
                     __float_as_uint(v[4 * qq + 2]), __float_as_uint(v[4 * qq + 3]));
          } else if (row_ok) {
            if (EPI == EPI_FWD_SIG && full) {
              uint32_t hp[8], sp[8];
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) {
                float h0, d0, h1, d1;
                sigmoid_d_fast2(v[2 * qq], v[2 * qq + 1], sb[c + 2 * qq], sb[c + 2 * qq + 1], h0, h1, d0, d1);
                hp[qq] = pack_bf16x2(h0, h1);
                sp[qq] = pack_bf16x2(d0, d1);
              }
              uint4* H = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out0) + (int64_t)r * ep.ld0 + nc);
              H[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
              H[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
              if (ep.out1) {
                uint4* S = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(ep.out1) + (int64_t)r * ep.ld1 + nc);
                S[0] = make_uint4(sp[0], sp[1], sp[2], sp[3]);
                S[1] = make_uint4(sp[4], sp[5], sp[6], sp[7]);
              }
            } else if (EPI == EPI_FWD_SIG || EPI == EPI_FWD_LOGITS) {
#pragma unroll
              for (int j = 0; j < 16; ++j)
                if (nc + j < ep.N) {
                  const float z = v[j] + sb[c + j];
                  if (EPI == EPI_FWD_LOGITS) {
                    static_cast<float*>(ep.out0)[(int64_t)r * ep.ld0 + nc + j] = z;
                  } else {
                    float hv, dv;
                    sigmoid_d_fast(z, hv, dv);
                    static_cast<__nv_bfloat16*>(ep.out0)[(int64_t)r * ep.ld0 + nc + j] = __float2bfloat16_rn(hv);
                    if (ep.out1)
                      static_cast<__nv_bfloat16*>(ep.out1)[(int64_t)r * ep.ld1 + nc + j] = __float2bfloat16_rn(dv);
                  }
                }
            } else {
              const bool vec_ok = full && !ep.transposed && (EPI != EPI_WGRAD_SGD || ep.shadow != nullptr) &&
                                  EPI != EPI_WGRAD_STORE;
              if (vec_ok) {
                epi_row16_bf16<EPI>(ep, r, nc, v);
              } else {
#pragma unroll
                for (int j = 0; j < 16; ++j)
                  if (nc + j < ep.N) epi_elem<EPI, __nv_bfloat16, false>(ep, r, nc + j, v[j]);
              }
            }
          }
        }
      }
      if (EPI == EPI_DGRAD_SIG && ep.bpart_out) {
        if (!TO::on) epi_bar_sync();
        for (int cc = et; cc < BN && n0 + cc < ep.N; cc += TC_EPI_THREADS)
          ep.bpart_out[(int64_t)m_tile * ep.ldp + n0 + cc] =
              (red[cc] + red[BN + cc]) + (red[2 * BN + cc] + red[3 * BN + cc]);
      }
      if ((EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) && ep.bpart_in && splits == 1) {
        // db = sum of the dZ producer's per-tile partials, fixed order; bias index = W row.
        // non-transposed: the n-tile-0 CTA owns bias rows m0..m0+127;
        // transposed (small head): the m-tile-0 CTA owns bias entries n0..n0+BN-1
        const bool own = !ep.transposed ? (n_tile == 0) : (m_tile == 0);
        const int lo = !ep.transposed ? m0 : n0;
        const int hi = !ep.transposed ? min(ep.M, m0 + TC_BM) : min(ep.hilo ? ep.n_real : ep.N, n0 + BN);
        if (own) bias_reduce_update<EPI>(ep, lo, hi, et);
      }
    }
    // release this accumulator to the MMA warp (all TMEM reads of the tile have completed)
    tc_fence_before();
    __syncwarp();
    if (lane == 0) {
      if (x.empty_remote)  // CTA pair: the leader's MMAs write both CTAs' accumulators
        mbar_arrive_cluster(x.empty_remote + (uint32_t)(acc * 8));
      else
        mbar_arrive(&tmem_empty_bar[acc]);
    }
}

template <int BN, bool A_MN, bool B_MN, int EPI, bool PAIR = false>
__global__ void __launch_bounds__(TC_THREADS, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmO0, const __grid_constant__ CUtensorMap tmO1,
                   int K, const int* __restrict__ offA, const int* __restrict__ offB, EpiArgs ep) {
  using Cfg = TcCfg<BN, B_MN, EPI, PAIR>;
  using TO = TmaOut<BN, EPI, PAIR>;
  constexpr int STAGES = Cfg::STAGES;
  static_assert(!PAIR || (A_MN && B_MN && BN >= 128 && !TO::on) || (!A_MN && BN == 256),
                "CTA pairs: split-K dW GEMMs or persistent 256 x 256 forward / dX tiles");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sout = smem + STAGES * Cfg::STAGE_BYTES;  // TMA-store staging [NOUT][NBOX][128 rows x 128 B]
  uint64_t* full_bar = reinterpret_cast<uint64_t*>(sout + Cfg::OUT_BYTES);
  uint64_t* empty_bar = full_bar + STAGES;
  uint64_t* tmem_full_bar = empty_bar + STAGES;   // [2]: accumulator a ready (MMA -> epilogue)
  uint64_t* tmem_empty_bar = tmem_full_bar + 2;    // [2]: accumulator a drained (epilogue -> MMA)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_empty_bar + 2);
  __shared__ float red[EPI == EPI_DGRAD_SIG || EPI == EPI_HEAD_XENT ? 4 * BN : 4];  // bias-gradient partials
  __shared__ float sbias[2][BN];   // bias of the tile, double-buffered across tiles
  __shared__ __align__(16) float dzs[EPI == EPI_HEAD_XENT ? TC_BM * 16 : 4];  // dZ_L rows (fused head dX)

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  unsigned long long* dbg = ep.dbg ? ep.dbg + 32 * ((size_t)(blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x) : nullptr;
  HB_STAMP(dbg && threadIdx.x == 0, dbg[0]);
  // Tiles: persistent CTAs walk tiles t = blockIdx.x, +gridDim.x, ... (n fastest, so CTAs running
  // together share the A row panel in L2).  Split-K launches (gridDim.z > 1) are one tile per CTA.
  const int tiles_n = (ep.N + BN - 1) / BN;
  const int tiles_m = (ep.M + TC_BM - 1) / TC_BM;
  // split-K (dW GEMMs with K = batch): the gridDim.z CTAs of one output tile form a cluster,
  // each accumulates k-blocks [kb_lo, kb_hi) in its own TMEM
  const int splits = gridDim.z;
  // persistent CTA pairs walk 256-row pair tiles; pair p is the cluster (2p, 2p+1) along x
  const bool pair_persist = PAIR && splits == 1;
  const int tiles_mp = pair_persist ? (tiles_m + 1) / 2 : tiles_m;
  const int num_tiles = tiles_n * tiles_mp;
  const int t_first = splits == 1 ? (int)(PAIR ? blockIdx.x >> 1 : blockIdx.x) : (int)(blockIdx.y * gridDim.x + blockIdx.x);
  const int t_step = splits == 1 ? (int)(PAIR ? gridDim.x >> 1 : gridDim.x) : num_tiles;
  const int kz = blockIdx.z;
  // CTA pair (grid x = M tiles, y = N tiles, z = splits; cluster (2, 1, S) — pairs must be along
  // the cluster's x): half = blockIdx.x & 1; cluster rank of split sp's CTA with the same half =
  // half + 2 sp; the pair's leader (half 0) has rank 2 kz
  const uint32_t half = PAIR ? (blockIdx.x & 1) : 0;
  const uint16_t pair_mask = (uint16_t)(3u << (2 * kz));
  const int num_kb_all = (K + TC_BK - 1) / TC_BK;
  const int kpb = (num_kb_all + splits - 1) / splits;
  const int kb_lo = min(num_kb_all, kz * kpb);
  const int num_kb = min(num_kb_all, kb_lo + kpb) - kb_lo;
  // output tile (m_tile, n_tile) of the CTA's tile index t
  auto tile_of = [&](int t, int& m_tile, int& n_tile) {
    if (PAIR && splits > 1) {  // split-K pair: one tile per CTA, from the grid
      m_tile = blockIdx.x;
      n_tile = blockIdx.y;
    } else if (PAIR) {
      int mp;
      tile_coords<TC_GROUP_M_PAIR>(t, tiles_mp, tiles_n, mp, n_tile);
      m_tile = 2 * mp + (int)half;
    } else {
      tile_coords<TC_GROUP_M>(t, tiles_m, tiles_n, m_tile, n_tile);
    }
  };

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tmem_full_bar[a], 1);
      mbar_init(&tmem_empty_bar[a], (PAIR ? 2 : 1) * TC_EPI_WARPS);  // one arrive per epilogue warp (of the pair)
    }
    fence_barrier_init();
  }
  if (warp == 2) {
    if (PAIR)
      tmem_alloc_pair<Cfg::TMEM_COLS>(tmem_slot);
    else
      tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  }
  tc_fence_before();
  __syncthreads();
  if (PAIR) cluster_sync_all();  // the leader's barriers are initialised before the peer's loads signal them
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  // programmatic dependent launch: everything above overlapped the previous kernel's tail;
  // no global memory produced by it is touched before this point
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  HB_STAMP(dbg && threadIdx.x == 0, dbg[1]);

  if (warp == 0 && lane == 0) {
    // ===== TMA producer =====
    const int oa = offA ? __ldg(offA) : 0;
    const int ob = offB ? __ldg(offB) : 0;
    int it = 0;  // k-blocks issued by this CTA (ring position across tiles)
    for (int t = t_first; t < num_tiles; t += t_step) {
    int mt_, nt_;
    tile_of(t, mt_, nt_);  // PAIR: this CTA's own M tile, the pair's N tile (its half of it)
    const int m0 = mt_ * TC_BM, n0 = nt_ * BN + (int)half * Cfg::B_TILE;
    const uint32_t lead_full = PAIR ? mapa_shared(smem_u32(full_bar), 2 * kz) : 0;
    for (int kb = 0; kb < num_kb; ++kb, ++it) {
      const int s = it % STAGES;
      const uint32_t ph = (it / STAGES) & 1;
      mbar_wait(&empty_bar[s], ph ^ 1);
      uint8_t* sA = smem + s * Cfg::STAGE_BYTES;
      uint8_t* sB = sA + Cfg::A_BYTES;
      const int k0 = (kb_lo + kb) * TC_BK;
      if (PAIR) {  // both CTAs' loads complete on the leader's barrier, which expects both
        const uint32_t fb = lead_full + (uint32_t)(s * 8);
        if (half == 0) mbar_arrive_expect_tx(&full_bar[s], 2 * Cfg::STAGE_BYTES);
        if (!A_MN) {
          tma_load_2d_pair(sA, &tmA, fb, k0, m0 + oa);
        } else {
          tma_load_2d_pair(sA, &tmA, fb, m0, k0 + oa);
          tma_load_2d_pair(sA + 8192, &tmA, fb, m0 + 64, k0 + oa);
        }
        if (!B_MN) {
          tma_load_2d_pair(sB, &tmB, fb, k0, n0 + ob);
        } else {
#pragma unroll
          for (int j = 0; j < Cfg::B_ROWS / 64; ++j) tma_load_2d_pair(sB + j * 8192, &tmB, fb, n0 + 64 * j, k0 + ob);
        }
        continue;
      }
      mbar_arrive_expect_tx(&full_bar[s], Cfg::STAGE_BYTES);
      if (!A_MN) {
        tma_load_2d(sA, &tmA, &full_bar[s], k0, m0 + oa);
      } else {
        tma_load_2d(sA, &tmA, &full_bar[s], m0, k0 + oa);
        tma_load_2d(sA + 8192, &tmA, &full_bar[s], m0 + 64, k0 + oa);
      }
      if (!B_MN) {
        tma_load_2d(sB, &tmB, &full_bar[s], k0, n0 + ob);
      } else {
#pragma unroll
        for (int j = 0; j < Cfg::B_ROWS / 64; ++j)
          tma_load_2d(sB + j * 8192, &tmB, &full_bar[s], n0 + 64 * j, k0 + ob);
      }
    }
    }
  } else if (warp == 1 && lane == 0 && half == 0) {
    // ===== MMA issuer (single thread; in a pair the leader issues for both CTAs) =====
    constexpr uint32_t idesc = make_idesc_bf16(PAIR ? 2 * TC_BM : TC_BM, BN, A_MN, B_MN);
    int it = 0, i = 0;
    for (int t = t_first; t < num_tiles; t += t_step, ++i) {
    const int acc = i & 1;
    if (PAIR)  // both CTAs' epilogues have drained this accumulator (remote arrivals)
      mbar_wait_cluster(&tmem_empty_bar[acc], ((i >> 1) & 1) ^ 1);
    else
      mbar_wait(&tmem_empty_bar[acc], ((i >> 1) & 1) ^ 1);  // epilogue has drained this accumulator
    tc_fence_after();
    const uint32_t tacc = tmem_base + (uint32_t)(acc * BN);
    for (int kb = 0; kb < num_kb; ++kb, ++it) {
      const int s = it % STAGES;
      const uint32_t ph = (it / STAGES) & 1;
      mbar_wait(&full_bar[s], ph);
      tc_fence_after();
      HB_STAMP(dbg && it == 0, dbg[2]);
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
        if (PAIR)
          umma_bf16_pair(tacc, ad, bd, idesc, (kb | kk) != 0);
        else
          umma_bf16(tacc, ad, bd, idesc, (kb | kk) != 0);
      }
      if (PAIR)
        umma_commit_pair(&empty_bar[s], pair_mask);  // both CTAs' slots
      else
        umma_commit(&empty_bar[s]);  // frees the smem slot when these MMAs complete
    }
    if (PAIR)
      umma_commit_pair(&tmem_full_bar[acc], pair_mask);
    else
      umma_commit(&tmem_full_bar[acc]);  // accumulator ready (arrives even if num_kb == 0)
    HB_STAMP(dbg && i == 0, dbg[3]);
    HB_STAMP(dbg && i < 5, dbg[12 + i]);  // tuning: MMAs of tile i issued
    }
  } else if (warp >= 4) {
    // ===== epilogue (8 warps): TMEM -> registers -> fused epilogue -> global =====
    // warp w reads TMEM lanes 32*(w%4).. (tile rows) and handles column half h = (w-4)/4
    const EpiTileCtx ectx{tmem_base, tmem_full_bar, tmem_empty_bar, &sbias[0][0], red, dzs, sout, smem, &tmO0,
                          &tmO1, splits, num_kb, warp, lane, dbg,
                          PAIR ? mapa_shared(smem_u32(tmem_empty_bar), 2 * kz) : 0u};
    int i = 0;
    for (int t = t_first; t < num_tiles; t += t_step, ++i) {
      int m_tile, n_tile;
      tile_of(t, m_tile, n_tile);
      HB_STAMP(dbg && threadIdx.x == 128 && i < 5, dbg[17 + i]);  // tuning: epilogue of tile i starts
      tc_epilogue_tile<BN, EPI, PAIR>(ep, ectx, m_tile, n_tile, i & 1, i);
      HB_STAMP(dbg && threadIdx.x == 128 && i < 5, dbg[22 + i]);  // tuning: epilogue of tile i done
    }
  }

  if ((EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) && splits > 1) {
    // ---- split-K reduce-scatter: CTA kz of the cluster reduces rows [kz*rps, (kz+1)*rps) of the
    //      tile over the `splits` partials (read from every CTA's shared memory, fixed order) and
    //      applies the fused SGD update ----
    static_assert(!(EPI == EPI_WGRAD_SGD || EPI == EPI_WGRAD_STORE) || TC_BM * (BN + 4) * 4 <= Cfg::STAGES * Cfg::STAGE_BYTES,
                  "split-K tile must fit the ring");
    // the fp32 master rows of this CTA's slice do not depend on the partials: fetch them (up to 8
    // float4 per thread) before the cluster barrier so their latency hides behind it
    constexpr int RED_MAXIT = 8;
    float4 wpre[RED_MAXIT];
    {
      const int t = t_first;
      int m_tile, n_tile;
      tile_of(t, m_tile, n_tile);
      const int tid = threadIdx.x - 128;
      const int rps = TC_BM / splits;
#pragma unroll
      for (int u = 0; u < RED_MAXIT; ++u) {
        wpre[u] = make_float4(0.f, 0.f, 0.f, 0.f);
        const int e = (tid + u * TC_EPI_THREADS) * 4;
        if (EPI == EPI_WGRAD_SGD && warp >= 4 && !ep.transposed && !ep.atomic && e < rps * BN) {
          const int gm = m_tile * TC_BM + kz * rps + e / BN, gn = n_tile * BN + e % BN;
          if (gm < ep.M && gn + 4 <= ep.N) wpre[u] = __ldcg(reinterpret_cast<const float4*>(ep.master + (int64_t)gm * ep.ldw + gn));
        }
      }
    }
    HB_STAMP(dbg && threadIdx.x == 128, dbg[8]);
    cluster_sync_all();  // every partial tile is in shared memory (release/acquire, cluster scope)
    HB_STAMP(dbg && threadIdx.x == 128, dbg[9]);
    if (warp >= 4) {
      const int t = t_first;
      int m_tile, n_tile;
      tile_of(t, m_tile, n_tile);
      const int m0 = m_tile * TC_BM, n0 = n_tile * BN;
      const int tid = threadIdx.x - 128;  // 0..255
      const int rps = TC_BM / splits;
      const uint32_t tile_s = smem_u32(smem);
      // every load of an element group is issued before the first add (the adds keep the fixed
      // split order, so the result is bitwise the same as a sequential sum): one DSMEM round trip
      // per group instead of `splits` dependent ones; the master row is fetched up front too
#pragma unroll 1
      for (int e = tid * 4, u = 0; e < rps * BN; e += TC_EPI_THREADS * 4, ++u) {
        const int rloc = kz * rps + e / BN, col = e % BN;
        const uint32_t off = (uint32_t)((rloc * (BN + 4) + col) * 4);
        const int gm = m0 + rloc, gn = n0 + col;
        if (ep.hilo && col >= ep.hilo) continue;  // R24: lo-plane columns are folded into [0, hilo)
        const bool in = gm < ep.M && gn < (ep.hilo ? ep.n_real : ep.N);
        const bool vec = in && !ep.transposed && gn + 4 <= ep.N && EPI == EPI_WGRAD_SGD;
        float4* W = vec ? reinterpret_cast<float4*>(ep.master + (int64_t)gm * ep.ldw + gn) : nullptr;
        float4 w = make_float4(0.f, 0.f, 0.f, 0.f);
        if (vec && !ep.atomic) {
          if (u < RED_MAXIT) {  // prefetched (static register index via the unrolled select)
#pragma unroll
            for (int k = 0; k < RED_MAXIT; ++k)
              if (k == u) w = wpre[k];
          } else {
            w = *W;
          }
        }
        float4 part[8];
#pragma unroll
        for (int sp = 0; sp < 8; ++sp)
          if (sp < splits) part[sp] = ld_dsmem_f4(mapa_shared(tile_s + off, PAIR ? half + 2u * sp : (uint32_t)sp));
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int sp = 0; sp < 8; ++sp)
          if (sp < splits) {
            acc.x += part[sp].x;
            acc.y += part[sp].y;
            acc.z += part[sp].z;
            acc.w += part[sp].w;
          }
        if (ep.hilo) {  // + the lo plane's column (same splits, same fixed order)
#pragma unroll
          for (int sp = 0; sp < 8; ++sp)
            if (sp < splits)
              part[sp] = ld_dsmem_f4(mapa_shared(tile_s + off + (uint32_t)(ep.hilo * 4), (uint32_t)sp));
          float4 lo4 = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
          for (int sp = 0; sp < 8; ++sp)
            if (sp < splits) {
              lo4.x += part[sp].x;
              lo4.y += part[sp].y;
              lo4.z += part[sp].z;
              lo4.w += part[sp].w;
            }
          acc.x += lo4.x;
          acc.y += lo4.y;
          acc.z += lo4.z;
          acc.w += lo4.w;
        }
        if (!in) continue;
        const float a4[4] = {acc.x, acc.y, acc.z, acc.w};
        if (vec) {
          const float4 d = sgd_delta4(ep.lr, acc.x, acc.y, acc.z, acc.w);
          if (ep.atomic) {
            w = sgd_atomic4(W, d);
          } else {
            w.x += d.x;
            w.y += d.y;
            w.z += d.z;
            w.w += d.w;
            *W = w;
          }
          uint2 sh = make_uint2(pack_bf16x2(w.x, w.y), pack_bf16x2(w.z, w.w));
          *reinterpret_cast<uint2*>(ep.shadow + (int64_t)gm * ep.ldw + gn) = sh;
          if (ep.npeer) {
            float* wl = ep.master + (int64_t)gm * ep.ldw + gn;
            __nv_bfloat16* sl = ep.shadow + (int64_t)gm * ep.ldw + gn;
            peer_push1(ep, wl, sl, acc.x);
            peer_push1(ep, wl + 1, sl + 1, acc.y);
            peer_push1(ep, wl + 2, sl + 2, acc.z);
            peer_push1(ep, wl + 3, sl + 3, acc.w);
          }
        } else {
#pragma unroll
          for (int j = 0; j < 4; ++j)
            if (gn + j < (ep.hilo ? ep.n_real : ep.N)) epi_elem<EPI, __nv_bfloat16, false>(ep, gm, gn + j, a4[j]);
        }
      }
      HB_STAMP(dbg && threadIdx.x == 128, dbg[10]);
      if (ep.bpart_in) {  // bias: rows of this CTA's slice (or, transposed, the tile's columns)
        int lo, hi;
        bool own;
        if (!ep.transposed) {
          own = n_tile == 0;
          lo = m0 + kz * rps;
          hi = min(ep.M, m0 + (kz + 1) * rps);
        } else {
          own = m_tile == 0 && kz == 0;
          lo = n0;
          hi = min(ep.hilo ? ep.n_real : ep.N, n0 + BN);
        }
        if (own) bias_reduce_update<EPI>(ep, lo, hi, tid);
      }
    }
    HB_STAMP(dbg && threadIdx.x == 128, dbg[11]);
    cluster_sync_all();  // no CTA leaves while another still reads its partial tile
  }

  if (TO::on && threadIdx.x == 128) tma_store_wait_all();  // bulk stores complete before exit
  // persistent pair: neither CTA leaves while the other may still arrive on its barriers
  if (PAIR && splits == 1) cluster_sync_all();
  HB_STAMP(dbg && threadIdx.x == 128, dbg[6]);
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    if (PAIR)
      tmem_dealloc_pair<Cfg::TMEM_COLS>(tmem_base);
    else
      tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
  }
  HB_STAMP(dbg && threadIdx.x == 64, dbg[7]);
}

}  // namespace hb
