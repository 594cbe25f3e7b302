// common.cuh — error plumbing and sm_100a PTX wrappers (mbarrier, TMA, tcgen05).
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "../../include/hogbatch.h"

namespace hb {

// thread-local last error message (hb_last_error)
void set_error(const std::string& msg);
int fail(int code, const std::string& msg);

#define HB_CUDA_TRY(expr)                                                                   \
  do {                                                                                      \
    cudaError_t _e = (expr);                                                                \
    if (_e != cudaSuccess)                                                                  \
      return ::hb::fail(HB_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(_e) +     \
                                       " (" + __FILE__ + ":" + std::to_string(__LINE__) + ")"); \
  } while (0)

#define HB_CHECK_ARG(cond, msg)                                   \
  do {                                                            \
    if (!(cond)) return ::hb::fail(HB_EINVAL, std::string(msg)); \
  } while (0)

static inline int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// ---------------------------------------------------------------------------------------
// device-side PTX wrappers
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// shared-memory vector store / load by 32-bit shared address (no "memory" clobber: ordering
// against barriers / fences comes from those volatile asm statements)
#ifndef HB_SMEM_CLOBBER
#define HB_SMEM_CLOBBER
#endif
__device__ __forceinline__ void sts128(uint32_t saddr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(saddr), "r"(a), "r"(b), "r"(c), "r"(d) HB_SMEM_CLOBBER);
}
__device__ __forceinline__ float4 lds128f(uint32_t saddr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(saddr) HB_SMEM_CLOBBER);
  return v;
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "HB_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra HB_WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* m) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(m)) : "memory");
}

// 2-D TMA tile load global -> shared, completion counted on an mbarrier (bytes)
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* m, uint64_t* bar,
                                            int32_t c0, int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}

// 2-D TMA tile store shared -> global (bulk group); out-of-bounds rows/columns are clipped
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* m, const void* src, int32_t c0, int32_t c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(smem_u32(src)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_store_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// the smem sources of all committed bulk stores have been read (buffer reusable)
__device__ __forceinline__ void tma_store_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
// the smem sources of all but the most recent committed bulk-store group have been read
__device__ __forceinline__ void tma_store_wait_read_1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
// all committed bulk stores are complete
__device__ __forceinline__ void tma_store_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// --- tcgen05 (5th-generation tensor cores, TMEM accumulators) ---
template <uint32_t kCols>
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(dst_smem)),
               "n"(kCols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}

// CTA pair (cta_group::2): executed by one warp in EACH CTA of the pair
template <uint32_t kCols>
__device__ __forceinline__ void tmem_alloc_pair(uint32_t* dst_smem) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
               "n"(kCols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
template <uint32_t kCols>
__device__ __forceinline__ void tmem_dealloc_pair(uint32_t taddr) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols) : "memory");
}
// 2-D TMA load into this CTA's shared memory whose completion (complete_tx) is counted on the
// mbarrier of the pair's leader CTA (bar_cluster: a shared::cluster address, e.g. from mapa)
__device__ __forceinline__ void tma_load_2d_pair(void* dst, const CUtensorMap* m, uint32_t bar_cluster, int32_t c0,
                                                 int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(bar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
// issued by the leader only: D[256 rows over both CTAs' TMEM] += A (128 rows per CTA) B (N/2 rows per CTA)
__device__ __forceinline__ void umma_bf16_pair(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                               uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// arrive on `bar` (same offset) in every CTA of cta_mask when the leader's MMAs complete
__device__ __forceinline__ void umma_commit_pair(uint64_t* bar, uint16_t cta_mask) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(cta_mask)
      : "memory");
}

template <uint32_t kCols>
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols)
               : "memory");
}

__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// D[tmem] (+)= A[smem] * B[smem]^T, kind::f16 (bf16 inputs, fp32 accumulate), issued by one thread
__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// arrive on an mbarrier when all previously issued tcgen05.mma of this thread complete
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          smem_u32(bar))
      : "memory");
}

// 32 lanes x 32 bits, 32 consecutive columns
__device__ __forceinline__ void tmem_ld_32x32b_x32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}

// 32 lanes x 32 bits, 16 consecutive columns: thread t of the warp gets row (lane_base+t)
__device__ __forceinline__ void tmem_ld_32x32b_x16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}

__device__ __forceinline__ void tmem_ld_wait() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// Shared-memory matrix descriptor for tcgen05 (SWIZZLE_128B canonical layouts).
//   start address >> 4 in bits [0,14), LBO >> 4 in [16,30), SBO >> 4 in [32,46),
//   descriptor version 1 (Blackwell) in [46,48), base offset 0, layout type 2 (128B swizzle)
//   in [61,64).
__device__ __forceinline__ uint64_t make_sw128_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

// Instruction descriptor, kind::f16: D fp32, A/B bf16, A/B major (0 = K, 1 = MN), N>>3, M>>4
__host__ __device__ constexpr uint32_t make_idesc_bf16(int M, int N, bool a_mn, bool b_mn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) |
         ((b_mn ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// all threads of all CTAs of the cluster (release/acquire: global writes before are visible after)
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// --- thread-block-cluster (distributed shared memory) helpers ---
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// shared::cta address -> the shared::cluster address of the same offset in CTA `rank`
__device__ __forceinline__ uint32_t mapa_shared(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
// 16-byte load from the shared memory of a CTA of the cluster (address from mapa_shared)
__device__ __forceinline__ float4 ld_dsmem_f4(uint32_t cluster_addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(cluster_addr)
               : "memory");
  return v;
}
// wait with cluster-scope acquire (arrivals / tx may come from another CTA of the cluster)
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "HB_WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra HB_WAITC_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// arrive on (and expect tx bytes at) an mbarrier of another CTA of the cluster; relaxed: the
// data it announces arrives through the async proxy (bulk copy, complete_tx), so no generic
// memory operation has to be ordered before it (a release.cluster arrive costs a MEMBAR.GPU)
__device__ __forceinline__ void mbar_arrive_expect_tx_remote(uint32_t cluster_bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.relaxed.cluster.shared::cluster.b64 _, [%0], %1;" ::"r"(cluster_bar),
               "r"(bytes)
               : "memory");
}
// arrive on an mbarrier of a CTA of the cluster (shared::cluster address), releasing this thread's
// prior memory operations (and, after tcgen05.fence::before_thread_sync, its TMEM reads) at cluster scope
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_bar) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_bar) : "memory");
}
// bulk copy local shared memory -> shared memory of another CTA of the cluster, completion
// (bytes) signalled on that CTA's mbarrier
__device__ __forceinline__ void bulk_copy_s2cluster(uint32_t cluster_dst, const void* src, uint32_t bytes,
                                                    uint32_t cluster_bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          cluster_dst),
      "r"(smem_u32(src)), "r"(bytes), "r"(cluster_bar)
      : "memory");
}
// arrive on the mbarrier at the same smem offset in every CTA of cta_mask when all previously
// issued tcgen05.mma of this thread complete
__device__ __forceinline__ void umma_commit_multicast(uint64_t* bar, uint16_t cta_mask) {
  asm volatile(
      "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(cta_mask)
      : "memory");
}

// Tuning builds (-DHB_TUNING, build.py --variant tuning HB_TUNING) record per-CTA phase timestamps
// into a caller-armed buffer; product builds compile every stamp away.
#ifdef HB_TUNING
#define HB_STAMP(cond, slot) \
  do {                        \
    if (cond) (slot) = gtimer(); \
  } while (0)
#else
#define HB_STAMP(cond, slot) \
  do {                        \
  } while (0)
#endif

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ float sigmoidf_(float z) { return __fdividef(1.0f, 1.0f + __expf(-z)); }

// h = sigma(z) and d = sigma'(z) = sigma(z) (1 - sigma(z)) without cancellation or overflow:
// with e = exp(-|z|) <= 1 and s = 1 / (1 + e):  sigma(|z|) = s, sigma(-|z|) = e s,  d = e s^2.
__device__ __forceinline__ void sigmoid_d(float z, float& h, float& d) {
  const float e = __expf(-fabsf(z));
  const float s = __fdividef(1.0f, 1.0f + e);
  const float es = e * s;
  h = z >= 0.f ? s : es;
  d = es * s;
}

// Tensor-core epilogues: the same formulas with ONE MUFU op per element (ex2).  1/(1+e), 1+e in
// (1, 2], starts from the minimax line 24/17 - 8/17 y (relative error <= 1/17) and takes two
// Newton steps s <- s (2 - y s) on the FMA pipe (error 1/17 -> 3.5e-3 -> 1.2e-5, far below the
// bf16 rounding of H and S).  The fp32 check mode keeps sigmoid_d.
__device__ __forceinline__ float ex2_ftz(float x) {  // MUFU.EX2 without __expf's denormal fix-up
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void sigmoid_d_fast(float z, float& h, float& d) {
  // e = exp(-|z|) flushed to 0 below 2^-126 (|z| > 87): then h = 0 or 1 and d = 0, exact in bf16
  const float e = ex2_ftz(fabsf(z) * -1.4426950408889634f);
  const float y = 1.0f + e;
#ifdef HB_SIG_RCP  // tuning only: MUFU reciprocal instead of the FMA-pipe Newton steps
  float s;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(s) : "f"(y));
#else
  float s = fmaf(-8.0f / 17.0f, y, 24.0f / 17.0f);
  s = s * fmaf(-y, s, 2.0f);
  s = s * fmaf(-y, s, 2.0f);
#endif
  const float es = e * s;
  h = z >= 0.f ? s : es;
  d = es * s;
}

// sigmoid_d_fast of two elements, z = acc + bias, on the packed fp32x2 pipe (FADD2 / FFMA2 / FMUL2,
// sm_100): the same IEEE operations per element in the same order — the negations are exact and
// fma(e, -1, -1) = -(1 + e) rounded — so the results are bitwise those of two sigmoid_d_fast
// calls, at about half the FP instructions (the tile epilogues are issue-bound on them)
__device__ __forceinline__ void sigmoid_d_fast2(float a0, float a1, float b0, float b1, float& h0, float& h1,
                                                float& d0, float& d1) {
  const float2 z = __fadd2_rn(make_float2(a0, a1), make_float2(b0, b1));
#ifdef HB_FAKE_SIG  // tuning only (wrong numerics): the epilogue's cost without the sigmoid math
  h0 = z.x; h1 = z.y; d0 = z.x * 0.25f; d1 = z.y * 0.25f;
  return;
#endif
  const float2 e = make_float2(ex2_ftz(fabsf(z.x) * -1.4426950408889634f), ex2_ftz(fabsf(z.y) * -1.4426950408889634f));
  const float2 ny = __ffma2_rn(e, make_float2(-1.0f, -1.0f), make_float2(-1.0f, -1.0f));
  const float2 two = make_float2(2.0f, 2.0f);
  float2 s = __ffma2_rn(make_float2(8.0f / 17.0f, 8.0f / 17.0f), ny, make_float2(24.0f / 17.0f, 24.0f / 17.0f));
  s = __fmul2_rn(s, __ffma2_rn(ny, s, two));
  s = __fmul2_rn(s, __ffma2_rn(ny, s, two));
  const float2 es = __fmul2_rn(e, s);
  const float2 dd = __fmul2_rn(es, s);
  h0 = z.x >= 0.f ? s.x : es.x;
  h1 = z.y >= 0.f ? s.y : es.y;
  d0 = dd.x;
  d1 = dd.y;
}

}  // namespace hb
