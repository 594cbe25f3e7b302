// pair_probe.cu — standalone check of the CTA-pair tensor-core path (tcgen05.mma.cta_group::2,
// M = 256) that DESIGN.md §10 ranks as the next lever: one 256 x 256 x K tile, A and B K-major
// bf16, each CTA of the pair loading its 128 A rows and its 128 B rows, the leader issuing the
// MMAs, both CTAs reading their 128 accumulator rows.  Not part of the library.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -I paper_conf_ipps_marws21_b200/csrc \
//        scripts/pair_probe.cu -o scripts/pair_probe -lcuda
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "common.cuh"

using namespace hb;

constexpr int NS = 4;
constexpr int STAGE_A = 128 * 128;  // 128 rows x 64 bf16
constexpr int STAGE = 2 * STAGE_A;  // A half + B half

__device__ __forceinline__ void tma_load_2d_pair(void* dst, const CUtensorMap* m, uint32_t bar_cluster, int32_t c0,
                                                 int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(bar_cluster), "r"(c0), "r"(c1)
      : "memory");
}

__device__ __forceinline__ void umma_bf16_pair(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                               uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

__device__ __forceinline__ void umma_commit_pair(uint64_t* bar, uint16_t mask) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(mask)
      : "memory");
}

__global__ void __launch_bounds__(256, 1) pair_kernel(const __grid_constant__ CUtensorMap tA,
                                                      const __grid_constant__ CUtensorMap tB, float* C, int K) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * STAGE);
  uint64_t* empty = full + NS;
  uint64_t* acc_full = empty + NS;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(acc_full + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const int nkb = K / 64;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < NS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    mbar_init(acc_full, 1);
    fence_barrier_init();
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0 && lane == 0) {
    // both CTAs: own 128 A rows and own 128 B rows of every k-block, completing on the LEADER's barrier
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % NS;
      mbar_wait(&empty[s], ((kb / NS) & 1) ^ 1);
      if (rank == 0) mbar_arrive_expect_tx(&full[s], 2 * STAGE);
      const uint32_t bar0 = mapa_shared(smem_u32(&full[s]), 0);
      uint8_t* st = smem + s * STAGE;
      tma_load_2d_pair(st, &tA, bar0, kb * 64, (int)rank * 128);
      tma_load_2d_pair(st + STAGE_A, &tB, bar0, kb * 64, (int)rank * 128);
    }
  } else if (warp == 1 && lane == 0 && rank == 0) {
    constexpr uint32_t idesc = make_idesc_bf16(256, 256, false, false);
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % NS;
      mbar_wait(&full[s], (kb / NS) & 1);
      tc_fence_after();
      const uint32_t a = smem_u32(smem + s * STAGE), b = a + STAGE_A;
      for (int kk = 0; kk < 4; ++kk)
        umma_bf16_pair(tmem, make_sw128_desc(a + kk * 32, 16, 1024), make_sw128_desc(b + kk * 32, 16, 1024), idesc,
                       (kb | kk) != 0);
      umma_commit_pair(&empty[s], 0x3);
    }
    umma_commit_pair(acc_full, 0x3);
  } else if (warp >= 4) {
    const int q = warp & 3;
    mbar_wait(acc_full, 0);
    tc_fence_after();
    const int row = (int)rank * 128 + q * 32 + lane;
    for (int c = 0; c < 256; c += 16) {
      uint32_t r[16];
      tmem_ld_32x32b_x16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)c, r);
      tmem_ld_wait();
      for (int j = 0; j < 16; ++j) C[(size_t)row * 256 + c + j] = __uint_as_float(r[j]);
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync_all();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 256;" ::"r"(tmem));
  }
}

static uint16_t f2bf(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}
static float bf2f(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return f;
}

int main(int argc, char** argv) {
  const int K = argc > 1 ? atoi(argv[1]) : 512;
  std::vector<uint16_t> A(256 * K), B(256 * K);
  srand(1);
  for (auto& v : A) v = f2bf((rand() / (float)RAND_MAX - 0.5f));
  for (auto& v : B) v = f2bf((rand() / (float)RAND_MAX - 0.5f));
  void *dA, *dB;
  float* dC;
  cudaMalloc(&dA, A.size() * 2);
  cudaMalloc(&dB, B.size() * 2);
  cudaMalloc(&dC, 256 * 256 * 4);
  cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
  cudaMemset(dC, 0, 256 * 256 * 4);
  CUtensorMap mA, mB;
  for (int i = 0; i < 2; ++i) {
    cuuint64_t dims[2] = {(cuuint64_t)K, 256};
    cuuint64_t strides[1] = {(cuuint64_t)K * 2};
    cuuint32_t box[2] = {64, 128};
    cuuint32_t es[2] = {1, 1};
    CUresult r = cuTensorMapEncodeTiled(i ? &mB : &mA, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, i ? dB : dA, dims, strides,
                                        box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r) {
      printf("encode failed %d\n", (int)r);
      return 1;
    }
  }
  const int smem = NS * STAGE + 2048;
  cudaFuncSetAttribute(pair_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, pair_kernel, mA, mB, dC, K);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  printf("launch: %s\n", cudaGetErrorString(e));
  if (e) return 1;
  std::vector<float> C(256 * 256);
  cudaMemcpy(C.data(), dC, C.size() * 4, cudaMemcpyDeviceToHost);
  double num = 0, den = 0, maxe = 0;
  int bad_i = -1, bad_j = -1;
  for (int i = 0; i < 256; ++i)
    for (int j = 0; j < 256; ++j) {
      double ref = 0;
      for (int k = 0; k < K; ++k) ref += (double)bf2f(A[i * K + k]) * bf2f(B[j * K + k]);
      const double d = C[i * 256 + j] - ref;
      num += d * d;
      den += ref * ref;
      if (fabs(d) > maxe) {
        maxe = fabs(d);
        bad_i = i;
        bad_j = j;
      }
    }
  printf("K=%d rel err %.3e  max abs err %.3e at (%d, %d)  C[0][0]=%f C[255][255]=%f\n", K, sqrt(num / den), maxe,
         bad_i, bad_j, C[0], C[255 * 256 + 255]);
  return sqrt(num / den) < 1e-3 ? 0 : 2;
}
