// comm.cu — multi-GPU replica merge over NCCL (NVLink 5 / NVSwitch).
//
// PAPER.md §V.B [L141]: "If the update is applied to the deep replica, this has to be
// subsequently integrated in the global model"; §VI.B [L174–L175]: the GPU replica is pushed to
// the global model.  With one replica per GPU (multi-GPU is the paper's future work, L277) the
// integration of every replica's delta is one all-reduce:
//     W <- W_base + gamma * sum_ranks (W_rank - W_base),   W_base <- W
// done over the whole flat fp32 parameter buffer (weights + biases) in a single ncclAllReduce.
#include <nccl.h>

#include <cstring>
#include <string>

#include "kernels.cuh"
#include "model.h"

struct hb_comm {
  ncclComm_t comm = nullptr;
  int device = 0, nranks = 1, rank = 0;
};

using namespace hb;

extern "C" {

int hb_nccl_unique_id(uint8_t out[128]) {
  HB_CHECK_ARG(out, "null out");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return fail(HB_ENCCL, std::string("ncclGetUniqueId: ") + ncclGetErrorString(r));
  static_assert(sizeof(id.internal) == 128, "ncclUniqueId size");
  std::memcpy(out, id.internal, 128);
  return HB_OK;
}

int hb_comm_create(const uint8_t id[128], int32_t nranks, int32_t rank, int32_t device, hb_comm** out) {
  HB_CHECK_ARG(id && out && nranks >= 1 && rank >= 0 && rank < nranks, "bad comm arguments");
  *out = nullptr;
  HB_CUDA_TRY(cudaSetDevice(device));
  ncclUniqueId uid;
  std::memcpy(uid.internal, id, 128);
  hb_comm* c = new hb_comm();
  ncclResult_t r = ncclCommInitRank(&c->comm, nranks, uid, rank);
  if (r != ncclSuccess) {
    delete c;
    return fail(HB_ENCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
  }
  c->device = device;
  c->nranks = nranks;
  c->rank = rank;
  *out = c;
  return HB_OK;
}

int hb_comm_destroy(hb_comm* c) {
  if (!c) return HB_OK;
  cudaSetDevice(c->device);
  if (c->comm) ncclCommDestroy(c->comm);
  delete c;
  return HB_OK;
}

int hb_merge_begin(hb_model* m) {
  HB_CHECK_ARG(m, "null model");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  if (!m->base) HB_CUDA_TRY(cudaMalloc(&m->base, m->total * 4));
  if (!m->delta) HB_CUDA_TRY(cudaMalloc(&m->delta, m->total * 4));
  HB_CUDA_TRY(cudaDeviceSynchronize());
  HB_CUDA_TRY(cudaMemcpyAsync(m->base, m->master, m->total * 4, cudaMemcpyDeviceToDevice, m->stream));
  HB_CUDA_TRY(cudaStreamSynchronize(m->stream));
  return HB_OK;
}

int hb_merge(hb_model* m, hb_comm* c, float gamma, void* cuda_stream) {
  HB_CHECK_ARG(m && c, "null arg");
  if (!m->base) return fail(HB_ESTATE, "hb_merge_begin was not called");
  HB_CUDA_TRY(cudaSetDevice(m->device));
  cudaStream_t s = cuda_stream ? static_cast<cudaStream_t>(cuda_stream) : m->stream;
  HB_CUDA_TRY(cudaDeviceSynchronize());  // every worker's in-place updates are visible
  const int64_t n = (int64_t)m->total;
  Prof pr(HB_PROF_OTHER, s);
  merge_delta_kernel<<<592, 256, 0, s>>>(m->master, m->base, m->delta, n);
  HB_CUDA_TRY(cudaGetLastError());
  ncclResult_t r = ncclAllReduce(m->delta, m->delta, (size_t)n, ncclFloat, ncclSum, c->comm, s);
  if (r != ncclSuccess) return fail(HB_ENCCL, std::string("ncclAllReduce: ") + ncclGetErrorString(r));
  merge_apply_kernel<<<592, 256, 0, s>>>(m->master, m->base, m->delta, gamma, m->shadow, n);
  HB_CUDA_TRY(cudaGetLastError());
  pr.done(2, 0.0, 4.0 * 7.0 * n);
  HB_CUDA_TRY(cudaStreamSynchronize(s));
  return HB_OK;
}

int hb_merge_replicas(hb_model* m, hb_worker* const* workers, int32_t n, float gamma) {
  HB_CHECK_ARG(m && (workers || n == 0) && n >= 0, "bad arguments");
  if (!m->base) return fail(HB_ESTATE, "hb_merge_begin was not called");
  ReplicaPtrs r{};
  int nr = 0;
  for (int i = 0; i < n; ++i) {
    hb_worker* w = workers[i];
    HB_CHECK_ARG(w && w->global == m, "every worker must belong to this model");
    if (w->m == m) continue;  // reference replica: its updates are already in the global model
    HB_CHECK_ARG(nr < 8, "at most 8 deep replicas per merge");
    r.w[nr] = w->m->master;
    r.sh[nr] = w->m->shadow;
    ++nr;
  }
  HB_CUDA_TRY(cudaSetDevice(m->device));
  HB_CUDA_TRY(cudaDeviceSynchronize());  // every worker's updates of its replica have landed
  Prof pr(HB_PROF_OTHER, m->stream);
  merge_replicas_kernel<<<592, 256, 0, m->stream>>>(m->master, m->base, m->shadow, r, nr, gamma, (int64_t)m->total);
  HB_CUDA_TRY(cudaGetLastError());
  pr.done(1, 0.0, 4.0 * (double)m->total * (4.0 + 2.0 * nr) + 2.0 * (double)m->total * (1 + nr));
  HB_CUDA_TRY(cudaStreamSynchronize(m->stream));
  return HB_OK;
}

}  // extern "C"
