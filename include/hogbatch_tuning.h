/*
 * hogbatch_tuning.h — tuning-only entry points of the TUNING build of libhogbatch
 * (python paper_conf_ipps_marws21_b200/build.py --variant tuning HB_TUNING ->
 *  paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so, loaded by the scripts with
 *  HB_LIB=<path>).  The product library does not export these symbols; the tuning build also
 * compiles the kernels' per-phase globaltimer stamps (HB_STAMP) and reads HB_* environment
 * overrides of launch choices (tile width, splits, cluster size, ring depth, k-block order).
 * Same conventions as hogbatch.h (int status, hb_last_error()).
 */
#ifndef HOGBATCH_TUNING_H
#define HOGBATCH_TUNING_H

#include "hogbatch.h"

#ifdef __cplusplus
extern "C" {
#endif

/* tuning only: mean device microseconds of one tensor-core GEMM launch of the given kind
 * (0 forward+sigmoid, 1 dgrad+sigma', 2 wgrad+SGD) and shape on zero-filled scratch buffers */
int hb_bench_gemm(int32_t kind, int32_t M, int32_t N, int32_t K, int32_t iters, float* us_out);
/* kind: 0 forward, 1 dX, 2 dW + fused SGD, 3 dW storing the fp32 gradient (unfused baseline).
 * hb_bench_sgd_apply: the unfused SGD update alone (W -= lr G, shadow rewritten) over n fp32
 * weights (n % 4 == 0), mean device microseconds per launch. */
int hb_bench_sgd_apply(int64_t n, int32_t iters, float* us_out);
/* tuning only: per-CTA phase timestamps (8 globaltimer ns values per CTA, cap entries) of one launch */
/* tuning only: hb_rc_trace(NULL, cap) arms per-step globaltimer stamps (10 per CTA per step, 24 steps
 * per CTA) in later fused row-block launches; hb_rc_trace(host, cap) reads the last launch's */
int hb_rc_trace(unsigned long long* host, int64_t cap);
/* tuning only: mean device microseconds of one SGD step (graph-replayed `iters` times, lr = 0) on
 * rows [0, batch) of X/y; part 0 = whole step, 1 = fused chain only, 2 = dW GEMMs only */
int hb_bench_step(hb_worker* w, const void* X, int64_t ldx, const int32_t* y, int32_t batch, int32_t iters,
                  int32_t part, float* us_out);
int hb_bench_gemm_phases(int32_t kind, int32_t M, int32_t N, int32_t K, unsigned long long* host_ts, int64_t cap);

#ifdef __cplusplus
}
#endif
#endif /* HOGBATCH_TUNING_H */
