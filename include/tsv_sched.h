/*
 * tsv_sched.h — TetriServe's round-based scheduler (paper §4.2), the consumer of the
 * step-latency table T(res, k) that tsv_latency_table exports.  Pure host code, no GPU.
 *
 * T is a row-major double[n_res][n_k] table of step latencies (seconds or any unit, consistently
 * with deadlines and tau); entries <= 0 mark unavailable (res, k) cells; ks[j] is the SP degree of
 * column j (powers of two).  N = number of GPUs in the pool.
 */
#ifndef TSV_SCHED_H_
#define TSV_SCHED_H_

#include <stdint.h>
#include "tsv.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  double deadline;      /* D_i, absolute time in the table's unit */
  int remaining_steps;  /* S_i still to run */
  int table_row;        /* row of T (the request's resolution class) */
} tsv_sched_request;

/* Deadline-aware GPU allocation (eq. at): the steps per degree (steps_per_k[n_k], summing to
 * remaining_steps) minimising sum_k s_k k T(k) subject to sum_k s_k T(k) <= deadline - now
 * (queueing taken as 0 at planning time).  Exact (enumerates all compositions).  If no
 * allocation meets the deadline, *late = 1 and all steps go to the smallest available degree
 * (best effort).  Ties: smaller total time, then larger degrees.  Errors: TSV_E_INVAL. */
tsv_status tsv_sched_allocate(const double* T, int n_res, const int* ks, int n_k, const tsv_sched_request* req,
                              double now, int N, int* steps_per_k, int* late);

/* One scheduling round of length tau starting at `now` (Alg. 1): per request the GPUs
 * (gpus_out[i], 0 = not scheduled) and steps (steps_out[i]) it runs this round, maximising the
 * number of requests that are not "definitely late" at now + tau under capacity N (group-knapsack
 * DP, O(R N)); late requests then receive one leftover GPU each, best effort.
 * *survivors (may be NULL) = the DP optimum.  Errors: TSV_E_INVAL. */
tsv_status tsv_sched_round(const double* T, int n_res, const int* ks, int n_k, const tsv_sched_request* reqs, int R,
                           double now, double tau, int N, int* gpus_out, int* steps_out, int* survivors);

/* tsv_sched_round with the tie at Alg. 1 line 21 (several capacities c attaining the optimum)
 * selectable: work_conserving = 0 takes the smallest c (= tsv_sched_round, reading S31: requests
 * with slack are deferred), != 0 the largest (reading S31b: every request that can make progress
 * now runs at its minimal allocation; the survivor count is the same optimum). */
tsv_status tsv_sched_round_ex(const double* T, int n_res, const int* ks, int n_k, const tsv_sched_request* reqs,
                              int R, double now, double tau, int N, int work_conserving, int* gpus_out,
                              int* steps_out, int* survivors);

/* GPU placement with preservation and elastic scale-up (S:§8(f) NEXT #4).  gpus[i] =
 * GPUs granted to request i this round (0 or a power of two, e.g. tsv_sched_round's gpus_out),
 * rows[i] its table row, prev_mask[i] the bitmask of the GPUs it held in the previous round (0 =
 * none).  N <= 64.  Placement: requests in decreasing size (ties: lower index) each take the free
 * aligned block (start % size == 0) with the largest overlap with prev_mask[i] (ties: lowest
 * start), so a request whose size is unchanged and whose block is free keeps its GPUs (no
 * reshard).  Elastic scale-up (scale_up != 0, work-conserving, "no GPU remains unused"):
 * first every request left without GPUs takes one idle GPU (one it held before if free, else the
 * lowest), in index order; then while some placed request of size
 * g has its buddy block (the other half of its aligned 2g block) entirely idle and T(row, 2g) <
 * T(row, g), the one with the largest T(g) / T(2g) (ties: lower index) doubles in place.  Output:
 * mask_out[i] (popcount = the final size).  Errors: TSV_E_INVAL (sizes, total > N, no fit). */
tsv_status tsv_sched_place(const double* T, int n_res, const int* ks, int n_k, const int* rows, const int* gpus,
                           const uint64_t* prev_mask, int R, int N, int scale_up, uint64_t* mask_out);

const char* tsv_sched_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* TSV_SCHED_H_ */
