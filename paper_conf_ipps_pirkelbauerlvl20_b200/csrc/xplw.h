/* xplw.h -- C interface of libxplwork.so: instrumented "user applications"
 * shaped like the paper's workloads, written against the
 * public xpl.h / xpl_device.cuh only.  Each app runs its whole program: host
 * loops traced with xpl_record_host, transfers traced with xpl_record_copy
 * (and performed when do_copies), instrumented kernels between
 * xpl_kernel_begin/_end, and xpl_diagnose at the paper's points.  With
 * run->ctx == NULL the same app runs uninstrumented (twin kernels compiled
 * without hooks, no xpl call) -- the baseline of the slowdown metric.
 *
 * Array order and sizes are fixed by xplgen/rodinia.py (the input generator);
 * the caller owns every array (device arrays in HBM, host arrays pinned). */
#ifndef XPLW_H
#define XPLW_H
#include <stddef.h>
#include <stdint.h>

#include "xpl.h"

#ifdef __cplusplus
extern "C" {
#endif

#define XPLW_MAX_ARRAYS 24

typedef struct {
  uint64_t addr[XPLW_MAX_ARRAYS];  /* base address of each array (app order)   */
  uint64_t bytes[XPLW_MAX_ARRAYS]; /* its size                                 */
  uint32_t kind[XPLW_MAX_ARRAYS];  /* xpl_alloc_kind it is registered as       */
  int n;
} xplw_arrays;

typedef struct {
  xpl_ctx* ctx;         /* NULL => uninstrumented twin                          */
  void* stream;         /* cudaStream_t of the app's kernels                    */
  int do_copies;        /* 1 = perform the app's cudaMemcpy calls too           */
  int diag_each;        /* diagnose after every iteration (else at the end only) */
  xpl_diag_params params;
  xpl_alloc_report* out; /* reports of every diagnose, appended                 */
  size_t out_cap, n_out;
  uint32_t* diag_rows;  /* rows of each diagnose                                */
  size_t diag_cap, n_diag;
  uint64_t dev_accesses;  /* counted by the app: hook calls                     */
  uint64_t host_accesses; /* host tracer calls                                  */
  uint64_t copy_words;    /* words moved by traced transfers                    */
  uint64_t epochs;
  int status;             /* first xpl_status / CUDA failure                    */
  int time_kernels;       /* 1 = time the app's kernels with CUDA events          */
  double kernel_ms;       /* sum of the app's kernel times (time_kernels)         */
  double host_ms;         /* host wall time spent in traced host loops + tracer   */
} xplw_run;

/* Rodinia hotspot: rows x cols temperatures, `iters` 5-point stencil steps.
 * arrays: 0 temp_host, 1 power_host, 2 result_host (HOST), 3 d_power,
 *         4 d_temp0, 5 d_temp1 (DEVICE). */
int xplw_hotspot(xplw_run* run, const xplw_arrays* a, int rows, int cols, int iters);

/* Rodinia backprop: `in` input units, `hid` hidden units, 16x16 tiles.
 * arrays: 0 input_units, 1 input_weights, 2 partial_sum, 3 hidden_delta,
 *         4 prev_weights (HOST), 5 input_cuda, 6 output_hidden_cuda,
 *         7 input_hidden_cuda, 8 hidden_partial_sum, 9 hidden_delta_cuda,
 *         10 input_prev_weights_cuda (DEVICE). */
int xplw_backprop(xplw_run* run, const xplw_arrays* a, int in, int hid);

#ifdef __cplusplus
}
#endif
#endif
