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

#define XPLW_MAX_ARRAYS 64

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
  int diag_no_reset;      /* 1 = diagnoses keep the interval bits (D25)            */
  int keep_allocs;        /* 1 = leave the arrays registered at the end (no final  *
                           *     frees + diagnose), for shadow dumps (LULESH)      */
  int rank, world;        /* world > 1: this process is rank `rank` of a sharded  *
                           * run (ctx sharded too); LULESH runs its slab only     */
  float* kernel_ms_each;  /* time_kernels: each launch's event time, in order (or NULL) */
  size_t kernel_cap;
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

/* Rodinia bfs: n nodes with `deg` out-edges each (node i: edges [deg*i, deg*i+deg)),
 * level-synchronous from node 0, two kernels per level, `over` flag round trip.
 * arrays: 0 h_nodes, 1 h_edges, 2 h_mask, 3 h_updating, 4 h_visited, 5 h_cost,
 *         6 h_over (HOST), 7 d_nodes, 8 d_edges, 9 d_mask, 10 d_updating,
 *         11 d_visited, 12 d_cost, 13 d_over (DEVICE).  h_edges holds the graph
 *         (input).  hook_count: device u64 the instrumented kernels add their
 *         hook calls to (data-dependent).  Returns the number of levels in *levels. */
int xplw_bfs(xplw_run* run, const xplw_arrays* a, int n, int deg, unsigned long long* hook_count,
             int* levels);

/* Rodinia nw (Needleman-Wunsch): (n+1) x (n+1) ints, 16 x 16 tiles, 2*(n/16)-1
 * block-diagonal kernels, host traceback over the D2H result.
 * arrays: 0 input_itemsets, 1 referrence, 2 output_itemsets (HOST), 3 referrence_cuda,
 *         4 matrix_cuda (DEVICE).  blosum: 24 x 24 substitution scores (host, not
 * traced).  input_itemsets row/column 0 hold the sequences (1..23) on entry;
 * output_itemsets holds the expected DP result (the traceback reads it when
 * do_copies == 0, i.e. when the D2H is not performed). */
int xplw_nw(xplw_run* run, const xplw_arrays* a, int n, int penalty, const int* blosum);

/* Smith-Waterman (Fig. 7/8 P:L341-349; cfg1 SW-128 and cfg3 SW-16K of SURVEY §8(d)):
 * managed a[n], b[m], H[(n+1) x (m+1)] ints; the CPU writes a, b and zero-fills H;
 * GPU epochs fill H (score +3 match / -3 mismatch, gap 2, floor 0):
 *   per_diagonal = 0: ONE launch of one CTA (n <= 1024 threads) sweeping all
 *                     anti-diagonals with __syncthreads (cfg1);
 *   per_diagonal = 1: one launch per anti-diagonal d = 2 .. n+m (cfg3); every
 *                     `tb_every` diagonals a host segment reads the finished diagonal,
 *                     every `diag_every` diagonals a diagnose (0 = never);
 * then the CPU scans H for the maximum and traces back from it; with
 * per_diagonal = 0 a final GPU epoch re-zeroes the interior (the next query).
 * arrays: 0 a, 1 b, 2 H (MANAGED).  a, b hold the sequences (0..3) on entry.
 * Returns the traceback length in *tb_len. */
int xplw_sw(xplw_run* run, const xplw_arrays* a, int n, int m, int per_diagonal, int tb_every,
            int diag_every, int* tb_len);

/* LULESH-shaped program (§II-C, §III-D, Fig. 4; cfg4/cfg5): edge s elements,
 * `steps` timesteps of 19 instrumented launches with two temporaries allocated
 * and freed per step (managed, registered by the program) and a diagnose after
 * each step.  arrays: 0 dom (3736 B), 1 dt_block (2*ceil(s^3/256) doubles),
 * 2 + k = the array of domain pointer slot k for k < 48 (all MANAGED; slots
 * 26..32 hold the mesh topology on entry).  hook_count: device u64.  tmp_addrs:
 * host array of 2*steps (the temporaries' addresses, for the CPU twin) or NULL. */
int xplw_lulesh(xplw_run* run, const xplw_arrays* a, int s, int steps, unsigned long long* hook_count,
                unsigned long long* tmp_addrs);
int xplw_lulesh_layout(int what);

#ifdef __cplusplus
}
#endif
#endif
