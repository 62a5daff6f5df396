/* oracle/xpl_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, sequential CPU oracle for XPlacer's recording + diagnosis
 * (Pirkelbauer et al., IPDPS 2020; "P:Lnnn" = line nnn of the paper text).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this.  It shares no code, header, table or
 * constant with the CUDA path (paper_conf_ipps_pirkelbauerlvl20_b200/), and
 * neither side includes the other.
 *
 * Every entry point returns 0 on success and a negative number on a usage
 * error (the event is then ignored).  Addresses are plain integers: the
 * oracle never dereferences them.
 */
#ifndef XPL_ORACLE_H
#define XPL_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct xo_state xo_state;

/* One row of the diagnosis (Fig. 4 columns + SURVEY §8c). */
typedef struct {
  uint64_t id, base, bytes, words;
  uint32_t kind, live, name_idx, flags;
  uint64_t w_c, w_g, r_cc, r_cg, r_gc, r_gg, any_acc, gpu_acc, alternating,
      density_pct_any, density_pct_gpu, low_density_blocks, low_density_words,
      h2d_unused_runs, h2d_unused_words, d2h_unneeded_runs, d2h_unneeded_words,
      ever_accessed;
} xo_report;

xo_state* xo_new(void);
void xo_delete(xo_state*);
/* kind: 0 = cudaMalloc, 1 = cudaMallocManaged, 2 = host. Returns id >= 0. */
int64_t xo_reg(xo_state*, uint64_t ptr, uint64_t bytes, uint32_t kind);
int xo_free(xo_state*, uint64_t ptr);
int xo_kb(xo_state*);
int xo_ke(xo_state*);
/* acc: 1 = R, 2 = W, 3 = RW (read, then write). */
int xo_host(xo_state*, uint64_t addr, uint32_t size, uint32_t acc);
int xo_host_batch(xo_state*, const uint64_t* addr, const uint32_t* size,
                  const uint8_t* acc, size_t n);
int xo_dev(xo_state*, uint64_t addr, uint32_t size, uint32_t acc);
int xo_dev_batch(xo_state*, const uint64_t* addr, const uint32_t* size,
                 const uint8_t* acc, size_t n);
/* dir: 0 H2D, 1 D2H, 2 H2H, 3 D2D, 4 device memset (dst only). */
int xo_copy(xo_state*, uint64_t dst, uint64_t src, uint64_t bytes, uint32_t dir);
/* Returns the number of rows written (or needed, if > cap), negative on error. */
int64_t xo_diag(xo_state*, uint32_t thr_pct, uint64_t block_words,
                uint64_t min_run, int reset, const uint64_t* name_addrs,
                size_t n_names, xo_report* out, size_t cap);
/* UM page view (D31-D33):
 * per live row, its pages of page_words words counted from the base. */
typedef struct {
  uint64_t id, base, words, page_words, pages;
  uint32_t kind, advice;
  uint64_t cpu_pages, gpu_pages, shared_pages, false_shared_pages, alternating_pages;
  uint32_t flags, pad;
} xo_page_report;
/* Rows written (or needed, if > cap); negative on error.  Changes nothing. */
int64_t xo_pages(xo_state*, uint64_t page_words, xo_page_report* out, size_t cap);
/* cudaMemAdvise: advice 1..6 in cudaMemoryAdvise order, device < 0 = CPU. */
int xo_advise(xo_state*, uint64_t ptr, uint32_t advice, int device);
/* The record byte of (allocation id, word); 0 if never touched. */
int xo_peek(xo_state*, uint64_t id, uint64_t word);

#ifdef __cplusplus
}
#endif
#endif
