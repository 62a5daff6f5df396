/* include/xpl_device.cuh -- header-only __device__ hooks of the B200-native
 * XPlacer runtime: traceR / traceW / traceRW for instrumented CUDA kernels
 * (Table I; Fig. 2).
 *
 * Usage (one context per process):
 *     #include "xpl_device.cuh"
 *     xpl_device_bind(ctx);                        // once per translation unit
 *     xpl_kernel_begin(ctx, stream);
 *     my_kernel<<<g, b, 0, stream>>>(...);         // calls xpl_read(a[i]), xpl_write(b[i]) ...
 *     xpl_kernel_end(ctx, stream);
 * Compile the same kernel with -DXPL_OFF to get the uninstrumented twin.
 *
 * What a hook does (design: DESIGN.md §5):
 *  1. lookup: binary search of the address in the live-allocation table
 *     (sorted by base, read-only while a kernel runs); a miss ignores the access;
 *  2. shadow update: every 32-bit word the access overlaps gets
 *       read  -> rCG (value written by the CPU) or rGG (by the GPU), chosen by the
 *                record's last-writer bit L, which is frozen for the whole epoch
 *                (snapshot semantics, D5);
 *       write -> wG and P ("GPU write pending"; the epoch close turns P into L=1);
 *  3. warp aggregation: lanes that hit the same shadow u32 (4 records) are grouped
 *     with __match_any_sync, their bits OR-reduced, and one leader issues a single
 *     atomicOr -- and only if some bit is still missing (test before set);
 *  4. the first pending write in a shadow u32 appends its index to the dirty list,
 *     so closing the epoch costs O(words written), not O(shadow).
 * Device hooks never fail: a dirty-list overflow makes the epoch close scan the
 * whole pool instead (results are unchanged).
 */
#ifndef XPL_DEVICE_CUH
#define XPL_DEVICE_CUH

#include <cuda_runtime.h>
#include <stdint.h>

#include "xpl.h"

/* One live allocation as the hooks see it (sorted by base). */
struct xpl_dev_row {
  unsigned long long base;  /* first byte                       */
  unsigned long long end;   /* one past the last byte           */
  unsigned long long off;   /* first shadow word in the pool    */
  unsigned long long words; /* ceil(bytes/4)                    */
};

struct xpl_dev_ctx {
  const struct xpl_dev_row* rows; /* live rows, sorted by base      */
  const unsigned int* n_rows;     /* number of live rows            */
  unsigned int* pool;             /* shadow pool, 4 records per u32 */
  unsigned int* dirty;            /* dirty list (u32 indices)       */
  unsigned int* dirty_count;
  unsigned int dirty_cap;
  unsigned int pad_;
};

#ifdef __CUDACC__

/* Translation-unit-local copy of the device context (set by xpl_device_bind). */
static __constant__ xpl_dev_ctx xpl_dctx;

static inline xpl_status xpl_device_bind(xpl_ctx* ctx) {
  xpl_dev_ctx d;
  xpl_status s = xpl_get_device_ctx(ctx, &d);
  if (s != XPL_OK) return s;
  return cudaMemcpyToSymbol(xpl_dctx, &d, sizeof d) == cudaSuccess ? XPL_OK : XPL_ERR_CUDA;
}

/* Record byte layout ("processor of the last write ... whether a CPU or
 * GPU wrote ... whether a CPU or GPU read ... and whether the data originated on
 * the CPU or GPU"; seven bits + the pending bit P in the spare eighth). */
#define XPLD_L 0x01u
#define XPLD_P 0x02u
#define XPLD_WG 0x08u
#define XPLD_RCG 0x40u
#define XPLD_RGG 0x80u
#define XPLD_P4 0x02020202u

static __device__ __forceinline__ unsigned xpld_lane() {
  unsigned l;
  asm("mov.u32 %0, %%laneid;" : "=r"(l));
  return l;
}

/* Apply a GPU access to the shadow words [g0, g1] (global pool word indices;
 * empty when g0 > g1).  All lanes of the calling warp that are active must call it. */
static __device__ __forceinline__ void xpl_dev_apply(unsigned long long g0,
                                                     unsigned long long g1,
                                                     unsigned acc) {
  const unsigned active = __activemask();
  const unsigned lane = xpld_lane();
  unsigned long long q = g0 >> 2;
  const unsigned long long ql = g1 >> 2;
  bool more = g0 <= g1;
  while (__any_sync(active, more)) {
    unsigned m = 0, cur = 0;
    if (more) {
      cur = xpl_dctx.pool[q];
#pragma unroll
      for (unsigned k = 0; k < 4; ++k) {
        const unsigned long long gw = q * 4 + k;
        if (gw >= g0 && gw <= g1) {
          unsigned b = 0;
          if (acc & XPL_ACC_R) b = ((cur >> (8 * k)) & XPLD_L) ? XPLD_RGG : XPLD_RCG;
          if (acc & XPL_ACC_W) b |= XPLD_WG | XPLD_P;
          m |= b << (8 * k);
        }
      }
    }
    const bool need = more && ((cur & m) != m);
    if (__any_sync(active, need)) {
      const unsigned long long key = need ? q : ~0ull;
      const unsigned grp = __match_any_sync(active, key);
      const unsigned M = __reduce_or_sync(grp, m);
      if (need && lane == (unsigned)(__ffs(grp) - 1)) {
        if (M & XPLD_P4) {
          const unsigned old = atomicOr(xpl_dctx.pool + q, M);
          if ((old & XPLD_P4) == 0) {
            const unsigned i = atomicAdd(xpl_dctx.dirty_count, 1u);
            if (i < xpl_dctx.dirty_cap) xpl_dctx.dirty[i] = (unsigned)q;
          }
        } else {
          atomicOr(xpl_dctx.pool + q, M);
        }
      }
    }
    more = more && q < ql;
    ++q;
  }
}

/* Lookup + apply.  size in bytes; acc = XPL_ACC_R / _W / _RW. */
static __device__ __forceinline__ void xpl_dev_record(const void* p, unsigned size,
                                                      unsigned acc) {
#ifndef XPL_OFF
  const unsigned long long a = (unsigned long long)p;
  const xpl_dev_row* rows = xpl_dctx.rows;
  unsigned lo = 0, hi = __ldg(xpl_dctx.n_rows);
  while (lo < hi) {
    const unsigned mid = (lo + hi) >> 1;
    if (__ldg(&rows[mid].base) <= a) lo = mid + 1;
    else hi = mid;
  }
  unsigned long long g0 = 1, g1 = 0;
  if (lo > 0 && size > 0) {
    const xpl_dev_row* r = rows + (lo - 1);
    const unsigned long long base = __ldg(&r->base);
    if (a < __ldg(&r->end)) {
      const unsigned long long w0 = (a - base) >> 2;
      unsigned long long wl = (a + size - 1 - base) >> 2;
      const unsigned long long wmax = __ldg(&r->words) - 1;
      if (wl > wmax) wl = wmax;
      const unsigned long long off = __ldg(&r->off);
      g0 = off + w0;
      g1 = off + wl;
    }
  }
  xpl_dev_apply(g0, g1, acc);
#else
  (void)p; (void)size; (void)acc;
#endif
}

/* traceR / traceW / traceRW: take the element, return it (Table I). */
template <class T>
static __device__ __forceinline__ const T& xpl_read(const T& x) {
  xpl_dev_record(&x, sizeof(T), XPL_ACC_R);
  return x;
}
template <class T>
static __device__ __forceinline__ T& xpl_write(T& x) {
  xpl_dev_record(&x, sizeof(T), XPL_ACC_W);
  return x;
}
template <class T>
static __device__ __forceinline__ T& xpl_rw(T& x) {
  xpl_dev_record(&x, sizeof(T), XPL_ACC_RW);
  return x;
}

#endif /* __CUDACC__ */
#endif /* XPL_DEVICE_CUH */
