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
 *  4. a write also marks its 128-word chunk (and 16K-word super-chunk) in two
 *     byte maps with plain idempotent stores (test before store, no atomics),
 *     so closing the epoch costs O(chunks written), not O(shadow).
 * A single-word access (the common case: an aligned scalar) takes a short path
 * with one ballot; multi-word accesses loop over the shadow u32s they cover.
 * Device hooks never fail and never block.
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
  const struct xpl_dev_row* rows; /* live rows, sorted by base                   */
  const unsigned int* n_rows;     /* number of live rows                         */
  unsigned int* pool;             /* shadow pool, 4 records per u32              */
  unsigned char* cmap;            /* 1 byte per 128-word chunk: GPU write pending */
  unsigned char* smap;            /* 1 byte per 128 chunks (16K words)            */
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

/* Mark the chunk (and super-chunk) of shadow u32 q as holding a pending GPU
 * write: plain idempotent byte stores, tested first (a stale cached 0 only
 * costs a redundant store).  Only first writes of a shadow u32 get here. */
static __device__ __forceinline__ void xpld_mark(unsigned q) {
  unsigned char* c = xpl_dctx.cmap + (q >> 5);
  if (!*c) *c = 1;
  unsigned char* s = xpl_dctx.smap + (q >> 12);
  if (!*s) *s = 1;
}

/* OR the record bits m into shadow u32 q for the lanes in `needers` (lanes with
 * bits still missing): lanes hitting the same u32 are grouped and one leader
 * issues the atomic.  Only the lanes of `needers` may call it. */
static __device__ __forceinline__ void xpld_commit(unsigned needers, unsigned q, unsigned m) {
  const unsigned grp = __match_any_sync(needers, q);
  const unsigned M = __reduce_or_sync(grp, m);
  if (xpld_lane() == (unsigned)(__ffs(grp) - 1)) {
    atomicOr(xpl_dctx.pool + q, M);  /* no return value needed: RED */
    if (M & XPLD_P4) xpld_mark(q);
  }
}

/* The record bits an access of kind acc sets on the 4 records of shadow u32 cur,
 * restricted to the byte lanes of `bytes` (0xFF per record touched). */
static __device__ __forceinline__ unsigned xpld_bits(unsigned cur, unsigned bytes, unsigned acc) {
  unsigned m = 0;
  if (acc & XPL_ACC_R) {
    const unsigned l = cur & 0x01010101u;                  /* L per record        */
    m = ((l << 7) | ((~l & 0x01010101u) << 6)) & bytes;    /* rGG if L else rCG   */
  }
  if (acc & XPL_ACC_W) m |= 0x0A0A0A0Au & bytes;           /* wG | P              */
  return m;
}

/* Apply a GPU access to the shadow words [g0, g1] (global pool word indices;
 * empty when g0 > g1).  All active lanes of the calling warp must call it. */
static __device__ __forceinline__ void xpl_dev_apply(unsigned long long g0,
                                                     unsigned long long g1,
                                                     unsigned acc) {
  const unsigned active = __activemask();
  const bool single = g0 >= g1; /* one word (g0 == g1) or none (g0 > g1) */
  const unsigned singles = __ballot_sync(active, single);
  if (single) { /* the short path */
    const bool hit = g0 == g1;
    const unsigned q = (unsigned)(g0 >> 2);
    unsigned cur = 0, m = 0;
    if (hit) {
      cur = xpl_dctx.pool[q];
      m = xpld_bits(cur, 0xFFu << (8 * (unsigned)(g0 & 3)), acc);
    }
    const bool need = hit && (cur & m) != m;
    const unsigned needers = __ballot_sync(singles, need);
    if (need) xpld_commit(needers, q, m);
  }
  if (singles == active) return;
  /* multi-word accesses: one shadow u32 per iteration */
  const bool multi = g0 < g1;
  unsigned long long q = g0 >> 2;
  const unsigned long long ql = g1 >> 2;
  bool more = multi;
  while (__any_sync(active, more)) {
    unsigned cur = 0, m = 0;
    if (more) {
      cur = xpl_dctx.pool[q];
      unsigned bytes = 0;
#pragma unroll
      for (unsigned k = 0; k < 4; ++k) {
        const unsigned long long gw = q * 4 + k;
        if (gw >= g0 && gw <= g1) bytes |= 0xFFu << (8 * k);
      }
      m = xpld_bits(cur, bytes, acc);
    }
    const bool need = more && (cur & m) != m;
    const unsigned needers = __ballot_sync(active, need);
    if (need) xpld_commit(needers, (unsigned)q, m);
    more = more && q < ql;
    ++q;
  }
}

/* Lookup + apply.  size in bytes; acc = XPL_ACC_R / _W / _RW.
 * A per-warp cache of the last row found (in shared memory, 32 slots per
 * block, validated against the row on every use, so stale or uninitialised
 * slots only cost the full search) skips the binary search when consecutive
 * accesses of a warp hit the same allocation -- the common case. */
static __device__ __forceinline__ void xpl_dev_record(const void* p, unsigned size,
                                                      unsigned acc) {
#ifndef XPL_OFF
  __shared__ unsigned xpl_row_cache[32];
  const unsigned long long a = (unsigned long long)p;
  const xpl_dev_row* rows = xpl_dctx.rows;
  const unsigned n = __ldg(xpl_dctx.n_rows);
  const unsigned slot = ((threadIdx.z * blockDim.y + threadIdx.y) * blockDim.x + threadIdx.x) >> 5 & 31;
  unsigned ri = xpl_row_cache[slot];
  bool hit = ri < n && __ldg(&rows[ri].base) <= a && a < __ldg(&rows[ri].end);
  if (!hit) {
    unsigned lo = 0, hi = n;
    while (lo < hi) {
      const unsigned mid = (lo + hi) >> 1;
      if (__ldg(&rows[mid].base) <= a) lo = mid + 1;
      else hi = mid;
    }
    if (lo > 0 && a < __ldg(&rows[lo - 1].end)) {
      ri = lo - 1;
      hit = true;
      xpl_row_cache[slot] = ri;  /* benign race: any lane's row is a valid entry */
    }
  }
  unsigned long long g0 = 1, g1 = 0;
  if (hit && size > 0) {
    const xpl_dev_row* r = rows + ri;
    const unsigned long long base = __ldg(&r->base);
    const unsigned long long w0 = (a - base) >> 2;
    unsigned long long wl = (a + size - 1 - base) >> 2;
    const unsigned long long wmax = __ldg(&r->words) - 1;
    if (wl > wmax) wl = wmax;
    const unsigned long long off = __ldg(&r->off);
    g0 = off + w0;
    g1 = off + wl;
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
