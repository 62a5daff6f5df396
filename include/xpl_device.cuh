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
 * Latency variants (same records, for latency-bound kernels -- few threads, one
 * access after another): xpl_read_lat(x) defers the commit to the end of the
 * full expression so its shadow load overlaps the user's load (C++17: the proxy
 * is returned by guaranteed copy elision); xpl_write_lat(x) stores the chunk
 * mark without testing it first.  Array handles (xpl_array<T>) hoist the
 * lookup of a base pointer out of repeated accesses.
 *
 * What a hook does (design: DESIGN.md §5):
 *  1. lookup: binary search of the address in the live-allocation table
 *     (sorted by base, read-only while a kernel runs); a miss ignores the access;
 *  2. shadow update: every 32-bit word the access overlaps gets
 *       read  -> rCG (value written by the CPU) or rGG (by the GPU), chosen by the
 *                record's last-writer bit L, which is frozen for the whole epoch
 *                (snapshot semantics, D5);
 *       write -> wG, and P ("GPU write pending"; the epoch close turns P into
 *                L=1) where L is still the CPU (where it is the GPU already,
 *                the epoch ends with L=1 anyway: no P, no fold work);
 *  3. warp aggregation: lanes that hit the same shadow u32 (4 records) are grouped
 *     with __match_any_sync, their bits combined (per-byte-lane ballots), and one
 *     leader issues a single atomicOr -- and only if some bit is still missing
 *     (test before set);
 *  4. a write that sets P also marks its 128-word chunk (and 16K-word
 *     super-chunk) in two byte maps with plain idempotent stores (test before
 *     store, no atomics), so closing the epoch costs O(chunks with P), not
 *     O(shadow).
 * Paths: a compile-time-kind call site whose active lanes all access words
 * inside one local shadow u32 (aligned scalars up to doubles) runs one
 * straight-line warp-convergent sequence (xpld_record_fast); per-lane kinds
 * and multi-u32 accesses take the general path (xpl_dev_apply), which loops
 * over the shadow u32s an access covers; in sharded mode (xpl.h) words of
 * another rank's pieces go to its peer-mapped pool (xpld_remote).
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
  const unsigned long long* n_super; /* super-chunks below the pool's high-water mark */
  unsigned int* flags;            /* [0]: a device-side epoch split ran in the open epoch */
  /* sharded mode (xpl.h): a row's `off` carries its owner rank in the top byte;
   * the other ranks' pools and chunk maps are mapped here (CUDA IPC, NVLink) */
  unsigned int rank, world;
  unsigned int* pools[XPL_MAX_RANKS];
  unsigned char* cmaps[XPL_MAX_RANKS];
  unsigned char* smaps[XPL_MAX_RANKS];
};

#ifdef __CUDACC__

#include <cooperative_groups.h>

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
/* The whole-warp consecutive-element path of the compile-time-kind hooks and
 * the array handles (xpld_record_fast, xpl_array::rec_contig).  A/B switch:
 * XPL_HANDLE_CONTIG=0. */
#ifndef XPL_HANDLE_CONTIG
#define XPL_HANDLE_CONTIG 1
#endif
/* The same check on the plain hooks' path (after the lookup): measured neutral
 * on streams and up to 10 % slower on gather kernels (profiles/r2z_contig_ab.txt),
 * so off by default. */
#ifndef XPL_PLAIN_CONTIG
#define XPL_PLAIN_CONTIG 0
#endif

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
 * costs a redundant store).  Both bytes are loaded before either store, so
 * the two loads overlap.  Only first writes of a shadow u32 get here.  The
 * first mark of a super-chunk also raises flags[2] ("the epoch close has
 * work"), so the close of an epoch that set no pending write ends at once.
 * flags[2] is one word every marking lane of the grid would store to (a
 * scattered writer, e.g. a wavefront's cells in 16K different rows, marks a
 * new super-chunk per lane): it is tested first (its line stays in L1), so
 * about one store per SM reaches L2 instead of one per lane; the latency
 * variant raises it with a RED (no wait, combined at L2). */
template <bool TESTED = true>
static __device__ __forceinline__ void xpld_mark(unsigned q) {
  unsigned char* c = xpl_dctx.cmap + (q >> 5);
  unsigned char* s = xpl_dctx.smap + (q >> 12);
  if (TESTED) {
#if XPL_MARK_FLAG_LAZY  /* A/B: the flag word loaded only on a super-chunk's first mark */
    const unsigned cv = *c, sv = *s;
    if (!cv) *c = 1;
    if (!sv) {
      *s = 1;
      if (!xpl_dctx.flags[2]) xpl_dctx.flags[2] = 1u;
    }
#else
    const unsigned cv = *c, sv = *s, fv = xpl_dctx.flags[2];
    if (!cv) *c = 1;
    if (!sv) {
      *s = 1;
      if (!fv) xpl_dctx.flags[2] = 1u;
    }
#endif
  } else {  /* latency variant: plain stores, nothing to wait for */
    *c = 1;
    *s = 1;
    atomicOr(xpl_dctx.flags + 2, 1u);
  }
}

/* The record bits a read of the byte lanes rb and a write of the byte lanes wb
 * (0xFF per record) set on the 4 records of shadow u32 cur.  A write sets wG,
 * and P ("make L = GPU at the epoch close") only where L is still the CPU: L is
 * constant within an epoch (D5), so a word the GPU wrote last already ends the
 * epoch with L = GPU -- no P, no chunk mark, no fold work for it. */
static __device__ __forceinline__ unsigned xpld_bits2(unsigned cur, unsigned rb, unsigned wb) {
  const unsigned l = cur & 0x01010101u;                           /* L per record      */
  const unsigned nl = ~l & 0x01010101u;                           /* L == CPU          */
  return (((l << 7) | (nl << 6)) & rb)                            /* rGG if L else rCG */
         | ((0x08080808u | (nl << 1)) & wb);                      /* wG, P if L == CPU */
}

/* The record bits an access of kind acc sets on the 4 records of shadow u32 cur,
 * restricted to the byte lanes of `bytes` (0xFF per record touched). */
static __device__ __forceinline__ unsigned xpld_bits(unsigned cur, unsigned bytes, unsigned acc) {
  return xpld_bits2(cur, (acc & XPL_ACC_R) ? bytes : 0u, (acc & XPL_ACC_W) ? bytes : 0u);
}

/* Commit the access of every lane of `needers` (lanes with bits still missing):
 * lanes hitting the same shadow u32 q are grouped (__match_any_sync) and one
 * leader issues a single atomicOr with the group's bits.  The group's bits are
 * formed from warp ballots (which byte lanes the group reads / writes), not
 * from a reduction over the group's own lane mask: that mask differs between
 * groups, and a reduction under a non-uniform mask serialises over the groups.
 * Any lane's `cur` gives the group's L bits (L is frozen for the epoch).
 * K = the access kind when it is the same for every lane (the hook's call site
 * fixes it), 0 when each lane brings its own (acc).  SINGLE: every lane touches
 * one byte lane, bytes == 0xFF << 8*b, so two ballots of b's bits name the
 * group's byte lanes.  Only the lanes of `needers` may call it. */
template <unsigned K, bool SINGLE, bool TM = true>
static __device__ __forceinline__ void xpld_commit(unsigned needers, unsigned q, unsigned cur,
                                                   unsigned bytes, unsigned acc) {
  const unsigned grp = __match_any_sync(needers, q);
  unsigned rb = 0, wb = 0;
  if (K != 0 && SINGLE) {
    const unsigned b = (unsigned)(__ffs(bytes) - 1) >> 3;
    const unsigned b0 = __ballot_sync(needers, b & 1) & grp, b1 = __ballot_sync(needers, b & 2) & grp;
    const unsigned n0 = grp & ~b0, n1 = grp & ~b1;
    const unsigned u = ((n0 & n1) ? 0x000000FFu : 0u) | ((b0 & n1) ? 0x0000FF00u : 0u) |
                       ((n0 & b1) ? 0x00FF0000u : 0u) | ((b0 & b1) ? 0xFF000000u : 0u);
    rb = (K & XPL_ACC_R) ? u : 0u;
    wb = (K & XPL_ACC_W) ? u : 0u;
  } else if (SINGLE) {
    /* per-lane kinds, one byte lane each: four ballots (byte-lane bits, R, W)
     * name, per byte lane, whether some lane of the group reads / writes it */
    const unsigned b = (unsigned)(__ffs(bytes) - 1) >> 3;
    const unsigned b0 = __ballot_sync(needers, b & 1) & grp, b1 = __ballot_sync(needers, b & 2) & grp;
    const unsigned r = __ballot_sync(needers, acc & XPL_ACC_R) & grp;
    const unsigned w = __ballot_sync(needers, acc & XPL_ACC_W) & grp;
    const unsigned n0 = grp & ~b0, n1 = grp & ~b1;
    const unsigned l0 = n0 & n1, l1 = b0 & n1, l2 = n0 & b1, l3 = b0 & b1;
    rb = ((l0 & r) ? 0x000000FFu : 0u) | ((l1 & r) ? 0x0000FF00u : 0u) | ((l2 & r) ? 0x00FF0000u : 0u) |
         ((l3 & r) ? 0xFF000000u : 0u);
    wb = ((l0 & w) ? 0x000000FFu : 0u) | ((l1 & w) ? 0x0000FF00u : 0u) | ((l2 & w) ? 0x00FF0000u : 0u) |
         ((l3 & w) ? 0xFF000000u : 0u);
  } else {
#pragma unroll
    for (unsigned k = 0; k < 4; ++k) {
      const unsigned sel = 0xFFu << (8 * k);
      const bool has = (bytes & sel) != 0;
      if (K != 0) {
        if (__ballot_sync(needers, has) & grp) {
          if (K & XPL_ACC_R) rb |= sel;
          if (K & XPL_ACC_W) wb |= sel;
        }
      } else {
        if (__ballot_sync(needers, has && (acc & XPL_ACC_R)) & grp) rb |= sel;
        if (__ballot_sync(needers, has && (acc & XPL_ACC_W)) & grp) wb |= sel;
      }
    }
  }
  if (xpld_lane() == (unsigned)(__ffs(grp) - 1)) {
    const unsigned bits = xpld_bits2(cur, rb, wb);
    atomicOr(xpl_dctx.pool + q, bits); /* no return value needed: RED */
    if (bits & XPLD_P4) xpld_mark<TM>(q);
  }
}

/* A row's `off` holds its owner rank in the top byte (sharded mode). */
#define XPLD_OFF_MASK 0x00FFFFFFFFFFFFFFull

/* Sharded mode: the lanes whose access falls in a piece another rank owns
 * record it in that rank's pool (peer-mapped, CUDA IPC), with the same bits
 * and test-before-set as a local hook; lanes on one (owner, shadow u32) are
 * grouped (match + OR) so one atomic crosses NVLink per group.  Out of line:
 * remote words are the exception (halo and small shared objects). */
template <unsigned K>
static __device__ __noinline__ void xpld_remote(unsigned owner, unsigned long long g0,
                                                unsigned long long g1, unsigned acc) {
  unsigned* const P = xpl_dctx.pools[owner];
  unsigned long long q = g0 >> 2;
  const unsigned long long ql = g1 >> 2;
  bool more = true;
  while (__any_sync(__activemask(), more)) {
    if (more) {
      unsigned bytes = 0;
#pragma unroll
      for (unsigned k = 0; k < 4; ++k) {
        const unsigned long long gw = q * 4 + k;
        if (gw >= g0 && gw <= g1) bytes |= 0xFFu << (8 * k);
      }
      const unsigned cur = __ldcg(P + q);
      const unsigned m = xpld_bits(cur, bytes, acc);
      const bool need = (cur & m) != m;
      const unsigned needers = __ballot_sync(__activemask(), need);
      if (need) {
        const unsigned grp = __match_any_sync(needers, ((unsigned long long)owner << 40) | q);
        const unsigned bits = __reduce_or_sync(grp, m);
        if (xpld_lane() == (unsigned)(__ffs(grp) - 1)) {
          atomicOr_system(P + q, bits); /* (system scope: another GPU's memory over NVLink) */
          if (bits & XPLD_P4) {
            unsigned char* c = xpl_dctx.cmaps[owner] + (q >> 5);
            unsigned char* sm = xpl_dctx.smaps[owner] + (q >> 12);
            if (!*c) *c = 1;
            if (!*sm) *sm = 1;
          }
        }
      }
    }
    more = more && q < ql;
    ++q;
  }
}

/* Test-before-set commit of one shadow u32 q by one lane: bits = the record
 * bits of the byte lanes rb (read) / wb (written) given the u32's value cur at
 * the hook (its L bits are the epoch's). */
template <unsigned K, bool TM>
static __device__ __forceinline__ void xpld_put(unsigned q, unsigned cur, unsigned rb, unsigned wb) {
  const unsigned bits = xpld_bits2(cur, rb, wb);
  if ((cur & bits) != bits) {
    atomicOr(xpl_dctx.pool + q, bits); /* no return value needed: RED */
    if (bits & XPLD_P4) xpld_mark<TM>(q);
  }
}

/* The lanes of `ones` each access words [g0, g0+nb1] inside ONE shadow u32
 * (every aligned access of <= 4 words: ints, floats, doubles, ...):
 *  1. each lane loads its shadow u32 and tests whether a bit of its access is
 *     still missing (test before set; a write-only call site K == W always
 *     commits: wG | P do not depend on the record, so it loads nothing); a warp
 *     with nothing missing (a re-touch) is done after one load and one ballot;
 *  2. lanes on the same u32 are grouped (__match_any_sync); a lane alone in its
 *     group (strided or scattered accesses) commits its own bits at once;
 *  3. a larger group's byte lanes come from four ballots (one per byte lane of
 *     the u32, uniform over the remaining lanes, so no serialisation over the
 *     groups) and its first lane commits.
 * K: the access kind if uniform (compile-time call site), else 0 (per lane). */
template <unsigned K, bool TM>
static __device__ __forceinline__ void xpld_one(unsigned ones, unsigned long long g0, unsigned nb1,
                                                unsigned acc) {
  const unsigned lane = xpld_lane();
  const unsigned q = (unsigned)(g0 >> 2);
  const unsigned bm = (0xFFFFFFFFu >> (24 - 8 * nb1)) << (8 * ((unsigned)g0 & 3u));
  const unsigned kind = K ? K : acc;
  const unsigned cur = xpl_dctx.pool[q];
  const unsigned rb = (kind & XPL_ACC_R) ? bm : 0u, wb = (kind & XPL_ACC_W) ? bm : 0u;
  const unsigned mine = xpld_bits2(cur, rb, wb);
  const bool need = (cur & mine) != mine;
  const unsigned needers = __ballot_sync(ones, need);
  if (!need) return;
  const unsigned grp = __match_any_sync(needers, q);
  const unsigned me = 1u << lane;
  const unsigned alone = __ballot_sync(needers, grp == me);
  if (grp == me) {
    xpld_put<K, TM>(q, cur, rb, wb);
    return;
  }
  const unsigned rest = needers & ~alone;
  unsigned gr = 0, gw = 0;
#pragma unroll
  for (unsigned k = 0; k < 4; ++k) {
    const unsigned sel = 0xFFu << (8 * k);
    if (K != 0) {
      if (__ballot_sync(rest, (bm & sel) != 0) & grp) {
        if (K & XPL_ACC_R) gr |= sel;
        if (K & XPL_ACC_W) gw |= sel;
      }
    } else {
      if (__ballot_sync(rest, (rb & sel) != 0) & grp) gr |= sel;
      if (__ballot_sync(rest, (wb & sel) != 0) & grp) gw |= sel;
    }
  }
  if (lane == (unsigned)(__ffs(grp) - 1)) xpld_put<K, TM>(q, cur, gr, gw);
}

/* Apply a GPU access to the shadow words [g0, g1] (global pool word indices;
 * empty when g0 > g1).  All active lanes of the calling warp must call it.
 * K: the access kind if uniform over the warp (a compile-time call site), else 0. */
template <unsigned K, bool TM = true>
static __device__ __forceinline__ void xpl_dev_apply(unsigned long long g0,
                                                     unsigned long long g1,
                                                     unsigned acc) {
  const unsigned active = __activemask();
  const bool hit = g0 <= g1;
  const bool one = hit && (g0 >> 2) == (g1 >> 2); /* inside one shadow u32 */
  const unsigned ones = __ballot_sync(active, one);
  if (one) xpld_one<K, TM>(ones, g0, (unsigned)(g1 - g0), acc);
  const bool multi = hit && !one;
  const unsigned multis = __ballot_sync(active, multi);
  if (!multi) return;
  /* accesses over several shadow u32s: one u32 per iteration */
  unsigned long long q = g0 >> 2;
  const unsigned long long ql = g1 >> 2;
  bool more = true;
  while (__any_sync(multis, more)) {
    unsigned cur = 0, m = 0, bytes = 0;
    if (more) {
      cur = xpl_dctx.pool[q];
#pragma unroll
      for (unsigned k = 0; k < 4; ++k) {
        const unsigned long long gw = q * 4 + k;
        if (gw >= g0 && gw <= g1) bytes |= 0xFFu << (8 * k);
      }
      m = xpld_bits(cur, bytes, acc);
    }
    const bool need = more && (cur & m) != m;
    const unsigned needers = __ballot_sync(multis, need);
    if (need) xpld_commit<K, false, TM>(needers, (unsigned)q, cur, bytes, acc);
    more = more && q < ql;
    ++q;
  }
}

/* Lookup + apply.  size in bytes; acc = XPL_ACC_R / _W / _RW.
 * A per-warp cache of the last row found (in shared memory, 32 slots per
 * block, validated against the row on every use, so stale or uninitialised
 * slots only cost the full search) skips the binary search when consecutive
 * accesses of a warp hit the same allocation -- the common case. */
/* The per-warp row cache (one per block, shared by every hook of the kernel). */
static __device__ __forceinline__ unsigned* xpld_row_cache() {
  __shared__ unsigned c[32];
  return c;
}

/* The row (live allocation) holding address a: (base, end) and (off | owner
 * << 56, words); false = untracked. */
static __device__ __forceinline__ bool xpld_find(unsigned long long a, ulonglong2& be, ulonglong2& ow) {
  unsigned* const xpl_row_cache = xpld_row_cache();
  const xpl_dev_row* rows = xpl_dctx.rows;
  const unsigned n = __ldg(xpl_dctx.n_rows);
  const unsigned slot = ((threadIdx.z * blockDim.y + threadIdx.y) * blockDim.x + threadIdx.x) >> 5 & 31;
  unsigned ri = xpl_row_cache[slot];
  const unsigned rc = ri < n ? ri : 0; /* (n == 0: nothing matches below) */
  be = __ldg(reinterpret_cast<const ulonglong2*>(rows + rc));     /* base, end  */
  ow = __ldg(reinterpret_cast<const ulonglong2*>(rows + rc) + 1); /* off, words */
  bool hit = ri < n && be.x <= a && a < be.y;
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
      atomicExch(xpl_row_cache + slot, ri); /* (lanes may store different rows: any is valid) */
      be = __ldg(reinterpret_cast<const ulonglong2*>(rows + ri));
      ow = __ldg(reinterpret_cast<const ulonglong2*>(rows + ri) + 1);
    }
  }
  return hit;
}

/* Words [g0, g1] (in the owner's pool) of an access of `size` bytes at a in the
 * row [base, end) whose shadow starts at pool word offo (owner rank in the top
 * byte): clipped to the row (D1, D18; its last word is (end - 1 - base) / 4). */
static __device__ __forceinline__ void xpld_words(unsigned long long a, unsigned size, unsigned long long base,
                                                  unsigned long long end, unsigned long long offo,
                                                  unsigned long long& g0, unsigned long long& g1,
                                                  unsigned& owner) {
  const unsigned long long w0 = (a - base) >> 2;
  unsigned long long wl = (a + size - 1 - base) >> 2;
  const unsigned long long wmax = (end - 1 - base) >> 2;
  if (wl > wmax) wl = wmax;
  owner = (unsigned)(offo >> 56);
  g0 = (offo & XPLD_OFF_MASK) + w0;
  g1 = (offo & XPLD_OFF_MASK) + wl;
}

/* Record words [g0, g1] of rank `owner`'s pool (g0 > g1: nothing).  All active
 * lanes of the warp call it. */
template <unsigned K, bool TM = true>
static __device__ __forceinline__ void xpld_record_words(unsigned long long g0, unsigned long long g1,
                                                         unsigned owner, unsigned acc) {
  /* sharded mode: words another rank owns go to its pool over NVLink (rare) */
  const bool remote = owner != xpl_dctx.rank && g0 <= g1;
  const unsigned long long l0 = remote ? 1ull : g0, l1 = remote ? 0ull : g1;
  xpl_dev_apply<K, TM>(l0, l1, acc);
  if (__any_sync(__activemask(), remote) && remote) xpld_remote<K>(owner, g0, g1, acc);
}

/* The compile-time-kind hook (every xpl_read / xpl_write / xpl_rw call site):
 * when every active lane's access is local and inside one shadow u32 (or
 * misses) -- the common case -- one straight-line, warp-convergent sequence:
 * a predicated shadow load, the test before set, one ballot (a re-touching
 * warp is done here), then match_any groups, four byte-lane ballots and one
 * atomicOr per group.  Every warp-synchronous op runs at the same level for
 * all active lanes (no divergent collectives).  Anything else (multi-u32
 * accesses, remote pieces) takes the general path, decided warp-uniformly. */
template <unsigned K, bool TM = true>
static __device__ __forceinline__ void xpld_record_fast(unsigned long long g0, unsigned long long g1,
                                                        unsigned owner) {
  const unsigned act = __activemask();
  const bool hit = g0 <= g1;
  const bool fast = !hit || (owner == xpl_dctx.rank && (g0 ^ g1) < 4ull);
  if (__ballot_sync(act, !fast)) { /* uniform: some lane needs the general path */
    xpld_record_words<K, TM>(g0, g1, owner, K);
    return;
  }
  const unsigned lane = xpld_lane();
  const unsigned q = (unsigned)(g0 >> 2);
  const unsigned bm = hit ? (0xFFFFFFFFu >> (24 - 8 * (unsigned)(g1 - g0))) << (8 * ((unsigned)g0 & 3u)) : 0u;
  const unsigned cur = hit ? xpl_dctx.pool[q] : 0u;
  const unsigned rb = (K & XPL_ACC_R) ? bm : 0u, wb = (K & XPL_ACC_W) ? bm : 0u;
  const unsigned mine = xpld_bits2(cur, rb, wb);
  const bool need = hit && (cur & mine) != mine;
  const unsigned needers = __ballot_sync(act, need);
  if (!needers) return; /* uniform: nothing missing (a re-touch) */
#if XPL_PLAIN_CONTIG
  /* a whole warp on consecutive 4- or 8-byte elements starting a shadow u32
   * (p[i0 + lane]): each u32 of the span is covered by 4 / W whole lanes --
   * its first lane commits the u32's bits, no grouping (as xpl_array::rec_contig) */
  if (act == 0xFFFFFFFFu) {
    const unsigned w = (unsigned)(g1 - g0) + 1u;
    const unsigned long long b = g0 - (unsigned long long)lane * w;
    const unsigned long long b0 = __shfl_sync(0xFFFFFFFFu, b, 0);
    const unsigned w0 = __shfl_sync(0xFFFFFFFFu, w, 0);
    if (__all_sync(0xFFFFFFFFu, hit && b == b0 && w == w0 && w <= 2u && (b & 3ull) == 0)) {
      if ((lane & (4u / w - 1u)) == 0)
        xpld_put<K, TM>(q, cur, (K & XPL_ACC_R) ? 0xFFFFFFFFu : 0u, (K & XPL_ACC_W) ? 0xFFFFFFFFu : 0u);
      return;
    }
  }
#endif
  const unsigned grp = __match_any_sync(act, need ? q : 0xFFFFFFFFu) & needers;
#if XPL_FAST_ALONE  /* A/B: scattered warps (every needer alone on its u32) commit at once */
  if (__all_sync(act, !need || grp == (1u << lane))) {
    if (need) xpld_put<K, TM>(q, cur, rb, wb);
    return;
  }
#endif
  unsigned gb = 0;
#pragma unroll
  for (unsigned k = 0; k < 4; ++k) {
    const unsigned sel = 0xFFu << (8 * k);
    if (__ballot_sync(act, need && (bm & sel)) & grp) gb |= sel;
  }
  if (need && lane == (unsigned)(__ffs(grp) - 1))
    xpld_put<K, TM>(q, cur, (K & XPL_ACC_R) ? gb : 0u, (K & XPL_ACC_W) ? gb : 0u);
}

/* A hooked read's own data load is issued after the hook (the hook returns the
 * reference the caller loads through), so its latency would add to the hook's
 * shadow load.  A prefetch of the data line at the start of the hook overlaps
 * the two (the caller's load then hits L1).  A/B switch: XPL_HOOK_PREFETCH=0. */
#ifndef XPL_HOOK_PREFETCH
#define XPL_HOOK_PREFETCH 1
#endif

static __device__ __forceinline__ void xpld_prefetch(const void* p) {
#if XPL_HOOK_PREFETCH
  asm volatile("prefetch.L1 [%0];" ::"l"(p));
#else
  (void)p;
#endif
}

template <unsigned K, bool TM = true>
static __device__ __forceinline__ void xpl_dev_record_k(const void* p, unsigned size,
                                                        unsigned acc) {
#ifndef XPL_OFF
  if (K & XPL_ACC_R) xpld_prefetch(p);
  const unsigned long long a = (unsigned long long)p;
  ulonglong2 be, ow;
  unsigned long long g0 = 1, g1 = 0;
  unsigned owner = xpl_dctx.rank;
  if (xpld_find(a, be, ow) && size > 0) xpld_words(a, size, be.x, be.y, ow.x, g0, g1, owner);
  if (K != 0) xpld_record_fast<K, TM>(g0, g1, owner);
  else xpld_record_words<K, TM>(g0, g1, owner, acc);
#else
  (void)p; (void)size; (void)acc;
#endif
}

/* traceR / traceW / traceRW through an array handle: the row lookup of the
 * array's base pointer is done once (when the handle is made) instead of once
 * per access -- the hoisting an instrumenting compiler does for a loop-invariant
 * base.  Same records as xpl_read(p[i]) etc.: an element outside the handle's
 * row falls back to the full lookup (D18: an access belongs to the row holding
 * its first byte). */
template <class T>
struct xpl_array {
  T* p;
  /* element i of p (0 <= i < nel: whole elements inside the row holding p)
   * covers pool words q0 + i * W .. q0 + i * W + W - 1 of rank `owner`; else
   * (outside the row, or T not a multiple of 4 bytes / p not word-aligned in
   * its row) the access takes the full lookup.  W = sizeof(T) / 4. */
  unsigned long long q0 = 0, nel = 0;
  unsigned owner = 0;
  __device__ __forceinline__ explicit xpl_array(T* ptr) : p(ptr) {
#ifndef XPL_OFF
    ulonglong2 be, ow;
    const unsigned long long a = (unsigned long long)ptr;
    if (sizeof(T) % 4 == 0 && xpld_find(a, be, ow) && ((a - be.x) & 3) == 0) {
      q0 = (ow.x & XPLD_OFF_MASK) + ((a - be.x) >> 2);
      nel = (be.y - a) / sizeof(T);
      owner = (unsigned)(ow.x >> 56);
    }
#endif
  }
  /* A whole warp on 32 consecutive elements (i = i0 + lane: the streaming
   * case, e.g. p[blockIdx.x * blockDim.x + threadIdx.x]) of 4- or 8-byte T,
   * local, inside the row, the first element's words starting a shadow u32:
   * every shadow u32 of the warp's span is covered by 4 / W whole lanes, so its
   * record bits are known without grouping -- the group's first lane loads,
   * tests and commits them (the same bits and test as the general path).
   * Checked at run time (one 64-bit shuffle, one vote); false: not the case. */
  template <unsigned K>
  __device__ __forceinline__ bool rec_contig(unsigned long long i) const {
    constexpr unsigned W = (unsigned)(sizeof(T) / 4);
    if (__activemask() != 0xFFFFFFFFu) return false; /* (uniform) */
    const unsigned lane = xpld_lane();
    const unsigned long long b = i - lane;
    const unsigned long long b0 = __shfl_sync(0xFFFFFFFFu, b, 0);
    const bool ok = b == b0 && i < nel && owner == xpl_dctx.rank && ((q0 + b * W) & 3ull) == 0;
    if (!__all_sync(0xFFFFFFFFu, ok)) return false;
    if ((lane & (4 / W - 1)) == 0) {
      const unsigned q = (unsigned)((q0 + i * W) >> 2);
      xpld_put<K, true>(q, xpl_dctx.pool[q], (K & XPL_ACC_R) ? 0xFFFFFFFFu : 0u,
                        (K & XPL_ACC_W) ? 0xFFFFFFFFu : 0u);
    }
    return true;
  }
  template <unsigned K>
  __device__ __forceinline__ void rec(unsigned long long i) const {
#ifndef XPL_OFF
    constexpr unsigned long long W = sizeof(T) / 4;
#if XPL_HANDLE_CONTIG
    if constexpr (sizeof(T) == 4 || sizeof(T) == 8)
      if (rec_contig<K>(i)) return;
#endif
    unsigned long long g0 = 1, g1 = 0;
    unsigned own = owner;
    if (i < nel) {
      g0 = q0 + i * W;
      g1 = g0 + (W - 1);
    } else {
      const unsigned long long a = (unsigned long long)(p + i);
      ulonglong2 b2, o2;
      own = xpl_dctx.rank;
      if (xpld_find(a, b2, o2)) xpld_words(a, sizeof(T), b2.x, b2.y, o2.x, g0, g1, own);
    }
    xpld_record_fast<K>(g0, g1, own);
#else
    (void)i;
#endif
  }
  /* read: the element is loaded before the hook runs, so the data load and the
   * hook's shadow load are in flight together (the value is returned) */
  __device__ __forceinline__ T read(unsigned long long i) const {
#if XPL_HOOK_PREFETCH
    const T v = p[i];
    rec<XPL_ACC_R>(i);
    return v;
#else
    rec<XPL_ACC_R>(i);
    return p[i];
#endif
  }
  __device__ __forceinline__ T& write(unsigned long long i) const { rec<XPL_ACC_W>(i); return p[i]; }
  __device__ __forceinline__ T& rw(unsigned long long i) const {
#ifndef XPL_OFF
    xpld_prefetch(p + i);
#endif
    rec<XPL_ACC_RW>(i);
    return p[i];
  }
};

/* A D-deep hook pipeline for an instrumented thread's straight-line code
 * (one object per thread, e.g. a local at the top of the kernel):
 * p.read(x) / p.write(x) / p.rw(x) record the same bits as xpl_read / _write /
 * _rw, but a hook's commit (test before set, grouping, atomicOr) runs D hooks
 * later, or when the object dies: its shadow load is in flight
 * while the thread goes on to its next access, instead of stalling it (a GPU
 * warp issues in order, so with immediate commits every hook costs one full
 * memory latency; kernels with a dozen hooks per thread are latency-bound by
 * them).  Record order inside an epoch does not matter (D5), so deferring the
 * commit within the kernel changes nothing.  Accesses that are not local and
 * inside one shadow u32 take the general path at once.  Commits group lanes by
 * shadow u32 with per-lane kinds (a lane's pending access may come from another
 * call site than its neighbours' after divergence).  Warp-synchronous like every
 * hook: all lanes that made a hook must reach the next one (or the object's end)
 * together with the lanes of their warp that are active there. */
template <unsigned D = 4>
struct xpl_pipe {
#ifndef XPL_OFF
  /* pending, newest first: shadow u32, its value (load in flight), byte lanes, kind (0 = none) */
  unsigned pq[D], pcur[D], pbm[D], pk[D];
#endif
  __device__ __forceinline__ xpl_pipe() {
#ifndef XPL_OFF
#pragma unroll
    for (unsigned j = 0; j < D; ++j) pq[j] = pcur[j] = pbm[j] = pk[j] = 0u;
#endif
  }
  xpl_pipe(const xpl_pipe&) = delete;
  xpl_pipe& operator=(const xpl_pipe&) = delete;
  __device__ __forceinline__ ~xpl_pipe() {
#ifndef XPL_OFF
#pragma unroll
    for (unsigned j = D; j-- > 0;) commit(j);
#endif
  }
#ifndef XPL_OFF
  __device__ __forceinline__ void commit(unsigned j) {
    const unsigned act = __activemask();
    const unsigned m = xpld_bits(pcur[j], pbm[j], pk[j]);
    const bool need = pk[j] != 0 && (pcur[j] & m) != m;
    const unsigned needers = __ballot_sync(act, need);
    if (need) xpld_commit<0, false, true>(needers, pq[j], pcur[j], pbm[j], pk[j]);
    pk[j] = 0;
  }
#endif
  template <unsigned K>
  __device__ __forceinline__ void hook(const void* x, unsigned size) {
#ifndef XPL_OFF
    const unsigned long long a = (unsigned long long)x;
    ulonglong2 be, ow;
    unsigned long long g0 = 1, g1 = 0;
    unsigned owner = xpl_dctx.rank;
    if (xpld_find(a, be, ow) && size > 0) xpld_words(a, size, be.x, be.y, ow.x, g0, g1, owner);
    const unsigned act = __activemask();
    const bool hit = g0 <= g1;
    const bool fast = !hit || (owner == xpl_dctx.rank && (g0 ^ g1) < 4ull);
    if (__ballot_sync(act, !fast)) { /* uniform: the general path, now */
      xpld_record_words<K>(g0, g1, owner, K);
      return;
    }
    const unsigned q = (unsigned)(g0 >> 2);
    const unsigned bm = hit ? (0xFFFFFFFFu >> (24 - 8 * (unsigned)(g1 - g0))) << (8 * ((unsigned)g0 & 3u)) : 0u;
    const unsigned cur = hit ? xpl_dctx.pool[q] : 0u; /* in flight until this entry is the oldest */
    commit(D - 1);
#pragma unroll
    for (unsigned j = D - 1; j > 0; --j) {
      pq[j] = pq[j - 1];
      pcur[j] = pcur[j - 1];
      pbm[j] = pbm[j - 1];
      pk[j] = pk[j - 1];
    }
    pq[0] = q;
    pcur[0] = cur;
    pbm[0] = bm;
    pk[0] = hit ? K : 0u;
#endif
  }
  template <class T>
  __device__ __forceinline__ const T& read(const T& x) {
    hook<XPL_ACC_R>(&x, sizeof(T));
    return x;
  }
  template <class T>
  __device__ __forceinline__ T& write(T& x) {
    hook<XPL_ACC_W>(&x, sizeof(T));
    return x;
  }
  template <class T>
  __device__ __forceinline__ T& rw(T& x) {
    hook<XPL_ACC_RW>(&x, sizeof(T));
    return x;
  }
};

/* Generic form: acc may differ from lane to lane. */
static __device__ __forceinline__ void xpl_dev_record(const void* p, unsigned size, unsigned acc) {
  xpl_dev_record_k<0>(p, size, acc);
}

/* traceR / traceW / traceRW: take the element, return it (Table I). */
template <class T>
static __device__ __forceinline__ const T& xpl_read(const T& x) {
  xpl_dev_record_k<XPL_ACC_R>(&x, sizeof(T), XPL_ACC_R);
  return x;
}
template <class T>
static __device__ __forceinline__ T& xpl_write(T& x) {
  xpl_dev_record_k<XPL_ACC_W>(&x, sizeof(T), XPL_ACC_W);
  return x;
}
template <class T>
static __device__ __forceinline__ T& xpl_rw(T& x) {
  xpl_dev_record_k<XPL_ACC_RW>(&x, sizeof(T), XPL_ACC_RW);
  return x;
}
/* traceR for latency-bound kernels: xpl_read_lat(x) returns a proxy.  The hook's
 * lookup and shadow load are issued when the proxy is made; the proxy converts
 * to `const T&` (the user's own load of x follows, with the shadow load still in
 * flight); its destructor -- at the end of the full expression, e.g. after
 * `v = xpl_read_lat(a[i]);` -- tests and commits the record exactly as xpl_read
 * does.  So the shadow load's latency overlaps the user's load instead of
 * adding to it.  All lanes that made the proxy must reach its destructor (it
 * is warp-synchronous, like every hook); accesses of more than one word commit
 * at once. */
template <class T>
struct xpl_read_proxy {
  const T& x;
  unsigned q, cur, bytes, active, singles;
  bool hit;
  __device__ __forceinline__ explicit xpl_read_proxy(const T& v) : x(v) {
#ifndef XPL_OFF
    const unsigned long long a = (unsigned long long)&v;
    ulonglong2 be, ow;
    unsigned long long g0 = 1, g1 = 0;
    unsigned owner = 0;
    const bool h = xpld_find(a, be, ow);
    if (h) xpld_words(a, sizeof(T), be.x, be.y, ow.x, g0, g1, owner);
    if (__any_sync(__activemask(), owner != xpl_dctx.rank && h)) {  /* sharded: remote words now */
      if (owner != xpl_dctx.rank && h) {
        xpld_remote<XPL_ACC_R>(owner, g0, g1, XPL_ACC_R);
        g0 = 1;
        g1 = 0;
      }
    }
    active = __activemask();
    const bool single = g0 >= g1;
    singles = __ballot_sync(active, single);
    hit = single && g0 == g1;
    q = (unsigned)(g0 >> 2);
    bytes = 0xFFu << (8 * (unsigned)(g0 & 3));
    cur = hit ? xpl_dctx.pool[q] : 0u;  /* issued now, consumed in the destructor */
    if (singles != active) xpl_dev_apply<XPL_ACC_R>(single ? 1ull : g0, single ? 0ull : g1, XPL_ACC_R);
#endif
  }
  __device__ __forceinline__ operator const T&() const { return x; }
  __device__ __forceinline__ ~xpl_read_proxy() {
#ifndef XPL_OFF
    if (singles & (1u << xpld_lane())) {
      const unsigned m = xpld_bits(cur, bytes, XPL_ACC_R);
      const bool need = hit && (cur & m) != m;
      const unsigned needers = __ballot_sync(singles, need);
      if (need) xpld_commit<XPL_ACC_R, true>(needers, q, cur, bytes, XPL_ACC_R);
    }
#endif
  }
  xpl_read_proxy(const xpl_read_proxy&) = delete;
  xpl_read_proxy& operator=(const xpl_read_proxy&) = delete;
};
template <class T>
static __device__ __forceinline__ xpl_read_proxy<T> xpl_read_lat(const T& x) {
  return xpl_read_proxy<T>(x);
}

/* traceW for latency-bound kernels (few threads, a few writes each, e.g. one
 * small block per tile of a wavefront): the same record, but the write's chunk
 * mark is stored without first testing it.  Do not use it where many warps
 * write one 2M-word region per epoch (every commit would store the same
 * super-chunk byte). */
template <class T>
static __device__ __forceinline__ T& xpl_write_lat(T& x) {
  xpl_dev_record_k<XPL_ACC_W, false>(&x, sizeof(T), XPL_ACC_W);
  return x;
}

/* Device-side epoch boundary (the paper's per-iteration
 * view of a wavefront, Fig. 8).  Inside ONE cooperative launch
 * (cudaLaunchCooperativeKernel), every thread of the grid calls it at the same
 * point: it closes the epoch the kernel's accesses so far belong to and opens a
 * new one, exactly like xpl_kernel_end + xpl_kernel_begin between two launches
 * (trace: KE KB).  Steps: grid barrier (all hooks of the segment have landed),
 * the fold of that segment's pending writes (P -> L, D5) spread over the warps
 * of the grid (a warp per marked super-chunk, a lane per marked chunk), grid barrier (reads of the next segment see the new L).  The
 * barrier's release/acquire at gpu scope orders the plain shadow loads of the
 * hooks after the fold.  Must not be called from a non-cooperative launch (the
 * grid barrier would deadlock or fault); a no-op under -DXPL_OFF except for the
 * barrier itself, which keeps the twin's control flow.  The fold stores whole
 * shadow vectors, so nothing else may record into the pool while it runs: the
 * epoch holding the launch must have a single stream and no D2D / memset
 * shadow work of the runtime (xpl_record_copy inside the epoch); the epoch
 * close checks this and the next xpl_sync / xpl_diagnose returns XPL_ERR_STATE
 * if it was violated. */
static __device__ __forceinline__ void xpl_grid_epoch() {
  cooperative_groups::grid_group g = cooperative_groups::this_grid();
  g.sync();
#ifndef XPL_OFF
  /* tell the epoch close a split ran: an epoch with a split must be one stream
   * without runtime range work of its own (else its close reports XPL_ERR_STATE) */
  if (g.thread_rank() == 0) xpl_dctx.flags[0] = 1u;
  const unsigned lane = xpld_lane();
  const unsigned long long nthreads = (unsigned long long)gridDim.x * gridDim.y * gridDim.z *
                                      blockDim.x * blockDim.y * blockDim.z;
  const unsigned long long nwarps = (nthreads + 31) / 32;
  const unsigned long long gw = g.thread_rank() / 32;
  const unsigned long long n_super = __ldcg(xpl_dctx.n_super);
  for (unsigned long long sc = gw; sc < n_super; sc += nwarps) {
    if (!__ldcg(xpl_dctx.smap + sc)) continue; /* (uniform over the warp) */
    for (unsigned c0 = 0; c0 < 128; c0 += 32) {
      const unsigned long long ch = sc * 128 + c0 + lane;
      if (__ldcg(xpl_dctx.cmap + ch)) {
        /* lane-per-chunk: the lane folds its own 128-word chunk (32 u32, one
         * 128 B line, 8 x 16 B loads in flight together), so a round of 32
         * chunks costs one round trip.  No hook runs between the two grid
         * barriers, so whole-vector stores race with nothing. */
        uint4* w = reinterpret_cast<uint4*>(xpl_dctx.pool + ch * 32);
        uint4 v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) v[k] = __ldcg(w + k);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const unsigned any = (v[k].x | v[k].y | v[k].z | v[k].w) & XPLD_P4;
          if (any) {
            v[k].x = (v[k].x & ~XPLD_P4) | ((v[k].x & XPLD_P4) >> 1); /* P -> L */
            v[k].y = (v[k].y & ~XPLD_P4) | ((v[k].y & XPLD_P4) >> 1);
            v[k].z = (v[k].z & ~XPLD_P4) | ((v[k].z & XPLD_P4) >> 1);
            v[k].w = (v[k].w & ~XPLD_P4) | ((v[k].w & XPLD_P4) >> 1);
            w[k] = v[k];
          }
        }
        xpl_dctx.cmap[ch] = 0;
      }
    }
    if (lane == 0) xpl_dctx.smap[sc] = 0;
  }
  g.sync();
#endif
}

#endif /* __CUDACC__ */
#endif /* XPL_DEVICE_CUH */
