// kernels.cu -- sm_100a kernels of the XPlacer runtime (everything but the
// inlined device hooks, which live in include/xpl_device.cuh).
//
//   fold          epoch close: pending GPU writes become "last writer = GPU"
//                 (snapshot semantics D5), O(chunks written)
//   merge_*       ordered host-record batches (host tracer), 3 passes
//   range_apply   transfers and other long ranges, 16 records / vector
//   diag_*        tracePrint: counts, density blocks, transfer runs,
//                 fused reset, one pass over the shadow at HBM speed
//
// Record byte: bit0 L, bit1 P, bit2 wC, bit3 wG, bit4 rCC, bit5 rGC, bit6 rCG,
// bit7 rGG.
#include <cuda_runtime.h>
#include <stdint.h>

#include "xpl_internal.h"

namespace xpl {

namespace {

constexpr uint32_t kL4 = 0x01010101u;
constexpr uint32_t kP4 = 0x02020202u;

// ---------------------------------------------------------------------------
// fold (epoch close): every 128-word chunk a GPU write marked (cmap) gets
// P -> L=1 and P cleared (snapshot semantics D5).  A one-wave grid of
// W warps; warp w owns the super-chunks (16K words) w, w + W, w + 2W, ... below
// the pool's high-water mark: it reads 32 of its super bytes at once (one per
// lane), and for each marked one folds its marked chunks lane-per-chunk (lane
// l checks chunks l, l+32, l+64, l+96; a marked chunk = one 128 B line, eight
// 16 B loads in flight together).  Spreading the super-chunks over all warps
// keeps the chain per warp short whatever the epoch's write pattern: an epoch
// that touched one word in every super-chunk (a Smith-Waterman anti-diagonal)
// costs every warp ~2 supers, not one CTA a long list.  No global list, no
// atomics; cost O(super map + chunks written).  Launched with programmatic
// stream serialization when it directly follows the epoch's kernels on their
// stream: griddepcontrol.wait holds it until they are complete, while its own
// launch overlaps their tail.
constexpr int kFoldThreads = 256;
#ifndef XPL_FOLD_CTAS
#define XPL_FOLD_CTAS (148 * 3)  // grid cap: one wave at 3 CTAs per SM (the register budget below)
#endif

// P -> L over the 128-word chunks ch0 (if m0) and ch1 (if m1) of one lane: all
// sixteen 16 B loads issued before the first store (one round trip for both).
__device__ __forceinline__ void fold_two(uint32_t* pool, uint64_t ch0, bool m0, uint64_t ch1, bool m1) {
  uint4* w0 = reinterpret_cast<uint4*>(pool + ch0 * 32);
  uint4* w1 = reinterpret_cast<uint4*>(pool + ch1 * 32);
  uint4 v[16];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    v[k] = m0 ? w0[k] : make_uint4(0, 0, 0, 0);
    v[8 + k] = m1 ? w1[k] : make_uint4(0, 0, 0, 0);
  }
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    if ((v[k].x | v[k].y | v[k].z | v[k].w) & kP4) {
      v[k].x = (v[k].x & ~kP4) | ((v[k].x & kP4) >> 1);
      v[k].y = (v[k].y & ~kP4) | ((v[k].y & kP4) >> 1);
      v[k].z = (v[k].z & ~kP4) | ((v[k].z & kP4) >> 1);
      v[k].w = (v[k].w & ~kP4) | ((v[k].w & kP4) >> 1);
      (k < 8 ? w0 : w1)[k & 7] = v[k];
    }
  }
}

__device__ __forceinline__ void fold_body(uint32_t* __restrict__ pool, uint8_t* __restrict__ cmap,
                                          uint8_t* __restrict__ smap, uint64_t n_super,
                                          unsigned long long* stats) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t W = (uint64_t)gridDim.x * (kFoldThreads / 32);
  const uint64_t w = (uint64_t)blockIdx.x * (kFoldThreads / 32) + (threadIdx.x >> 5);
  uint32_t folded = 0;
  for (uint64_t k0 = 0; w + k0 * W < n_super; k0 += 32) {
    const uint64_t sc = w + (k0 + lane) * W;
    const bool marked = sc < n_super && smap[sc] != 0;
    uint32_t ms = __ballot_sync(0xFFFFFFFFu, marked);
    if (!ms) continue;
    // Sparse super-chunks (<= 2 marked chunks: e.g. an anti-diagonal touches one
    // word per row) are folded lane-per-super-chunk, all of the warp's at once:
    // one 128 B read of the super's chunk bytes, then its one or two chunks.
    bool dense = false;
    if (marked) {
      uint4 cm[8];
      const uint4* cp = reinterpret_cast<const uint4*>(cmap + sc * 128);
#pragma unroll
      for (int k = 0; k < 8; ++k) cm[k] = cp[k];
      uint32_t cnt = 0;  // (chunk bytes are 0 or 1)
#pragma unroll
      for (int k = 0; k < 8; ++k) cnt += __popc(cm[k].x) + __popc(cm[k].y) + __popc(cm[k].z) + __popc(cm[k].w);
      dense = cnt > 2;
      if (!dense) {
        int ca = -1, cb = -1;
#pragma unroll
        for (int k = 0; k < 32; ++k) {
          const uint32_t v = k % 4 == 0 ? cm[k / 4].x : k % 4 == 1 ? cm[k / 4].y : k % 4 == 2 ? cm[k / 4].z : cm[k / 4].w;
          if (v) {
            const int b0 = 4 * k + (__ffs(v) - 1) / 8;
            const uint32_t rest = v & ~(0xFFu << (8 * ((__ffs(v) - 1) / 8)));
            if (ca < 0) {
              ca = b0;
              if (rest) cb = 4 * k + (__ffs(rest) - 1) / 8;
            } else if (cb < 0) {
              cb = b0;
            }
          }
        }
        if (ca >= 0) {
          fold_two(pool, sc * 128 + ca, true, sc * 128 + (cb >= 0 ? cb : ca), cb >= 0);
          cmap[sc * 128 + ca] = 0;
          if (cb >= 0) cmap[sc * 128 + cb] = 0;
        }
        folded += cnt;
        smap[sc] = 0;
      }
    }
    ms = __ballot_sync(0xFFFFFFFFu, marked && dense);
    while (ms) {
      const uint32_t j = __ffs(ms) - 1;
      ms &= ms - 1;
      const uint64_t s = w + (k0 + j) * W;
      const uint64_t c0 = s * 128 + lane;
      const bool m0 = cmap[c0], m1 = cmap[c0 + 32], m2 = cmap[c0 + 64], m3 = cmap[c0 + 96];
      if (m0 || m1) fold_two(pool, c0, m0, c0 + 32, m1);
      if (m2 || m3) fold_two(pool, c0 + 64, m2, c0 + 96, m3);
      folded += m0 + m1 + m2 + m3;
      if (m0) cmap[c0] = 0;
      if (m1) cmap[c0 + 32] = 0;
      if (m2) cmap[c0 + 64] = 0;
      if (m3) cmap[c0 + 96] = 0;
      if (lane == 0) smap[s] = 0;
    }
  }
  folded = __reduce_add_sync(0xFFFFFFFFu, folded);
  if (lane == 0 && folded) atomicAdd(stats + 3, (unsigned long long)folded);
}

__global__ void __launch_bounds__(kFoldThreads, 3) fold_kernel(uint32_t* __restrict__ pool,
                                                            uint8_t* __restrict__ cmap,
                                                            uint8_t* __restrict__ smap,
                                                            uint64_t n_super,
                                                            unsigned long long* stats,
                                                            uint32_t* flags, int strict, int force) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (blockIdx.x == 0 && threadIdx.x == 0) {  // a device-side split in an epoch that forbids it
    if (strict && flags[0]) flags[1] = 1u;
    flags[0] = 0u;
  }
  // flags[2]: some pending write was marked since the last close (hooks, range
  // kernel); without one the close has nothing to fold.  The last CTA to finish
  // clears it (flags[3] counts the finished CTAs).  (A sharded epoch's remote
  // writers mark another rank's maps: there flags[2] is not used, force = 1.)
  const bool work = force || *reinterpret_cast<volatile uint32_t*>(flags + 2) != 0;
  __syncthreads();  // (every thread read the flag before any CTA can clear it below)
  if (work) fold_body(pool, cmap, smap, n_super, stats);
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(flags + 3, 1u) == gridDim.x - 1) {
      flags[2] = 0u;
      flags[3] = 0u;
    }
  }
}

// ---------------------------------------------------------------------------
// Host merge.  A batch of host records is one ordered stream (D7b).  Per word:
// a read before the first write of the batch sees the batch-start last writer;
// a read after it sees the CPU; any write sets wC and makes the CPU the last
// writer.  Pass 1 finds each word's first writing record
// (atomicMin of the record index), pass 2 sets read/write bits, pass 3 clears L
// of written words and resets the scratch.  The scratch covers only the pool
// words [fw0, fw0 + span) the batch touches (fw[w - fw0]).

__device__ __forceinline__ void merge_firstw_rec(const uint64_t* __restrict__ recs, uint32_t i,
                                                 uint32_t* __restrict__ fw, uint64_t fw0) {
  const uint64_t r = recs[i];
  if (!(rec_acc(r) & XPL_ACC_W)) return;
  const uint64_t g0 = rec_g0(r), nw = rec_nw(r);
  for (uint64_t w = g0; w < g0 + nw; ++w) atomicMin(fw + (w - fw0), i);
}

// Record i's bits on shadow u32 q (one of the u32s its words [g0, g1] cover).
__device__ __forceinline__ void merge_apply_q(uint32_t acc, uint64_t g0, uint64_t g1, uint32_t i, uint64_t q,
                                              const uint32_t* __restrict__ fw, uint64_t fw0, uint32_t* pool) {
  const uint32_t cur = pool[q];  // L bits do not change during this pass
  uint32_t m = 0;
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {
    const uint64_t w = q * 4 + k;
    if (w < g0 || w > g1) continue;
    uint32_t b = 0;
    if (acc & XPL_ACC_R) {
      const bool before = (fw == nullptr) || i <= fw[w - fw0];
      b = before ? (((cur >> (8 * k)) & 1u) ? kRGC : kRCC) : kRCC;
    }
    if (acc & XPL_ACC_W) b |= kWC;
    m |= b << (8 * k);
  }
  if ((cur & m) != m) atomicOr(pool + q, m);
}

__device__ __forceinline__ void merge_apply_rec(const uint64_t* __restrict__ recs, uint32_t i,
                                                const uint32_t* __restrict__ fw, uint64_t fw0, uint32_t* pool) {
  const uint64_t r = recs[i];
  const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
  for (uint64_t q = g0 >> 2; q <= (g1 >> 2); ++q) merge_apply_q(rec_acc(r), g0, g1, i, q, fw, fw0, pool);
}

// A written record's u32 q: clear L of its words (the CPU is now the last writer).
__device__ __forceinline__ void merge_clear_q(uint64_t g0, uint64_t g1, uint64_t q, uint32_t* pool) {
  uint32_t lm = 0;
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {
    const uint64_t w = q * 4 + k;
    if (w >= g0 && w <= g1) lm |= kL << (8 * k);
  }
  if (pool[q] & lm) atomicAnd(pool + q, ~lm);
}

__device__ __forceinline__ void merge_clear_rec(const uint64_t* __restrict__ recs, uint32_t i,
                                                uint32_t* __restrict__ fw, uint64_t fw0, uint32_t* pool) {
  const uint64_t r = recs[i];
  if (!(rec_acc(r) & XPL_ACC_W)) return;
  const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
  for (uint64_t q = g0 >> 2; q <= (g1 >> 2); ++q) merge_clear_q(g0, g1, q, pool);
  if (fw)
    for (uint64_t w = g0; w <= g1; ++w) fw[w - fw0] = 0xFFFFFFFFu;
}

__global__ void merge_firstw_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                    uint32_t* __restrict__ fw, uint64_t fw0) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    merge_firstw_rec(recs, i, fw, fw0);
}

__global__ void merge_apply_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                   const uint32_t* __restrict__ fw, uint64_t fw0, uint32_t* pool) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    merge_apply_rec(recs, i, fw, fw0, pool);
}

__global__ void merge_clear_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                   uint32_t* __restrict__ fw, uint64_t fw0, uint32_t* pool) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    merge_clear_rec(recs, i, fw, fw0, pool);
}

// A small batch (a host segment of a few thousand records, the common case
// between epochs): the three passes in one CTA, separated by CTA barriers
// instead of kernel boundaries -- one launch instead of three.  The apply and
// clear passes are spread over (record, shadow u32) items, not records: a
// record of up to kPieceWords words covers up to 65 u32s, and one thread
// walking them would chain as many dependent L2 round trips.  The items'
// offsets are an exclusive scan of the records' u32 counts in shared memory;
// an item finds its record by binary search.
constexpr uint32_t kMergeSmall = 8192;
constexpr uint32_t kMergeThreads = 1024;
constexpr uint32_t kMergePer = kMergeSmall / kMergeThreads;
__global__ void __launch_bounds__(kMergeThreads) merge_small_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                                                    bool has_r, bool has_w,
                                                                    uint32_t* __restrict__ fw, uint64_t fw0,
                                                                    uint32_t* pool) {
  __shared__ uint32_t s_off[kMergeSmall + 1];  // exclusive scan of u32 counts; s_off[n] = items
  __shared__ uint32_t s_warp[kMergeThreads / 32];
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const bool both = has_r && has_w;
  // scan: thread tid owns records [tid * kMergePer, +kMergePer)
  uint32_t cnt[kMergePer], sum = 0;
#pragma unroll
  for (uint32_t k = 0; k < kMergePer; ++k) {
    const uint32_t i = tid * kMergePer + k;
    cnt[k] = 0;
    if (i < n) {
      const uint64_t r = recs[i];
      const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
      cnt[k] = (uint32_t)((g1 >> 2) - (g0 >> 2) + 1);
      if (both) merge_firstw_rec(recs, i, fw, fw0);
    }
    sum += cnt[k];
  }
  uint32_t incl = sum;
#pragma unroll
  for (uint32_t o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += v;
  }
  if (lane == 31) s_warp[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    uint32_t w = s_warp[lane], wi = w;
#pragma unroll
    for (uint32_t o = 1; o < 32; o <<= 1) {
      const uint32_t v = __shfl_up_sync(0xFFFFFFFFu, wi, o);
      if (lane >= o) wi += v;
    }
    s_warp[lane] = wi - w;  // exclusive over warps
  }
  __syncthreads();
  uint32_t off = s_warp[wid] + incl - sum;
#pragma unroll
  for (uint32_t k = 0; k < kMergePer; ++k) {
    const uint32_t i = tid * kMergePer + k;
    if (i <= n) s_off[i] = off;  // (i == n: the total)
    off += cnt[k];
  }
  if (tid == kMergeThreads - 1) s_off[n] = off;  // (the total; n == kMergeSmall has no owner above)
  __syncthreads();  // (also orders pass 1's first writers before pass 2)
  const uint32_t items = s_off[n];
  auto rec_of = [&](uint32_t x) {  // the last record with s_off <= x
    uint32_t lo = 0, hi = n;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (s_off[mid] <= x) lo = mid;
      else hi = mid;
    }
    return lo;
  };
  for (uint32_t x = tid; x < items; x += kMergeThreads) {
    const uint32_t i = rec_of(x);
    const uint64_t r = recs[i];
    const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
    merge_apply_q(rec_acc(r), g0, g1, i, (g0 >> 2) + (x - s_off[i]), both ? fw : nullptr, fw0, pool);
  }
  if (!has_w) return;
  __syncthreads();
  for (uint32_t x = tid; x < items; x += kMergeThreads) {
    const uint32_t i = rec_of(x);
    const uint64_t r = recs[i];
    if (!(rec_acc(r) & XPL_ACC_W)) continue;
    const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
    merge_clear_q(g0, g1, (g0 >> 2) + (x - s_off[i]), pool);
  }
  if (both) {  // the first-writer scratch back to all-ones
    for (uint32_t i = tid; i < n; i += kMergeThreads) {
      const uint64_t r = recs[i];
      if (!(rec_acc(r) & XPL_ACC_W)) continue;
      const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
      for (uint64_t w = g0; w <= g1; ++w) fw[w - fw0] = 0xFFFFFFFFu;
    }
  }
}

// ---------------------------------------------------------------------------
// range_apply: a list of ranges, 16-word vectors spread over the grid.
// CPU side: one RMW per word -- R sets rGC/rCC by L, W sets wC and clears L
// (H2D = W, D2H = R).  Ranges of one launch are pairwise disjoint
// (the runtime guarantees it), so a u32 wholly inside a range is owned by one
// thread; u32s shared with a neighbour range use a CAS loop.
// GPU side (D2D, memset; D7): the hooks' rule with atomics, ranges may overlap.
__device__ __forceinline__ uint32_t cpu_range_op(uint32_t v, uint32_t bm, uint32_t acc) {
  if (acc & XPL_ACC_R) {
    const uint32_t lb = v & kL4;
    v |= ((lb << 5) | ((~lb & kL4) << 4)) & bm;
  }
  if (acc & XPL_ACC_W) v = (v | (0x04040404u & bm)) & ~(kL4 & bm);
  return v;
}

__global__ void __launch_bounds__(256) range_kernel(const RangeDesc* __restrict__ rd, uint32_t nr,
                                                    uint64_t nvec, uint32_t* pool,
                                                    uint8_t* cmap, uint8_t* smap, uint32_t* flags) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nvec;
       v += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t lo = 0, hi = nr;  // last range with vbase <= v
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (rd[mid].vbase <= v) lo = mid;
      else hi = mid;
    }
    const RangeDesc r = rd[lo];
    const uint64_t g1 = r.g0 + r.nw - 1;
    const uint64_t vi = (r.g0 >> 4) + (v - r.vbase);
    uint4* p4 = reinterpret_cast<uint4*>(pool) + vi;
    const uint4 val = *p4;
    const uint32_t in[4] = {val.x, val.y, val.z, val.w};
    uint32_t out[4];
    uint32_t bms[4];
    bool all_full = true;
#pragma unroll
    for (uint32_t c = 0; c < 4; ++c) {
      uint32_t bm = 0;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint64_t w = vi * 16 + c * 4 + k;
        if (w >= r.g0 && w <= g1) bm |= 0xFFu << (8 * k);
      }
      bms[c] = bm;
      all_full = all_full && bm == 0xFFFFFFFFu;
    }
    if (r.side == 0) {
#pragma unroll
      for (uint32_t c = 0; c < 4; ++c) out[c] = cpu_range_op(in[c], bms[c], r.acc);
      if (all_full) {
        if (out[0] != in[0] || out[1] != in[1] || out[2] != in[2] || out[3] != in[3])
          *p4 = make_uint4(out[0], out[1], out[2], out[3]);
      } else {
        for (uint32_t c = 0; c < 4; ++c) {
          if (!bms[c]) continue;
          uint32_t* p = pool + vi * 4 + c;
          if (bms[c] == 0xFFFFFFFFu) {
            if (out[c] != in[c]) *p = out[c];
          } else {
            uint32_t old = *p, assumed;
            do {
              assumed = old;
              const uint32_t nv = cpu_range_op(assumed, bms[c], r.acc);
              if (nv == assumed) break;
              old = atomicCAS(p, assumed, nv);
            } while (old != assumed);
          }
        }
      }
    } else {
#pragma unroll
      for (uint32_t c = 0; c < 4; ++c) {
        if (!bms[c]) continue;
        const uint32_t lb = in[c] & kL4;
        uint32_t m = 0;
        if (r.acc & XPL_ACC_R) m |= ((lb << 7) | ((~lb & kL4) << 6)) & bms[c];
        if (r.acc & XPL_ACC_W) m |= (0x08080808u | ((~lb & kL4) << 1)) & bms[c];  // P only where L = CPU
        if ((in[c] & m) == m) continue;
        const uint32_t q = (uint32_t)(vi * 4 + c);
        atomicOr(pool + q, m);
        if (m & kP4) {
          if (!cmap[q >> 5]) cmap[q >> 5] = 1;
          if (!smap[q >> 12]) {
            smap[q >> 12] = 1;
            flags[2] = 1u;
          }
        }
      }
    }
  }
}

// ---------------------------------------------------------------------------
// Diagnose.

// Run summary combine: the monoid of maximal runs of ones.  pre/suf = leading /
// trailing ones; cnt/sum = complete runs (bounded by zeros on both sides) of
// length >= min_run.  "full" = pre == len.
template <class S>
__device__ __forceinline__ S rs_combine(const S& a, const S& b, uint64_t min_run) {
  S r;
  const bool af = a.pre == a.len, bf = b.pre == b.len;
  r.len = a.len + b.len;
  r.pre = af ? a.len + b.pre : a.pre;
  r.suf = bf ? b.len + a.suf : b.suf;
  r.cnt = a.cnt + b.cnt;
  r.sum = a.sum + b.sum;
  if (!af && !bf) {
    const uint64_t mid = (uint64_t)a.suf + b.pre;
    if (mid > 0 && mid >= min_run) {
      r.cnt += 1;
      r.sum += mid;
    }
  }
  return r;
}

struct RunSum64 {
  uint64_t len, pre, suf, cnt, sum;
};

__device__ __forceinline__ uint32_t pack4(uint32_t t) {  // bit0 of each byte -> 4 bits
  return (t | (t >> 7) | (t >> 14) | (t >> 21)) & 0xFu;
}

// Warp summary of one predicate over the warp's 512 consecutive words; lane l
// owns words [16l, 16l+16) as the 16-bit mask m.  Returns a warp-uniform RunSum.
__device__ __noinline__ RunSum warp_runs(uint32_t m, uint32_t lane, uint32_t min_run) {
  const bool full = m == 0xFFFFu;
  const uint32_t pre = __ffs(~m) - 1;  // 16 when full
  const uint32_t x = ~m & 0xFFFFu;
  const uint32_t suf = x ? __clz(x) - 16 : 16;
  uint32_t cnt = 0, sum = 0;
  if (min_run <= 14 && !full) {  // runs strictly inside the lane
    uint32_t y = m & ~((1u << pre) - 1u) & ((1u << (16 - suf)) - 1u);
    while (y) {
      const uint32_t s = __ffs(y) - 1;
      const uint32_t l = __ffs(~(y >> s)) - 1;
      if (l >= min_run) {
        cnt += 1;
        sum += l;
      }
      y &= ~(((1u << l) - 1u) << s);
    }
  }
  const uint32_t F = __ballot_sync(0xFFFFFFFFu, full);
  uint32_t suf_prev = __shfl_up_sync(0xFFFFFFFFu, suf, 1);
  const uint32_t after = lane == 31 ? 0u : (~F & (0xFFFFFFFFu << (lane + 1)));
  const uint32_t b = after ? (uint32_t)(__ffs(after) - 1) : 32u;
  const uint32_t pre_b = __shfl_sync(0xFFFFFFFFu, pre, b & 31);
  if (!full) {
    if (suf > 0 && b < 32) {
      const uint32_t L = suf + 16 * (b - lane - 1) + pre_b;
      if (L >= min_run) { cnt += 1; sum += L; }
    }
    if (pre > 0 && lane > 0 && suf_prev == 0 && pre >= min_run) { cnt += 1; sum += pre; }
  } else if (lane > 0 && suf_prev == 0 && b < 32) {
    const uint32_t L = 16 * (b - lane) + pre_b;
    if (L >= min_run) { cnt += 1; sum += L; }
  }
  RunSum r;
  r.len = 512;
  r.cnt = __reduce_add_sync(0xFFFFFFFFu, cnt);
  r.sum = __reduce_add_sync(0xFFFFFFFFu, sum);
  if (F == 0xFFFFFFFFu) {
    r.pre = r.suf = 512;
  } else {
    const uint32_t f0 = __ffs(~F) - 1;
    const uint32_t l0 = 31 - __clz(~F);
    r.pre = 16 * f0 + __shfl_sync(0xFFFFFFFFu, pre, f0);
    r.suf = 16 * (31 - l0) + __shfl_sync(0xFFFFFFFFu, suf, l0);
  }
  return r;
}

// Harley-Seal style vertical counter: bit j of plane k is bit k of the number of
// ones seen at bit position j.  Up to 4 x kDiagIters = 128 u32 per lane per tile
// -> 8 planes (counts up to 255).
struct VCount {
  uint32_t p0 = 0, p1 = 0, p2 = 0, p3 = 0, p4 = 0, p5 = 0, p6 = 0, p7 = 0;
  __device__ __forceinline__ void add4(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    // two full adders into (p0, carries), then carries into p1, ripple up
    uint32_t u = p0 ^ a ^ b;
    uint32_t c1 = (p0 & a) | (p0 & b) | (a & b);
    p0 = u;
    u = p0 ^ c ^ d;
    uint32_t c2 = (p0 & c) | (p0 & d) | (c & d);
    p0 = u;
    uint32_t s = p1 ^ c1 ^ c2;
    uint32_t c4 = (p1 & c1) | (p1 & c2) | (c1 & c2);
    p1 = s;
    uint32_t t = p2 & c4; p2 ^= c4;
    uint32_t t2 = p3 & t; p3 ^= t;
    uint32_t t3 = p4 & t2; p4 ^= t2;
    uint32_t t4 = p5 & t3; p5 ^= t3;
    uint32_t t5 = p6 & t4; p6 ^= t4;
    p7 ^= t5;
  }
  __device__ __forceinline__ uint32_t count(uint32_t mask) const {
    return __popc(p0 & mask) + 2 * __popc(p1 & mask) + 4 * __popc(p2 & mask) +
           8 * __popc(p3 & mask) + 16 * __popc(p4 & mask) + 32 * __popc(p5 & mask) +
           64 * __popc(p6 & mask) + 128 * __popc(p7 & mask);
  }
};
static_assert(4 * kDiagIters <= 255, "vertical counter planes");

// Per-byte flags, 0x80 in each byte where the predicate holds.
__device__ __forceinline__ uint32_t derived_flags(uint32_t x) {
  const uint32_t cpu = ((x & 0x34343434u) + 0x7F7F7F7Fu) & 0x80808080u;  // wC|rCC|rGC
  const uint32_t gpu = (((x & 0x48484848u) + 0x7F7F7F7Fu) | x) & 0x80808080u;  // wG|rCG|rGG
  const uint32_t wr = ((x & 0x0C0C0C0Cu) + 0x7F7F7F7Fu) & 0x80808080u;  // wC|wG
  const uint32_t any = cpu | gpu;
  const uint32_t alt = cpu & gpu & wr;
  return any | (gpu >> 1) | (alt >> 2);  // bit7 any, bit6 gpu, bit5 alternating
}

// Run summary updates of a warp's running summary A by one 512-word step that
// is all zeros / all ones (the common cases; u32 arithmetic inside a tile).
__device__ __forceinline__ void rs_append_zero(RunSum& a, uint32_t min_run, uint32_t n = 512) {
  if (a.pre != a.len && a.suf >= min_run && a.suf > 0) {  // an inner run ends here
    a.cnt += 1;
    a.sum += a.suf;
  }  // (pre == len: the leading run ends here and stays the prefix)
  a.suf = 0;
  a.len += n;
}
__device__ __forceinline__ void rs_append_full(RunSum& a, uint32_t n = 512) {
  if (a.pre == a.len) a.pre += n;
  a.suf += n;
  a.len += n;
}
__device__ __forceinline__ RunSum rs_combine32(const RunSum& a, const RunSum& b, uint32_t min_run) {
  RunSum r;
  const bool af = a.pre == a.len, bf = b.pre == b.len;
  r.len = a.len + b.len;
  r.pre = af ? a.len + b.pre : a.pre;
  r.suf = bf ? b.len + a.suf : b.suf;
  r.cnt = a.cnt + b.cnt;
  r.sum = a.sum + b.sum;
  if (!af && !bf) {
    const uint32_t mid = a.suf + b.pre;
    if (mid > 0 && mid >= min_run) {
      r.cnt += 1;
      r.sum += mid;
    }
  }
  return r;
}

// The mixed (slow) case of one 512-word run step, out of line to keep the hot
// loop small (instruction cache).
__device__ __noinline__ RunSum run_step_mixed(RunSum a, const uint32_t* bits, uint32_t shift,
                                              uint32_t lane, uint32_t min_run) {
  const uint32_t m = pack4(bits[0] >> shift) | (pack4(bits[1] >> shift) << 4) |
                     (pack4(bits[2] >> shift) << 8) | (pack4(bits[3] >> shift) << 12);
  return rs_combine32(a, warp_runs(m, lane, min_run), min_run);
}

// rw = logical word of the lane's first word; blk = counters of this row, the
// first one being logical block goff / B.
// The step holding the row's end: the exact summary of its first n words (no
// padding words, so a run reaching the row end stays open -- what a piece of a
// sharded allocation needs).  Streams the 32 lane masks; rare (once per row).
__device__ __noinline__ RunSum run_step_exact(RunSum a, const uint32_t* bits, uint32_t shift,
                                              uint32_t n, uint32_t min_run) {
  // warp-parallel: the 512-word summary of the step with the words >= n as
  // zeros (warp_runs), then the run that reaches word n-1 is reopened -- it is
  // the exact summary's suffix, not a closed run (len = n).  n in [1, 512).
  const uint32_t lane = threadIdx.x & 31, base = lane * 16;
  const uint32_t valid = base >= n ? 0u : (n - base >= 16 ? 0xFFFFu : ((1u << (n - base)) - 1u));
  const uint32_t m = (pack4(bits[0] >> shift) | (pack4(bits[1] >> shift) << 4) |
                      (pack4(bits[2] >> shift) << 8) | (pack4(bits[3] >> shift) << 12)) & valid;
  const RunSum w = warp_runs(m, lane, min_run);
  RunSum b;
  b.len = n;
  if (w.pre >= n) {  // all ones in [0, n)
    b.pre = b.suf = n;
    b.cnt = b.sum = 0;
  } else {
    const uint32_t z = ~m & valid;  // zeros inside [0, n)
    const uint32_t lz1 = z ? base + 32 - __clz(z) : 0u;  // (last zero of the lane) + 1
    const uint32_t t = n - __reduce_max_sync(0xFFFFFFFFu, lz1);  // ones ending at n-1
    b.pre = w.pre;
    b.suf = t;
    b.cnt = w.cnt;
    b.sum = w.sum;
    if (t > 0 && t >= min_run) {  // warp_runs closed it at the padding
      b.cnt -= 1;
      b.sum -= t;
    }
  }
  return rs_combine32(a, b, min_run);
}

__device__ __noinline__ void block_counts(uint32_t f0, uint32_t f1, uint32_t f2, uint32_t f3,
                                          uint64_t rw, uint64_t B, uint32_t* blk, uint64_t kb0) {
  const uint32_t g = ((f0 >> 6) & kL4) | (((f1 >> 6) & kL4) << 1) | (((f2 >> 6) & kL4) << 2) |
                     (((f3 >> 6) & kL4) << 3);
  uint32_t gm = 0;  // bit i = GPU-accessed flag of word rw + i
#pragma unroll
  for (uint32_t c = 0; c < 4; ++c)
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) gm |= ((g >> (8 * k + c)) & 1u) << (4 * c + k);
  if (!gm) return;
  uint64_t a = rw;
  const uint64_t e = rw + 16;
  while (a < e) {
    const uint64_t k = a / B;
    const uint64_t be = (k + 1) * B < e ? (k + 1) * B : e;
    const uint32_t lo = (uint32_t)(a - rw), hi = (uint32_t)(be - rw);
    const uint32_t seg = ((hi >= 32 ? 0xFFFFFFFFu : ((1u << hi) - 1u)) & ~((1u << lo) - 1u));
    const uint32_t c = __popc(gm & seg);
    if (c) atomicAdd(blk + (k - kb0), c);
    a = be;
  }
}

struct TileAcc {
  VCount raw, der;
  RunSum wu = {0, 0, 0, 0, 0}, wd = {0, 0, 0, 0, 0};
  // uniform 512-word steps (every record byte equal): counted by byte value,
  // warp-uniform -- ub = the byte of the current stretch, un = its steps; the
  // stretches already closed are added to the warp's counters in shared memory
  uint32_t ub = 0, un = 0;
  uint32_t* uc = nullptr;  // this warp's 9 counters (shared memory)
  // Close the current stretch: its counts (lane 0, shared memory) and its run
  // steps (warp-uniform; must precede any other step's run update).
  __device__ __forceinline__ void close_uniform(uint32_t lane, uint32_t min_run) {
    if (!un) return;
    const uint32_t b = ub, n = un * 512;
    if (lane == 0) {
      const bool cpu = (b & 0x34u) != 0, gpu = (b & 0xC8u) != 0, wr = (b & 0x0Cu) != 0;
      uc[0] += (b >> 2 & 1u) * n;  // wC
      uc[1] += (b >> 3 & 1u) * n;  // wG
      uc[2] += (b >> 4 & 1u) * n;  // rCC
      uc[3] += (b >> 6 & 1u) * n;  // rCG
      uc[4] += (b >> 5 & 1u) * n;  // rGC
      uc[5] += (b >> 7 & 1u) * n;  // rGG
      uc[6] += (cpu || gpu) ? n : 0u;
      uc[7] += gpu ? n : 0u;
      uc[8] += (cpu && gpu && wr) ? n : 0u;
    }
    if ((b & 0x44u) == 0x04u) rs_append_full(wu, n);  // u = wC & !rCG
    else rs_append_zero(wu, min_run, n);
    if (b & 0x10u) rs_append_full(wd, n);  // d = rCC
    else rs_append_zero(wd, min_run, n);
    un = 0;
  }
};

// One 16-word lane step: TAIL = the warp's range may end inside the row.
template <bool TAIL, bool RESET, bool BLOCKS>
__device__ __forceinline__ void tile_step(TileAcc& A, uint4 y, uint4* dst, uint32_t w, uint32_t live,
                                          uint32_t lane, uint32_t min_run, uint64_t rw0,
                                          uint64_t B, uint32_t* blk, uint64_t kb0) {
  if (!BLOCKS) {
    // Fast path: the warp's 512 words all hold the same record byte (long
    // stretches of one access pattern are the common case of a real shadow).
    const uint32_t u = y.x;
    const bool lu = y.y == u && y.z == u && y.w == u && __byte_perm(u, 0, 0) == u &&
                    (!TAIL || w - lane * 16 + 512 <= live);
    const uint32_t u0 = __shfl_sync(0xFFFFFFFFu, u, 0);
    if (__all_sync(0xFFFFFFFFu, lu && u == u0)) {
      const uint32_t b = u0 & 0xFFu;
      if (b != A.ub) {
        A.close_uniform(lane, min_run);
        A.ub = b;
      }
      A.un += 1;
      if (RESET && (b & 0xFEu)) {
        const uint32_t k = u0 & kL4;
        *dst = make_uint4(k, k, k, k);
      }
      return;
    }
  }
  A.close_uniform(lane, min_run);  // (a pending stretch precedes this step)
  uint32_t x[4] = {y.x, y.y, y.z, y.w};
  uint32_t keep[4] = {kL4, kL4, kL4, kL4};
  if (TAIL && w + 16 > live) {  // mask the words past the row's end
#pragma unroll
    for (uint32_t c = 0; c < 4; ++c) {
      uint32_t m = 0;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k)
        if (w + c * 4 + k < live) m |= 0xFFu << (8 * k);
      x[c] &= m;
      keep[c] |= ~m;
    }
  }
  A.raw.add4(x[0], x[1], x[2], x[3]);
  const uint32_t f0 = derived_flags(x[0]), f1 = derived_flags(x[1]), f2 = derived_flags(x[2]),
                 f3 = derived_flags(x[3]);
  A.der.add4(f0, f1, f2, f3);
  // transfer runs: u = wC & !rCG (bit 2), d = rCC (bit 4)
  uint32_t uu[4], dd[4];
#pragma unroll
  for (uint32_t c = 0; c < 4; ++c) {
    uu[c] = x[c] & ~(x[c] >> 4) & 0x04040404u;
    dd[c] = x[c] & 0x10101010u;
  }
  const uint32_t step0 = w - lane * 16;  // first (warp-relative) word of this 512-word step
  if (TAIL && step0 + 512 > live) {      // the row ends in (or before) this step
    if (step0 < live) {
      A.wu = run_step_exact(A.wu, uu, 2, live - step0, min_run);
      A.wd = run_step_exact(A.wd, dd, 4, live - step0, min_run);
    }
  } else {
  if (__ballot_sync(0xFFFFFFFFu, (uu[0] | uu[1] | uu[2] | uu[3]) != 0) == 0)
    rs_append_zero(A.wu, min_run);
  else if (__all_sync(0xFFFFFFFFu, (uu[0] & uu[1] & uu[2] & uu[3]) == 0x04040404u))
    rs_append_full(A.wu);
  else
    A.wu = run_step_mixed(A.wu, uu, 2, lane, min_run);
  if (__ballot_sync(0xFFFFFFFFu, (dd[0] | dd[1] | dd[2] | dd[3]) != 0) == 0)
    rs_append_zero(A.wd, min_run);
  else if (__all_sync(0xFFFFFFFFu, (dd[0] & dd[1] & dd[2] & dd[3]) == 0x10101010u))
    rs_append_full(A.wd);
  else
    A.wd = run_step_mixed(A.wd, dd, 4, lane, min_run);
  }
  if (BLOCKS && (!TAIL || w < live)) block_counts(f0, f1, f2, f3, rw0 + w, B, blk, kb0);
  // fused reset (D4): keep L only, words of this row only
  if (RESET && (!TAIL || w < live)) {
    if (((y.x & ~keep[0]) | (y.y & ~keep[1]) | (y.z & ~keep[2]) | (y.w & ~keep[3])) != 0)
      *dst = make_uint4(y.x & keep[0], y.y & keep[1], y.z & keep[2], y.w & keep[3]);
  }
}

// ---- 1D TMA (cp.async.bulk) staging of the shadow, one mbarrier per stage ----
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!ok);
}

// The warp's staging ring: kDiagStages slots of kStageSteps 512-word steps each
// (kStageSteps x 512 B of records), filled by 1D bulk copies (TMA) that lane 0
// issues a whole ring ahead; each slot's mbarrier counts the bytes in.  No
// register staging, so the prefetch depth (8 KB per warp) does not cost
// registers (occupancy), and the wait + refill is paid once per kStageSteps.
#ifndef XPL_DIAG_STAGE_STEPS
#define XPL_DIAG_STAGE_STEPS 2
#endif
#ifndef XPL_DIAG_STAGES
#define XPL_DIAG_STAGES 4
#endif
constexpr uint32_t kStageSteps = XPL_DIAG_STAGE_STEPS;
constexpr uint32_t kDiagStages = XPL_DIAG_STAGES;
struct WarpRing {
  uint4 buf[kDiagStages][kStageSteps * 32];
  uint64_t bar[kDiagStages];
};
constexpr size_t kDiagSmem = (kDiagThreads / 32) * sizeof(WarpRing);

template <bool TAIL, bool RESET, bool BLOCKS>
__device__ __forceinline__ void tile_loop(TileAcc& A, WarpRing& R, uint4* p4, uint32_t live,
                                          uint32_t lane, uint32_t min_run, uint64_t rw0, uint64_t B,
                                          uint32_t* blk, uint64_t kb0 = 0) {
  const uint32_t n = (live + 511) / 512;  // steps holding row words (live = the tile size unless TAIL)
  const uint32_t ns = (n + kStageSteps - 1) / kStageSteps;     // stages
  // bytes of stage j: whole 16-word vectors up to the row's end (the row's
  // shadow span is a multiple of 16 words, so they are all inside it)
  auto issue = [&](uint32_t j) {
    const uint32_t words = TAIL ? min(kStageSteps * 512u, live - j * kStageSteps * 512) : kStageSteps * 512u;
    bulk_load(R.buf[j % kDiagStages], p4 + j * kStageSteps * 32, ((words + 15) & ~15u),
              &R.bar[j % kDiagStages]);
  };
  if (lane == 0)
    for (uint32_t j = 0; j < ns && j < kDiagStages; ++j) issue(j);
#pragma unroll 1
  for (uint32_t j = 0; j < ns; ++j) {
    const uint32_t st = j % kDiagStages;
    mbar_wait(&R.bar[st], (j / kDiagStages) & 1u);
#pragma unroll 1
    for (uint32_t k = 0; k < kStageSteps; ++k) {
      const uint32_t it = j * kStageSteps + k;
      if (TAIL && it >= n) break;
      const uint32_t w = it * 512 + lane * 16;
      uint4 y = R.buf[st][k * 32 + lane];
      if (TAIL && w >= live) y = make_uint4(0, 0, 0, 0);  // (bytes not copied this round)
      tile_step<TAIL, RESET, BLOCKS>(A, y, p4 + it * 32 + lane, w, live, lane, min_run, rw0, B, blk, kb0);
    }
    __syncwarp();
    if (lane == 0 && j + kDiagStages < ns) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // our reads before the refill
      issue(j + kDiagStages);
    }
  }
}

// One warp = one tile of p.tile_words words of one row (no CTA-wide barrier: the
// warps of a CTA are independent, so a warp on a cheap uniform stretch never
// waits for one on a mixed stretch); per step lane l owns 16 words (one uint4
// of records).  Counts: two Harley-Seal vertical counters (raw record bits;
// derived per-word any/gpu/alternating flags) popcounted once per tile, plus
// the uniform-step counts.  Runs: ballot fast paths for all-zero/all-one
// 512-word steps, warp_runs() for mixed ones.  Reset fused.  The tile's counts
// and run summaries go to tiles[t]; the stitch adds and combines them in order.
// The stitch in one kernel launched right behind the tile kernel (programmatic
// dependent launch; no block counts: p.block_words == 0): a warp per segment
// combines its <= kSegTiles tiles; the warp that finishes its row's last
// segment (last-warp-done: release fence + done counter, which that warp resets
// to 0 for the next call) combines the row and writes its report.  Null
// row_done = the separate stitch kernels.
struct FusedStitch {
  uint32_t* row_done;               // per row: segments done (kept zero between calls)
  unsigned long long* segcnt;       // 9 counters per segment
  unsigned long long* cnt;          // C_NCNT counters per row (partials)
  xpl_alloc_report* out;
  RowPartial* parts;
  const uint32_t* flags_in;         // d_misc[0..1], copied to flags_out by row 0's finalizer
  uint32_t* flags_out;
};

#ifndef XPL_DIAG_MINB
#define XPL_DIAG_MINB 4  // CTAs per SM the register budget is sized for (A/B: profiles/r1h_diag_variants.txt)
#endif
__global__ void __launch_bounds__(kDiagThreads, XPL_DIAG_MINB) diag_tile_kernel(
    const DiagRow* __restrict__ rows, const uint32_t* __restrict__ tile_row, uint64_t ntiles,
    DiagParams p, uint32_t* __restrict__ pool, TileSum* __restrict__ tiles,
    uint32_t* __restrict__ blk_cnt) {
  constexpr uint32_t kWarps = kDiagThreads / 32;
  __shared__ uint32_t s_uc[kWarps][9];
  extern __shared__ __align__(128) unsigned char s_dyn[];
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint64_t t = (uint64_t)blockIdx.x * kWarps + warp;
  if (t >= ntiles) return;
  WarpRing& R = reinterpret_cast<WarpRing*>(s_dyn)[warp];
  if (lane == 0) {
    for (uint32_t k = 0; k < kDiagStages; ++k) mbar_init(&R.bar[k], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const uint32_t ri = tile_row[t];
  const DiagRow row = rows[ri];
  const uint32_t tw = p.tile_words;
  const uint64_t ww0 = (t - row.tile0) * tw;  // row word
  const uint32_t min_run = (uint32_t)(p.min_run < 0xFFFFFFFFull ? p.min_run : 0xFFFFFFFFull);
  const uint32_t live = (uint32_t)min(row.words - ww0, (uint64_t)tw);
  uint4* p4 = reinterpret_cast<uint4*>(pool) + ((row.off + ww0) >> 4);
  uint32_t* blk = blk_cnt + row.blk0;
  TileAcc A;
  if (lane < 9) s_uc[warp][lane] = 0;
  __syncwarp();
  A.uc = s_uc[warp];
  const bool tail = live < tw;
  if (p.block_words) {  // rare: blocks need per-lane counter atomics (logical block index)
    const uint64_t kb0 = row.goff / p.block_words;
    if (p.reset) tile_loop<true, true, true>(A, R, p4, live, lane, min_run, row.goff + ww0, p.block_words, blk, kb0);
    else tile_loop<true, false, true>(A, R, p4, live, lane, min_run, row.goff + ww0, p.block_words, blk, kb0);
  } else if (p.reset) {
    if (tail) tile_loop<true, true, false>(A, R, p4, live, lane, min_run, ww0, 0, blk);
    else tile_loop<false, true, false>(A, R, p4, live, lane, min_run, ww0, 0, blk);
  } else {
    if (tail) tile_loop<true, false, false>(A, R, p4, live, lane, min_run, ww0, 0, blk);
    else tile_loop<false, false, false>(A, R, p4, live, lane, min_run, ww0, 0, blk);
  }

  // counters: 6 raw bit classes + any/gpu/alternating
  uint32_t c9[9];
  c9[0] = A.raw.count(0x04040404u);  // wC
  c9[1] = A.raw.count(0x08080808u);  // wG
  c9[2] = A.raw.count(0x10101010u);  // rCC
  c9[3] = A.raw.count(0x40404040u);  // rCG
  c9[4] = A.raw.count(0x20202020u);  // rGC
  c9[5] = A.raw.count(0x80808080u);  // rGG
  c9[6] = A.der.count(0x80808080u);  // any
  c9[7] = A.der.count(0x40404040u);  // gpu
  c9[8] = A.der.count(0x20202020u);  // alternating
  A.close_uniform(lane, min_run);
  __syncwarp();
  TileSum* ts = tiles + t;
#pragma unroll
  for (int k = 0; k < 9; ++k) {
    const uint32_t s = __reduce_add_sync(0xFFFFFFFFu, c9[k]);
    if (lane == k) ts->cnt[k] = s + A.uc[k];
  }
  if (lane == 0) {
    ts->u = A.wu;
    ts->d = A.wd;
  }
}

__device__ __forceinline__ void run_final(const RunSum64& s, uint64_t min_run, uint64_t* runs,
                                          uint64_t* words) {
  uint64_t r = s.cnt, w = s.sum;
  if (s.pre == s.len) {
    if (s.len >= min_run && s.len > 0) { r += 1; w += s.len; }
  } else {
    if (s.pre >= min_run && s.pre > 0) { r += 1; w += s.pre; }
    if (s.suf >= min_run && s.suf > 0) { r += 1; w += s.suf; }
  }
  *runs = r;
  *words = w;
}

struct RunPair {
  RunSum64 u, d;
};
static_assert(sizeof(RunPair) == kRunPairBytes, "RunPair size");

__device__ __forceinline__ RunSum64 shfl_down_rs(const RunSum64& a, uint32_t s) {
  RunSum64 o;
  o.len = __shfl_down_sync(0xFFFFFFFFu, a.len, s);
  o.pre = __shfl_down_sync(0xFFFFFFFFu, a.pre, s);
  o.suf = __shfl_down_sync(0xFFFFFFFFu, a.suf, s);
  o.cnt = __shfl_down_sync(0xFFFFFFFFu, a.cnt, s);
  o.sum = __shfl_down_sync(0xFFFFFFFFu, a.sum, s);
  return o;
}

// Ordered warp reduction: lane 0 ends with combine(lane 0, ..., lane 31).
__device__ __forceinline__ void warp_combine(RunSum64& a, RunSum64& b, uint32_t lane, uint64_t min_run) {
  for (uint32_t s = 1; s < 32; s <<= 1) {
    const RunSum64 oa = shfl_down_rs(a, s), ob = shfl_down_rs(b, s);
    if ((lane & (2 * s - 1)) == 0 && lane + s < 32) {
      a = rs_combine(a, oa, min_run);
      b = rs_combine(b, ob, min_run);
    }
  }
}

// Stitch, level 1: one warp per segment of <= kSegTiles consecutive tiles of a
// row; lanes combine contiguous sub-ranges, then an ordered warp reduction.
__global__ void stitch_seg_kernel(const StitchSeg* __restrict__ segs, uint32_t nseg,
                                  const TileSum* __restrict__ tiles, uint64_t min_run,
                                  RunPair* __restrict__ out, unsigned long long* __restrict__ cnt) {
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  if (gw >= nseg) return;
  const StitchSeg sg = segs[gw];
  const uint64_t per = (sg.n + 31) / 32;
  const uint64_t t0 = sg.t0 + lane * per;
  const uint64_t t1 = min(sg.t0 + sg.n, t0 + per);
  RunSum64 a = {0, 0, 0, 0, 0}, b = {0, 0, 0, 0, 0};
  uint64_t c9[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0};
  for (uint64_t t = t0; t < t1; ++t) {
    const RunSum u = tiles[t].u, d = tiles[t].d;
    a = rs_combine(a, RunSum64{u.len, u.pre, u.suf, u.cnt, u.sum}, min_run);
    b = rs_combine(b, RunSum64{d.len, d.pre, d.suf, d.cnt, d.sum}, min_run);
#pragma unroll
    for (int k = 0; k < 9; ++k) c9[k] += tiles[t].cnt[k];
  }
  warp_combine(a, b, lane, min_run);
  if (lane == 0) out[gw] = RunPair{a, b};
#pragma unroll
  for (int k = 0; k < 9; ++k) {
    uint64_t v = c9[k];
    for (uint32_t o = 16; o; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
    if (lane == 0 && v) atomicAdd(cnt + (uint64_t)sg.row * C_NCNT + k, (unsigned long long)v);
  }
}

// One report row from the row's combined run summaries and counters c (D8).
__device__ __forceinline__ void row_finalize(const DiagRow& r, uint32_t gw, const RunSum64& a, const RunSum64& b,
                                             const unsigned long long* c, const DiagParams& p,
                                             xpl_alloc_report* __restrict__ out, RowPartial* __restrict__ parts,
                                             const uint32_t* __restrict__ blk_cnt) {
  if (parts) {
    RowPartial& q = parts[gw];
    q.u[0] = a.len; q.u[1] = a.pre; q.u[2] = a.suf; q.u[3] = a.cnt; q.u[4] = a.sum;
    q.d[0] = b.len; q.d[1] = b.pre; q.d[2] = b.suf; q.d[3] = b.cnt; q.d[4] = b.sum;
    q.blk_first_g = (p.block_words && r.nblk) ? blk_cnt[r.blk0] : 0;
    q.blk_last_g = (p.block_words && r.nblk) ? blk_cnt[r.blk0 + r.nblk - 1] : 0;
  }
  xpl_alloc_report o;
  o.id = o.base = o.bytes = 0;
  o.words = r.words;
  o.kind = r.kind;
  o.live = 0;
  o.name_idx = 0xFFFFFFFFu;
  o.w_c = c[C_WC];
  o.w_g = c[C_WG];
  o.r_cc = c[C_RCC];
  o.r_cg = c[C_RCG];
  o.r_gc = c[C_RGC];
  o.r_gg = c[C_RGG];
  o.any_acc = c[C_ANY];
  o.gpu_acc = c[C_GPU];
  o.alternating = c[C_ALT];
  o.density_pct_any = o.any_acc * 100 / r.words;
  o.density_pct_gpu = o.gpu_acc * 100 / r.words;
  if (p.block_words == 0) {
    const bool f = o.gpu_acc >= 1 && 100ull * o.gpu_acc <= (uint64_t)p.thr * r.words;
    o.low_density_blocks = f ? 1 : 0;
    o.low_density_words = f ? r.words : 0;
  } else {
    o.low_density_blocks = c[C_LDB];
    o.low_density_words = c[C_LDW];
  }
  uint64_t rr, ww;
  run_final(a, p.min_run, &rr, &ww);
  o.h2d_unused_runs = rr;
  o.h2d_unused_words = ww;
  run_final(b, p.min_run, &rr, &ww);
  o.d2h_unneeded_runs = rr;
  o.d2h_unneeded_words = ww;
  o.ever_accessed = 0;
  uint32_t f = 0;
  if (r.kind == XPL_ALLOC_MANAGED && o.alternating > 0) f |= XPL_PAT_ALTERNATING;
  if (r.kind != XPL_ALLOC_HOST && o.low_density_blocks > 0) f |= XPL_PAT_LOW_DENSITY;
  if (r.kind == XPL_ALLOC_DEVICE && o.h2d_unused_runs > 0) f |= XPL_PAT_UNNEEDED_H2D;
  if (r.kind == XPL_ALLOC_DEVICE && o.d2h_unneeded_runs > 0) f |= XPL_PAT_UNNEEDED_D2H;
  if (o.any_acc == 0) f |= XPL_PAT_UNUSED;
  o.flags = f;
  out[gw] = o;
}

// Stitch, level 2 + finalize: one warp per row combines its segment summaries,
// then lane 0 turns the counters into the report row (flags P:L84-114, D8).
__global__ void stitch_row_finalize_kernel(const DiagRow* __restrict__ rows, uint32_t nrows,
                                           const RunPair* __restrict__ segsum, DiagParams p,
                                           unsigned long long* __restrict__ cnt,
                                           xpl_alloc_report* __restrict__ out,
                                           RowPartial* __restrict__ parts,
                                           const uint32_t* __restrict__ blk_cnt) {
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  if (gw >= nrows) return;
  const DiagRow r = rows[gw];
  const uint64_t per = (r.nseg + 31) / 32;
  const uint64_t s0 = r.seg0 + lane * per;
  const uint64_t s1 = min(r.seg0 + r.nseg, s0 + per);
  RunSum64 a = {0, 0, 0, 0, 0}, b = {0, 0, 0, 0, 0};
  for (uint64_t s = s0; s < s1; ++s) {
    a = rs_combine(a, segsum[s].u, p.min_run);
    b = rs_combine(b, segsum[s].d, p.min_run);
  }
  warp_combine(a, b, lane, p.min_run);
  if (lane == 0) row_finalize(r, gw, a, b, cnt + (uint64_t)gw * C_NCNT, p, out, parts, blk_cnt);
}

__device__ __forceinline__ void fused_flags(const FusedStitch& fs) {
  if (!fs.flags_out) return;
  fs.flags_out[0] = *reinterpret_cast<const volatile uint32_t*>(fs.flags_in);
  fs.flags_out[1] = *reinterpret_cast<const volatile uint32_t*>(fs.flags_in + 1);
}

__device__ __forceinline__ RunSum64 rs64(const RunSum& u) { return RunSum64{u.len, u.pre, u.suf, u.cnt, u.sum}; }

__global__ void __launch_bounds__(256) stitch_fused_kernel(const StitchSeg* __restrict__ segs, uint32_t nseg,
                                                           const DiagRow* __restrict__ rows,
                                                           const TileSum* __restrict__ tiles, DiagParams p,
                                                           RunPair* __restrict__ ss, FusedStitch fs) {
  asm volatile("griddepcontrol.wait;" ::: "memory");  // (the tile kernel's summaries are complete)
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  if (gw >= nseg) return;
  const StitchSeg sg = segs[gw];
  const uint32_t ri = (uint32_t)sg.row;
  const DiagRow row = rows[ri];
  // level 1: the segment's tiles in order (lanes take contiguous sub-ranges)
  RunSum64 a = {0, 0, 0, 0, 0}, b = {0, 0, 0, 0, 0};
  uint64_t c9[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0};
  {
    // (kSegTiles / 32 tiles per lane: every load is issued before the first combine)
    constexpr uint32_t kPer = (uint32_t)(kSegTiles / 32);
    const uint64_t per = (sg.n + 31) / 32;
    const uint64_t t0 = sg.t0 + lane * per, t1 = min(sg.t0 + sg.n, t0 + per);
    TileSum ts[kPer];
#pragma unroll
    for (uint32_t k = 0; k < kPer; ++k)
      if (t0 + k < t1) ts[k] = tiles[t0 + k];
#pragma unroll
    for (uint32_t k = 0; k < kPer; ++k) {
      if (t0 + k >= t1) break;
      a = rs_combine(a, rs64(ts[k].u), p.min_run);
      b = rs_combine(b, rs64(ts[k].d), p.min_run);
#pragma unroll
      for (int j = 0; j < 9; ++j) c9[j] += ts[k].cnt[j];
    }
  }
  warp_combine(a, b, lane, p.min_run);
#pragma unroll
  for (int j = 0; j < 9; ++j)
    for (uint32_t o = 16; o; o >>= 1) c9[j] += __shfl_down_sync(0xFFFFFFFFu, c9[j], o);
  if (row.nseg > 1) {
    uint32_t last = 0;
    if (lane == 0) {
      ss[gw] = RunPair{a, b};
      for (int j = 0; j < 9; ++j) fs.segcnt[(uint64_t)gw * 9 + j] = c9[j];
      __threadfence();  // (release: the segment's summary before the count)
      last = atomicAdd(fs.row_done + ri, 1u) == row.nseg - 1;
    }
    if (!__shfl_sync(0xFFFFFFFFu, last, 0)) return;
    __threadfence();  // (acquire: the row's other segment summaries)
    // level 2: the row's segments in order
    a = RunSum64{0, 0, 0, 0, 0};
    b = RunSum64{0, 0, 0, 0, 0};
#pragma unroll
    for (int j = 0; j < 9; ++j) c9[j] = 0;
    const uint64_t per = (row.nseg + 31) / 32;
    const uint64_t s0 = row.seg0 + lane * per, s1 = min(row.seg0 + row.nseg, s0 + per);
    for (uint64_t u = s0; u < s1; ++u) {
      const uint64_t* q = reinterpret_cast<const uint64_t*>(ss + u);
      const RunSum64 x = {__ldcg(q + 0), __ldcg(q + 1), __ldcg(q + 2), __ldcg(q + 3), __ldcg(q + 4)};
      const RunSum64 y = {__ldcg(q + 5), __ldcg(q + 6), __ldcg(q + 7), __ldcg(q + 8), __ldcg(q + 9)};
      a = rs_combine(a, x, p.min_run);
      b = rs_combine(b, y, p.min_run);
#pragma unroll
      for (int j = 0; j < 9; ++j) c9[j] += __ldcg(fs.segcnt + u * 9 + j);
    }
    warp_combine(a, b, lane, p.min_run);
#pragma unroll
    for (int j = 0; j < 9; ++j)
      for (uint32_t o = 16; o; o >>= 1) c9[j] += __shfl_down_sync(0xFFFFFFFFu, c9[j], o);
  }
  if (lane == 0) {
    if (row.nseg > 1) fs.row_done[ri] = 0;
    unsigned long long* c = fs.cnt + (uint64_t)ri * C_NCNT;
    for (int j = 0; j < 9; ++j) c[j] = c9[j];
    for (int j = 9; j < (int)C_NCNT; ++j) c[j] = 0;
    row_finalize(row, ri, a, b, c, p, fs.out, fs.parts, nullptr);
    if (ri == 0) fused_flags(fs);
  }
}

// Low-density blocks (Eq. P:L102, D11-D13): block flagged iff it has
// >= 1 GPU-accessed word and 100*g <= thr*size.
__global__ void block_eval_kernel(const DiagRow* __restrict__ rows, uint32_t nrows,
                                  uint64_t nblocks, const uint32_t* __restrict__ blk_cnt,
                                  uint64_t B, uint32_t thr, unsigned long long* cnt) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nblocks;
       j += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t g = blk_cnt[j];
    if (!g) continue;
    uint32_t lo = 0, hi = nrows;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (rows[mid].blk0 <= j) lo = mid;
      else hi = mid;
    }
    const DiagRow r = rows[lo];
    const uint64_t k = r.goff / B + (j - r.blk0);  // logical block
    const uint64_t s = min(B, r.lwords - k * B);   // its size in the logical allocation
    if (k * B < r.goff || k * B + s > r.goff + r.words) continue;  // cut by the piece: combined later
    if (100ull * g <= (uint64_t)thr * s) {
      atomicAdd(cnt + (uint64_t)lo * C_NCNT + C_LDB, 1ull);
      atomicAdd(cnt + (uint64_t)lo * C_NCNT + C_LDW, (unsigned long long)s);
    }
  }
}

__global__ void fill_u32_kernel(uint32_t* p, uint64_t n, uint32_t v) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

int grid_for(uint64_t n, int threads, int max_ctas) {
  uint64_t g = (n + threads - 1) / threads;
  if (g < 1) g = 1;
  if (g > (uint64_t)max_ctas) g = max_ctas;
  return (int)g;
}


// ---------------------------------------------------------------------------
// UM page view (NEXT-3): per page of P words of a row, the
// OR over its records of: CPU access, GPU access, a word accessed by both, an
// alternating word (D9), CPU write, GPU write.  One warp per contiguous chunk of
// pages (so the row changes rarely); lanes stride over the page's shadow u32s,
// bytes outside the page masked; per-row page counts in registers, flushed with
// one atomicAdd per counter when the warp leaves a row.
__device__ __forceinline__ uint32_t page_bits(uint32_t x) {
  const uint32_t cpu = ((x & 0x34343434u) + 0x7F7F7F7Fu) & 0x80808080u;          // wC|rCC|rGC
  const uint32_t gpu = (((x & 0x48484848u) + 0x7F7F7F7Fu) | x) & 0x80808080u;    // wG|rCG|rGG
  const uint32_t wr = ((x & 0x0C0C0C0Cu) + 0x7F7F7F7Fu) & 0x80808080u;           // wC|wG
  const uint32_t both = cpu & gpu;
  return (cpu ? 1u : 0u) | (gpu ? 2u : 0u) | (both ? 4u : 0u) | ((both & wr) ? 8u : 0u) |
         ((x & 0x04040404u) ? 16u : 0u) | ((x & 0x08080808u) ? 32u : 0u);
}

__global__ void __launch_bounds__(256) page_kernel(const PageRow* __restrict__ rows, uint32_t nrows,
                                                   uint64_t npages, uint64_t P,
                                                   const uint32_t* __restrict__ pool,
                                                   uint8_t* __restrict__ flags,
                                                   unsigned long long* __restrict__ cnt) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
  const uint64_t wi = (uint64_t)blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  const uint64_t chunk = (npages + nw - 1) / nw;
  const uint64_t p0 = wi * chunk, p1 = min(npages, p0 + chunk);
  if (p0 >= p1) return;
  uint32_t lo = 0, hi = nrows;  // the row holding page p0: last row with page0 <= p0
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) / 2;
    if (rows[mid].page0 <= p0) lo = mid;
    else hi = mid;
  }
  // the warp's row state lives in registers: the row, the first page of the next
  // row, the pool word where page p starts; counters are 32-bit (a warp's chunk
  // of pages fits) and go out with one atomicAdd each when the row changes
  uint32_t r = lo;
  PageRow R = rows[r];
  uint64_t next0 = r + 1 < nrows ? rows[r + 1].page0 : npages;
  uint64_t pw = R.off + (p0 - R.page0) * P;  // pool word of page p's first record
  // per-lane counts (the lane that judged a page counts it), summed over the
  // warp when the row changes
  uint32_t c0 = 0, c1 = 0, c2 = 0, c3 = 0, c4 = 0;
  auto flush_counts = [&]() {
    const uint32_t s0 = __reduce_add_sync(0xFFFFFFFFu, c0), s1 = __reduce_add_sync(0xFFFFFFFFu, c1),
                   s2 = __reduce_add_sync(0xFFFFFFFFu, c2), s3 = __reduce_add_sync(0xFFFFFFFFu, c3),
                   s4 = __reduce_add_sync(0xFFFFFFFFu, c4);
    const uint32_t v = lane == 0 ? s0 : lane == 1 ? s1 : lane == 2 ? s2 : lane == 3 ? s3 : s4;
    if (lane < 5 && v) atomicAdd(cnt + 5ull * r + lane, (unsigned long long)v);
    c0 = c1 = c2 = c3 = c4 = 0;
  };
  auto count = [&](uint32_t f) {
    const uint32_t shared = (f & 3u) == 3u;
    c0 += f & 1u;
    c1 += (f >> 1) & 1u;
    c2 += shared;
    c3 += shared & ((f >> 2) ^ 1u);
    c4 += (f >> 3) & 1u;
  };
  const ulonglong2* p4 = reinterpret_cast<const ulonglong2*>(pool);
  // small pages (P % 16 == 0, at most 128 uint4 of records): L lanes per page,
  // 32 / L pages per warp step, so the per-page bookkeeping is shared by the warp
  const uint64_t u4 = P >> 4;  // uint4 per page
  uint32_t L = 32;
  if ((P & 15) == 0 && u4 <= 128)
    while (L > 1 && (uint64_t)(L >> 1) * 4 >= u4) L >>= 1;  // smallest power of 2 with 4 L >= u4
  const uint32_t G = 32 / L, gi = lane / L, li = lane % L;
  const uint32_t gmask = L == 32 ? 0xFFFFFFFFu : ((1u << L) - 1u) << (gi * L);
  for (uint64_t p = p0; p < p1;) {
    while (p >= next0) {  // the next row (empty rows have no pages: skipped)
      flush_counts();
      ++r;
      R = rows[r];
      next0 = r + 1 < nrows ? rows[r + 1].page0 : npages;
      pw = R.off;
    }
    if (G > 1 && p + G <= p1 && p + G <= next0 && (p + G - R.page0) * P <= R.words) {
      // G whole pages of this row, page p + gi for lane group gi (16-byte aligned:
      // rows start on 16 words, P % 16 == 0)
      const uint64_t v0 = (pw + (uint64_t)gi * P) >> 4;
      ulonglong2 x[4];
#pragma unroll
      for (int k = 0; k < 4; ++k)
        x[k] = li + L * k < u4 ? __ldg(p4 + v0 + li + L * k) : make_ulonglong2(0, 0);
      unsigned long long o = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) o |= x[k].x | x[k].y;
      const uint32_t o32 = (uint32_t)o | (uint32_t)(o >> 32);
      unsigned long long a_both = 0, a_alt = 0;
      if ((o32 & 0x34343434u) && (o32 & 0xC8C8C8C8u)) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const unsigned long long y = (k & 1) ? x[k >> 1].y : x[k >> 1].x;
          const unsigned long long c = (y & 0x3434343434343434ull) + 0x7F7F7F7F7F7F7F7Full;
          const unsigned long long g = ((y & 0x4848484848484848ull) + 0x7F7F7F7F7F7F7F7Full) | y;
          const unsigned long long cg = c & g & 0x8080808080808080ull;
          a_both |= cg;
          a_alt |= cg & ((y & 0x0C0C0C0C0C0C0C0Cull) + 0x7F7F7F7F7F7F7F7Full);
        }
      }
      uint32_t f = ((o32 & 0x34343434u) ? 1u : 0u) | ((o32 & 0xC8C8C8C8u) ? 2u : 0u) | (a_both ? 4u : 0u) |
                   (a_alt ? 8u : 0u) | ((o32 & 0x04040404u) ? 16u : 0u) | ((o32 & 0x08080808u) ? 32u : 0u);
      f = __reduce_or_sync(gmask, f);
      if (li == 0) {
        if (flags) flags[p + gi] = (uint8_t)f;
        count(f);
      }
      p += G;
      pw += (uint64_t)G * P;
      continue;
    }
    const uint64_t w0 = pw;                                 // pool words [w0, w1)
    const uint64_t w1 = min(pw + P, R.off + R.words);
    uint32_t f = 0;
    uint64_t wa = w0;  // words [w0, wa) done by the 16-byte path
    if ((w0 & 15) == 0) {  // page starts on a uint4 (pool rows are 16-word aligned): 16 records
      // per lane, up to 4 loads in flight; the class bits are accumulated per
      // record byte in 64-bit SWAR registers and turned into page bits once
      const uint64_t v0 = w0 >> 4, v1 = w1 >> 4;
      // CPU / GPU / CPU-write / GPU-write presence is a property of the OR of
      // the records; only "both on one word" and "alternating" need per-record
      // work, and only where the lane's 64 records hold both classes at all
      uint32_t a_raw = 0;
      unsigned long long a_both = 0, a_alt = 0;
      for (uint64_t b = v0; b < v1; b += 128) {  // (b is warp-uniform)
        ulonglong2 x[4];
#pragma unroll
        for (int k = 0; k < 4; ++k)
          x[k] = b + 32 * k + lane < v1 ? __ldg(p4 + b + 32 * k + lane) : make_ulonglong2(0, 0);
        unsigned long long o = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) o |= x[k].x | x[k].y;  // (zeros past the page add nothing)
        const uint32_t o32 = (uint32_t)o | (uint32_t)(o >> 32);
        a_raw |= o32;
        if ((o32 & 0x34343434u) && (o32 & 0xC8C8C8C8u)) {
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const unsigned long long y = (k & 1) ? x[k >> 1].y : x[k >> 1].x;
            const unsigned long long c = (y & 0x3434343434343434ull) + 0x7F7F7F7F7F7F7F7Full;
            const unsigned long long g = ((y & 0x4848484848484848ull) + 0x7F7F7F7F7F7F7F7Full) | y;
            const unsigned long long cg = c & g & 0x8080808080808080ull;
            a_both |= cg;
            a_alt |= cg & ((y & 0x0C0C0C0C0C0C0C0Cull) + 0x7F7F7F7F7F7F7F7Full);
          }
        }
      }
      f = ((a_raw & 0x34343434u) ? 1u : 0u) | ((a_raw & 0xC8C8C8C8u) ? 2u : 0u) | (a_both ? 4u : 0u) |
          (a_alt ? 8u : 0u) | ((a_raw & 0x04040404u) ? 16u : 0u) | ((a_raw & 0x08080808u) ? 32u : 0u);
      wa = v1 << 4;
    }
    if (wa < w1) {  // unaligned page start or a tail of < 16 words: u32 loads, bytes outside masked
      for (uint64_t q = (wa >> 2) + lane; q <= ((w1 - 1) >> 2); q += 32) {
        uint32_t x = pool[q];
        if (q * 4 < wa || q * 4 + 4 > w1) {
          uint32_t m = 0;
#pragma unroll
          for (uint32_t k = 0; k < 4; ++k)
            if (q * 4 + k >= wa && q * 4 + k < w1) m |= 0xFFu << (8 * k);
          x &= m;
        }
        f |= page_bits(x);
      }
    }
    f = __reduce_or_sync(0xFFFFFFFFu, f);
    if (lane == 0) {
      if (flags) flags[p] = (uint8_t)f;
      count(f);
    }
    ++p;
    pw += P;
  }
  flush_counts();
}
}  // namespace

void launch_fold(cudaStream_t s, bool pdl, uint32_t* pool, uint8_t* cmap, uint8_t* smap,
                 uint64_t n_super, unsigned long long* stats, uint32_t* flags, int strict, int force) {
  cudaLaunchConfig_t cfg = {};
  const uint64_t ctas = (n_super + 7) / 8;  // (one warp per super-chunk at most)
  cfg.gridDim = dim3((unsigned)(ctas == 0 ? 1 : ctas < XPL_FOLD_CTAS ? ctas : XPL_FOLD_CTAS));  // one wave
  cfg.blockDim = dim3(kFoldThreads);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  cudaLaunchKernelEx(&cfg, fold_kernel, pool, cmap, smap, n_super, stats, flags, strict, force);
}

void launch_merge(cudaStream_t s, const uint64_t* recs, uint32_t n, bool has_r, bool has_w,
                  uint32_t* first_w, uint64_t fw0, uint32_t* pool) {
  if (n <= kMergeSmall) {
    merge_small_kernel<<<1, kMergeThreads, 0, s>>>(recs, n, has_r, has_w, first_w, fw0, pool);
    return;
  }
  const int g = grid_for(n, 256, 148 * 16);
  const bool both = has_r && has_w;
  if (both) merge_firstw_kernel<<<g, 256, 0, s>>>(recs, n, first_w, fw0);
  merge_apply_kernel<<<g, 256, 0, s>>>(recs, n, both ? first_w : nullptr, fw0, pool);
  if (has_w) merge_clear_kernel<<<g, 256, 0, s>>>(recs, n, both ? first_w : nullptr, fw0, pool);
}

void launch_range(cudaStream_t s, const RangeDesc* d_ranges, uint32_t nr, uint64_t nvec,
                  uint32_t* pool, uint8_t* cmap, uint8_t* smap, uint32_t* flags) {
  const int g = grid_for(nvec, 256, 148 * 8);
  range_kernel<<<g, 256, 0, s>>>(d_ranges, nr, nvec, pool, cmap, smap, flags);
}

void launch_diag(cudaStream_t s, const DiagRow* rows, uint32_t nrows, const uint32_t* tile_row,
                 uint64_t ntiles, const StitchSeg* segs, uint32_t nseg, uint64_t nblocks,
                 const DiagParams& p, uint32_t* pool, unsigned long long* cnt, TileSum* tiles,
                 void* segsum, uint32_t* blk_cnt, xpl_alloc_report* out, RowPartial* parts,
                 cudaEvent_t tile_ev0, cudaEvent_t tile_ev1, uint32_t* row_done, unsigned long long* segcnt,
                 const uint32_t* flags_in, uint32_t* flags_out) {
  // fused: tile kernel + one stitch kernel (PDL); block counts (p.block_words)
  // need the block pass between them: separate kernels
  const bool fused = row_done != nullptr && p.block_words == 0;
  if (!fused) {
    cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * C_NCNT * nrows, s);
    if (p.block_words && nblocks) cudaMemsetAsync(blk_cnt, 0, sizeof(uint32_t) * nblocks, s);
  }
  if (tile_ev0) cudaEventRecord(tile_ev0, s);
  constexpr uint32_t kWarps = kDiagThreads / 32;
  // (per device; cheap next to a diagnose)
  cudaFuncSetAttribute(diag_tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kDiagSmem);
  if (ntiles)
    diag_tile_kernel<<<(unsigned)((ntiles + kWarps - 1) / kWarps), kDiagThreads, kDiagSmem, s>>>(
        rows, tile_row, ntiles, p, pool, tiles, blk_cnt);
  if (tile_ev1) cudaEventRecord(tile_ev1, s);
  if (fused) {
    const FusedStitch fs = {row_done, segcnt, cnt, out, parts, flags_in, flags_out};
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((nseg * 32 + 255) / 256);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = tile_ev1 ? 0 : 1;  // (profiled: no overlap with the timed tile kernel)
    cudaLaunchKernelEx(&cfg, stitch_fused_kernel, segs, nseg, rows, (const TileSum*)tiles, p, (RunPair*)segsum, fs);
    return;
  }
  if (p.block_words && nblocks)
    block_eval_kernel<<<grid_for(nblocks, 256, 148 * 8), 256, 0, s>>>(rows, nrows, nblocks, blk_cnt,
                                                                    p.block_words, p.thr, cnt);
  stitch_seg_kernel<<<(nseg * 32 + 255) / 256, 256, 0, s>>>(segs, nseg, tiles, p.min_run,
                                                             (RunPair*)segsum, cnt);
  stitch_row_finalize_kernel<<<(nrows * 32 + 255) / 256, 256, 0, s>>>(rows, nrows, (const RunPair*)segsum,
                                                                       p, cnt, out, parts, blk_cnt);
}

void launch_pages(cudaStream_t s, const PageRow* rows, uint32_t nrows, uint64_t npages, uint64_t page_words,
                  const uint32_t* pool, uint8_t* flags, unsigned long long* cnt) {
  if (!npages || !nrows) return;
  const uint64_t warps = npages < 148ull * 64 ? npages : 148ull * 64;  // <= 8 pages' chunk per warp at small n
  page_kernel<<<(unsigned)((warps + 7) / 8), 256, 0, s>>>(rows, nrows, npages, page_words, pool, flags, cnt);
}

void launch_fill_u32(cudaStream_t s, uint32_t* p, uint64_t n, uint32_t v) {
  fill_u32_kernel<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(p, n, v);
}

}  // namespace xpl
