// kernels.cu -- sm_100a kernels of the XPlacer runtime (everything but the
// inlined device hooks, which live in include/xpl_device.cuh).
//
//   fold          epoch close: pending GPU writes become "last writer = GPU"
//                 (snapshot semantics D5), O(dirty u32s)
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
// fold: for every shadow u32 in the dirty list, P -> L=1 and clear P.  If the
// list overflowed during the epoch, scan the whole pool instead.  The last CTA
// to finish resets the list for the next epoch (no host round trip).
__global__ void __launch_bounds__(256) fold_kernel(uint32_t* __restrict__ pool,
                                                   uint64_t pool_u32,
                                                   const uint32_t* __restrict__ dirty,
                                                   uint32_t* dirty_count, uint32_t cap,
                                                   uint32_t* done_ctr,
                                                   unsigned long long* stats) {
  const uint32_t n = *((volatile uint32_t*)dirty_count);
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  if (n <= cap) {
    for (uint64_t i = tid; i < n; i += stride) {
      const uint32_t q = dirty[i];
      const uint32_t v = pool[q];
      const uint32_t p = v & kP4;
      pool[q] = (v & ~kP4) | (p >> 1);
    }
  } else {
    uint4* p4 = reinterpret_cast<uint4*>(pool);
    for (uint64_t i = tid; i < pool_u32 / 4; i += stride) {
      uint4 v = p4[i];
      if ((v.x | v.y | v.z | v.w) & kP4) {
        v.x = (v.x & ~kP4) | ((v.x & kP4) >> 1);
        v.y = (v.y & ~kP4) | ((v.y & kP4) >> 1);
        v.z = (v.z & ~kP4) | ((v.z & kP4) >> 1);
        v.w = (v.w & ~kP4) | ((v.w & kP4) >> 1);
        p4[i] = v;
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t t = atomicAdd(done_ctr, 1u);
    if (t == gridDim.x - 1) {
      if (n > stats[0]) stats[0] = n;
      if (n > cap) stats[1] += 1;
      stats[2] += 1;
      stats[3] += n <= cap ? n : pool_u32;
      *dirty_count = 0;
      *done_ctr = 0;
      __threadfence();
    }
  }
}

// ---------------------------------------------------------------------------
// Host merge.  A batch of host records is one ordered stream (D7b).  Per word:
// a read before the first write of the batch sees the batch-start last writer;
// a read after it sees the CPU; any write sets wC and makes the CPU the last
// writer.  Pass 1 finds each word's first writing record
// (atomicMin of the record index), pass 2 sets read/write bits, pass 3 clears L
// of written words and resets the scratch.

__global__ void merge_firstw_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                    uint32_t* __restrict__ fw) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint64_t r = recs[i];
    if (!(rec_acc(r) & XPL_ACC_W)) continue;
    const uint64_t g0 = rec_g0(r), nw = rec_nw(r);
    for (uint64_t w = g0; w < g0 + nw; ++w) atomicMin(fw + w, i);
  }
}

__global__ void merge_apply_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                   const uint32_t* __restrict__ fw, uint32_t* pool) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint64_t r = recs[i];
    const uint32_t acc = rec_acc(r);
    const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
    for (uint64_t q = g0 >> 2; q <= (g1 >> 2); ++q) {
      const uint32_t cur = pool[q];  // L bits do not change during this kernel
      uint32_t m = 0;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint64_t w = q * 4 + k;
        if (w < g0 || w > g1) continue;
        uint32_t b = 0;
        if (acc & XPL_ACC_R) {
          const bool before = (fw == nullptr) || i <= fw[w];
          b = before ? (((cur >> (8 * k)) & 1u) ? kRGC : kRCC) : kRCC;
        }
        if (acc & XPL_ACC_W) b |= kWC;
        m |= b << (8 * k);
      }
      if ((cur & m) != m) atomicOr(pool + q, m);
    }
  }
}

__global__ void merge_clear_kernel(const uint64_t* __restrict__ recs, uint32_t n,
                                   uint32_t* __restrict__ fw, uint32_t* pool) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint64_t r = recs[i];
    if (!(rec_acc(r) & XPL_ACC_W)) continue;
    const uint64_t g0 = rec_g0(r), g1 = g0 + rec_nw(r) - 1;
    for (uint64_t q = g0 >> 2; q <= (g1 >> 2); ++q) {
      uint32_t lm = 0;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint64_t w = q * 4 + k;
        if (w >= g0 && w <= g1) lm |= kL << (8 * k);
      }
      if (pool[q] & lm) atomicAnd(pool + q, ~lm);
    }
    if (fw)
      for (uint64_t w = g0; w <= g1; ++w) fw[w] = 0xFFFFFFFFu;
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
                                                    uint32_t* dirty, uint32_t* dirty_count,
                                                    uint32_t dirty_cap) {
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
        if (r.acc & XPL_ACC_W) m |= 0x0A0A0A0Au & bms[c];
        if ((in[c] & m) == m) continue;
        const uint32_t q = (uint32_t)(vi * 4 + c);
        const uint32_t old = atomicOr(pool + q, m);
        if ((m & kP4) && !(old & kP4)) {
          const uint32_t i = atomicAdd(dirty_count, 1u);
          if (i < dirty_cap) dirty[i] = q;
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
__device__ __forceinline__ RunSum warp_runs(uint32_t m, uint32_t lane, uint32_t min_run) {
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
// ones seen at bit position j.  32 words per lane per tile -> 6 planes.
struct VCount {
  uint32_t p0 = 0, p1 = 0, p2 = 0, p3 = 0, p4 = 0, p5 = 0;
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
    p5 ^= t3;
  }
  __device__ __forceinline__ uint32_t count(uint32_t mask) const {
    return __popc(p0 & mask) + 2 * __popc(p1 & mask) + 4 * __popc(p2 & mask) +
           8 * __popc(p3 & mask) + 16 * __popc(p4 & mask) + 32 * __popc(p5 & mask);
  }
};

// Per-byte flags, 0x80 in each byte where the predicate holds.
__device__ __forceinline__ uint32_t derived_flags(uint32_t x) {
  const uint32_t cpu = ((x & 0x34343434u) + 0x7F7F7F7Fu) & 0x80808080u;  // wC|rCC|rGC
  const uint32_t gpu = (((x & 0x48484848u) + 0x7F7F7F7Fu) | x) & 0x80808080u;  // wG|rCG|rGG
  const uint32_t wr = ((x & 0x0C0C0C0Cu) + 0x7F7F7F7Fu) & 0x80808080u;  // wC|wG
  const uint32_t any = cpu | gpu;
  const uint32_t alt = cpu & gpu & wr;
  return any | (gpu >> 1) | (alt >> 2);  // bit7 any, bit6 gpu, bit5 alternating
}

__global__ void __launch_bounds__(kDiagThreads) diag_tile_kernel(
    const DiagRow* __restrict__ rows, const uint32_t* __restrict__ tile_row, DiagParams p,
    uint32_t* __restrict__ pool, unsigned long long* __restrict__ cnt, TileSum* __restrict__ tiles,
    uint32_t* __restrict__ blk_cnt) {
  __shared__ uint32_t s_cnt[kDiagThreads / 32][9];
  __shared__ RunSum s_u[kDiagThreads / 32], s_d[kDiagThreads / 32];
  const uint64_t t = blockIdx.x;
  const uint32_t ri = tile_row[t];
  const DiagRow row = rows[ri];
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint64_t tw0 = (t - row.tile0) * kTileWords;
  const uint64_t ww0 = tw0 + (uint64_t)warp * (kTileWords / (kDiagThreads / 32));
  const uint32_t min_run = (uint32_t)(p.min_run < 0xFFFFFFFFull ? p.min_run : 0xFFFFFFFFull);
  uint4* p4 = reinterpret_cast<uint4*>(pool);

  uint4 v[kDiagIters];
#pragma unroll
  for (uint32_t it = 0; it < kDiagIters; ++it) {
    const uint64_t w = ww0 + it * 512 + lane * 16;
    v[it] = w < row.words ? p4[(row.off + w) >> 4] : make_uint4(0, 0, 0, 0);
  }

  VCount raw, der;
  RunSum wu = {0, 0, 0, 0, 0}, wd = {0, 0, 0, 0, 0};
#pragma unroll
  for (uint32_t it = 0; it < kDiagIters; ++it) {
    const uint64_t w = ww0 + it * 512 + lane * 16;
    uint32_t x[4] = {v[it].x, v[it].y, v[it].z, v[it].w};
    uint32_t bm[4] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu};
    if (w + 16 > row.words) {  // tail of the row (or beyond it): mask the words
#pragma unroll
      for (uint32_t c = 0; c < 4; ++c) {
        uint32_t m = 0;
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k)
          if (w + c * 4 + k < row.words) m |= 0xFFu << (8 * k);
        bm[c] = m;
        x[c] &= m;
      }
    }
    raw.add4(x[0], x[1], x[2], x[3]);
    const uint32_t f0 = derived_flags(x[0]), f1 = derived_flags(x[1]), f2 = derived_flags(x[2]),
                   f3 = derived_flags(x[3]);
    der.add4(f0, f1, f2, f3);

    // transfer runs: u = wC & !rCG at bit 2, d = rCC at bit 4
    uint32_t uu[4], dd[4];
#pragma unroll
    for (uint32_t c = 0; c < 4; ++c) {
      uu[c] = x[c] & ~(x[c] >> 4) & 0x04040404u;
      dd[c] = x[c] & 0x10101010u;
    }
    const uint32_t uor = uu[0] | uu[1] | uu[2] | uu[3];
    const uint32_t uand = uu[0] & uu[1] & uu[2] & uu[3];
    const uint32_t dor = dd[0] | dd[1] | dd[2] | dd[3];
    const uint32_t dand = dd[0] & dd[1] & dd[2] & dd[3];
    RunSum su, sd;
    const unsigned any_u = __ballot_sync(0xFFFFFFFFu, uor != 0);
    const unsigned full_u = __ballot_sync(0xFFFFFFFFu, uand == 0x04040404u);
    if (any_u == 0) su = {512, 0, 0, 0, 0};
    else if (full_u == 0xFFFFFFFFu) su = {512, 512, 512, 0, 0};
    else {
      const uint32_t m = pack4(uu[0] >> 2) | (pack4(uu[1] >> 2) << 4) | (pack4(uu[2] >> 2) << 8) |
                         (pack4(uu[3] >> 2) << 12);
      su = warp_runs(m, lane, min_run);
    }
    const unsigned any_d = __ballot_sync(0xFFFFFFFFu, dor != 0);
    const unsigned full_d = __ballot_sync(0xFFFFFFFFu, dand == 0x10101010u);
    if (any_d == 0) sd = {512, 0, 0, 0, 0};
    else if (full_d == 0xFFFFFFFFu) sd = {512, 512, 512, 0, 0};
    else {
      const uint32_t m = pack4(dd[0] >> 4) | (pack4(dd[1] >> 4) << 4) | (pack4(dd[2] >> 4) << 8) |
                         (pack4(dd[3] >> 4) << 12);
      sd = warp_runs(m, lane, min_run);
    }
    wu = rs_combine(wu, su, min_run);
    wd = rs_combine(wd, sd, min_run);

    // density blocks when block_words > 0
    if (p.block_words && w < row.words) {
      const uint64_t B = p.block_words;
      const uint32_t g = ((f0 >> 6) & kL4) | (((f1 >> 6) & kL4) << 1) |
                         (((f2 >> 6) & kL4) << 2) | (((f3 >> 6) & kL4) << 3);
      // bit (c + 8k) of g = gpu flag of word 4c + k; build the word-ordered 16-bit mask
      uint32_t gm = 0;
#pragma unroll
      for (uint32_t c = 0; c < 4; ++c)
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k) gm |= ((g >> (8 * k + c)) & 1u) << (4 * c + k);
      if (gm) {
        uint64_t a = w;
        const uint64_t e = w + 16;
        while (a < e) {
          const uint64_t k = a / B;
          const uint64_t be = (k + 1) * B < e ? (k + 1) * B : e;
          const uint32_t lo = (uint32_t)(a - w), hi = (uint32_t)(be - w);
          const uint32_t seg = ((hi >= 32 ? 0xFFFFFFFFu : ((1u << hi) - 1u)) & ~((1u << lo) - 1u));
          const uint32_t c = __popc(gm & seg);
          if (c) atomicAdd(blk_cnt + row.blk0 + k, c);
          a = be;
        }
      }
    }

    // fused reset (D4): keep L only
    if (p.reset && w < row.words) {
      const uint32_t y[4] = {v[it].x, v[it].y, v[it].z, v[it].w};
      uint32_t n[4];
      bool ch = false;
#pragma unroll
      for (uint32_t c = 0; c < 4; ++c) {
        n[c] = y[c] & (~bm[c] | kL4);
        ch = ch || n[c] != y[c];
      }
      if (ch) p4[(row.off + w) >> 4] = make_uint4(n[0], n[1], n[2], n[3]);
    }
  }

  // counters: 6 raw bit classes + any/gpu/alternating
  uint32_t c9[9];
  c9[0] = raw.count(0x04040404u);  // wC
  c9[1] = raw.count(0x08080808u);  // wG
  c9[2] = raw.count(0x10101010u);  // rCC
  c9[3] = raw.count(0x40404040u);  // rCG
  c9[4] = raw.count(0x20202020u);  // rGC
  c9[5] = raw.count(0x80808080u);  // rGG
  c9[6] = der.count(0x80808080u);  // any
  c9[7] = der.count(0x40404040u);  // gpu
  c9[8] = der.count(0x20202020u);  // alternating
#pragma unroll
  for (int k = 0; k < 9; ++k) {
    const uint32_t s = __reduce_add_sync(0xFFFFFFFFu, c9[k]);
    if (lane == 0) s_cnt[warp][k] = s;
  }
  if (lane == 0) {
    s_u[warp] = wu;
    s_d[warp] = wd;
  }
  __syncthreads();
  if (threadIdx.x < 9) {
    uint32_t s = 0;
    for (uint32_t w = 0; w < kDiagThreads / 32; ++w) s += s_cnt[w][threadIdx.x];
    if (s) atomicAdd(cnt + (uint64_t)ri * C_NCNT + threadIdx.x, (unsigned long long)s);
  } else if (threadIdx.x == 32) {
    RunSum a = s_u[0], b = s_d[0];
    for (uint32_t w = 1; w < kDiagThreads / 32; ++w) {
      a = rs_combine(a, s_u[w], min_run);
      b = rs_combine(b, s_d[w], min_run);
    }
    tiles[t].u = a;
    tiles[t].d = b;
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

// One warp per row: ordered combine of the row's tile summaries.
__global__ void stitch_kernel(const DiagRow* __restrict__ rows, uint32_t nrows,
                              const TileSum* __restrict__ tiles, uint64_t min_run,
                              unsigned long long* __restrict__ cnt) {
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  if (gw >= nrows) return;
  const DiagRow row = rows[gw];
  const uint64_t per = (row.ntiles + 31) / 32;
  const uint64_t t0 = row.tile0 + lane * per;
  const uint64_t t1 = min(row.tile0 + row.ntiles, t0 + per);
  RunSum64 a = {0, 0, 0, 0, 0}, b = {0, 0, 0, 0, 0};
  for (uint64_t t = t0; t < t1; ++t) {
    const RunSum u = tiles[t].u, d = tiles[t].d;
    a = rs_combine(a, RunSum64{u.len, u.pre, u.suf, u.cnt, u.sum}, min_run);
    b = rs_combine(b, RunSum64{d.len, d.pre, d.suf, d.cnt, d.sum}, min_run);
  }
  for (uint32_t s = 1; s < 32; s <<= 1) {
    RunSum64 oa, ob;
    oa.len = __shfl_down_sync(0xFFFFFFFFu, a.len, s);
    oa.pre = __shfl_down_sync(0xFFFFFFFFu, a.pre, s);
    oa.suf = __shfl_down_sync(0xFFFFFFFFu, a.suf, s);
    oa.cnt = __shfl_down_sync(0xFFFFFFFFu, a.cnt, s);
    oa.sum = __shfl_down_sync(0xFFFFFFFFu, a.sum, s);
    ob.len = __shfl_down_sync(0xFFFFFFFFu, b.len, s);
    ob.pre = __shfl_down_sync(0xFFFFFFFFu, b.pre, s);
    ob.suf = __shfl_down_sync(0xFFFFFFFFu, b.suf, s);
    ob.cnt = __shfl_down_sync(0xFFFFFFFFu, b.cnt, s);
    ob.sum = __shfl_down_sync(0xFFFFFFFFu, b.sum, s);
    if ((lane & (2 * s - 1)) == 0 && lane + s < 32) {
      a = rs_combine(a, oa, min_run);
      b = rs_combine(b, ob, min_run);
    }
  }
  if (lane == 0) {
    uint64_t r, w;
    unsigned long long* c = cnt + (uint64_t)gw * C_NCNT;
    run_final(a, min_run, &r, &w);
    c[C_UR] = r;
    c[C_UW] = w;
    run_final(b, min_run, &r, &w);
    c[C_DR] = r;
    c[C_DW] = w;
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
    const uint64_t k = j - r.blk0;
    const uint64_t s = min(B, r.words - k * B);
    if (100ull * g <= (uint64_t)thr * s) {
      atomicAdd(cnt + (uint64_t)lo * C_NCNT + C_LDB, 1ull);
      atomicAdd(cnt + (uint64_t)lo * C_NCNT + C_LDW, (unsigned long long)s);
    }
  }
}

__global__ void finalize_kernel(const DiagRow* __restrict__ rows, uint32_t nrows, DiagParams p,
                                const unsigned long long* __restrict__ cnt,
                                xpl_alloc_report* __restrict__ out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nrows) return;
  const DiagRow r = rows[i];
  const unsigned long long* c = cnt + (uint64_t)i * C_NCNT;
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
  o.h2d_unused_runs = c[C_UR];
  o.h2d_unused_words = c[C_UW];
  o.d2h_unneeded_runs = c[C_DR];
  o.d2h_unneeded_words = c[C_DW];
  o.ever_accessed = 0;
  uint32_t f = 0;
  if (r.kind == XPL_ALLOC_MANAGED && o.alternating > 0) f |= XPL_PAT_ALTERNATING;
  if (r.kind != XPL_ALLOC_HOST && o.low_density_blocks > 0) f |= XPL_PAT_LOW_DENSITY;
  if (r.kind == XPL_ALLOC_DEVICE && o.h2d_unused_runs > 0) f |= XPL_PAT_UNNEEDED_H2D;
  if (r.kind == XPL_ALLOC_DEVICE && o.d2h_unneeded_runs > 0) f |= XPL_PAT_UNNEEDED_D2H;
  if (o.any_acc == 0) f |= XPL_PAT_UNUSED;
  o.flags = f;
  out[i] = o;
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

}  // namespace

void launch_fold(cudaStream_t s, uint32_t* pool, uint64_t pool_u32, const uint32_t* dirty,
                 uint32_t* dirty_count, uint32_t dirty_cap, uint32_t* done_ctr,
                 unsigned long long* stats) {
  fold_kernel<<<148, 256, 0, s>>>(pool, pool_u32, dirty, dirty_count, dirty_cap, done_ctr, stats);
}

void launch_merge(cudaStream_t s, const uint64_t* recs, uint32_t n, bool has_r, bool has_w,
                  uint32_t* first_w, uint32_t* pool) {
  const int g = grid_for(n, 256, 148 * 16);
  const bool both = has_r && has_w;
  if (both) merge_firstw_kernel<<<g, 256, 0, s>>>(recs, n, first_w);
  merge_apply_kernel<<<g, 256, 0, s>>>(recs, n, both ? first_w : nullptr, pool);
  if (has_w) merge_clear_kernel<<<g, 256, 0, s>>>(recs, n, both ? first_w : nullptr, pool);
}

void launch_range(cudaStream_t s, const RangeDesc* d_ranges, uint32_t nr, uint64_t nvec,
                  uint32_t* pool, uint32_t* dirty, uint32_t* dirty_count, uint32_t dirty_cap) {
  const int g = grid_for(nvec, 256, 148 * 8);
  range_kernel<<<g, 256, 0, s>>>(d_ranges, nr, nvec, pool, dirty, dirty_count, dirty_cap);
}

void launch_diag(cudaStream_t s, const DiagRow* rows, uint32_t nrows, const uint32_t* tile_row,
                 uint64_t ntiles, uint64_t nblocks, const DiagParams& p, uint32_t* pool,
                 unsigned long long* cnt, TileSum* tiles, uint32_t* blk_cnt,
                 xpl_alloc_report* out, cudaEvent_t tile_ev0, cudaEvent_t tile_ev1) {
  cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * C_NCNT * nrows, s);
  if (p.block_words && nblocks) cudaMemsetAsync(blk_cnt, 0, sizeof(uint32_t) * nblocks, s);
  if (tile_ev0) cudaEventRecord(tile_ev0, s);
  if (ntiles) diag_tile_kernel<<<(unsigned)ntiles, kDiagThreads, 0, s>>>(rows, tile_row, p, pool, cnt, tiles, blk_cnt);
  if (tile_ev1) cudaEventRecord(tile_ev1, s);
  stitch_kernel<<<(nrows * 32 + 255) / 256, 256, 0, s>>>(rows, nrows, tiles, p.min_run, cnt);
  if (p.block_words && nblocks)
    block_eval_kernel<<<grid_for(nblocks, 256, 148 * 8), 256, 0, s>>>(rows, nrows, nblocks, blk_cnt,
                                                                    p.block_words, p.thr, cnt);
  finalize_kernel<<<(nrows + 127) / 128, 128, 0, s>>>(rows, nrows, p, cnt, out);
}

void launch_fill_u32(cudaStream_t s, uint32_t* p, uint64_t n, uint32_t v) {
  fill_u32_kernel<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(p, n, v);
}

}  // namespace xpl
