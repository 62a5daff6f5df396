// xpl_internal.h -- private declarations shared by runtime.cu and kernels.cu.
// (CUDA path only; the oracle never sees this file.)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "xpl.h"
#include "xpl_device.cuh"

namespace xpl {

// Record byte (P:L243 + the pending bit): see include/xpl_device.cuh.
constexpr uint32_t kL = 0x01, kP = 0x02, kWC = 0x04, kWG = 0x08, kRCC = 0x10, kRGC = 0x20,
                   kRCG = 0x40, kRGG = 0x80;

// Packed host record (8 B): bits [0,38) first pool word g0, [38,62) nwords-1,
// [62,64) acc (R=1, W=2, RW=3).  The host runtime has already looked the address
// up and clipped it to its allocation (D18).
constexpr int kG0Bits = 38;
constexpr uint64_t kG0Mask = (1ull << kG0Bits) - 1;
constexpr uint64_t kMaxRecWords = 1ull << 24;
__host__ __device__ inline uint64_t pack_rec(uint64_t g0, uint64_t nw, uint32_t acc) {
  return g0 | ((nw - 1) << kG0Bits) | ((uint64_t)acc << 62);
}
__host__ __device__ inline uint64_t rec_g0(uint64_t r) { return r & kG0Mask; }
__host__ __device__ inline uint64_t rec_nw(uint64_t r) { return ((r >> kG0Bits) & (kMaxRecWords - 1)) + 1; }
__host__ __device__ inline uint32_t rec_acc(uint64_t r) { return (uint32_t)(r >> 62); }

// Records of more than kBigRange words are "ranges" and go through range_apply
// (2 B/word, cutting the batch into segments); shorter ones are merged, split
// into pieces of at most kPieceWords (one thread each, program order kept).
constexpr uint64_t kRangeWords = 65536;  // (kBigRange)
constexpr uint64_t kPieceWords = 256;

// A range for the vectorised range kernels (host transfers, D2D/memset).
struct RangeDesc {
  uint64_t g0, nw;     // first pool word, number of words
  uint64_t vbase;      // prefix sum of the 16-word vectors the ranges touch
  uint32_t acc, side;  // side 0 = CPU, 1 = GPU
};

// Diagnose geometry.
constexpr uint32_t kTileWords = 16384;         // max words per diagnose tile (one warp)
constexpr uint32_t kMinTileWords = 2048;       // min: small diagnoses use smaller tiles (more warps)
constexpr uint32_t kDiagIters = kTileWords / 512;  // max 512-word steps per tile (32 lanes x 16 words)
constexpr uint32_t kDiagThreads = 256;         // 8 independent warps (tiles) per CTA

struct DiagRow {        // one row to analyse (live or dead-since-last-reset)
  uint64_t off, words;  // pool offset (multiple of 16), words
  uint64_t tile0;       // first tile index of this row
  uint64_t ntiles;
  uint64_t blk0;        // first block-counter index (block_words > 0)
  uint64_t nblk;
  uint64_t seg0, nseg;  // its stitch segments
  uint64_t goff;        // first logical word (pieces of a sharded allocation; else 0)
  uint64_t lwords;      // logical words (== words unless sharded)
  uint32_t kind, pad;
};

// What a row contributes to a sharded diagnosis besides its counters.
struct RowPartial {
  uint64_t u[5], d[5];             // run summaries (len, pre, suf, cnt, sum)
  uint64_t blk_first_g, blk_last_g;  // GPU words of the first / last block of the row
};

// Stitch segment: <= kSegTiles consecutive tiles of one row.
constexpr uint64_t kSegTiles = 128;
struct StitchSeg {
  uint64_t t0, n;
  uint64_t row;  // the row (report index) the segment belongs to
};

// Per-row counters accumulated by the diagnose kernels (u64 each).
enum Cnt {
  C_WC, C_WG, C_RCC, C_RCG, C_RGC, C_RGG, C_ANY, C_GPU, C_ALT,
  C_LDB, C_LDW, C_UR, C_UW, C_DR, C_DW, C_NCNT
};

// Run summary of a predicate over a contiguous word range (see kernels.cu).
struct RunSum {
  uint32_t len, pre, suf, cnt, sum;
};
struct TileSum {
  RunSum u, d;      // u = wC & !rCG (unneeded H2D), d = rCC (unneeded D2H)
  uint32_t cnt[9];  // wC wG rCC rCG rGC rGG any gpu alternating (C_WC .. C_ALT)
  uint32_t pad;
};

struct DiagParams {
  uint32_t thr;
  uint32_t reset;
  uint64_t block_words;
  uint64_t min_run;
  uint32_t tile_words;  // this call's tile size (power of two in [kMinTileWords, kTileWords])
  uint32_t pad;
};

// ---- launchers (kernels.cu) ----
void launch_fold(cudaStream_t s, bool pdl, uint32_t* pool, uint8_t* cmap, uint8_t* smap,
                 uint64_t n_super, unsigned long long* stats, uint32_t* flags, int strict, int force);
void launch_merge(cudaStream_t s, const uint64_t* recs, uint32_t n, bool has_r, bool has_w,
                  uint32_t* first_w, uint64_t fw0, uint32_t* pool);
void launch_range(cudaStream_t s, const RangeDesc* d_ranges, uint32_t nr, uint64_t nvec,
                  uint32_t* pool, uint8_t* cmap, uint8_t* smap, uint32_t* flags);
void launch_diag(cudaStream_t s, const DiagRow* rows, uint32_t nrows, const uint32_t* tile_row,
                 uint64_t ntiles, const StitchSeg* segs, uint32_t nseg, uint64_t nblocks,
                 const DiagParams& p, uint32_t* pool, unsigned long long* cnt, TileSum* tiles,
                 void* segsum, uint32_t* blk_cnt, xpl_alloc_report* out, RowPartial* parts,
                 cudaEvent_t tile_ev0, cudaEvent_t tile_ev1, uint32_t* row_done, unsigned long long* segcnt,
                 const uint32_t* flags_in, uint32_t* flags_out);
// row_done: nrows zero u32s (row done counters, left zero), or null for the
// separate stitch kernels; segcnt: 9 u64 per segment.  Fused, the stitch kernel
// may write out / parts / cnt and flags_out (<- flags_in[0..1]) straight into
// pinned host memory (unified addressing): no copies back.
constexpr size_t kRunPairBytes = 80;  // sizeof(RunPair) in kernels.cu
struct PageRow {  // one live row of a page pass (NEXT-3)
  uint64_t off, words, page0;  // pool word offset, words, first global page index
};
void launch_pages(cudaStream_t s, const PageRow* rows, uint32_t nrows, uint64_t npages, uint64_t page_words,
                  const uint32_t* pool, uint8_t* flags, unsigned long long* cnt);
void launch_fill_u32(cudaStream_t s, uint32_t* p, uint64_t n, uint32_t v);

}  // namespace xpl
