// runtime.cu -- host side of the B200-native XPlacer runtime: the C-ABI of
// include/xpl.h.  Owns the shadow memory table, the shadow pool,
// the epoch state machine around kernel launches, host-record staging
// with run-length coalescing (host tracer) and the diagnose driver
// (tracePrint).  Every data-parallel step runs in kernels.cu or in the
// inlined hooks of xpl_device.cuh; this file only orders and launches them.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <array>
#include <map>
#include <new>
#include <string>
#include <unordered_map>
#include <vector>

#include <nvtx3/nvToolsExt.h>  // (header-only NVTX 3: ranges cost nothing without a tool attached)

#include "xpl_internal.h"

using namespace xpl;

namespace {
// An NVTX range over one runtime call (nsight / ncu timelines show the
// runtime's host work next to its kernels).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace

#define CK(x)                                      \
  do {                                             \
    if ((x) != cudaSuccess) return XPL_ERR_CUDA;   \
  } while (0)

namespace {

struct Row {
  uint64_t id, base, bytes, words, off, span;  // span = pool words reserved
  uint64_t logical_id, goff, lbytes;           // sharded pieces (else id, 0, bytes)
  uint32_t kind;
  bool live, dropped, ever;
  uint32_t advice = 0;  // XPL_ADVICE_* bits (xpl_mem_advise)
  uint32_t owner = 0;   // rank whose pool holds the shadow (sharded mode; else 0)
};

// First-fit allocator of shadow-pool ranges (16-word granules so every row
// starts on a 16-byte boundary for the vector loads of diagnose).
struct PoolAlloc {
  std::map<uint64_t, uint64_t> free_;  // off -> len
  uint64_t hwm = 0;                    // high-water mark: no row ever extended past it
  void init(uint64_t cap) { free_.clear(); free_[0] = cap; hwm = 0; }
  bool alloc(uint64_t n, uint64_t* off) {
    for (auto it = free_.begin(); it != free_.end(); ++it) {
      if (it->second >= n) {
        *off = it->first;
        if (it->first + n > hwm) hwm = it->first + n;
        const uint64_t rest = it->second - n, o = it->first + n;
        free_.erase(it);
        if (rest) free_[o] = rest;
        return true;
      }
    }
    return false;
  }
  void release(uint64_t off, uint64_t n) {
    auto it = free_.emplace(off, n).first;
    auto nx = std::next(it);
    if (nx != free_.end() && it->first + it->second == nx->first) {
      it->second += nx->second;
      free_.erase(nx);
    }
    if (it != free_.begin()) {
      auto pv = std::prev(it);
      if (pv->first + pv->second == it->first) {
        pv->second += it->second;
        free_.erase(it);
      }
    }
  }
};

template <class T>
cudaError_t host_alloc(T** p, size_t n) {
  return cudaMallocHost((void**)p, sizeof(T) * (n ? n : 1));
}

}  // namespace

struct xpl_ctx {
  xpl_config cfg;
  cudaStream_t rs = nullptr;  // the runtime's own stream
  // The stream the runtime's latest work is on: rs, or the stream of the last
  // single-stream epoch (its fold was enqueued right behind the epoch's kernels,
  // so the next epoch on that stream needs no cross-stream event).  Every
  // runtime enqueue goes to cs; switching streams always goes through an event.
  cudaStream_t cs = nullptr;

  // shadow pool: 1 byte per word
  uint8_t* d_pool = nullptr;
  uint64_t pool_words = 0;
  // every rank's pool allocator: in sharded mode all ranks replay the same
  // registrations and frees, so each computes every piece's offset identically
  std::vector<PoolAlloc> pas;

  // sharded mode (world > 1, xpl.h): collectives, routing lists, peer pools
  int rank = 0, world = 1;
  const xpl_comm* comm = nullptr;
  std::vector<std::vector<uint64_t>> route;  // staged host records per owner rank
  uint64_t n_logical = 0;                    // logical ids handed out by xpl_register_alloc
  std::unordered_map<uint64_t, std::vector<uint64_t>> lrows;  // logical id -> its rows (pieces)
  void* peer_pool[XPL_MAX_RANKS] = {};       // IPC-mapped pools / chunk maps of the other ranks
  void* peer_cmap[XPL_MAX_RANKS] = {};
  void* peer_smap[XPL_MAX_RANKS] = {};
  bool ready = false;                        // xpl_init completed
  uint32_t* d_first_w = nullptr;  // merge scratch (first writer per word of a batch's span), grown lazily
  uint64_t first_w_cap = 0;

  // shadow memory table
  std::vector<Row> rows;               // by id
  std::vector<uint64_t> active;        // ids of the rows a diagnose reports (live, or freed since the
                                       // last reset), ascending: the walks below skip dropped rows
  std::map<uint64_t, uint64_t> live;   // base -> id
  uint32_t n_dead = 0;
  uint8_t* d_tab = nullptr;            // [u32 n | pad to 32 B | xpl_dev_row[max_rows]]
  uint8_t* h_tab = nullptr;
  bool table_dirty = true;
  cudaEvent_t table_ev = nullptr;
  const Row* cache = nullptr;          // last host lookup hit

  // epoch close: chunk maps (1 B per 128 words, 1 B per 16K words) + chunk list
  uint8_t* d_cmap = nullptr;           // 1 byte per 128-word chunk: GPU write pending
  uint8_t* d_smap = nullptr;           // 1 byte per 16K-word super-chunk
  uint32_t* d_misc = nullptr;          // [0] split seen in the open epoch, [1] split in a forbidden epoch
  uint32_t* h_misc = nullptr;          // pinned mirror of d_misc (read back with the diagnose copies)
  unsigned long long* d_stats = nullptr;

  // epochs (D19)
  int depth = 0;
  std::vector<cudaStream_t> epoch_streams;  // streams that joined the open epoch
  std::vector<cudaEvent_t> ev_pool;
  cudaEvent_t ev_begin = nullptr;
  bool ev_begin_valid = false;       // ev_begin recorded on cs for this epoch
  bool cs_in_epoch = false;          // runtime work (D2D / memset) enqueued inside the epoch
  cudaEvent_t ev_join = nullptr;

  // host-record staging (8-byte packed records)
  uint64_t* h_stage[2] = {nullptr, nullptr};
  cudaEvent_t stage_ev[2] = {nullptr, nullptr};
  int cur = 0;
  size_t stage_n = 0, stage_cap = 0, stage_ranges = 0;
  bool stage_has_r = false, stage_has_w = false;
  uint64_t* d_stage = nullptr;
  std::vector<std::pair<uint32_t, uint64_t>> deferred;  // (owner, record) inside an open epoch (D20)

  // merge pieces (records split to <= kPieceWords words)
  uint64_t* h_pieces = nullptr;
  uint64_t* d_pieces = nullptr;
  size_t pieces_cap = 0;
  cudaEvent_t pieces_ev = nullptr;

  // range descriptors
  RangeDesc* h_ranges = nullptr;
  RangeDesc* d_ranges = nullptr;
  size_t ranges_cap = 0;
  cudaEvent_t ranges_ev = nullptr;

  // diagnose buffers (grown on demand)
  size_t drows_cap = 0;
  TileSum* d_tiles = nullptr;
  size_t tiles_cap = 0;
  uint32_t* d_blk = nullptr;
  size_t blk_cap = 0;
  void* d_segsum = nullptr;
  unsigned long long* d_segcnt = nullptr;  // fused stitch: 9 counters per segment
  size_t segs_cap = 0;
  uint32_t* d_done = nullptr;  // fused stitch: row done counters (kept zero)
  // one diagnose's upload (row table | tile -> row | segments): one pinned
  // buffer, one device buffer, one copy
  unsigned char* h_up = nullptr;
  unsigned char* d_up = nullptr;
  size_t up_cap = 0;
  size_t done_cap = 0;
  unsigned long long* d_cnt = nullptr;
  xpl_alloc_report* d_rep = nullptr;
  xpl_alloc_report* h_rep = nullptr;
  RowPartial* d_rpart = nullptr;
  RowPartial* h_rpart = nullptr;
  unsigned long long* h_cnt = nullptr;

  xpl_stats st;

  // live kernel timing (xpl_profile)
  struct ProfRec {
    int cls;
    cudaEvent_t a, b;
    uint64_t bytes;
  };
  bool prof = false;
  std::vector<ProfRec> prof_pending;
  std::vector<cudaEvent_t> prof_free;
  xpl_kernel_time prof_acc[XPL_K_NCLASS];
  unsigned long long fold_entries_seen = 0;
  uint64_t folds_host = 0;

  // kernel-launch log (NEXT-4)
  struct EpochRec {
    cudaEvent_t a = nullptr, b = nullptr;  // begin on the epoch's first stream / after its fold
    cudaEvent_t c = nullptr;               // after the end snapshot copy (what a read waits for)
  };
  bool llog = false;
  std::vector<xpl_launch_record> lrecs;
  std::vector<EpochRec> lepochs;           // logged epochs, in order
  std::vector<uint64_t> lepoch_no;         // their epoch numbers
  std::vector<cudaEvent_t> lev_free;
  unsigned long long* h_lcum = nullptr;    // pinned: d_stats[3] (folded chunks) after each logged fold
  size_t lcum_cap = 0;
  bool lepoch_open = false;                // the open epoch has a log entry
  std::vector<std::string> lnames;
  std::unordered_map<std::string, uint32_t> lname_idx;
};

namespace {

// ---------------------------------------------------------------------------
// host lookup: the live row holding addr; nullptr = untracked
const Row* lookup(xpl_ctx* c, uint64_t addr) {
  if (c->cache && addr >= c->cache->base && addr < c->cache->base + c->cache->bytes) return c->cache;
  auto it = c->live.upper_bound(addr);
  if (it == c->live.begin()) return nullptr;
  --it;
  const Row* r = &c->rows[it->second];
  if (addr >= r->base + r->bytes) return nullptr;
  c->cache = r;
  return r;
}

// words [g0, g0+nw) of the access (addr, size), clipped (D1, D18); *owner =
// the rank whose pool holds them (sharded mode; D36: clipped to the piece)
bool to_words(xpl_ctx* c, uint64_t addr, uint64_t size, uint64_t* g0, uint64_t* nw,
              uint32_t* owner = nullptr) {
  if (size == 0) return false;
  const Row* r = lookup(c, addr);
  if (!r) return false;
  if (owner) *owner = r->owner;
  const uint64_t w0 = (addr - r->base) >> 2;
  uint64_t wl = (addr + size - 1 - r->base) >> 2;
  if (wl > r->words - 1) wl = r->words - 1;
  *g0 = r->off + w0;
  *nw = wl - w0 + 1;
  return true;
}

xpl_status flush(xpl_ctx* c);
xpl_status flush_local(xpl_ctx* c);

cudaEvent_t prof_event(xpl_ctx* c) {
  if (!c->prof_free.empty()) {
    cudaEvent_t e = c->prof_free.back();
    c->prof_free.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// Bracket the next launches on the runtime stream (only when profiling).
int prof_begin(xpl_ctx* c, int cls, uint64_t bytes, bool record = true) {
  if (!c->prof) return -1;
  xpl_ctx::ProfRec r{cls, prof_event(c), prof_event(c), bytes};
  if (record) cudaEventRecord(r.a, c->cs);
  c->prof_pending.push_back(r);
  return (int)c->prof_pending.size() - 1;
}
void prof_end(xpl_ctx* c, int i) {
  if (i >= 0) cudaEventRecord(c->prof_pending[i].b, c->cs);
}

uint64_t words_of(const uint64_t* h, size_t n) {
  uint64_t w = 0;
  for (size_t i = 0; i < n; ++i) w += rec_nw(h[i]);
  return w;
}


// Coalesce record (g0, nw, acc) into `last` when that is exact: same access
// kind and touching/overlapping words for R or W (idempotent per word),
// adjacent disjoint words for RW.  Returns whether it did.
bool coalesce(uint64_t& last, uint64_t g0, uint64_t nw, uint32_t acc, bool* became_range) {
  const uint32_t la = rec_acc(last);
  const uint64_t l0 = rec_g0(last), ln = rec_nw(last);
  if (la != acc) return false;
  uint64_t u0 = 0, u1 = 0;
  bool ok = false;
  if (acc != XPL_ACC_RW) {
    if (g0 <= l0 + ln && g0 + nw >= l0) {
      u0 = std::min(g0, l0);
      u1 = std::max(g0 + nw, l0 + ln);
      ok = true;
    }
  } else if (g0 == l0 + ln) {
    u0 = l0;
    u1 = g0 + nw;
    ok = true;
  }
  if (!ok || u1 - u0 > kMaxRecWords) return false;
  *became_range = ln <= kRangeWords && u1 - u0 > kRangeWords;
  last = pack_rec(u0, u1 - u0, acc);
  return true;
}

// Sharded mode: stage a record on its owner's routing list (sent at the next
// collective call).  Lists are per owner, so coalescing with the list's last
// record never reorders accesses of one word.
xpl_status route_push(xpl_ctx* c, uint32_t owner, uint64_t g0, uint64_t nw, uint32_t acc) {
  for (; nw > kMaxRecWords; g0 += kMaxRecWords, nw -= kMaxRecWords) {
    xpl_status s = route_push(c, owner, g0, kMaxRecWords, acc);
    if (s) return s;
  }
  c->st.host_records++;
  std::vector<uint64_t>& L = c->route[owner];
  bool rng = false;
  if (!L.empty() && coalesce(L.back(), g0, nw, acc, &rng)) return XPL_OK;
  L.push_back(pack_rec(g0, nw, acc));
  c->st.host_records_packed++;
  return XPL_OK;
}

// Append one packed record to staging, coalescing with the previous one when
// that is exact (coalesce()).  owner: the rank holding the words (sharded mode).
xpl_status stage_push(xpl_ctx* c, uint64_t g0, uint64_t nw, uint32_t acc, uint32_t owner = 0) {
  if (c->world > 1) return route_push(c, owner, g0, nw, acc);
  while (nw > kMaxRecWords) {  // split very long ranges (disjoint pieces)
    xpl_status s = stage_push(c, g0, kMaxRecWords, acc);
    if (s) return s;
    g0 += kMaxRecWords;
    nw -= kMaxRecWords;
  }
  c->st.host_records++;
  if (c->stage_n) {
    bool rng = false;
    if (coalesce(c->h_stage[c->cur][c->stage_n - 1], g0, nw, acc, &rng)) {
      if (rng) c->stage_ranges++;
      return XPL_OK;
    }
  }
  if (c->stage_n == c->stage_cap) {
    xpl_status s = flush(c);
    if (s) return s;
  }
  c->h_stage[c->cur][c->stage_n++] = pack_rec(g0, nw, acc);
  c->st.host_records_packed++;
  if (nw > kRangeWords) c->stage_ranges++;
  if (acc & XPL_ACC_R) c->stage_has_r = true;
  if (acc & XPL_ACC_W) c->stage_has_w = true;
  return XPL_OK;
}

xpl_status ensure_ranges(xpl_ctx* c, size_t n) {
  if (n <= c->ranges_cap) {
    CK(cudaEventSynchronize(c->ranges_ev));
    return XPL_OK;
  }
  CK(cudaStreamSynchronize(c->cs));
  if (c->h_ranges) cudaFreeHost(c->h_ranges);
  if (c->d_ranges) cudaFree(c->d_ranges);
  size_t cap = std::max<size_t>(n, 1024);
  CK(host_alloc(&c->h_ranges, cap));
  CK(cudaMalloc(&c->d_ranges, sizeof(RangeDesc) * cap));
  c->ranges_cap = cap;
  return XPL_OK;
}

// The merge scratch for a batch of records h[0, n) mixing reads and writes: one
// u32 per pool word of the batch's span [*lo, hi) (not per pool word: 4 B x the
// span, e.g. a host segment over two small allocations); all-ones between uses.
xpl_status ensure_first_w(xpl_ctx* c, const uint64_t* h, size_t n, uint64_t* lo) {
  uint64_t a = ~0ull, b = 0;
  for (size_t i = 0; i < n; ++i) {
    a = std::min(a, rec_g0(h[i]));
    b = std::max(b, rec_g0(h[i]) + rec_nw(h[i]));
  }
  *lo = a;
  const uint64_t span = b > a ? b - a : 1;
  if (span <= c->first_w_cap) return XPL_OK;
  if (c->d_first_w) {
    CK(cudaStreamSynchronize(c->cs));
    cudaFree(c->d_first_w);
  }
  const uint64_t cap = std::max<uint64_t>(span + span / 2, 1 << 16);
  CK(cudaMalloc(&c->d_first_w, sizeof(uint32_t) * cap));
  launch_fill_u32(c->cs, c->d_first_w, cap, 0xFFFFFFFFu);
  c->first_w_cap = cap;
  c->st.kernel_launches += 1;
  return XPL_OK;
}

// Sharded mode: route every rank's staged records to their owners (all-gather
// of the per-owner byte counts, then one all-to-all of the records) and apply
// what this rank received, in source-rank order = the logical host stream's
// order (xpl.h).  COLLECTIVE.
xpl_status route_flush(xpl_ctx* c) {
  const int R = c->world;
  std::vector<uint64_t> sb(R), all((size_t)R * R), rb(R);
  for (int q = 0; q < R; ++q) sb[q] = 8 * c->route[q].size();
  if (c->comm->allgather(c->comm->user, sb.data(), 8 * (size_t)R, all.data())) return XPL_ERR_NCCL;
  uint64_t tot = 0, any = 0;
  for (int q = 0; q < R; ++q) {
    rb[q] = all[(size_t)q * R + c->rank];
    tot += rb[q];
  }
  for (uint64_t v : all) any |= v;
  if (!any) return XPL_OK;  // (every rank sees the same matrix: all skip together)
  std::vector<uint64_t> send;
  for (int q = 0; q < R; ++q) {
    send.insert(send.end(), c->route[q].begin(), c->route[q].end());
    c->route[q].clear();
  }
  std::vector<uint64_t> recv(tot / 8 + 1);
  if (c->comm->alltoallv(c->comm->user, send.data(), sb.data(), recv.data(), rb.data())) return XPL_ERR_NCCL;
  const size_t n = tot / 8;
  for (size_t i = 0; i < n;) {
    const size_t k = std::min(n - i, c->stage_cap);
    memcpy(c->h_stage[c->cur], recv.data() + i, 8 * k);
    c->stage_n = k;
    c->stage_ranges = 0;
    c->stage_has_r = c->stage_has_w = false;
    for (size_t j = 0; j < k; ++j) {
      const uint64_t r = recv[i + j];
      if (rec_acc(r) & XPL_ACC_R) c->stage_has_r = true;
      if (rec_acc(r) & XPL_ACC_W) c->stage_has_w = true;
      if (rec_nw(r) > kRangeWords) c->stage_ranges++;
    }
    xpl_status s = flush_local(c);
    if (s) return s;
    i += k;
  }
  return XPL_OK;
}

xpl_status flush(xpl_ctx* c) {
  if (c->world <= 1 && c->stage_n == 0) return XPL_OK;
  NvtxRange nv("xpl host-record flush");
  return c->world > 1 ? route_flush(c) : flush_local(c);
}

// Apply all staged host records on the runtime stream, in order.  Records of
// more than kRangeWords words cut the batch and go through range_apply (runs of
// pairwise-disjoint ones share a launch); everything between them is one merge
// segment, with records longer than kPieceWords split into consecutive pieces
// (pieces of one record are disjoint, so program order is kept).
xpl_status flush_local(xpl_ctx* c) {
  if (c->stage_n == 0) return XPL_OK;
  const size_t n = c->stage_n;
  uint64_t* h = c->h_stage[c->cur];
  size_t n_pieces = 0, n_long = 0;
  for (size_t i = 0; i < n; ++i) {
    const uint64_t nw = rec_nw(h[i]);
    if (nw > kRangeWords) ++n_long;
    else n_pieces += (nw + kPieceWords - 1) / kPieceWords;
  }
  if (n_long == 0 && n_pieces == n) {  // the common case: one merge segment as staged
    CK(cudaMemcpyAsync(c->d_stage, h, n * sizeof(uint64_t), cudaMemcpyHostToDevice, c->cs));
    CK(cudaEventRecord(c->stage_ev[c->cur], c->cs));
    xpl_status s = XPL_OK;
    uint64_t fw0 = 0;
    if (c->stage_has_r && c->stage_has_w) s = ensure_first_w(c, h, n, &fw0);
    if (s) return s;
    const int pi = prof_begin(c, XPL_K_MERGE, c->prof ? 8 * n + 2 * words_of(h, n) : 0);
    launch_merge(c->cs, c->d_stage, (uint32_t)n, c->stage_has_r, c->stage_has_w, c->d_first_w, fw0,
                 (uint32_t*)c->d_pool);
    prof_end(c, pi);
    c->st.kernel_launches += n <= 8192 ? 1 : 1 + c->stage_has_w + (c->stage_has_r && c->stage_has_w);
    c->st.merge_segments++;
  } else {
    // pieces go to a pinned buffer of their own, uploaded once
    xpl_status s = ensure_ranges(c, n_long);
    if (s) return s;
    if (n_pieces > c->pieces_cap) {
      CK(cudaStreamSynchronize(c->cs));
      cudaFreeHost(c->h_pieces);
      cudaFree(c->d_pieces);
      c->pieces_cap = std::max<size_t>(n_pieces, 1 << 16);
      CK(host_alloc(&c->h_pieces, c->pieces_cap));
      CK(cudaMalloc(&c->d_pieces, sizeof(uint64_t) * c->pieces_cap));
    } else {
      CK(cudaEventSynchronize(c->pieces_ev));
    }
    struct Seg { size_t start, n; bool range, has_r, has_w; };
    std::vector<Seg> segs;
    std::map<uint64_t, uint64_t> iv;  // disjointness of the open range segment
    size_t nr_total = 0, np = 0;
    for (size_t i = 0; i < n; ++i) {
      const uint64_t r = h[i];
      const uint64_t g0 = rec_g0(r), nw = rec_nw(r);
      const uint32_t acc = rec_acc(r);
      if (nw > kRangeWords) {
        bool join = !segs.empty() && segs.back().range;
        if (join) {
          auto it = iv.lower_bound(g0);
          if (it != iv.end() && it->first < g0 + nw) join = false;
          if (join && it != iv.begin()) {
            --it;
            if (it->second > g0) join = false;
          }
        }
        if (!join) {
          segs.push_back({nr_total, 0, true, false, false});
          iv.clear();
        }
        iv[g0] = g0 + nw;
        RangeDesc& d = c->h_ranges[nr_total++];
        d.g0 = g0;
        d.nw = nw;
        d.acc = acc;
        d.side = 0;
        segs.back().n++;
      } else {
        if (segs.empty() || segs.back().range) segs.push_back({np, 0, false, false, false});
        Seg& sg = segs.back();
        for (uint64_t o = 0; o < nw; o += kPieceWords) {
          c->h_pieces[np++] = pack_rec(g0 + o, std::min<uint64_t>(kPieceWords, nw - o), acc);
          sg.n++;
        }
        if (acc & XPL_ACC_R) sg.has_r = true;
        if (acc & XPL_ACC_W) sg.has_w = true;
      }
    }
    for (const Seg& sg : segs) {  // vbase per range segment
      if (!sg.range) continue;
      uint64_t v = 0;
      for (size_t i = sg.start; i < sg.start + sg.n; ++i) {
        c->h_ranges[i].vbase = v;
        v += ((c->h_ranges[i].g0 + c->h_ranges[i].nw - 1) >> 4) - (c->h_ranges[i].g0 >> 4) + 1;
      }
    }
    if (np) CK(cudaMemcpyAsync(c->d_pieces, c->h_pieces, sizeof(uint64_t) * np, cudaMemcpyHostToDevice, c->cs));
    CK(cudaEventRecord(c->pieces_ev, c->cs));
    if (nr_total)
      CK(cudaMemcpyAsync(c->d_ranges, c->h_ranges, sizeof(RangeDesc) * nr_total,
                         cudaMemcpyHostToDevice, c->cs));
    CK(cudaEventRecord(c->ranges_ev, c->cs));
    CK(cudaEventRecord(c->stage_ev[c->cur], c->cs));  // (staging itself was not uploaded)
    for (const Seg& sg : segs) {
      if (sg.range) {
        const RangeDesc& last = c->h_ranges[sg.start + sg.n - 1];
        const uint64_t nvec = last.vbase + ((last.g0 + last.nw - 1) >> 4) - (last.g0 >> 4) + 1;
        uint64_t rw = 0;
        for (size_t i = sg.start; i < sg.start + sg.n; ++i) rw += c->h_ranges[i].nw;
        const int pi = prof_begin(c, XPL_K_RANGE, 2 * rw);
        launch_range(c->cs, c->d_ranges + sg.start, (uint32_t)sg.n, nvec, (uint32_t*)c->d_pool,
                     c->d_cmap, c->d_smap, c->d_misc);
        prof_end(c, pi);
        c->st.kernel_launches += 1;
        c->st.range_segments++;
      } else {
        uint64_t fw0 = 0;
        if (sg.has_r && sg.has_w) {
          s = ensure_first_w(c, c->h_pieces + sg.start, sg.n, &fw0);
          if (s) return s;
        }
        const int pi = prof_begin(c, XPL_K_MERGE, c->prof ? 8 * sg.n + 2 * words_of(c->h_pieces + sg.start, sg.n) : 0);
        launch_merge(c->cs, c->d_pieces + sg.start, (uint32_t)sg.n, sg.has_r, sg.has_w,
                     c->d_first_w, fw0, (uint32_t*)c->d_pool);
        prof_end(c, pi);
        c->st.kernel_launches += sg.n <= 8192 ? 1 : 1 + sg.has_w + (sg.has_r && sg.has_w);
        c->st.merge_segments++;
      }
    }
  }
  if (cudaGetLastError() != cudaSuccess) return XPL_ERR_CUDA;
  c->cur ^= 1;
  CK(cudaEventSynchronize(c->stage_ev[c->cur]));  // the other buffer's copy is done
  c->stage_n = 0;
  c->stage_ranges = 0;
  c->stage_has_r = c->stage_has_w = false;
  return XPL_OK;
}

xpl_status upload_table(xpl_ctx* c) {
  if (!c->table_dirty) return XPL_OK;
  CK(cudaEventSynchronize(c->table_ev));
  uint32_t n = 0;
  xpl_dev_row* hr = (xpl_dev_row*)(c->h_tab + 32);
  for (auto& kv : c->live) {  // sorted by base
    const Row& r = c->rows[kv.second];
    hr[n].base = r.base;
    hr[n].end = r.base + r.bytes;
    hr[n].off = r.off | (uint64_t)r.owner << 56;  // the owner rank rides in the top byte
    hr[n].words = r.words;
    ++n;
  }
  memcpy(c->h_tab, &n, sizeof n);
  const unsigned long long n_super = (c->pas[c->rank].hwm + 16383) / 16384;  // for xpl_grid_epoch
  memcpy(c->h_tab + 8, &n_super, sizeof n_super);
  CK(cudaMemcpyAsync(c->d_tab, c->h_tab, 32 + sizeof(xpl_dev_row) * n, cudaMemcpyHostToDevice, c->cs));
  CK(cudaEventRecord(c->table_ev, c->cs));
  c->table_dirty = false;
  return XPL_OK;
}

cudaEvent_t pool_event(xpl_ctx* c, size_t i) {
  while (c->ev_pool.size() <= i) {
    cudaEvent_t e;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    c->ev_pool.push_back(e);
  }
  return c->ev_pool[i];
}

// GPU-side range accesses (D2D, memset; D7) inside the current epoch.
xpl_status gpu_ranges(xpl_ctx* c, const RangeDesc* rd, size_t nr) {
  if (!nr) return XPL_OK;
  xpl_status s = ensure_ranges(c, nr);
  if (s) return s;
  memcpy(c->h_ranges, rd, sizeof(RangeDesc) * nr);
  uint64_t v = 0;
  for (size_t i = 0; i < nr; ++i) {
    c->h_ranges[i].vbase = v;
    v += ((c->h_ranges[i].g0 + c->h_ranges[i].nw - 1) >> 4) - (c->h_ranges[i].g0 >> 4) + 1;
  }
  CK(cudaMemcpyAsync(c->d_ranges, c->h_ranges, sizeof(RangeDesc) * nr, cudaMemcpyHostToDevice, c->cs));
  CK(cudaEventRecord(c->ranges_ev, c->cs));
  uint64_t rw = 0;
  for (size_t i = 0; i < nr; ++i) rw += rd[i].nw;
  const int pi = prof_begin(c, XPL_K_RANGE, 2 * rw);
  launch_range(c->cs, c->d_ranges, (uint32_t)nr, v, (uint32_t*)c->d_pool, c->d_cmap, c->d_smap, c->d_misc);
  if (c->depth) c->cs_in_epoch = true;
  c->st.kernel_launches += 1;
  prof_end(c, pi);
  return cudaGetLastError() == cudaSuccess ? XPL_OK : XPL_ERR_CUDA;
}

// Epoch close (D5): the fold on cs.  pdl = it directly follows the
// epoch's kernels on the same stream (programmatic stream serialization).
// strict = the epoch had several streams or runtime range work of its own, so a
// device-side split (xpl_grid_epoch) inside it is an error (its fold would race).
// The fold skips its scan when no pending write was marked since the last close
// (d_misc[2], raised by the hooks and the range kernel); in sharded mode other
// ranks' writers mark this rank's maps without raising it, so the scan is forced.
void fold(xpl_ctx* c, bool pdl, bool strict = false) {
  const int pi = prof_begin(c, XPL_K_FOLD, 0);
  // only super-chunks below the pool's high-water mark can be flagged
  launch_fold(c->cs, pdl && pi < 0, (uint32_t*)c->d_pool, c->d_cmap, c->d_smap,
              (c->pas[c->rank].hwm + 16383) / 16384, c->d_stats, c->d_misc, strict ? 1 : 0,
              c->world > 1 ? 1 : 0);
  c->folds_host++;
  c->st.kernel_launches += 1;
  prof_end(c, pi);
}

// Make stream s wait for every runtime enqueue so far (no-op when s is cs).
xpl_status join(xpl_ctx* c, cudaStream_t s) {
  if (s == c->cs) return XPL_OK;
  CK(cudaEventRecord(c->ev_join, c->cs));
  CK(cudaStreamWaitEvent(s, c->ev_join, 0));
  return XPL_OK;
}

// ---- kernel-launch log (NEXT-4) -------------------------------------
cudaEvent_t log_event(xpl_ctx* c) {
  if (!c->lev_free.empty()) {
    cudaEvent_t e = c->lev_free.back();
    c->lev_free.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
  return e;
}

void log_clear(xpl_ctx* c) {
  for (auto& r : c->lepochs)
    for (cudaEvent_t e : {r.a, r.b, r.c})
      if (e) c->lev_free.push_back(e);
  c->lepochs.clear();
  c->lepoch_no.clear();
  c->lrecs.clear();
}

// Open the log entry of the epoch beginning on stream s (after s joined the
// runtime's pending work): begin event + the folded-chunk counter before it.
xpl_status log_epoch_begin(xpl_ctx* c, cudaStream_t s) {
  const size_t i = c->lepochs.size();
  if (2 * (i + 1) > c->lcum_cap) {  // grow the pinned snapshot array (rare: doubling)
    const size_t cap = c->lcum_cap ? 2 * c->lcum_cap : 8192;
    unsigned long long* h = nullptr;
    CK(cudaDeviceSynchronize());  // pending snapshot copies target the old array
    CK(cudaMallocHost((void**)&h, cap * sizeof(unsigned long long)));
    if (c->h_lcum) {
      memcpy(h, c->h_lcum, c->lcum_cap * sizeof(unsigned long long));
      cudaFreeHost(c->h_lcum);
    }
    c->h_lcum = h;
    c->lcum_cap = cap;
  }
  xpl_ctx::EpochRec r;
  r.a = log_event(c);
  r.b = log_event(c);
  r.c = log_event(c);
  if (!r.a || !r.b || !r.c) return XPL_ERR_CUDA;
  CK(cudaMemcpyAsync(c->h_lcum + 2 * i, c->d_stats + 3, sizeof(unsigned long long),
                     cudaMemcpyDeviceToHost, s));
  CK(cudaEventRecord(r.a, s));
  c->lepochs.push_back(r);
  c->lepoch_no.push_back(c->st.epochs);
  c->lepoch_open = true;
  return XPL_OK;
}

// A device-side epoch split ran in an epoch that forbids it (see fold()): reported
// once, by the first blocking call that reads the flags back (h_misc).
xpl_status split_error(xpl_ctx* c) {
  if (!c->h_misc[1]) return XPL_OK;
  c->h_misc[1] = 0;
  const uint32_t zero = 0;
  CK(cudaMemcpyAsync(c->d_misc + 1, &zero, 4, cudaMemcpyHostToDevice, c->cs));
  CK(cudaStreamSynchronize(c->cs));
  return XPL_ERR_STATE;
}

}  // namespace

extern "C" {

xpl_status xpl_launch_log_enable(xpl_ctx* c, int enable) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  CK(cudaDeviceSynchronize());  // pending snapshot copies / events of the old log
  log_clear(c);
  c->llog = enable != 0;
  return XPL_OK;
}

xpl_status xpl_kernel_launch(xpl_ctx* c, void* stream, const xpl_launch_info* li) {
  if (!c || !li) return XPL_ERR_INVALID_ARG;
  if (!c->depth) return XPL_ERR_STATE;
  if (!c->llog) return XPL_OK;
  xpl_launch_record r;
  memset(&r, 0, sizeof r);
  r.seq = c->lrecs.size();
  r.epoch = c->st.epochs;
  r.stream = (uint64_t)stream;
  for (int k = 0; k < 3; ++k) {
    r.grid[k] = li->grid[k];
    r.block[k] = li->block[k];
  }
  r.shmem = li->shmem;
  r.threads = (uint64_t)li->grid[0] * li->grid[1] * li->grid[2] * li->block[0] * li->block[1] * li->block[2];
  r.name_idx = UINT32_MAX;
  if (li->name) {
    auto it = c->lname_idx.find(li->name);
    if (it == c->lname_idx.end()) {
      it = c->lname_idx.emplace(li->name, (uint32_t)c->lnames.size()).first;
      c->lnames.push_back(li->name);
    }
    r.name_idx = it->second;
  }
  r.epoch_ms = -1.0;
  c->lrecs.push_back(r);
  return XPL_OK;
}

xpl_status xpl_launch_log(xpl_ctx* c, xpl_launch_record* out, size_t cap, size_t* n_out, int reset) {
  if (!c || !n_out || (cap && !out)) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  *n_out = c->lrecs.size();
  if (cap < c->lrecs.size()) return XPL_ERR_INVALID_ARG;
  // per logged epoch: GPU time and written chunks (waits for its events / copies)
  std::unordered_map<uint64_t, size_t> at;
  std::vector<double> ms(c->lepochs.size(), -1.0);
  std::vector<uint64_t> chunks(c->lepochs.size(), 0), nl(c->lepochs.size(), 0);
  for (size_t i = 0; i < c->lepochs.size(); ++i) {
    at[c->lepoch_no[i]] = i;
    CK(cudaEventSynchronize(c->lepochs[i].c));  // (after b and the end snapshot copy)
    float f = 0.f;
    if (cudaEventElapsedTime(&f, c->lepochs[i].a, c->lepochs[i].b) == cudaSuccess) ms[i] = f;
    chunks[i] = c->h_lcum[2 * i + 1] - c->h_lcum[2 * i];
  }
  for (const auto& r : c->lrecs) {
    auto it = at.find(r.epoch);
    if (it != at.end()) nl[it->second]++;
  }
  for (size_t k = 0; k < c->lrecs.size(); ++k) {
    out[k] = c->lrecs[k];
    auto it = at.find(out[k].epoch);
    if (it == at.end()) continue;
    out[k].epoch_ms = ms[it->second];
    out[k].epoch_written_chunks = chunks[it->second];
    out[k].launches_in_epoch = nl[it->second];
  }
  if (reset) log_clear(c);
  return XPL_OK;
}

const char* xpl_launch_name(xpl_ctx* c, uint32_t idx) {
  if (!c || idx >= c->lnames.size()) return nullptr;
  return c->lnames[idx].c_str();
}

// ---- UM page view (NEXT-3; D31-D33) ----------------------
static xpl_status page_pass(xpl_ctx* c, const std::vector<const Row*>& rows, uint64_t P,
                            uint8_t* h_flags, unsigned long long* h_cnt) {
  std::vector<PageRow> pr(rows.size());
  uint64_t np = 0;
  for (size_t i = 0; i < rows.size(); ++i) {
    pr[i].off = rows[i]->off;
    pr[i].words = rows[i]->words;
    pr[i].page0 = np;
    np += (rows[i]->words + P - 1) / P;
  }
  PageRow* d_rows = nullptr;
  unsigned long long* d_cnt = nullptr;
  uint8_t* d_flags = nullptr;
  const size_t ncnt = 5 * rows.size();
  CK(cudaMallocAsync((void**)&d_rows, sizeof(PageRow) * pr.size() + 1, c->cs));
  CK(cudaMallocAsync((void**)&d_cnt, sizeof(unsigned long long) * ncnt + 8, c->cs));
  if (h_flags) CK(cudaMallocAsync((void**)&d_flags, np + 1, c->cs));
  CK(cudaMemcpyAsync(d_rows, pr.data(), sizeof(PageRow) * pr.size(), cudaMemcpyHostToDevice, c->cs));
  CK(cudaMemsetAsync(d_cnt, 0, sizeof(unsigned long long) * ncnt + 8, c->cs));
  uint64_t words = 0;
  for (const Row* r : rows) words += r->words;
  const int pi = prof_begin(c, XPL_K_PAGES, words);
  launch_pages(c->cs, d_rows, (uint32_t)pr.size(), np, P, (const uint32_t*)c->d_pool, d_flags, d_cnt);
  prof_end(c, pi);
  c->st.kernel_launches += 1;
  CK(cudaMemcpyAsync(h_cnt, d_cnt, sizeof(unsigned long long) * ncnt, cudaMemcpyDeviceToHost, c->cs));
  if (h_flags) CK(cudaMemcpyAsync(h_flags, d_flags, np, cudaMemcpyDeviceToHost, c->cs));
  CK(cudaFreeAsync(d_rows, c->cs));
  CK(cudaFreeAsync(d_cnt, c->cs));
  if (d_flags) CK(cudaFreeAsync(d_flags, c->cs));
  CK(cudaStreamSynchronize(c->cs));
  return XPL_OK;
}

xpl_status xpl_page_summary(xpl_ctx* c, uint64_t P, xpl_page_report* out, size_t cap, size_t* n_out) {
  if (!c || !n_out || P == 0 || (cap && !out)) return XPL_ERR_INVALID_ARG;
  if (c->depth || c->world > 1) return XPL_ERR_STATE;  // (the page view is single-GPU)
  std::vector<const Row*> rows;
  for (uint64_t id : c->active)
    if (c->rows[id].live) rows.push_back(&c->rows[id]);  // (active is in id order)
  *n_out = rows.size();
  if (cap < rows.size()) return XPL_ERR_INVALID_ARG;
  xpl_status st = flush(c);
  if (st) return st;
  std::vector<unsigned long long> cnt(5 * rows.size() + 1);
  if (!rows.empty()) {
    st = page_pass(c, rows, P, nullptr, cnt.data());
    if (st) return st;
  }
  for (size_t i = 0; i < rows.size(); ++i) {
    const Row& r = *rows[i];
    xpl_page_report& o = out[i];
    memset(&o, 0, sizeof o);
    o.id = r.id;
    o.base = r.base;
    o.words = r.words;
    o.page_words = P;
    o.pages = (r.words + P - 1) / P;
    o.kind = r.kind;
    o.advice = r.advice;
    o.cpu_pages = cnt[5 * i + 0];
    o.gpu_pages = cnt[5 * i + 1];
    o.shared_pages = cnt[5 * i + 2];
    o.false_shared_pages = cnt[5 * i + 3];
    o.alternating_pages = cnt[5 * i + 4];
    if (r.kind == XPL_ALLOC_MANAGED) {  // D8: page effects exist for unified memory only
      if (o.false_shared_pages) o.flags |= XPL_PAGE_PAT_FALSE_SHARING;
      if ((r.advice & XPL_ADVICE_READ_MOSTLY) && o.alternating_pages) o.flags |= XPL_PAGE_PAT_ADVICE_MISMATCH;
    }
  }
  return XPL_OK;
}

xpl_status xpl_page_flags(xpl_ctx* c, const void* base, uint64_t P, uint8_t* out, uint64_t n_pages) {
  if (!c || !out || P == 0) return XPL_ERR_INVALID_ARG;
  if (c->depth || c->world > 1) return XPL_ERR_STATE;
  auto it = c->live.find((uint64_t)base);
  if (it == c->live.end()) return XPL_ERR_UNKNOWN_PTR;
  const Row* r = &c->rows[it->second];
  if (n_pages != (r->words + P - 1) / P) return XPL_ERR_INVALID_ARG;
  xpl_status st = flush(c);
  if (st) return st;
  unsigned long long cnt[5];
  return page_pass(c, std::vector<const Row*>{r}, P, out, cnt);
}

xpl_status xpl_mem_advise(xpl_ctx* c, const void* ptr, size_t bytes, int advice, int device) {
  (void)bytes;  // D33: advice is tracked per allocation
  if (!c || advice < 1 || advice > 6) return XPL_ERR_INVALID_ARG;
  const Row* cr = lookup(c, (uint64_t)ptr);
  if (!cr) return XPL_OK;  // untracked
  Row& r = c->rows[cr->id];
  const bool cpu = device < 0;
  switch (advice) {
    case 1: r.advice |= XPL_ADVICE_READ_MOSTLY; break;
    case 2: r.advice &= ~XPL_ADVICE_READ_MOSTLY; break;
    case 3:
      r.advice &= ~(XPL_ADVICE_PREFERRED_GPU | XPL_ADVICE_PREFERRED_CPU);
      r.advice |= cpu ? XPL_ADVICE_PREFERRED_CPU : XPL_ADVICE_PREFERRED_GPU;
      break;
    case 4: r.advice &= ~(XPL_ADVICE_PREFERRED_GPU | XPL_ADVICE_PREFERRED_CPU); break;
    case 5: r.advice |= cpu ? XPL_ADVICE_ACCESSED_BY_CPU : XPL_ADVICE_ACCESSED_BY_GPU; break;
    default: r.advice &= ~(cpu ? XPL_ADVICE_ACCESSED_BY_CPU : XPL_ADVICE_ACCESSED_BY_GPU); break;
  }
  return XPL_OK;
}

const char* xpl_status_string(xpl_status s) {
  switch (s) {
    case XPL_OK: return "ok";
    case XPL_ERR_INVALID_ARG: return "invalid argument";
    case XPL_ERR_OOM: return "out of memory (shadow pool, table or staging)";
    case XPL_ERR_OVERLAP: return "allocation overlaps a live allocation";
    case XPL_ERR_UNKNOWN_PTR: return "pointer is not the base of a live allocation";
    case XPL_ERR_STATE: return "call not allowed in the current epoch state";
    case XPL_ERR_CUDA: return "CUDA runtime error";
    case XPL_ERR_NCCL: return "NCCL error";
    case XPL_ERR_DEVICE_OVERFLOW: return "device-side capacity exceeded";
  }
  return "unknown status";
}

xpl_status xpl_init(const xpl_config* cfg, xpl_ctx** out) {
  if (!cfg || !out) return XPL_ERR_INVALID_ARG;
  const int world = cfg->world > 1 ? cfg->world : 1;
  if (world > XPL_MAX_RANKS || (world > 1 && (!cfg->comm || cfg->rank < 0 || cfg->rank >= world)))
    return XPL_ERR_INVALID_ARG;
  xpl_ctx* c = new (std::nothrow) xpl_ctx();
  if (!c) return XPL_ERR_OOM;
  c->cfg = *cfg;
  c->world = world;
  c->rank = world > 1 ? cfg->rank : 0;
  c->comm = world > 1 ? cfg->comm : nullptr;
  c->route.assign(world, {});
  if (!c->cfg.pool_words) c->cfg.pool_words = 1ull << 28;
  if (!c->cfg.staging_recs) c->cfg.staging_recs = 1ull << 22;
  if (!c->cfg.max_rows) c->cfg.max_rows = 4096;
  c->pool_words = (c->cfg.pool_words + 65535) & ~65535ull;  // whole 4-byte words of the super map
  if (c->pool_words / 4 > 0xFFFFFFFFull) { delete c; return XPL_ERR_INVALID_ARG; }
#define CKI(x)                  \
  do {                          \
    if ((x) != cudaSuccess) {   \
      xpl_finalize(c);          \
      return XPL_ERR_CUDA;      \
    }                           \
  } while (0)
  CKI(cudaSetDevice(cfg->device));
  CKI(cudaStreamCreateWithFlags(&c->rs, cudaStreamNonBlocking));
  c->cs = c->rs;
  CKI(cudaMalloc(&c->d_pool, c->pool_words));
  CKI(cudaMemsetAsync(c->d_pool, 0, c->pool_words, c->cs));
  c->pas.assign(world, PoolAlloc());
  for (PoolAlloc& a : c->pas) a.init(c->pool_words);
  CKI(cudaMalloc(&c->d_tab, 32 + sizeof(xpl_dev_row) * c->cfg.max_rows));
  CKI(cudaMemsetAsync(c->d_tab, 0, 32, c->cs));
  CKI(host_alloc(&c->h_tab, 32 + sizeof(xpl_dev_row) * c->cfg.max_rows));
  CKI(cudaMalloc(&c->d_cmap, c->pool_words / 128));
  CKI(cudaMemsetAsync(c->d_cmap, 0, c->pool_words / 128, c->cs));
  CKI(cudaMalloc(&c->d_smap, c->pool_words / 16384));
  CKI(cudaMemsetAsync(c->d_smap, 0, c->pool_words / 16384, c->cs));
  CKI(cudaMalloc(&c->d_misc, 64));
  CKI(cudaMemsetAsync(c->d_misc, 0, 64, c->cs));
  CKI(host_alloc(&c->h_misc, 16));
  memset(c->h_misc, 0, 64);
  CKI(cudaMalloc(&c->d_stats, 64));
  CKI(cudaMemsetAsync(c->d_stats, 0, 64, c->cs));
  c->stage_cap = c->cfg.staging_recs;
  CKI(host_alloc(&c->h_stage[0], c->stage_cap));
  CKI(host_alloc(&c->h_stage[1], c->stage_cap));
  CKI(cudaMalloc(&c->d_stage, sizeof(uint64_t) * c->stage_cap));
  CKI(cudaEventCreateWithFlags(&c->stage_ev[0], cudaEventDisableTiming));
  CKI(cudaEventCreateWithFlags(&c->stage_ev[1], cudaEventDisableTiming));
  CKI(cudaEventCreateWithFlags(&c->table_ev, cudaEventDisableTiming));
  CKI(cudaEventCreateWithFlags(&c->ranges_ev, cudaEventDisableTiming));
  CKI(cudaEventCreateWithFlags(&c->pieces_ev, cudaEventDisableTiming));
  CKI(cudaEventRecord(c->pieces_ev, c->cs));
  CKI(cudaEventCreateWithFlags(&c->ev_begin, cudaEventDisableTiming));
  CKI(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  CKI(cudaEventRecord(c->stage_ev[0], c->cs));
  CKI(cudaEventRecord(c->stage_ev[1], c->cs));
  CKI(cudaEventRecord(c->table_ev, c->cs));
  CKI(cudaEventRecord(c->ranges_ev, c->cs));
  xpl_status s = ensure_ranges(c, 1024);
  if (s) { xpl_finalize(c); return s; }
  CKI(cudaStreamSynchronize(c->cs));
  if (world > 1) {  // map the other ranks' pools and chunk maps (CUDA IPC; NVLink / NVSwitch peers)
    struct Ex { cudaIpcMemHandle_t h[3]; uint64_t pool_words; };
    Ex mine;
    memset(&mine, 0, sizeof mine);
    CKI(cudaIpcGetMemHandle(&mine.h[0], c->d_pool));
    CKI(cudaIpcGetMemHandle(&mine.h[1], c->d_cmap));
    CKI(cudaIpcGetMemHandle(&mine.h[2], c->d_smap));
    mine.pool_words = c->pool_words;
    std::vector<Ex> all(world);
    if (c->comm->allgather(c->comm->user, &mine, sizeof(Ex), all.data())) { xpl_finalize(c); return XPL_ERR_NCCL; }
    for (int q = 0; q < world; ++q) {
      if (all[q].pool_words != c->pool_words) { xpl_finalize(c); return XPL_ERR_INVALID_ARG; }
      if (q == c->rank) continue;
      CKI(cudaIpcOpenMemHandle(&c->peer_pool[q], all[q].h[0], cudaIpcMemLazyEnablePeerAccess));
      CKI(cudaIpcOpenMemHandle(&c->peer_cmap[q], all[q].h[1], cudaIpcMemLazyEnablePeerAccess));
      CKI(cudaIpcOpenMemHandle(&c->peer_smap[q], all[q].h[2], cudaIpcMemLazyEnablePeerAccess));
    }
    if (c->comm->barrier(c->comm->user)) { xpl_finalize(c); return XPL_ERR_NCCL; }
  }
  memset(&c->st, 0, sizeof c->st);
  c->ready = true;
  *out = c;
  return XPL_OK;
#undef CKI
}

xpl_status xpl_finalize(xpl_ctx* c) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->cs) cudaStreamSynchronize(c->cs);
  if (c->rs) cudaStreamSynchronize(c->rs);
  // (sharded: every rank finalises; no rank may unmap a pool a peer still writes --
  // only once xpl_init completed, so a rank failing inside xpl_init does not wait)
  if (c->world > 1 && c->comm && c->ready) c->comm->barrier(c->comm->user);
  for (int q = 0; q < XPL_MAX_RANKS; ++q)
    for (void* p : {c->peer_pool[q], c->peer_cmap[q], c->peer_smap[q]})
      if (p) cudaIpcCloseMemHandle(p);
  cudaFree(c->d_pool);
  cudaFree(c->d_first_w);
  cudaFree(c->d_tab);
  cudaFreeHost(c->h_tab);
  cudaFree(c->d_cmap);
  cudaFree(c->d_smap);
  cudaFree(c->d_misc);
  cudaFreeHost(c->h_misc);
  cudaFree(c->d_stats);
  cudaFreeHost(c->h_stage[0]);
  cudaFreeHost(c->h_stage[1]);
  cudaFree(c->d_stage);
  cudaFreeHost(c->h_ranges);
  cudaFree(c->d_ranges);
  cudaFree(c->d_tiles);
  cudaFree(c->d_blk);
  cudaFree(c->d_segsum);
  cudaFree(c->d_segcnt);
  cudaFree(c->d_done);
  cudaFreeHost(c->h_up);
  cudaFree(c->d_up);
  cudaFree(c->d_cnt);
  cudaFree(c->d_rep);
  cudaFreeHost(c->h_rep);
  cudaFree(c->d_rpart);
  cudaFreeHost(c->h_rpart);
  cudaFreeHost(c->h_cnt);
  for (cudaEvent_t e : c->ev_pool) cudaEventDestroy(e);
  for (cudaEvent_t e : c->prof_free) cudaEventDestroy(e);
  for (cudaEvent_t e : c->lev_free) cudaEventDestroy(e);
  for (auto& r : c->lepochs)
    for (cudaEvent_t e : {r.a, r.b, r.c})
      if (e) cudaEventDestroy(e);
  cudaFreeHost(c->h_lcum);
  for (auto& r : c->prof_pending) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  cudaFreeHost(c->h_pieces);
  cudaFree(c->d_pieces);
  for (cudaEvent_t e : {c->stage_ev[0], c->stage_ev[1], c->table_ev, c->ranges_ev, c->ev_begin,
                        c->pieces_ev, c->ev_join})
    if (e) cudaEventDestroy(e);
  if (c->rs) cudaStreamDestroy(c->rs);
  delete c;
  return XPL_OK;
}

static xpl_status register_row(xpl_ctx* c, const void* ptr, size_t bytes, xpl_alloc_kind kind,
                               bool piece, uint64_t logical_id, uint64_t goff, uint64_t lbytes,
                               uint32_t owner = 0) {
  if (!c || !ptr || bytes == 0 || (unsigned)kind > 2) return XPL_ERR_INVALID_ARG;
  if (piece && (lbytes == 0 || goff + (bytes + 3) / 4 > (lbytes + 3) / 4)) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  const uint64_t p = (uint64_t)ptr;
  auto it = c->live.lower_bound(p);
  if (it != c->live.end() && it->first < p + bytes) return XPL_ERR_OVERLAP;
  if (it != c->live.begin()) {
    auto pv = std::prev(it);
    const Row& r = c->rows[pv->second];
    if (r.base + r.bytes > p) return XPL_ERR_OVERLAP;
  }
  if (c->live.size() >= c->cfg.max_rows) return XPL_ERR_OOM;
  Row r;
  r.id = c->rows.size();
  r.base = p;
  r.bytes = bytes;
  r.words = (bytes + 3) / 4;
  r.span = (r.words + 15) & ~15ull;
  r.kind = kind;
  r.live = true;
  r.dropped = false;
  r.ever = false;
  r.advice = 0;
  r.logical_id = piece ? logical_id : r.id;
  r.goff = piece ? goff : 0;
  r.lbytes = piece ? lbytes : bytes;
  r.owner = owner;
  if (!c->pas[owner].alloc(r.span, &r.off)) return XPL_ERR_OOM;
  if (owner == (uint32_t)c->rank)
    CK(cudaMemsetAsync(c->d_pool + r.off, 0, r.span, c->cs));  // D3: last writer = CPU
  const size_t cap_before = c->rows.capacity();
  c->rows.push_back(r);
  if (c->rows.capacity() != cap_before) c->cache = nullptr;
  c->live[p] = r.id;
  c->active.push_back(r.id);
  c->lrows[r.logical_id].push_back(r.id);
  c->table_dirty = true;
  c->cache = nullptr;
  return XPL_OK;
}

// The pieces of a logical allocation of lw words over R ranks (xpl.h sharded
// mode): < 65536 words -> one piece owned by rank (lid mod R); else R pieces of
// ceil(lw/R) words rounded up to 1024, piece r owned by rank r (empty tail
// pieces dropped).  (goff, words, owner) each.
static std::vector<std::array<uint64_t, 3>> shard_pieces(uint64_t lid, uint64_t lw, int R) {
  std::vector<std::array<uint64_t, 3>> v;
  if (lw < 65536) {
    v.push_back({0, lw, lid % (uint64_t)R});
    return v;
  }
  const uint64_t chunk = ((lw + R - 1) / R + 1023) & ~1023ull;
  for (int r = 0; r < R; ++r) {
    const uint64_t g = (uint64_t)r * chunk;
    if (g >= lw) break;
    v.push_back({g, std::min(lw, g + chunk) - g, (uint64_t)r});
  }
  return v;
}

xpl_status xpl_register_alloc(xpl_ctx* c, const void* ptr, size_t bytes, xpl_alloc_kind kind) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->world <= 1) return register_row(c, ptr, bytes, kind, false, 0, 0, 0);
  // sharded mode (COLLECTIVE): one row per piece, each in its owner's pool
  if (!ptr || bytes == 0 || (unsigned)kind > 2) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  const uint64_t lid = c->n_logical;
  const uint64_t lw = (bytes + 3) / 4;
  const auto pcs = shard_pieces(lid, lw, c->world);
  if (c->live.size() + pcs.size() > c->cfg.max_rows) return XPL_ERR_OOM;
  const size_t first_row = c->rows.size();
  for (const auto& pc : pcs) {
    const uint64_t b0 = 4 * pc[0], b1 = std::min<uint64_t>(bytes, 4 * (pc[0] + pc[1]));
    xpl_status st = register_row(c, (const uint8_t*)ptr + b0, b1 - b0, kind, true, lid, pc[0], bytes,
                                 (uint32_t)pc[2]);
    if (st) {  // undo the pieces registered so far (every rank fails alike: same tables)
      for (size_t id = first_row; id < c->rows.size(); ++id) {
        Row& r = c->rows[id];
        c->live.erase(r.base);
        c->pas[r.owner].release(r.off, r.span);
        r.live = false;
        r.dropped = true;
      }
      c->active.erase(std::remove_if(c->active.begin(), c->active.end(),
                                     [&](uint64_t id) { return id >= first_row; }),
                      c->active.end());
      c->lrows.erase(lid);
      c->table_dirty = true;
      c->cache = nullptr;
      return st;
    }
  }
  c->n_logical++;
  return XPL_OK;
}

xpl_status xpl_register_alloc_piece(xpl_ctx* c, const void* ptr, size_t bytes, xpl_alloc_kind kind,
                                    uint64_t logical_id, uint64_t word_offset, uint64_t logical_bytes) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->world > 1) return XPL_ERR_STATE;  // sharded mode cuts the pieces itself
  return register_row(c, ptr, bytes, kind, true, logical_id, word_offset, logical_bytes);
}

static void kill_row(xpl_ctx* c, uint64_t id) {
  Row& r = c->rows[id];
  r.live = false;  // shadow kept until the next diagnose
  c->live.erase(r.base);
  c->n_dead++;
}

xpl_status xpl_free(xpl_ctx* c, const void* ptr) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  auto it = c->live.find((uint64_t)ptr);
  if (it == c->live.end()) return XPL_ERR_UNKNOWN_PTR;
  if (c->world > 1) {  // every piece of the logical allocation (COLLECTIVE)
    const Row& r = c->rows[it->second];
    if (r.goff != 0) return XPL_ERR_UNKNOWN_PTR;  // not the allocation's base
    const std::vector<uint64_t> ids = c->lrows[r.logical_id];
    for (uint64_t id : ids) kill_row(c, id);
  } else {
    kill_row(c, it->second);
  }
  c->table_dirty = true;
  c->cache = nullptr;
  return XPL_OK;
}

// Epochs (D19).  The runtime's pending work (host merges, table
// upload) sits on cs; a stream joining the epoch waits for it through ev_begin,
// unless it is cs itself.  At the close, a single-stream epoch gets its fold
// enqueued right behind its kernels on that stream (which becomes cs); several
// streams are joined on rs first.
xpl_status xpl_kernel_begin(xpl_ctx* c, void* stream) {
  if (!c) return XPL_ERR_INVALID_ARG;
  NvtxRange nv("xpl_kernel_begin");
  cudaStream_t s = (cudaStream_t)stream;
  if (c->depth == 0) {
    xpl_status st = flush(c);
    if (st) return st;
    st = upload_table(c);
    if (st) return st;
    if (c->world > 1) {
      // sharded: every rank's shadow work before this epoch -- its fold of the
      // last epoch, its merges of the routed host records, a diagnose's reset --
      // has completed before any rank's kernels record into its pool again
      // (a remote write landing before the owner's fold would be folded early)
      CK(cudaStreamSynchronize(c->cs));
      if (c->comm->barrier(c->comm->user)) return XPL_ERR_NCCL;
    }
    c->ev_begin_valid = false;
    c->cs_in_epoch = false;
    c->epoch_streams.clear();
    c->st.epochs++;
  }
  if (std::find(c->epoch_streams.begin(), c->epoch_streams.end(), s) == c->epoch_streams.end()) {
    if (s != c->cs) {
      if (!c->ev_begin_valid) {
        CK(cudaEventRecord(c->ev_begin, c->cs));
        c->ev_begin_valid = true;
      }
      CK(cudaStreamWaitEvent(s, c->ev_begin, 0));
    }
    c->epoch_streams.push_back(s);
  }
  if (c->llog && !c->lepoch_open) {  // NEXT-4: the epoch starts on its first stream
    xpl_status st = log_epoch_begin(c, s);
    if (st) return st;
  }
  c->depth++;
  return XPL_OK;
}

xpl_status xpl_kernel_end(xpl_ctx* c, void* stream) {
  if (!c) return XPL_ERR_INVALID_ARG;
  NvtxRange nv("xpl_kernel_end");
  if (c->depth == 0) return XPL_ERR_STATE;
  cudaStream_t s = (cudaStream_t)stream;
  if (std::find(c->epoch_streams.begin(), c->epoch_streams.end(), s) == c->epoch_streams.end()) {
    if (s != c->cs && !c->ev_begin_valid) {  // (ended on a stream that never began)
      CK(cudaEventRecord(c->ev_begin, c->cs));
      c->ev_begin_valid = true;
    }
    if (s != c->cs) CK(cudaStreamWaitEvent(s, c->ev_begin, 0));
    c->epoch_streams.push_back(s);
  }
  if (--c->depth) return XPL_OK;
  if (c->world > 1) {
    // sharded: every rank's kernels of the epoch -- including their atomics into
    // this rank's pool over NVLink -- have completed before any owner folds
    for (cudaStream_t x : c->epoch_streams) CK(cudaStreamSynchronize(x));
    CK(cudaStreamSynchronize(c->cs));
    if (c->comm->barrier(c->comm->user)) return XPL_ERR_NCCL;
  }
  // the stream the fold goes on, and everything of the epoch that must precede it
  const bool single = c->epoch_streams.size() == 1;
  cudaStream_t t = single ? c->epoch_streams[0] : c->rs;
  std::vector<cudaStream_t> wait = c->epoch_streams;
  // cs: only in-epoch D2D / memset work is not yet ordered before the epoch's
  // streams (everything earlier was, through ev_begin)
  if (c->cs_in_epoch) wait.push_back(c->cs);
  size_t k = 0;
  bool crossed = false;
  for (size_t i = 0; i < wait.size(); ++i) {
    const cudaStream_t x = wait[i];
    if (x == t || std::find(wait.begin(), wait.begin() + i, x) != wait.begin() + i) continue;
    cudaEvent_t e = pool_event(c, k++);
    CK(cudaEventRecord(e, x));
    CK(cudaStreamWaitEvent(t, e, 0));
    crossed = true;
  }
  const bool strict = !single || c->cs_in_epoch || c->world > 1;  // (a split cannot span ranks)
  c->cs = t;
  fold(c, !crossed, strict);
  if (c->lepoch_open) {  // NEXT-4: after the fold, on its stream
    const size_t i = c->lepochs.size() - 1;
    CK(cudaEventRecord(c->lepochs[i].b, c->cs));
    CK(cudaMemcpyAsync(c->h_lcum + 2 * i + 1, c->d_stats + 3, sizeof(unsigned long long),
                       cudaMemcpyDeviceToHost, c->cs));
    CK(cudaEventRecord(c->lepochs[i].c, c->cs));
    c->lepoch_open = false;
  }
  if (t == nullptr || t == cudaStreamLegacy || t == cudaStreamPerThread) {
    // never adopt a default stream as the runtime's stream: it would serialise the
    // runtime's later work with every blocking stream of the process
    CK(cudaEventRecord(c->ev_join, t));
    CK(cudaStreamWaitEvent(c->rs, c->ev_join, 0));
    c->cs = c->rs;
  }
  if (cudaGetLastError() != cudaSuccess) return XPL_ERR_CUDA;
  std::vector<std::pair<uint32_t, uint64_t>> q;
  q.swap(c->deferred);
  for (const auto& d : q) {
    const uint64_t r = d.second;
    xpl_status st = stage_push(c, rec_g0(r), rec_nw(r), rec_acc(r), d.first);
    if (st) return st;
  }
  return XPL_OK;
}

xpl_status xpl_record_host(xpl_ctx* c, const xpl_host_access* recs, size_t n) {
  if (!c || (!recs && n)) return XPL_ERR_INVALID_ARG;
  for (size_t i = 0; i < n; ++i) {
    const uint32_t acc = recs[i].kind;
    if (acc < 1 || acc > 3) return XPL_ERR_INVALID_ARG;
    uint64_t g0, nw;
    uint32_t own = 0;
    if (!to_words(c, recs[i].addr, recs[i].size, &g0, &nw, &own)) continue;  // untracked
    if (c->depth) {
      while (nw > kMaxRecWords) {
        c->deferred.push_back({own, pack_rec(g0, kMaxRecWords, acc)});
        g0 += kMaxRecWords;
        nw -= kMaxRecWords;
      }
      c->deferred.push_back({own, pack_rec(g0, nw, acc)});
      continue;
    }
    xpl_status s = stage_push(c, g0, nw, acc, own);
    if (s) return s;
  }
  return XPL_OK;
}

xpl_status xpl_record_host_ranges(xpl_ctx* c, const xpl_host_access* recs, size_t n) {
  if (!c || (!recs && n)) return XPL_ERR_INVALID_ARG;
  for (size_t i = 0; i < n; ++i) {
    const uint32_t acc = recs[i].kind;
    if (acc < 1 || acc > 3) return XPL_ERR_INVALID_ARG;
    uint64_t a = recs[i].addr;
    const uint64_t e = a + recs[i].size;
    while (a < e) {
      const Row* r = lookup(c, a);
      if (!r) {  // skip to the next live allocation inside the range, if any
        auto it = c->live.upper_bound(a);
        if (it == c->live.end() || it->first >= e) break;
        a = it->first;
        continue;
      }
      const uint64_t re = r->base + r->bytes;
      const uint64_t pe = e < re ? e : re;
      uint64_t g0, nw;
      uint32_t own = 0;
      if (to_words(c, a, pe - a, &g0, &nw, &own)) {
        if (c->depth) {
          while (nw > kMaxRecWords) {
            c->deferred.push_back({own, pack_rec(g0, kMaxRecWords, acc)});
            g0 += kMaxRecWords;
            nw -= kMaxRecWords;
          }
          c->deferred.push_back({own, pack_rec(g0, nw, acc)});
        } else {
          xpl_status s = stage_push(c, g0, nw, acc, own);
          if (s) return s;
        }
      }
      a = pe;
    }
  }
  return XPL_OK;
}

xpl_status xpl_record_host_strided(xpl_ctx* c, const xpl_host_strided* recs, size_t n) {
  if (!c || (!recs && n)) return XPL_ERR_INVALID_ARG;
  for (size_t i = 0; i < n; ++i) {
    const xpl_host_strided& q = recs[i];
    if (q.kind < 1 || q.kind > 3 || q.size == 0 || q.count == 0) return XPL_ERR_INVALID_ARG;
    if (q.count == 1) {
      const xpl_host_access one = {q.addr, q.size, q.kind};
      xpl_status s = xpl_record_host_ranges(c, &one, 1);
      if (s) return s;
      continue;
    }
    // the lowest and highest element: if both lie inside one live row, so do all
    const uint64_t last = q.addr + (uint64_t)q.stride * (q.count - 1);
    const uint64_t lo = q.stride >= 0 ? q.addr : last, hi = q.stride >= 0 ? last : q.addr;
    const Row* r = lookup(c, lo);
    if (r && hi + q.size <= r->base + r->bytes && hi + q.size > hi) {
      uint64_t a = q.addr;
      for (uint64_t j = 0; j < q.count; ++j, a += (uint64_t)q.stride) {
        const uint64_t w0 = (a - r->base) >> 2, wl = (a + q.size - 1 - r->base) >> 2;
        uint64_t g0 = r->off + w0, nw = wl - w0 + 1;
        if (c->depth) {
          for (; nw > kMaxRecWords; g0 += kMaxRecWords, nw -= kMaxRecWords)
            c->deferred.push_back({r->owner, pack_rec(g0, kMaxRecWords, q.kind)});
          c->deferred.push_back({r->owner, pack_rec(g0, nw, q.kind)});
        } else {
          xpl_status s = stage_push(c, g0, nw, q.kind, r->owner);
          if (s) return s;
        }
      }
      continue;
    }
    uint64_t a = q.addr;  // elements in several rows (or untracked): one by one
    for (uint64_t j = 0; j < q.count; ++j, a += (uint64_t)q.stride) {
      const xpl_host_access one = {a, q.size, q.kind};
      xpl_status s = xpl_record_host_ranges(c, &one, 1);
      if (s) return s;
    }
  }
  return XPL_OK;
}

}  // extern "C"

// The pieces (row, first pool word, words) of [addr, addr+bytes) clipped to the
// logical allocation holding addr (D18): its one row, or, in sharded mode, the
// pieces it spans.  False if addr is untracked.
template <class F>
static bool for_logical_range(xpl_ctx* c, uint64_t addr, uint64_t bytes, F fn) {
  const Row* r = lookup(c, addr);
  if (!r) return false;
  const uint64_t lend = r->base - 4 * r->goff + r->lbytes;  // pieces are contiguous in address
  const uint64_t e = bytes < lend - addr ? addr + bytes : lend;
  const std::vector<uint64_t> ids = c->lrows[r->logical_id];
  for (uint64_t id : ids) {
    const Row& p = c->rows[id];
    if (!p.live) continue;
    const uint64_t a0 = std::max(addr, p.base), a1 = std::min(e, p.base + p.bytes);
    if (a0 >= a1) continue;
    const uint64_t w0 = (a0 - p.base) >> 2, wl = std::min((a1 - 1 - p.base) >> 2, p.words - 1);
    fn(p, p.off + w0, wl - w0 + 1);
  }
  return true;
}

static xpl_status push_or_defer(xpl_ctx* c, uint32_t owner, uint64_t g0, uint64_t nw, uint32_t acc) {
  if (!c->depth) return stage_push(c, g0, nw, acc, owner);
  for (; nw > kMaxRecWords; g0 += kMaxRecWords, nw -= kMaxRecWords)
    c->deferred.push_back({owner, pack_rec(g0, kMaxRecWords, acc)});
  c->deferred.push_back({owner, pack_rec(g0, nw, acc)});
  return XPL_OK;
}

extern "C" {

xpl_status xpl_record_copy(xpl_ctx* c, const void* dst, const void* src, size_t bytes,
                           xpl_copy_dir dir) {
  if (!c || (unsigned)dir > 4) return XPL_ERR_INVALID_ARG;
  if (bytes == 0) return XPL_OK;
  if (dir <= XPL_COPY_H2H) {  // CPU-side: one ordered range per side
    if (c->world > 1) {
      // COLLECTIVE: route what came before; rank 0's call is the one recorded
      // (first in the next slice order, xpl.h)
      if (!c->depth) {
        xpl_status s = flush(c);
        if (s) return s;
      }
      if (c->rank != 0) return XPL_OK;
    }
    struct Side { uint64_t addr; uint32_t acc; } a[2];
    size_t n = 0;
    if (dir == XPL_COPY_H2D) a[n++] = {(uint64_t)dst, XPL_ACC_W};
    if (dir == XPL_COPY_D2H) a[n++] = {(uint64_t)src, XPL_ACC_R};
    if (dir == XPL_COPY_H2H) {
      a[n++] = {(uint64_t)src, XPL_ACC_R};
      a[n++] = {(uint64_t)dst, XPL_ACC_W};
    }
    xpl_status st = XPL_OK;
    for (size_t i = 0; i < n; ++i)
      for_logical_range(c, a[i].addr, bytes, [&](const Row& p, uint64_t g0, uint64_t nw) {
        if (!st) st = push_or_defer(c, p.owner, g0, nw, a[i].acc);
      });
    return st;
  }
  // GPU-side: D2D = GPU read src + GPU write dst; memset = GPU write dst (D7).
  // One range per side and piece, of any length (RangeDesc.nw and the range
  // kernel's vector indices are 64-bit); in sharded mode each owner applies
  // its own pieces.
  std::vector<RangeDesc> rd;
  auto add = [&](uint64_t addr, uint32_t acc) {
    for_logical_range(c, addr, bytes, [&](const Row& p, uint64_t g0, uint64_t nw) {
      if (p.owner == (uint32_t)c->rank) rd.push_back({g0, nw, 0, acc, 1});
    });
  };
  if (dir == XPL_COPY_D2D) add((uint64_t)src, XPL_ACC_R);
  add((uint64_t)dst, XPL_ACC_W);
  const bool own = c->depth == 0;
  if (own) {
    xpl_status s = flush(c);
    if (s) return s;
    c->st.epochs++;
  }
  xpl_status s = gpu_ranges(c, rd.data(), rd.size());
  if (s) return s;
  if (own) fold(c, false);
  return cudaGetLastError() == cudaSuccess ? XPL_OK : XPL_ERR_CUDA;
}

xpl_status xpl_flush(xpl_ctx* c) {
  if (!c) return XPL_ERR_INVALID_ARG;
  return flush(c);
}

xpl_status xpl_sync(xpl_ctx* c) {
  if (!c) return XPL_ERR_INVALID_ARG;
  CK(cudaMemcpyAsync(c->h_misc, c->d_misc, 8, cudaMemcpyDeviceToHost, c->cs));
  CK(cudaStreamSynchronize(c->cs));
  if (c->cs != c->rs) CK(cudaStreamSynchronize(c->rs));
  return split_error(c);
}

xpl_status xpl_release_stream(xpl_ctx* c, void* stream) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  cudaStream_t s = (cudaStream_t)stream;
  if (c->cs == s && s != c->rs) {  // move the runtime's pending work back onto its own stream
    CK(cudaEventRecord(c->ev_join, s));
    CK(cudaStreamWaitEvent(c->rs, c->ev_join, 0));
    c->cs = c->rs;
  }
  return XPL_OK;
}

xpl_status xpl_join(xpl_ctx* c, void* stream) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  return join(c, (cudaStream_t)stream);
}

xpl_status xpl_runtime_stream(xpl_ctx* c, void** s) {
  if (!c || !s) return XPL_ERR_INVALID_ARG;
  *s = (void*)c->rs;
  return XPL_OK;
}

xpl_status xpl_get_device_ctx(xpl_ctx* c, struct xpl_dev_ctx* d) {
  if (!c || !d) return XPL_ERR_INVALID_ARG;
  d->rows = (const xpl_dev_row*)(c->d_tab + 32);
  d->n_rows = (const unsigned int*)c->d_tab;
  d->pool = (unsigned int*)c->d_pool;
  d->cmap = c->d_cmap;
  d->smap = c->d_smap;
  d->n_super = (const unsigned long long*)(c->d_tab + 8);
  d->flags = c->d_misc;
  d->rank = (unsigned)c->rank;
  d->world = (unsigned)c->world;
  for (int q = 0; q < XPL_MAX_RANKS; ++q) {
    const bool me = q == c->rank;
    d->pools[q] = (unsigned int*)(me ? (void*)c->d_pool : c->peer_pool[q]);
    d->cmaps[q] = (unsigned char*)(me ? (void*)c->d_cmap : c->peer_cmap[q]);
    d->smaps[q] = (unsigned char*)(me ? (void*)c->d_smap : c->peer_smap[q]);
  }
  return XPL_OK;
}

xpl_status xpl_get_stats(xpl_ctx* c, xpl_stats* o) {
  if (!c || !o) return XPL_ERR_INVALID_ARG;
  unsigned long long ds[8];
  CK(cudaStreamSynchronize(c->cs));
  CK(cudaMemcpy(ds, c->d_stats, sizeof ds, cudaMemcpyDeviceToHost));
  *o = c->st;
  o->fold_chunks_max = 0;  // (not tracked by the one-kernel fold)
  o->fold_chunks = ds[3];
  o->folds = c->folds_host;
  return XPL_OK;
}

xpl_status xpl_profile(xpl_ctx* c, int enable) {
  if (!c) return XPL_ERR_INVALID_ARG;
  if (enable && !c->prof) {
    memset(c->prof_acc, 0, sizeof c->prof_acc);
    CK(cudaStreamSynchronize(c->cs));
    unsigned long long ds[8];
    CK(cudaMemcpy(ds, c->d_stats, sizeof ds, cudaMemcpyDeviceToHost));
    c->fold_entries_seen = ds[3];
  }
  c->prof = enable != 0;
  return XPL_OK;
}

xpl_status xpl_profile_read(xpl_ctx* c, xpl_kernel_time* out, int reset) {
  if (!c || !out) return XPL_ERR_INVALID_ARG;
  CK(cudaStreamSynchronize(c->cs));
  for (auto& r : c->prof_pending) {
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, r.a, r.b));
    c->prof_acc[r.cls].launches += 1;
    c->prof_acc[r.cls].ms += ms;
    c->prof_acc[r.cls].bytes += r.bytes;
    c->prof_free.push_back(r.a);
    c->prof_free.push_back(r.b);
  }
  c->prof_pending.clear();
  unsigned long long ds[8];
  CK(cudaMemcpy(ds, c->d_stats, sizeof ds, cudaMemcpyDeviceToHost));
  c->prof_acc[XPL_K_FOLD].bytes += 256ull * (ds[3] - c->fold_entries_seen);  // 128 B read + 128 B written
  c->fold_entries_seen = ds[3];
  for (int k = 0; k < XPL_K_NCLASS; ++k) out[k] = c->prof_acc[k];
  if (reset) memset(c->prof_acc, 0, sizeof c->prof_acc);
  return XPL_OK;
}

xpl_status xpl_shadow_dump(xpl_ctx* c, const void* base, uint64_t word0, uint64_t n, uint8_t* out) {
  if (!c || !out) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  auto it = c->live.find((uint64_t)base);
  if (it == c->live.end()) return XPL_ERR_UNKNOWN_PTR;
  const Row& r = c->rows[it->second];
  if (word0 > r.words || n > r.words - word0) return XPL_ERR_INVALID_ARG;
  if (r.owner != (uint32_t)c->rank) return XPL_ERR_INVALID_ARG;  // (sharded: another rank's piece)
  xpl_status s = flush(c);
  if (s) return s;
  CK(cudaMemcpyAsync(out, c->d_pool + r.off + word0, n, cudaMemcpyDeviceToHost, c->cs));
  CK(cudaStreamSynchronize(c->cs));
  return XPL_OK;
}

// A resetting diagnose drops the rows freed since the last one and recycles
// their shadow (D17); in sharded mode every rank drops every piece
// (each rank keeps every owner's pool allocator in step).
static void drop_dead(xpl_ctx* c) {
  std::vector<uint64_t> keep;
  for (uint64_t id : c->active) {
    Row& r = c->rows[id];
    if (r.live) keep.push_back(id);
    if (!r.live && !r.dropped) {
      r.dropped = true;
      c->pas[r.owner].release(r.off, r.span);
      auto it = c->lrows.find(r.logical_id);
      if (it != c->lrows.end()) {
        auto& v = it->second;
        v.erase(std::remove(v.begin(), v.end(), r.id), v.end());
        if (v.empty()) c->lrows.erase(it);
      }
    }
  }
  c->active.swap(keep);
  c->n_dead = 0;
}

// The diagnosis of every live row and every row freed since the last reset
// (tracePrint).  Fills `out` (reports) or `pout` (sharding partials).
static xpl_status diagnose_impl(xpl_ctx* c, const xpl_diag_params* params, const xpl_name* names,
                                size_t n_names, xpl_alloc_report* out, xpl_partial* pout, size_t cap,
                                size_t* n_out, int reset) {
  // (sharded mode: this rank analyses the pieces it owns)
  NvtxRange nv("xpl_diagnose");
  if (!c || !n_out || (n_names && !names)) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  DiagParams p;
  p.thr = params ? params->density_threshold_pct : 50;
  p.block_words = params ? params->block_words : 0;
  p.min_run = params ? params->min_run_words : 256;
  if (p.min_run == 0) p.min_run = 1;
  p.reset = reset ? 1 : 0;
  const uint64_t B = p.block_words;

  std::vector<uint64_t> ids;  // live rows + rows freed since the last reset, id order (D23)
  for (uint64_t id : c->active)
    if (c->rows[id].owner == (uint32_t)c->rank) ids.push_back(id);
  *n_out = ids.size();
  if (cap < ids.size() || (!out && !pout && ids.size())) return XPL_ERR_INVALID_ARG;

  xpl_status s = flush(c);
  if (s) return s;
  const size_t nr = ids.size();
  c->st.diagnoses++;
  if (nr == 0) {
    if (reset) drop_dead(c);
    return XPL_OK;
  }

  auto row_blocks = [&](const Row& r) -> uint64_t {  // logical blocks the row touches
    return B ? (r.goff + r.words - 1) / B - r.goff / B + 1 : 0;
  };
  // geometry: the tile size is halved (down to kMinTileWords) while the call
  // would not fill every SM with several warps -- small diagnoses get more,
  // shorter warps instead of a partial wave of long ones
  uint64_t total_words = 0;
  for (uint64_t id : ids) total_words += c->rows[id].words;
  uint32_t tw = kTileWords;
  while (tw > kMinTileWords && total_words / tw < 148ull * 24) tw >>= 1;
  if (const char* e = getenv("XPL_DIAG_TILE_WORDS")) {  // test knob: force a tile size
    const unsigned long v = strtoul(e, nullptr, 10);
    if (v >= kMinTileWords && v <= kTileWords && (v & (v - 1)) == 0) tw = (uint32_t)v;
  }
  p.tile_words = tw;
  p.pad = 0;
  uint64_t ntiles = 0, nblocks = 0, nseg = 0;
  for (uint64_t id : ids) {
    const Row& r = c->rows[id];
    const uint64_t nt = (r.words + tw - 1) / tw;
    ntiles += nt;
    nseg += (nt + kSegTiles - 1) / kSegTiles;
    nblocks += row_blocks(r);
  }
  if (ntiles > 0x7FFFFFFFull) return XPL_ERR_OOM;
  if (nr > c->drows_cap) {
    cudaFree(c->d_cnt);
    cudaFree(c->d_rep);
    cudaFreeHost(c->h_rep);
    cudaFree(c->d_rpart);
    cudaFreeHost(c->h_rpart);
    cudaFreeHost(c->h_cnt);
    c->drows_cap = std::max<size_t>(nr, 256);
    CK(cudaMalloc(&c->d_cnt, sizeof(unsigned long long) * C_NCNT * c->drows_cap));
    CK(cudaMalloc(&c->d_rep, sizeof(xpl_alloc_report) * c->drows_cap));
    CK(host_alloc(&c->h_rep, c->drows_cap));
    CK(cudaMalloc(&c->d_rpart, sizeof(RowPartial) * c->drows_cap));
    CK(host_alloc(&c->h_rpart, c->drows_cap));
    CK(host_alloc(&c->h_cnt, C_NCNT * c->drows_cap));
  }
  if (ntiles > c->tiles_cap) {
    cudaFree(c->d_tiles);
    c->tiles_cap = std::max<uint64_t>(ntiles, 1024);
    CK(cudaMalloc(&c->d_tiles, sizeof(TileSum) * c->tiles_cap));
  }
  if (nseg > c->segs_cap) {
    cudaFree(c->d_segsum);
    cudaFree(c->d_segcnt);
    c->segs_cap = std::max<uint64_t>(nseg, 1024);
    CK(cudaMalloc(&c->d_segsum, kRunPairBytes * c->segs_cap));
    CK(cudaMalloc(&c->d_segcnt, sizeof(unsigned long long) * 9 * c->segs_cap));
  }
  if (nblocks > c->blk_cap) {
    cudaFree(c->d_blk);
    c->blk_cap = std::max<uint64_t>(nblocks, 1024);
    CK(cudaMalloc(&c->d_blk, sizeof(uint32_t) * c->blk_cap));
  }
  auto al = [](size_t b) { return (b + 255) & ~(size_t)255; };
  const size_t o_tr = al(sizeof(DiagRow) * nr), o_sg = o_tr + al(sizeof(uint32_t) * ntiles);
  const size_t up_bytes = o_sg + sizeof(StitchSeg) * nseg;
  if (up_bytes > c->up_cap) {
    if (c->d_up) {
      CK(cudaStreamSynchronize(c->cs));
      cudaFreeHost(c->h_up);
      cudaFree(c->d_up);
    }
    c->up_cap = std::max<size_t>(up_bytes + up_bytes / 2, 1 << 16);
    CK(host_alloc(&c->h_up, c->up_cap));
    CK(cudaMalloc(&c->d_up, c->up_cap));
  }
  DiagRow* const h_drows = reinterpret_cast<DiagRow*>(c->h_up);
  uint32_t* const h_tile_row = reinterpret_cast<uint32_t*>(c->h_up + o_tr);
  StitchSeg* const h_segs = reinterpret_cast<StitchSeg*>(c->h_up + o_sg);
  const DiagRow* const d_drows = reinterpret_cast<const DiagRow*>(c->d_up);
  const uint32_t* const d_tile_row = reinterpret_cast<const uint32_t*>(c->d_up + o_tr);
  const StitchSeg* const d_segs = reinterpret_cast<const StitchSeg*>(c->d_up + o_sg);
  // fused stitch (tile kernel + one stitch kernel): no block counts, no empty row
  bool fused = B == 0 && getenv("XPL_DIAG_UNFUSED") == nullptr;
  for (uint64_t id : ids) fused = fused && c->rows[id].words > 0;
  if (fused && nr > c->done_cap) {
    if (c->d_done) {
      CK(cudaStreamSynchronize(c->cs));
      cudaFree(c->d_done);
    }
    c->done_cap = std::max<size_t>(nr, 4096);
    CK(cudaMalloc(&c->d_done, sizeof(uint32_t) * c->done_cap));
    CK(cudaMemsetAsync(c->d_done, 0, sizeof(uint32_t) * c->done_cap, c->cs));
  }
  uint64_t t = 0, b = 0, sgi = 0;
  for (size_t i = 0; i < nr; ++i) {
    const Row& r = c->rows[ids[i]];
    DiagRow& d = h_drows[i];
    d.off = r.off;
    d.words = r.words;
    d.tile0 = t;
    d.ntiles = (r.words + tw - 1) / tw;
    d.blk0 = b;
    d.nblk = row_blocks(r);
    d.goff = r.goff;
    d.lwords = (r.lbytes + 3) / 4;
    d.kind = r.kind;
    d.pad = 0;
    d.seg0 = sgi;
    d.nseg = (d.ntiles + kSegTiles - 1) / kSegTiles;
    for (uint64_t k = 0; k < d.nseg; ++k) {
      h_segs[sgi + k].t0 = t + k * kSegTiles;
      h_segs[sgi + k].n = std::min<uint64_t>(kSegTiles, d.ntiles - k * kSegTiles);
      h_segs[sgi + k].row = i;
    }
    for (uint64_t k = 0; k < d.ntiles; ++k) h_tile_row[t + k] = (uint32_t)i;
    sgi += d.nseg;
    t += d.ntiles;
    b += d.nblk;
  }
  CK(cudaMemcpyAsync(c->d_up, c->h_up, up_bytes, cudaMemcpyHostToDevice, c->cs));
  const uint64_t dbytes = total_words * (reset ? 2 : 1);
  const int pall = prof_begin(c, XPL_K_DIAGNOSE, dbytes);
  const int ptile = prof_begin(c, XPL_K_DIAG_TILE, dbytes, false);  // recorded by launch_diag
  // fused: the kernel writes the report rows (and partials, counters, the
  // epoch-split flags) straight into the pinned host buffers -- no copies back
  launch_diag(c->cs, d_drows, (uint32_t)nr, d_tile_row, ntiles, d_segs, (uint32_t)nseg,
              nblocks, p, (uint32_t*)c->d_pool, fused ? c->h_cnt : c->d_cnt, c->d_tiles, c->d_segsum, c->d_blk,
              fused ? c->h_rep : c->d_rep, pout ? (fused ? c->h_rpart : c->d_rpart) : nullptr,
              ptile >= 0 ? c->prof_pending[ptile].a : nullptr, ptile >= 0 ? c->prof_pending[ptile].b : nullptr,
              fused ? c->d_done : nullptr, c->d_segcnt, c->d_misc, fused ? c->h_misc : nullptr);
  CK(cudaGetLastError());
  c->st.kernel_launches += fused ? 2 : 3 + (B && nblocks ? 1 : 0);
  if (!fused) {
    CK(cudaMemcpyAsync(c->h_rep, c->d_rep, sizeof(xpl_alloc_report) * nr, cudaMemcpyDeviceToHost, c->cs));
    if (pout) {
      CK(cudaMemcpyAsync(c->h_rpart, c->d_rpart, sizeof(RowPartial) * nr, cudaMemcpyDeviceToHost, c->cs));
      CK(cudaMemcpyAsync(c->h_cnt, c->d_cnt, sizeof(unsigned long long) * C_NCNT * nr,
                         cudaMemcpyDeviceToHost, c->cs));
    }
    CK(cudaMemcpyAsync(c->h_misc, c->d_misc, 8, cudaMemcpyDeviceToHost, c->cs));
  }
  prof_end(c, pall);
  CK(cudaStreamSynchronize(c->cs));
  s = split_error(c);
  if (s) return s;

  std::vector<uint32_t> name_of(nr, 0xFFFFFFFFu);
  c->cache = nullptr;  // names (XplAllocData): the first name inside a live row
  for (size_t j = 0; j < n_names; ++j) {
    const Row* r = lookup(c, (uint64_t)names[j].addr);
    if (!r) continue;
    for (size_t i = 0; i < nr; ++i)
      if (ids[i] == r->id && name_of[i] == 0xFFFFFFFFu) name_of[i] = (uint32_t)j;
  }
  for (size_t i = 0; i < nr; ++i) {
    Row& r = c->rows[ids[i]];
    const xpl_alloc_report& h = c->h_rep[i];
    if (h.any_acc) r.ever = true;
    if (out) {
      xpl_alloc_report o = h;
      o.id = r.id;
      o.base = r.base;
      o.bytes = r.bytes;
      o.live = r.live ? 1 : 0;
      o.name_idx = name_of[i];
      o.ever_accessed = r.ever ? 1 : 0;
      out[i] = o;
    }
    if (pout) {
      const DiagRow& d = h_drows[i];
      const RowPartial& q = c->h_rpart[i];
      const unsigned long long* cn = c->h_cnt + (uint64_t)C_NCNT * i;
      xpl_partial o;
      memset(&o, 0, sizeof o);
      o.logical_id = r.logical_id;
      o.word_offset = r.goff;
      o.words = r.words;
      o.logical_words = d.lwords;
      o.logical_bytes = r.lbytes;
      o.base = r.base;
      o.kind = r.kind;
      o.live = r.live ? 1 : 0;
      o.name_idx = name_of[i];
      for (int k = 0; k < 9; ++k) o.cnt[k] = cn[k];
      for (int k = 0; k < 5; ++k) {
        o.u_run[k] = q.u[k];
        o.d_run[k] = q.d[k];
      }
      o.low_density_blocks = B ? cn[C_LDB] : 0;
      o.low_density_words = B ? cn[C_LDW] : 0;
      o.blk_first = o.blk_last = ~0ull;
      if (B) {  // the blocks cut by the piece's ends are combined across pieces
        const uint64_t k0 = r.goff / B, k1 = (r.goff + r.words - 1) / B;
        auto cut = [&](uint64_t k) {
          const uint64_t lo = k * B, hi = std::min(lo + B, d.lwords);
          return lo < r.goff || hi > r.goff + r.words;
        };
        auto in_piece = [&](uint64_t k) {
          const uint64_t lo = std::max(k * B, r.goff), hi = std::min(std::min(k * B + B, d.lwords), r.goff + r.words);
          return hi - lo;
        };
        if (cut(k0)) {
          o.blk_first = k0;
          o.blk_first_g = q.blk_first_g;
          o.blk_first_s = in_piece(k0);
        }
        if (k1 != k0 && cut(k1)) {
          o.blk_last = k1;
          o.blk_last_g = q.blk_last_g;
          o.blk_last_s = in_piece(k1);
        }
      }
      o.ever_accessed = r.ever ? 1 : 0;
      pout[i] = o;
    }
  }
  if (reset) drop_dead(c);
  return XPL_OK;
}

xpl_status xpl_diagnose(xpl_ctx* c, const xpl_diag_params* params, const xpl_name* names,
                        size_t n_names, xpl_alloc_report* out, size_t cap, size_t* n_out,
                        int reset) {
  if (!c || c->world <= 1) return diagnose_impl(c, params, names, n_names, out, nullptr, cap, n_out, reset);
  // sharded (COLLECTIVE): partials of the owned pieces -> all-gather -> combine
  if (!n_out || (n_names && !names)) return XPL_ERR_INVALID_ARG;
  if (c->depth) return XPL_ERR_STATE;
  std::vector<uint64_t> lids;
  size_t n_own = 0;
  for (uint64_t id : c->active) {
    const Row& r = c->rows[id];
    lids.push_back(r.logical_id);
    if (r.owner == (uint32_t)c->rank) ++n_own;
  }
  std::sort(lids.begin(), lids.end());
  lids.erase(std::unique(lids.begin(), lids.end()), lids.end());
  *n_out = lids.size();
  if (cap < lids.size() || (!out && !lids.empty())) return XPL_ERR_INVALID_ARG;  // (before any collective)
  std::vector<xpl_partial> mine(n_own + 1);
  size_t k = 0;
  xpl_status s = diagnose_impl(c, params, names, n_names, nullptr, mine.data(), n_own, &k, reset);
  if (s) return s;
  const int R = c->world;
  std::vector<uint64_t> cnt(R), sb(R), rb(R);
  const uint64_t my = k * sizeof(xpl_partial);
  if (c->comm->allgather(c->comm->user, &my, 8, cnt.data())) return XPL_ERR_NCCL;
  std::vector<uint8_t> send((size_t)my * R + 1);
  uint64_t tot = 0;
  for (int q = 0; q < R; ++q) {
    sb[q] = my;
    rb[q] = cnt[q];
    tot += cnt[q];
    memcpy(send.data() + (size_t)q * my, mine.data(), my);
  }
  std::vector<uint8_t> recv(tot + 1);
  if (c->comm->alltoallv(c->comm->user, send.data(), sb.data(), recv.data(), rb.data())) return XPL_ERR_NCCL;
  size_t no = 0;
  s = xpl_combine_partials((const xpl_partial*)recv.data(), tot / sizeof(xpl_partial), params, out, cap, &no);
  if (s) return s;
  *n_out = no;
  return XPL_OK;
}

xpl_status xpl_diagnose_partials(xpl_ctx* c, const xpl_diag_params* params, const xpl_name* names,
                                 size_t n_names, xpl_partial* out, size_t cap, size_t* n_out,
                                 int reset) {
  return diagnose_impl(c, params, names, n_names, nullptr, out, cap, n_out, reset);
}

}  // extern "C"
