// combine.cpp -- host-side combination of sharded diagnosis partials (SURVEY
// §8(e)): one report per logical allocation, byte-identical to the report of
// the unsharded allocation.  Counters add; transfer runs are stitched with the
// run monoid in logical word order (exactly associative); density blocks cut
// by piece ends are summed by logical block index, then judged (P:L253,
// Eq. P:L102, D11-D13).  Needs no GPU (the partials are plain data).
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <map>
#include <vector>

#include "xpl.h"

namespace {

struct Run {
  uint64_t len, pre, suf, cnt, sum;
};

Run combine(const Run& a, const Run& b, uint64_t min_run) {
  Run r;
  const bool af = a.pre == a.len, bf = b.pre == b.len;
  r.len = a.len + b.len;
  r.pre = af ? a.len + b.pre : a.pre;
  r.suf = bf ? b.len + a.suf : b.suf;
  r.cnt = a.cnt + b.cnt;
  r.sum = a.sum + b.sum;
  if (!af && !bf) {
    const uint64_t mid = a.suf + b.pre;
    if (mid > 0 && mid >= min_run) {
      r.cnt += 1;
      r.sum += mid;
    }
  }
  return r;
}

void finish(const Run& s, uint64_t min_run, uint64_t* runs, uint64_t* words) {
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

Run run_of(const uint64_t* v) { return Run{v[0], v[1], v[2], v[3], v[4]}; }

}  // namespace

extern "C" xpl_status xpl_combine_partials(const xpl_partial* parts, size_t n,
                                           const xpl_diag_params* params, xpl_alloc_report* out,
                                           size_t cap, size_t* n_out) {
  if ((!parts && n) || !n_out) return XPL_ERR_INVALID_ARG;
  const uint32_t thr = params ? params->density_threshold_pct : 50;
  const uint64_t B = params ? params->block_words : 0;
  uint64_t min_run = params ? params->min_run_words : 256;
  if (min_run == 0) min_run = 1;
  std::map<uint64_t, std::vector<const xpl_partial*>> by;
  for (size_t i = 0; i < n; ++i) by[parts[i].logical_id].push_back(&parts[i]);
  *n_out = by.size();
  if (cap < by.size() || (!out && !by.empty())) return XPL_ERR_INVALID_ARG;
  size_t k = 0;
  for (auto& kv : by) {
    std::vector<const xpl_partial*>& v = kv.second;
    std::sort(v.begin(), v.end(), [](const xpl_partial* a, const xpl_partial* b) {
      return a->word_offset < b->word_offset;
    });
    const uint64_t lw = v[0]->logical_words;
    uint64_t at = 0;
    for (const xpl_partial* p : v) {  // the pieces must tile [0, lw)
      if (p->word_offset != at || p->logical_words != lw) return XPL_ERR_INVALID_ARG;
      at += p->words;
    }
    if (at != lw) return XPL_ERR_INVALID_ARG;
    xpl_alloc_report o;
    memset(&o, 0, sizeof o);
    o.id = kv.first;
    o.base = v[0]->base;
    o.bytes = v[0]->logical_bytes;
    o.words = lw;
    o.kind = v[0]->kind;
    o.live = 1;
    o.name_idx = 0xFFFFFFFFu;
    uint64_t c[9] = {0};
    Run u = {0, 0, 0, 0, 0}, d = {0, 0, 0, 0, 0};
    std::map<uint64_t, std::pair<uint64_t, uint64_t>> cut;  // block -> (gpu words, words)
    for (const xpl_partial* p : v) {
      for (int j = 0; j < 9; ++j) c[j] += p->cnt[j];
      u = combine(u, run_of(p->u_run), min_run);
      d = combine(d, run_of(p->d_run), min_run);
      o.low_density_blocks += p->low_density_blocks;
      o.low_density_words += p->low_density_words;
      if (p->blk_first != ~0ull) {
        cut[p->blk_first].first += p->blk_first_g;
        cut[p->blk_first].second += p->blk_first_s;
      }
      if (p->blk_last != ~0ull) {
        cut[p->blk_last].first += p->blk_last_g;
        cut[p->blk_last].second += p->blk_last_s;
      }
      o.live = o.live && p->live;
      o.name_idx = std::min(o.name_idx, p->name_idx);
      o.ever_accessed |= p->ever_accessed;
    }
    o.w_c = c[0];
    o.w_g = c[1];
    o.r_cc = c[2];
    o.r_cg = c[3];
    o.r_gc = c[4];
    o.r_gg = c[5];
    o.any_acc = c[6];
    o.gpu_acc = c[7];
    o.alternating = c[8];
    o.density_pct_any = o.any_acc * 100 / lw;
    o.density_pct_gpu = o.gpu_acc * 100 / lw;
    if (B == 0) {  // the whole allocation is one block
      const bool f = o.gpu_acc >= 1 && 100ull * o.gpu_acc <= (uint64_t)thr * lw;
      o.low_density_blocks = f ? 1 : 0;
      o.low_density_words = f ? lw : 0;
    } else {
      for (auto& b : cut) {
        const uint64_t s = std::min(B, lw - b.first * B);
        if (b.second.second != s) return XPL_ERR_INVALID_ARG;  // a piece is missing
        if (b.second.first >= 1 && 100ull * b.second.first <= (uint64_t)thr * s) {
          o.low_density_blocks += 1;
          o.low_density_words += s;
        }
      }
    }
    finish(u, min_run, &o.h2d_unused_runs, &o.h2d_unused_words);
    finish(d, min_run, &o.d2h_unneeded_runs, &o.d2h_unneeded_words);
    uint32_t f = 0;
    if (o.kind == XPL_ALLOC_MANAGED && o.alternating > 0) f |= XPL_PAT_ALTERNATING;
    if (o.kind != XPL_ALLOC_HOST && o.low_density_blocks > 0) f |= XPL_PAT_LOW_DENSITY;
    if (o.kind == XPL_ALLOC_DEVICE && o.h2d_unused_runs > 0) f |= XPL_PAT_UNNEEDED_H2D;
    if (o.kind == XPL_ALLOC_DEVICE && o.d2h_unneeded_runs > 0) f |= XPL_PAT_UNNEEDED_D2H;
    if (o.any_acc == 0) f |= XPL_PAT_UNUSED;
    o.flags = f;
    out[k++] = o;
  }
  return XPL_OK;
}
