// tests/native/host_tracer_check.cpp -- compiled and run by tests/test_host_tracer.py (no GPU).
// CPU check of xpl_host.h's coalescing: random access streams over a few
// arrays, emitted ranges expanded to per-word sequences must equal the
// per-word sequences of the raw accesses (up to idempotent repeats).
#include <cstdio>
#include <cstdlib>
#include <map>
#include <vector>
#include <random>
#include "xpl.h"
static std::vector<xpl_host_access> got;
static size_t n_strided = 0;
extern "C" xpl_status xpl_record_host_strided(xpl_ctx*, const xpl_host_strided* r, size_t n) {
  for (size_t i = 0; i < n; ++i) {
    if (r[i].count > 1) ++n_strided;
    for (uint64_t j = 0; j < r[i].count; ++j)
      got.push_back(xpl_host_access{r[i].addr + (uint64_t)r[i].stride * j, r[i].size, r[i].kind});
  }
  return XPL_OK;
}
#include "xpl_host.h"
typedef std::map<uint64_t, std::vector<int>> Seq;
static void add(Seq& s, uint64_t a, uint32_t size, int k) {
  for (uint64_t w = a / 4; w <= (a + size - 1) / 4; ++w) {
    std::vector<int>& v = s[w];
    // canonical: R/W repeats collapse (R after R, W after W); RW = R then W
    if (k == 3) { if (v.empty() || v.back() != 1) v.push_back(1); v.push_back(2); continue; }
    if (v.empty() || v.back() != k) v.push_back(k);
  }
}
int main() {
  std::mt19937_64 rng(1);
  for (int trial = 0; trial < 2000; ++trial) {
    got.clear();
    Seq want, have;
    {
      xpl_host_tracer tr(nullptr);
      int nstreams = 1 + rng() % 6;
      std::vector<uint64_t> pos(nstreams), base(nstreams);
      std::vector<int> kind(nstreams), sz(nstreams);
      std::vector<xpl_host_site> site(nstreams);
      for (int s = 0; s < nstreams; ++s) {
        base[s] = 0x1000 + (rng() % 8) * 64 + (rng() % 3);  // arrays may overlap / be adjacent
        pos[s] = base[s];
        kind[s] = 1 + rng() % 3;
        int sizes[4] = {1, 2, 4, 8};
        sz[s] = sizes[rng() % 4];
      }
      int n = 1 + rng() % (trial % 3 == 2 ? 3000 : 300);
      for (int i = 0; i < n; ++i) {
        int s = rng() % nstreams;
        const bool scatter = (trial % 3 == 2) && (rng() % 2 == 0);  // scattered mode
        // trial % 5 == 4: column walks (strided) mixed in
        const bool walk = (trial % 5 == 4) && (rng() % 4 != 0);
        uint64_t a = walk ? base[s] + ((uint64_t)(i / nstreams) * (16 + 8 * s)) % 8192
                   : scatter ? 0x1000 + rng() % 4096 : (rng() % 10 == 0) ? base[s] + (rng() % 64) : pos[s];
        int k = (rng() % 15 == 0) ? 1 + rng() % 3 : kind[s];
        // trial % 4: 0 no hint (current-run prediction), 1 one site per stream,
        // 2 one site shared by all streams, 3 per-stream sites scrambled now and then
        const int mode = trial % 4;
        if (mode == 0) {
          tr.access((void*)a, sz[s], k);
        } else {
          xpl_host_site& h = site[mode == 2 ? 0 : s];
          if (mode == 3 && rng() % 7 == 0) h.slot = rng() % 9;  // stale / foreign / never-open slot
          tr.access((void*)a, sz[s], k, h);
        }
        add(want, a, sz[s], k);
        pos[s] = a + sz[s];
      }
      tr.flush();
    }
    for (auto& r : got) add(have, r.addr, r.size, r.kind);
    if (want != have) { printf("MISMATCH trial %d\n", trial); return 1; }
  }
  printf("tracer ok, last trial %zu records, %zu strided records overall\n", got.size(), n_strided);
  if (n_strided == 0) { printf("no strided record was ever formed\n"); return 1; }
  return 0;
}
