// oracle/xpl_oracle.cpp -- TEST INFRASTRUCTURE ONLY (see xpl_oracle.h).
//
// The plain definition of XPlacer's bookkeeping, replayed sequentially:
// an ordered map (allocation id, word) -> shadow record, exactly as the
// north_star asks ("an ordered map of word to shadow record, replaying the
// trace sequentially").  Nothing is blocked, fused, vectorised or reordered.
// Readings where the paper is silent are SURVEY.md §8(c) D1-D24, restated
// in DESIGN.md §3; each is cited where it is used.
//
// Record layout (one byte per 32-bit word):
//   bit0 L   processor of the last write, 0 = CPU, 1 = GPU
//   bit2 wC  written by the CPU in this interval          (Fig. 4 "C")
//   bit3 wG  written by the GPU in this interval          (Fig. 4 "G")
//   bit4 rCC CPU read a CPU-origin value                  (Fig. 4 "C>C")
//   bit5 rGC CPU read a GPU-origin value                  (Fig. 4 "G>C")
//   bit6 rCG GPU read a CPU-origin value                  (Fig. 4 "C>G")
//   bit7 rGG GPU read a GPU-origin value                  (Fig. 4 "G>G")
// (bit1 is the GPU path's pending-write bit; the oracle has no use for it:
//  it keeps the epoch's read and write sets instead.)

#include "xpl_oracle.h"

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <set>
#include <string>
#include <utility>
#include <vector>

namespace {

const uint8_t kL = 1u << 0;
const uint8_t kWC = 1u << 2;
const uint8_t kWG = 1u << 3;
const uint8_t kRCC = 1u << 4;
const uint8_t kRGC = 1u << 5;
const uint8_t kRCG = 1u << 6;
const uint8_t kRGG = 1u << 7;

const uint32_t kAccR = 1, kAccW = 2;
const uint32_t kDevice = 0, kManaged = 1;

const uint32_t kFlagAlternating = 1, kFlagLowDensity = 2, kFlagUnneededH2D = 4,
               kFlagUnneededD2H = 8, kFlagUnused = 16;

struct Row {
  uint64_t id, base, bytes, words;
  uint32_t kind;
  bool live;
  bool ever;
  uint32_t advice;  // cudaMemAdvise hints in force (bits below), D33
};

// cudaMemAdvise hints as bits: ReadMostly, PreferredLocation GPU /
// CPU, AccessedBy GPU / CPU.
const uint32_t kAdvReadMostly = 1, kAdvPrefGpu = 2, kAdvPrefCpu = 4, kAdvByGpu = 8, kAdvByCpu = 16;

typedef std::pair<uint64_t, uint64_t> Key;  // (allocation id, word)

struct HostOp {  // a host event queued while a GPU epoch is open (D20)
  int type;      // 0 = access, 1 = copy
  uint64_t a, b, c;
  uint32_t d;
};

}  // namespace

struct xo_state {
  std::vector<Row> rows;                 // every row ever registered, by id
  std::map<uint64_t, uint64_t> live;     // base -> id, live rows only
  std::set<uint64_t> dead;               // ids freed since the last reset (D17)
  std::map<Key, uint8_t> shadow;         // missing key = record 0 (D3: L = CPU)
  int gpu_open = 0;                      // epoch nesting depth (D19)
  std::set<Key> rset, wset;              // GPU reads / writes of the open epoch
  std::vector<HostOp> pending;           // host events during an open epoch (D20)
};

namespace {

uint8_t get(xo_state* s, const Key& k) {
  std::map<Key, uint8_t>::iterator it = s->shadow.find(k);
  return it == s->shadow.end() ? 0 : it->second;
}

void put(xo_state* s, const Key& k, uint8_t v) { s->shadow[k] = v; }

// Lookup: the live row whose [base, base+bytes) holds addr; a miss
// means the access is ignored.  The access covers words
// (addr-base)>>2 .. (addr+size-1-base)>>2, clipped to the allocation (D1, D18).
bool lookup(xo_state* s, uint64_t addr, uint64_t size, uint64_t* id,
            uint64_t* w0, uint64_t* w1) {
  if (size == 0) return false;
  std::map<uint64_t, uint64_t>::iterator it = s->live.upper_bound(addr);
  if (it == s->live.begin()) return false;
  --it;
  const Row& r = s->rows[it->second];
  if (addr >= r.base + r.bytes) return false;
  *id = r.id;
  *w0 = (addr - r.base) >> 2;
  uint64_t last = (addr + size - 1 - r.base) >> 2;
  *w1 = last < r.words - 1 ? last : r.words - 1;
  return true;
}

// A host access, applied immediately in program order (host tracer, the
// !__CUDA_ARCH__ branch).  R sets the read bit of the value's origin
// (the last writer); W sets wC and makes the CPU the last writer.
// RW = read, then write (D6).
void host_access(xo_state* s, uint64_t addr, uint64_t size, uint32_t acc) {
  uint64_t id, w0, w1;
  if (!lookup(s, addr, size, &id, &w0, &w1)) return;
  s->rows[id].ever = true;
  for (uint64_t w = w0; w <= w1; ++w) {
    Key k(id, w);
    uint8_t rec = get(s, k);
    if (acc & kAccR) rec |= (rec & kL) ? kRGC : kRCC;
    if (acc & kAccW) rec = (uint8_t)((rec | kWC) & ~kL);
    put(s, k, rec);
  }
}

// A device access inside an open GPU epoch: only remembered; its effect is
// applied when the epoch closes (snapshot semantics, D5).
void dev_access(xo_state* s, uint64_t addr, uint64_t size, uint32_t acc) {
  uint64_t id, w0, w1;
  if (!lookup(s, addr, size, &id, &w0, &w1)) return;
  s->rows[id].ever = true;
  for (uint64_t w = w0; w <= w1; ++w) {
    if (acc & kAccR) s->rset.insert(Key(id, w));
    if (acc & kAccW) s->wset.insert(Key(id, w));
  }
}

void kernel_begin(xo_state* s) {
  if (s->gpu_open++ == 0) {
    s->rset.clear();
    s->wset.clear();
  }
}

void apply_copy(xo_state* s, uint64_t dst, uint64_t src, uint64_t bytes,
                uint32_t dir);

void kernel_end(xo_state* s) {
  if (--s->gpu_open != 0) return;
  // Reads first, with the last writer as of the epoch start (D5) ...
  for (std::set<Key>::iterator it = s->rset.begin(); it != s->rset.end(); ++it) {
    uint8_t rec = get(s, *it);
    rec |= (rec & kL) ? kRGG : kRCG;
    put(s, *it, rec);
  }
  // ... then writes: wG, and the GPU becomes the last writer.
  for (std::set<Key>::iterator it = s->wset.begin(); it != s->wset.end(); ++it) {
    uint8_t rec = get(s, *it);
    rec = (uint8_t)(rec | kWG | kL);
    put(s, *it, rec);
  }
  s->rset.clear();
  s->wset.clear();
  // Host events issued while the epoch was open form the next host segment (D20).
  std::vector<HostOp> q;
  q.swap(s->pending);
  for (size_t i = 0; i < q.size(); ++i) {
    if (q[i].type == 0) host_access(s, q[i].a, q[i].b, q[i].d);
    else apply_copy(s, q[i].a, q[i].b, q[i].c, q[i].d);
  }
}

// Transfers (D7): H2D = a CPU write of every destination word;
// D2H = a CPU read of every source word; H2H = read src, write dst;
// D2D and device memset = GPU accesses, in their own epoch unless one is open.
void apply_copy(xo_state* s, uint64_t dst, uint64_t src, uint64_t bytes,
                uint32_t dir) {
  switch (dir) {
    case 0: host_access(s, dst, bytes, kAccW); break;
    case 1: host_access(s, src, bytes, kAccR); break;
    case 2:
      host_access(s, src, bytes, kAccR);
      host_access(s, dst, bytes, kAccW);
      break;
    case 3:
      kernel_begin(s);
      dev_access(s, src, bytes, kAccR);
      dev_access(s, dst, bytes, kAccW);
      kernel_end(s);
      break;
    case 4:
      kernel_begin(s);
      dev_access(s, dst, bytes, kAccW);
      kernel_end(s);
      break;
  }
}

// Maximal runs of a per-word predicate inside one allocation; a run counts
// when its length is >= min_run ("minimum block size ... is
// parametrizable", D16).
void runs(const std::vector<bool>& f, uint64_t min_run, uint64_t* count,
          uint64_t* words) {
  *count = 0;
  *words = 0;
  uint64_t i = 0, n = f.size();
  while (i < n) {
    if (!f[i]) { ++i; continue; }
    uint64_t j = i;
    while (j < n && f[j]) ++j;
    if (j - i >= min_run) { *count += 1; *words += j - i; }
    i = j;
  }
}

}  // namespace

extern "C" {

xo_state* xo_new(void) { return new xo_state(); }
void xo_delete(xo_state* s) { delete s; }

// Registration (the cudaMalloc/cudaMallocManaged/malloc wrappers):
// ceil(bytes/4) records, all zero (D3).  Overlap with a live row is an error.
int64_t xo_reg(xo_state* s, uint64_t ptr, uint64_t bytes, uint32_t kind) {
  if (bytes == 0 || kind > 2 || s->gpu_open) return -1;
  std::map<uint64_t, uint64_t>::iterator it = s->live.lower_bound(ptr);
  if (it != s->live.end() && it->first < ptr + bytes) return -2;
  if (it != s->live.begin()) {
    --it;
    const Row& p = s->rows[it->second];
    if (p.base + p.bytes > ptr) return -2;
  }
  Row r;
  r.id = s->rows.size();
  r.base = ptr;
  r.bytes = bytes;
  r.words = (bytes + 3) / 4;
  r.kind = kind;
  r.live = true;
  r.ever = false;
  r.advice = 0;
  s->rows.push_back(r);
  s->live[ptr] = r.id;
  return (int64_t)r.id;
}

// Free: the memory goes now, its shadow stays until the next
// diagnostic (D17).
int xo_free(xo_state* s, uint64_t ptr) {
  if (s->gpu_open) return -1;
  std::map<uint64_t, uint64_t>::iterator it = s->live.find(ptr);
  if (it == s->live.end()) return -3;
  s->rows[it->second].live = false;
  s->dead.insert(it->second);
  s->live.erase(it);
  return 0;
}

int xo_kb(xo_state* s) {
  kernel_begin(s);
  return 0;
}

int xo_ke(xo_state* s) {
  if (s->gpu_open == 0) return -1;
  kernel_end(s);
  return 0;
}

int xo_host(xo_state* s, uint64_t addr, uint32_t size, uint32_t acc) {
  if (acc < 1 || acc > 3) return -1;
  if (s->gpu_open) {
    HostOp op = {0, addr, size, 0, acc};
    s->pending.push_back(op);
  } else {
    host_access(s, addr, size, acc);
  }
  return 0;
}

int xo_host_batch(xo_state* s, const uint64_t* addr, const uint32_t* size,
                  const uint8_t* acc, size_t n) {
  for (size_t i = 0; i < n; ++i)
    if (xo_host(s, addr[i], size[i], acc[i]) != 0) return -1;
  return 0;
}

int xo_dev(xo_state* s, uint64_t addr, uint32_t size, uint32_t acc) {
  if (s->gpu_open == 0 || acc < 1 || acc > 3) return -1;
  dev_access(s, addr, size, acc);
  return 0;
}

int xo_dev_batch(xo_state* s, const uint64_t* addr, const uint32_t* size,
                 const uint8_t* acc, size_t n) {
  for (size_t i = 0; i < n; ++i)
    if (xo_dev(s, addr[i], size[i], acc[i]) != 0) return -1;
  return 0;
}

int xo_copy(xo_state* s, uint64_t dst, uint64_t src, uint64_t bytes,
            uint32_t dir) {
  if (dir > 4) return -1;
  if (s->gpu_open && dir <= 2) {  // host-side effect: next host segment (D20)
    HostOp op = {1, dst, src, bytes, dir};
    s->pending.push_back(op);
    return 0;
  }
  apply_copy(s, dst, src, bytes, dir);  // D2D / memset join an open epoch (D19)
  return 0;
}

// The diagnosis (tracePrint; summary counts, Fig. 4 / P:L301).
int64_t xo_diag(xo_state* s, uint32_t thr_pct, uint64_t block_words,
                uint64_t min_run, int reset, const uint64_t* name_addrs,
                size_t n_names, xo_report* out, size_t cap) {
  if (s->gpu_open) return -1;
  if (min_run == 0) min_run = 1;
  std::vector<uint64_t> ids;  // live and dead rows, in id order (D23)
  for (size_t i = 0; i < s->rows.size(); ++i)
    if (s->rows[i].live || s->dead.count(i)) ids.push_back(i);
  if (ids.size() > cap) return (int64_t)ids.size();

  for (size_t k = 0; k < ids.size(); ++k) {
    const Row& r = s->rows[ids[k]];
    xo_report rep;
    std::memset(&rep, 0, sizeof(rep));
    rep.id = r.id;
    rep.base = r.base;
    rep.bytes = r.bytes;
    rep.words = r.words;
    rep.kind = r.kind;
    rep.live = r.live ? 1 : 0;
    rep.name_idx = 0xFFFFFFFFu;
    std::vector<bool> gpu(r.words), u(r.words), d(r.words);
    for (uint64_t w = 0; w < r.words; ++w) {
      uint8_t rec = get(s, Key(r.id, w));
      bool wc = rec & kWC, wg = rec & kWG, rcc = rec & kRCC, rgc = rec & kRGC,
           rcg = rec & kRCG, rgg = rec & kRGG;
      bool cpu_acc = wc || rcc || rgc;
      bool gpu_acc = wg || rcg || rgg;
      // Each address counted at most once per column (D21).
      rep.w_c += wc;
      rep.w_g += wg;
      rep.r_cc += rcc;
      rep.r_cg += rcg;
      rep.r_gc += rgc;
      rep.r_gg += rgg;
      rep.any_acc += (cpu_acc || gpu_acc);
      rep.gpu_acc += gpu_acc;
      // Alternating: accessed by both CPU and GPU, at least one a write (D9).
      rep.alternating += (cpu_acc && gpu_acc && (wc || wg));
      gpu[w] = gpu_acc;
      u[w] = wc && !rcg;  // sent to the GPU, never consumed there (D14)
      d[w] = rcc;         // read back by the CPU, not updated by the GPU (D15)
    }
    // Density = accessed / size (Eq. P:L102) with GPU accesses as "accessed" (D10),
    // printed as a floored integer percent (Fig. 4, D22).
    rep.density_pct_any = rep.any_acc * 100 / r.words;
    rep.density_pct_gpu = rep.gpu_acc * 100 / r.words;
    // Low density per block: a block is diagnosed when it has at least
    // one access and sum(accessed)/size <= threshold (Eq. P:L102, D11-D13).
    uint64_t B = block_words ? block_words : r.words;
    for (uint64_t b0 = 0; b0 < r.words; b0 += B) {
      uint64_t b1 = b0 + B < r.words ? b0 + B : r.words;
      uint64_t g = 0;
      for (uint64_t w = b0; w < b1; ++w) g += gpu[w];
      uint64_t sz = b1 - b0;
      if (g >= 1 && 100 * g <= (uint64_t)thr_pct * sz) {
        rep.low_density_blocks += 1;
        rep.low_density_words += sz;
      }
    }
    runs(u, min_run, &rep.h2d_unused_runs, &rep.h2d_unused_words);
    runs(d, min_run, &rep.d2h_unneeded_runs, &rep.d2h_unneeded_words);
    bool ever = r.ever;
    rep.ever_accessed = ever ? 1 : 0;
    // Pattern flags, gated by how the memory was allocated (P:L84, P:L97-99,
    // P:L114, D8).
    if (r.kind == kManaged && rep.alternating > 0) rep.flags |= kFlagAlternating;
    if ((r.kind == kDevice || r.kind == kManaged) && rep.low_density_blocks > 0)
      rep.flags |= kFlagLowDensity;
    if (r.kind == kDevice && rep.h2d_unused_runs > 0) rep.flags |= kFlagUnneededH2D;
    if (r.kind == kDevice && rep.d2h_unneeded_runs > 0) rep.flags |= kFlagUnneededD2H;
    if (rep.any_acc == 0) rep.flags |= kFlagUnused;
    out[k] = rep;
  }
  // Names (XplAllocData): the first name whose address lies in a
  // live row names it (D23).
  for (size_t j = 0; j < n_names; ++j) {
    uint64_t id, w0, w1;
    if (!lookup(s, name_addrs[j], 1, &id, &w0, &w1)) continue;
    for (size_t k = 0; k < ids.size(); ++k)
      if (out[k].id == id && out[k].name_idx == 0xFFFFFFFFu)
        out[k].name_idx = (uint32_t)j;
  }
  // Reset: clear the interval bits, keep the last writer (D4);
  // dead rows are dropped (D17).
  if (reset) {
    for (std::map<Key, uint8_t>::iterator it = s->shadow.begin();
         it != s->shadow.end();) {
      if (!s->rows[it->first.first].live) {
        s->shadow.erase(it++);
      } else {
        it->second &= kL;
        ++it;
      }
    }
    s->dead.clear();
  }
  return (int64_t)ids.size();
}

// UM page view (NEXT-3).  For page p of a live row (words [p*P, min((p+1)*P,
// words)), D31) the OR over its words of: accessed by the CPU (wC, rCC or rGC),
// by the GPU (wG, rCG or rGG), by both, alternating (both and written, D9).
// A page is shared if both processors touched it -- under unified memory it
// would move between them; false-shared if no single word was
// touched by both ("an effect similar to false sharing").  Flags only
// for managed allocations (D8): FALSE_SHARING = some false-shared page;
// ADVICE_MISMATCH = ReadMostly advised yet some page alternates, i.e. a write
// to data the other processor also uses invalidates its read copies (P:L47,
// P:L86, D32).
int64_t xo_pages(xo_state* s, uint64_t P, xo_page_report* out, size_t cap) {
  if (P == 0) return -1;
  size_t n = 0;
  for (size_t id = 0; id < s->rows.size(); ++id) {
    const Row& r = s->rows[id];
    if (!r.live) continue;
    if (n < cap) {
      xo_page_report& o = out[n];
      std::memset(&o, 0, sizeof o);
      o.id = r.id;
      o.base = r.base;
      o.words = r.words;
      o.page_words = P;
      o.pages = (r.words + P - 1) / P;
      o.kind = r.kind;
      o.advice = r.advice;
      for (uint64_t p = 0; p < o.pages; ++p) {
        bool cpu = false, gpu = false, both = false, alt = false;
        for (uint64_t w = p * P; w < (p + 1) * P && w < r.words; ++w) {
          const uint8_t rec = get(s, Key(r.id, w));
          const bool c = (rec & kWC) || (rec & kRCC) || (rec & kRGC);
          const bool g = (rec & kWG) || (rec & kRCG) || (rec & kRGG);
          cpu = cpu || c;
          gpu = gpu || g;
          both = both || (c && g);
          alt = alt || (c && g && ((rec & kWC) || (rec & kWG)));
        }
        if (cpu) o.cpu_pages++;
        if (gpu) o.gpu_pages++;
        if (cpu && gpu) o.shared_pages++;
        if (cpu && gpu && !both) o.false_shared_pages++;
        if (alt) o.alternating_pages++;
      }
      if (r.kind == kManaged) {
        if (o.false_shared_pages > 0) o.flags |= 1;
        if ((r.advice & kAdvReadMostly) && o.alternating_pages > 0) o.flags |= 2;
      }
    }
    ++n;
  }
  return (int64_t)n;
}

// cudaMemAdvise wrapper: the hint applies to the whole allocation holding ptr
// (D33); untracked pointers are ignored.  Set/Unset pairs in the
// order of the cudaMemoryAdvise enum: 1/2 ReadMostly, 3/4 PreferredLocation,
// 5/6 AccessedBy; a negative device means the CPU (cudaCpuDeviceId).
int xo_advise(xo_state* s, uint64_t ptr, uint32_t advice, int device) {
  if (advice < 1 || advice > 6) return -1;
  uint64_t id, w0, w1;
  if (!lookup(s, ptr, 1, &id, &w0, &w1)) return 0;
  uint32_t& a = s->rows[id].advice;
  const bool cpu = device < 0;
  if (advice == 1) a |= kAdvReadMostly;
  if (advice == 2) a &= ~kAdvReadMostly;
  if (advice == 3) a = (a & ~(kAdvPrefGpu | kAdvPrefCpu)) | (cpu ? kAdvPrefCpu : kAdvPrefGpu);
  if (advice == 4) a &= ~(kAdvPrefGpu | kAdvPrefCpu);
  if (advice == 5) a |= cpu ? kAdvByCpu : kAdvByGpu;
  if (advice == 6) a &= ~(cpu ? kAdvByCpu : kAdvByGpu);
  return 0;
}

int xo_peek(xo_state* s, uint64_t id, uint64_t word) {
  if (id >= s->rows.size()) return -1;
  return get(s, Key(id, word));
}

}  // extern "C"

// ---------------------------------------------------------------------------
// Command-line driver: replays a text trace (SURVEY §8c trace language) and
// prints one JSON object per DIAG row.  Used for the golden hand traces.
//   REG ptr bytes kind | FREE ptr | KB | KE | H addr size acc | D addr size acc
//   X dir dst src bytes | DIAG thr block_words min_run reset [name_addr ...]
// kind: D|M|H or 0|1|2; acc: R|W|RW or 1|2|3; numbers may be 0x-hex.
#ifdef XPL_ORACLE_MAIN
#include <sstream>
#include <fstream>
#include <iostream>

static uint64_t num(const std::string& t) { return std::strtoull(t.c_str(), 0, 0); }
static uint32_t kind_of(const std::string& t) {
  if (t == "D") return 0;
  if (t == "M") return 1;
  if (t == "H") return 2;
  return (uint32_t)num(t);
}
static uint32_t acc_of(const std::string& t) {
  if (t == "R") return 1;
  if (t == "W") return 2;
  if (t == "RW") return 3;
  return (uint32_t)num(t);
}

int main(int argc, char** argv) {
  if (argc < 2) {
    std::fprintf(stderr, "usage: %s trace.txt\n", argv[0]);
    return 2;
  }
  std::ifstream in(argv[1]);
  xo_state* s = xo_new();
  std::string line;
  int diag_no = 0, lineno = 0;
  while (std::getline(in, line)) {
    ++lineno;
    size_t h = line.find('#');
    if (h != std::string::npos) line = line.substr(0, h);
    std::istringstream ss(line);
    std::vector<std::string> t;
    std::string w;
    while (ss >> w) t.push_back(w);
    if (t.empty()) continue;
    int rc = 0;
    if (t[0] == "REG") rc = xo_reg(s, num(t[1]), num(t[2]), kind_of(t[3])) < 0 ? -1 : 0;
    else if (t[0] == "FREE") rc = xo_free(s, num(t[1]));
    else if (t[0] == "KB") rc = xo_kb(s);
    else if (t[0] == "KE") rc = xo_ke(s);
    else if (t[0] == "H") rc = xo_host(s, num(t[1]), (uint32_t)num(t[2]), acc_of(t[3]));
    else if (t[0] == "D") rc = xo_dev(s, num(t[1]), (uint32_t)num(t[2]), acc_of(t[3]));
    else if (t[0] == "X") rc = xo_copy(s, num(t[2]), num(t[3]), num(t[4]), (uint32_t)num(t[1]));
    else if (t[0] == "DIAG") {
      std::vector<uint64_t> names;
      for (size_t i = 5; i < t.size(); ++i) names.push_back(num(t[i]));
      std::vector<xo_report> rep(s->rows.size() + 1);
      int64_t n = xo_diag(s, (uint32_t)num(t[1]), num(t[2]), num(t[3]), (int)num(t[4]),
                          names.data(), names.size(), rep.data(), rep.size());
      if (n < 0) rc = -1;
      for (int64_t i = 0; i < n; ++i) {
        const xo_report& r = rep[i];
        std::printf(
            "{\"diag\":%d,\"id\":%llu,\"base\":%llu,\"bytes\":%llu,\"words\":%llu,"
            "\"kind\":%u,\"live\":%u,\"name_idx\":%u,\"flags\":%u,\"w_c\":%llu,"
            "\"w_g\":%llu,\"r_cc\":%llu,\"r_cg\":%llu,\"r_gc\":%llu,\"r_gg\":%llu,"
            "\"any_acc\":%llu,\"gpu_acc\":%llu,\"alternating\":%llu,"
            "\"density_pct_any\":%llu,\"density_pct_gpu\":%llu,"
            "\"low_density_blocks\":%llu,\"low_density_words\":%llu,"
            "\"h2d_unused_runs\":%llu,\"h2d_unused_words\":%llu,"
            "\"d2h_unneeded_runs\":%llu,\"d2h_unneeded_words\":%llu,"
            "\"ever_accessed\":%llu}\n",
            diag_no, (unsigned long long)r.id, (unsigned long long)r.base,
            (unsigned long long)r.bytes, (unsigned long long)r.words, r.kind, r.live,
            r.name_idx, r.flags, (unsigned long long)r.w_c, (unsigned long long)r.w_g,
            (unsigned long long)r.r_cc, (unsigned long long)r.r_cg,
            (unsigned long long)r.r_gc, (unsigned long long)r.r_gg,
            (unsigned long long)r.any_acc, (unsigned long long)r.gpu_acc,
            (unsigned long long)r.alternating, (unsigned long long)r.density_pct_any,
            (unsigned long long)r.density_pct_gpu,
            (unsigned long long)r.low_density_blocks,
            (unsigned long long)r.low_density_words,
            (unsigned long long)r.h2d_unused_runs, (unsigned long long)r.h2d_unused_words,
            (unsigned long long)r.d2h_unneeded_runs,
            (unsigned long long)r.d2h_unneeded_words,
            (unsigned long long)r.ever_accessed);
      }
      ++diag_no;
    } else {
      std::fprintf(stderr, "line %d: unknown op %s\n", lineno, t[0].c_str());
      return 2;
    }
    if (rc != 0) {
      std::fprintf(stderr, "line %d: rejected (%d)\n", lineno, rc);
      return 3;
    }
  }
  xo_delete(s);
  return 0;
}
#endif
