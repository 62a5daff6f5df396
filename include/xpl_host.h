/* include/xpl_host.h -- header-only host tracer: the !__CUDA_ARCH__ branch of
 * traceR / traceW / traceRW (Table I) as an inline C++
 * object the instrumented host code calls per access.
 *
 *     xpl_host_tracer tr(ctx);
 *     for (i...) tr.write(a[i]) = ...;       // = traceW(a[i]) = ...
 *     x = tr.read(b[i]);                     // = traceR(b[i])
 *     tr.flush();                            // before kernel launches / diagnose
 *
 * Coalescing, in the caller's thread: the tracer keeps up to kRuns open runs,
 * each a byte range [beg, end) of one access kind.  Invariant: the open runs
 * are pairwise disjoint at 32-bit-word granularity.  An access
 *   - that lies inside an open run of its kind (R or W) is dropped: repeating
 *     a read or a write of a word with no other access in between changes
 *     nothing (the invariant guarantees there was none);
 *   - that starts where an open run of its kind ends and overlaps no other
 *     open run extends it (RW only with word-aligned pieces, so no word sees
 *     RW twice);
 *   - otherwise first closes every open run it overlaps (emitting them in
 *     their order), then opens a new run (closing the oldest if all are used).
 * Every word therefore sees its accesses in program order, so the emitted
 * ranges (xpl_record_host_ranges) mean exactly what the individual accesses
 * mean -- for programs whose individual accesses never straddle two
 * allocations (every valid C/C++ object access; D28).
 *
 * Site hints.  An instrumenting tool knows the static access site; giving each
 * site a local `xpl_host_site` (the run slot that site hit last) lets the fast
 * path go straight to that run instead of through the shared "current run"
 * prediction, so interleaved streams (a[i], b[i], c[i] in one loop body) do
 * not form a dependency chain through the tracer's state:
 *
 *     xpl_host_site sa, sb;
 *     for (i...) tr.write(a[i], sa) = tr.read(b[i], sb);
 *
 * A hint is only a starting point: whatever run it names is checked like any
 * other, so a stale hint costs a slow-path call, never a wrong record.
 */
#ifndef XPL_HOST_H
#define XPL_HOST_H

#include <stddef.h>
#include <stdint.h>

#include "xpl.h"

#ifdef __cplusplus

/* Per-access-site hint (a local of the instrumented code; see above). */
struct xpl_host_site {
  uint32_t slot = 0;
};

class xpl_host_tracer {
 public:
  explicit xpl_host_tracer(xpl_ctx* ctx) : ctx_(ctx) {}
  ~xpl_host_tracer() { flush(); }
  xpl_host_tracer(const xpl_host_tracer&) = delete;
  xpl_host_tracer& operator=(const xpl_host_tracer&) = delete;

  /* One access of `size` bytes at p, kind = XPL_ACC_R / _W / _RW. */
  __attribute__((always_inline)) inline void access(const void* p, uint32_t size, uint32_t kind) {
    const uint64_t a = (uint64_t)p;
    Run* r = cur_;
    if (hit(r, a, size, kind)) return;  // the run used last
    Run* n = r->next;                    // the run that followed it last time
    if (n && hit(n, a, size, kind)) {
      cur_ = n;
      return;
    }
    slow(a, size, kind);
  }
  /* The same access with a site hint: try the run the site used last. */
  __attribute__((always_inline)) inline void access(const void* p, uint32_t size, uint32_t kind,
                                                    xpl_host_site& s) {
    const uint64_t a = (uint64_t)p;
    if (hit(&run_[s.slot], a, size, kind)) return;
    s.slot = slow(a, size, kind);
  }
  template <class T>
  inline const T& read(const T& x, xpl_host_site& s) {
    access(&x, sizeof(T), XPL_ACC_R, s);
    return x;
  }
  template <class T>
  inline T& write(T& x, xpl_host_site& s) {
    access(&x, sizeof(T), XPL_ACC_W, s);
    return x;
  }
  template <class T>
  inline T& rw(T& x, xpl_host_site& s) {
    access(&x, sizeof(T), XPL_ACC_RW, s);
    return x;
  }
  template <class T>
  inline const T& read(const T& x) {
    access(&x, sizeof(T), XPL_ACC_R);
    return x;
  }
  template <class T>
  inline T& write(T& x) {
    access(&x, sizeof(T), XPL_ACC_W);
    return x;
  }
  template <class T>
  inline T& rw(T& x) {
    access(&x, sizeof(T), XPL_ACC_RW);
    return x;
  }
  /* Hand everything traced so far to the runtime (program order kept). */
  xpl_status flush() {
    for (;;) {  // close the open runs, oldest first
      int o = -1;
      for (int i = 0; i < kRuns; ++i)
        if (run_[i].kind && (o < 0 || run_[i].seq < run_[o].seq)) o = i;
      if (o < 0) break;
      close(o);
    }
    drain();
    return status_;
  }
  xpl_status status() const { return status_; }

 private:
  static const int kRuns = 8;
  static const uint64_t kMaxRun = 0xFFFFFFF0ull;
  static const size_t kBuf = 4096;
  struct Run {
    uint64_t beg = 0, end = 0;  // bytes [beg, end)
    uint64_t end0 = 0;          // end when opened
    uint64_t limit = 0;         // word-aligned start of the next open run above (or max)
    uint64_t cap = 0;           // min(limit, beg + kMaxRun): the run may grow up to here
    uint64_t seq = 0;           // opening order
    uint16_t kind = 0;          // 0 = slot free (16 bits: no aliasing with int/uint32 data)
    uint16_t grew = 0;          // repeated since opened (extension: end != end0)
    Run* next = nullptr;        // the run used after this one last time (a prediction)
  };
  /* The access joins run r (extension at its end, or a repeat inside it). */
  static inline bool hit(Run* r, uint64_t a, uint32_t size, uint32_t kind) {
    if (kind != r->kind) return false;
    if (a == r->end) {
      if (a + size > r->cap) return false;
      if (kind == XPL_ACC_RW && ((a | size) & 3u)) return false;
      r->end = a + size;  // (growth is seen at close: end != end0)
      return true;
    }
    if (kind != XPL_ACC_RW && a >= r->beg && a + size <= r->end) {  // repeat (R or W)
      r->grew = 1;
      return true;
    }
    return false;
  }
  static uint64_t wlo(uint64_t a) { return a & ~3ull; }
  static uint64_t whi(uint64_t e) { return (e + 3) & ~3ull; }

  void drain() {
    if (n_) {
      const xpl_status s = xpl_record_host_strided(ctx_, buf_, n_);
      if (s != XPL_OK && status_ == XPL_OK) status_ = s;
    }
    n_ = 0;
  }
  static void set_limit(Run& r, uint64_t lim) {
    r.limit = lim;
    r.cap = lim < r.beg + kMaxRun ? lim : r.beg + kMaxRun;
  }
  void close(int i) {
    if (n_ == kBuf) drain();
    buf_[n_++] = xpl_host_strided{run_[i].beg, (uint32_t)(run_[i].end - run_[i].beg), run_[i].kind, 0, 1};
    run_[i].kind = 0;
    const uint64_t b = wlo(run_[i].beg);
    for (int j = 0; j < kRuns; ++j) {
      if (run_[j].next == &run_[i]) run_[j].next = nullptr;  // forget predictions into the slot
      if (run_[j].kind && run_[j].limit == b) set_limit(run_[j], limit_of(j));  // it was the run above
    }
    run_[i].next = nullptr;
  }
  // word start of the closest open run above run i (the furthest i may grow)
  uint64_t limit_of(int i) const {
    uint64_t lim = ~0ull;
    for (int j = 0; j < kRuns; ++j)
      if (j != i && run_[j].kind && wlo(run_[j].beg) >= whi(run_[i].end) && wlo(run_[j].beg) < lim)
        lim = wlo(run_[j].beg);
    return lim;
  }
  bool overlaps(int i, uint64_t lo, uint64_t hi) const {  // word ranges intersect
    return run_[i].kind && wlo(run_[i].beg) < hi && lo < whi(run_[i].end);
  }
  void touch(int k) {  // move mru_[k] to the front; learn the successor of the current run
    const uint8_t i = mru_[k];
    for (; k > 0; --k) mru_[k] = mru_[k - 1];
    mru_[0] = i;
    if (cur_ != &run_[i]) cur_->next = &run_[i];
    cur_ = &run_[i];
  }
  /* Returns the slot that now holds the access (kRuns: emitted directly). */
  __attribute__((noinline)) uint32_t slow(uint64_t a, uint32_t size, uint32_t kind) {
    const uint64_t lo = wlo(a), hi = whi(a + size);
    for (int k = 0; k < kRuns; ++k) {  // most recently used first: a run a starts in or right after
      const uint32_t i = mru_[k];
      Run& r = run_[i];
      if (r.kind != kind || a < r.beg || a > r.end) continue;
      if (kind != XPL_ACC_RW) {  // R / W: idempotent per word -> union
        if (a + size <= r.end) {  // repeat inside the run (its words are no other run's)
          r.grew = 1;
          churn_ = 0;
          touch(k);
          return i;
        }
        if (a + size <= r.cap) {
          r.end = a + size;
          churn_ = 0;
          touch(k);
          return i;
        }
      } else if (a == r.end && ((a | size) & 3u) == 0 && a + size <= r.cap) {
        r.end = a + size;
        churn_ = 0;
        touch(k);
        return i;
      }
      break;
    }
    // close the runs this access overlaps (oldest first), then open a new one
    for (;;) {
      int o = -1;
      for (int i = 0; i < kRuns; ++i)
        if (overlaps(i, lo, hi) && (o < 0 || run_[i].seq < run_[o].seq)) o = i;
      if (o < 0) break;
      close(o);
    }
    // Scattered accesses (no run ever grows): emit them directly, re-trying
    // runs every 64th access -- same records, without the slot churn.  An
    // emitted access that continues the arithmetic progression of the record
    // emitted last (same kind and size, nothing emitted in between) joins it.
    if (churn_ >= 32 && (++tick_ & 63) != 0) {
      if (n_) {
        xpl_host_strided& l = buf_[n_ - 1];
        if (l.kind == kind && l.size == size) {
          if (l.count == 1) {
            l.stride = (int64_t)(a - l.addr);
            l.count = 2;
            return kRuns;
          }
          if (a == l.addr + (uint64_t)l.stride * l.count) {
            ++l.count;
            return kRuns;
          }
        }
      }
      if (n_ == kBuf) drain();
      buf_[n_++] = xpl_host_strided{a, size, kind, 0, 1};
      return kRuns;
    }
    int slot = -1;
    for (int i = 0; i < kRuns && slot < 0; ++i)
      if (!run_[i].kind) slot = i;
    if (slot < 0) {  // all used: close the oldest
      slot = 0;
      for (int i = 1; i < kRuns; ++i)
        if (run_[i].seq < run_[slot].seq) slot = i;
      churn_ = (run_[slot].grew || run_[slot].end != run_[slot].end0) ? 0 : churn_ + 1;
      close(slot);
    }
    Run& r = run_[slot];
    r.beg = a;
    r.end = r.end0 = a + size;
    r.kind = (uint16_t)kind;
    r.grew = 0;
    r.seq = ++seq_;
    set_limit(r, limit_of(slot));
    for (int j = 0; j < kRuns; ++j)  // runs below the new one may now grow only up to it
      if (j != slot && run_[j].kind && whi(run_[j].end) <= lo && run_[j].limit > lo) set_limit(run_[j], lo);
    for (int k = 0; k < kRuns; ++k)
      if (mru_[k] == slot) {
        touch(k);
        break;
      }
    return (uint32_t)slot;
  }

  xpl_ctx* ctx_;
  Run run_[kRuns + 1];  // run_[kRuns]: never open (the hint of a directly emitted access)
  uint8_t mru_[kRuns] = {0, 1, 2, 3, 4, 5, 6, 7};  // run slots, most recently used first
  Run* cur_ = &run_[0];                              // == &run_[mru_[0]]
  uint64_t seq_ = 0;
  uint32_t churn_ = 0;  // consecutive evictions of runs that never grew
  uint32_t tick_ = 0;
  size_t n_ = 0;
  xpl_status status_ = XPL_OK;
  xpl_host_strided buf_[kBuf];
};

#endif /* __cplusplus */
#endif /* XPL_HOST_H */
