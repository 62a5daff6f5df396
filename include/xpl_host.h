/* include/xpl_host.h -- header-only host tracer: the !__CUDA_ARCH__ branch of
 * traceR / traceW / traceRW (Table I) as an inline C++
 * object the instrumented host code calls per access.
 *
 *     xpl_host_tracer tr(ctx);
 *     for (i...) tr.write(&a[i]);            // = traceW(a[i]) = ...
 *     x = tr.read(b[i]);                     // = traceR(b[i])
 *     tr.flush();                            // before kernel launches / diagnose
 *
 * The tracer coalesces consecutive accesses of one kind to adjacent bytes into
 * one byte range in the caller's thread (R and W are idempotent per word;
 * RW only when every piece is word aligned, so no word sees RW twice) and
 * hands ranges to xpl_record_host_ranges.  For programs whose individual
 * accesses never straddle two allocations (every valid C/C++ object access)
 * this is exactly the per-access semantics of xpl_record_host.
 */
#ifndef XPL_HOST_H
#define XPL_HOST_H

#include <stddef.h>
#include <stdint.h>

#include "xpl.h"

#ifdef __cplusplus

class xpl_host_tracer {
 public:
  explicit xpl_host_tracer(xpl_ctx* ctx) : ctx_(ctx) {}
  ~xpl_host_tracer() { flush(); }
  xpl_host_tracer(const xpl_host_tracer&) = delete;
  xpl_host_tracer& operator=(const xpl_host_tracer&) = delete;

  /* One access of `size` bytes at p, kind = XPL_ACC_R / _W / _RW. */
  inline void access(const void* p, uint32_t size, uint32_t kind) {
    const uint64_t a = (uint64_t)p;
    if (kind == kind_ && a == end_ && size <= kMaxRun - (end_ - beg_) &&
        (kind != XPL_ACC_RW || ((a | size) & 3u) == 0)) {
      end_ = a + size;
      return;
    }
    if (kind == kind_ && kind != XPL_ACC_RW && a >= beg_ && a + size <= end_) return;  // repeat
    slow(a, size, kind);
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
    close_run();
    xpl_status s = XPL_OK;
    if (n_) s = xpl_record_host_ranges(ctx_, buf_, n_);
    n_ = 0;
    if (s != XPL_OK && status_ == XPL_OK) status_ = s;
    return status_;
  }
  xpl_status status() const { return status_; }

 private:
  static const uint64_t kMaxRun = 0xFFFFFFF0ull;
  static const size_t kBuf = 4096;
  void close_run() {
    if (kind_) buf_[n_++] = xpl_host_access{beg_, (uint32_t)(end_ - beg_), kind_};
    kind_ = 0;
    beg_ = end_ = 0;
  }
  void slow(uint64_t a, uint32_t size, uint32_t kind) {
    close_run();
    if (n_ == kBuf) flush();
    beg_ = a;
    end_ = a + size;
    kind_ = kind;
  }
  xpl_ctx* ctx_;
  uint64_t beg_ = 0, end_ = 0;
  uint32_t kind_ = 0;
  size_t n_ = 0;
  xpl_status status_ = XPL_OK;
  xpl_host_access buf_[kBuf];
};

#endif /* __cplusplus */
#endif /* XPL_HOST_H */
