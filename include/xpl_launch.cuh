/* include/xpl_launch.cuh -- the kernel-launch wrapper (traceKernelLaunch,
 * P:L227).  The paper's `#pragma xpl replace
 * kernel-launch` turns every `kernel<<<grd, blk, shmem, stream>>>(args...)`
 * into `traceKernelLaunch(grd, blk, shmem, stream, kernel, args...)`; this is
 * that function for the xpl runtime:
 *
 *     xpl_trace_kernel_launch(ctx, "hotspot", grd, blk, 0, stream, hotspot_kernel<true>, a, b, n);
 *
 * opens a GPU epoch on `stream` (xpl_kernel_begin), logs the launch parameters
 * (xpl_kernel_launch; kept when the launch log is on), launches the kernel, and
 * closes the epoch (xpl_kernel_end: the fold, plus the epoch's GPU time and
 * written-chunk count when the log is on).  Inside an already open epoch the
 * begin/end only nest (D19), so several wrapped launches can share one epoch.
 * Returns the launch's cudaError_t, or cudaErrorUnknown if the runtime refused
 * a call (its xpl_status is then in *st when st is given).
 */
#ifndef XPL_LAUNCH_CUH
#define XPL_LAUNCH_CUH

#include <cuda_runtime.h>

#include <utility>

#include "xpl.h"

template <class... KArgs, class... Args>
inline cudaError_t xpl_trace_kernel_launch_st(xpl_ctx* ctx, xpl_status* st, const char* name, dim3 grd,
                                              dim3 blk, size_t shmem, cudaStream_t stream,
                                              void (*kernel)(KArgs...), Args&&... args) {
  xpl_status s = xpl_kernel_begin(ctx, (void*)stream);
  if (st) *st = s;
  if (s != XPL_OK) return cudaErrorUnknown;
  const xpl_launch_info li = {name, {grd.x, grd.y, grd.z}, {blk.x, blk.y, blk.z}, (uint32_t)shmem};
  const xpl_status sl = xpl_kernel_launch(ctx, (void*)stream, &li);
  kernel<<<grd, blk, shmem, stream>>>(std::forward<Args>(args)...);
  const cudaError_t e = cudaGetLastError();
  s = xpl_kernel_end(ctx, (void*)stream);  // always closes what begin opened
  if (s == XPL_OK) s = sl;
  if (st) *st = s;
  return e != cudaSuccess ? e : (s == XPL_OK ? cudaSuccess : cudaErrorUnknown);
}

template <class... KArgs, class... Args>
inline cudaError_t xpl_trace_kernel_launch(xpl_ctx* ctx, const char* name, dim3 grd, dim3 blk,
                                           size_t shmem, cudaStream_t stream, void (*kernel)(KArgs...),
                                           Args&&... args) {
  return xpl_trace_kernel_launch_st(ctx, nullptr, name, grd, blk, shmem, stream, kernel,
                                    std::forward<Args>(args)...);
}

#endif /* XPL_LAUNCH_CUH */
