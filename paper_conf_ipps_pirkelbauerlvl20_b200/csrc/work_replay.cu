// work_replay.cu -- an instrumented "user" kernel that replays a list of device
// accesses through the public __device__ hooks (include/xpl_device.cuh).  It is
// user code of libxpl, not part of it: it only sees xpl.h and xpl_device.cuh.
// Used by the parity tests (any trace, any launch shape, any permutation) and
// as the generic device-event source of the benchmarks.
#include <cuda_runtime.h>
#include <stdint.h>

#include "xpl.h"
#include "xpl_device.cuh"
#include "xpl_launch.cuh"

namespace {

__global__ void replay_kernel(const unsigned long long* __restrict__ addr,
                              const unsigned int* __restrict__ size,
                              const unsigned char* __restrict__ acc, unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    xpl_dev_record((const void*)addr[i], size[i], acc[i]);
}

// The replay with a compile-time access kind (every event of the launch has
// kind K): the K-uniform form of the hooks that xpl_read / xpl_write / xpl_rw
// call sites use (fast paths of xpl_device.cuh).
template <unsigned K>
__global__ void replay_k_kernel(const unsigned long long* __restrict__ addr,
                                const unsigned int* __restrict__ size, unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    xpl_dev_record_k<K>((const void*)addr[i], size[i], K);
}

// The same replay as ONE cooperative launch over several epochs: segment k is
// events [seg[k], seg[k+1]); a device-side epoch split (xpl_grid_epoch,
// NEXT-2) separates consecutive segments.  Equal to one launch per segment.
__global__ void replay_split_kernel(const unsigned long long* __restrict__ addr,
                                    const unsigned int* __restrict__ size,
                                    const unsigned char* __restrict__ acc,
                                    const unsigned long long* __restrict__ seg, int nseg) {
  for (int k = 0; k < nseg; ++k) {
    if (k) xpl_grid_epoch();
    for (unsigned long long i = seg[k] + (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
         i < seg[k + 1]; i += (unsigned long long)gridDim.x * blockDim.x)
      xpl_dev_record((const void*)addr[i], size[i], acc[i]);
  }
}

__device__ __forceinline__ unsigned hash32(unsigned x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

// A synthetic instrumented kernel over n words at address `base` (no memory
// behind it: hooks only use addresses).  Per 4096-word block one of: untouched,
// all read, all written, or a per-word random R/W/RW mix -- long runs and
// mixed regions, like a real shadow.
__global__ void touch_kernel(unsigned long long base, unsigned long long n, unsigned seed,
                             unsigned long long i0) {
  for (unsigned long long j = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; j < n;
       j += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned long long i = i0 + j;  // the pattern is a function of the logical word
    const unsigned hb = hash32((unsigned)(i >> 12) ^ seed);
    unsigned acc = 0;
    switch (hb & 3) {
      case 1: acc = XPL_ACC_R; break;
      case 2: acc = XPL_ACC_W; break;
      case 3: {
        const unsigned h = hash32((unsigned)i ^ (seed * 0x9E3779B9u));
        acc = (h & 3);  // 0 = no access
        break;
      }
      default: break;
    }
    if (acc) xpl_dev_record((const void*)(base + 4 * j), 4, acc);
  }
}

// Atomic-throughput microbenchmark (the recording roofline):
// one 32-bit OR per u32 of p[0, n), grid-stride, coalesced.  mode 0: RED
// (no return value -- what a hook's commit issues); mode 1: ATOM (return value
// consumed); mode 2: every lane of a warp on the same u32 (the same-word case
// without warp aggregation).
__global__ void atomic_bench_kernel(unsigned* p, unsigned long long n, int mode, unsigned* sink) {
  unsigned acc = 0;
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned v = 1u << (i & 31);
    if (mode == 0) atomicOr(p + i, v);
    else if (mode == 1) acc ^= atomicOr(p + i, v);
    else atomicOr(p + (i >> 5), v);
  }
  if (mode == 1 && acc == 0x9E3779B9u) *sink = acc;  // keep the return values live
}

// Streaming user kernel with real data (the recording roofline and the
// slowdown floor of a bandwidth-bound kernel): y[i] = x[i] + x[i]
// over n elements of T, every read through traceR and every write through
// traceW (I = instrumented), or the uninstrumented twin (I = false).
template <class T, bool I>
__global__ void __launch_bounds__(256) stream_kernel(const T* __restrict__ x, T* __restrict__ y,
                                                     unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    if constexpr (I) {
      const T v = xpl_read(x[i]);
      xpl_write(y[i]) = v + v;
    } else {
      const T v = x[i];
      y[i] = v + v;
    }
  }
}

// The same streaming kernel through array handles (the lookups of x and y
// hoisted out of the loop, as an instrumenting compiler would for a
// loop-invariant base): same records.
template <class T>
__global__ void __launch_bounds__(256) stream_kernel_h(const T* __restrict__ x, T* __restrict__ y,
                                                       unsigned long long n) {
  const xpl_array<const T> hx(x);
  const xpl_array<T> hy(y);
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const T v = hx.read(i);
    hy.write(i) = v + v;
  }
}

struct T12 {  // a 12-byte element (3 words: handles of non-power-of-two sizes)
  unsigned a, b, c;
};

// Accesses through one array handle made from `base` (addresses only): event i
// is element idx[i] of the handle (any index, negative too: elements outside
// the handle's row take the full lookup), with kind K.  The handle's parity test.
template <class T, unsigned K>
__global__ void handle_replay_kernel(unsigned long long base, const long long* __restrict__ idx,
                                     unsigned long long n) {
  const xpl_array<T> h(reinterpret_cast<T*>(base));
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    h.template rec<K>((unsigned long long)idx[i]);
}

// A user kernel that really touches memory (managed memory for the UM-counter
// check, NEXT-4): word k*stride of base for k < n/stride is read (write = 0) or
// incremented (write = 1: read then write, hooked as RW), hooks on.
__global__ void touch_mem_kernel(unsigned* base, unsigned long long n, unsigned long long stride, int write,
                                 unsigned* sink) {
  unsigned acc = 0;
  for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k * stride < n;
       k += (unsigned long long)gridDim.x * blockDim.x) {
    unsigned& w = base[k * stride];
    if (write) xpl_rw(w) += 1u;
    else acc ^= xpl_read(w);
  }
  if (acc == 0x9E3779B9u) *sink = acc;
}

// Reads through the deferred-commit hook (xpl_read_lat): element i reads a T at
// addr[i] (addresses only: the proxy is never converted, so no user load).
template <class T>
__global__ void read_lat_kernel(const unsigned long long* __restrict__ addr, unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    auto pr = xpl_read_lat(*reinterpret_cast<const T*>(addr[i]));
    (void)pr;
  }
}

}  // namespace

extern "C" {

// Launch read_lat_kernel<T> with sizeof(T) = size (1, 2, 4, 8 or 16) on `stream`
// (between xpl_kernel_begin/_end); grid-stride, so odd grids are allowed.
int xplw_read_lat(const unsigned long long* d_addr, unsigned long long n, int size, int grid, int block,
                  void* stream) {
  if (n == 0) return 0;
  cudaStream_t s = (cudaStream_t)stream;
  switch (size) {
    case 1: read_lat_kernel<unsigned char><<<grid, block, 0, s>>>(d_addr, n); break;
    case 2: read_lat_kernel<unsigned short><<<grid, block, 0, s>>>(d_addr, n); break;
    case 4: read_lat_kernel<unsigned int><<<grid, block, 0, s>>>(d_addr, n); break;
    case 8: read_lat_kernel<unsigned long long><<<grid, block, 0, s>>>(d_addr, n); break;
    case 16: read_lat_kernel<uint4><<<grid, block, 0, s>>>(d_addr, n); break;
    default: return (int)XPL_ERR_INVALID_ARG;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// Launch touch_mem_kernel on `stream` (between xpl_kernel_begin/_end).
int xplw_touch_mem(void* base, unsigned long long n_words, unsigned long long stride, int write, void* stream) {
  if (!stride || !n_words) return 0;
  const unsigned long long m = (n_words + stride - 1) / stride;
  const unsigned g = (unsigned)(m < 148ull * 8 * 256 ? (m + 255) / 256 : 148 * 8);
  touch_mem_kernel<<<g, 256, 0, (cudaStream_t)stream>>>((unsigned*)base, n_words, stride, write,
                                                        (unsigned*)base);
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// Launch the streaming kernel: elem = 4 or 8 bytes, instrumented (1: traceR /
// traceW per element, 2: through array handles; between xpl_kernel_begin/_end)
// or the twin (0); one wave of 148 x 8 CTAs, grid-stride.
int xplw_stream(const void* x, void* y, unsigned long long n, int elem, int instrumented, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  const unsigned g = 148 * 8;
  if (instrumented == 2) {  // through array handles
    if (elem == 4) stream_kernel_h<unsigned><<<g, 256, 0, s>>>((const unsigned*)x, (unsigned*)y, n);
    else if (elem == 8)
      stream_kernel_h<unsigned long long><<<g, 256, 0, s>>>((const unsigned long long*)x, (unsigned long long*)y, n);
    else return (int)XPL_ERR_INVALID_ARG;
  } else if (elem == 4) {
    if (instrumented) stream_kernel<unsigned, true><<<g, 256, 0, s>>>((const unsigned*)x, (unsigned*)y, n);
    else stream_kernel<unsigned, false><<<g, 256, 0, s>>>((const unsigned*)x, (unsigned*)y, n);
  } else if (elem == 8) {
    if (instrumented) stream_kernel<unsigned long long, true><<<g, 256, 0, s>>>(
        (const unsigned long long*)x, (unsigned long long*)y, n);
    else stream_kernel<unsigned long long, false><<<g, 256, 0, s>>>(
        (const unsigned long long*)x, (unsigned long long*)y, n);
  } else {
    return (int)XPL_ERR_INVALID_ARG;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// Launch the handle replay: elem = 4, 8 or 12 bytes, kind = 1 R, 2 W, 3 RW.
int xplw_handle_replay(unsigned long long base, int elem, const long long* d_idx, unsigned long long n,
                       int kind, int grid, int block, void* stream) {
  if (n == 0) return 0;
  cudaStream_t s = (cudaStream_t)stream;
#define XPLW_HR(T)                                                                                     \
  switch (kind) {                                                                                     \
    case 1: handle_replay_kernel<T, XPL_ACC_R><<<grid, block, 0, s>>>(base, d_idx, n); break;        \
    case 2: handle_replay_kernel<T, XPL_ACC_W><<<grid, block, 0, s>>>(base, d_idx, n); break;        \
    case 3: handle_replay_kernel<T, XPL_ACC_RW><<<grid, block, 0, s>>>(base, d_idx, n); break;       \
    default: return (int)XPL_ERR_INVALID_ARG;                                                         \
  }
  if (elem == 4) { XPLW_HR(unsigned) }
  else if (elem == 8) { XPLW_HR(unsigned long long) }
  else if (elem == 12) { XPLW_HR(T12) }
  else return (int)XPL_ERR_INVALID_ARG;
#undef XPLW_HR
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

int xplw_atomic_bench(void* buf, unsigned long long n_u32, int mode, void* stream) {
  atomic_bench_kernel<<<148 * 16, 256, 0, (cudaStream_t)stream>>>((unsigned*)buf, n_u32, mode,
                                                                  (unsigned*)buf);
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}


// Launch the synthetic touch kernel (between xpl_kernel_begin/_end) over the n
// words at base, which are logical words i0 .. i0+n-1 of the pattern.
int xplw_touch(unsigned long long base, unsigned long long n, unsigned seed, void* stream,
               unsigned long long i0) {
  touch_kernel<<<148 * 16, 256, 0, (cudaStream_t)stream>>>(base, n, seed, i0);
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}


int xplw_bind_rodinia(xpl_ctx* ctx);
int xplw_bind_sw(xpl_ctx* ctx);
int xplw_bind_lulesh(xpl_ctx* ctx);

// Bind the hooks of every instrumented translation unit of this library to ctx
// (xpl_device_bind copies the device context into each TU's __constant__).
int xplw_bind(xpl_ctx* ctx) {
  int s = (int)xpl_device_bind(ctx);
  if (!s) s = xplw_bind_rodinia(ctx);
  if (!s) s = xplw_bind_sw(ctx);
  if (!s) s = xplw_bind_lulesh(ctx);
  return s;
}

// Launch the replay kernel on `stream` (between xpl_kernel_begin/_end).
int xplw_replay(const unsigned long long* d_addr, const unsigned int* d_size,
                const unsigned char* d_acc, unsigned long long n, int grid, int block,
                void* stream) {
  if (n == 0) return 0;
  replay_kernel<<<grid, block, 0, (cudaStream_t)stream>>>(d_addr, d_size, d_acc, n);
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// Launch the K-uniform replay kernel (kind = 1 R, 2 W, 3 RW) on `stream`.
int xplw_replay_k(const unsigned long long* d_addr, const unsigned int* d_size, unsigned long long n,
                  int kind, int grid, int block, void* stream) {
  if (n == 0) return 0;
  cudaStream_t s = (cudaStream_t)stream;
  switch (kind) {
    case XPL_ACC_R: replay_k_kernel<XPL_ACC_R><<<grid, block, 0, s>>>(d_addr, d_size, n); break;
    case XPL_ACC_W: replay_k_kernel<XPL_ACC_W><<<grid, block, 0, s>>>(d_addr, d_size, n); break;
    case XPL_ACC_RW: replay_k_kernel<XPL_ACC_RW><<<grid, block, 0, s>>>(d_addr, d_size, n); break;
    default: return (int)XPL_ERR_INVALID_ARG;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// The same launch through the kernel-launch wrapper (traceKernelLaunch, P:L227;
// NEXT-4): opens (or nests into) an epoch on `stream`, logs the launch, closes it.
int xplw_replay_traced(xpl_ctx* ctx, const unsigned long long* d_addr, const unsigned int* d_size,
                       const unsigned char* d_acc, unsigned long long n, int grid, int block,
                       void* stream) {
  xpl_status st = XPL_OK;
  const cudaError_t e = xpl_trace_kernel_launch_st(ctx, &st, "replay_kernel", dim3(grid), dim3(block), 0,
                                                   (cudaStream_t)stream, replay_kernel, d_addr, d_size,
                                                   d_acc, n);
  if (st != XPL_OK) return (int)st;
  return e == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}

// One cooperative launch replaying nseg epochs (between one xpl_kernel_begin/_end);
// d_seg: nseg+1 event offsets (device).  grid is capped at the co-resident limit.
int xplw_replay_split(const unsigned long long* d_addr, const unsigned int* d_size,
                      const unsigned char* d_acc, const unsigned long long* d_seg, int nseg,
                      int grid, int block, void* stream) {
  if (nseg <= 0) return 0;
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, replay_split_kernel, block, 0);
  const int cap = sms * per_sm;
  if (grid <= 0 || grid > cap) grid = cap;
  void* args[] = {&d_addr, &d_size, &d_acc, &d_seg, &nseg};
  const cudaError_t e = cudaLaunchCooperativeKernel((const void*)replay_split_kernel, dim3(grid), dim3(block),
                                                    args, 0, (cudaStream_t)stream);
  return e == cudaSuccess ? 0 : (int)XPL_ERR_CUDA;
}
}
