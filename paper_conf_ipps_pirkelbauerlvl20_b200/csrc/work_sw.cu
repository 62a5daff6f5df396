// work_sw.cu -- Smith-Waterman instrumented program (the paper's SW study,
// Fig. 7/8 P:L341-349; configs cfg1 SW-128 and cfg3 SW-16K).
// User code of libxpl: only xpl.h / xpl_device.cuh / xpl_host.h.  The CPU twin
// (event trace for the oracle) is xplgen/sw.py.
#include <cuda_runtime.h>
#include <stdint.h>

#include <chrono>

#include "xpl.h"
#include "xpl_device.cuh"
#include "xpl_host.h"
#include "xplw.h"

namespace {

constexpr int kMatch = 3, kMismatch = -3, kGap = 2;

template <bool I, class T>
__device__ __forceinline__ const T& RD(const T& x) {
  if constexpr (I) return xpl_read(x);
  else return x;
}
template <bool I, class T>
__device__ __forceinline__ T& WR(T& x) {
  if constexpr (I) return xpl_write(x);
  else return x;
}

// H through an array handle (its row lookup hoisted out of the cell's four
// accesses, as an instrumenting compiler would); the twin gets the pointer.
template <bool I>
struct HArr : xpl_array<int> {
  __device__ __forceinline__ explicit HArr(int* q) : xpl_array<int>(q) {}
};
template <>
struct HArr<false> {
  int* p;
  __device__ __forceinline__ explicit HArr(int* q) : p(q) {}
  __device__ __forceinline__ const int& read(long long i) const { return p[i]; }
  __device__ __forceinline__ int& write(long long i) const { return p[i]; }
};

template <bool I>
__device__ __forceinline__ void sw_cell(const int* a, const int* b, const HArr<I>& H, int ld, int i, int j) {
  const int s = RD<I>(a[i - 1]) == RD<I>(b[j - 1]) ? kMatch : kMismatch;
  const int d = H.read((long long)(i - 1) * ld + j - 1) + s;
  const int u = H.read((long long)(i - 1) * ld + j) - kGap;
  const int l = H.read((long long)i * ld + j - 1) - kGap;
  int h = d > u ? d : u;
  h = h > l ? h : l;
  H.write((long long)i * ld + j) = h > 0 ? h : 0;
}

// cfg1: one CTA, thread t owns row i = t + 1, sweeping the anti-diagonals.
template <bool I>
__global__ void sw_wavefront(const int* a, const int* b, int* H, int n, int m) {
  const int ld = m + 1, i = threadIdx.x + 1;
  const HArr<I> Hh(H);
  for (int d = 2; d <= n + m; ++d) {
    const int j = d - i;
    if (i <= n && j >= 1 && j <= m) sw_cell<I>(a, b, Hh, ld, i, j);
    __syncthreads();
  }
}

// cfg1 with device-side epoch splits (NEXT-2): the same single launch, but each
// anti-diagonal is its own epoch (xpl_grid_epoch; launched cooperatively), so
// the wavefront's reads of the previous diagonal see the GPU as the last writer
// -- the paper's per-iteration view (Fig. 8).
template <bool I>
__global__ void sw_wavefront_split(const int* a, const int* b, int* H, int n, int m) {
  const int ld = m + 1, i = threadIdx.x + 1;
  const HArr<I> Hh(H);
  for (int d = 2; d <= n + m; ++d) {
    const int j = d - i;
    if (i <= n && j >= 1 && j <= m) sw_cell<I>(a, b, Hh, ld, i, j);
    if constexpr (I) {
      if (d < n + m) xpl_grid_epoch();  // (the last diagonal's epoch closes at xpl_kernel_end)
    } else {
      __syncthreads();
    }
  }
}

// cfg3: one launch per anti-diagonal d, thread per cell.
template <bool I>
__global__ void __launch_bounds__(256) sw_diagonal(const int* a, const int* b, int* H, int n, int m,
                                                   int d) {
  const int i = max(1, d - m) + blockIdx.x * blockDim.x + threadIdx.x;
  const int j = d - i;
  if (i > n || j < 1) return;
  const HArr<I> Hh(H);
  sw_cell<I>(a, b, Hh, m + 1, i, j);
}

template <bool I>
__global__ void sw_rezero(int* H, int n, int m) {
  const int ld = m + 1;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < (int64_t)n * m;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int i = 1 + (int)(k / m), j = 1 + (int)(k % m);
    WR<I>(H[i * ld + j]) = 0;
  }
}

}  // namespace

extern "C" {

int xplw_bind_sw(xpl_ctx* ctx) { return (int)xpl_device_bind(ctx); }

int xplw_sw(xplw_run* run, const xplw_arrays* arr, int n, int m, int per_diagonal, int tb_every,
            int diag_every, int* tb_len) {
  const bool on = run->ctx != nullptr;
  cudaStream_t s = (cudaStream_t)run->stream;
  int *a = (int*)arr->addr[0], *b = (int*)arr->addr[1], *H = (int*)arr->addr[2];
  const int ld = m + 1;
  const int64_t hn = (int64_t)(n + 1) * (m + 1);
  xpl_host_tracer* tr = on ? new xpl_host_tracer(run->ctx) : nullptr;
  auto ok = [&](int st) {
    if (st && !run->status) run->status = st;
  };
  auto okc = [&](cudaError_t e) {
    if (e != cudaSuccess && !run->status) run->status = XPL_ERR_CUDA;
  };
  auto flush = [&]() {
    if (tr) ok(tr->flush());
  };
  auto diag = [&]() {
    flush();
    if (!on) return;
    size_t nr = 0;
    xpl_alloc_report* o = run->out ? run->out + run->n_out : nullptr;
    const size_t cap = run->out ? run->out_cap - run->n_out : 0;
    const int st = xpl_diagnose(run->ctx, &run->params, nullptr, 0, o, cap, &nr, 1);
    if (st == XPL_OK) {
      run->n_out += nr;
      if (run->diag_rows && run->n_diag < run->diag_cap) run->diag_rows[run->n_diag] = (uint32_t)nr;
      run->n_diag++;
    } else {
      ok(st);
    }
  };
  auto begin = [&]() {
    flush();
    if (on) ok(xpl_kernel_begin(run->ctx, s));
  };
  auto end = [&]() {
    okc(cudaGetLastError());
    if (on) ok(xpl_kernel_end(run->ctx, s));
    run->epochs++;
  };
  auto host_ms = [&](std::chrono::steady_clock::time_point t0) {
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  };
  if (on)
    for (int k = 0; k < arr->n; ++k)
      ok(xpl_register_alloc(run->ctx, (const void*)arr->addr[k], arr->bytes[k], (xpl_alloc_kind)arr->kind[k]));
  // E0 (host): the sequences are stored, H is zeroed (Fig. 7a)
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) {
    const int v = a[i];
    if (tr) tr->write(a[i]) = v;
  }
  for (int j = 0; j < m; ++j) {
    const int v = b[j];
    if (tr) tr->write(b[j]) = v;
  }
  if (tr)
    for (int64_t k = 0; k < hn; ++k) tr->write(H[k]) = 0;
  else
    for (int64_t k = 0; k < hn; ++k) H[k] = 0;
  run->host_accesses += n + m + hn;
  host_ms(t0);
  // the GPU fills H
  if (per_diagonal == 2) {  // one cooperative launch, one epoch per anti-diagonal
    begin();
    if (on) {
      void* args[] = {&a, &b, &H, &n, &m};
      okc(cudaLaunchCooperativeKernel((const void*)sw_wavefront_split<true>, dim3(1), dim3(n), args, 0, s));
    } else {
      sw_wavefront_split<false><<<1, n, 0, s>>>(a, b, H, n, m);
    }
    end();
    run->dev_accesses += 6ull * n * m;
  } else if (!per_diagonal) {
    begin();
    if (on) sw_wavefront<true><<<1, n, 0, s>>>(a, b, H, n, m);
    else sw_wavefront<false><<<1, n, 0, s>>>(a, b, H, n, m);
    end();
    run->dev_accesses += 6ull * n * m;
  } else {
    for (int d = 2; d <= n + m; ++d) {
      const int i0 = d - m > 1 ? d - m : 1, i1 = d - 1 < n ? d - 1 : n;
      const int cells = i1 - i0 + 1;
      begin();
      if (on) sw_diagonal<true><<<(cells + 255) / 256, 256, 0, s>>>(a, b, H, n, m, d);
      else sw_diagonal<false><<<(cells + 255) / 256, 256, 0, s>>>(a, b, H, n, m, d);
      end();
      run->dev_accesses += 6ull * cells;
      if (tb_every > 0 && (d - 1) % tb_every == 0) {  // a host segment reads the finished diagonal
        okc(cudaStreamSynchronize(s));                 // (managed memory: wait for the kernel)
        const auto t1 = std::chrono::steady_clock::now();
        int64_t mx = 0;
        for (int i = i0; i <= i1; ++i) mx += tr ? tr->read(H[i * ld + d - i]) : H[i * ld + d - i];
        run->host_accesses += cells;
        host_ms(t1);
        (void)mx;
      }
      if (diag_every > 0 && (d - 1) % diag_every == 0) diag();
    }
  }
  okc(cudaStreamSynchronize(s));
  // the CPU: maximum scan of H, then the traceback from the (first) maximum
  t0 = std::chrono::steady_clock::now();
  int best = -1;
  int64_t at = 0;
  for (int64_t k = 0; k < hn; ++k) {
    const int v = tr ? tr->read(H[k]) : H[k];
    if (v > best) {
      best = v;
      at = k;
    }
  }
  run->host_accesses += hn;
  int i = (int)(at / ld), j = (int)(at % ld), len = 0;
  auto R = [&](const int& x) -> int {
    run->host_accesses += 1;
    return tr ? tr->read(x) : x;
  };
  while (i > 0 && j > 0) {
    const int h = R(H[i * ld + j]);
    if (h == 0) break;
    ++len;
    const int sc = R(a[i - 1]) == R(b[j - 1]) ? kMatch : kMismatch;
    if (R(H[(i - 1) * ld + j - 1]) + sc == h) {
      --i;
      --j;
    } else if (R(H[(i - 1) * ld + j]) - kGap == h) {
      --i;
    } else {
      --j;
    }
  }
  *tb_len = len;
  host_ms(t0);
  if (per_diagonal != 1) {  // E3: the GPU re-zeroes the interior for the next query
    begin();
    if (on) sw_rezero<true><<<(n * m + 255) / 256, 256, 0, s>>>(H, n, m);
    else sw_rezero<false><<<(n * m + 255) / 256, 256, 0, s>>>(H, n, m);
    end();
    run->dev_accesses += (uint64_t)n * m;
  }
  flush();
  delete tr;
  tr = nullptr;
  if (on)
    for (int k = 0; k < arr->n; ++k) ok(xpl_free(run->ctx, (const void*)arr->addr[k]));
  diag();
  okc(cudaStreamSynchronize(s));
  return run->status;
}

}  // extern "C"

extern "C" {
// Unified memory for the managed-memory programs (cudaMallocManaged).
void* xplw_alloc_managed(unsigned long long bytes) {
  void* p = nullptr;
  return cudaMallocManaged(&p, bytes) == cudaSuccess ? p : nullptr;
}
int xplw_free_managed(void* p) { return cudaFree(p) == cudaSuccess ? 0 : (int)XPL_ERR_CUDA; }
// The programs' input upload (bench e2e: pinned host -> managed/device, on a stream).
int xplw_memcpy_async(void* dst, const void* src, unsigned long long bytes, void* stream) {
  return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault, (cudaStream_t)stream) == cudaSuccess
             ? 0 : (int)XPL_ERR_CUDA;
}
}
