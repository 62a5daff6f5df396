// work_rodinia.cu -- Rodinia-shaped instrumented applications (configs[1]:
// backprop, hotspot), written as a user of the public
// API: kernels call xpl_read / xpl_write / xpl_rw (include/xpl_device.cuh),
// host loops feed xpl_record_host, cudaMemcpy calls are traced with
// xpl_record_copy (the `#pragma xpl replace` wrappers).
// Every kernel is compiled twice: I = true (instrumented) and I = false (the
// uninstrumented twin of the slowdown metric, Table III).
// The CPU twin of these programs (the event trace the oracle replays) is
// xplgen/rodinia.py; the two are written independently and must agree.
#include <cuda_runtime.h>
#include <stdint.h>

#include <chrono>
#include <vector>

#include "xpl.h"
#include "xpl_device.cuh"
#include "xpl_host.h"
#include "xplw.h"

namespace {

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
template <bool I, class T>
__device__ __forceinline__ T& RW(T& x) {
  if constexpr (I) return xpl_rw(x);
  else return x;
}

// ---------------------------------------------------------------------------
// The app-side helpers: host tracer buffer, traced copies, epochs, diagnoses.
struct App {
  xplw_run* run;
  cudaStream_t s;
  std::vector<cudaEvent_t> evs;  // pairs around kernels (time_kernels)
  explicit App(xplw_run* r) : run(r), s((cudaStream_t)r->stream) {
    if (r->ctx) tr = new xpl_host_tracer(r->ctx);
  }
  ~App() {
    delete tr;
    if (!evs.empty()) {
      cudaStreamSynchronize(s);
      for (size_t i = 0; i + 1 < evs.size(); i += 2) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, evs[i], evs[i + 1]);
        run->kernel_ms += ms;
      }
      for (cudaEvent_t e : evs) cudaEventDestroy(e);
    }
  }
  void mark() {
    if (!run->time_kernels) return;
    cudaEvent_t e;
    cudaEventCreate(&e);
    cudaEventRecord(e, s);
    evs.push_back(e);
  }
  bool on() const { return run->ctx != nullptr; }
  void ok(int st) {
    if (st && !run->status) run->status = st;
  }
  void ok_cuda(cudaError_t e) {
    if (e != cudaSuccess && !run->status) run->status = XPL_ERR_CUDA;
  }
  // host tracer: the inline coalescing tracer of xpl_host.h
  xpl_host_tracer* tr = nullptr;
  double t_host = 0;
  void flush() {
    if (tr) ok(tr->flush());
  }
  // for (i < n) p[i] = f(i)   -- a traced host write loop doing the real stores
  template <class T>
  void write_loop(T* p, uint64_t n) {
    const auto t0 = std::chrono::steady_clock::now();
    if (tr)
      for (uint64_t i = 0; i < n; ++i) tr->write(p[i]) = (T)(i & 1023) * (T)0.001;
    else
      for (uint64_t i = 0; i < n; ++i) p[i] = (T)(i & 1023) * (T)0.001;
    run->host_accesses += n;
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  // s += p[i * stride + off] for i < n  -- a traced host read loop
  template <class T>
  T read_loop(const T* p, uint64_t n, uint64_t stride = 1, uint64_t off = 0) {
    const auto t0 = std::chrono::steady_clock::now();
    T acc = 0;
    if (tr)
      for (uint64_t i = 0; i < n; ++i) acc += tr->read(p[i * stride + off]);
    else
      for (uint64_t i = 0; i < n; ++i) acc += p[i * stride + off];
    run->host_accesses += n;
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    sink += (double)acc;
    return acc;
  }
  double sink = 0;
  void copy(void* dst, const void* src, size_t bytes, xpl_copy_dir dir) {
    flush();
    if (on()) ok(xpl_record_copy(run->ctx, dst, src, bytes, dir));
    run->copy_words += (bytes + 3) / 4;
    if (run->do_copies) {
      const cudaMemcpyKind k = dir == XPL_COPY_H2D ? cudaMemcpyHostToDevice
                              : dir == XPL_COPY_D2H ? cudaMemcpyDeviceToHost
                                                    : cudaMemcpyDefault;
      ok_cuda(cudaMemcpyAsync(dst, src, bytes, k, s));
      if (dir == XPL_COPY_D2H) ok_cuda(cudaStreamSynchronize(s));  // cudaMemcpy semantics
    }
  }
  void begin() {
    flush();
    if (on()) ok(xpl_kernel_begin(run->ctx, s));
    mark();
  }
  void end() {
    ok_cuda(cudaGetLastError());
    mark();
    if (on()) ok(xpl_kernel_end(run->ctx, s));
    run->epochs++;
  }
  void reg(const xplw_arrays* a) {
    if (!on()) return;
    for (int i = 0; i < a->n; ++i)
      ok(xpl_register_alloc(run->ctx, (const void*)a->addr[i], a->bytes[i], (xpl_alloc_kind)a->kind[i]));
  }
  void unreg(const xplw_arrays* a) {
    flush();
    if (!on()) return;
    for (int i = 0; i < a->n; ++i) ok(xpl_free(run->ctx, (const void*)a->addr[i]));
  }
  void diag() {
    flush();
    if (!on()) return;
    size_t n = 0;
    xpl_alloc_report* o = run->out ? run->out + run->n_out : nullptr;
    const size_t cap = run->out ? run->out_cap - run->n_out : 0;
    const int st = xpl_diagnose(run->ctx, &run->params, nullptr, 0, o, cap, &n, 1);
    if (st == XPL_OK) {
      run->n_out += n;
      if (run->diag_rows && run->n_diag < run->diag_cap) run->diag_rows[run->n_diag] = (uint32_t)n;
      run->n_diag++;
    } else {
      ok(st);
    }
  }
};

template <class T>
T* A(const xplw_arrays* a, int i) {
  return reinterpret_cast<T*>(a->addr[i]);
}

// ---------------------------------------------------------------------------
// hotspot: 5-point thermal stencil (Rodinia hotspot shape: temperature read at
// the cell and its 4 clamped neighbours, power at the cell, one write).
template <bool I>
__global__ void __launch_bounds__(256) hotspot_kernel(const float* power, const float* src,
                                                      float* dst, int R, int C, float k_step,
                                                      float rx1, float ry1, float rz1, float amb) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  const int i = blockIdx.y * blockDim.y + threadIdx.y;
  if (i >= R || j >= C) return;
  const int idx = i * C + j;
  const float c = RD<I>(src[idx]);
  const float n = RD<I>(src[(i > 0 ? i - 1 : 0) * C + j]);
  const float s = RD<I>(src[(i < R - 1 ? i + 1 : R - 1) * C + j]);
  const float w = RD<I>(src[i * C + (j > 0 ? j - 1 : 0)]);
  const float e = RD<I>(src[i * C + (j < C - 1 ? j + 1 : C - 1)]);
  const float p = RD<I>(power[idx]);
  WR<I>(dst[idx]) = c + k_step * (p + (s + n - 2.f * c) * ry1 + (e + w - 2.f * c) * rx1 + (amb - c) * rz1);
}

// ---------------------------------------------------------------------------
// backprop: layerforward and adjust_weights over 16x16 tiles of the
// (in+1) x (hid+1) weight matrix (Rodinia backprop shape).
constexpr int BP = 16;

template <bool I>
__global__ void __launch_bounds__(256) bp_layerforward(const float* input, float* weights,
                                                       float* partial, int hid) {
  __shared__ float in_node[BP];
  __shared__ float wm[BP][BP];
  const int by = blockIdx.x, tx = threadIdx.x, ty = threadIdx.y;
  const int index = (hid + 1) * BP * by + (hid + 1) * ty + tx + 1 + (hid + 1);
  const int index_in = BP * by + ty + 1;
  if (tx == 0) in_node[ty] = RD<I>(input[index_in]);
  __syncthreads();
  wm[ty][tx] = RD<I>(weights[index]) * in_node[ty];
  WR<I>(weights[index]) = wm[ty][tx];
  __syncthreads();
  for (int stride = 1; stride < BP; stride <<= 1) {
    if ((ty % (2 * stride)) == 0) wm[ty][tx] += wm[ty + stride][tx];
    __syncthreads();
  }
  if (ty == 0) WR<I>(partial[by * hid + tx]) = wm[0][tx];
}

template <bool I>
__global__ void __launch_bounds__(256) bp_adjust(const float* delta, const float* ly, float* w,
                                                 float* oldw, int hid) {
  const int by = blockIdx.x, tx = threadIdx.x, ty = threadIdx.y;
  const int index = (hid + 1) * BP * by + (hid + 1) * ty + tx + 1 + (hid + 1);
  const int index_y = BP * by + ty + 1;
  const int index_x = tx + 1;
  const float eta = 0.3f, momentum = 0.3f;
  const float d = RD<I>(delta[index_x]) * RD<I>(ly[index_y]);
  const float nw = eta * d + momentum * RW<I>(oldw[index]);
  RW<I>(w[index]) += nw;
  RW<I>(oldw[index]) = nw;
  if (ty == 0 && by == 0) {  // the bias row
    const float nb = eta * RD<I>(delta[index_x]) + momentum * RW<I>(oldw[index_x]);
    RW<I>(w[index_x]) += nb;
    RW<I>(oldw[index_x]) = nb;
  }
}

}  // namespace

extern "C" {

int xplw_bind_rodinia(xpl_ctx* ctx) { return (int)xpl_device_bind(ctx); }

int xplw_hotspot(xplw_run* run, const xplw_arrays* a, int R, int C, int iters) {
  App app(run);
  const uint64_t n = (uint64_t)R * C;
  float *temp_h = A<float>(a, 0), *power_h = A<float>(a, 1), *result_h = A<float>(a, 2);
  float *d_power = A<float>(a, 3), *d_temp[2] = {A<float>(a, 4), A<float>(a, 5)};
  app.reg(a);
  app.write_loop(temp_h, n);  // read the input files into host arrays
  app.write_loop(power_h, n);
  app.copy(d_power, power_h, n * 4, XPL_COPY_H2D);
  app.copy(d_temp[0], temp_h, n * 4, XPL_COPY_H2D);
  const dim3 blk(32, 8), grd((C + 31) / 32, (R + 7) / 8);
  int src = 0;
  for (int it = 0; it < iters; ++it) {
    app.begin();
    if (app.on())
      hotspot_kernel<true><<<grd, blk, 0, app.s>>>(d_power, d_temp[src], d_temp[1 - src], R, C, 0.5f, 0.1f, 0.1f, 0.01f, 80.f);
    else
      hotspot_kernel<false><<<grd, blk, 0, app.s>>>(d_power, d_temp[src], d_temp[1 - src], R, C, 0.5f, 0.1f, 0.1f, 0.01f, 80.f);
    app.end();
    run->dev_accesses += 7 * n;
    src = 1 - src;
    if (run->diag_each) app.diag();  // "after each iteration"
  }
  app.copy(result_h, d_temp[src], n * 4, XPL_COPY_D2H);
  app.read_loop(result_h, n);  // write the output file
  app.unreg(a);
  app.diag();  // "and at the end of the program"
  return run->status;
}

int xplw_backprop(xplw_run* run, const xplw_arrays* a, int in, int hid) {
  App app(run);
  const int nblk = in / BP;
  const uint64_t nw = (uint64_t)(in + 1) * (hid + 1);
  float *input_units = A<float>(a, 0), *input_weights = A<float>(a, 1), *partial_sum = A<float>(a, 2),
        *hidden_delta = A<float>(a, 3), *prev_weights = A<float>(a, 4);
  float *input_cuda = A<float>(a, 5), *input_hidden_cuda = A<float>(a, 7),
        *hidden_partial_sum = A<float>(a, 8), *hidden_delta_cuda = A<float>(a, 9),
        *input_prev_weights_cuda = A<float>(a, 10);
  app.reg(a);
  // bpnn_create + load: random inputs and weights, zero previous weights
  app.write_loop(input_units, in + 1);
  app.write_loop(input_weights, nw);
  app.write_loop(prev_weights, nw);
  app.copy(input_cuda, input_units, (in + 1) * 4, XPL_COPY_H2D);
  app.copy(input_hidden_cuda, input_weights, nw * 4, XPL_COPY_H2D);
  const dim3 blk(BP, BP), grd(nblk);
  app.begin();
  if (app.on()) bp_layerforward<true><<<grd, blk, 0, app.s>>>(input_cuda, input_hidden_cuda, hidden_partial_sum, hid);
  else bp_layerforward<false><<<grd, blk, 0, app.s>>>(input_cuda, input_hidden_cuda, hidden_partial_sum, hid);
  app.end();
  run->dev_accesses += (uint64_t)nblk * BP * BP * 2 + (uint64_t)nblk * BP * 2;
  app.copy(partial_sum, hidden_partial_sum, (uint64_t)nblk * hid * 4, XPL_COPY_D2H);
  // host: hidden sums, output layer and error terms (small), hidden deltas
  for (int j = 0; j < hid; ++j) app.read_loop(partial_sum, nblk, hid, j);  // sum over tiles
  app.write_loop(hidden_delta, hid + 1);
  app.copy(hidden_delta_cuda, hidden_delta, (hid + 1) * 4, XPL_COPY_H2D);
  app.copy(input_prev_weights_cuda, prev_weights, nw * 4, XPL_COPY_H2D);
  app.begin();
  if (app.on()) bp_adjust<true><<<grd, blk, 0, app.s>>>(hidden_delta_cuda, input_cuda, input_hidden_cuda, input_prev_weights_cuda, hid);
  else bp_adjust<false><<<grd, blk, 0, app.s>>>(hidden_delta_cuda, input_cuda, input_hidden_cuda, input_prev_weights_cuda, hid);
  app.end();
  run->dev_accesses += (uint64_t)nblk * BP * BP * 5 + (uint64_t)BP * 4;
  app.copy(input_weights, input_hidden_cuda, nw * 4, XPL_COPY_D2H);
  app.copy(input_units, input_cuda, (in + 1) * 4, XPL_COPY_D2H);  // Table II: not modified
  app.unreg(a);
  app.diag();
  return run->status;
}

}  // extern "C"
