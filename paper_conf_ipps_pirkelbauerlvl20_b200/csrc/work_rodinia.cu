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
__device__ __forceinline__ decltype(auto) RDL(const T& x) {  // the latency-variant read hook (xpl_read_lat)
  if constexpr (I) return xpl_read_lat(x);
  else return (x);
}
template <bool I, class T>
__device__ __forceinline__ T& WRL(T& x) {  // the latency-variant write hook (xpl_write_lat)
  if constexpr (I) return xpl_write_lat(x);
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
  // (noinline: the loops get their own register allocation instead of sharing
  // the program's large driver function; the same for the twin)
  template <class T>
  __attribute__((noinline)) void write_loop(T* p, uint64_t n) {
    const auto t0 = std::chrono::steady_clock::now();
    xpl_host_site st;  // one per static access site (xpl_host.h)
    if (tr)
      for (uint64_t i = 0; i < n; ++i) tr->write(p[i], st) = (T)(i & 1023) * (T)0.001;
    else
      for (uint64_t i = 0; i < n; ++i) p[i] = (T)(i & 1023) * (T)0.001;
    run->host_accesses += n;
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  // s += p[i * stride + off] for i < n  -- a traced host read loop
  template <class T>
  __attribute__((noinline)) T read_loop(const T* p, uint64_t n, uint64_t stride = 1, uint64_t off = 0) {
    const auto t0 = std::chrono::steady_clock::now();
    T acc = 0;
    xpl_host_site st;
    if (tr)
      for (uint64_t i = 0; i < n; ++i) acc += tr->read(p[i * stride + off], st);
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
  // epoch around one launch; the launch parameters go to the runtime's launch
  // log (xpl_kernel_launch: a no-op unless the log is on; NEXT-4)
  void begin(const char* name, dim3 grd, dim3 blk) {
    flush();
    if (on()) {
      ok(xpl_kernel_begin(run->ctx, s));
      const xpl_launch_info li = {name, {grd.x, grd.y, grd.z}, {blk.x, blk.y, blk.z}, 0};
      ok(xpl_kernel_launch(run->ctx, s, &li));
    }
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


// ---------------------------------------------------------------------------
// bfs: Rodinia's two-kernel level-synchronous BFS (graph in CSR with uniform
// degree).  Every hook call is counted per thread and added once per block.
struct BfsNode {
  int starting, no_of_edges;
};

template <bool I>
__device__ __forceinline__ void count_hooks(unsigned long long* hc, unsigned c) {
  if constexpr (I) {
    __shared__ unsigned s_c;
    if (threadIdx.x == 0) s_c = 0;
    __syncthreads();
    if (c) atomicAdd(&s_c, c);
    __syncthreads();
    if (threadIdx.x == 0 && s_c) atomicAdd(hc, (unsigned long long)s_c);
  }
}

template <bool I>
__global__ void __launch_bounds__(512) bfs_kernel1(BfsNode* nodes, int* edges, bool* mask,
                                                   bool* updating, bool* visited, int* cost, int n,
                                                   unsigned long long* hc) {
  const int tid = blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  if (tid < n) {
    ++c;
    if (RD<I>(mask[tid])) {
      WR<I>(mask[tid]) = false;
      c += 4;  // the write, the loop init and the first loop test (2 reads)
      for (int i = RD<I>(nodes[tid].starting);
           i < (RD<I>(nodes[tid].no_of_edges) + RD<I>(nodes[tid].starting)); i++) {
        const int id = RD<I>(edges[i]);
        c += 4;  // edges, visited, and the next loop test (2 reads)
        if (!RD<I>(visited[id])) {
          WR<I>(cost[id]) = RD<I>(cost[tid]) + 1;
          WR<I>(updating[id]) = true;
          c += 3;
        }
      }
    }
  }
  count_hooks<I>(hc, c);
}

template <bool I>
__global__ void __launch_bounds__(512) bfs_kernel2(bool* mask, bool* updating, bool* visited,
                                                   bool* over, int n, unsigned long long* hc) {
  const int tid = blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  if (tid < n) {
    ++c;
    if (RD<I>(updating[tid])) {
      WR<I>(mask[tid]) = true;
      WR<I>(visited[tid]) = true;
      WR<I>(*over) = true;
      WR<I>(updating[tid]) = false;
      c += 4;
    }
  }
  count_hooks<I>(hc, c);
}

// ---------------------------------------------------------------------------
// nw: Rodinia's Needleman-Wunsch, 16x16 tiles, one block-diagonal per launch.
constexpr int NWB = 16;

__host__ __device__ __forceinline__ int nw_max(int a, int b, int c) {
  const int k = a <= b ? b : a;
  return k <= c ? c : k;
}

template <bool I, bool UPPER>
__global__ void __launch_bounds__(NWB) nw_kernel(int* ref, int* mat, int cols, int penalty, int i,
                                                 int block_width) {
  const int bx = blockIdx.x, tx = threadIdx.x;
  const int b_index_x = UPPER ? bx : bx + block_width - i;
  const int b_index_y = UPPER ? i - 1 - bx : block_width - bx - 1;
  const int index = cols * NWB * b_index_y + NWB * b_index_x + tx + (cols + 1);
  const int index_n = cols * NWB * b_index_y + NWB * b_index_x + tx + 1;
  const int index_w = cols * NWB * b_index_y + NWB * b_index_x + cols;
  const int index_nw = cols * NWB * b_index_y + NWB * b_index_x;
  __shared__ int temp[NWB + 1][NWB + 1];
  __shared__ int rf[NWB][NWB];
  if (tx == 0) temp[tx][0] = RDL<I>(mat[index_nw]);
  for (int ty = 0; ty < NWB; ty++) rf[ty][tx] = RDL<I>(ref[index + cols * ty]);
  __syncthreads();
  temp[tx + 1][0] = RDL<I>(mat[index_w + cols * tx]);
  __syncthreads();
  temp[0][tx + 1] = RDL<I>(mat[index_n]);
  __syncthreads();
  for (int m = 0; m < NWB; m++) {
    if (tx <= m) {
      const int t_x = tx + 1, t_y = m - tx + 1;
      temp[t_y][t_x] = nw_max(temp[t_y - 1][t_x - 1] + rf[t_y - 1][t_x - 1],
                              temp[t_y][t_x - 1] - penalty, temp[t_y - 1][t_x] - penalty);
    }
    __syncthreads();
  }
  for (int m = NWB - 2; m >= 0; m--) {
    if (tx <= m) {
      const int t_x = tx + NWB - m, t_y = NWB - tx;
      temp[t_y][t_x] = nw_max(temp[t_y - 1][t_x - 1] + rf[t_y - 1][t_x - 1],
                              temp[t_y][t_x - 1] - penalty, temp[t_y - 1][t_x] - penalty);
    }
    __syncthreads();
  }
  for (int ty = 0; ty < NWB; ty++) WRL<I>(mat[index + ty * cols]) = temp[ty + 1][tx + 1];  // 16-thread blocks
}

// ---------------------------------------------------------------------------
// Host loops of the programs, as separate functions (their own register
// allocation; tr == nullptr is the uninstrumented twin).  Each static access
// site has its own xpl_host_site (xpl_host.h).
__attribute__((noinline)) void bfs_read_nodes(xpl_host_tracer* tr, BfsNode* h_nodes, bool* h_mask,
                                              bool* h_updating, bool* h_visited, int n, int deg) {
  if (tr) {
    xpl_host_site s0, s1, s2, s3, s4;
    for (int i = 0; i < n; i++) {
      tr->write(h_nodes[i].starting, s0) = i * deg;
      tr->write(h_nodes[i].no_of_edges, s1) = deg;
      tr->write(h_mask[i], s2) = false;
      tr->write(h_updating[i], s3) = false;
      tr->write(h_visited[i], s4) = false;
    }
  } else {
    for (int i = 0; i < n; i++) {
      h_nodes[i].starting = i * deg;
      h_nodes[i].no_of_edges = deg;
      h_mask[i] = h_updating[i] = h_visited[i] = false;
    }
  }
}

// the edge list is stored as read from the input; costs -1
__attribute__((noinline)) void bfs_read_edges(xpl_host_tracer* tr, int* h_edges, uint64_t ne,
                                              int* h_cost, int n) {
  if (tr) {
    xpl_host_site s0, s1;
    for (uint64_t i = 0; i < ne; ++i) {
      const int e = h_edges[i];  // (the input buffer; the traced store is the program's)
      tr->write(h_edges[i], s0) = e;
    }
    for (int i = 0; i < n; ++i) tr->write(h_cost[i], s1) = -1;
  } else {
    for (int i = 0; i < n; ++i) h_cost[i] = -1;
  }
}

// the substitution matrix from the sequences (row / column 0), then the gap row and column
__attribute__((noinline)) void nw_fill_reference(xpl_host_tracer* tr, int* in, int* refh,
                                                 const int* blosum, int rows, int cols, int penalty) {
  if (tr) {
    xpl_host_site s0, s1, s2, s3, s4;
    for (int i = 1; i < rows; i++)
      for (int j = 1; j < cols; j++) {
        const int x = tr->read(in[i * cols], s0), y = tr->read(in[j], s1);
        tr->write(refh[i * cols + j], s2) = blosum[x * 24 + y];
      }
    for (int i = 1; i < rows; i++) tr->write(in[i * cols], s3) = -i * penalty;
    for (int j = 1; j < cols; j++) tr->write(in[j], s4) = -j * penalty;
  } else {
    for (int i = 1; i < rows; i++)
      for (int j = 1; j < cols; j++) refh[i * cols + j] = blosum[in[i * cols] * 24 + in[j]];
    for (int i = 1; i < rows; i++) in[i * cols] = -i * penalty;
    for (int j = 1; j < cols; j++) in[j] = -j * penalty;
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
    app.begin("hotspot_kernel", grd, blk);
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
  app.begin("bp_layerforward", grd, blk);
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
  app.begin("bp_adjust", grd, blk);
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


int xplw_bfs(xplw_run* run, const xplw_arrays* a, int n, int deg, unsigned long long* hook_count,
             int* levels) {
  App app(run);
  BfsNode* h_nodes = A<BfsNode>(a, 0);
  int* h_edges = A<int>(a, 1);
  bool *h_mask = A<bool>(a, 2), *h_updating = A<bool>(a, 3), *h_visited = A<bool>(a, 4);
  int* h_cost = A<int>(a, 5);
  bool* h_over = A<bool>(a, 6);
  BfsNode* d_nodes = A<BfsNode>(a, 7);
  int* d_edges = A<int>(a, 8);
  bool *d_mask = A<bool>(a, 9), *d_updating = A<bool>(a, 10), *d_visited = A<bool>(a, 11);
  int* d_cost = A<int>(a, 12);
  bool* d_over = A<bool>(a, 13);
  const uint64_t ne = (uint64_t)n * deg;
  app.reg(a);
  // read the graph "file": node records, masks, edges, costs (Rodinia bfs.cu order)
  {
    const auto t0 = std::chrono::steady_clock::now();
    bfs_read_nodes(app.tr, h_nodes, h_mask, h_updating, h_visited, n, deg);
    run->host_accesses += 5ull * n;
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  if (app.tr) {
    app.tr->write(h_mask[0]) = true;
    app.tr->write(h_visited[0]) = true;
  } else {
    h_mask[0] = h_visited[0] = true;
  }
  run->host_accesses += 2;
  {  // the edge list is stored as read from the input; costs -1, source 0
    const auto t0 = std::chrono::steady_clock::now();
    bfs_read_edges(app.tr, h_edges, ne, h_cost, n);
    if (app.tr) app.tr->write(h_cost[0]) = 0;
    else h_cost[0] = 0;
    run->host_accesses += ne + n + 1;
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  app.copy(d_nodes, h_nodes, sizeof(BfsNode) * n, XPL_COPY_H2D);
  app.copy(d_edges, h_edges, sizeof(int) * ne, XPL_COPY_H2D);
  app.copy(d_mask, h_mask, n, XPL_COPY_H2D);
  app.copy(d_updating, h_updating, n, XPL_COPY_H2D);
  app.copy(d_visited, h_visited, n, XPL_COPY_H2D);
  app.copy(d_cost, h_cost, sizeof(int) * n, XPL_COPY_H2D);
  const int blocks = (n + 511) / 512;
  int k = 0;
  bool stop = false;
  do {
    if (app.tr) app.tr->write(*h_over) = false;
    else *h_over = false;
    run->host_accesses += 1;
    app.copy(d_over, h_over, 1, XPL_COPY_H2D);
    if (!run->do_copies)  // control data: the loop needs it even when bulk data is resident
      app.ok_cuda(cudaMemcpyAsync(d_over, h_over, 1, cudaMemcpyHostToDevice, app.s));
    app.begin("bfs_kernel1", dim3(blocks), dim3(512));
    if (app.on()) bfs_kernel1<true><<<blocks, 512, 0, app.s>>>(d_nodes, d_edges, d_mask, d_updating, d_visited, d_cost, n, hook_count);
    else bfs_kernel1<false><<<blocks, 512, 0, app.s>>>(d_nodes, d_edges, d_mask, d_updating, d_visited, d_cost, n, hook_count);
    app.end();
    app.begin("bfs_kernel2", dim3(blocks), dim3(512));
    if (app.on()) bfs_kernel2<true><<<blocks, 512, 0, app.s>>>(d_mask, d_updating, d_visited, d_over, n, hook_count);
    else bfs_kernel2<false><<<blocks, 512, 0, app.s>>>(d_mask, d_updating, d_visited, d_over, n, hook_count);
    app.end();
    app.copy(h_over, d_over, 1, XPL_COPY_D2H);
    if (!run->do_copies) {  // the control flow needs the flag even with resident data
      app.ok_cuda(cudaMemcpyAsync(h_over, d_over, 1, cudaMemcpyDeviceToHost, app.s));
      app.ok_cuda(cudaStreamSynchronize(app.s));
    }
    stop = app.tr ? app.tr->read(*h_over) : *h_over;
    run->host_accesses += 1;
    ++k;
    if (run->diag_each) app.diag();
  } while (stop && k < n + 1 && !run->status);  // (a BFS has at most n levels)
  *levels = k;
  app.copy(h_cost, d_cost, sizeof(int) * n, XPL_COPY_D2H);
  app.read_loop(h_cost, n);  // write the result file
  app.unreg(a);
  app.diag();
  return run->status;
}

int xplw_nw(xplw_run* run, const xplw_arrays* a, int n, int penalty, const int* blosum) {
  App app(run);
  const int cols = n + 1, rows = n + 1;
  int *in = A<int>(a, 0), *refh = A<int>(a, 1), *out = A<int>(a, 2);
  int *ref_d = A<int>(a, 3), *mat_d = A<int>(a, 4);
  app.reg(a);
  // the sequences (row / column 0) are the input; the substitution matrix from them
  {
    const auto t0 = std::chrono::steady_clock::now();
    nw_fill_reference(app.tr, in, refh, blosum, rows, cols, penalty);
    run->host_accesses += 3ull * (rows - 1) * (cols - 1);
    run->host_accesses += (uint64_t)(rows - 1) + (cols - 1);
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  app.copy(ref_d, refh, sizeof(int) * rows * cols, XPL_COPY_H2D);
  app.copy(mat_d, in, sizeof(int) * rows * cols, XPL_COPY_H2D);
  const int bw = (cols - 1) / NWB;
  for (int i = 1; i <= bw; i++) {
    app.begin("nw_kernel_upper", dim3(i), dim3(NWB));
    if (app.on()) nw_kernel<true, true><<<i, NWB, 0, app.s>>>(ref_d, mat_d, cols, penalty, i, bw);
    else nw_kernel<false, true><<<i, NWB, 0, app.s>>>(ref_d, mat_d, cols, penalty, i, bw);
    app.end();
    run->dev_accesses += (uint64_t)i * (1 + 2 * NWB * NWB + 2 * NWB);
  }
  for (int i = bw - 1; i >= 1; i--) {
    app.begin("nw_kernel_lower", dim3(i), dim3(NWB));
    if (app.on()) nw_kernel<true, false><<<i, NWB, 0, app.s>>>(ref_d, mat_d, cols, penalty, i, bw);
    else nw_kernel<false, false><<<i, NWB, 0, app.s>>>(ref_d, mat_d, cols, penalty, i, bw);
    app.end();
    run->dev_accesses += (uint64_t)i * (1 + 2 * NWB * NWB + 2 * NWB);
  }
  app.copy(out, mat_d, sizeof(int) * rows * cols, XPL_COPY_D2H);
  // traceback (Rodinia nw): from the bottom-right corner towards (0, 0)
  {
    const auto t0 = std::chrono::steady_clock::now();
    const int LIMIT = -999;
    xpl_host_site s_nw, s_w, s_n, s_ref;  // the traceback's read sites
    auto R = [&](int* p, xpl_host_site& st) -> int {
      run->host_accesses += 1;
      return app.tr ? app.tr->read(*p, st) : *p;
    };
    app.sink += R(&out[(rows - 2) * cols + rows - 2], s_nw);  // the score printed first
    for (int i = rows - 2, j = rows - 2; i >= 0 && j >= 0;) {
      if (i == 0 && j == 0) break;
      int nw, w, nn;
      if (i > 0 && j > 0) {
        nw = R(&out[(i - 1) * cols + j - 1], s_nw);
        w = R(&out[i * cols + j - 1], s_w);
        nn = R(&out[(i - 1) * cols + j], s_n);
      } else if (i == 0) {
        nw = nn = LIMIT;
        w = R(&out[i * cols + j - 1], s_w);
      } else {
        nw = w = LIMIT;
        nn = R(&out[(i - 1) * cols + j], s_n);
      }
      const int new_nw = nw + R(&refh[i * cols + j], s_ref);
      const int new_w = w - penalty, new_n = nn - penalty;
      int tb = nw_max(new_nw, new_w, new_n);
      if (tb == new_nw) tb = nw;
      if (tb == new_w) tb = w;
      if (tb == new_n) tb = nn;
      if (tb == nw) { i--; j--; continue; }
      else if (tb == w) { j--; continue; }
      else if (tb == nn) { i--; continue; }
      else break;
    }
    app.flush();
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
  app.unreg(a);
  app.diag();
  return run->status;
}

}  // extern "C"
