// tools/host_tracer_bench.cpp -- CPU microbenchmark of the inline host tracer
// (include/xpl_host.h) on the host-loop shapes of the bench workloads, with a
// stub xpl_record_host_ranges that only counts.  No GPU.
//   g++ -O3 -march=native -std=c++17 -Iinclude tools/host_tracer_bench.cpp -o /tmp/htb && /tmp/htb
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "xpl.h"
static size_t g_ranges = 0;
extern "C" xpl_status xpl_record_host_strided(xpl_ctx*, const xpl_host_strided*, size_t n) {
  g_ranges += n;
  return XPL_OK;
}
#include "xpl_host.h"
#ifdef HTB_PINNED
#include <cuda_runtime.h>
#endif

// The workload's shape: a noinline member loop reading the tracer from its object.
struct AppLike {
  xpl_host_tracer* tr = nullptr;
  template <class T>
  __attribute__((noinline)) void write_loop(T* p, uint64_t n) {
    xpl_host_site st;
    if (tr)
      for (uint64_t i = 0; i < n; ++i) tr->write(p[i], st) = (T)(i & 1023) * (T)0.001;
    else
      for (uint64_t i = 0; i < n; ++i) p[i] = (T)(i & 1023) * (T)0.001;
  }
};

template <class F>
static double t_ms(F f) {
  auto t0 = std::chrono::steady_clock::now();
  f();
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

struct Node {
  int starting, no_of_edges;
};
volatile double g_sink;

int main(int argc, char** argv) {
  const int reps = argc > 1 ? atoi(argv[1]) : 5;
  const uint64_t n = 11u << 20;  // backprop weights (640K x 17)
  std::vector<float> f(n);
  float* pin = nullptr;
#ifdef HTB_PINNED
  if (cudaHostAlloc((void**)&pin, n * sizeof(float), cudaHostAllocDefault) != cudaSuccess) pin = nullptr;
#endif
  const int bn = 1 << 20, deg = 6;
  std::vector<Node> nodes(bn);
  std::vector<char> m1(bn), m2(bn), m3(bn);
  std::vector<int> edges((size_t)bn * deg), cost(bn);
  const int N = 2049;
  std::vector<int> in((size_t)N * N), ref((size_t)N * N);
  int blosum[24 * 24];
  for (int i = 0; i < 24 * 24; ++i) blosum[i] = i % 11 - 5;
  for (size_t i = 0; i < in.size(); ++i) in[i] = (int)(i * 2654435761u >> 27) % 24;

  for (int traced = 0; traced < 3; ++traced) {  // 0 plain, 1 traced, 2 traced with site hints
    double best[4] = {1e30, 1e30, 1e30, 1e30};
    for (int r = 0; r < reps; ++r) {
      xpl_host_tracer* tr = traced ? new xpl_host_tracer(nullptr) : nullptr;
      // 1: float write loop (hotspot / backprop init)
      double t = t_ms([&] {
        xpl_host_site s0;
        if (traced == 2)
          for (uint64_t i = 0; i < n; ++i) tr->write(f[i], s0) = (float)(i & 1023) * 0.001f;
        else if (tr)
          for (uint64_t i = 0; i < n; ++i) tr->write(f[i]) = (float)(i & 1023) * 0.001f;
        else
          for (uint64_t i = 0; i < n; ++i) f[i] = (float)(i & 1023) * 0.001f;
        if (tr) tr->flush();
      });
      best[0] = std::min(best[0], t / n * 1e6);
      // 2: bfs init: 5 interleaved streams incl. bool arrays
      t = t_ms([&] {
        xpl_host_site s0, s1, s2, s3, s4;
        for (int i = 0; i < bn; ++i) {
          if (traced == 2) {
            tr->write(nodes[i].starting, s0) = i * deg;
            tr->write(nodes[i].no_of_edges, s1) = deg;
            tr->write(m1[i], s2) = false;
            tr->write(m2[i], s3) = false;
            tr->write(m3[i], s4) = false;
          } else if (tr) {
            tr->write(nodes[i].starting) = i * deg;
            tr->write(nodes[i].no_of_edges) = deg;
            tr->write(m1[i]) = false;
            tr->write(m2[i]) = false;
            tr->write(m3[i]) = false;
          } else {
            nodes[i].starting = i * deg;
            nodes[i].no_of_edges = deg;
            m1[i] = m2[i] = m3[i] = false;
          }
        }
        if (tr) tr->flush();
      });
      best[1] = std::min(best[1], t / (5.0 * bn) * 1e6);
      // 3: nw reference matrix: 2 reads + 1 write per element
      t = t_ms([&] {
        xpl_host_site s0, s1, s2;
        if (traced == 2) {
          for (int i = 1; i < N; i++)
            for (int j = 1; j < N; j++) {
              const int x = tr->read(in[i * N], s0), y = tr->read(in[j], s1);
              tr->write(ref[i * N + j], s2) = blosum[x * 24 + y];
            }
          tr->flush();
        } else if (tr) {
          for (int i = 1; i < N; i++)
            for (int j = 1; j < N; j++) {
              const int x = tr->read(in[i * N]), y = tr->read(in[j]);
              tr->write(ref[i * N + j]) = blosum[x * 24 + y];
            }
          tr->flush();
        } else {
          for (int i = 1; i < N; i++)
            for (int j = 1; j < N; j++) ref[i * N + j] = blosum[in[i * N] * 24 + in[j]];
        }
      });
      best[2] = std::min(best[2], t / (3.0 * (N - 1) * (N - 1)) * 1e6);
      // 4: read loop with a sum (result files)
      t = t_ms([&] {
        double acc = 0;
        xpl_host_site s0;
        if (traced == 2)
          for (uint64_t i = 0; i < n; ++i) acc += tr->read(f[i], s0);
        else if (tr)
          for (uint64_t i = 0; i < n; ++i) acc += tr->read(f[i]);
        else
          for (uint64_t i = 0; i < n; ++i) acc += f[i];
        if (tr) tr->flush();
        g_sink = acc;
      });
      best[3] = std::min(best[3], t / n * 1e6);
      delete tr;
    }
    printf("%s  ns/access: float-write %.3f  bfs-init %.3f  nw-ref %.3f  float-read %.3f   (ranges %zu)\n",
           traced == 2 ? "sites " : traced ? "traced" : "plain ", best[0], best[1], best[2], best[3], g_ranges);
    // the app's shape: noinline member loop, over pageable and pinned memory
    double b_pg = 1e30, b_pin = 1e30;
    for (int r = 0; r < reps; ++r) {
      AppLike app;
      app.tr = traced ? new xpl_host_tracer(nullptr) : nullptr;
      double t = t_ms([&] { app.write_loop(f.data(), n); if (app.tr) app.tr->flush(); });
      b_pg = std::min(b_pg, t / n * 1e6);
      if (pin) {
        t = t_ms([&] { app.write_loop(pin, n); if (app.tr) app.tr->flush(); });
        b_pin = std::min(b_pin, t / n * 1e6);
      }
      delete app.tr;
    }
    printf("        app-shaped write_loop<float>: pageable %.3f  pinned %.3f\n", b_pg, pin ? b_pin : -1.0);
  }
  return 0;
}
