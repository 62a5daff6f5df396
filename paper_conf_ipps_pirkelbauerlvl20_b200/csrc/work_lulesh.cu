// work_lulesh.cu -- a LULESH-shaped instrumented program (the paper's main case
// study, §II-C, §III-D, Fig. 4).
//
// Shape, not physics: a managed singleton "domain" object of 3736 bytes
// holds the pointers of 50 managed arrays and the scalar
// parameters; every kernel reads the array pointers it uses from the domain
// (RAJA lambdas capture the domain), so all GPU threads hit the same domain
// words.  Per timestep: 16 kernel stages (19 launches) -- nodal force zeroing,
// element stress and hourglass forces gathered through the 8-node lists into a
// temporary, corner sums back to nodes through node->corner lists, nodal
// acceleration / symmetry planes / velocity / position, element kinematics into
// a second temporary, Q gradients over face neighbours, four EOS stages, volume
// update, courant and hydro dt reductions.  Two temporaries are allocated,
// published through the domain, and freed every timestep.  The
// host then reads the dt reductions and updates the domain (TimeIncrement): it
// writes 27 domain words and reads 680; the kernels read 85 domain words, 18 of
// them CPU-written -- the dom row of Fig. 4 (C=27, C>C=680, 9 %, 18
// alternating).  The CPU twin (oracle trace) is xplgen/lulesh.py.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <chrono>
#include <vector>

#include "xpl.h"
#include "xpl_device.cuh"
#include "xpl_host.h"
#include "xplw.h"

namespace {

// ---- the domain object (3736 bytes = 934 words) ----
enum Slot {
  X, Y, Z, XD, YD, ZD, XDD, YDD, ZDD, FX, FY, FZ, NODALMASS,                   // nodal reals
  E, P, Q, V, VOLO, VNEW, DELV, VDOV, AREALG, SS, ELEMMASS, QL, QQ,             // element reals
  NODELIST, LXIM, LXIP, NODEELEMSTART, CORNERLIST, SYMMX, ELEMBC,               // topology
  LETAM, LETAP, LZETAM, LZETAP, SYMMY, SYMMZ,                                   // never used
  DELV_XI, DELV_ETA, DELV_ZETA, DELX_XI, DELX_ETA, DELX_ZETA, DXX, DYY, DZZ,    // never used
  TMP_FORCE, TMP_DVDX, NSLOT
};
struct Dom {
  void* ptr[NSLOT];  // words 0..99
  uint32_t numElem;  // word 100 (read by every kernel)
  uint32_t numNode;  // word 101
  double dt;         // words 102-103
  double time;       // words 104-105
  uint32_t cycle;    // word 106
  uint32_t pad107;
  double dtcourant;  // words 108-109
  double dthydro;    // words 110-111
  uint32_t misc[14]; // words 112-125: written by the host each step; 112-121 read by kernels
  uint32_t params[808];
};
static_assert(NSLOT == 50, "50 pointer slots");
static_assert(sizeof(Dom) == 3736, "the domain object of Fig. 5 has 3736 bytes (P:L315)");

// The index ranges one rank's kernels cover (sharded program, xplw_run.world >
// 1): elements [e0, e1) (e0 a multiple of 256, so dt blocks stay whole), nodes
// [n0, n1), symmetry-plane nodes [s0, s1).  One rank: everything.
struct Part {
  int e0, e1, n0, n1, s0, s1;
};

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

// Arrays a thread accesses several times go through array handles (the row
// lookup of the base pointer hoisted out of the accesses, xpl_array); the twin
// gets a plain pointer with the same interface.
template <bool I, class T>
struct Arr : xpl_array<T> {
  __device__ __forceinline__ explicit Arr(T* q) : xpl_array<T>(q) {}
};
template <class T>
struct Arr<false, T> {
  T* p;
  __device__ __forceinline__ explicit Arr(T* q) : p(q) {}
  __device__ __forceinline__ const T& read(unsigned long long i) const { return p[i]; }
  __device__ __forceinline__ T& write(unsigned long long i) const { return p[i]; }
  __device__ __forceinline__ T& rw(unsigned long long i) const { return p[i]; }
};

// Instrumented kernels: CTAs per SM the register budget is sized for (the hooks'
// dependent loads want occupancy more than registers).
#ifndef XPL_LULESH_MINB
#define XPL_LULESH_MINB 3
#endif

// Hook calls are counted per thread (c) and added once per block (exact counts).
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

// every traced access goes through one of these (and is counted)
#ifndef XPL_LULESH_PIPE
#define XPL_LULESH_PIPE 1  // (profiles/r2p_pipe_ab.txt: paired hook cost -25 % at depth 1)
#endif
#if XPL_LULESH_PIPE
// the plain hooks through a hook pipeline (xpl_pipe: each commit deferred by
// XPL_LULESH_PIPE_DEPTH hooks, so consecutive shadow loads overlap); A/B switch
#ifndef XPL_LULESH_PIPE_DEPTH
#define XPL_LULESH_PIPE_DEPTH 1  // (depth 4 and 8 measured no better: the hooks are mostly issue-bound)
#endif
template <bool I>
struct Pipe : xpl_pipe<XPL_LULESH_PIPE_DEPTH> {};
template <>
struct Pipe<false> {
  template <class T> __device__ __forceinline__ const T& read(const T& x) { return x; }
  template <class T> __device__ __forceinline__ T& write(T& x) { return x; }
  template <class T> __device__ __forceinline__ T& rw(T& x) { return x; }
};
#define R_(x) (++c, xp_.read(x))
#define W_(x) (++c, xp_.write(x))
#define RW_(x) (++c, xp_.rw(x))
#define PIPE_DECL Pipe<I> xp_
#else
#define R_(x) (++c, RD<I>(x))
#define W_(x) (++c, WR<I>(x))
#define RW_(x) (++c, RW<I>(x))
#define PIPE_DECL
#endif
#define PTR(T, slot) static_cast<T*>(R_(d->ptr[slot]))
#define ARR(T, slot) Arr<I, T>(PTR(T, slot))
#define RA_(h, i) (++c, (h).read(i))
#define WA_(h, i) (++c, (h).write(i))
#define RWA_(h, i) (++c, (h).rw(i))
#define NE() (int)R_(d->numElem)

// 1. zero the nodal forces
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_zero_forces(Part P_, Dom* d, int nn, unsigned long long* hc) {
  const int n = P_.n0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (n < P_.n1 && n < nn) {
    WA_(ARR(double, FX), n) = 0.0;
    WA_(ARR(double, FY), n) = 0.0;
    WA_(ARR(double, FZ), n) = 0.0;
  }
  count_hooks<I>(hc, c);
}

// 2. stress integration: gather the 8 nodes, write 8 corner forces x 3
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_integrate_stress(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const auto nl = ARR(const int, NODELIST);
    const auto x = ARR(const double, X), y = ARR(const double, Y), z = ARR(const double, Z);
    const double sig = -(RA_(ARR(const double, P), e) + RA_(ARR(const double, Q), e));
    const auto f = ARR(double, TMP_FORCE);
    for (int k = 0; k < 8; ++k) {
      const int n = RA_(nl, 8 * e + k);
      const double g = RA_(x, n) + RA_(y, n) + RA_(z, n);
      WA_(f, 24 * e + 3 * k + 0) = sig * g;
      WA_(f, 24 * e + 3 * k + 1) = sig * g * 0.5;
      WA_(f, 24 * e + 3 * k + 2) = sig * g * 0.25;
    }
  }
  count_hooks<I>(hc, c);
}

// 3. hourglass control: gather nodal velocities, add to the corner forces
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_hourglass(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const auto nl = ARR(const int, NODELIST);
    const auto xd = ARR(const double, XD), yd = ARR(const double, YD), zd = ARR(const double, ZD);
    const double coef = RA_(ARR(const double, SS), e) * RA_(ARR(const double, ELEMMASS), e) /
                        (RA_(ARR(const double, VOLO), e) * RA_(ARR(const double, V), e) + 1.0);
    const auto f = ARR(double, TMP_FORCE);
    for (int k = 0; k < 8; ++k) {
      const int n = RA_(nl, 8 * e + k);
      const double a = RA_(xd, n), b = RA_(yd, n), g = RA_(zd, n);
      RWA_(f, 24 * e + 3 * k + 0) += coef * a;
      RWA_(f, 24 * e + 3 * k + 1) += coef * b;
      RWA_(f, 24 * e + 3 * k + 2) += coef * g;
    }
  }
  count_hooks<I>(hc, c);
}

// 4. sum the corner forces into the nodes through the node->corner lists
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_corner_sum(Part P_, Dom* d, int nn, unsigned long long* hc) {
  const int n = P_.n0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (n < P_.n1 && n < nn) {
    const auto st = ARR(const int, NODEELEMSTART), cl = ARR(const int, CORNERLIST);
    const auto f = ARR(const double, TMP_FORCE);
    double *fx = PTR(double, FX), *fy = PTR(double, FY), *fz = PTR(double, FZ);
    const int b = RA_(st, n), en = RA_(st, n + 1);
    double sx = 0, sy = 0, sz = 0;
    for (int k = b; k < en; ++k) {
      const int corner = RA_(cl, k);
      sx += RA_(f, 3 * corner + 0);
      sy += RA_(f, 3 * corner + 1);
      sz += RA_(f, 3 * corner + 2);
    }
    W_(fx[n]) = sx;
    W_(fy[n]) = sy;
    W_(fz[n]) = sz;
  }
  count_hooks<I>(hc, c);
}

// 5. nodal accelerations
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_accel(Part P_, Dom* d, int nn, unsigned long long* hc) {
  const int n = P_.n0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (n < P_.n1 && n < nn) {
    const double m = RA_(ARR(const double, NODALMASS), n);
    const double ax = RA_(ARR(const double, FX), n) / m, ay = RA_(ARR(const double, FY), n) / m,
                 az = RA_(ARR(const double, FZ), n) / m;
    WA_(ARR(double, XDD), n) = ax;
    WA_(ARR(double, YDD), n) = ay;
    WA_(ARR(double, ZDD), n) = az;
  }
  count_hooks<I>(hc, c);
}

// 6. symmetry plane: zero the accelerations of the plane's nodes
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_symm(Part P_, Dom* d, int ns, unsigned long long* hc) {
  const int k = P_.s0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (k < P_.s1 && k < ns) {
    const int n = R_(PTR(const int, SYMMX)[k]);
    WA_(ARR(double, XDD), n) = 0.0;
    WA_(ARR(double, YDD), n) = 0.0;
    WA_(ARR(double, ZDD), n) = 0.0;
  }
  count_hooks<I>(hc, c);
}

// 7./8. velocity and position updates
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_velocity(Part P_, Dom* d, int nn, unsigned long long* hc) {
  const int n = P_.n0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (n < P_.n1 && n < nn) {
    const double dt = R_(d->dt);
    const double ax = RA_(ARR(const double, XDD), n), ay = RA_(ARR(const double, YDD), n),
                 az = RA_(ARR(const double, ZDD), n);
    RWA_(ARR(double, XD), n) += dt * ax;
    RWA_(ARR(double, YD), n) += dt * ay;
    RWA_(ARR(double, ZD), n) += dt * az;
  }
  count_hooks<I>(hc, c);
}
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_position(Part P_, Dom* d, int nn, unsigned long long* hc) {
  const int n = P_.n0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (n < P_.n1 && n < nn) {
    const double dt = R_(d->dt);
    const double vx = RA_(ARR(const double, XD), n), vy = RA_(ARR(const double, YD), n),
                 vz = RA_(ARR(const double, ZD), n);
    RWA_(ARR(double, X), n) += dt * vx;
    RWA_(ARR(double, Y), n) += dt * vy;
    RWA_(ARR(double, Z), n) += dt * vz;
  }
  count_hooks<I>(hc, c);
}

// 9. element kinematics: gather positions and velocities, new volume, gradients
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_kinematics(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const auto nl = ARR(const int, NODELIST);
    const auto x = ARR(const double, X), y = ARR(const double, Y), z = ARR(const double, Z);
    const auto xd = ARR(const double, XD), yd = ARR(const double, YD), zd = ARR(const double, ZD);
    double vol = 0, dv = 0;
    for (int k = 0; k < 8; ++k) {
      const int n = RA_(nl, 8 * e + k);
      vol += RA_(x, n) * RA_(y, n) + RA_(z, n);
      dv += RA_(xd, n) + RA_(yd, n) + RA_(zd, n);
    }
    const double vnew = vol / (RA_(ARR(const double, VOLO), e) + 1.0);
    const double vold = RA_(ARR(const double, V), e);
    WA_(ARR(double, VNEW), e) = vnew;
    WA_(ARR(double, DELV), e) = vnew - vold;
    WA_(ARR(double, AREALG), e) = vol;
    const auto g = ARR(double, TMP_DVDX);
    WA_(g, 3 * e + 0) = dv;
    WA_(g, 3 * e + 1) = dv * 0.5;
    WA_(g, 3 * e + 2) = dv * 0.25;
  }
  count_hooks<I>(hc, c);
}

// 10. strain rate from the gradients
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_lagrange(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const auto g = ARR(const double, TMP_DVDX);
    const double r = (RA_(g, 3 * e) + RA_(g, 3 * e + 1) + RA_(g, 3 * e + 2)) / (RA_(ARR(const double, VNEW), e) + 1.0);
    WA_(ARR(double, VDOV), e) = r;
  }
  count_hooks<I>(hc, c);
}

// 11./12. monotonic Q: gradients over the xi face neighbours, region limiter
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_monoq_grad(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const double* vdov = PTR(const double, VDOV);
    const int m = RA_(ARR(const int, LXIM), e), p = RA_(ARR(const int, LXIP), e);
    const double r = R_(vdov[p]) - R_(vdov[m]) + RA_(ARR(const double, VNEW), e);
    WA_(ARR(double, QL), e) = r;
  }
  count_hooks<I>(hc, c);
}
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_monoq_region(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const int bc = RA_(ARR(const int, ELEMBC), e);
    const double r = (bc & 1 ? 0.5 : 1.0) * RA_(ARR(const double, QL), e) * RA_(ARR(const double, VDOV), e);
    WA_(ARR(double, QQ), e) = r;
  }
  count_hooks<I>(hc, c);
}

// 13. the four EOS stages (they read material parameters from the domain)
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_eos(Part P_, Dom* d, int stage, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const double t = R_(d->time);
    if (stage == 0) {  // energy
      const double w = R_(d->misc[0]) * 1e-6 + R_(d->misc[1]) * 1e-6 + R_(d->misc[2]);
      const double de = RA_(ARR(const double, DELV), e) *
                        (RA_(ARR(const double, P), e) + RA_(ARR(const double, Q), e) +
                         RA_(ARR(const double, QQ), e) + RA_(ARR(const double, QL), e));
      RWA_(ARR(double, E), e) += w - de;
    } else if (stage == 1) {  // pressure
      const double pmin = R_(d->misc[3]) * 1e-6 + R_(d->misc[4]);
      const double r = pmin + RA_(ARR(const double, E), e) / (RA_(ARR(const double, VNEW), e) + t);
      WA_(ARR(double, P), e) = r;
    } else if (stage == 2) {  // sound speed
      const double ss4o3 = R_(d->misc[5]) * 1e-6 + R_(d->misc[6]);
      const double r = ss4o3 * (RA_(ARR(const double, P), e) + RA_(ARR(const double, E), e)) /
                       (RA_(ARR(const double, VNEW), e) + 1.0);
      WA_(ARR(double, SS), e) = r;
    } else {  // artificial viscosity
      const double qstop = R_(d->misc[7]) * 1e-6 + R_(d->misc[8]) + R_(d->misc[9]);
      const double r = qstop + RA_(ARR(const double, QL), e) + RA_(ARR(const double, QQ), e) +
                       0.0 * RA_(ARR(const double, P), e);
      WA_(ARR(double, Q), e) = r;
    }
  }
  count_hooks<I>(hc, c);
}

// 14. volumes
template <bool I>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_update_volumes(Part P_, Dom* d, unsigned long long* hc) {
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    const double v = RA_(ARR(const double, VNEW), e);
    WA_(ARR(double, V), e) = v;
  }
  count_hooks<I>(hc, c);
}

// 15./16. dt reductions: one minimum per 256-element block into dtb (GPU W, host R)
template <bool I, bool COURANT>
__global__ void __launch_bounds__(256, I ? XPL_LULESH_MINB : 1) k_dt(Part P_, Dom* d, double* dtb, int nblk, unsigned long long* hc) {
  __shared__ double s_min[256];
  const int e = P_.e0 + blockIdx.x * blockDim.x + threadIdx.x;
  unsigned c = 0;
  PIPE_DECL;
  double v = 1e30;
  if (e < NE() && e < P_.e1) {  // (every thread reads numElem, as the twin counts)
    if (COURANT) {
      const double ss = RA_(ARR(const double, SS), e), vd = RA_(ARR(const double, VDOV), e),
                   ar = RA_(ARR(const double, AREALG), e);
      v = ar / (ss * ss + vd * vd + 1.0);
    } else {
      const double vd = RA_(ARR(const double, VDOV), e);
      v = 1.0 / (vd * vd + 1e-3);
    }
  }
  s_min[threadIdx.x] = v;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o && s_min[threadIdx.x + o] < s_min[threadIdx.x]) s_min[threadIdx.x] = s_min[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) W_(dtb[(COURANT ? 0 : nblk) + P_.e0 / 256 + blockIdx.x]) = s_min[0];
  count_hooks<I>(hc, c);
}

}  // namespace

extern "C" {

int xplw_bind_lulesh(xpl_ctx* ctx) { return (int)xpl_device_bind(ctx); }

// Word-level layout of the domain for the CPU twin: byte offset of a field.
int xplw_lulesh_layout(int what) {
  switch (what) {
    case 0: return (int)sizeof(Dom);
    case 1: return (int)offsetof(Dom, numElem);
    case 2: return (int)offsetof(Dom, dt);
    case 3: return (int)offsetof(Dom, time);
    case 4: return (int)offsetof(Dom, cycle);
    case 5: return (int)offsetof(Dom, dtcourant);
    case 6: return (int)offsetof(Dom, dthydro);
    case 7: return (int)offsetof(Dom, misc);
    case 8: return (int)offsetof(Dom, params);
    default: return -1;
  }
}

int xplw_lulesh(xplw_run* run, const xplw_arrays* arr, int s, int steps, unsigned long long* hook_count,
                unsigned long long* tmp_addrs) {
  const bool on = run->ctx != nullptr;
  cudaStream_t st = (cudaStream_t)run->stream;
  const int ne = s * s * s, nn = (s + 1) * (s + 1) * (s + 1), nsym = (s + 1) * (s + 1);
  const int nblk = (ne + 255) / 256;
  // sharded program (run->world > 1, one rank per GPU, a sharded context): this
  // rank's kernels cover an element range (whole dt blocks), a node range and a
  // symmetry-node range; its host traces its slice of every array's init; rank 0
  // traces the single-copy host segments (domain init, TimeIncrement).
  const int R = run->world > 1 ? run->world : 1, rk = R > 1 ? run->rank : 0;
  Part P;
  {
    const int pe = ((ne + R - 1) / R + 255) / 256 * 256, pn = (nn + R - 1) / R, ps = (nsym + R - 1) / R;
    P.e0 = std::min(ne, rk * pe), P.e1 = std::min(ne, P.e0 + pe);
    P.n0 = std::min(nn, rk * pn), P.n1 = std::min(nn, P.n0 + pn);
    P.s0 = std::min(nsym, rk * ps), P.s1 = std::min(nsym, P.s0 + ps);
  }
  const int GE = std::max(1, (P.e1 - P.e0 + 255) / 256), GN = std::max(1, (P.n1 - P.n0 + 255) / 256),
            GS = std::max(1, (P.s1 - P.s0 + 255) / 256);
  Dom* dom = (Dom*)arr->addr[0];
  double* dtb = (double*)arr->addr[1];
  // arr->addr[2 + k] = the array of pointer slot k (k < TMP_FORCE)
  xpl_host_tracer* tr = on ? new xpl_host_tracer(run->ctx) : nullptr;
  auto ok = [&](int x) {
    if (x && !run->status) run->status = x;
  };
  auto okc = [&](cudaError_t e) {
    if (e != cudaSuccess && !run->status) run->status = XPL_ERR_CUDA;
  };
  auto flush = [&]() {
    if (tr) ok(tr->flush());
  };
  auto host_t = [&](std::chrono::steady_clock::time_point t0) {
    run->host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  };
  auto diag = [&]() {
    flush();
    if (!on) return;
    size_t nr = 0;
    xpl_alloc_report* o = run->out ? run->out + run->n_out : nullptr;
    const size_t cap = run->out ? run->out_cap - run->n_out : 0;
    const int x = xpl_diagnose(run->ctx, &run->params, nullptr, 0, o, cap, &nr, run->diag_no_reset ? 0 : 1);
    if (x == XPL_OK) {
      run->n_out += nr;
      if (run->diag_rows && run->n_diag < run->diag_cap) run->diag_rows[run->n_diag] = (uint32_t)nr;
      run->n_diag++;
    } else {
      ok(x);
    }
  };
  // one instrumented launch = one GPU epoch (the kernel-launch wrapper);
  // time_kernels: CUDA events around the kernel alone (its epoch close excluded)
  std::vector<cudaEvent_t> evs;
  auto mark = [&]() {
    if (!run->time_kernels) return;
    cudaEvent_t e;
    okc(cudaEventCreate(&e));
    okc(cudaEventRecord(e, st));
    evs.push_back(e);
  };
  // time_kernels == 2 (a measurement run of the instrumented program): the twin
  // kernel runs too, right before or after the instrumented one (alternating by
  // launch index), each timed, each after an L2 flush (a 256 MB memset, untimed):
  // the pair sees the same cache state and, up to order, the same page
  // residency, so the hooks' cost (instrumented - twin) is not buried under the
  // application's unified-memory faults.  The data then evolves twice per
  // launch; such a run is for timing only.
  const bool paired = on && run->time_kernels == 2;
  const size_t kFlush = 256ull << 20;
  void* l2flush = nullptr;
  if (paired) okc(cudaMalloc(&l2flush, kFlush));
  auto launch = [&](auto fi, auto ft, int grid) {
    flush();
    if (on) ok(xpl_kernel_begin(run->ctx, st));
    if (paired) {
      const bool twin_first = (run->epochs & 1) != 0;
      if (l2flush) okc(cudaMemsetAsync(l2flush, 1, kFlush, st));
      mark();
      if (twin_first) ft(grid);
      else fi(grid);
      mark();
      if (l2flush) okc(cudaMemsetAsync(l2flush, 2, kFlush, st));
      mark();
      if (twin_first) fi(grid);
      else ft(grid);
      mark();
    } else {
      mark();
      if (on) fi(grid);
      else ft(grid);
      mark();
    }
    okc(cudaGetLastError());
    if (on) ok(xpl_kernel_end(run->ctx, st));
    run->epochs++;
  };
  auto sum_events = [&]() {
    if (evs.empty()) return;
    okc(cudaStreamSynchronize(st));
    for (size_t i = 0; i + 1 < evs.size(); i += 2) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, evs[i], evs[i + 1]);
      run->kernel_ms += ms;
      if (run->kernel_ms_each && i / 2 < run->kernel_cap) run->kernel_ms_each[i / 2] = ms;
    }
    for (cudaEvent_t e : evs) cudaEventDestroy(e);
    evs.clear();
  };
#define LAUNCH(KER, GRID, ...)                                                          \
  launch([&](int g) { KER<true><<<g, 256, 0, st>>>(P, __VA_ARGS__); },                 \
         [&](int g) { KER<false><<<g, 256, 0, st>>>(P, __VA_ARGS__); }, GRID)
  auto managed = [&](size_t bytes) -> void* {
    void* p = nullptr;
    okc(cudaMallocManaged(&p, bytes));
    if (on && p) ok(xpl_register_alloc(run->ctx, p, bytes, XPL_ALLOC_MANAGED));
    return p;
  };
  auto release = [&](void* p) {
    if (on) ok(xpl_free(run->ctx, p));
    okc(cudaFree(p));  // (synchronises, like the application's cudaFree)
  };
  auto hw = [&](auto& x, auto v) {  // a traced host write
    if (tr) tr->write(x) = v;
    else x = v;
    run->host_accesses++;
  };
  xpl_host_tracer* const tr0 = rk == 0 ? tr : nullptr;  // the single-copy host segments
  auto hw0 = [&](auto& x, auto v) {
    if (tr0) {
      tr0->write(x) = v;
      run->host_accesses++;
    } else {
      x = v;
      if (!tr) run->host_accesses++;
    }
  };

  if (on)
    for (int k = 0; k < arr->n; ++k)
      ok(xpl_register_alloc(run->ctx, (const void*)arr->addr[k], arr->bytes[k], (xpl_alloc_kind)arr->kind[k]));
  // ---- initialisation (host): the domain, the arrays, the mesh topology ----
  auto t0 = std::chrono::steady_clock::now();
  for (int k = 0; k < NSLOT; ++k) hw0(dom->ptr[k], k < TMP_FORCE ? (void*)arr->addr[2 + k] : (void*)nullptr);
  hw0(dom->numElem, (uint32_t)ne);
  hw0(dom->numNode, (uint32_t)nn);
  hw0(dom->dt, 1e-3);
  hw0(dom->time, 0.0);
  hw0(dom->cycle, 0u);
  hw0(dom->pad107, 0u);
  hw0(dom->dtcourant, 1e20);
  hw0(dom->dthydro, 1e20);
  for (int k = 0; k < 14; ++k) hw0(dom->misc[k], (uint32_t)(k + 1));
  for (int k = 0; k < 808; ++k) hw0(dom->params[k], (uint32_t)k);
  // every array: its initial values (topology arrays: the input); a rank traces
  // its slice [i0, i1) of the element indices and writes the rest untraced
  auto slice = [&](uint64_t n, uint64_t* i0, uint64_t* i1) {
    const uint64_t per = (n + R - 1) / R;
    *i0 = std::min<uint64_t>(n, per * rk);
    *i1 = std::min<uint64_t>(n, *i0 + per);
  };
  for (int k = 0; k < TMP_FORCE; ++k) {
    const uint64_t bytes = arr->bytes[2 + k];
    uint64_t i0, i1;
    if (k >= NODELIST) {
      int* a = (int*)arr->addr[2 + k];
      slice(bytes / 4, &i0, &i1);
      const bool topo = k <= ELEMBC;
      for (uint64_t i = 0; i < bytes / 4; ++i) {
        const int v = topo ? a[i] : 0;
        if (i >= i0 && i < i1) hw(a[i], v);
        else a[i] = v;
      }
    } else {
      double* a = (double*)arr->addr[2 + k];
      slice(bytes / 8, &i0, &i1);
      for (uint64_t i = 0; i < bytes / 8; ++i) {
        const double v = 1.0 + (double)(i & 7) * 0.125;
        if (i >= i0 && i < i1) hw(a[i], v);
        else a[i] = v;
      }
    }
  }
  {
    uint64_t i0, i1;
    slice(2 * nblk, &i0, &i1);
    for (int b = 0; b < 2 * nblk; ++b) {
      if ((uint64_t)b >= i0 && (uint64_t)b < i1) hw(dtb[b], 0.0);
      else dtb[b] = 0.0;
    }
  }
  host_t(t0);

  for (int step = 0; step < steps; ++step) {
    // forces: a temporary for the 8 corner forces of every element
    void* tf = managed(sizeof(double) * 24 * (size_t)ne);
    if (tmp_addrs) tmp_addrs[2 * step] = (unsigned long long)tf;
    hw0(dom->ptr[TMP_FORCE], tf);
    LAUNCH(k_zero_forces, GN, dom, nn, hook_count);
    LAUNCH(k_integrate_stress, GE, dom, hook_count);
    LAUNCH(k_hourglass, GE, dom, hook_count);
    LAUNCH(k_corner_sum, GN, dom, nn, hook_count);
    okc(cudaStreamSynchronize(st));
    hw0(dom->ptr[TMP_FORCE], (void*)nullptr);
    flush();
    release(tf);
    LAUNCH(k_accel, GN, dom, nn, hook_count);
    LAUNCH(k_symm, GS, dom, nsym, hook_count);
    LAUNCH(k_velocity, GN, dom, nn, hook_count);
    LAUNCH(k_position, GN, dom, nn, hook_count);
    // kinematics: a temporary for the velocity gradients
    void* tg = managed(sizeof(double) * 3 * (size_t)ne);
    if (tmp_addrs) tmp_addrs[2 * step + 1] = (unsigned long long)tg;
    hw0(dom->ptr[TMP_DVDX], tg);
    LAUNCH(k_kinematics, GE, dom, hook_count);
    LAUNCH(k_lagrange, GE, dom, hook_count);
    okc(cudaStreamSynchronize(st));
    hw0(dom->ptr[TMP_DVDX], (void*)nullptr);
    flush();
    release(tg);
    LAUNCH(k_monoq_grad, GE, dom, hook_count);
    LAUNCH(k_monoq_region, GE, dom, hook_count);
    for (int stage = 0; stage < 4; ++stage) LAUNCH(k_eos, GE, dom, stage, hook_count);
    LAUNCH(k_update_volumes, GE, dom, hook_count);
    launch([&](int g) { k_dt<true, true><<<g, 256, 0, st>>>(P, dom, dtb, nblk, hook_count); },
           [&](int g) { k_dt<false, true><<<g, 256, 0, st>>>(P, dom, dtb, nblk, hook_count); }, GE);
    launch([&](int g) { k_dt<true, false><<<g, 256, 0, st>>>(P, dom, dtb, nblk, hook_count); },
           [&](int g) { k_dt<false, false><<<g, 256, 0, st>>>(P, dom, dtb, nblk, hook_count); }, GE);
    okc(cudaStreamSynchronize(st));
    // TimeIncrement (host): the dt minima, the domain's parameters, the new dt
    // (traced by rank 0: one copy in the logical program)
    t0 = std::chrono::steady_clock::now();
    double dc = 1e30, dh = 1e30;
    for (int b = 0; b < nblk; ++b) {
      const double v = tr0 ? tr0->read(dtb[b]) : dtb[b];
      dc = v < dc ? v : dc;
    }
    for (int b = 0; b < nblk; ++b) {
      const double v = tr0 ? tr0->read(dtb[nblk + b]) : dtb[nblk + b];
      dh = v < dh ? v : dh;
    }
    if (rk == 0) run->host_accesses += 2 * nblk;
    hw0(dom->dtcourant, dc);
    hw0(dom->dthydro, dh);
    const uint32_t* w = (const uint32_t*)dom;
    uint64_t chk = 0;
    for (int k = 100; k < 780; ++k) chk += tr0 ? tr0->read(w[k]) : w[k];  // 680 words of parameters
    if (rk == 0) run->host_accesses += 680;
    hw0(dom->dt, 1e-3 + (double)(chk & 1) * 1e-9);
    hw0(dom->time, dom->time + 1e-3);
    hw0(dom->cycle, (uint32_t)(step + 1));
    for (int k = 0; k < 14; ++k) hw0(dom->misc[k], (uint32_t)(k + 1));
    host_t(t0);
    if (run->diag_each) diag();  // "diagnostics are called at the end of every timestep"
  }
  flush();
  delete tr;
  tr = nullptr;
  if (run->keep_allocs) {
    if (on) ok(xpl_sync(run->ctx));
    okc(cudaStreamSynchronize(st));
    sum_events();
    if (l2flush) cudaFree(l2flush);
    return run->status;
  }
  if (on)
    for (int k = 0; k < arr->n; ++k) ok(xpl_free(run->ctx, (const void*)arr->addr[k]));
  diag();
  okc(cudaStreamSynchronize(st));
  sum_events();
  if (l2flush) cudaFree(l2flush);
  return run->status;
}

}  // extern "C"
