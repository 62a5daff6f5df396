// comm_nccl.cpp -- the collectives of a sharded context (xpl.h xpl_comm) over
// NCCL: one communicator per rank and GPU, the exchange over NVLink / NVSwitch.
// The runtime hands host buffers (routing lists, partials, IPC handles); they
// bounce through a device buffer on a private stream: H2D, the NCCL call(s),
// D2H, then the host waits.  All-to-all = grouped ncclSend / ncclRecv.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>
#include <string.h>

#include <new>
#include <vector>

#include "xpl.h"

namespace {

struct NcclComm {
  xpl_comm api;  // first member: the xpl_comm* handed out points here
  ncclComm_t nc = nullptr;
  int rank = 0, world = 1, device = 0;
  cudaStream_t s = nullptr;
  uint8_t* d = nullptr;  // bounce buffer
  size_t cap = 0;
};

bool reserve(NcclComm* c, size_t bytes) {
  if (bytes <= c->cap) return true;
  if (c->d) cudaFree(c->d);
  c->d = nullptr;
  c->cap = 0;
  size_t n = bytes < (1u << 20) ? (1u << 20) : bytes;
  if (cudaMalloc(&c->d, n) != cudaSuccess) return false;
  c->cap = n;
  return true;
}

int allgather(void* user, const void* send, size_t bytes, void* recv) {
  NcclComm* c = (NcclComm*)user;
  if (cudaSetDevice(c->device) != cudaSuccess) return 1;
  if (!reserve(c, bytes * (c->world + 1))) return 2;
  uint8_t* ds = c->d;
  uint8_t* dr = c->d + bytes;
  if (bytes && cudaMemcpyAsync(ds, send, bytes, cudaMemcpyHostToDevice, c->s) != cudaSuccess) return 3;
  if (ncclAllGather(ds, dr, bytes, ncclUint8, c->nc, c->s) != ncclSuccess) return 4;
  if (bytes && cudaMemcpyAsync(recv, dr, bytes * c->world, cudaMemcpyDeviceToHost, c->s) != cudaSuccess) return 5;
  return cudaStreamSynchronize(c->s) == cudaSuccess ? 0 : 6;
}

int alltoallv(void* user, const void* send, const uint64_t* sb, void* recv, const uint64_t* rb) {
  NcclComm* c = (NcclComm*)user;
  if (cudaSetDevice(c->device) != cudaSuccess) return 1;
  uint64_t ts = 0, tr = 0;
  for (int q = 0; q < c->world; ++q) {
    ts += sb[q];
    tr += rb[q];
  }
  if (!reserve(c, ts + tr + 16)) return 2;
  uint8_t* ds = c->d;
  uint8_t* dr = c->d + ts;
  if (ts && cudaMemcpyAsync(ds, send, ts, cudaMemcpyHostToDevice, c->s) != cudaSuccess) return 3;
  if (ncclGroupStart() != ncclSuccess) return 4;
  uint64_t so = 0, ro = 0;
  for (int q = 0; q < c->world; ++q) {
    if (sb[q] && ncclSend(ds + so, sb[q], ncclUint8, q, c->nc, c->s) != ncclSuccess) return 5;
    if (rb[q] && ncclRecv(dr + ro, rb[q], ncclUint8, q, c->nc, c->s) != ncclSuccess) return 6;
    so += sb[q];
    ro += rb[q];
  }
  if (ncclGroupEnd() != ncclSuccess) return 7;
  if (tr && cudaMemcpyAsync(recv, dr, tr, cudaMemcpyDeviceToHost, c->s) != cudaSuccess) return 8;
  return cudaStreamSynchronize(c->s) == cudaSuccess ? 0 : 9;
}

int barrier(void* user) {
  NcclComm* c = (NcclComm*)user;
  if (cudaSetDevice(c->device) != cudaSuccess) return 1;
  if (!reserve(c, 64)) return 2;
  if (ncclAllReduce(c->d, c->d, 1, ncclInt32, ncclSum, c->nc, c->s) != ncclSuccess) return 3;
  return cudaStreamSynchronize(c->s) == cudaSuccess ? 0 : 4;
}

}  // namespace

extern "C" {

xpl_status xpl_comm_nccl_unique_id(uint8_t id[128]) {
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  if (!id) return XPL_ERR_INVALID_ARG;
  ncclUniqueId u;
  if (ncclGetUniqueId(&u) != ncclSuccess) return XPL_ERR_NCCL;
  memcpy(id, &u, 128);
  return XPL_OK;
}

xpl_status xpl_comm_nccl_create(const uint8_t id[128], int rank, int world, int device, xpl_comm** out) {
  if (!id || !out || world < 1 || rank < 0 || rank >= world) return XPL_ERR_INVALID_ARG;
  NcclComm* c = new (std::nothrow) NcclComm();
  if (!c) return XPL_ERR_OOM;
  c->rank = rank;
  c->world = world;
  c->device = device;
  if (cudaSetDevice(device) != cudaSuccess || cudaStreamCreateWithFlags(&c->s, cudaStreamNonBlocking) != cudaSuccess) {
    delete c;
    return XPL_ERR_CUDA;
  }
  ncclUniqueId u;
  memcpy(&u, id, 128);
  if (ncclCommInitRank(&c->nc, world, u, rank) != ncclSuccess) {
    cudaStreamDestroy(c->s);
    delete c;
    return XPL_ERR_NCCL;
  }
  c->api.user = c;
  c->api.allgather = allgather;
  c->api.alltoallv = alltoallv;
  c->api.barrier = barrier;
  *out = &c->api;
  return XPL_OK;
}

xpl_status xpl_comm_nccl_destroy(xpl_comm* comm) {
  if (!comm) return XPL_ERR_INVALID_ARG;
  NcclComm* c = (NcclComm*)comm->user;
  cudaSetDevice(c->device);
  if (c->s) cudaStreamSynchronize(c->s);
  if (c->nc) ncclCommDestroy(c->nc);
  if (c->d) cudaFree(c->d);
  if (c->s) cudaStreamDestroy(c->s);
  delete c;
  return XPL_OK;
}

}  // extern "C"
