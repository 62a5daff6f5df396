// um_counters.cpp -- libxplum.so: CUPTI unified-memory counters kept per record
// with their addresses (include/xpl_um.h; NEXT-4).
#include <cupti.h>
#include <dlfcn.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>
#include <vector>

#include "xpl_um.h"

namespace {

struct Rec {
  uint64_t addr, value;
  uint32_t kind;
};

std::mutex g_mu;
std::vector<Rec> g_recs;
uint64_t g_dropped = 0;
bool g_callbacks = false;
uint32_t g_kinds = 0;  // 1 << CUpti_ActivityUnifiedMemoryCounterKind accepted
constexpr size_t kCap = size_t(1) << 22;
constexpr size_t kBuf = size_t(8) << 20;

void CUPTIAPI buffer_requested(uint8_t** buf, size_t* size, size_t* max_records) {
  *buf = (uint8_t*)aligned_alloc(8, kBuf);
  *size = *buf ? kBuf : 0;
  *max_records = 0;
}

void CUPTIAPI buffer_completed(CUcontext, uint32_t, uint8_t* buf, size_t, size_t valid) {
  CUpti_Activity* rec = nullptr;
  std::lock_guard<std::mutex> g(g_mu);
  while (cuptiActivityGetNextRecord(buf, valid, &rec) == CUPTI_SUCCESS) {
    if (rec->kind != CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER) continue;
    const auto* u = (const CUpti_ActivityUnifiedMemoryCounter3*)rec;
    if (g_recs.size() >= kCap) {
      ++g_dropped;
      continue;
    }
    g_recs.push_back(Rec{u->address, u->value, (uint32_t)u->counterKind});
  }
  free(buf);
}

}  // namespace

extern "C" {

int xpl_um_enable(int device) {
  // "should be called after CUDA driver initialization" (cupti_activity.h): init
  // the driver, but create no context -- the counters must be set up before it
  // (libcuda is opened here, not linked: the library must load on driverless hosts)
  void* drv = dlopen("libcuda.so.1", RTLD_NOW | RTLD_GLOBAL);
  auto cu_init = drv ? (int (*)(unsigned))dlsym(drv, "cuInit") : nullptr;
  if (!cu_init) return 1000 + 100;  // CUDA_ERROR_NO_DEVICE-like: no driver
  const int cr = cu_init(0);
  if (cr != 0) return 1000 + cr;
  CUptiResult r;
  if (!g_callbacks) {
    r = cuptiActivityRegisterCallbacks(buffer_requested, buffer_completed);
    if (r != CUPTI_SUCCESS) return 4000 + (int)r;
    g_callbacks = true;
  }
  const CUpti_ActivityUnifiedMemoryCounterKind kinds[] = {
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_HTOD,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_DTOH,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_CPU_PAGE_FAULT_COUNT,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_THRASHING,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_THROTTLING,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_REMOTE_MAP,
      CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_DTOD};
  // Which kinds / scopes CUPTI accepts differs by platform: probe each kind alone
  // (single-device scope first, then all devices), then configure the accepted set.
  const uint32_t n = sizeof kinds / sizeof kinds[0];
  CUpti_ActivityUnifiedMemoryCounterConfig cfg[sizeof kinds / sizeof kinds[0]];
  uint32_t m = 0;
  int first_err = 0;
  g_kinds = 0;
  for (uint32_t i = 0; i < n; ++i) {
    for (CUpti_ActivityUnifiedMemoryCounterScope sc : {CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_SCOPE_PROCESS_SINGLE_DEVICE,
                                                       CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_SCOPE_PROCESS_ALL_DEVICES}) {
      CUpti_ActivityUnifiedMemoryCounterConfig c;
      c.scope = sc;
      c.kind = kinds[i];
      c.deviceId = (uint32_t)device;
      c.enable = 1;
      r = cuptiActivityConfigureUnifiedMemoryCounter(&c, 1);
      if (r == CUPTI_SUCCESS) {
        cfg[m++] = c;
        g_kinds |= 1u << (uint32_t)kinds[i];
        break;
      }
      if (!first_err) first_err = (int)r;
    }
  }
  if (!m) return first_err ? first_err : -1;
  r = cuptiActivityConfigureUnifiedMemoryCounter(cfg, m);
  if (r != CUPTI_SUCCESS) return 3000 + (int)r;
  r = cuptiActivityEnable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER);
  return r == CUPTI_SUCCESS ? 0 : 2000 + (int)r;
}

int xpl_um_disable(void) {
  cuptiActivityFlushAll(0);
  return (int)cuptiActivityDisable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER);
}

int xpl_um_read(uint64_t base, uint64_t bytes, xpl_um_counts* out, int reset) {
  if (!out) return -1;
  memset(out, 0, sizeof *out);
  const CUptiResult r = cuptiActivityFlushAll(1);  // CUPTI_ACTIVITY_FLAG_FLUSH_FORCED
  if (r != CUPTI_SUCCESS) return (int)r;
  std::lock_guard<std::mutex> g(g_mu);
  for (const Rec& x : g_recs) {
    if (bytes && (x.addr < base || x.addr - base >= bytes)) continue;
    ++out->records;
    switch (x.kind) {
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_HTOD: out->htod_bytes += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_DTOH: out->dtoh_bytes += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_DTOD: out->dtod_bytes += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_CPU_PAGE_FAULT_COUNT: out->cpu_page_faults += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT: out->gpu_page_fault_groups += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_THRASHING: out->thrashing += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_THROTTLING: out->throttling += x.value; break;
      case CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_REMOTE_MAP: out->remote_map += x.value; break;
      default: break;
    }
  }
  if (reset) g_recs.clear();
  return 0;
}

uint32_t xpl_um_kinds(void) { return g_kinds; }

uint64_t xpl_um_dropped(void) {
  std::lock_guard<std::mutex> g(g_mu);
  return g_dropped;
}

}  // extern "C"
