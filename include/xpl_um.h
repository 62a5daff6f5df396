/* include/xpl_um.h -- unified-memory fault and migration counters (SURVEY §8(f)
 * NEXT-4, optional part): the CUPTI counters the paper proposes to collect
 * around kernel launches "in order to more precisely pinpoint" page faults
 * (P:L227).  A separate library, libxplum.so, so that the
 * runtime (libxpl.so) does not depend on CUPTI.
 *
 * Collects CUPTI unified-memory counter records (HtoD / DtoH / DtoD migrated
 * bytes, CPU page faults, GPU page-fault groups, thrashing, throttling, remote
 * maps) for one device and keeps each record's kind, value and virtual address,
 * so counts can be taken per address range -- per allocation, next to the
 * xpl page view (xpl_page_summary) of the same interval.
 *
 * Call xpl_um_enable before the process creates its CUDA context where the
 * platform requires it (CUPTI may refuse unified-memory counters otherwise);
 * every function returns 0 or an error: xpl_um_enable returns 1000 + CUresult
 * (driver init), 4000 + / 3000 + / 2000 + CUptiResult (callback registration /
 * counter configuration / activity enable), or the CUptiResult of the probe of
 * the first kind when no kind is accepted; the others return the CUptiResult.
 * Not thread-safe; one collector per process. */
#ifndef XPL_UM_H
#define XPL_UM_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  uint64_t htod_bytes, dtoh_bytes, dtod_bytes;
  uint64_t cpu_page_faults;       /* CPU page faults (count)                          */
  uint64_t gpu_page_fault_groups; /* GPU fault groups (CUPTI's GPU_PAGE_FAULT value)  */
  uint64_t thrashing, throttling, remote_map;
  uint64_t records;               /* counter records that fell in the range           */
} xpl_um_counts;

/* Configure and enable the counters for `device`.  0 on success. */
int xpl_um_enable(int device);
/* Stop collecting (records already kept stay readable). */
int xpl_um_disable(void);
/* Flush CUPTI's buffers (synchronise the device first) and sum the kept records whose
 * address lies in [base, base + bytes) -- bytes == 0: all records, whatever their
 * address.  reset != 0 drops every kept record afterwards.  0 on success. */
int xpl_um_read(uint64_t base, uint64_t bytes, xpl_um_counts* out, int reset);
/* The counter kinds the platform accepted at xpl_um_enable, as bits 1 << k in
 * CUPTI's numbering: 1 HtoD bytes, 2 DtoH bytes, 3 CPU page faults, 4 GPU page
 * faults, 5 thrashing, 6 throttling, 7 remote map, 8 DtoD bytes. */
uint32_t xpl_um_kinds(void);
/* Records dropped because the keep buffer was full (cap 2^22 records). */
uint64_t xpl_um_dropped(void);

#ifdef __cplusplus
}
#endif
#endif /* XPL_UM_H */
