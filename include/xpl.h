/* include/xpl.h -- the C-ABI of the B200-native XPlacer recording + diagnosis
 * runtime (libxpl.so).
 *
 * Paper: P. Pirkelbauer, P.-H. Lin, T. Vanderbruggen, C. Liao, "XPlacer:
 * Automatic Analysis of Data Access Patterns on Heterogeneous CPU/GPU
 * Systems", IPDPS 2020.  "P:Lnnn" cites line nnn of the paper's text;
 * "Dnn" cites a reading of DESIGN.md §3 (= SURVEY.md §8(c)).
 *
 * Conventions for every entry point:
 *  - all functions return xpl_status; nothing throws across the ABI;
 *  - pointers to user memory are only used as numbers: the library never
 *    dereferences user data (only the address is looked up);
 *  - "host" arguments are host pointers; the library copies what it needs
 *    before returning, so the caller may reuse its buffers at once;
 *  - one host thread per context; one context per process and GPU.  With
 *    world > 1 (sharded mode, below) every rank makes every call marked
 *    COLLECTIVE, in the same order;
 *  - `stream` arguments are cudaStream_t values passed as void*.
 */
#ifndef XPL_H
#define XPL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  XPL_OK = 0,
  XPL_ERR_INVALID_ARG = 1,    /* NULL pointer, zero size, unknown enum, cap too small */
  XPL_ERR_OOM = 2,            /* shadow pool / table / staging capacity exhausted   */
  XPL_ERR_OVERLAP = 3,        /* xpl_register_alloc intersects a live allocation     */
  XPL_ERR_UNKNOWN_PTR = 4,    /* xpl_free of a pointer that is no live base          */
  XPL_ERR_STATE = 5,          /* call not allowed now (e.g. diagnose in an epoch)    */
  XPL_ERR_CUDA = 6,           /* a CUDA runtime call failed                           */
  XPL_ERR_NCCL = 7,           /* a collective failed (world > 1)                      */
  XPL_ERR_DEVICE_OVERFLOW = 8 /* a device-side capacity was exceeded                  */
} xpl_status;

/* How the memory was allocated; stored in the shadow memory table and
 * used to gate the anti-pattern flags (D8). */
typedef enum {
  XPL_ALLOC_DEVICE = 0,  /* cudaMalloc               */
  XPL_ALLOC_MANAGED = 1, /* cudaMallocManaged        */
  XPL_ALLOC_HOST = 2     /* malloc/new/cudaMallocHost */
} xpl_alloc_kind;

/* traceR / traceW / traceRW (Table I).  RW = read, then write (D6). */
typedef enum { XPL_ACC_R = 1, XPL_ACC_W = 2, XPL_ACC_RW = 3 } xpl_acc_kind;

/* The cudaMemcpy / cudaMemset wrappers of `#pragma xpl replace`.
 * H2D = a CPU write of dst, D2H = a CPU read of src; H2H = CPU read of src
 * and write of dst; D2D and MEMSET_DEV = GPU accesses in their own epoch, or in the
 * open one (D7, D19). */
typedef enum {
  XPL_COPY_H2D = 0,
  XPL_COPY_D2H = 1,
  XPL_COPY_H2H = 2,
  XPL_COPY_D2D = 3,
  XPL_MEMSET_DEV = 4
} xpl_copy_dir;

/* One host-side access as the host tracer saw it (16 bytes).  An access marks every
 * 32-bit word overlapping [addr, addr+size) of the allocation holding `addr`,
 * clipped to that allocation (D1, D2, D18). */
typedef struct {
  uint64_t addr;
  uint32_t size; /* bytes, >= 1; any size (large sizes are ranges) */
  uint32_t kind; /* xpl_acc_kind */
} xpl_host_access;

/* A strided sequence of host accesses (what xpl_host.h emits for scattered
 * accesses with a constant stride, e.g. a column walk): `count` accesses, the
 * j-th covering [addr + j*stride, addr + j*stride + size), in order j = 0, 1, ...
 * (32 bytes).  count == 1 is one xpl_record_host_ranges record. */
typedef struct {
  uint64_t addr;
  uint32_t size;  /* bytes, >= 1 */
  uint32_t kind;  /* xpl_acc_kind */
  int64_t stride; /* bytes between consecutive accesses (any sign, 0 = repeats) */
  uint64_t count; /* >= 1 */
} xpl_host_strided;

/* XplAllocData: names an allocation in the report. */
typedef struct {
  const void* addr;
  const char* expr;
  uint32_t elem_size;
} xpl_name;

/* ---- Sharded mode (world > 1) --------------------------------
 * One logical program runs SPMD over `world` processes, one GPU each; its shadow
 * memory is partitioned over the ranks' pools by logical word:
 *  - every allocation is registered by every rank (COLLECTIVE, same bytes and
 *    kind in the same order; the address may differ per rank -- each rank's
 *    table maps ITS address range).  An allocation of < 65536 words is owned
 *    whole by rank (logical id mod world); a larger one is cut into world
 *    pieces of ceil(words / world) words rounded up to 1024 (4 KiB), piece r
 *    owned by rank r.  Logical ids count registrations, as with one rank;
 *  - device hooks record into the owner's pool: local atomics for owned words,
 *    atomics over NVLink/NVSwitch into the peer-mapped pool for the others;
 *  - host records: between two collective calls each rank records its own
 *    slice of the logical host stream; the slices are ordered by rank (the
 *    logical host stream = rank 0's slice, then rank 1's, ...).  At the next
 *    collective call the records are routed to their owners (all-to-all) and
 *    merged there in that order;
 *  - epochs are collective (all ranks' kernels between kernel_begin/_end form
 *    one GPU epoch); the close waits for every rank's kernels (barrier) before
 *    each owner folds its pool, and the next begin waits for every rank's
 *    shadow work (folds, merges, resets) before any rank records again;
 *  - xpl_diagnose is collective: each owner analyses its pieces, the partials
 *    are exchanged (all-gather) and combined on every rank: every rank gets the
 *    same reports, equal to the unsharded run's (field `base`: the piece-0
 *    owner's address);
 *  - xpl_record_copy is collective; rank 0's call is the one recorded.
 * Reading D36: pieces are cut on 4 KiB boundaries of the
 * allocation, so only an access that is not aligned to its size can straddle
 * two pieces; such an access records only its words in the first piece.
 *
 * The collectives, on HOST buffers, blocking; every rank calls them in the same
 * order.  Return 0 on success.  Provided by xpl_comm_nccl_create (NCCL over
 * NVLink / NVSwitch) or by the caller (e.g. a gloo process group). */
typedef struct {
  void* user;
  /* recv[world * bytes] = every rank's send[bytes], in rank order */
  int (*allgather)(void* user, const void* send, size_t bytes, void* recv);
  /* rank r sends send_bytes[q] bytes (packed in q order in send) to every rank q
   * and receives recv_bytes[q] bytes from every q (packed in q order in recv) */
  int (*alltoallv)(void* user, const void* send, const uint64_t* send_bytes, void* recv,
                   const uint64_t* recv_bytes);
  int (*barrier)(void* user);
} xpl_comm;

#define XPL_MAX_RANKS 8

typedef struct {
  int device;            /* CUDA device ordinal                                   */
  int rank, world;       /* world > 1 => sharded mode (above), world <= XPL_MAX_RANKS */
  const xpl_comm* comm;  /* the collectives when world > 1 (kept by pointer), else NULL */
  uint64_t pool_words;   /* shadow pool capacity in words (1 byte each)   */
  uint64_t staging_recs; /* host-record staging capacity (records)                */
  uint32_t max_rows;     /* capacity of the allocation table                      */
} xpl_config;

/* NCCL collectives for a sharded context: rank 0 creates the id, the caller
 * broadcasts its 128 bytes (any transport), every rank creates its comm (one
 * NCCL communicator on `device`; buffers bounce through device memory, the
 * exchange runs over NVLink / NVSwitch).  *out is owned by the caller until
 * xpl_comm_nccl_destroy (after xpl_finalize of the contexts using it). */
xpl_status xpl_comm_nccl_unique_id(uint8_t id[128]);
xpl_status xpl_comm_nccl_create(const uint8_t id[128], int rank, int world, int device, xpl_comm** out);
xpl_status xpl_comm_nccl_destroy(xpl_comm* comm);

/* Diagnosis parameters. */
typedef struct {
  uint32_t density_threshold_pct; /* default 50 ("e.g., 50%"); "<=" per Eq. P:L102 (D11) */
  uint64_t block_words;           /* 0 = the whole allocation is one block (D12)           */
  uint64_t min_run_words;         /* minimum transfer run, default 256 (D16); 0 acts as 1  */
} xpl_diag_params;

/* Report flags (the three anti-patterns of §III-A, plus "unused"). */
#define XPL_PAT_ALTERNATING 1u  /* managed, CPU and GPU on one word, >= 1 a write */
#define XPL_PAT_LOW_DENSITY 2u  /* device/managed block with <= threshold density  */
#define XPL_PAT_UNNEEDED_H2D 4u /* device: CPU-written run the GPU never read     */
#define XPL_PAT_UNNEEDED_D2H 8u /* device: CPU read back a run the GPU never updated       */
#define XPL_PAT_UNUSED 16u      /* no access in the interval (Table II Backprop)   */

/* One row of the diagnosis (Fig. 4).  Counts are numbers of words,
 * each counted at most once per column. */
typedef struct {
  uint64_t id, base, bytes, words;
  uint32_t kind, live, name_idx /* index into the xpl_name array, or 0xFFFFFFFF */, flags;
  uint64_t w_c, w_g;                /* Fig. 4 "write counts C G"                   */
  uint64_t r_cc, r_cg, r_gc, r_gg;  /* Fig. 4 "C>C C>G G>C G>G" (origin>reader)    */
  uint64_t any_acc, gpu_acc, alternating;
  uint64_t density_pct_any, density_pct_gpu; /* floor(100*accessed/words) (D10, D22) */
  uint64_t low_density_blocks, low_density_words;
  uint64_t h2d_unused_runs, h2d_unused_words;
  uint64_t d2h_unneeded_runs, d2h_unneeded_words;
  uint64_t ever_accessed; /* any access since registration */
} xpl_alloc_report;

typedef struct xpl_ctx xpl_ctx;
struct xpl_dev_ctx; /* defined in xpl_device.cuh */

/* Counters the runtime keeps about itself (not part of the paper's output). */
typedef struct {
  uint64_t epochs, folds, fold_chunks /* 128-word chunks folded */, host_records,
      host_records_packed, merge_segments, range_segments, diagnoses,
      fold_chunks_max /* largest single fold */,
      kernel_launches; /* runtime kernels launched (not counting user kernels) */
} xpl_stats;

/* Create a context on cfg->device.  *out is owned by the caller until
 * xpl_finalize.  Zero fields of cfg take defaults (pool_words 2^28,
 * staging_recs 2^22, max_rows 4096).  Allocates the shadow pool in HBM (plus
 * 1/128 of it for the chunk maps of the epoch close).  world > 1: COLLECTIVE;
 * INVALID_ARG without cfg->comm, with rank outside [0, world) or world >
 * XPL_MAX_RANKS; the ranks' pools are mapped into each other (CUDA IPC) for the
 * hooks' remote atomics (every rank's pool_words must be equal). */
xpl_status xpl_init(const xpl_config* cfg, xpl_ctx** out);
/* Sharded mode: COLLECTIVE (no rank unmaps its pool while a peer may write it). */
xpl_status xpl_finalize(xpl_ctx* ctx);

/* The allocation wrappers.  register: ceil(bytes/4) zeroed records
 * (last writer = CPU, D3); OVERLAP if [ptr, ptr+bytes) intersects a live row;
 * STATE inside an open GPU epoch.  free: UNKNOWN_PTR unless ptr is a live
 * base; the row stops matching lookups now and is reported once more at the
 * next diagnose before its shadow is recycled (D17).
 * Sharded mode: both COLLECTIVE (same bytes / kind / order on every rank; free
 * takes each rank's own base of the allocation). */
xpl_status xpl_register_alloc(xpl_ctx* ctx, const void* ptr, size_t bytes, xpl_alloc_kind kind);
xpl_status xpl_free(xpl_ctx* ctx, const void* ptr);

/* GPU epoch delimiters around kernel launches (traceKernelLaunch).
 * Epochs nest; the epoch is the outermost begin..end (D19).  begin orders
 * `stream` after all pending runtime work; end orders the runtime after
 * `stream` (and every stream that began inside the epoch) and enqueues the
 * epoch close (fold).  Nothing synchronises the host.  end without an open
 * epoch -> STATE.
 * Stream lifetime: after an epoch whose kernels all ran on one (non-default)
 * stream, the epoch close is enqueued right behind them on that stream and the
 * runtime keeps using it for its next work (no cross-stream event for the next
 * epoch there).  Such a stream must stay valid until xpl_release_stream() names
 * it or xpl_finalize(); the legacy / per-thread default streams are never
 * adopted.  Sharded mode: COLLECTIVE; end waits for this rank's epoch streams
 * and for every rank (barrier) before the owner folds; begin (outermost) waits
 * for this rank's runtime stream and for every rank (barrier). */
xpl_status xpl_kernel_begin(xpl_ctx* ctx, void* stream);
xpl_status xpl_kernel_end(xpl_ctx* ctx, void* stream);

/* Host tracer batch (the !__CUDA_ARCH__ branch of traceR/traceW/traceRW).
 * recs: host array of n records in program order.  Untracked addresses are
 * ignored.  Inside an open GPU epoch the records are applied after
 * the epoch closes (D20). */
xpl_status xpl_record_host(xpl_ctx* ctx, const xpl_host_access* recs, size_t n);

/* Coalesced host ranges (what xpl_host.h's inline tracer emits): each record
 * stands for a run of consecutive accesses of one kind covering the bytes
 * [addr, addr+size); every word of every live allocation overlapping it is
 * accessed once, in program order with the other records.  Equal to
 * xpl_record_host on the individual accesses whenever no individual access
 * straddles two allocations.  Same ordering and epoch rules as xpl_record_host. */
xpl_status xpl_record_host_ranges(xpl_ctx* ctx, const xpl_host_access* recs, size_t n);

/* Strided host ranges: record i stands for recs[i].count ranges records
 * (addr + j*stride, size, kind), j = 0 .. count-1, in that order; the records
 * are in program order with each other.  Exactly xpl_record_host_ranges on the
 * expanded list (same ordering and epoch rules).  INVALID_ARG on kind outside
 * 1..3, size 0 or count 0. */
xpl_status xpl_record_host_strided(xpl_ctx* ctx, const xpl_host_strided* recs, size_t n);

/* The transfer wrappers (D7).  dst/src are the cudaMemcpy arguments.
 * A range is clipped to the allocation holding its first byte (D18).  Sharded
 * mode: COLLECTIVE; rank 0's call is the one recorded (D37). */
xpl_status xpl_record_copy(xpl_ctx* ctx, const void* dst, const void* src, size_t bytes,
                           xpl_copy_dir dir);

/* tracePrint: analyse every live row and every row freed since the
 * last reset, write one report per row in id order into out[0..cap), set
 * *n_out.  INVALID_ARG with *n_out = rows needed if cap is too small.  With
 * reset != 0 the interval bits are cleared (the last writer is kept, D4) and
 * freed rows are dropped.  STATE inside an open epoch, or (like xpl_sync) after
 * a forbidden device-side split.  Blocks until done.
 * params NULL = defaults; names may be NULL when n_names == 0.  Sharded mode:
 * COLLECTIVE; every rank gets the same reports (one per logical allocation). */
xpl_status xpl_diagnose(xpl_ctx* ctx, const xpl_diag_params* params, const xpl_name* names,
                        size_t n_names, xpl_alloc_report* out, size_t cap, size_t* n_out,
                        int reset);

/* ---- Address-range sharding: one logical allocation split into
 * pieces held by different contexts (ranks).  A piece is the contiguous range of
 * logical words [word_offset, word_offset + ceil(bytes/4)) of the logical
 * allocation `logical_id` (logical size logical_bytes); its address range
 * [ptr, ptr+bytes) is registered like xpl_register_alloc.  Pieces of one logical
 * allocation must tile [0, ceil(logical_bytes/4)) exactly.  (Virtual shards of
 * world-1 contexts; a sharded context cuts its pieces itself: STATE there.) */
xpl_status xpl_register_alloc_piece(xpl_ctx* ctx, const void* ptr, size_t bytes,
                                    xpl_alloc_kind kind, uint64_t logical_id,
                                    uint64_t word_offset, uint64_t logical_bytes);

/* One piece's share of a diagnosis: exchanged between ranks (all-gather of the
 * raw bytes) and combined by xpl_combine_partials.  Run summaries are the run
 * monoid (len, pre, suf, cnt, sum) of DESIGN.md §5; `blk_*` are the density
 * blocks cut by the piece's ends (block_words > 0): global block index, GPU
 * words in the piece, piece words in the block. */
typedef struct {
  uint64_t logical_id, word_offset, words, logical_words, logical_bytes, base;
  uint32_t kind, live, name_idx, pad;
  uint64_t cnt[9]; /* w_c w_g r_cc r_cg r_gc r_gg any gpu alternating */
  uint64_t u_run[5], d_run[5];
  uint64_t low_density_blocks, low_density_words; /* blocks wholly inside the piece */
  uint64_t blk_first, blk_first_g, blk_first_s, blk_last, blk_last_g, blk_last_s;
  uint64_t ever_accessed;
} xpl_partial;

/* xpl_diagnose, but every row is returned as a partial (out[0..cap), *n_out);
 * rows registered with xpl_register_alloc are single pieces of themselves. */
xpl_status xpl_diagnose_partials(xpl_ctx* ctx, const xpl_diag_params* params,
                                 const xpl_name* names, size_t n_names, xpl_partial* out,
                                 size_t cap, size_t* n_out, int reset);

/* Combine the partials of all ranks (host only, no GPU needed): one report per
 * logical allocation, in logical id order -- byte-identical to the report of
 * the unsharded allocation.  INVALID_ARG if the pieces do not tile their
 * logical allocation; *n_out = reports needed if cap is too small. */
xpl_status xpl_combine_partials(const xpl_partial* parts, size_t n, const xpl_diag_params* params,
                                xpl_alloc_report* out, size_t cap, size_t* n_out);

/* tracePrint's output: format reports as the textual summary of
 * Fig. 4 -- per allocation its name, write counts C G, read counts
 * C>C C>G G>C G>G, access density, alternating elements and the anti-pattern
 * findings -- or (csv != 0) as comma-separated raw counts with a header line.
 * names/n_names: the XplAllocData list the reports' name_idx refer to (may be
 * NULL); unnamed rows print as "alloc <id>".  only_named != 0 prints named rows
 * only ("checking N named allocations").  Writes at most cap bytes including the
 * terminating NUL into buf and sets *needed to the full length + 1; INVALID_ARG
 * if it did not fit (the caller retries with a larger buffer). */
xpl_status xpl_format_reports(const xpl_alloc_report* reps, size_t n, const xpl_name* names,
                              size_t n_names, int csv, int only_named, char* buf, size_t cap,
                              size_t* needed);

/* The device-side context the __device__ hooks of xpl_device.cuh use: copies
 * it into *out (a host struct of device pointers; valid until xpl_finalize). */
xpl_status xpl_get_device_ctx(xpl_ctx* ctx, struct xpl_dev_ctx* out);

/* Per-word records of the live row whose base is `base`, words
 * [word0, word0+n), copied into the host array out[n] (access maps, Fig. 5/7/8/10;
 * also the sampled-parity hook of the tests).  Blocks until done.  Sharded mode:
 * COLLECTIVE; `base` must be a piece this rank owns (INVALID_ARG otherwise). */
xpl_status xpl_shadow_dump(xpl_ctx* ctx, const void* base, uint64_t word0, uint64_t n,
                           uint8_t* out);

/* ---- Unified-memory page view ----
 * The current interval's records aggregated per page of `page_words` words (pages
 * counted from the allocation base, D31; the last page may be partial): which
 * processors touched the page, whether some single word was touched by both
 * (true sharing) or only disjoint words were (the "effect similar to false
 * sharing" of P:L90), and whether some word alternated (D9).  Page bits: */
#define XPL_PAGE_CPU 1u    /* some word accessed by the CPU (wC | rCC | rGC)  */
#define XPL_PAGE_GPU 2u    /* some word accessed by the GPU (wG | rCG | rGG)  */
#define XPL_PAGE_BOTH 4u   /* some word accessed by both                       */
#define XPL_PAGE_ALT 8u    /* some alternating word (both, >= 1 a write, D9)   */
#define XPL_PAGE_CPU_W 16u /* some word written by the CPU                     */
#define XPL_PAGE_GPU_W 32u /* some word written by the GPU                     */

/* cudaMemAdvise hints recorded per allocation, as bits: */
#define XPL_ADVICE_READ_MOSTLY 1u
#define XPL_ADVICE_PREFERRED_GPU 2u
#define XPL_ADVICE_PREFERRED_CPU 4u
#define XPL_ADVICE_ACCESSED_BY_GPU 8u
#define XPL_ADVICE_ACCESSED_BY_CPU 16u

/* Page-report flags (managed allocations only, D8 / P:L84): */
#define XPL_PAGE_PAT_FALSE_SHARING 1u   /* a page used by both sides on disjoint words */
#define XPL_PAGE_PAT_ADVICE_MISMATCH 2u /* ReadMostly advised, yet a page alternates (D32) */

typedef struct {
  uint64_t id, base, words, page_words, pages;
  uint32_t kind, advice; /* xpl_alloc_kind; XPL_ADVICE_* bits in force           */
  uint64_t cpu_pages, gpu_pages;
  uint64_t shared_pages;       /* CPU and GPU pages                                 */
  uint64_t false_shared_pages; /* shared pages on which no word was used by both    */
  uint64_t alternating_pages;  /* pages holding an alternating word                 */
  uint32_t flags, pad;         /* XPL_PAGE_PAT_*                                    */
} xpl_page_report;

/* The page view of every live row, in id order, into out[0..cap) (*n_out rows;
 * INVALID_ARG with *n_out = rows needed if cap is too small, or page_words == 0).
 * Reads the interval bits without changing them: call it before the resetting
 * diagnose of the interval.  STATE inside an open epoch, or in sharded mode.
 * Blocks until done. */
xpl_status xpl_page_summary(xpl_ctx* ctx, uint64_t page_words, xpl_page_report* out, size_t cap,
                            size_t* n_out);

/* The page bits (XPL_PAGE_*) of the live row whose base is `base`: out[n_pages],
 * n_pages must be ceil(words / page_words) (else INVALID_ARG).  The page map
 * of Fig. 5-style plots.  Blocks until done. */
xpl_status xpl_page_flags(xpl_ctx* ctx, const void* base, uint64_t page_words, uint8_t* out,
                          uint64_t n_pages);

/* The cudaMemAdvise wrapper: records advice (cudaMemoryAdvise numbering: 1 Set/2
 * Unset ReadMostly, 3 Set/4 Unset PreferredLocation, 5 Set/6 Unset AccessedBy;
 * device < 0 = the CPU) for the allocation holding `ptr`, as a whole (D33).
 * Untracked pointers are ignored.  INVALID_ARG on another advice value. */
xpl_status xpl_mem_advise(xpl_ctx* ctx, const void* ptr, size_t bytes, int advice, int device);

/* ---- Kernel-launch log (traceKernelLaunch) ----
 * The paper's launch wrapper "can be used to ... record data before and after
 * the launch of a CUDA kernel".  With the log on, every launch the
 * instrumented code reports inside an epoch (xpl_kernel_launch, or the
 * xpl_trace_kernel_launch template of xpl_launch.cuh) is kept with its launch
 * parameters, and every epoch gets two measurements taken on the device, in
 * stream order, without synchronising the host: its GPU time (CUDA events from
 * the epoch's begin on its first stream to the end of its fold) and the number
 * of 128-word shadow chunks its fold found GPU-written (the epoch's write
 * footprint).  Off by default; costs three event records and two 8-byte
 * device->host copies per epoch when on. */
typedef struct {
  const char* name; /* kernel name; copied (interned) by the runtime, may be NULL */
  uint32_t grid[3], block[3];
  uint32_t shmem; /* dynamic shared memory bytes */
} xpl_launch_info;

typedef struct {
  uint64_t seq;         /* launch number since the log was enabled/reset (0-based)   */
  uint64_t epoch;       /* epoch number (xpl_stats.epochs counted at its begin)      */
  uint64_t stream;      /* cudaStream_t of the launch, as an integer                 */
  uint32_t grid[3], block[3];
  uint32_t shmem, name_idx; /* name_idx: xpl_launch_name(), UINT32_MAX = none        */
  uint64_t threads;         /* grid x block                                          */
  uint64_t launches_in_epoch;
  uint64_t epoch_written_chunks; /* 128-word chunks the epoch's fold folded: chunks
                                  * holding a word the epoch wrote while its last
                                  * writer was the CPU (D34)                         */
  double epoch_ms;               /* GPU time of the epoch incl. its fold, -1 if n/a  */
} xpl_launch_record;

/* Turn the log on (1) or off (0); either clears it.  Synchronises the device
 * (pending per-epoch copies of the old log).  STATE inside an open epoch. */
xpl_status xpl_launch_log_enable(xpl_ctx* ctx, int enable);
/* Log one launch of the open epoch (call between xpl_kernel_begin and _end,
 * before or after the launch itself).  STATE outside an epoch; INVALID_ARG on
 * a NULL info; a no-op when the log is off. */
xpl_status xpl_kernel_launch(xpl_ctx* ctx, void* stream, const xpl_launch_info* info);
/* The logged launches in order into out[0..cap) (*n_out records; INVALID_ARG
 * with *n_out = records needed if cap is too small).  Waits for the logged
 * epochs' events and copies.  reset != 0 clears the log after reading.  STATE
 * inside an open epoch. */
xpl_status xpl_launch_log(xpl_ctx* ctx, xpl_launch_record* out, size_t cap, size_t* n_out,
                          int reset);
/* The interned kernel name with index idx (owned by the context, valid until
 * xpl_finalize); NULL if idx is out of range. */
const char* xpl_launch_name(xpl_ctx* ctx, uint32_t idx);

/* Apply every staged host record now (normally done lazily at kernel_begin,
 * diagnose and when staging fills up).  Asynchronous.  Sharded mode:
 * COLLECTIVE (the records are routed to their owners). */
xpl_status xpl_flush(xpl_ctx* ctx);
/* Wait for all runtime work enqueued so far.  STATE if a device-side epoch split
 * (xpl_grid_epoch) ran in an epoch with several streams or with D2D / memset
 * shadow work (reported once; the records of that epoch are unreliable). */
xpl_status xpl_sync(xpl_ctx* ctx);
/* The runtime stops using `stream` for its own work (moves it back onto its own
 * stream, ordered after everything enqueued on `stream` so far).  Call before
 * destroying a stream that ended an epoch.  STATE inside an epoch. */
xpl_status xpl_release_stream(xpl_ctx* ctx, void* stream);
/* Make `stream` (cudaStream_t as void*) wait on the device for every runtime
 * operation enqueued so far (host merges, transfers' shadow updates, the last
 * epoch's fold).  Runtime work runs on the runtime's own stream, or on the
 * stream of the last single-stream epoch (its fold directly follows that
 * epoch's kernels there).  No host blocking.  XPL_ERR_STATE inside an epoch. */
xpl_status xpl_join(xpl_ctx* ctx, void* stream);
/* The runtime's own stream (cudaStream_t as void*).  To order work or timing
 * events after the runtime's work, use xpl_join on the stream first. */
xpl_status xpl_runtime_stream(xpl_ctx* ctx, void** stream);
xpl_status xpl_get_stats(xpl_ctx* ctx, xpl_stats* out);

/* Live kernel timing (for the roofline numbers of bench.py): with profiling on,
 * every runtime kernel is bracketed by CUDA events on the runtime stream.
 * xpl_profile_read waits for the runtime stream and returns, per kernel class,
 * the launches, the summed event time and the ALGORITHMIC bytes moved
 * (fold 256 B per written 128-word chunk; merge 8 B per record + 2 B per word;
 * range 2 B per word; diagnose 1 B per word + 1 B per word when resetting;
 * page view 1 B per word). */
typedef enum {
  XPL_K_FOLD = 0,
  XPL_K_MERGE = 1,
  XPL_K_RANGE = 2,
  XPL_K_DIAG_TILE = 3, /* the one-pass shadow kernel of diagnose               */
  XPL_K_DIAGNOSE = 4,  /* the whole diagnose call (all its kernels + copies)   */
  XPL_K_PAGES = 5,     /* the page-view kernel (NEXT-3; 1 B per word read)    */
  XPL_K_NCLASS = 6
} xpl_kernel_class;
typedef struct {
  uint64_t launches;
  double ms;
  uint64_t bytes;
} xpl_kernel_time;
xpl_status xpl_profile(xpl_ctx* ctx, int enable);
xpl_status xpl_profile_read(xpl_ctx* ctx, xpl_kernel_time out[XPL_K_NCLASS], int reset);

const char* xpl_status_string(xpl_status s);

#ifdef __cplusplus
}
#endif
#endif /* XPL_H */
