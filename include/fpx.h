/*
 * fpx.h — C ABI of the B200-native GPU-FPX exception-scan hot path.
 *
 * What this library computes (the method, restated from the paper; "P:<line>"
 * cites /root/reference/PAPER.md, "SURVEY §8" the scope table in SURVEY.md):
 *
 *   GPU-FPX checks, on the device, every executed floating-point instruction:
 *   it classifies the destination value(s) of each active lane as NaN, INF or
 *   subnormal from the IEEE-754 bit pattern (§2.1), reports
 *   division by zero when a MUFU.RCP(64H) destination holds NaN/INF (§3.1.1
 *   P:179, Alg1), and — in the analyzer — tags how an exceptional
 *   value (EV) flows through the instruction (Table 2: Appearance,
 *   Propagation, Disappearance = GEN, PROP, KILL here). Results of a warp are
 *   reduced to a leader and deduplicated in a device table GT keyed by
 *   <E_exce, E_loc, E_fp> (Fig 3 / P:234-244, Alg2) so that only
 *   combinations not seen before are reported to the host,
 *   while GT holds the complete record at the end.
 *
 *   This library runs that check as a streaming scan over *records* of
 *   executed FP instructions (capture by NVBit is out of scope, SURVEY §8 f/OUT)
 *   and over plain FP32/FP64/FP16/BF16 buffers, into a device table whose key
 *   is widened to <site 32b, fmt 2b, flow 2b, kind 2b> and whose value is
 *   (count of lane-values, first record/element index) instead of a 1-bit
 *   "occurred" flag (readings R14, R15 in DESIGN.md).
 *
 * Threading / streams: a handle belongs to one device and is used from one
 * host thread at a time.  Scans are enqueued on the caller's stream and never
 * synchronise; fetch / stats synchronise the stream of the last scan.
 *
 * Error model: argument errors are returned immediately and nothing is
 * enqueued.  Device-side conditions (bad record, table full) are STICKY
 * counters inside the handle: the kernel counts and skips, it never traps;
 * they are reported as the status of the next fpx_table_fetch* call (entries
 * are still written) and readable through fpx_get_stats.
 */
#ifndef FPX_H
#define FPX_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------------ */
/* Status codes                                                              */
/* ------------------------------------------------------------------------ */
typedef enum {
  FPX_OK = 0,
  FPX_ERR_INVALID = -1,     /* bad argument (NULL handle, misaligned pointer, bad enum) */
  FPX_ERR_CUDA = -2,        /* a CUDA runtime call failed (see fpx_last_cuda_error) */
  FPX_ERR_NOMEM = -3,       /* device or host allocation failed */
  FPX_ERR_TABLE_FULL = -4,  /* sticky: an insert found no free slot; events dropped */
  FPX_ERR_BAD_RECORD = -5,  /* sticky: >=1 record failed validation and was skipped */
  FPX_ERR_TRUNCATED = -6    /* fetch: capacity < n_total; first `capacity` entries written */
} fpx_status;

/* ------------------------------------------------------------------------ */
/* Enumerations (values are part of the ABI and of the table key)            */
/* ------------------------------------------------------------------------ */

/* E_fp, Fig 3 / P:240: "up to four FP formats". */
enum { FPX_FP32 = 0, FPX_FP64 = 1, FPX_FP16 = 2, FPX_BF16 = 3 };

/* E_exce: NaN, INF, SUB (subnormal), DIV0. */
enum { FPX_NAN = 0, FPX_INF = 1, FPX_SUB = 2, FPX_DIV0 = 3 };

/* Flow tag, Table 2 P:421-433.  NONE = detector (destination-only) result;
 * GEN = Appearance (dest EV, no source EV); PROP = Propagation (dest EV and a
 * source EV); KILL = Disappearance (no dest EV, a source EV; also compare /
 * select / min-max that consume an EV, Listing 4). */
enum { FPX_FLOW_NONE = 0, FPX_GEN = 1, FPX_PROP = 2, FPX_KILL = 3 };

/* Scan modes: the detector (dest-only, §3.1) and the analyzer (flow, §3.2);
 * the two-phase workflow of Fig 2 / P:167, 230.  FPX_MODE_FLOW_DETAIL is the
 * analyzer plus Table 2's separate "Comparison" state and per-source
 * attribution (fn4 P:99 "INF flowed from R3 to R1"): entries
 * also carry `detail` (below). */
enum { FPX_MODE_DEST = 0, FPX_MODE_FLOW = 1, FPX_MODE_FLOW_DETAIL = 2 };

/* detail byte of an entry (0 outside FPX_MODE_FLOW_DETAIL):
 *   bits [1:0]  1 + index of the source operand that set the source class S
 *               (the lowest-index source with the most severe class), 0 if no
 *               source was exceptional;
 *   bit 2       FPX_DETAIL_CMP: the instruction is a control-flow opcode
 *               (Table 1's right column: FSEL, FSET, FSETP, FMNMX, DSETP) and a
 *               source was exceptional — Table 2's "Comparison" state. */
#define FPX_DETAIL_SRC(d) ((uint32_t)(d) & 3u)
#define FPX_DETAIL_CMP 4u

/* Opcode classes (Table 1; Alg1 dispatch; SASS opcode -> opcode_id
 * map of P:332).  HADD2..HMMA are the FP16/BF16 "future" formats;
 * DIV is a synthetic IEEE divide used by producers that record a whole
 * division rather than its MUFU.RCP expansion. */
enum {
  FPX_OP_OTHER = 0,
  FPX_OP_FADD = 1, FPX_OP_FMUL = 2, FPX_OP_FFMA = 3,
  FPX_OP_MUFU_RCP = 4, FPX_OP_MUFU_RCP64H = 5, FPX_OP_MUFU_OTHER = 6,
  FPX_OP_DADD = 7, FPX_OP_DMUL = 8, FPX_OP_DFMA = 9,
  FPX_OP_FSEL = 10, FPX_OP_FSET = 11, FPX_OP_FSETP = 12, FPX_OP_FMNMX = 13,
  FPX_OP_DSETP = 14,
  FPX_OP_HADD2 = 15, FPX_OP_HFMA2 = 16, FPX_OP_HMUL2 = 17, FPX_OP_HMMA = 18,
  FPX_OP_DIV = 19,
  FPX_OP_COUNT = 20
};

/* Fetch flags. */
enum { FPX_FETCH_ALL = 0, FPX_FETCH_NEW = 1 };

/* ------------------------------------------------------------------------ */
/* Record layout (the input of fpx_scan_records)                             */
/* ------------------------------------------------------------------------ */
/*
 * One record = one executed FP SASS instruction of one warp (the unit the
 * paper's injected code sees, Alg2).  Records are an array of
 * 16-byte headers plus an "arena" of 128-byte planes; a plane is one 32-bit
 * register word for all 32 lanes (lane l at byte 4*l), i.e. exactly the
 * register-granular view of P:151-155.
 *
 *   site        E_loc widened to 32 bits: kernel id + SASS offset, as
 *               assigned by the producer.  0xFFFFFFFF is reserved (bad record).
 *   active_mask bit l set = lane l executed the instruction.  Inactive lanes
 *               are ignored entirely (their plane words may hold garbage).
 *   meta        bits [7:0]   opclass (FPX_OP_*, < FPX_OP_COUNT)
 *               bits [9:8]   fmt (FPX_FP32..FPX_BF16)
 *               bits [11:10] nsrc, number of source operands (0..3)
 *               bits [14:12] dwords, 32-bit words per lane of the destination
 *                            (0..4); 0 = no FP destination (FSETP/DSETP/FSET)
 *               bits [31:15] reserved, must be 0
 *   val_off     index (in planes) of the record's first plane in the arena.
 *
 * Planes of a record, in order, starting at arena[val_off]:
 *   dest word 0 .. dwords-1, then for each source k < nsrc: sw words,
 *   sw = 2 for FP64 and 1 otherwise.
 *   FP64 values: word 2i = low half (R_d), word 2i+1 = high half (R_{d+1});
 *   the producer resolves the "64H" pairing (R_{d-1}, R_d) of Alg1 lines 3-4
 *   and 12-13 into this (lo, hi) order.
 *   FP16/BF16: each 32-bit word packs two values, low half first.
 *   Sources hold PRE-execution values (shared dest/src registers);
 *   immediates / constant-bank operands are broadcast planes.
 *
 * Values per lane of the destination: FP32 dwords, FP64 dwords/2 (dwords must
 * be even), FP16/BF16 2*dwords.
 */
typedef struct {
  uint32_t site;
  uint32_t active_mask;
  uint32_t meta;
  uint32_t val_off;
} fpx_rec_hdr;

#define FPX_META(opclass, fmt, nsrc, dwords) \
  ((uint32_t)(opclass) | ((uint32_t)(fmt) << 8) | ((uint32_t)(nsrc) << 10) | ((uint32_t)(dwords) << 12))

#define FPX_SITE_INVALID 0xFFFFFFFFu

/* ------------------------------------------------------------------------ */
/* Table key and entries                                                     */
/* ------------------------------------------------------------------------ */
/* key = site << 32 | detail << 6 | fmt << 4 | flow << 2 | kind.  Ascending
 * key order = (site, detail, fmt, flow, kind) order; fetch always returns
 * entries in this order (detail is 0 except in FPX_MODE_FLOW_DETAIL). */
#define FPX_KEY(site, fmt, flow, kind) \
  (((uint64_t)(site) << 32) | ((uint64_t)(fmt) << 4) | ((uint64_t)(flow) << 2) | (uint64_t)(kind))
#define FPX_KEY_DETAIL(site, detail, fmt, flow, kind) (FPX_KEY(site, fmt, flow, kind) | ((uint64_t)(detail) << 6))
#define FPX_KEY_EMPTY 0xFFFFFFFFFFFFFFFFull

typedef struct {
  uint32_t site;
  uint8_t kind;          /* FPX_NAN..FPX_DIV0 */
  uint8_t flow;          /* FPX_FLOW_NONE..FPX_KILL */
  uint8_t fmt;           /* FPX_FP32..FPX_BF16 */
  uint8_t detail;        /* FPX_MODE_FLOW_DETAIL attribution, else 0 */
  uint64_t count;        /* number of lane-values with this key */
  uint64_t first_index;  /* min base_index + record (or element) index */
} fpx_entry;             /* 24 bytes */

/* ------------------------------------------------------------------------ */
/* Handle, options, stats                                                    */
/* ------------------------------------------------------------------------ */
typedef struct fpx_ctx* fpx_handle;

typedef struct {
  uint32_t table_log2_slots;  /* 0 = default 20 (2^20 slots x 32 B = 32 MiB, L2-sized); valid 4..30 */
  uint32_t newlog_capacity;   /* 0 = default (= number of slots) */
  uint32_t flags;             /* 0, or FPX_OPT_* below (ablations) */
} fpx_options;

/* Option flags.  FPX_OPT_LIVE_NEW enables early notification (fpx_poll_new
 * below).  FPX_OPT_STORM always runs the record scan's storm kernel (a
 * shared-memory pre-aggregation of the table updates per CTA; every tile
 * straight to the exact path while a storm lasts); without it a DEST scan
 * uses that kernel when the handle's previous scan sent at least a quarter
 * of its tiles to the exact path — the table is the same either way.  The
 * other two are ablations that compute the same table:
 * FPX_OPT_SCAN_LDG selects the register-staged LDG record-scan kernel instead
 * of the default TMA (cp.async.bulk) shared-memory ring.
 * FPX_OPT_NO_WARP_AGG turns off warp aggregation (Alg2) in the
 * record scans' exact path: every lane issues its own table updates, one per
 * distinct code it holds (SURVEY §8(d) stress ablation; record scans only). */
enum { FPX_OPT_SCAN_LDG = 1, FPX_OPT_NO_WARP_AGG = 2, FPX_OPT_LIVE_NEW = 4, FPX_OPT_STORM = 8 };

typedef struct {
  uint64_t bad_records;       /* records skipped by validation (sticky, cumulative) */
  uint64_t dropped_events;    /* lane-values lost because the table was full */
  uint64_t table_entries;     /* distinct keys currently in the table */
  uint64_t newlog_overflow;   /* inserts not logged because the new-key log was full */
} fpx_stats;

/* Create a context on `device` (cudaSetDevice is called; the caller's current
 * device is restored).  Allocates the table (32 B per slot), the new-key log
 * (8 B per entry) and fetch scratch, and clears them.  opt may be NULL.
 * Errors: FPX_ERR_INVALID (out==NULL, bad options), FPX_ERR_NOMEM, FPX_ERR_CUDA. */
fpx_status fpx_open(int device, const fpx_options* opt, fpx_handle* out);

/* Enqueue the record scan on `stream` (cudaStream_t; NULL
 * = legacy default stream).
 *   d_hdr      device pointer to n_records headers (16-B aligned), caller-owned
 *   d_arena    device pointer to arena_planes planes of 128 B (16-B aligned)
 *   base_index global index of d_hdr[0]; record r reports first_index
 *              base_index + r (lets a stream be scanned in batches / shards)
 *   mode       FPX_MODE_DEST (detector), FPX_MODE_FLOW (analyzer) or
 *              FPX_MODE_FLOW_DETAIL (analyzer + Comparison state + source)
 * Every lane-value of every active lane is classified; per warp the events
 * are reduced before any atomic; the table gets count += lane-values,
 * first = min(first, base_index + r).  Records that fail validation (reserved
 * bits, enum ranges, planes outside the arena, invalid site, and in the FLOW
 * modes records other than scalar FP32/FP64) are counted and skipped.
 * n_records == 0 is a no-op.  Buffers must stay valid until the stream passes
 * the scan.  Large scans balance work across warps with two device counters
 * owned by the handle; a handle keeps 64 counter pairs and hands them out in
 * turn, so at most 64 record scans of one handle may be in flight at once on
 * different streams (scans on one stream are always safe).  Errors:
 * FPX_ERR_INVALID, FPX_ERR_CUDA. */
fpx_status fpx_scan_records(fpx_handle h, const fpx_rec_hdr* d_hdr, uint64_t n_records,
                            const uint32_t* d_arena, uint64_t arena_planes,
                            uint64_t base_index, uint32_t mode, void* stream);

/* Enqueue a destination-only scan of a contiguous buffer of
 * n_elems values of format fmt, all attributed to `site`; element i reports
 * first_index base_index + i.  Any alignment of d_ptr to the element size is
 * accepted (misaligned heads/tails are handled).  Errors: FPX_ERR_INVALID,
 * FPX_ERR_CUDA. */
fpx_status fpx_scan_tensor(fpx_handle h, const void* d_ptr, uint64_t n_elems, uint32_t fmt,
                           uint32_t site, uint64_t base_index, void* stream);

/* Many tensors in ONE launch (e.g. every module output of a forward pass, the
 * activation detector of SURVEY §8 f1): descs[i] is scanned exactly as
 * fpx_scan_tensor(h, ptr, n_elems, fmt, site, base_index) would.  descs is
 * host memory (copied before the call returns); the device pointers must stay
 * valid until the stream passes the scan.  n == 0 is a no-op.  Errors:
 * FPX_ERR_INVALID (bad fmt / alignment in any descriptor: nothing is
 * enqueued), FPX_ERR_NOMEM, FPX_ERR_CUDA. */
typedef struct {
  const void* ptr;       /* device pointer, aligned to the element size */
  uint64_t n_elems;
  uint64_t base_index;
  uint32_t fmt;          /* FPX_FP32..FPX_BF16 */
  uint32_t site;
} fpx_tensor_desc;       /* 32 bytes */

fpx_status fpx_scan_tensors(fpx_handle h, const fpx_tensor_desc* descs, uint32_t n, void* stream);

/* Synchronise the last scan's stream and copy entries, ascending by key, into
 * caller-allocated host memory.  flags = FPX_FETCH_ALL: every entry;
 * FPX_FETCH_NEW: only keys first inserted since the previous FETCH_NEW call
 * (the paper's "only push new combinations", served from the device
 * new-key log).  *n_total receives the number of entries available (FETCH_NEW:
 * the number of new keys not yet returned).  If capacity < *n_total the first
 * `capacity` are written and FPX_ERR_TRUNCATED is returned — FETCH_ALL: the
 * first in key order; FETCH_NEW: the first `capacity` new keys in insertion
 * order (sorted by key among themselves), and only those count as returned,
 * so the next FETCH_NEW call continues with the rest (capacity 0 only
 * queries).  Otherwise the sticky device status (FPX_ERR_TABLE_FULL before
 * FPX_ERR_BAD_RECORD) or FPX_OK.  host_out may be NULL when capacity == 0. */
fpx_status fpx_table_fetch(fpx_handle h, fpx_entry* host_out, uint64_t capacity,
                           uint64_t* n_total, uint32_t flags);

/* Device-side fetch for the multi-GPU merge: writes the table's keys (sorted
 * ascending), counts and first indices to caller-owned device arrays on
 * `stream`, then synchronises it to return *n_total.  Same truncation /
 * sticky-status rules as fpx_table_fetch. */
fpx_status fpx_table_fetch_device(fpx_handle h, uint64_t* d_keys, uint64_t* d_counts,
                                  uint64_t* d_first, uint64_t capacity, uint64_t* n_total,
                                  void* stream);

/* For every key d_keys[i] (i < n; FPX_KEY_EMPTY allowed as padding) write
 * this table's count (0 if absent) and first index (INT64_MAX if absent — the
 * int64 sentinel lets NCCL MIN-reduce it as signed) to d_counts[i], d_first[i].
 * This is the dense-scatter step of the NCCL merge (SURVEY §8 e). Async. */
fpx_status fpx_table_lookup_device(fpx_handle h, const uint64_t* d_keys, uint64_t n,
                                   uint64_t* d_counts, uint64_t* d_first, void* stream);

/* Sort-unique n device keys (in place semantics: result in d_out, which may
 * alias d_keys), dropping FPX_KEY_EMPTY; writes the number of unique keys to
 * *n_out (synchronises `stream`).  Union step of the merge. */
fpx_status fpx_keys_unique_device(fpx_handle h, const uint64_t* d_keys, uint64_t n,
                                  uint64_t* d_out, uint64_t* n_out, void* stream);

/* Add n (key, count, first) triples into the table (count added, first
 * min-ed, keys inserted and logged as new if absent).  Re-imports a fetched
 * or merged table (checkpoint/resume).  Async. */
fpx_status fpx_table_merge_device(fpx_handle h, const uint64_t* d_keys, const uint64_t* d_counts,
                                  const uint64_t* d_first, uint64_t n, void* stream);

/* Clear the table, the new-key log, its cursor and the sticky counters
 * (async on `stream`). */
fpx_status fpx_table_reset(fpx_handle h, void* stream);

/* Early notification, without waiting for scans (§3.1.2: new
 * exceptions are pushed to the host so that users are alerted "before
 * (hour-long) GPU runs finish").  On a handle opened with FPX_OPT_LIVE_NEW,
 * the thread whose insert creates a key also publishes it to a ring in mapped
 * pinned host memory (one 32-B slot per new-key-log position; capacity =
 * newlog_capacity).  fpx_poll_new copies the keys published since the previous
 * poll, in insertion order, into host_out (at most `capacity`; *n_out = number
 * written) and returns at once: it calls no CUDA API and synchronises no
 * stream, so it may run while scans are in flight.  A polled entry's key
 * (site, kind, flow, fmt, detail) is final; its count and first_index are
 * those of the event that inserted the key (provisional: fpx_table_fetch
 * gives the final values once the scans are done).  fpx_table_reset restarts
 * the ring.  Keys first inserted by another process's attached handle
 * (fpx_open_attached) are not published here (FETCH_NEW still reports them).
 * Latency: the sparse record kernels, the tensor scans and the analyzer
 * modes insert (and publish) a key as soon as a warp finds it; the storm
 * kernel (FPX_OPT_STORM, or picked after a storm) pre-aggregates per CTA and
 * inserts a key when the CTA that found it finishes, within the same launch.
 * This poll cursor is independent of FPX_FETCH_NEW's.  A handle is used from
 * one host thread at a time, polls included.  Errors: FPX_ERR_INVALID (no
 * FPX_OPT_LIVE_NEW, NULL arguments). */
fpx_status fpx_poll_new(fpx_handle h, fpx_entry* host_out, uint64_t capacity, uint64_t* n_out);

/* Synchronise and read the sticky counters. */
fpx_status fpx_get_stats(fpx_handle h, fpx_stats* out);

/* ------------------------------------------------------------------------ */
/* Shared table across processes / GPUs (SURVEY §5, §8 e alternative)       */
/* ------------------------------------------------------------------------ */
/* One device table that scans on other GPUs update in place through CUDA IPC
 * peer mappings (NVLink / NVSwitch on a B200 box: remote atomicCAS / Add /
 * Min), so a multi-GPU scan needs no merge step: the home handle's table is
 * the union.  Events are rare (the fast path never touches the table), so the
 * remote traffic is a few atomics per exceptional warp-record.
 *
 * fpx_table_export: describe the handle's table (slots, new-key log, counters)
 * as CUDA IPC handles; *out is plain bytes to pass to other processes.
 * fpx_open_attached: open a handle on `device` (in another process) whose
 * scans update the exported table.  Attached handles may scan, fetch and read
 * stats (peer reads); fpx_table_reset is the home handle's job.  Ordering
 * across processes is the caller's: synchronise the scanning streams and
 * barrier before the home fetch.  Errors: FPX_ERR_INVALID, FPX_ERR_CUDA (e.g.
 * no IPC / peer access between the devices). */
typedef struct {
  unsigned char ipc[4][64];   /* cudaIpcMemHandle_t: slots, newlog, newlog_slot, ctl */
  uint32_t table_log2_slots;
  uint32_t newlog_capacity;
  int32_t home_device;
  uint32_t magic;             /* FPX_IPC_MAGIC */
} fpx_ipc_table;
#define FPX_IPC_MAGIC 0x46505831u /* "FPX1" */

fpx_status fpx_table_export(fpx_handle h, fpx_ipc_table* out);
fpx_status fpx_open_attached(int device, const fpx_ipc_table* table, fpx_handle* out);

/* Free everything owned by the handle (synchronises the device first).  An
 * attached handle unmaps the shared table; the home handle frees it. */
fpx_status fpx_close(fpx_handle h);

/* Static string for a status code. */
const char* fpx_strerror(fpx_status s);

/* Last CUDA error string seen by any call in this process ("" if none). */
const char* fpx_last_cuda_error(void);

/* ABI self-description for bindings: sizeof(fpx_rec_hdr), sizeof(fpx_entry),
 * library version.  Never fails. */
uint32_t fpx_abi_version(void);
uint32_t fpx_sizeof_rec_hdr(void);
uint32_t fpx_sizeof_entry(void);

#ifdef __cplusplus
}
#endif

#endif /* FPX_H */
