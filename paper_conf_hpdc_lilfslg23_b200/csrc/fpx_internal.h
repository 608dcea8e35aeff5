// fpx_internal.h — types shared by the C-ABI layer and the sm_100a kernels.
//
// Device state of one handle:
//   table   2^k slots x 32 B {key, count, first, pad}: one L2 sector per slot,
//           open addressing with linear probing (the paper's GT, P:223, 236-244,
//           widened per readings R14/R15)
//   newlog  append-only log of keys in insertion order (the paper's
//           "push only new combinations to the host", P:244 / Alg2 P:271-273,
//           read at fetch instead of through a GPU->CPU channel)
//   ctl     sticky counters (bad records, dropped events, log tail, overflow)
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "fpx.h"

namespace fpx {

struct alignas(32) Slot {
  unsigned long long key;    // FPX_KEY_EMPTY when free
  unsigned long long count;  // lane-values with this key
  unsigned long long first;  // min global record / element index
  unsigned long long pad;
};
static_assert(sizeof(Slot) == 32, "slot = one 32-B L2 sector");

struct LiveSlot;
struct alignas(64) Ctl {
  unsigned long long bad_records;
  unsigned long long dropped_events;
  unsigned long long newlog_tail;      // number of inserts ever (= table entries)
  unsigned long long newlog_overflow;
  LiveSlot* live;                      // device view of the live ring (TV_LIVE handles only)
  unsigned long long live_gen;         // its generation, set by every reset
  unsigned long long pad[2];
};

// Early notification ring (FPX_OPT_LIVE_NEW): one slot per new-key-log
// position, in mapped pinned HOST memory.  The thread that inserts a key
// writes key / count / first, fences at system scope, then publishes
// seq = gen << 32 | (position + 1); the host polls seq in log order without
// synchronising any stream (fpx_poll_new).  gen changes at every table reset
// so slots of an earlier table are never taken for new ones.
struct alignas(32) LiveSlot {
  unsigned long long key;
  unsigned long long first;  // index of the inserting event (provisional first)
  unsigned long long count;  // lane-values of the inserting event (provisional count)
  unsigned long long seq;
};
static_assert(sizeof(LiveSlot) == 32, "live slot is 32 B");

// TableView::flags bit: the table is shared with other GPUs / processes
// (fpx_table_export on the home handle, fpx_open_attached on the others), so
// its atomics run at system scope (fpx_device.cuh t_cas / t_add / t_min).
constexpr uint32_t TV_SHARED = 1u << 16;
// TableView::flags bit: this handle publishes new keys to its live ring
// (ctl->live; FPX_OPT_LIVE_NEW on the home handle; never on attached ones,
// whose process cannot see the home's host ring).
constexpr uint32_t TV_LIVE = 1u << 17;
// TableView::flags bit, set per launch by the sparse record-scan kernels'
// launcher: table_add tries the key's home slot with the CAS straight away
// (most of their events are new keys); storm kernels, whose events mostly hit
// present hot keys, and the per-lane ablation read the slot first.
constexpr uint32_t TV_CAS_FIRST = 1u << 18;

// Everything a scan kernel needs to update the table, passed by value.
struct TableView {
  Slot* slots;
  unsigned long long mask;       // slots - 1
  unsigned long long* newlog;
  unsigned int* newlog_slot;     // slot index of each logged key (for the touched-slot reset)
  unsigned long long newlog_cap;
  Ctl* ctl;
  uint32_t flags;                // FPX_OPT_NO_WARP_AGG (ablation) | TV_SHARED | TV_LIVE | TV_CAS_FIRST
};

// One tensor of a fused multi-tensor scan (host-prepared, device-resident).
struct alignas(16) ListEntry {
  const uint8_t* ptr;   // tensor base
  uint64_t base;        // first_index of element 0
  uint64_t vbegin;      // first body vector of this tensor in the launch
  uint64_t sbegin;      // first head/tail scalar of this tensor in the launch
  uint64_t nvec;        // 16-B body vectors (starting after `head` elements)
  uint32_t head, tail;  // scalars before / after the aligned body
  uint32_t fmt, site;
};
static_assert(sizeof(ListEntry) == 64, "list entry is 64 B");

// Density feedback of the record scan (mapped pinned host memory, one per
// handle): the last warp of a launch with a dynamic tail writes the launch's
// hit tiles (tiles that took the exact path) and record count; the launcher
// reads it, without synchronising, to pick the storm kernel for the next
// launch of the handle.
struct ScanFeedback {
  unsigned long long hit_tiles;
  unsigned long long records;
};
struct FeedbackPtrs {
  unsigned long long* dev;  // device accumulator (zeroed again by the last warp), or nullptr
  ScanFeedback* host;       // device view of the mapped host struct
};

// ---- launchers (fpx_scan_records.cu, fpx_scan_tensor.cu, fpx_table.cu) --------------------------------
// variant 0 = TMA ring (default), 1 = register-staged LDG (FPX_OPT_SCAN_LDG ablation).
// sched_ctr: two zeroed u32 counters of the TMA kernel's dynamic tail, left
// zeroed again when the launch completes (nullptr: static ranges only).
// storm: launch the DEST storm instantiation (CTA pre-aggregation, storm mode).
cudaError_t launch_scan_records(const fpx_rec_hdr* d_hdr, uint64_t n, const uint32_t* d_arena,
                                uint64_t arena_planes, uint64_t base_index, uint32_t mode,
                                const TableView& tv, int num_sms, uint32_t variant, unsigned int* sched_ctr,
                                const FeedbackPtrs& fbp, bool storm, cudaStream_t s);
cudaError_t launch_scan_tensor(const void* d_ptr, uint64_t n_elems, uint32_t fmt, uint32_t site,
                               uint64_t base_index, const TableView& tv, int num_sms, cudaStream_t s);
cudaError_t launch_scan_tensor_list(const ListEntry* d_entries, uint32_t n, uint64_t total_vec,
                                    uint64_t total_scalar, const TableView& tv, int num_sms, cudaStream_t s);
// Both resets also (re)write ctl->live / live_gen (the early-notification ring).
cudaError_t launch_table_reset(const TableView& tv, uint64_t slots, LiveSlot* live, uint32_t live_gen, cudaStream_t s);
// Clear only the slots recorded in the new-key log (every occupied slot is
// there unless the log overflowed, in which case the whole table is cleared),
// then the counters.  O(entries) instead of O(slots); stream-ordered, no sync.
cudaError_t launch_table_reset_touched(const TableView& tv, uint64_t slots, LiveSlot* live, uint32_t live_gen,
                                      cudaStream_t s);
// Compact non-empty slots into (keys, counts, firsts); *d_n receives the count.
cudaError_t launch_table_compact(const TableView& tv, uint64_t slots, uint64_t* d_keys,
                                 uint64_t* d_counts, uint64_t* d_first, unsigned long long* d_n,
                                 cudaStream_t s);
// Look keys up: count (0 if absent) and first (INT64_MAX if absent).
cudaError_t launch_table_lookup(const TableView& tv, const uint64_t* d_keys, uint64_t n,
                                uint64_t* d_counts, uint64_t* d_first, cudaStream_t s);
cudaError_t launch_table_merge(const TableView& tv, const uint64_t* d_keys, const uint64_t* d_counts,
                               const uint64_t* d_first, uint64_t n, cudaStream_t s);
// Radix-sort keys (with a permutation of 0..n-1 as values); temp via cub.
cudaError_t sort_keys_with_index(void* d_temp, size_t* temp_bytes, const uint64_t* d_keys_in,
                                 uint64_t* d_keys_out, const uint64_t* d_idx_in, uint64_t* d_idx_out,
                                 uint64_t n, cudaStream_t s);
cudaError_t launch_iota(uint64_t* d, uint64_t n, cudaStream_t s);
cudaError_t launch_gather3(const uint64_t* d_idx, uint64_t n, const uint64_t* c_in, const uint64_t* f_in,
                           uint64_t* c_out, uint64_t* f_out, cudaStream_t s);
cudaError_t unique_keys(void* d_temp, size_t* temp_bytes, const uint64_t* d_in, uint64_t* d_out,
                        unsigned long long* d_nout, uint64_t n, cudaStream_t s);

}  // namespace fpx
