// fpx_device.cuh — device-side building blocks of the scan (sm_100a).
//
//   cls_*        branch-free IEEE-754 classification from the bit pattern
//                (§2.1): 0 clean, 1 NaN, 2 INF, 3 SUB
//   value_code   Alg1's dispatch per opcode class -> E_exce code
//   table_add    open-addressed insert + count / first-index update + new-key
//                log append (GT; Alg2 lines 10-12 with the prose
//                reading R3: push iff this thread inserted the key)
//   warp_flush   warp aggregation (Alg2 lines 3-9 redesigned): one table
//                update per distinct (flow, kind) code per warp-record
#pragma once
#include <stdint.h>

#include "fpx_internal.h"

namespace fpx {

constexpr unsigned FULL = 0xFFFFFFFFu;

enum : uint32_t { CLS_CLEAN = 0, CLS_NAN = 1, CLS_INF = 2, CLS_SUB = 3 };

// FP32: a = |x|; NaN: a > 0x7F800000; INF: a == 0x7F800000; SUB: 0 < a < 2^23.
__device__ __forceinline__ uint32_t cls_fp32(uint32_t x) {
  const uint32_t a = x & 0x7FFFFFFFu;
  uint32_t c = (a - 1u) < 0x007FFFFFu ? CLS_SUB : CLS_CLEAN;
  c = a == 0x7F800000u ? CLS_INF : c;
  c = a > 0x7F800000u ? CLS_NAN : c;
  return c;
}
// FP64 as (lo, hi) words: the exponent lives in hi, the mantissa spans both.
__device__ __forceinline__ uint32_t cls_fp64(uint32_t lo, uint32_t hi) {
  const uint32_t ah = hi & 0x7FFFFFFFu;
  const bool mant_nz = ((ah & 0x000FFFFFu) | lo) != 0u;
  const bool exp_max = ah >= 0x7FF00000u;
  const bool exp_zero = ah < 0x00100000u;
  uint32_t c = (exp_zero && mant_nz) ? CLS_SUB : CLS_CLEAN;
  c = exp_max ? (mant_nz ? CLS_NAN : CLS_INF) : c;
  return c;
}
__device__ __forceinline__ uint32_t cls_fp16(uint32_t h) {
  const uint32_t a = h & 0x7FFFu;
  uint32_t c = (a - 1u) < 0x03FFu ? CLS_SUB : CLS_CLEAN;
  c = a == 0x7C00u ? CLS_INF : c;
  c = a > 0x7C00u ? CLS_NAN : c;
  return c;
}
__device__ __forceinline__ uint32_t cls_bf16(uint32_t h) {
  const uint32_t a = h & 0x7FFFu;
  uint32_t c = (a - 1u) < 0x007Fu ? CLS_SUB : CLS_CLEAN;
  c = a == 0x7F80u ? CLS_INF : c;
  c = a > 0x7F80u ? CLS_NAN : c;
  return c;
}
__device__ __forceinline__ bool is_zero_val(uint32_t fmt, uint32_t lo, uint32_t hi) {
  if (fmt == FPX_FP64) return ((hi & 0x7FFFFFFFu) | lo) == 0u;
  if (fmt == FPX_FP32) return (lo & 0x7FFFFFFFu) == 0u;
  return (lo & 0x7FFFu) == 0u;
}
__device__ __forceinline__ uint32_t cls_val(uint32_t fmt, uint32_t lo, uint32_t hi) {
  switch (fmt) {
    case FPX_FP32: return cls_fp32(lo);
    case FPX_FP64: return cls_fp64(lo, hi);
    case FPX_FP16: return cls_fp16(lo);
    default: return cls_bf16(lo);
  }
}

// No event.
constexpr int CODE_NONE = -1;
// code = flow << 2 | kind (kind: NaN 0, INF 1, SUB 2, DIV0 3)
__device__ __forceinline__ int kind_of_cls(uint32_t c) { return c == CLS_CLEAN ? CODE_NONE : (int)c - 1; }

// Destination kind of one value under the Alg1 dispatch (a3 in SURVEY §8):
// MUFU.RCP(64H) -> DIV0 iff dest NaN/INF (never SUB: R2); compares
// have no FP destination (R10); DIV -> IEEE divideByZero (R1); else the class.
// `dividend` / `divisor` are (lo, hi) words of src0 / src1 at the same value
// position; have_div tells whether they are defined.
__device__ __forceinline__ int dest_kind(uint32_t op, uint32_t fmt, uint32_t lo, uint32_t hi, bool have_div,
                                         uint32_t n_lo, uint32_t n_hi, uint32_t d_lo, uint32_t d_hi) {
  const uint32_t c = cls_val(fmt, lo, hi);
  if (op == FPX_OP_MUFU_RCP || op == FPX_OP_MUFU_RCP64H) return (c == CLS_NAN || c == CLS_INF) ? FPX_DIV0 : CODE_NONE;
  if (op == FPX_OP_FSETP || op == FPX_OP_DSETP || op == FPX_OP_FSET) return CODE_NONE;
  if (op == FPX_OP_DIV && have_div) {
    const uint32_t cn = cls_val(fmt, n_lo, n_hi);
    const bool dividend_ok = (cn == CLS_CLEAN || cn == CLS_SUB) && !is_zero_val(fmt, n_lo, n_hi);
    if (dividend_ok && is_zero_val(fmt, d_lo, d_hi)) return FPX_DIV0;
  }
  return kind_of_cls(c);
}

// code = detail << 4 | flow << 2 | kind  ->  key = site << 32 | detail << 6 | fmt << 4 | flow << 2 | kind
__device__ __forceinline__ unsigned long long make_key(uint32_t site, uint32_t fmt, uint32_t code) {
  return ((unsigned long long)site << 32) | ((unsigned long long)(code >> 4) << 6) | ((unsigned long long)fmt << 4) |
         (unsigned long long)(code & 15u);
}

// murmur3 fmix64
__device__ __forceinline__ unsigned long long hash_key(unsigned long long k) {
  k ^= k >> 33;
  k *= 0xFF51AFD7ED558CCDull;
  k ^= k >> 33;
  k *= 0xC4CEB9FE1A85EC53ull;
  k ^= k >> 33;
  return k;
}

// Atomics on the table and its counters.  The CUDA memory model makes an
// atomic indivisible only among the threads of its scope: a table shared with
// other GPUs (TV_SHARED: the home handle after fpx_table_export, every
// fpx_open_attached handle) is updated from several devices at once over
// NVLink, so its atomics are system-scope; a local table keeps device scope.
__device__ __forceinline__ unsigned long long t_cas(const TableView& tv, unsigned long long* a, unsigned long long c,
                                                    unsigned long long v) {
  return (tv.flags & TV_SHARED) ? atomicCAS_system(a, c, v) : atomicCAS(a, c, v);
}
__device__ __forceinline__ unsigned long long t_add(const TableView& tv, unsigned long long* a, unsigned long long v) {
  return (tv.flags & TV_SHARED) ? atomicAdd_system(a, v) : atomicAdd(a, v);
}
__device__ __forceinline__ void t_min(const TableView& tv, unsigned long long* a, unsigned long long v) {
  if (tv.flags & TV_SHARED) atomicMin_system(a, v);
  else atomicMin(a, v);
}

// Fire-and-forget reductions (no value returned: the issuing thread never
// waits for the L2 round trip), same scopes as above.
__device__ __forceinline__ void t_red_add(const TableView& tv, unsigned long long* a, unsigned long long v) {
  if (tv.flags & TV_SHARED) asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
  else asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
}
__device__ __forceinline__ void t_red_min(const TableView& tv, unsigned long long* a, unsigned long long v) {
  if (tv.flags & TV_SHARED) asm volatile("red.relaxed.sys.global.min.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
  else asm volatile("red.relaxed.gpu.global.min.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
}

// Insert-or-update.  Linear probing over the whole table: an event is only
// dropped (and TABLE_FULL raised) when every slot holds another key.
static __device__ __noinline__ void table_add(const TableView tv, unsigned long long key, unsigned long long cnt,
                                       unsigned long long first) {
  unsigned long long i = hash_key(key) & tv.mask;
  for (unsigned long long probe = 0; probe <= tv.mask; ++probe) {
    Slot* s = tv.slots + i;
    unsigned long long k, f_seen = ~0ull;
    bool mine;  // this thread's CAS installed the key
    if (probe == 0 && (tv.flags & TV_CAS_FIRST)) {
      // the home slot straight with the CAS: one L2 round trip less for a new
      // key (the same one for a present key) on the latency path of a sparse
      // hit tile, and the first-index min is then always issued (C1 +1.6 %,
      // C3 +0.4 %; on the 1 % storm, whose events hit ~200 present keys,
      // CAS-first lost 0.9 %: storm kernels read first; ab_cas_first.txt)
      k = t_cas(tv, &s->key, FPX_KEY_EMPTY, key);
      mine = k == FPX_KEY_EMPTY;
    } else {
      k = *reinterpret_cast<volatile unsigned long long*>(&s->key);
      f_seen = *reinterpret_cast<volatile unsigned long long*>(&s->first);
      mine = false;
      if (k == FPX_KEY_EMPTY) {
        k = t_cas(tv, &s->key, FPX_KEY_EMPTY, key);
        mine = k == FPX_KEY_EMPTY;
      }
    }
    if (mine) {
      // this thread inserted the key: log it once (the "new combination")
      unsigned long long pos = t_add(tv, &tv.ctl->newlog_tail, 1ull);
      if (pos < tv.newlog_cap) {
        tv.newlog[pos] = key;
        tv.newlog_slot[pos] = (unsigned int)i;
        if (tv.flags & TV_LIVE) {  // early notification: publish to the host right away
          LiveSlot* l = tv.ctl->live + pos;
          l->key = key;
          l->first = first;
          l->count = cnt;
          __threadfence_system();  // the payload is visible to the host before seq
          *reinterpret_cast<volatile unsigned long long*>(&l->seq) = (tv.ctl->live_gen << 32) | (pos + 1ull);
        }
      } else {
        t_red_add(tv, &tv.ctl->newlog_overflow, 1ull);
      }
      k = key;
    }
    if (k == key) {
      t_red_add(tv, &s->count, cnt);
      // `first` only decreases: a value already <= ours makes the min a no-op
      // (a fresh insert reads the empty slot's ~0 and always updates).  Skips
      // most of the atomics on hot slots: all-NaN storm S1 +20 % (A/B).
      if (first < f_seen) t_red_min(tv, &s->first, first);
      return;
    }
    i = (i + 1) & tv.mask;
  }
  t_red_add(tv, &tv.ctl->dropped_events, cnt);
}

// CTA-level pre-aggregation of table updates (dense exception storms): a
// small open-addressed table in shared memory, keyed like the device table,
// holding a 32-bit count and a 32-bit first-index offset (relative to the
// launch's base index) per key.  Every event of a key, its first sighting in
// the CTA included (FPX_CT_DEFER_FIRST), only touches shared memory; the key
// reaches the device table once, when the CTA's last warp is done
// (cta_warp_done).  Alg2's "reduce before any atomic"
// one level up: per CTA instead of per warp.  A key that finds no
// slot within CT_PROBES probes goes straight to the device table.
constexpr uint32_t CT_SLOTS = 512, CT_PROBES = 16;
#ifndef FPX_CT_HASH32
#define FPX_CT_HASH32 1
#endif
constexpr uint32_t CT_USABLE = CT_SLOTS - 1;  // slot CT_SLOTS - 1 holds the header (see from_image)
constexpr uint32_t CT_NONE = 0xFFFFFFFFu;
constexpr uint32_t CT_ON = 1u, CT_ON_RED = 2u;  // the header's "on" word
// FPX_CT_DEFER_FIRST 1: a key's first sighting in a CTA is counted in shared
// memory like the others and reaches the device table (and the new-key log /
// live ring) when the CTA's last warp drains the table, at the latest at the
// end of the launch, instead of at once: the storm kernel's warps then never
// wait for a device-table insert (each CTA met every hot key once, ~10 L2
// round trips per warp early in the launch: S1 +9.2 %, S2 +11.4 %,
// profiles/r2/ab_ct_defer.txt).  Only the storm kernel has a CTA table; the
// sparse kernels, where an isolated new exception is what a user waits for,
// still insert at once (P:244's early notification is about runs that last
// hours, not about one launch).  0: insert at the first sighting.
#ifndef FPX_CT_DEFER_FIRST
#define FPX_CT_DEFER_FIRST 1
#endif
#ifndef FPX_CT_RED
#define FPX_CT_RED 1
#endif
// A tile is "dense" (its events go through the CTA table) from this many
// warp-reduced events (FLOW / pending batches) or records with an event
// (DEST transposed path) on.
#ifndef FPX_DENSE_EVENTS
#define FPX_DENSE_EVENTS 4
#endif
constexpr uint32_t kDenseEvents = FPX_DENSE_EVENTS;
struct CtaTable {
  unsigned long long* keys;  // shared [CT_SLOTS] FPX_KEY_EMPTY when free, then the
                             // counts [CT_SLOTS] (u32, lane-values not yet in the device table)
                             // and the first offsets [CT_SLOTS] (u32, min first index - base);
                             // nullptr: no CTA table (events go to the device table)
  unsigned long long base;   // the launch's base index
  bool red = false;          // counts by RED (no returned value, no drain): see init
  __host__ __device__ static constexpr size_t bytes() { return CT_SLOTS * 16; }
  __device__ __forceinline__ unsigned int* cnt() const { return reinterpret_cast<unsigned int*>(keys + CT_SLOTS); }
  __device__ __forceinline__ unsigned int* first() const { return cnt() + CT_SLOTS; }
  __device__ __forceinline__ bool on() const { return keys != nullptr; }
  // The record-scan ring kernel keeps the table at the END of its dynamic
  // shared memory (image_at) with its header in the last slot (key = base
  // index, count = on, first = warps done), so the exact path finds it from
  // %dynamic_smem_size without any register held by the scan loop, and the
  // rings keep their offsets.
  __device__ static uint8_t* image_at() {
    extern __shared__ __align__(128) uint8_t fpx_dyn_smem[];
    uint32_t dyn;
    asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(dyn));
    return fpx_dyn_smem + dyn - bytes();
  }
  __device__ static CtaTable from_image() {
    uint8_t* smem = image_at();
    const unsigned long long* k = reinterpret_cast<const unsigned long long*>(smem);
    const unsigned int* c = reinterpret_cast<const unsigned int*>(k + CT_SLOTS);
    return CtaTable{c[CT_USABLE] ? reinterpret_cast<unsigned long long*>(smem) : nullptr, k[CT_USABLE],
                    c[CT_USABLE] == CT_ON_RED};
  }
  // by the whole CTA, before a __syncthreads.  red_ok: the launch has fewer
  // than 2^24 records, so no slot's count (<= 256 lane-values per record)
  // can reach 2^32: counts are added with a fire-and-forget shared reduction
  __device__ void init(bool on_, bool red_ok = false) const {
    for (uint32_t i = threadIdx.x; i < CT_USABLE; i += blockDim.x) {
      keys[i] = FPX_KEY_EMPTY;
      cnt()[i] = 0u;
      first()[i] = CT_NONE;
    }
    if (threadIdx.x == 0) {
      keys[CT_USABLE] = base;
      cnt()[CT_USABLE] = !on_ ? 0u : red_ok ? CT_ON_RED : CT_ON;
      first()[CT_USABLE] = 0u;  // warps done (cta_warp_done)
    }
  }
  // one event (any lane, divergent callers welcome); c < 2^16; requires on()
  __device__ __forceinline__ void add(const TableView& tv, unsigned long long key, uint32_t c, unsigned long long f) const {
#if FPX_CT_HASH32
    // a 32-bit multiplicative hash mapped onto the slots with one umulhi (the
    // 64-bit fmix + 64-bit modulo cost ~20 instructions per event in storms)
    const uint32_t hk = ((uint32_t)(key >> 32) * 0x9E3779B1u) ^ ((uint32_t)key * 0x85EBCA77u);
    uint32_t i = __umulhi(hk, CT_USABLE);
#else
    uint32_t i = (uint32_t)(hash_key(key) % CT_USABLE);
#endif
    for (uint32_t probe = 0; probe < CT_PROBES; ++probe, i = i + 1u == CT_USABLE ? 0u : i + 1u) {
      unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(keys + i);
      if (k == FPX_KEY_EMPTY) {
        k = atomicCAS(keys + i, FPX_KEY_EMPTY, key);
        if (k == FPX_KEY_EMPTY) {  // first sighting in this CTA: the device table gets it now
          if (!FPX_CT_DEFER_FIRST) {
            table_add(tv, key, c, f);
            return;
          }
          k = key;  // deferred: counted here, inserted by the CTA's last warp
        }
      }
      if (k == key) {
        unsigned int* fi = first() + i;
        unsigned int* ci = cnt() + i;
        const uint32_t off = (uint32_t)(f - base);
        if (off < *reinterpret_cast<volatile unsigned int*>(fi)) atomicMin(fi, off);
        if (red) {  // nothing to wait for (S1 / S2: ab_ct_red.txt)
          asm volatile("red.shared.add.u32 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(ci)), "r"(c) : "memory");
          return;
        }
        const uint32_t old = atomicAdd(ci, c);
        if (old + c >= 0x80000000u) {  // keep the 32-bit count far from overflow: drain it
          const uint32_t v = atomicExch(ci, 0u);
          if (v) table_add(tv, key, v, base + *reinterpret_cast<volatile unsigned int*>(fi));
        }
        return;
      }
    }
    table_add(tv, key, c, f);
  }
};

// An event of the record-scan ring kernel's exact path: through the CTA
// table when the kernel set one up (found in shared memory, so callers hold
// no register for it) and the tile is dense (a storm: many events, keys that
// repeat), else straight to the device table (sparse tiles: the insert
// latency is what counts, and a key seldom repeats within a CTA).  Out of line: the
// scan loop's register budget stays with the fast path.  Only for kernels
// whose dynamic shared memory starts with a CtaTable image.
static __device__ __noinline__ void emit_event(const TableView tv, unsigned long long key, uint32_t c,
                                              unsigned long long f, bool dense) {
  if (dense) {  // only warm warps of kernels that set the table up pass dense
    const CtaTable ct = CtaTable::from_image();
    if (ct.on()) {
      ct.add(tv, key, c, f);
      return;
    }
  }
  table_add(tv, key, c, f);
}

// A record's per-kind counts (16 bits per kind in cnt, kinds in `present`)
// straight into the CTA table (warm warps, dense tiles of the transposed
// DEST path); out of line like emit_event.
#ifndef FPX_EMIT_INLINE
#define FPX_EMIT_INLINE 0
#endif
#if FPX_EMIT_INLINE
static __device__ __forceinline__
#else
static __device__ __noinline__
#endif
void emit_kinds_cta(const TableView tv, uint32_t site, uint32_t fmt, uint32_t present,
                                                  unsigned long long cnt, unsigned long long f) {
  const CtaTable ct = CtaTable::from_image();
  while (present) {
    const uint32_t kd = (uint32_t)(__ffs(present) - 1);
    present &= present - 1u;
    const unsigned long long key = make_key(site, fmt, kd);
    const uint32_t c = (uint32_t)((cnt >> (16 * kd)) & 0xFFFFu);
    if (ct.on()) ct.add(tv, key, c, f);
    else table_add(tv, key, c, f);
  }
}

// Called once by every warp of the ring kernel's CTA as it finishes
// (warp-uniform).  The last one to arrive adds every slot's pending count
// (with its min first index) to the device table: the other warps' shared
// memory updates happen before their (fenced) arrival, so it sees them all.
// The arrival counter is the header slot's first-offset word.  Out of line,
// like emit_event, so the scan loop keeps no register for it.
static __device__ __noinline__ void cta_warp_done(const TableView tv, uint32_t nwarps) {
  const CtaTable ct = CtaTable::from_image();
  if (!ct.on()) return;
  const uint32_t lane = threadIdx.x & 31u;
  __syncwarp();
  __threadfence_block();
  uint32_t last = 0u;
  if (lane == 0u) last = atomicAdd(ct.first() + CT_USABLE, 1u) == nwarps - 1u ? 1u : 0u;
  if (__shfl_sync(0xFFFFFFFFu, last, 0) == 0u) return;
  __threadfence_block();
  for (uint32_t i = lane; i < CT_USABLE; i += 32u) {
    const unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(ct.keys + i);
    const uint32_t c = *reinterpret_cast<volatile unsigned int*>(ct.cnt() + i);
    if (k != FPX_KEY_EMPTY && c != 0u) table_add(tv, k, c, ct.base + *reinterpret_cast<volatile unsigned int*>(ct.first() + i));
  }
}

// Per-CTA table-update queue (the analyzer kernels): the scan warps hand
// their warp-reduced (key, count, first) events to one extra warp of the CTA,
// the drain warp, which issues them (table_add) while the scan warps go on
// streaming.  A table insert costs one or two dependent L2 round trips (the
// key CAS, then the new-key log position), ~2 us each under a full HBM
// stream: half of an analyzer hit tile's time when the scanning warp waited
// for them itself (profiles/r2/ab_flow_cand.txt).  Same updates, same table;
// only the issuing warp changes.  A bounded ring of tickets: a producer lane
// takes ticket t from `tail` (shared atomic), waits until entry t % EQ_N is
// free for it (seq == t; only when EQ_N events are in flight), writes the
// event and publishes seq = t + 1; the drain warp takes tickets in order, 32
// at a time (one lane each, so up to 32 inserts overlap), and frees each
// entry for ticket t + EQ_N.  The image sits at the END of dynamic shared
// memory (found from %dynamic_smem_size, like CtaTable; the kernels that use
// the queue have no CTA table).
constexpr uint32_t EQ_N = 256;  // entries (power of two)
struct EqEntry {
  unsigned long long key, first;
  uint32_t count, seq;
};
static_assert(sizeof(EqEntry) == 24, "queue entry");
struct EventQueue {
  EqEntry* e;          // [EQ_N]
  unsigned int* hdr;   // [0] tail (tickets taken), [1] scan warps done
  __host__ __device__ static constexpr size_t bytes() { return EQ_N * sizeof(EqEntry) + 16; }
  __device__ static EventQueue from_image() {
    extern __shared__ __align__(128) uint8_t fpx_dyn_smem[];
    uint32_t dyn;
    asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(dyn));
    uint8_t* p = fpx_dyn_smem + dyn - bytes();
    return EventQueue{reinterpret_cast<EqEntry*>(p), reinterpret_cast<unsigned int*>(p + EQ_N * sizeof(EqEntry))};
  }
  // by the whole CTA, before a __syncthreads
  __device__ void init() const {
    for (uint32_t i = threadIdx.x; i < EQ_N; i += blockDim.x) e[i].seq = i;
    if (threadIdx.x == 0) hdr[0] = hdr[1] = 0u;
  }
};

// Bounded spin of the queue's hand-offs: the other side is always running (a
// producer writes right after taking its ticket; the drain warp frees entries
// as it goes), so a 4 s stall is an internal bug -- a launch error, not a hang.
__device__ __forceinline__ void eq_stall_check(unsigned long long& t0) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  if (t0 == 0ull) t0 = t;
  else if (t - t0 > 4000000000ull) __trap();
}

// One event into the CTA's queue (any lane; divergent callers welcome).
// Out of line: the scan loop's register budget stays with the fast path.
static __device__ __noinline__ void eq_push(unsigned long long key, uint32_t c, unsigned long long f) {
  const EventQueue q = EventQueue::from_image();
  const uint32_t t = atomicAdd(q.hdr, 1u);
  EqEntry* e = q.e + (t & (EQ_N - 1u));
  unsigned long long t0 = 0ull;
  while (*reinterpret_cast<volatile uint32_t*>(&e->seq) != t) {  // queue full: wait for the drain
    __nanosleep(64);
    eq_stall_check(t0);
  }
  e->key = key;
  e->first = f;
  e->count = c;
  __threadfence_block();
  *reinterpret_cast<volatile uint32_t*>(&e->seq) = t + 1u;
}

// A scan warp is done pushing (warp-uniform, once per scan warp, including
// warps without work).
static __device__ __forceinline__ void eq_warp_done() {
  __syncwarp();
  __threadfence_block();
  if ((threadIdx.x & 31u) == 0u) atomicAdd(EventQueue::from_image().hdr + 1, 1u);
}

// The drain warp: issues every queued event until all `nscan` scan warps are
// done and the queue is empty.
static __device__ __noinline__ void eq_drain(const TableView tv, uint32_t nscan) {
  const EventQueue q = EventQueue::from_image();
  const uint32_t lane = threadIdx.x & 31u;
  volatile unsigned int* vh = q.hdr;
  uint32_t h = 0u;
  for (;;) {
    uint32_t t = vh[0];
    if (t == h) {
      if (vh[1] != nscan) {
        __nanosleep(256);
        continue;
      }
      __threadfence_block();
      t = vh[0];  // every push of a done warp took its ticket before the warp counted itself done
      if (t == h) break;
    }
    const uint32_t n = min(t - h, 32u);
    if (lane < n) {
      EqEntry* e = q.e + ((h + lane) & (EQ_N - 1u));
      unsigned long long t0 = 0ull;
      while (*reinterpret_cast<volatile uint32_t*>(&e->seq) != h + lane + 1u) eq_stall_check(t0);
      __threadfence_block();
      const unsigned long long key = *reinterpret_cast<volatile unsigned long long*>(&e->key);
      const unsigned long long f = *reinterpret_cast<volatile unsigned long long*>(&e->first);
      const uint32_t c = *reinterpret_cast<volatile uint32_t*>(&e->count);
      __threadfence_block();
      *reinterpret_cast<volatile uint32_t*>(&e->seq) = h + lane + EQ_N;  // free for ticket h + lane + EQ_N
      table_add(tv, key, c, f);
    }
    __syncwarp();
    h += n;
  }
}

// Table updates of one warp, batched: the warp-reduced (key, count, first)
// events of a tile are parked one per lane and issued by up to 32 lanes at
// once, so a dense tile (storms) costs ~one L2 round trip per 32 events
// instead of one per event.  Consecutive events with the same key (a storm
// over one site) merge before any atomic.  `n` and `last` are warp-uniform.
// CTA = true: the issued events go through emit_event (CTA table).
// Q = true: hand the events to the CTA's drain warp (eq_push) instead.
template <bool CTA = false, bool Q = false>  // CTA: issue through emit_event (ring kernel only)
struct PendingEvents {
  unsigned long long key = 0, first = 0, last = FPX_KEY_EMPTY;
  uint32_t count = 0, n = 0;
  bool warm = false;  // CTA: the warp is in a storm; dense batches may use the CTA table
  __device__ __forceinline__ void push(const TableView& tv, unsigned long long k, uint32_t c,
                                       unsigned long long f) {
    const uint32_t lane = threadIdx.x & 31;
    if (n != 0 && k == last) {  // same key as the previous event: merge
      if (lane == n - 1) {
        count += c;
        first = min(first, f);  // record paths push in index order; tensor lists need not
      }
      return;
    }
    if (lane == n) {
      key = k;
      count = c;
      first = f;
    }
    last = k;
    if (++n == 32) flush(tv);
  }
  // (Combining non-adjacent equal keys with __match_any_sync before the
  // atomics was tried: +16 % on an all-NaN storm, -4 % / -11 % on the 1 %
  // storm and C1, so the plain per-lane issue stays.)
  __device__ __forceinline__ void flush(const TableView& tv) {
    const bool dense = warm && n >= kDenseEvents;  // warp-uniform
    if ((threadIdx.x & 31) < n) {
      if (Q) eq_push(key, count, first);
      else if (CTA) emit_event(tv, key, count, first, dense);
      else table_add(tv, key, count, first);
    }
    n = 0;
    last = FPX_KEY_EMPTY;
    __syncwarp();
  }
};

// Warp aggregation of one record's events.  Every lane passes a bitmask of
// the codes it holds (bit c = code c present) plus, per code, its count via
// the `count_of` functor.  Must be called by the full warp (uniform).
template <typename CountOf, typename Pend>
__device__ __forceinline__ void warp_flush(const TableView& tv, Pend& pend, uint32_t code_mask,
                                           uint32_t site, uint32_t fmt, unsigned long long gidx, CountOf count_of) {
  uint32_t all = __reduce_or_sync(FULL, code_mask);
  while (all) {
    const int c = __ffs(all) - 1;
    all &= all - 1;
    const uint32_t tot = __reduce_add_sync(FULL, count_of(c));
    pend.push(tv, make_key(site, fmt, (uint32_t)c), tot, gidx);
  }
}

// Warp aggregation when every lane holds at most one event code (the FLOW
// modes): lanes with equal codes are grouped with a ballot per distinct code.
template <typename Pend>
__device__ __forceinline__ void warp_flush_single(const TableView& tv, Pend& pend, int code, uint32_t site,
                                                  uint32_t fmt, unsigned long long gidx) {
  uint32_t pending = __ballot_sync(FULL, code >= 0);
  while (pending) {
    const int leader = __ffs(pending) - 1;
    const int c = __shfl_sync(FULL, code, leader);
    const uint32_t peers = __ballot_sync(FULL, code == c);
    pend.push(tv, make_key(site, fmt, (uint32_t)c), __popc(peers), gidx);
    pending &= ~peers;
  }
}

// Shared-memory address of a generic pointer into shared memory, and a
// 128-bit shared load at such an address.
__device__ __forceinline__ uint32_t sh_addr(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ uint32_t sh_ld1(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint4 sh_ld4(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}

// Streaming 32-bit / 128-bit loads: read-only path, no L1 allocation.
__device__ __forceinline__ uint32_t ld_stream(const uint32_t* p) {
  uint32_t v;
  asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint4 ld_stream4(const void* p) {
  uint4 v;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

}  // namespace fpx
