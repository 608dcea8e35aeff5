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

// Insert-or-update.  Linear probing over the whole table: an event is only
// dropped (and TABLE_FULL raised) when every slot holds another key.
static __device__ __noinline__ void table_add(const TableView tv, unsigned long long key, unsigned long long cnt,
                                       unsigned long long first) {
  unsigned long long i = hash_key(key) & tv.mask;
  for (unsigned long long probe = 0; probe <= tv.mask; ++probe) {
    Slot* s = tv.slots + i;
    unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(&s->key);
    const unsigned long long f_seen = *reinterpret_cast<volatile unsigned long long*>(&s->first);
    if (k == FPX_KEY_EMPTY) {
      k = t_cas(tv, &s->key, FPX_KEY_EMPTY, key);
      if (k == FPX_KEY_EMPTY) {
        // this thread inserted the key: log it once (the "new combination")
        unsigned long long pos = t_add(tv, &tv.ctl->newlog_tail, 1ull);
        if (pos < tv.newlog_cap) {
          tv.newlog[pos] = key;
          tv.newlog_slot[pos] = (unsigned int)i;
          if (tv.live != nullptr) {  // early notification: publish to the host right away
            LiveSlot* l = tv.live + pos;
            l->key = key;
            l->first = first;
            l->count = cnt;
            __threadfence_system();  // the payload is visible to the host before seq
            *reinterpret_cast<volatile unsigned long long*>(&l->seq) =
                ((unsigned long long)tv.live_gen << 32) | (pos + 1ull);
          }
        } else {
          t_add(tv, &tv.ctl->newlog_overflow, 1ull);
        }
        k = key;
      }
    }
    if (k == key) {
      t_add(tv, &s->count, cnt);
      // `first` only decreases: a value already <= ours makes the min a no-op
      // (a fresh insert reads the empty slot's ~0 and always updates).  Skips
      // most of the atomics on hot slots: all-NaN storm S1 +20 % (A/B).
      if (first < f_seen) t_min(tv, &s->first, first);
      return;
    }
    i = (i + 1) & tv.mask;
  }
  t_add(tv, &tv.ctl->dropped_events, cnt);
}

// Table updates of one warp, batched: the warp-reduced (key, count, first)
// events of a tile are parked one per lane and issued by up to 32 lanes at
// once, so a dense tile (storms) costs ~one L2 round trip per 32 events
// instead of one per event.  Consecutive events with the same key (a storm
// over one site) merge before any atomic.  `n` and `last` are warp-uniform.
struct PendingEvents {
  unsigned long long key = 0, first = 0, last = FPX_KEY_EMPTY;
  uint32_t count = 0, n = 0;
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
    if ((threadIdx.x & 31) < n) table_add(tv, key, count, first);
    n = 0;
    last = FPX_KEY_EMPTY;
    __syncwarp();
  }
};

// Warp aggregation of one record's events.  Every lane passes a bitmask of
// the codes it holds (bit c = code c present) plus, per code, its count via
// the `count_of` functor.  Must be called by the full warp (uniform).
template <typename CountOf>
__device__ __forceinline__ void warp_flush(const TableView& tv, PendingEvents& pend, uint32_t code_mask,
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
__device__ __forceinline__ void warp_flush_single(const TableView& tv, PendingEvents& pend, int code, uint32_t site,
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
