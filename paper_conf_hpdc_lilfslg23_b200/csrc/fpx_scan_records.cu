// fpx_scan_records.cu — the record scan for sm_100a.
//
// One warp owns a contiguous range of records and walks it in tiles of up to
// 32 records (one header per lane) whose needed planes fit one stage of a
// per-warp shared-memory ring.  Lane l of the scanning warp reads lane l of
// every plane: exactly the lane of the instrumented warp whose register it
// holds (Alg2, "each thread checks its own value").
//
// k_scan_records_tma (default)
//   produce   lane j decodes + validates header j (prefetched one tile ahead),
//             a warp scan assigns each record's needed planes (DEST: the
//             destination words; FLOW: destination + sources) a contiguous
//             slot range in the stage; when the tile's needed planes are
//             one arena-contiguous range (the common case: one min-reduce and
//             one vote decide it) lane 0 issues ONE cp.async.bulk (TMA) copy
//             global -> shared, otherwise one copy per run of adjacent planes;
//             copies complete on the stage's mbarrier.  Tiles are issued
//             STAGES-1 ahead, so memory parallelism is bounded by shared
//             memory, not registers.
//   consume   lane-quad layout (8 threads per plane, one 128-bit LDS each);
//             a few integer ops per value keep min / max witnesses of
//             "subnormal" and "exponent all ones"; one vote per tile (the
//             common case at 1e-6 density is "nothing exceptional")
//   exact     hit tiles only: rec::exact_tile (kind rule, flow states, warp
//             aggregation, table) — fpx_records.cuh
//
// k_scan_records_ldg (ablation, FPX_OPT_SCAN_LDG): the same fast path with
// register-staged LDG loads, batched U per warp; kept to show what the TMA
// ring buys (profiles/).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <mutex>

#include "fpx_records.cuh"

namespace fpx {
namespace {

using namespace rec;

// ---- PTX wrappers: mbarrier + bulk async copy -------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_init_fence() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// Bounded wait: the copies of a stage always complete unless the byte count
// promised by expect_tx and the bytes issued disagree (an internal bug); a
// watchdog turns such a deadlock into a launch error instead of a hang.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  if (mbar_try_wait(bar, parity)) return;
  const uint64_t t0 = globaltimer_ns();
  while (!mbar_try_wait(bar, parity)) {
    if (globaltimer_ns() - t0 > 4000000000ull) __trap();
  }
}
// global -> shared bulk copy (TMA), completion counted in bytes on `bar`;
// streaming data: evict-first in L2.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ---- TMA-ring kernel ------------------------------------------------------------
// Ring geometry: WARPS warps per CTA (one CTA per SM), STAGES stages per warp
// (STAGES-1 tiles in flight while one is consumed), PLANES planes per stage.
template <int WARPS_, int STAGES_, int PLANES_, bool STASH_ = false>
struct RingCfg {
  static constexpr int WARPS = WARPS_, STAGES = STAGES_, PLANES = PLANES_;
  static constexpr bool STASH = STASH_;  // the producer keeps each tile's headers in shared memory
};

// Fast-path item lists of a stage: 4 formats x {full, partial active mask}.
// list l = 2 * fmt + partial.
constexpr int NLISTS = 8;

// StageMeta::k bit 31: the tile holds a record that must take the exact path
constexpr uint32_t kForceBit = 0x80000000u;
// StageMeta::k bit 30: the producer built no item lists (a storm kernel warp
// in storm mode): the tile goes to the exact path
constexpr uint32_t kNoListBit = 0x40000000u;
constexpr uint32_t kFlagBits = kForceBit | kNoListBit;
struct StageMeta {
  uint32_t k;      // records in the tile (0 = no tile) | kForceBit | kNoListBit
  uint32_t tot;    // items in the tile (end of the last list)
  uint64_t gidx0;  // global index of the tile's first record
  uint32_t sb;     // byte f: first item of format f's full-mask list
  uint32_t sp;     // byte f: first item of format f's partial-mask list
  uint32_t pad[2];
};

template <class C>
struct alignas(128) WarpSmem {  // 128-B multiple: every warp's planes stay 16-B (TMA / LDS.128) aligned
  uint32_t planes[C::STAGES][C::PLANES * 32];  // 128 B per plane
  uint2 items[C::STAGES][C::PLANES];           // {plane slot, active mask}
  StageMeta meta[C::STAGES];
  uint64_t bar[C::STAGES];
  uint4 hdrs[C::STASH ? C::STAGES : 1][C::STASH ? 32 : 1];  // STASH: the tile's headers (lane = record)
};
// Header-decode table, one byte per (opclass < 32, fmt, nsrc, dwords):
// low nibble = fast-path items (0..4), DECODE_FORCE (DIV: exact path) or
// DECODE_BAD (meta violates the contract of include/fpx.h); high nibble = the
// record's arena footprint in planes.  Built per CTA from decode_items().
constexpr int DECODE_ENTRIES = 4096;
constexpr uint32_t DECODE_FORCE = 5u, DECODE_BAD = 15u;
__device__ __forceinline__ uint32_t decode_index(uint32_t meta) { return ((meta >> 3) & 0xFE0u) | (meta & 31u); }
// meta bits outside the table index that a valid record keeps zero
constexpr uint32_t META_RESERVED = 0xFFFF80E0u;

// shared memory of the ring kernel: per-warp rings, the decode table, the
// CTA pre-aggregation table (fpx_device.cuh CtaTable)
template <class C>
constexpr size_t ring_smem(bool cta_table = true, bool eq = false) {
  // with the event queue the last warp drains it and has no ring
  return sizeof(WarpSmem<C>) * (C::WARPS - (eq ? 1 : 0)) + DECODE_ENTRIES + (cta_table ? CtaTable::bytes() : 0u) +
         (eq ? EventQueue::bytes() : 0u);
}

// Header decode for the fast path, branch-free: validity (the contract of
// include/fpx.h, same rules as rec::record_valid), the number of fast-path
// items (they enumerate exactly the planes the mode must look at — DEST: the
// destination words; FLOW: destination + source words — contiguous from plane
// 0 of the record; an FP64 item is a (lo, hi) pair), and `force` for DIV
// records, whose DIV0 rule needs the sources: the exact path reads them.
template <int MODE>
__device__ __forceinline__ uint32_t decode_items(const uint4 h, uint64_t arena_planes, bool inrange, bool& ok,
                                                 bool& force) {
  const uint32_t meta = h.z;
  const uint32_t op = meta & 0xFFu, fmt = (meta >> 8) & 3u, ns = (meta >> 10) & 3u, dw = (meta >> 12) & 7u;
  const uint32_t is64 = fmt == FPX_FP64 ? 1u : 0u;
  const uint32_t all_planes = dw + (ns << is64);
  bool v = inrange & (h.x != FPX_SITE_INVALID) & (meta < 0x8000u) & (op < (uint32_t)FPX_OP_COUNT) & (dw <= 4u) &
           !((is64 != 0u) & ((dw & 1u) != 0u));
  v &= (uint64_t)h.w + all_planes <= arena_planes;
  if (MODE != FPX_MODE_DEST) v &= (fmt <= 1u) & ((dw == 0u) | (dw == 1u + is64));
  ok = v;
  const bool live = v & (h.y != 0u);
  force = live & (op == FPX_OP_DIV);
  uint32_t p = all_planes;
  if (MODE == FPX_MODE_DEST) p = ((0x5800u >> (op & 31u)) & 1u) ? 0u : dw;  // FSET / FSETP / DSETP: no dest kind
  return (live & !force) ? (p >> is64) : 0u;
}
// arena planes a record occupies (destination + all sources)
__device__ __forceinline__ uint32_t footprint(uint32_t meta) {
  return dwords_of(meta) + (nsrc_of(meta) << (fmt_of(meta) == FPX_FP64 ? 1u : 0u));
}

template <int MODE>
__device__ void build_decode_table(uint8_t* lut) {
  for (uint32_t i = threadIdx.x; i < (uint32_t)DECODE_ENTRIES; i += blockDim.x) {
    const uint32_t meta = (i & 31u) | ((i >> 5) << 8);
    bool ok, force;
    const uint32_t ni = decode_items<MODE>(make_uint4(0u, FULL, meta, 0u), ~0ull, true, ok, force);
    const uint32_t code = !ok ? DECODE_BAD : force ? DECODE_FORCE : ni;
    lut[i] = (uint8_t)((footprint(meta) << 4) | code);
  }
}

// Same result as decode_items() from the table: validity, items, force, footprint.
__device__ __forceinline__ uint32_t decode_fast(const uint8_t* lut, const uint4 h, uint64_t arena_planes,
                                                bool inrange, bool& ok, bool& force, uint32_t& foot) {
  const uint32_t e = lut[decode_index(h.z)];
  const uint32_t code = e & 15u;
  foot = e >> 4;
  const bool v = inrange & (h.x != FPX_SITE_INVALID) & ((h.z & META_RESERVED) == 0u) & (code != DECODE_BAD) &
                 ((uint64_t)h.w + foot <= arena_planes);
  ok = v;
  const bool live = v & (h.y != 0u);
  force = live & (code == DECODE_FORCE);
  return (live & (code < DECODE_FORCE)) ? code : 0u;
}

// inclusive warp scan step: v += value of lane - o (lanes >= o)
template <int O>
__device__ __forceinline__ void scan_step(uint32_t& v) {
  asm("{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
      "shfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t"
      "@p add.u32 %0, %0, t;\n\t}"
      : "+r"(v)
      : "n"(O));
}

// planes covered by packed item counts (bytes: FP32, FP64 pairs, FP16, BF16;
// each byte <= 128 so the byte sum cannot overflow)
__device__ __forceinline__ uint32_t planes_of_items(uint32_t p) {
  return ((p * 0x01010101u) >> 24) + ((p >> 8) & 0xFFu);
}

// Witnesses of one 32-bit word (no false negatives; exact thresholds in hit()):
//   FP32  a2 = |x| << 1:  subnormal <=> a2 - 2 < 0xFFFFFE;  INF/NaN <=> a2 >= 0xFF000000
//   FP64  a3 = 2|hi| + (lo != 0):  subnormal <=> a3 - 1 < 0x1FFFFF;  INF/NaN <=> a3 >= 0xFFE00000
//   FP16 / BF16 per doubled half h (see half4):  subnormal <=> h - 2 < 0x7FE / 0xFE;
//                         INF/NaN <=> h >= 0xF800 / 0xFF00
// Inactive lanes are masked to zero first (zero is clean in every format).
// min(x, 1) as one VIMNMX (the compiler otherwise emits ISETP + SEL)
__device__ __forceinline__ uint32_t umin1(uint32_t x) {
  uint32_t r;
  asm("min.u32 %0, %1, 1;" : "=r"(r) : "r"(x));
  return r;
}
// x * 2 + y kept on the FMA pipe (IMAD) instead of an ALU IADD3
__device__ __forceinline__ uint32_t imad2(uint32_t x, uint32_t y) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, 2, %2;" : "=r"(r) : "r"(x), "r"(y));
  return r;
}
struct Witness {
  uint32_t mn32 = 0xFFFFFFFFu, mx32 = 0u, mn64 = 0xFFFFFFFFu, mx64 = 0u;
  uint32_t mn16 = 0xFFFFFFFFu, mx16 = 0u, mnb = 0xFFFFFFFFu, mxb = 0u;
  __device__ __forceinline__ void fp32(uint32_t x) {
    const uint32_t a2 = x << 1;
    mn32 = min(mn32, a2 - 2u);
    mx32 = max(mx32, a2);
  }
  __device__ __forceinline__ void fp64(uint32_t lo, uint32_t hi) {
    const uint32_t a3 = imad2(hi, umin1(lo));  // 2|hi| + (lo != 0): IMAD on the FMA pipe + one VIMNMX
    mn64 = min(mn64, a3 - 1u);
    mx64 = max(mx64, a3);
  }
  // packed halves, doubled (x + x: FMA pipe): each half's exponent moves to
  // the top of its halfword and the signs drop out (the low half's sign lands
  // in bit 0 of the high half, below every threshold that matters); then
  // per-halfword DPX min / max (VIADDMNMX.U16x2, VIMNMX.U16x2)
  template <bool BF>
  __device__ __forceinline__ void half4(uint4 x) {
    x = make_uint4(x.x + x.x, x.y + x.y, x.z + x.z, x.w + x.w);
    uint32_t& mn = BF ? mnb : mn16;
    uint32_t& mx = BF ? mxb : mx16;
    mn = __viaddmin_u16x2(x.x, 0xFFFEFFFEu, mn);  // h - 2 per half (0, 1 -> 0xFFFE, 0xFFFF)
    mn = __viaddmin_u16x2(x.y, 0xFFFEFFFEu, mn);
    mn = __viaddmin_u16x2(x.z, 0xFFFEFFFEu, mn);
    mn = __viaddmin_u16x2(x.w, 0xFFFEFFFEu, mn);
    mx = __vimax3_u16x2(x.x, x.y, mx);
    mx = __vimax3_u16x2(x.z, x.w, mx);
  }
  __device__ __forceinline__ bool hit() const {
    return hit_wide() || hit_half();
  }
  __device__ __forceinline__ bool hit_wide() const {
    return mn32 < 0x00FFFFFEu || mx32 >= 0xFF000000u || mn64 < 0x001FFFFFu || mx64 >= 0xFFE00000u;
  }
  __device__ __forceinline__ bool hit_half() const {
    // doubled halves h = 2|x| (+ 1 for a high half whose low half is negative):
    // subnormal <=> 2 <= h <= 2 * max_mantissa + 1; INF/NaN <=> h >= 2 * exponent mask
    return min(mn16 & 0xFFFFu, mn16 >> 16) < 0x07FEu || max(mx16 & 0xFFFFu, mx16 >> 16) >= 0xF800u ||
           min(mnb & 0xFFFFu, mnb >> 16) < 0x00FEu || max(mxb & 0xFFFFu, mxb >> 16) >= 0xFF00u;
  }
};

// Predicated streaming 128-bit global load (zeros when !p), without a branch.
__device__ __forceinline__ uint4 ld_stream4_if(bool p, const void* ptr) {
  uint4 v;
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %4, 0;\n\t"
      "mov.u32 %0, 0;\n\tmov.u32 %1, 0;\n\tmov.u32 %2, 0;\n\tmov.u32 %3, 0;\n\t"
      "@q ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%5];\n\t}"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
      : "r"((uint32_t)p), "l"(ptr));
  return v;
}

// 128-bit shared load at a byte address.
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint2 lds64(uint32_t addr) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr));
  return v;
}
// Per-value activity masks of lanes 4q .. 4q+3 (all ones = active).
__device__ __forceinline__ uint4 quad_ext(uint32_t mask, uint32_t q) {
  const uint32_t m = mask >> (4 * q);
  return make_uint4((uint32_t)((int32_t)(m << 31) >> 31), (uint32_t)((int32_t)(m << 30) >> 31),
                    (uint32_t)((int32_t)(m << 29) >> 31), (uint32_t)((int32_t)(m << 28) >> 31));
}
__device__ __forceinline__ uint4 and4(uint4 a, uint4 b) { return make_uint4(a.x & b.x, a.y & b.y, a.z & b.z, a.w & b.w); }

#ifndef FPX_CONSUME_UNROLL
#define FPX_CONSUME_UNROLL 1  // A/B on B200 (tools/ab.sh): 1 beats 2 and 4 by 2-5 %
#endif
constexpr int kConsumeUnroll = FPX_CONSUME_UNROLL;
#ifndef FPX_CTA_FLOW
#define FPX_CTA_FLOW 0
#endif
// The sparse DEST kernel's exact path: 0 inlined, 1 a direct call, 2 through
// g_exact_fn.  A call keeps the exact path's code out of the scan loop's
// register allocation (C2 -3.1 %, C5 -2.6 % warp instructions) but the scan
// runs 3 % slower on C2 (more stalls per instruction; interleaved bisection
// over this round's commits, profiles/r2/bisect_c2.txt), and C1 20 % slower:
// inlined.
// The analyzer kernels' exact path: 1 = the lean path (exact_tile_flow)
// inlined, 0 = called through g_flow_fn, 2 = the generic record path inlined.
// Inlined, ptxas spills 40 B on the rare exact path, but the call (an ABI
// frame in the scan loop) cost C3 0.8 % with the FLOW work split and 4.5 %
// with the DEST one (profiles/r2/ab_flow_inline.txt; bisected to the commit
// that introduced the call, profiles/r2/bisect_c3.txt).
#ifndef FPX_FLOW_INLINE
#define FPX_FLOW_INLINE 1
#endif
#ifndef FPX_CAS_FIRST
#define FPX_CAS_FIRST 1  // TV_CAS_FIRST for the sparse kernels (fpx_internal.h)
#endif
#ifndef FPX_SPARSE_DEST_CALL
#define FPX_SPARSE_DEST_CALL 0
#endif
template <class C>
constexpr int kSparseDestCall = C::WARPS == 24 ? 0 : FPX_SPARSE_DEST_CALL;
// The storm machinery (CTA pre-aggregation table, storm mode) lives in a
// separate DEST kernel instantiation (STORM = true) that the launcher picks
// when the handle's previous launch found a storm (ScanFeedback): it costs
// the sparse fast path 1-2 % of its instructions (C2 / C5), and gains 2.7-3x
// on storms.  The analyzer kernels never use it (it cost 5 % of C3).
template <int MODE, bool STORM>
constexpr bool kCtaTable = STORM && (MODE == FPX_MODE_DEST || FPX_CTA_FLOW);
// In the analyzer kernels the last warp of each CTA is the drain warp: it
// issues the exact path's table updates (fpx_device.cuh EventQueue), so the
// scan warps do not wait for the inserts' L2 round trips.  It replaces a scan
// warp rather than adding one: a 21st warp puts 6 warps on one SM
// sub-partition and caps the kernel at 80 registers (spills in the scan
// loop).  0: every warp scans and issues its own updates (A/B).
#ifndef FPX_EQ
#define FPX_EQ 1
#endif
template <int MODE, bool STORM>
constexpr bool kEq = FPX_EQ && MODE != FPX_MODE_DEST && !kCtaTable<MODE, STORM>;
template <int MODE, class C, bool STORM>
constexpr int kScanWarps = C::WARPS - (kEq<MODE, STORM> ? 1 : 0);
#ifndef FPX_BAD_SYS
#define FPX_BAD_SYS 1
#endif

// Consume one item list with the lane-quad layout: thread (g = lane / 8,
// q = lane % 8) reads words 4q..4q+3 (lanes 4q..4q+3 of the instrumented
// warp) of item i + g, so one warp step covers four items with one 128-bit
// shared load per thread (two for an FP64 pair).
template <uint32_t FMT, bool PARTIAL>
__device__ __forceinline__ void consume_list(Witness& w, uint32_t b, uint32_t e, uint32_t items_addr,
                                             uint32_t planes_addr, uint32_t g, uint32_t q) {
#pragma unroll kConsumeUnroll
  for (uint32_t i = b + g; i < e; i += 4) {
    const uint2 it = lds64(items_addr + i * 8);
    const uint32_t a = planes_addr + it.x * 128 + q * 16;
    uint4 x = lds128(a);
    uint4 mk = make_uint4(~0u, ~0u, ~0u, ~0u);
    if (PARTIAL) mk = quad_ext(it.y, q);
    if (FMT == FPX_FP64) {
      uint4 hi = lds128(a + 128);
      if (PARTIAL) {
        x = and4(x, mk);
        hi = and4(hi, mk);
      }
      w.fp64(x.x, hi.x);
      w.fp64(x.y, hi.y);
      w.fp64(x.z, hi.z);
      w.fp64(x.w, hi.w);
    } else {
      if (PARTIAL) x = and4(x, mk);
      if (FMT == FPX_FP32) {
        w.fp32(x.x);
        w.fp32(x.y);
        w.fp32(x.z);
        w.fp32(x.w);
      } else {
        w.half4<FMT == FPX_BF16>(x);
      }
    }
  }
}

// Load balance of the record scan.  Every warp first scans a static
// contiguous range (recs_per_warp records, 3/4 of the trace); the rest,
// [dyn0, n), is cut into chunks that warps claim with an atomicAdd on ctr[0]
// as they run out of work: nbig chunks of `chunk` records over [dyn0, dyn1),
// then one-tile chunks over [dyn1, n) (kTailTiles per warp), so that the last
// claims are short and the warps finish within a tile or two of each other.
// Equal record counts are not equal work: FP64-heavy stretches of a trace
// carry twice the bytes and exception storms take the exact path, so static
// ranges alone leave the SMs idle for 12-14 % of a C2 launch while the
// slowest warps finish (tools/warp_times.py, profiles/r1/ab_sched.txt).
// ctr[1] counts finished warps; the last one resets both counters, so each
// launch finds them at zero (the API gives concurrent launches different
// counter pairs).  nchunks = 0: static ranges only.
constexpr uint64_t kDynMinTiles = 16;  // dynamic tail only from 16 tiles per warp up
constexpr uint32_t kDynChunk = 256;     // records per claimed chunk (8 tiles)
// FLOW / FLOW_DETAIL: 128 (their tiles hold ~12 records with the sources, so
// a 256-record chunk is ~21 tiles): C3 +0.9 % (profiles/r2/ab_flow_sched.txt)
constexpr uint32_t kDynChunkFlow = 128;
// share of the trace in static ranges (DEST).  A warp whose SM streams x
// times slower than the average finishes its static range after the others
// have drained the dynamic tail when x > 100 / static share: 75 % covers
// SMs up to 1.33x slower, 60 % up to 1.67x (boxes with 1.33x SMs idle 5.5 %
// of a C2 launch at 75 %: profiles/r2/warp_times_r2fin.txt)
#ifndef FPX_STATIC_PCT_DEST
#define FPX_STATIC_PCT_DEST 75
#endif
constexpr int kStaticPct = FPX_STATIC_PCT_DEST;
// FLOW / FLOW_DETAIL: a smaller static share.  Some SMs stream 1.4-1.6x
// slower than the median (tools/warp_times.py: their warps finish 255 tiles
// of a static range while others do 313 with 15 claimed chunks), and the
// analyzer traces are short (C3: 0.65 ms), so a 75 % static range alone
// outlasts the kernel on them; 45 %: C3 +1.3 %, C2 (DEST) would lose 0.7 %
// (profiles/r2/ab_static.txt).
constexpr int kStaticPctFlow = 45;
constexpr uint32_t kTailTiles = 8;      // one-tile chunks at the end, per warp
struct SchedCfg {
  int static_pct;
  uint32_t chunk, tail_tiles;
};
struct Sched {
  unsigned int* ctr;
  uint64_t dyn0, dyn1;
  uint32_t chunk, nbig, nchunks, nwarps;
  // density feedback: every warp adds its hit tiles to *fb_dev; the last warp
  // out publishes the launch's total to mapped host memory (fb_host)
  unsigned long long* fb_dev;
  ScanFeedback* fb_host;
};

#ifdef FPX_WARP_TIMES
// Diagnostics build only (tools/warp_times.py): %globaltimer at each warp's
// start and end of the last record-scan launch, to measure load imbalance.
constexpr int kMaxWarpTimes = 148 * 32;
__device__ unsigned long long g_warp_t0[kMaxWarpTimes], g_warp_t1[kMaxWarpTimes];
// per warp: hit tiles and time spent in the exact path (ns)
__device__ unsigned long long g_warp_hits[kMaxWarpTimes], g_warp_exact_ns[kMaxWarpTimes];
// per warp: tiles consumed, chunks claimed, ns waiting on the stage mbarrier
__device__ unsigned long long g_warp_tiles[kMaxWarpTimes], g_warp_chunks[kMaxWarpTimes], g_warp_wait_ns[kMaxWarpTimes];
#endif

// The exact path of a hit tile (rec::exact_tile_hdr with this kernel's
// needed-plane count).  `warm`: this warp has met enough hit tiles for the
// CTA pre-aggregation table to pay (a storm); dense tiles then go through it.
template <int MODE>
__device__ __forceinline__ bool exact_tile_ring(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                                const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                                int lane, uint64_t gidx0, const TableView tv, bool warm,
                                                const uint4* pre = nullptr) {
  return exact_tile_hdr<MODE>(hdr_tile, k, arena_planes, lane_base, stage_lane, lane, gidx0, tv, warm, [](uint32_t meta) {
    bool f;
    const uint32_t ni = decode_items<MODE>(make_uint4(0u, FULL, meta, 0u), ~0ull, true, f, f);
    return fmt_of(meta) == FPX_FP64 ? 2u * ni : ni;
  }, pre);
}
// DEST: inlined (its transposed path fits the scan loop's registers: no
// spill).  FLOW / FLOW_DETAIL (exact_tile_flow) and the no-aggregation
// ablation (exact_tile_records): called through function pointers -- a
// direct call lets ptxas allocate caller and callee registers together and
// the record-walking path's demands then spill the scan loop's live values
// (up to 230 B per tile); an indirect call uses the ABI calling convention,
// whose saves and restores sit around the call, on the rare path only.
template <int MODE>
__device__ __noinline__ void exact_tile_ring_call(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                                  const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                                  int lane, uint64_t gidx0, const TableView tv, bool warm) {
  exact_tile_ring<MODE>(hdr_tile, k, arena_planes, lane_base, stage_lane, lane, gidx0, tv, warm);
}
// The analyzer's lean exact path (rec::exact_tile_flow), out of line.
template <int MODE>
__device__ __noinline__ void exact_tile_flow_call(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                                  const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                                  int lane, uint64_t gidx0, const TableView tv, bool warm) {
  exact_tile_flow<MODE>(hdr_tile, k, arena_planes, lane_base, stage_lane, lane, gidx0, tv, warm, [](uint32_t meta) {
    bool f;
    const uint32_t ni = decode_items<MODE>(make_uint4(0u, FULL, meta, 0u), ~0ull, true, f, f);
    return fmt_of(meta) == FPX_FP64 ? 2u * ni : ni;
  });
}
using ExactFn = void (*)(const uint4*, uint32_t, uint64_t, const uint32_t*, const uint32_t*, int, uint64_t,
                         const TableView, bool);
template <int MODE>
__device__ ExactFn g_exact_fn = exact_tile_ring_call<MODE>;
template <int MODE>
__device__ ExactFn g_flow_fn = exact_tile_flow_call<MODE>;
// storm mode (witnesses skipped) after this many dense exact tiles in a row
constexpr uint32_t kStormTiles = 16;
// Hysteresis of storm mode: a dense tile adds 1 to the run (up to kStormCap),
// a tile that is not dense takes kStormDrop off; storm mode while the run is
// >= kStormTiles.  On the 1 % storm S2 about one tile in 75 has fewer than 4
// records with an event: resetting the run on it sent ~17 % of S2's tiles
// through the fast path and its lists before the exact path (line profile,
// profiles/r2/lines_s2_r2v5.txt).  Leaving a storm costs (kStormCap -
// kStormTiles) / kStormDrop + 1 = 3 extra exact tiles.
#ifndef FPX_STORM_CAP
#define FPX_STORM_CAP 24
#endif
constexpr uint32_t kStormCap = FPX_STORM_CAP, kStormDrop = 4;
// the CTA table is used by a warp from its kWarmTiles-th hit tile on.  The
// storm kernel only runs after a launch that found a storm, so it needs no
// warm-up: 0 (8, the threshold from when one kernel served both: S1 -18 %,
// S2 -12 %; 0 without the reconvergence below: S2 -33 %;
// profiles/r2/ab_storm_warm.txt)
#ifndef FPX_POLICY_PER_TILE
#define FPX_POLICY_PER_TILE 0  // 1: recomputed per tile (no spill in the sparse DEST kernel, but C2 / C5 -0.5-1.2 %: ab_policy.txt)
#endif
#ifndef FPX_STORM_NO_LISTS
#define FPX_STORM_NO_LISTS 1
#endif
#ifndef FPX_STORM_LEAN
#define FPX_STORM_LEAN 1  // storm mode: one producer scan instead of two (no lists)
#endif
#ifndef FPX_DEST_RING
#define FPX_DEST_RING 1  // the sparse DEST kernels' ring for large traces (1: Ring1, 4: Ring4)
#endif
// BF16 items go into the FP16 lists and take the FP16 witness, which never
// misses a BF16 exception: a doubled BF16 half is subnormal iff it lies in
// [2, 0xFF] (inside FP16's [2, 0x7FF]) and INF / NaN iff >= 0xFF00 (inside
// FP16's >= 0xF800).  Its false positives are BF16 values below 2^-119 or
// above 2^120 in magnitude, which a hit tile's exact path then finds clean.
// Two list loops fewer per tile of packed records (C4a: ab_merge_halves.txt).
#ifndef FPX_MERGE_HALVES
#define FPX_MERGE_HALVES 1
#endif
constexpr bool kMergeHalves = FPX_MERGE_HALVES != 0;
#ifndef FPX_ONE_PLANE_RING
#define FPX_ONE_PLANE_RING 1
#endif
#ifndef FPX_STORM_HPRE
#define FPX_STORM_HPRE 1  // 1: loaded before the producer of the same iteration, 2: one iteration ahead (S1 / S2 -3.5 %: ab_storm_hpre.txt)
#endif
#ifndef FPX_STORM_RING
#define FPX_STORM_RING 5  // Ring5: 36-plane stages + header stash (S1 +3.0 %, S2 +3.4 %: ab_storm_stash.txt)
#endif
#ifndef FPX_STORM_START
#define FPX_STORM_START 1
#endif
#ifndef FPX_WARM_TILES
#define FPX_WARM_TILES 0
#endif
constexpr uint32_t kWarmTiles = FPX_WARM_TILES;

template <int MODE, class C, bool STORM>
__global__ void __launch_bounds__(C::WARPS * 32, 1)
k_scan_records_tma(const uint4* __restrict__ hdr, uint64_t n, const uint32_t* __restrict__ arena,
                   uint64_t arena_planes, uint64_t base_index, uint64_t recs_per_warp, const Sched sch,
                   const TableView tv) {
  constexpr int STAGES = C::STAGES, PLANES = C::PLANES;
  static_assert(PLANES <= 64, "stage sizes keep the byte fields of the packed scan exact");
  // dynamic shared memory: [per-warp rings][decode table][CTA table]
  extern __shared__ __align__(128) uint8_t fpx_dyn_smem[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* rings = fpx_dyn_smem;
  WarpSmem<C>& sm = reinterpret_cast<WarpSmem<C>*>(rings)[warp];
  uint8_t* lut = rings + sizeof(WarpSmem<C>) * kScanWarps<MODE, C, STORM>;
  build_decode_table<MODE>(lut);
  // CTA pre-aggregation of the exact path's table updates (fpx_device.cuh
  // CtaTable; the exact path finds it through emit_event); off for the
  // no-aggregation ablation and for launches whose record offsets need more
  // than 32 bits
  if (kCtaTable<MODE, STORM>)
    CtaTable{reinterpret_cast<unsigned long long*>(CtaTable::image_at()), base_index}
        .init((tv.flags & FPX_OPT_NO_WARP_AGG) == 0u && n < (uint64_t)CT_NONE, FPX_CT_RED && n < (1ull << 24));
  if (kEq<MODE, STORM>) EventQueue::from_image().init();
  __syncthreads();
  constexpr int SW = kScanWarps<MODE, C, STORM>;
  if (kEq<MODE, STORM> && warp == SW) {  // the drain warp (no block-wide barriers below)
    eq_drain(tv, SW);
    return;
  }
  const uint64_t gw = blockIdx.x * (uint64_t)SW + warp;
  const uint64_t start = gw * recs_per_warp;
  if (start >= n) {  // warp-uniform; no block-wide barriers below this line
    if (kCtaTable<MODE, STORM>) cta_warp_done(tv, C::WARPS);
    if (kEq<MODE, STORM>) eq_warp_done();
    return;
  }
#ifdef FPX_WARP_TIMES
  if (lane == 0 && gw < kMaxWarpTimes) {
    g_warp_t0[gw] = globaltimer_ns();
    g_warp_hits[gw] = 0;
    g_warp_exact_ns[gw] = 0;
    g_warp_tiles[gw] = g_warp_chunks[gw] = g_warp_wait_ns[gw] = 0;
    g_phase_ns[3 * gw] = g_phase_ns[3 * gw + 1] = g_phase_ns[3 * gw + 2] = 0;
  }
#endif
  const uint64_t end = min(n, start + recs_per_warp);
  // dynamic tail (Sched): the chunk this warp takes after its current range,
  // claimed one range ahead so the atomic's latency stays off the critical path
  uint32_t claim = 0;
  if (sch.nchunks != 0u && lane == 0) claim = atomicAdd(sch.ctr, 1u);
  const uint32_t* __restrict__ lane_base = arena + lane;
  const uint4* __restrict__ hdr_lane = hdr + lane;  // this lane's header of a tile = hdr_lane[tile start]
#if !FPX_POLICY_PER_TILE
  const uint64_t policy = policy_evict_first();
#endif
  const uint32_t g = (uint32_t)lane >> 3, q = (uint32_t)lane & 7u;

  if (lane == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) mbar_init(&sm.bar[s], 1);
    mbar_init_fence();
    sm.meta[0].pad[0] = 0u;  // hit tiles of this warp (exact path, CTA-table warm-up)
    // the storm run (storm mode, kStormCap).  The storm kernel starts in
    // storm mode (it runs after a launch that found a storm; tiles that are
    // not dense wear it off)
    sm.meta[0].pad[1] = kCtaTable<MODE, STORM> && FPX_STORM_START ? kStormCap : 0u;
  }
  __syncwarp();

  // cursor = global record index of the next tile; rem = records left in
  // this warp's range (< 2^31, checked at launch: 32-bit lane tests)
  uint64_t cursor = start;
  uint32_t rem = (uint32_t)(end - start);
  // at the end of a range: move into the claimed chunk and claim the next
  auto next_range = [&]() {
    if (rem == 0u) {
      if (sch.nchunks == 0u) return;
      const uint32_t c = __shfl_sync(FULL, claim, 0);
      if (c < sch.nchunks) {
        cursor = c < sch.nbig ? sch.dyn0 + (uint64_t)c * sch.chunk : sch.dyn1 + (uint64_t)(c - sch.nbig) * TILE;
#ifdef FPX_WARP_TIMES
        if (lane == 0 && gw < kMaxWarpTimes) g_warp_chunks[gw] += 1;
#endif
        rem = (uint32_t)min((uint64_t)(c < sch.nbig ? sch.chunk : TILE), n - cursor);
        if (lane == 0) claim = atomicAdd(sch.ctr, 1u);
      }
    }
  };
  next_range();
  uint4 h = ld_stream4_if((uint32_t)lane < rem, hdr_lane + cursor);

  // Build tile `s` from the prefetched headers and issue its copies.
  auto produce = [&](int s) {
    StageMeta& m = sm.meta[s];
    if (rem == 0u) {
      __syncwarp();
      if (lane == 0) m.k = 0;
      __syncwarp();
      return;
    }
    const bool inrange = (uint32_t)lane < rem;
    if (C::STASH) sm.hdrs[s][lane] = h;  // the exact path reads them from here (no L2 reload)
    bool ok, force;
    uint32_t foot_all;
    const uint32_t ni = decode_fast(lut, h, arena_planes, inrange, ok, force, foot_all);
    const uint32_t mask = ok ? h.y : 0u;
    const uint32_t fmt = fmt_of(h.z);
    const bool part = mask != FULL;
    // two packed scans (full / partial active mask; byte = format).  Bytes
    // stay <= 128 over the warp, so no field overflows into the next.
    // list format: BF16 items share the FP16 lists (kMergeHalves)
    const uint32_t lfmt = kMergeHalves ? min(fmt, (uint32_t)FPX_FP16) : fmt;
    const uint32_t c8 = ni << (8 * lfmt);
    // storm mode: the consumer skips the witnesses, so the lists are not built
    const bool lists = !kCtaTable<MODE, STORM> || !FPX_STORM_NO_LISTS || sm.meta[0].pad[1] < kStormTiles;
    uint32_t cf = part ? 0u : c8, cp = part ? c8 : 0u;
    uint32_t sf, sp;
    if (kCtaTable<MODE, STORM> && FPX_STORM_LEAN && !lists) {
      // no lists: one scan gives the stage slots (every item counted as full)
      cf = c8, cp = 0u;
      sf = c8, sp = 0u;
      scan_step<1>(sf), scan_step<2>(sf), scan_step<4>(sf), scan_step<8>(sf), scan_step<16>(sf);
    } else {
      sf = cf, sp = cp;
      scan_step<1>(sf), scan_step<1>(sp);
      scan_step<2>(sf), scan_step<2>(sp);
      scan_step<4>(sf), scan_step<4>(sp);
      scan_step<8>(sf), scan_step<8>(sp);
      scan_step<16>(sf), scan_step<16>(sp);
    }
    // a lane is in one of the two lists, so sf + sp stays <= 128 per byte
    const uint32_t incl_planes = planes_of_items(sf + sp);
    // the tile = leading records whose planes fit the stage (>= 1 record);
    // incl_planes never decreases over the lanes, so `fits` is a lane prefix
    const uint32_t fits = __ballot_sync(FULL, inrange && incl_planes <= (uint32_t)PLANES);
    const uint32_t k = (uint32_t)__popc(fits);
    const bool in_tile = (uint32_t)lane < k;
    // bad records and forced (DIV) records are rare: one vote finds both
    uint32_t force_any = 0u;
    if (__any_sync(FULL, in_tile && (!ok || force))) {
      const uint32_t bad = __ballot_sync(FULL, in_tile && !ok);
#if FPX_BAD_SYS
      if (bad != 0u && lane == 0) atomicAdd_system(&tv.ctl->bad_records, (unsigned long long)__popc(bad));  // rare; system scope covers shared tables
#else
      if (bad != 0u && lane == 0) atomicAdd(&tv.ctl->bad_records, (unsigned long long)__popc(bad));
#endif
      force_any = __ballot_sync(FULL, in_tile && force);
    }
    const uint32_t my_planes = ni << (fmt == FPX_FP64 ? 1u : 0u);  // = planes_of_items(c8)
    const uint32_t c = in_tile ? my_planes : 0u;
    const uint32_t slot = incl_planes - my_planes;
    const uint32_t tf = __shfl_sync(FULL, sf, k - 1), tp = __shfl_sync(FULL, sp, k - 1);
    const uint32_t total = __shfl_sync(FULL, incl_planes, k - 1);  // the tile's planes
    // the ring slot may still be read by the previous consume of this stage:
    // order those generic reads before the async-proxy writes below
    __syncwarp();
    fence_proxy_async_smem();
    // list l = 2 * fmt + partial; lists of lower formats come first
    const uint32_t tot_f = tf + tp;  // packed per-format item totals (<= 128 each)
    // byte f of `below`: items of the formats before f (= the start of format
    // f's full-mask list).  Every byte stays <= 40 (items <= planes), so the
    // packed sums never carry.
    const uint32_t below = (tot_f * 0x01010101u) << 8;
    const bool writes = lists && in_tile && ni != 0u;
    uint32_t at = 0u;
    if (writes) {
      // byte f of `own`: this record's place among format f's items (full list first)
      const uint32_t own = part ? tf + (sp - cp) : sf - cf;
      at = ((below + own) >> (8 * lfmt)) & 0xFFu;
      sm.items[s][at] = make_uint2(slot, mask);
    }
#ifndef FPX_ITEMS_PREDICATED
    // records with several items (HMMA fragments, FLOW sources) are absent
    // from many traces: one vote skips their writes
    if (__any_sync(FULL, writes && ni > 1u))
#endif
    {
      const uint32_t step = fmt == FPX_FP64 ? 2u : 1u;
#pragma unroll
      for (uint32_t j = 1; j < 4; ++j)  // ni <= 4
        if (writes && j < ni) sm.items[s][at + j] = make_uint2(slot + j * step, mask);
    }
    if (lane == 0) {
      m.k = k | (force_any != 0u ? kForceBit : 0u) | (lists ? 0u : kNoListBit);
      m.gidx0 = base_index + cursor;
      m.sb = below;              // list starts, packed (consumer: one PRMT per bound)
      m.sp = below + tf;
      m.tot = (tot_f * 0x01010101u) >> 24;
    }
    // Copies.  Common case: every in-tile record with an arena footprint
    // needs all of it and the footprints are arena-adjacent in record order
    // (records with no footprint are transparent), i.e. arena plane - stage
    // slot is the same for all of them: ONE bulk copy of the tile.
    const uint32_t a = h.w;
    const uint32_t foot = in_tile ? foot_all : 0u;
    const uint32_t d = a - slot;
    const uint32_t dmin = __reduce_min_sync(FULL, foot != 0u ? d : 0xFFFFFFFFu);
    // (dmin + total <= 2^32: the run's arena planes fit the 32-bit plane index)
    const bool one_run = __all_sync(FULL, foot == 0u || (c == foot && d == dmin)) &&
                         (total == 0u || dmin <= 0u - total);
    if (one_run) {
      if (lane == 0) {
        mbar_arrive_expect_tx(&sm.bar[s], total * 128u);
#if FPX_POLICY_PER_TILE
        const uint64_t policy = policy_evict_first();  // one instruction; not a register held by the scan loop
#endif
        if (total != 0u) bulk_g2s(&sm.planes[s][0], arena + (uint64_t)dmin * 32, total * 128u, &sm.bar[s], policy);
      }
    } else {
      // general case: runs of arena-adjacent needed planes -> one bulk copy
      // each.  A record whose needed planes stop before the end of its
      // footprint (DEST with sources) ends a run.
      const uint32_t rel = __ballot_sync(FULL, foot != 0u);
      const uint32_t below = rel & ((1u << lane) - 1u);
      const int prev = below ? 31 - __clz(below) : -1;
      const uint32_t prev_end = __shfl_sync(FULL, (c == foot) ? a + c : 0xFFFFFFFFu, prev < 0 ? 0 : prev);
      const bool head = c != 0u && (prev < 0 || prev_end != a);
      const uint32_t heads = __ballot_sync(FULL, head);
      const uint32_t above = lane == 31 ? 0u : heads & (0xFFFFFFFFu << (lane + 1));  // heads above this lane
      const uint32_t next = above ? (uint32_t)(__ffs(above) - 1) : 32u;
      const uint32_t next_slot_raw = __shfl_sync(FULL, slot, next & 31u);
      const uint32_t run_end = next < k ? next_slot_raw : total;
      if (lane == 0) mbar_arrive_expect_tx(&sm.bar[s], total * 128u);
      __syncwarp();
      if (head)
      {
#if FPX_POLICY_PER_TILE
        const uint64_t policy = policy_evict_first();
#endif
        bulk_g2s(&sm.planes[s][slot * 32], arena + (uint64_t)a * 32, (run_end - slot) * 128u, &sm.bar[s], policy);
      }
    }
    // advance and prefetch the next tile's headers
    cursor += k;
    rem -= k;
    next_range();
    h = ld_stream4_if((uint32_t)lane < rem, hdr_lane + cursor);
  };

  uint32_t phase = 0;  // bit s = parity to wait for on stage s
#pragma unroll 1
  for (int s = 0; s < STAGES - 1; ++s) produce(s);
  // storm kernel, FPX_STORM_HPRE 2: the exact path's headers of the tile
  // consumed next, loaded one loop iteration ahead (the first use of the
  // headers loaded before the producer was still 7.7 % of S2's stall samples,
  // r2v15) -- but holding them across the loop spills: S1 / S2 -3.5 %, so the
  // default stays 1 (ab_storm_hpre.txt)
  auto load_hx = [&](int st) {
    const uint32_t k0 = sm.meta[st].k & ~kFlagBits;
    return ld_stream4_if((uint32_t)lane < k0, hdr + (sm.meta[st].gidx0 - base_index) + lane);
  };
  uint4 hx_next = make_uint4(0u, 0u, 0u, 0u);
  if (kCtaTable<MODE, STORM> && FPX_STORM_HPRE == 2) hx_next = load_hx(0);
#pragma unroll 1
  for (uint32_t i = 0;; ++i) {
    const int s = (int)(i % STAGES);
    // storm kernel: the headers of the tile about to be consumed, loaded
    // before the producer runs so that the load's latency hides behind it
    // (every tile of a storm takes the exact path, which needs them)
    uint4 hx = make_uint4(0u, 0u, 0u, 0u);
    if (kCtaTable<MODE, STORM> && FPX_STORM_HPRE == 1 && !C::STASH) hx = load_hx(s);
    produce((int)((i + STAGES - 1) % STAGES));
    if (kCtaTable<MODE, STORM> && FPX_STORM_HPRE == 2) {
      hx = hx_next;
      hx_next = load_hx((int)((i + 1) % STAGES));
    }
    const StageMeta& m = sm.meta[s];
    const uint32_t mk = m.k;  // records in the tile | kForceBit | kNoListBit
    if (mk == 0u) {
#ifdef FPX_WARP_TIMES
      if (lane == 0 && gw < kMaxWarpTimes) g_warp_t1[gw] = globaltimer_ns();
#endif
      // the last warp out re-arms the launch's chunk counters for reuse and
      // publishes the launch's hit tiles (density feedback for the launcher)
      if (sch.nchunks != 0u && lane == 0) {
        const uint32_t my_hits = sm.meta[0].pad[0];
        if (my_hits != 0u && sch.fb_dev != nullptr) atomicAdd(sch.fb_dev, (unsigned long long)my_hits);
        __threadfence();
        if (atomicAdd(sch.ctr + 1, 1u) == sch.nwarps - 1u) {
          atomicExch(sch.ctr, 0u);
          atomicExch(sch.ctr + 1, 0u);
          if (sch.fb_dev != nullptr) {
            const unsigned long long total = atomicExch(sch.fb_dev, 0ull);
            volatile ScanFeedback* fb = sch.fb_host;
            fb->hit_tiles = total;
            fb->records = n;
          }
        }
      }
      break;
    }
#ifdef FPX_WARP_TIMES
    const uint64_t tw0 = globaltimer_ns();
#endif
    mbar_wait(&sm.bar[s], (phase >> s) & 1u);
    phase ^= 1u << s;
#ifdef FPX_WARP_TIMES
    if (lane == 0 && gw < kMaxWarpTimes) {
      g_warp_wait_ns[gw] += globaltimer_ns() - tw0;
      g_warp_tiles[gw] += 1;
    }
#endif

    // Storm mode (DEST): after kStormTiles dense exact tiles in a row a warp
    // skips the witnesses -- in a storm every tile is hit anyway -- and
    // sends each tile straight to the exact path, until tiles that are not
    // dense bring the run below kStormTiles (hysteresis: kStormCap).
    // (the run length lives in the stage-0 descriptor's spare word: a register
    // held across the loop cost S2 6 %, profiles/r2/ab_storm_state.txt)
    const uint32_t storm_run = kCtaTable<MODE, STORM> ? sm.meta[0].pad[1] : 0u;
    bool hit = kCtaTable<MODE, STORM> && (storm_run >= kStormTiles || (mk & kNoListBit) != 0u);
    if (!hit) {
      // ---- fast path over the staged planes (lane-quad layout) ------------
      const uint32_t ia = smem_u32(sm.items[s]), pa = smem_u32(sm.planes[s]);
      // lists in order (fmt, full / partial): format f's full list is
      // [sb_f, sp_f), its partial list [sp_f, sb_{f+1}) (the last ends at tot)
      const uint32_t sb = m.sb, sp = m.sp, tot = m.tot;
      auto byte_of = [](uint32_t x, uint32_t f) { return __byte_perm(x, 0u, 0x4440u | f); };
      Witness w;
      const uint32_t s1 = byte_of(sb, 1), s2 = byte_of(sb, 2);
      consume_list<FPX_FP32, false>(w, 0u, byte_of(sp, 0), ia, pa, g, q);
      consume_list<FPX_FP32, true>(w, byte_of(sp, 0), s1, ia, pa, g, q);
      consume_list<FPX_FP64, false>(w, s1, byte_of(sp, 1), ia, pa, g, q);
      consume_list<FPX_FP64, true>(w, byte_of(sp, 1), s2, ia, pa, g, q);
      const bool halves = s2 != tot;
      if (halves) {
        if (kMergeHalves) {
          consume_list<FPX_FP16, false>(w, s2, byte_of(sp, 2), ia, pa, g, q);
          consume_list<FPX_FP16, true>(w, byte_of(sp, 2), tot, ia, pa, g, q);
        } else {
          const uint32_t s3 = byte_of(sb, 3);
          consume_list<FPX_FP16, false>(w, s2, byte_of(sp, 2), ia, pa, g, q);
          consume_list<FPX_FP16, true>(w, byte_of(sp, 2), s3, ia, pa, g, q);
          consume_list<FPX_BF16, false>(w, s3, byte_of(sp, 3), ia, pa, g, q);
          consume_list<FPX_BF16, true>(w, byte_of(sp, 3), tot, ia, pa, g, q);
        }
      }
      hit = __any_sync(FULL, w.hit_wide() || (halves && w.hit_half())) || (mk & kForceBit) != 0u;
    }
    if (hit) {
      // hit tiles of this warp so far: kept in shared memory (the stage-0
      // descriptor's spare word), not in a register of the scan loop
      const uint32_t hits = sm.meta[0].pad[0];
      __syncwarp();
      if (lane == 0) sm.meta[0].pad[0] = hits + 1u;
      const bool warm = kCtaTable<MODE, STORM> && hits >= kWarmTiles;
#ifdef FPX_WARP_TIMES
      const uint64_t te0 = globaltimer_ns();
#endif
      if (MODE == FPX_MODE_DEST && (STORM || kSparseDestCall<C> == 0)) {
        if (C::STASH) hx = sm.hdrs[s][lane];
        const bool dense = exact_tile_ring<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes,
                                                 lane_base, sm.planes[s] + lane, lane, m.gidx0, tv, warm,
                                                 kCtaTable<MODE, STORM> && (FPX_STORM_HPRE || C::STASH) ? &hx : nullptr);
        if (kCtaTable<MODE, STORM> && lane == 0)
          sm.meta[0].pad[1] = dense ? min(storm_run + 1u, kStormCap) : storm_run - min(storm_run, kStormDrop);
      } else if (MODE == FPX_MODE_DEST && kSparseDestCall<C> == 1)
        exact_tile_ring_call<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base,
                                   sm.planes[s] + lane, lane, m.gidx0, tv, warm);
      else if (MODE == FPX_MODE_DEST)
        g_exact_fn<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base, sm.planes[s] + lane,
                         lane, m.gidx0, tv, warm);
      else if (!(tv.flags & FPX_OPT_NO_WARP_AGG)) {
#if FPX_FLOW_INLINE == 2
        exact_tile_ring<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base,
                              sm.planes[s] + lane, lane, m.gidx0, tv, warm);
#elif FPX_FLOW_INLINE
        exact_tile_flow<MODE, kEq<MODE, STORM>>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base,
                              sm.planes[s] + lane, lane, m.gidx0, tv, warm, [](uint32_t meta) {
                                bool f;
                                const uint32_t ni = decode_items<MODE>(make_uint4(0u, FULL, meta, 0u), ~0ull, true, f, f);
                                return fmt_of(meta) == FPX_FP64 ? 2u * ni : ni;
                              });
#else
        g_flow_fn<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base, sm.planes[s] + lane,
                        lane, m.gidx0, tv, warm);
#endif
      }
      else  // the no-aggregation ablation's record-by-record path
        g_exact_fn<MODE>(hdr + (m.gidx0 - base_index), mk & ~kFlagBits, arena_planes, lane_base, sm.planes[s] + lane,
                         lane, m.gidx0, tv, warm);
#ifdef FPX_WARP_TIMES
      if (lane == 0 && gw < kMaxWarpTimes) {
        g_warp_hits[gw] = hits + 1;
        g_warp_exact_ns[gw] += globaltimer_ns() - te0;
      }
#endif
      // storm kernel: reconverge after the exact path.  Lanes leave it at
      // different points (the table updates of a dense tile), and unless the
      // warp syncs here ptxas may let the groups run the next tiles apart:
      // S1 +3 %, S2 +4 %, and with it the warm-up can go (kWarmTiles)
      if (STORM) __syncwarp();
    }
  }
  // out of the loop: the call's register conventions stay off the scan loop
  if (kCtaTable<MODE, STORM>) cta_warp_done(tv, C::WARPS);
  if (kEq<MODE, STORM>) eq_warp_done();
}

// Ring configurations compiled in; FPX_RING (environment, tuning only) picks
// one, default RING_DEFAULT.
using Ring0 = RingCfg<16, 2, 50>;
using Ring1 = RingCfg<20, 2, 40>;
using Ring2 = RingCfg<28, 2, 28>;
using Ring3 = RingCfg<24, 2, 32>;
// the analyzer kernels with the drain warp (kEq): 19 scan warps x 42 planes
// keep Ring1's bytes in flight
using Ring1E = RingCfg<20, 2, 42>;
// the storm kernel (FPX_STORM_RING 5): Ring1's warps with 36-plane stages and
// the tiles' headers kept in the freed shared memory, so the exact path,
// which every storm tile takes, reads them with LDS instead of reloading
// them from L2 (the first use of the reloaded headers was 7.7 % of S2's stall
// samples, r2v15); one-plane storm tiles use 32 planes anyway
using Ring5 = RingCfg<20, 2, 36, true>;
// 18 warps x 46 planes (A/B: FPX_DEST_RING=4): tiles of mixed FP32 / FP64
// records reach 32 records (C2 averages ~26 per 40-plane tile)
using Ring4 = RingCfg<18, 2, 46>;
static_assert(sizeof(WarpSmem<Ring2>) % 128 == 0 && ring_smem<Ring0>() <= 227 * 1024 && ring_smem<Ring1>() <= 227 * 1024 &&
                  ring_smem<Ring2>() <= 227 * 1024 && ring_smem<Ring3>() <= 227 * 1024,
              "ring exceeds shared memory");
static_assert(ring_smem<Ring4>(false) <= 227 * 1024, "ring 4 exceeds shared memory");
static_assert(ring_smem<Ring5>(true) <= 227 * 1024, "ring 5 exceeds shared memory");
static_assert(ring_smem<Ring0>(false, true) <= 227 * 1024 && ring_smem<Ring1E>(false, true) <= 227 * 1024 &&
                  ring_smem<Ring2>(false, true) <= 227 * 1024 && ring_smem<Ring3>(false, true) <= 227 * 1024,
              "ring + event queue exceeds shared memory");

constexpr int kMaxDevices = 64;

template <int MODE, class C, bool STORM>
cudaError_t launch_ring(const uint4* hdr, uint64_t n, const uint32_t* arena, uint64_t arena_planes, uint64_t base_index,
                        const TableView& tv, int num_sms, unsigned int* sched_ctr, const SchedCfg& scfg,
                        const FeedbackPtrs& fbp, cudaStream_t s) {
  // the shared-memory opt-in, once per device and kernel instantiation;
  // handles may live on different host threads
  static std::once_flag once[kMaxDevices];
  static cudaError_t once_err[kMaxDevices];
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  auto set_attr = [] {
    return cudaFuncSetAttribute(k_scan_records_tma<MODE, C, STORM>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)ring_smem<C>(kCtaTable<MODE, STORM>, kEq<MODE, STORM>));
  };
  if (dev < kMaxDevices) {
    std::call_once(once[dev], [&] { once_err[dev] = set_attr(); });
    e = once_err[dev];
  } else {
    e = set_attr();
  }
  if (e != cudaSuccess) return e;
  // one CTA per SM; each warp a contiguous range of records (whole tiles of 32
  // where possible, so that ranges stay 512-B aligned in the header array)
  constexpr int SW = kScanWarps<MODE, C, STORM>;
  const uint64_t warps = (uint64_t)num_sms * SW;
  Sched sch{sched_ctr, n, n, 0u, 0u, 0u, 0u, fbp.dev, fbp.host};
  uint64_t per, blocks;
  if (sched_ctr != nullptr && n >= warps * TILE * kDynMinTiles) {
    // static ranges: 3/4 of the trace in whole tiles; the rest in chunks
    per = n / 100 * (uint64_t)scfg.static_pct / warps / TILE * TILE;
    sch.dyn0 = per * warps;
    sch.chunk = scfg.chunk;
    const uint64_t rest = n - sch.dyn0, small = std::min<uint64_t>(rest, warps * scfg.tail_tiles * TILE);
    const uint64_t nbig = (rest - small) / scfg.chunk;
    sch.dyn1 = sch.dyn0 + nbig * scfg.chunk;
    const uint64_t nch = nbig + (n - sch.dyn1 + TILE - 1) / TILE;
    if (nch >= (1ull << 31)) return cudaErrorInvalidValue;
    sch.nbig = (uint32_t)nbig;
    sch.nchunks = (uint32_t)nch;
    sch.nwarps = (uint32_t)warps;
    blocks = (uint64_t)num_sms;
  } else {
    per = (n + warps - 1) / warps;
    per = (per + TILE - 1) / TILE * TILE;
    blocks = ((n + per - 1) / per + SW - 1) / SW;
  }
  if (per >= (1ull << 31)) return cudaErrorInvalidValue;  // the kernel counts a warp's records in 32 bits
  k_scan_records_tma<MODE, C, STORM><<<(unsigned)blocks, C::WARPS * 32,
                                       ring_smem<C>(kCtaTable<MODE, STORM>, kEq<MODE, STORM>), s>>>(hdr, n, arena, arena_planes,
                                                                                      base_index, per, sch, tv);
  return cudaGetLastError();
}

// ---- register-staged LDG kernel (ablation) ------------------------------------
constexpr int LDG_WARPS = 8;
constexpr int MAXITEMS = 128;  // <= 4 items per record
constexpr int U32 = 8;         // FP32 / packed items per load batch
constexpr int U64 = 4;         // FP64 pairs per load batch

template <int MODE>
__global__ void __launch_bounds__(LDG_WARPS * 32, 4)
k_scan_records_ldg(const uint4* __restrict__ hdr, uint64_t n, const uint32_t* __restrict__ arena,
               uint64_t arena_planes, uint64_t base_index, const TableView tv) {
  __shared__ RecDesc s_rec[LDG_WARPS][TILE];
  __shared__ uint2 s_item[LDG_WARPS][MAXITEMS];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t nwarps = (uint64_t)gridDim.x * LDG_WARPS;
  const uint64_t ntiles = (n + TILE - 1) / TILE;
  const uint32_t* __restrict__ lane_base = arena + lane;
  RecDesc* __restrict__ recs = s_rec[warp];
  uint2* __restrict__ items = s_item[warp];

  uint64_t tile = blockIdx.x * (uint64_t)LDG_WARPS + warp;
  uint4 h_next = make_uint4(0, 0, 0, 0);
  if (tile < ntiles && tile * TILE + lane < n) h_next = ld_stream4(hdr + tile * TILE + lane);

  for (; tile < ntiles; tile += nwarps) {
    // ---- prologue: lane = record --------------------------------------------
    const uint64_t r = tile * TILE + lane;
    const bool inrange = r < n;
    const uint4 h = h_next;
    {
      const uint64_t nt = tile + nwarps;  // prefetch the next tile's header
      if (nt < ntiles && nt * TILE + lane < n) h_next = ld_stream4(hdr + nt * TILE + lane);
    }
    const bool ok = inrange && record_valid<MODE>(h, arena_planes);
    const uint32_t bad = __ballot_sync(FULL, inrange && !ok);
    if (bad != 0u && lane == 0) atomicAdd_system(&tv.ctl->bad_records, (unsigned long long)__popc(bad));  // rare; system scope covers shared tables
    const uint32_t mask = ok ? h.y : 0u;
    bool force;
    const uint32_t cnt = item_counts<MODE>(h.z, ok && mask != 0u, force);
    __syncwarp();
    recs[lane] = RecDesc{h.w, mask, h.z, h.x};
    // exclusive scan of the four packed 8-bit counts (sums stay <= 128)
    uint32_t incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(FULL, incl, o);
      if (lane >= o) incl += t;
    }
    const uint32_t tot = __shfl_sync(FULL, incl, 31);
    const uint32_t excl = incl - cnt;
    const uint32_t n32 = tot & 0xFFu, n64 = (tot >> 8) & 0xFFu, n16 = (tot >> 16) & 0xFFu, nb16 = tot >> 24;
    if (cnt != 0u) {
      const uint32_t fmt = fmt_of(h.z);
      const uint32_t my = (cnt >> (8 * fmt)) & 0xFFu;
      const uint32_t seg = fmt == 0u ? 0u : fmt == 1u ? n32 : fmt == 2u ? n32 + n64 : n32 + n64 + n16;
      const uint32_t at = seg + ((excl >> (8 * fmt)) & 0xFFu);
      const uint32_t step = fmt == FPX_FP64 ? 2u : 1u;
      for (uint32_t k = 0; k < my; ++k) items[at + k] = make_uint2(h.w + k * step, mask);
    }
    const bool force_any = __any_sync(FULL, force);
    __syncwarp();

    // ---- fast path: min / max witnesses per format ---------------------------
    uint32_t mn32 = 0xFFFFFFFFu, mx32 = 0u, mn64 = 0xFFFFFFFFu, mx64 = 0u;
    uint32_t mn16 = 0xFFFFFFFFu, mx16 = 0u, mnb = 0xFFFFFFFFu, mxb = 0u;
    for (uint32_t i = 0; i < n32; i += U32) {
      uint32_t w[U32], m[U32];
#pragma unroll
      for (int u = 0; u < U32; ++u) {
        m[u] = 0u;
        w[u] = 0u;
        if (i + u < n32) {
          const uint2 it = items[i + u];
          m[u] = it.y;
          w[u] = ld_stream(lane_base + (uint64_t)it.x * 32);
        }
      }
#pragma unroll
      for (int u = 0; u < U32; ++u) {
        const uint32_t a = w[u] & 0x7FFFFFFFu & lane_ext(m[u], lane);
        mn32 = min(mn32, a - 1u);  // < 0x7FFFFF  <=> subnormal
        mx32 = max(mx32, a);       // > 0x7F7FFFFF <=> INF / NaN
      }
    }
    for (uint32_t i = 0; i < n64; i += U64) {
      uint32_t lo[U64], hi[U64], m[U64];
#pragma unroll
      for (int u = 0; u < U64; ++u) {
        m[u] = 0u;
        lo[u] = 0u;
        hi[u] = 0u;
        if (i + u < n64) {
          const uint2 it = items[n32 + i + u];
          m[u] = it.y;
          const uint32_t* p = lane_base + (uint64_t)it.x * 32;
          lo[u] = ld_stream(p);
          hi[u] = ld_stream(p + 32);
        }
      }
#pragma unroll
      for (int u = 0; u < U64; ++u) {
        const uint32_t e = lane_ext(m[u], lane);
        const uint32_t ah = hi[u] & 0x7FFFFFFFu & e;
        const uint32_t a2 = (ah << 1) | min(lo[u] & e, 1u);  // 0 zero, [1,0x1FFFFF] SUB, >=0xFFE00000 INF/NaN
        mn64 = min(mn64, a2 - 1u);
        mx64 = max(mx64, a2);
      }
    }
    for (uint32_t i = 0; i < n16 + nb16; i += U32) {
      uint32_t w[U32], m[U32];
#pragma unroll
      for (int u = 0; u < U32; ++u) {
        m[u] = 0u;
        w[u] = 0u;
        if (i + u < n16 + nb16) {
          const uint2 it = items[n32 + n64 + i + u];
          m[u] = it.y;
          w[u] = ld_stream(lane_base + (uint64_t)it.x * 32);
        }
      }
#pragma unroll
      for (int u = 0; u < U32; ++u) {
        const uint32_t x = w[u] & 0x7FFF7FFFu & lane_ext(m[u], lane);
        const uint32_t l = x & 0xFFFFu, hh = x >> 16;
        if (i + u < n16) {
          mn16 = min(mn16, min(l - 1u, hh - 1u));
          mx16 = max(mx16, max(l, hh));
        } else {
          mnb = min(mnb, min(l - 1u, hh - 1u));
          mxb = max(mxb, max(l, hh));
        }
      }
    }
    const bool hit = mn32 < 0x007FFFFFu || mx32 > 0x7F7FFFFFu || mn64 < 0x001FFFFFu || mx64 >= 0xFFE00000u ||
                     mn16 < 0x03FFu || mx16 > 0x7BFFu || mnb < 0x007Fu || mxb > 0x7F7Fu;
    if (__any_sync(FULL, hit) || force_any) exact_tile<MODE>(recs, lane_base, lane, base_index + tile * TILE, tv);
  }
}


// Launch-shape knobs.  The product build uses the A/B-chosen constants; a
// tuning build (-DFPX_TUNING, tools/ab_env.sh / ab_sched.sh only) reads them
// once from the environment: FPX_RING (ring geometry), FPX_SCHED (0 static
// ranges only, 2 no one-tile chunks), FPX_STATIC_PCT, FPX_DYN_CHUNK,
// FPX_TAIL_TILES.
struct Tuning {
  int ring = -1;  // -1: by trace size
  int sched = 1;
  int static_pct = -1;  // -1: by mode (kStaticPct / kStaticPctFlow)
  uint32_t dyn_chunk = 0, tail_tiles = kTailTiles;  // dyn_chunk 0: by mode
};
#ifdef FPX_TUNING
Tuning read_tuning() {
  Tuning t;
  if (const char* e = getenv("FPX_RING")) t.ring = atoi(e);
  if (const char* e = getenv("FPX_SCHED")) t.sched = atoi(e);
  if (const char* e = getenv("FPX_STATIC_PCT")) t.static_pct = std::max(0, std::min(100, atoi(e)));
  if (const char* e = getenv("FPX_DYN_CHUNK")) t.dyn_chunk = (uint32_t)(std::max(1, atoi(e) / TILE) * TILE);
  if (const char* e = getenv("FPX_TAIL_TILES")) t.tail_tiles = (uint32_t)std::max(0, atoi(e));
  return t;
}
const Tuning& tuning() {
  static const Tuning t = read_tuning();  // thread-safe initialisation (C++11 magic static)
  return t;
}
#else
const Tuning& tuning() {
  static const Tuning t;
  return t;
}
#endif

template <int MODE>
cudaError_t launch_records_t(const fpx_rec_hdr* d_hdr, uint64_t n, const uint32_t* d_arena, uint64_t arena_planes,
                             uint64_t base_index, const TableView& tv, int num_sms, uint32_t variant,
                             unsigned int* sched_ctr, const FeedbackPtrs& fbp, bool storm, cudaStream_t s) {
  if (variant == 1u) {
    const uint64_t tiles = (n + TILE - 1) / TILE;
    uint64_t blocks = (tiles + LDG_WARPS - 1) / LDG_WARPS;
    const uint64_t cap = (uint64_t)num_sms * 4;
    if (blocks > cap) blocks = cap;
    k_scan_records_ldg<MODE><<<(unsigned)blocks, LDG_WARPS * 32, 0, s>>>(reinterpret_cast<const uint4*>(d_hdr), n,
                                                                         d_arena, arena_planes, base_index, tv);
    return cudaGetLastError();
  }
  // Ring geometry, from interleaved A/B runs on B200 (tools/ab_env.sh,
  // profiles/r1/ab_rings.txt): 20 warps x 2 stages x 40 planes by default;
  // 12-warp rings with 64-plane or 3-deep stages lose 10-15 %.
  // The 24-warp ring for small traces, which are latency-bound: every warp
  // gets at most one tile up to 24 x 32 records per SM (C1: 30 us instead of
  // 45 us).  On large one-plane traces the 20-warp ring wins C5 by 2.8 % (the
  // 24-warp build is capped at 80 registers and spills) and loses the 1 %
  // NaN storm S2 by 11 % (its exact path wants more warps): the common case
  // decides.
  const Tuning& tu = tuning();
  int ring = tu.ring;
  const bool small = n <= (uint64_t)num_sms * 24 * TILE;
  // one-plane DEST traces (an arena of at most 1.1 planes per record: FP32 /
  // packed scalar ops) fill only 32 of a 40-plane stage -- a tile holds at
  // most 32 records -- so they take the 24-warp x 32-plane ring: 20 % more
  // bytes in flight (C5 +2.1 %; multi-plane traces lose 3-6 % on it, C2 /
  // C4a: profiles/r2/ab_dest_ring3.txt).  Host-side, from the call's own
  // arguments; an arena with other data in it only keeps the default ring.
  const bool one_plane = MODE == FPX_MODE_DEST && FPX_ONE_PLANE_RING && arena_planes * 10 <= n * 11;
  if (ring < 0) ring = small || one_plane ? 3 : MODE == FPX_MODE_DEST ? FPX_DEST_RING : 1;
  if (tu.sched == 0) sched_ctr = nullptr;
  const int static_pct = tu.static_pct >= 0 ? tu.static_pct : MODE == FPX_MODE_DEST ? kStaticPct : kStaticPctFlow;
  const uint32_t chunk = tu.dyn_chunk ? tu.dyn_chunk : MODE == FPX_MODE_DEST ? kDynChunk : kDynChunkFlow;
  const SchedCfg scfg{static_pct, chunk, tu.sched == 2 ? 0u : tu.tail_tiles};
  const uint4* h4 = reinterpret_cast<const uint4*>(d_hdr);
  if constexpr (MODE == FPX_MODE_DEST) {
    if (storm) {  // the storm instantiation (CTA table, storm mode)
    // large traces: Ring5, 36-plane stages with the headers stashed in shared
    // memory (FPX_STORM_RING; the 24-warp Ring3 lost 6 % on both storms:
    // profiles/r2/ab_storm_ring.txt)
    if (tu.ring < 0) ring = small ? 3 : FPX_STORM_RING;
    switch (ring) {
      case 1: return launch_ring<MODE, Ring1, true>(h4, n, d_arena, arena_planes, base_index, tv, num_sms, sched_ctr, scfg, fbp, s);
      case 5: return launch_ring<MODE, Ring5, true>(h4, n, d_arena, arena_planes, base_index, tv, num_sms, sched_ctr, scfg, fbp, s);
      case 2: return launch_ring<MODE, Ring2, true>(h4, n, d_arena, arena_planes, base_index, tv, num_sms, sched_ctr, scfg, fbp, s);
      case 3: return launch_ring<MODE, Ring3, true>(h4, n, d_arena, arena_planes, base_index, tv, num_sms, sched_ctr, scfg, fbp, s);
      default: return launch_ring<MODE, Ring0, true>(h4, n, d_arena, arena_planes, base_index, tv, num_sms, sched_ctr, scfg, fbp, s);
      }
    }
  }
  // sparse kernels: new keys dominate their table updates (TV_CAS_FIRST)
  TableView tvs = tv;
  if (FPX_CAS_FIRST && !(tv.flags & FPX_OPT_NO_WARP_AGG)) tvs.flags |= TV_CAS_FIRST;
  switch (ring) {
    case 1:
      if constexpr (kEq<MODE, false>)
        return launch_ring<MODE, Ring1E, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
      return launch_ring<MODE, Ring1, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
    case 2: return launch_ring<MODE, Ring2, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
    case 3: return launch_ring<MODE, Ring3, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
    case 4:
      if constexpr (MODE == FPX_MODE_DEST && FPX_DEST_RING == 4)
        return launch_ring<MODE, Ring4, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
      [[fallthrough]];
    default: return launch_ring<MODE, Ring0, false>(h4, n, d_arena, arena_planes, base_index, tvs, num_sms, sched_ctr, scfg, fbp, s);
  }
}

}  // namespace

cudaError_t launch_scan_records(const fpx_rec_hdr* d_hdr, uint64_t n, const uint32_t* d_arena, uint64_t arena_planes,
                                uint64_t base_index, uint32_t mode, const TableView& tv, int num_sms, uint32_t variant,
                                unsigned int* sched_ctr, const FeedbackPtrs& fbp, bool storm, cudaStream_t s) {
  if (mode == FPX_MODE_DEST)
    return launch_records_t<FPX_MODE_DEST>(d_hdr, n, d_arena, arena_planes, base_index, tv, num_sms, variant, sched_ctr,
                                           fbp, storm, s);
  if (mode == FPX_MODE_FLOW)
    return launch_records_t<FPX_MODE_FLOW>(d_hdr, n, d_arena, arena_planes, base_index, tv, num_sms, variant, sched_ctr,
                                           fbp, false, s);
  return launch_records_t<FPX_MODE_FLOW_DETAIL>(d_hdr, n, d_arena, arena_planes, base_index, tv, num_sms, variant,
                                                sched_ctr, fbp, false, s);
}

}  // namespace fpx

#ifdef FPX_WARP_TIMES
// Copies the per-warp start / end times of the last record-scan launch
// (diagnostics build only; not part of include/fpx.h).
extern "C" __attribute__((visibility("default"))) int fpx_debug_warp_times(unsigned long long* t0,
                                                                            unsigned long long* t1, int n) {
  if (n > fpx::kMaxWarpTimes) n = fpx::kMaxWarpTimes;
  if (cudaMemcpyFromSymbol(t0, fpx::g_warp_t0, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(t1, fpx::g_warp_t1, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  return n;
}
extern "C" __attribute__((visibility("default"))) int fpx_debug_warp_exact(unsigned long long* hits,
                                                                            unsigned long long* ns, int n) {
  if (n > fpx::kMaxWarpTimes) n = fpx::kMaxWarpTimes;
  if (cudaMemcpyFromSymbol(hits, fpx::g_warp_hits, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(ns, fpx::g_warp_exact_ns, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  return n;
}
extern "C" __attribute__((visibility("default"))) int fpx_debug_warp_counts(unsigned long long* tiles,
                                                                             unsigned long long* chunks,
                                                                             unsigned long long* wait_ns, int n) {
  if (n > fpx::kMaxWarpTimes) n = fpx::kMaxWarpTimes;
  if (cudaMemcpyFromSymbol(tiles, fpx::g_warp_tiles, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(chunks, fpx::g_warp_chunks, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(wait_ns, fpx::g_warp_wait_ns, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  return n;
}
extern "C" __attribute__((visibility("default"))) int fpx_debug_warp_phases(unsigned long long* ph, int n) {
  if (n > fpx::kMaxWarpTimes) n = fpx::kMaxWarpTimes;
  if (cudaMemcpyFromSymbol(ph, fpx::g_phase_ns, 3 * n * sizeof(unsigned long long)) != cudaSuccess) return -1;
  return n;
}
#endif
