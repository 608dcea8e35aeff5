// fpx_records.cuh — record decoding, validation and the exact per-record
// evaluation shared by the record-scan kernels.
//
//   record_valid  the header contract of include/fpx.h
//   eval_record   one lane of one record, exactly: Alg1's kind dispatch
//                  on every destination value (detector) or the
//                 Table 2 state over dest + pre-execution sources
//                 (analyzer)
//   exact_tile    eval_record + warp aggregation + table update for every
//                 record of a tile (the rare path: tiles with an exception)
//   item_counts   planes of a record the fast path must look at, per format
#pragma once
#include "fpx_device.cuh"

namespace fpx {
#ifdef FPX_WARP_TIMES
// diagnostics build: per warp, ns in the FLOW exact path's prologue / record loop / final flush
__device__ unsigned long long g_phase_ns[3 * 148 * 32];
#endif
namespace rec {


constexpr int TILE = 32;  // records per warp tile (one header per lane)

struct alignas(16) RecDesc {
  uint32_t val_off, mask, meta, site;
};

__device__ __forceinline__ uint32_t op_of(uint32_t meta) { return meta & 0xFFu; }
__device__ __forceinline__ uint32_t fmt_of(uint32_t meta) { return (meta >> 8) & 3u; }
__device__ __forceinline__ uint32_t nsrc_of(uint32_t meta) { return (meta >> 10) & 3u; }
__device__ __forceinline__ uint32_t dwords_of(uint32_t meta) { return (meta >> 12) & 7u; }
__device__ __forceinline__ uint32_t sw_of(uint32_t fmt) { return fmt == FPX_FP64 ? 2u : 1u; }
__device__ __forceinline__ bool is_compare(uint32_t op) {
  return op == FPX_OP_FSETP || op == FPX_OP_DSETP || op == FPX_OP_FSET;
}

// Header validation (include/fpx.h record contract).
template <int MODE>
__device__ __forceinline__ bool record_valid(const uint4 h, uint64_t arena_planes) {
  const uint32_t meta = h.z, fmt = fmt_of(meta), dw = dwords_of(meta);
  bool ok = h.x != FPX_SITE_INVALID;
  ok &= (meta >> 15) == 0u;
  ok &= op_of(meta) < FPX_OP_COUNT;
  ok &= dw <= 4u;
  ok &= !(fmt == FPX_FP64 && (dw & 1u));
  const uint64_t planes = dw + (uint64_t)nsrc_of(meta) * sw_of(fmt);
  ok &= (uint64_t)h.w + planes <= arena_planes;
  if (MODE != FPX_MODE_DEST) {
    ok &= (fmt == FPX_FP32 || fmt == FPX_FP64);
    ok &= (dw == 0u || dw == sw_of(fmt));
  }
  return ok;
}

// Sign-extended "lane is active" mask: all ones if bit `lane` of m is set.
__device__ __forceinline__ uint32_t lane_ext(uint32_t m, int lane) {
  return (uint32_t)((int32_t)(m << (31 - lane)) >> 31);
}

// Destination kinds of one lane of a DEST-mode record: calls f(v, kind) for
// every destination value v whose Alg1 kind (dest_kind) is an exception.
// dv = destination words, sv = source words (only read when have_div).
template <typename F>
__device__ __forceinline__ void for_each_dest_kind(uint32_t op, uint32_t fmt, uint32_t dw, bool have_div,
                                                   const uint32_t dv[4], const uint32_t sv[6], F f) {
  const uint32_t nv = fmt == FPX_FP64 ? dw / 2 : fmt == FPX_FP32 ? dw : 2 * dw;
#pragma unroll
  for (uint32_t v = 0; v < 8; ++v) {
    if (v >= nv) break;
    uint32_t lo, hi = 0, nlo, nhi = 0, dlo, dhi = 0;  // value, dividend, divisor
    if (fmt == FPX_FP64) {
      lo = dv[(2 * v) & 3];
      hi = dv[(2 * v + 1) & 3];
      nlo = sv[0]; nhi = sv[1]; dlo = sv[2]; dhi = sv[3];
    } else if (fmt == FPX_FP32) {
      lo = dv[v & 3];
      nlo = sv[0]; dlo = sv[1];
    } else {
      const uint32_t sh = 16u * (v & 1u);
      lo = (dv[(v / 2) & 3] >> sh) & 0xFFFFu;
      nlo = (sv[0] >> sh) & 0xFFFFu;
      dlo = (sv[1] >> sh) & 0xFFFFu;
    }
    const int k = dest_kind(op, fmt, lo, hi, have_div, nlo, nhi, dlo, dhi);
    if (k >= 0) f(v, k);
  }
}

// Table 2's state of one lane-value of a scalar FP32 / FP64 record (FLOW
// modes): S = the most severe class among the pre-execution sources (NaN > INF
// > SUB, R5), src = the lowest-index source holding it (R21); D = the
// destination kind (dest_kind).  Returns flow << 2 | kind, or CODE_NONE.
__device__ __forceinline__ int flow_code(uint32_t op, uint32_t fmt, uint32_t nsrc, uint32_t dw, bool have_div,
                                         const uint32_t* dv, const uint32_t* sv, int& S, uint32_t& src) {
  S = CODE_NONE;
  src = 0;
  int sev = 0;
#pragma unroll
  for (uint32_t k = 0; k < 3; ++k) {
    if (k >= nsrc) break;
    const uint32_t c = fmt == FPX_FP64 ? cls_fp64(sv[2 * k], sv[2 * k + 1]) : cls_fp32(sv[k]);
    const int sv_ = c == CLS_NAN ? 3 : c == CLS_INF ? 2 : c == CLS_SUB ? 1 : 0;
    if (sv_ > sev) { sev = sv_; S = kind_of_cls(c); src = k; }
  }
  int D = CODE_NONE;
  if (dw != 0u) {
    if (fmt == FPX_FP64) D = dest_kind(op, fmt, dv[0], dv[1], have_div, sv[0], sv[1], sv[2], sv[3]);
    else D = dest_kind(op, fmt, dv[0], 0u, have_div, sv[0], 0u, sv[1], 0u);
  }
  if (D >= 0 && S < 0) return (FPX_GEN << 2) | D;
  if (D >= 0) return (FPX_PROP << 2) | D;
  if (S >= 0) return (FPX_KILL << 2) | S;
  return CODE_NONE;
}

// Exact evaluation of one record for this lane (both modes).  Returns the
// bitmask of event codes held by this lane; codes / evm describe per-value
// codes for count_of().
template <int MODE>
__device__ __forceinline__ uint32_t eval_record(const RecDesc& d, const uint32_t* __restrict__ lane_base, int lane,
                                                uint32_t& codes, uint32_t& evm, const uint32_t* staged = nullptr) {
  codes = 0;
  evm = 0;
  if (((d.mask >> lane) & 1u) == 0u) return 0u;
  const uint32_t op = op_of(d.meta), fmt = fmt_of(d.meta), nsrc = nsrc_of(d.meta), dw = dwords_of(d.meta);
  const uint32_t sw = sw_of(fmt);
  const bool have_div = (op == FPX_OP_DIV) && nsrc >= 2 && dw == sw;
  // destination words d[0..dw) and source words s[0..ns_words) of this lane
  uint32_t ns_words = 0;
  if (MODE != FPX_MODE_DEST) ns_words = nsrc * sw;
  else if (have_div) ns_words = 2 * sw;
  // `staged`: this lane's word of the record's first plane in the shared-memory
  // stage, which then holds every plane read below (no HBM re-read)
  const uint32_t* p = staged ? staged : lane_base + (uint64_t)d.val_off * 32;
  uint32_t dv[4], sv[6];
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) dv[k] = k < dw ? p[(uint64_t)k * 32] : 0u;
#pragma unroll
  for (uint32_t k = 0; k < 6; ++k) sv[k] = k < ns_words ? p[(uint64_t)(dw + k) * 32] : 0u;

  if (MODE == FPX_MODE_DEST) {
    uint32_t cm = 0;
    for_each_dest_kind(op, fmt, dw, have_div, dv, sv, [&](uint32_t v, int k) {
      codes |= (uint32_t)k << (4 * v);
      evm |= 1u << v;
      cm |= 1u << k;
    });
    return cm;
  } else {
    int S;
    uint32_t src;
    int code = flow_code(op, fmt, nsrc, dw, have_div, dv, sv, S, src);
    if (code < 0) return 0u;
    // FLOW_DETAIL: detail = 1 + src, | CMP for Table 1's control-flow opcodes (R22)
    if (MODE == FPX_MODE_FLOW_DETAIL && S >= 0) {
      const bool cf = op == FPX_OP_FSEL || op == FPX_OP_FSET || op == FPX_OP_FSETP || op == FPX_OP_FMNMX ||
                      op == FPX_OP_DSETP;
      code |= (int)((src + 1u) | (cf ? (uint32_t)FPX_DETAIL_CMP : 0u)) << 4;
    }
    codes = (uint32_t)code;
    evm = 1u;
    return 1u;
  }
}

// Exact evaluation + warp aggregation + table update of one record.
template <int MODE, typename Pend>
__device__ __forceinline__ void flush_record(const RecDesc& d, const uint32_t* __restrict__ lane_base, int lane,
                                             uint64_t gidx, const TableView& tv, Pend& pend,
                                             const uint32_t* staged = nullptr) {
  uint32_t codes, evm;
  const uint32_t cm = eval_record<MODE>(d, lane_base, lane, codes, evm, staged);
  if (tv.flags & FPX_OPT_NO_WARP_AGG) {  // ablation: no warp aggregation, every lane updates the table
    if (MODE != FPX_MODE_DEST) {
      if (cm) table_add(tv, make_key(d.site, fmt_of(d.meta), codes), 1u, gidx);  // one code per lane
      return;
    }
    uint32_t mine = cm;  // DEST: bit k = kind k among this lane's values
    while (mine) {
      const uint32_t c = (uint32_t)(__ffs(mine) - 1);
      mine &= mine - 1u;
      uint32_t n = 0u;
#pragma unroll
      for (int v = 0; v < 8; ++v) n += (((evm >> v) & 1u) && (((codes >> (4 * v)) & 15u) == c)) ? 1u : 0u;
      table_add(tv, make_key(d.site, fmt_of(d.meta), c), n, gidx);
    }
    return;
  }
  if (MODE == FPX_MODE_DEST) {
    warp_flush(tv, pend, cm, d.site, fmt_of(d.meta), gidx, [&](int c) {
      uint32_t n = 0;
#pragma unroll
      for (int v = 0; v < 8; ++v) n += (((evm >> v) & 1u) && (((codes >> (4 * v)) & 15u) == (uint32_t)c)) ? 1u : 0u;
      return n;
    });
  } else {
    warp_flush_single(tv, pend, cm ? (int)codes : CODE_NONE, d.site, fmt_of(d.meta), gidx);
  }
}

template <int MODE>
__device__ __noinline__ void exact_tile(const RecDesc* __restrict__ recs, const uint32_t* __restrict__ lane_base,
                                        int lane, uint64_t gidx0, const TableView tv) {
  PendingEvents<> pend;
  for (int j = 0; j < TILE; ++j) {
    const RecDesc d = recs[j];
    if (d.mask == 0u) continue;  // warp-uniform
    if (MODE == FPX_MODE_DEST && is_compare(op_of(d.meta))) continue;
    flush_record<MODE>(d, lane_base, lane, gidx0 + j, tv, pend);
  }
  pend.flush(tv);
}

// Same as exact_tile for the TMA ring: the tile's k headers are re-read from
// global memory, while every plane the mode needs is read from the tile's
// shared-memory stage (`stage_lane` = this lane's word of slot 0; a record's
// planes sit at the exclusive prefix sum of the needed-plane counts, exactly
// as the producer laid them out).  `needed(meta)` gives that count for a
// valid, active record (0 for DIV records, which the producer does not stage:
// their sources come from global memory).
template <int MODE, typename Needed>
__device__ __forceinline__ void exact_tile_records(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                            const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                            int lane, uint64_t gidx0, const TableView tv, bool warm, Needed needed) {
  uint4 h = make_uint4(0u, 0u, 0u, 0u);
  if ((uint32_t)lane < k) h = hdr_tile[lane];
  const bool ok = (uint32_t)lane < k && record_valid<MODE>(h, arena_planes);
  const uint32_t mask = ok ? h.y : 0u;
  const uint32_t c = (ok && mask != 0u) ? needed(h.z) : 0u;
  uint32_t slot = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(FULL, slot, o);
    if (lane >= o) slot += t;
  }
  slot -= c;
  const uint32_t staged_slot = c != 0u ? slot : 0xFFFFFFFFu;
  PendingEvents<true> pend;
  pend.warm = warm;
  for (uint32_t j = 0; j < k; ++j) {
    const RecDesc d{__shfl_sync(FULL, h.w, j), __shfl_sync(FULL, mask, j), __shfl_sync(FULL, h.z, j),
                    __shfl_sync(FULL, h.x, j)};
    const uint32_t sl = __shfl_sync(FULL, staged_slot, j);
    if (d.mask == 0u) continue;  // warp-uniform
    if (MODE == FPX_MODE_DEST && is_compare(op_of(d.meta))) continue;
    flush_record<MODE>(d, lane_base, lane, gidx0 + j, tv, pend, sl != 0xFFFFFFFFu ? stage_lane + sl * 32 : nullptr);
  }
  pend.flush(tv);
}

// Class counts (NaN, INF, SUB) over the active lanes' values in the `dw`
// staged destination planes of this lane's record (plane 0 at shared
// address sp).  Each load reads 16 B = instrumented lanes 4v..4v+3, with v
// skewed by the lane so that each 8-lane phase of a warp's LDS.128 touches
// all 32 banks once.  Thresholds on doubled magnitudes (the sign drops out):
//   FP32  a = 2x:                 NaN a > 0xFF000000, INF a == 0xFF000000, SUB a - 2 < 0xFFFFFE
//   FP64  a = 2 hi + min(lo, 1):  NaN a > 0xFFE00000, INF a == 0xFFE00000, SUB a - 1 < 0x1FFFFF
//   FP16 / BF16 per half h = |x|: NaN h > E, INF h == E, SUB h - 1 < M (E, M = 0x7C00, 0x3FF / 0x7F80, 0x7F)
// (the same definitions as cls_*, §2.1).
// Class counting of 4 transformed values (a[k] -- see count_staged) of one
// quad whose activity bits are m4[3:0]: NaN a > E, INF a == E, SUB
// a - S0 < S1, each compare combined with the lane's activity predicate in
// the setp itself and counted with a predicated add (PTX: ~8 instructions
// per value instead of ~12 from the C++ form).
template <uint32_t E, uint32_t S0, uint32_t S1>
__device__ __forceinline__ void count4(const uint32_t (&a)[4], uint32_t m4, uint32_t& n_nan, uint32_t& n_inf,
                                       uint32_t& n_sub) {
  asm("{\n\t.reg .pred p0, p1, p2, p3, q;\n\t.reg .u32 t;\n\t"
      "and.b32 t, %3, 1;\n\tsetp.ne.u32 p0, t, 0;\n\t"
      "and.b32 t, %3, 2;\n\tsetp.ne.u32 p1, t, 0;\n\t"
      "and.b32 t, %3, 4;\n\tsetp.ne.u32 p2, t, 0;\n\t"
      "and.b32 t, %3, 8;\n\tsetp.ne.u32 p3, t, 0;\n\t"
#define FPX_COUNT1(R, P)                                                                           \
  "setp.gt.and.u32 q, " R ", %8, " P ";\n\t@q add.u32 %0, %0, 1;\n\t"                           \
  "setp.eq.and.u32 q, " R ", %8, " P ";\n\t@q add.u32 %1, %1, 1;\n\t"                           \
  "sub.u32 t, " R ", %9;\n\tsetp.lt.and.u32 q, t, %10, " P ";\n\t@q add.u32 %2, %2, 1;\n\t"
      FPX_COUNT1("%4", "p0") FPX_COUNT1("%5", "p1") FPX_COUNT1("%6", "p2") FPX_COUNT1("%7", "p3")
#undef FPX_COUNT1
      "}"
      : "+r"(n_nan), "+r"(n_inf), "+r"(n_sub)
      : "r"(m4), "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "n"(E), "n"(S0), "n"(S1));
}

// FP32 class counting of 4 raw words (no doubling): NaN by an unordered
// float compare of x with itself, INF by |x| == +INF (float compares do not
// flush subnormals without .ftz), SUB by x + x - 2 < 0xFFFFFE (one IADD3):
// ~7 instructions per value instead of ~8 (storms).
__device__ __forceinline__ void count4_fp32(const uint4 x, uint32_t m4, uint32_t& n_nan, uint32_t& n_inf,
                                            uint32_t& n_sub) {
  asm("{\n\t.reg .pred p0, p1, p2, p3, q;\n\t.reg .u32 t;\n\t.reg .f32 f;\n\t"
      "and.b32 t, %3, 1;\n\tsetp.ne.u32 p0, t, 0;\n\t"
      "and.b32 t, %3, 2;\n\tsetp.ne.u32 p1, t, 0;\n\t"
      "and.b32 t, %3, 4;\n\tsetp.ne.u32 p2, t, 0;\n\t"
      "and.b32 t, %3, 8;\n\tsetp.ne.u32 p3, t, 0;\n\t"
#define FPX_COUNT1F(R, P)                                                                    \
  "mov.b32 f, " R ";\n\tsetp.nan.and.f32 q, f, f, " P ";\n\t@q add.u32 %0, %0, 1;\n\t"     \
  "abs.f32 f, f;\n\tsetp.eq.and.f32 q, f, 0f7F800000, " P ";\n\t@q add.u32 %1, %1, 1;\n\t" \
  "add.u32 t, " R ", " R ";\n\tadd.u32 t, t, -2;\n\t"                                         \
  "setp.lt.and.u32 q, t, 0x00FFFFFE, " P ";\n\t@q add.u32 %2, %2, 1;\n\t"
      FPX_COUNT1F("%4", "p0") FPX_COUNT1F("%5", "p1") FPX_COUNT1F("%6", "p2") FPX_COUNT1F("%7", "p3")
#undef FPX_COUNT1F
      "}"
      : "+r"(n_nan), "+r"(n_inf), "+r"(n_sub)
      : "r"(m4), "r"(x.x), "r"(x.y), "r"(x.z), "r"(x.w));
}
#ifndef FPX_COUNT_FP
#define FPX_COUNT_FP 1
#endif
#ifndef FPX_COUNT_UNROLL
#define FPX_COUNT_UNROLL 4  // quads per unrolled step of the transposed class count
#endif
constexpr int kCountUnroll = FPX_COUNT_UNROLL;

template <uint32_t FMT>
__device__ __forceinline__ void count_staged(uint32_t sp, uint32_t dw, uint32_t mask, uint32_t lane, uint32_t& n_nan,
                                             uint32_t& n_inf, uint32_t& n_sub) {
  constexpr uint32_t STEP = FMT == FPX_FP64 ? 2u : 1u;
  for (uint32_t w = 0; w < dw; w += STEP) {
#pragma unroll kCountUnroll
    for (uint32_t u = 0; u < 8; ++u) {
      const uint32_t v = (u + lane) & 7u;
      const uint32_t m4 = mask >> (4u * v);
      const uint4 x = sh_ld4(sp + w * 128u + v * 16u);
      if (FMT == FPX_FP32 && FPX_COUNT_FP) {
        count4_fp32(x, m4, n_nan, n_inf, n_sub);
      } else if (FMT == FPX_FP32) {
        const uint32_t a[4] = {x.x + x.x, x.y + x.y, x.z + x.z, x.w + x.w};
        count4<0xFF000000u, 2u, 0x00FFFFFEu>(a, m4, n_nan, n_inf, n_sub);
      } else if (FMT == FPX_FP64) {
        const uint4 y = sh_ld4(sp + (w + 1u) * 128u + v * 16u);
        const uint32_t a[4] = {y.x * 2u + min(x.x, 1u), y.y * 2u + min(x.y, 1u), y.z * 2u + min(x.z, 1u),
                               y.w * 2u + min(x.w, 1u)};
        count4<0xFFE00000u, 1u, 0x001FFFFFu>(a, m4, n_nan, n_inf, n_sub);
      } else {
        constexpr uint32_t E = FMT == FPX_FP16 ? 0x7C00u : 0x7F80u, M = FMT == FPX_FP16 ? 0x03FFu : 0x007Fu;
        // the two halves of a word share its activity bit: count the low
        // halves of words 0-1 and the high halves as a quad with m4 bits doubled
        const uint32_t m01 = (m4 & 1u) | ((m4 & 1u) << 1) | ((m4 & 2u) << 1) | ((m4 & 2u) << 2);
        const uint32_t m23 = ((m4 >> 2) & 1u) | (((m4 >> 2) & 1u) << 1) | ((m4 & 8u) >> 1) | (m4 & 8u);
        const uint32_t h01[4] = {x.x & 0x7FFFu, (x.x >> 16) & 0x7FFFu, x.y & 0x7FFFu, (x.y >> 16) & 0x7FFFu};
        count4<E, 1u, M>(h01, m01, n_nan, n_inf, n_sub);
        const uint32_t h23[4] = {x.z & 0x7FFFu, (x.z >> 16) & 0x7FFFu, x.w & 0x7FFFu, (x.w >> 16) & 0x7FFFu};
        count4<E, 1u, M>(h23, m23, n_nan, n_inf, n_sub);
      }
    }
  }
}

// One record evaluated from global memory (a recorded division, whose
// sources the producer does not stage), out of line: rare, and kept out of
// the lean FLOW path's register budget.
template <int MODE>
__device__ __noinline__ void flush_record_global(const RecDesc d, const uint32_t* __restrict__ lane_base, int lane,
                                                 uint64_t gidx, const TableView tv, bool warm) {
  PendingEvents<true> pend;
  pend.warm = warm;
  flush_record<MODE>(d, lane_base, lane, gidx, tv, pend, nullptr);
  pend.flush(tv);
}

// The analyzer's exact path of a TMA tile (FLOW / FLOW_DETAIL, with warp
// aggregation): record by record as the state of each lane depends on its
// own destination and sources (Table 2), but lean: header fields
// broadcast once, the planes read straight from the stage with LDS (lane l
// reads its own word: conflict-free), the class / severity / kind rules
// specialised per format, one code per lane, then Alg2's warp reduction per
// distinct code (warp_flush_single).  Same result as exact_tile_records
// (flow_code), ~4x fewer instructions per record: a NaN storm late in a
// warp's work no longer keeps it busy long after the others (the C3 tail).
// Records whose planes are not staged (recorded divisions, R1) take the
// generic flush_record from global memory.
// Q: the table updates go to the CTA's drain warp (eq_push) -- the caller's
// kernel runs one.
template <int MODE, bool Q = false, typename Needed>
__device__ __forceinline__ void exact_tile_flow(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                                const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                                int lane, uint64_t gidx0, const TableView tv, bool warm,
                                                Needed needed) {
#ifdef FPX_WARP_TIMES
  unsigned long long tph0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tph0));
#endif
  uint4 h = make_uint4(0u, 0u, 0u, 0u);
  if ((uint32_t)lane < k) h = hdr_tile[lane];
  const bool ok = (uint32_t)lane < k && record_valid<MODE>(h, arena_planes);
  const uint32_t mask = ok ? h.y : 0u;
  const uint32_t c = (ok && mask != 0u) ? needed(h.z) : 0u;
  uint32_t slot = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(FULL, slot, o);
    if (lane >= o) slot += t;
  }
  slot -= c;
#ifdef FPX_WARP_TIMES
  unsigned long long tph1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tph1));
#endif
  // per record, packed: stage slot (bits 0-7, 0xFF = not staged) | meta << 8
  // (meta < 2^15 for a valid record)
  const uint32_t packed = (c != 0u ? slot : 0xFFu) | (h.z << 8);
  const uint32_t sbase = sh_addr(stage_lane);  // this lane's word of stage slot 0
  PendingEvents<true, Q> pend;
  pend.warm = warm;
  uint32_t todo = __ballot_sync(FULL, mask != 0u);
  while (todo) {
    const uint32_t j = (uint32_t)(__ffs(todo) - 1);
    todo &= todo - 1u;
    const uint32_t pk = __shfl_sync(FULL, packed, j), m = __shfl_sync(FULL, mask, j);
    const uint32_t site = __shfl_sync(FULL, h.x, j);
    const uint32_t meta = pk >> 8, sl = pk & 0xFFu;
    if (sl == 0xFFu) {  // not staged: a recorded division (or no planes at all)
      const RecDesc d{__shfl_sync(FULL, h.w, j), m, meta, site};
      pend.flush(tv);  // keep the events in record order (PendingEvents merges neighbours)
      flush_record_global<MODE>(d, lane_base, lane, gidx0 + j, tv, warm);
      continue;
    }
    const uint32_t op = op_of(meta), fmt = fmt_of(meta), ns = nsrc_of(meta), dw = dwords_of(meta);
    const uint32_t a = sbase + sl * 128u;  // this lane's word of the record's plane 0
    // S: most severe source class (NaN > INF > SUB, R5), src: lowest index holding it (R21)
    uint32_t sev = 0u, src = 0u, dcls = CLS_CLEAN;
    if (fmt == FPX_FP64) {
      for (uint32_t q = 0; q < ns; ++q) {
        const uint32_t lo = sh_ld1(a + (dw + 2u * q) * 128u), hi = sh_ld1(a + (dw + 2u * q + 1u) * 128u);
        const uint32_t cl = cls_fp64(lo, hi), sv = cl == CLS_CLEAN ? 0u : 4u - cl;
        if (sv > sev) sev = sv, src = q;
      }
      if (dw != 0u) dcls = cls_fp64(sh_ld1(a), sh_ld1(a + 128u));
    } else {
      for (uint32_t q = 0; q < ns; ++q) {
        const uint32_t cl = cls_fp32(sh_ld1(a + (dw + q) * 128u)), sv = cl == CLS_CLEAN ? 0u : 4u - cl;
        if (sv > sev) sev = sv, src = q;
      }
      if (dw != 0u) dcls = cls_fp32(sh_ld1(a));
    }
    // D: Alg1's dispatch (dest_kind): RCP -> DIV0 iff NaN / INF; compares: none
    int D = CODE_NONE;
    if (op == FPX_OP_MUFU_RCP || op == FPX_OP_MUFU_RCP64H) D = (dcls == CLS_NAN || dcls == CLS_INF) ? FPX_DIV0 : CODE_NONE;
    else if (!is_compare(op)) D = kind_of_cls(dcls);
    // Table 2: GEN / PROP / KILL (the kind of a KILL is the source's, 4 - sev - 1)
    int code = CODE_NONE;
    if (D >= 0) code = ((sev ? FPX_PROP : FPX_GEN) << 2) | D;
    else if (sev) code = (FPX_KILL << 2) | (int)(3u - sev);
    if (MODE == FPX_MODE_FLOW_DETAIL && sev && code >= 0) {
      const bool cf = op == FPX_OP_FSEL || op == FPX_OP_FSET || op == FPX_OP_FSETP || op == FPX_OP_FMNMX ||
                      op == FPX_OP_DSETP;
      code |= (int)((src + 1u) | (cf ? (uint32_t)FPX_DETAIL_CMP : 0u)) << 4;
    }
    if (((m >> lane) & 1u) == 0u) code = CODE_NONE;
    warp_flush_single(tv, pend, code, site, fmt, gidx0 + j);
  }
#ifdef FPX_WARP_TIMES
  unsigned long long tph2, tph3;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tph2));
#endif
  pend.flush(tv);
#ifdef FPX_WARP_TIMES
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tph3));
  if (lane == 0) {
    // scan warps per CTA (the analyzer kernels' last warp drains the event queue)
    const uint64_t gw = blockIdx.x * (uint64_t)(blockDim.x / 32 - 1) + threadIdx.x / 32;
    if (gw < 148 * 32) {
      g_phase_ns[3 * gw] += tph1 - tph0;
      g_phase_ns[3 * gw + 1] += tph2 - tph1;
      g_phase_ns[3 * gw + 2] += tph3 - tph2;
    }
  }
#endif
}

// DEST-mode exact path of a TMA tile, transposed: lane j evaluates ALL lanes of
// record j (the k <= 32 records at once) instead of the warp walking the
// records one by one; then records with equal keys are combined across the
// warp (Alg2's warp reduction, over records instead of lanes:
// __match_any_sync + REDUX) and every group leader updates the table, all in
// parallel.  Same table as exact_tile_records: count = lane-values per key,
// first = the smallest record index of the group (lanes are in record order).
// Shared-memory reads are skewed (lane j reads instrumented lane (t + j) mod
// 32 at step t) so the 32 lanes hit 32 different banks.  `h`, `c`, `slot`:
// this lane's header, staged planes and stage slot.
__device__ __forceinline__ bool exact_tile_transposed(const uint4 h, uint32_t mask, uint32_t c, uint32_t slot,
                                                      const uint32_t* __restrict__ arena, const uint32_t* stage,
                                                      int lane, uint64_t gidx0, const TableView& tv, bool warm) {
  // group leaders' updates go through the CTA table when there is one
  bool dense = false;  // set below, warp-uniform: warm and records of the tile with an event >= kDenseEvents
  auto emit = [&](unsigned long long key, uint32_t cnt_, unsigned long long f) { emit_event(tv, key, cnt_, f, dense); };
  const uint32_t op = op_of(h.z), fmt = fmt_of(h.z), nsrc = nsrc_of(h.z), dw = dwords_of(h.z);
  const uint32_t sw = sw_of(fmt);
  const bool have_div = (op == FPX_OP_DIV) && nsrc >= 2 && dw == sw;
  // per-kind lane-value counts of this record, 16 bits each (<= 32 lanes x 8 values)
  unsigned long long cnt = 0ull;
  if (mask != 0u && dw != 0u && !is_compare(op)) {
    // plane 0 of the record: staged (c != 0) or in global memory (DIV records)
    const uint32_t* p = c != 0u ? stage + slot * 32 : arena + (uint64_t)h.w * 32;
    if (have_div) {
      // a recorded division with its operands (R1): the full per-value rule
      const uint32_t ns_words = 2 * sw;
      for (uint32_t t = 0; t < 32; ++t) {
        const uint32_t i = (t + (uint32_t)lane) & 31u;
        if (((mask >> i) & 1u) == 0u) continue;
        uint32_t dv[4], sv[6];
#pragma unroll
        for (uint32_t w = 0; w < 4; ++w) dv[w] = w < dw ? p[w * 32 + i] : 0u;
#pragma unroll
        for (uint32_t w = 0; w < 6; ++w) sv[w] = w < ns_words ? p[(dw + w) * 32 + i] : 0u;
        for_each_dest_kind(op, fmt, dw, have_div, dv, sv, [&](uint32_t, int kd) { cnt += 1ull << (16 * kd); });
      }
    } else {
      // Every other opclass maps the destination CLASS to a kind per record
      // (dest_kind: RCP -> DIV0 for NaN / INF, nothing for SUB; else the
      // class), so the loop only counts classes, per format (lanes of one
      // format run together).
      uint32_t n_nan = 0u, n_inf = 0u, n_sub = 0u;
      if (c != 0u) {
        // staged planes: 16 B per load (count_staged)
        const uint32_t sp = sh_addr(stage) + slot * 128u;
        switch (fmt) {
          case FPX_FP32: count_staged<FPX_FP32>(sp, dw, mask, (uint32_t)lane, n_nan, n_inf, n_sub); break;
          case FPX_FP64: count_staged<FPX_FP64>(sp, dw, mask, (uint32_t)lane, n_nan, n_inf, n_sub); break;
          case FPX_FP16: count_staged<FPX_FP16>(sp, dw, mask, (uint32_t)lane, n_nan, n_inf, n_sub); break;
          default: count_staged<FPX_BF16>(sp, dw, mask, (uint32_t)lane, n_nan, n_inf, n_sub);
        }
      } else {
        // planes in global memory (a recorded division whose destination is
        // not one source wide, R19: not staged): the plain per-value class
        for (uint32_t t = 0; t < 32; ++t) {
          if (((mask >> t) & 1u) == 0u) continue;
          for (uint32_t w = 0; w < dw; w += fmt == FPX_FP64 ? 2u : 1u) {
            const uint32_t lo = p[w * 32 + t], hi = fmt == FPX_FP64 ? p[(w + 1) * 32 + t] : 0u;
            for (uint32_t hv = 0; hv < (fmt >= FPX_FP16 ? 2u : 1u); ++hv) {
              const uint32_t cl = cls_val(fmt, fmt >= FPX_FP16 ? (lo >> (16 * hv)) & 0xFFFFu : lo, hi);
              n_nan += cl == CLS_NAN;
              n_inf += cl == CLS_INF;
              n_sub += cl == CLS_SUB;
            }
          }
        }
      }
      if (op == FPX_OP_MUFU_RCP || op == FPX_OP_MUFU_RCP64H)
        cnt = (unsigned long long)(n_nan + n_inf) << (16 * FPX_DIV0);
      else
        cnt = (unsigned long long)n_nan << (16 * FPX_NAN) | (unsigned long long)n_inf << (16 * FPX_INF) |
              (unsigned long long)n_sub << (16 * FPX_SUB);
    }
  }
  uint32_t present = 0u;
#pragma unroll
  for (int kd = 0; kd < 4; ++kd) present |= ((cnt >> (16 * kd)) & 0xFFFFu) ? 1u << kd : 0u;
  // Group per kind, then issue every group's table update at once: a leader
  // parks its sums (one per kind it leads) and the updates of different kinds
  // and records run in parallel instead of one warp-wide round per kind (C1
  // +11 %).  A single kind (storms) updates right away (S2 -2 % otherwise).
  dense = warm && __popc(__ballot_sync(FULL, present != 0u)) >= kDenseEvents;
  if (dense) {
    // a warm warp in a storm: every record's per-kind counts go straight to
    // the CTA table, whose shared-memory atomics merge equal keys -- no warp
    // grouping (a segmented REDUX over many distinct peer groups is a loop)
    if (present) emit_kinds_cta(tv, h.x, fmt, present, cnt, gidx0 + (uint64_t)lane);
    return true;
  }
  uint32_t all = __reduce_or_sync(FULL, present), lead = 0u;
  if (__popc(all) == 1) {
    const uint32_t kd = (uint32_t)(__ffs(all) - 1);
    const bool has = present != 0u;
    const unsigned long long key = has ? make_key(h.x, fmt, kd) : FPX_KEY_EMPTY - (unsigned long long)lane;
    const uint32_t peers = __match_any_sync(FULL, key);
    if (has) {
      const uint32_t sum = __reduce_add_sync(peers, (uint32_t)((cnt >> (16 * kd)) & 0xFFFFu));
      if ((uint32_t)lane == (uint32_t)(__ffs(peers) - 1)) emit(key, sum, gidx0 + (uint64_t)lane);
    }
    return false;
  }
  unsigned long long sums = 0ull;  // 16 bits per kind led by this lane
  while (all) {
    const uint32_t kd = (uint32_t)(__ffs(all) - 1);
    all &= all - 1u;
    const bool has = (present >> kd) & 1u;
    // lanes without this kind get lane-unique keys no record can have
    const unsigned long long key = has ? make_key(h.x, fmt, kd) : FPX_KEY_EMPTY - (unsigned long long)lane;
    const uint32_t peers = __match_any_sync(FULL, key);
    if (has) {
      const uint32_t sum = __reduce_add_sync(peers, (uint32_t)((cnt >> (16 * kd)) & 0xFFFFu));
      if ((uint32_t)lane == (uint32_t)(__ffs(peers) - 1)) {
        lead |= 1u << kd;
        sums |= (unsigned long long)sum << (16 * kd);
      }
    }
  }
  while (lead) {
    const uint32_t kd = (uint32_t)(__ffs(lead) - 1);
    lead &= lead - 1u;
    emit(make_key(h.x, fmt, kd), (uint32_t)((sums >> (16 * kd)) & 0xFFFFu), gidx0 + (uint64_t)lane);
  }
  return false;
}

// Exact path of a hit TMA tile: DEST mode goes transposed
// (exact_tile_transposed; a tile mixing formats runs each present format's
// class loop in turn, still far cheaper than walking the records), the
// analyzer modes and the no-aggregation ablation record by record
// (exact_tile_records).  A transposed FLOW path (lane groups per record,
// (destination, source) severity bins) was tried and lost 1.7-2.3x on
// storm-heavy FLOW traces: FLOW tiles hold ~10 records, so most lanes idle,
// and per-record operand counts and formats diverge inside the loop
// (profiles/r1/ab_sched.txt).  A/B in profiles/r1/ab_producer.txt (ab9-ab16).
// Table updates go through emit_event (the CTA pre-aggregation table, if the
// kernel set one up, then the device table).
// Returns whether the tile was dense (DEST transposed path, warm warp).
// `pre`: this lane's header, already loaded by the caller (nullptr: load it).
template <int MODE, typename Needed>
__device__ __forceinline__ bool exact_tile_hdr(const uint4* __restrict__ hdr_tile, uint32_t k, uint64_t arena_planes,
                                            const uint32_t* __restrict__ lane_base, const uint32_t* stage_lane,
                                            int lane, uint64_t gidx0, const TableView tv, bool warm, Needed needed,
                                            const uint4* pre = nullptr) {
  if (MODE == FPX_MODE_DEST && !(tv.flags & FPX_OPT_NO_WARP_AGG)) {
    uint4 h = make_uint4(0u, 0u, 0u, 0u);
    if (pre != nullptr) h = *pre;
    else if ((uint32_t)lane < k) h = hdr_tile[lane];
    const bool ok = (uint32_t)lane < k && record_valid<MODE>(h, arena_planes);
    const uint32_t mask = ok ? h.y : 0u;
    const uint32_t c = (ok && mask != 0u) ? needed(h.z) : 0u;
    uint32_t slot = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(FULL, slot, o);
      if (lane >= o) slot += t;
    }
    return exact_tile_transposed(h, mask, c, slot - c, lane_base - lane, stage_lane - lane, lane, gidx0, tv, warm);
  }
  exact_tile_records<MODE>(hdr_tile, k, arena_planes, lane_base, stage_lane, lane, gidx0, tv, warm, needed);
  return false;
}

// Plane items of one record for the fast path, by list:
//   0: FP32 words, 1: FP64 (lo, hi) pairs, 2: FP16x2 words, 3: BF16x2 words.
template <int MODE>
__device__ __forceinline__ uint32_t item_counts(uint32_t meta, bool ok, bool& force) {
  force = false;
  if (!ok) return 0u;
  const uint32_t op = op_of(meta), fmt = fmt_of(meta), dw = dwords_of(meta), ns = nsrc_of(meta);
  if (op == FPX_OP_DIV) { force = true; return 0u; }  // DIV0 needs the sources: exact path
  uint32_t n;
  if (MODE == FPX_MODE_DEST) {
    if (is_compare(op)) return 0u;
    n = fmt == FPX_FP64 ? dw / 2 : dw;
  } else {
    n = fmt == FPX_FP64 ? (dw + 2 * ns) / 2 : dw + ns;
  }
  return n << (8 * fmt);
}

}  // namespace rec
}  // namespace fpx
