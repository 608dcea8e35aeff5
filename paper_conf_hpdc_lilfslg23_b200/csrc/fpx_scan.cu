// fpx_scan.cu — the two scan kernels of the hot path (sm_100a).
//
// k_scan_records: one warp owns a tile of 32 consecutive
// records.  Lane l of the scanning warp reads lane l of every plane, exactly
// the lane of the instrumented warp whose register it holds (Alg2 P:249-281:
// "each thread checks its own value").
//   prologue  lane j decodes + validates header j, and flattens the planes the
//             mode needs into per-format item lists in shared memory
//             (FP32 words, FP64 (lo, hi) pairs, FP16x2 / BF16x2 words)
//   fast      each item is one coalesced 128-B warp load; a few integer ops
//             per value keep min / max witnesses of "subnormal" and
//             "exponent all ones"; one vote per tile decides if anything is
//             exceptional (the common case at 1e-6 density is "no")
//   exact     only for hit tiles: every record is re-read and evaluated with
//             the full kind rule (Alg1) and flow states (Table 2,
//             P:421-433), reduced per warp and written to the table
//
// k_scan_tensor: 128-bit loads of a plain buffer, unrolled,
// grid-stride over a persistent grid; one vote per unrolled batch, exact
// classification and warp reduction only on hit batches.
#include <cuda_runtime.h>

#include "fpx_device.cuh"

namespace fpx {
namespace {

constexpr int WARPS = 8;       // warps per block
constexpr int TILE = 32;       // records per warp tile (one header per lane)
constexpr int MAXITEMS = 128;  // <= 4 items per record
constexpr int U32 = 8;         // FP32 / packed items per load batch
constexpr int U64 = 4;         // FP64 pairs per load batch

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
  if (MODE == FPX_MODE_FLOW) {
    ok &= (fmt == FPX_FP32 || fmt == FPX_FP64);
    ok &= (dw == 0u || dw == sw_of(fmt));
  }
  return ok;
}

// Sign-extended "lane is active" mask: all ones if bit `lane` of m is set.
__device__ __forceinline__ uint32_t lane_ext(uint32_t m, int lane) {
  return (uint32_t)((int32_t)(m << (31 - lane)) >> 31);
}

// Exact evaluation of one record for this lane (both modes).  Returns the
// bitmask of event codes held by this lane; codes / evm describe per-value
// codes for count_of().
template <int MODE>
__device__ __forceinline__ uint32_t eval_record(const RecDesc& d, const uint32_t* __restrict__ lane_base, int lane,
                                                uint32_t& codes, uint32_t& evm) {
  codes = 0;
  evm = 0;
  if (((d.mask >> lane) & 1u) == 0u) return 0u;
  const uint32_t op = op_of(d.meta), fmt = fmt_of(d.meta), nsrc = nsrc_of(d.meta), dw = dwords_of(d.meta);
  const uint32_t sw = sw_of(fmt);
  const bool have_div = (op == FPX_OP_DIV) && nsrc >= 2 && dw == sw;
  // destination words d[0..dw) and source words s[0..ns_words) of this lane
  uint32_t ns_words = 0;
  if (MODE == FPX_MODE_FLOW) ns_words = nsrc * sw;
  else if (have_div) ns_words = 2 * sw;
  const uint32_t* p = lane_base + (uint64_t)d.val_off * 32;
  uint32_t dv[4], sv[6];
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) dv[k] = k < dw ? p[(uint64_t)k * 32] : 0u;
#pragma unroll
  for (uint32_t k = 0; k < 6; ++k) sv[k] = k < ns_words ? p[(uint64_t)(dw + k) * 32] : 0u;

  if (MODE == FPX_MODE_DEST) {
    const uint32_t nv = fmt == FPX_FP64 ? dw / 2 : fmt == FPX_FP32 ? dw : 2 * dw;
    uint32_t cm = 0;
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
      if (k >= 0) {
        codes |= (uint32_t)k << (4 * v);
        evm |= 1u << v;
        cm |= 1u << k;
      }
    }
    return cm;
  } else {
    // Analyzer: S = most severe class among the pre-execution sources.
    int S = CODE_NONE, sev = 0;
#pragma unroll
    for (uint32_t k = 0; k < 3; ++k) {
      if (k >= nsrc) break;
      const uint32_t c = fmt == FPX_FP64 ? cls_fp64(sv[2 * k], sv[2 * k + 1]) : cls_fp32(sv[k]);
      const int sv_ = c == CLS_NAN ? 3 : c == CLS_INF ? 2 : c == CLS_SUB ? 1 : 0;
      if (sv_ > sev) { sev = sv_; S = kind_of_cls(c); }
    }
    int D = CODE_NONE;
    if (dw != 0u) {
      if (fmt == FPX_FP64) D = dest_kind(op, fmt, dv[0], dv[1], have_div, sv[0], sv[1], sv[2], sv[3]);
      else D = dest_kind(op, fmt, dv[0], 0u, have_div, sv[0], 0u, sv[1], 0u);
    }
    int code = CODE_NONE;
    if (D >= 0 && S < 0) code = (FPX_GEN << 2) | D;
    else if (D >= 0) code = (FPX_PROP << 2) | D;
    else if (S >= 0) code = (FPX_KILL << 2) | S;
    if (code < 0) return 0u;
    codes = (uint32_t)code;
    evm = 1u;
    return 1u << code;
  }
}

template <int MODE>
__device__ __noinline__ void exact_tile(const RecDesc* __restrict__ recs, const uint32_t* __restrict__ lane_base,
                                        int lane, uint64_t gidx0, const TableView tv) {
  for (int j = 0; j < TILE; ++j) {
    const RecDesc d = recs[j];
    if (d.mask == 0u) continue;  // warp-uniform
    if (MODE == FPX_MODE_DEST && is_compare(op_of(d.meta))) continue;
    uint32_t codes, evm;
    const uint32_t cm = eval_record<MODE>(d, lane_base, lane, codes, evm);
    warp_flush(tv, cm, d.site, fmt_of(d.meta), gidx0 + j, [&](int c) {
      uint32_t n = 0;
#pragma unroll
      for (int v = 0; v < 8; ++v) n += (((evm >> v) & 1u) && (((codes >> (4 * v)) & 15u) == (uint32_t)c)) ? 1u : 0u;
      return n;
    });
  }
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

template <int MODE>
__global__ void __launch_bounds__(WARPS * 32, 4)
k_scan_records(const uint4* __restrict__ hdr, uint64_t n, const uint32_t* __restrict__ arena,
               uint64_t arena_planes, uint64_t base_index, const TableView tv) {
  __shared__ RecDesc s_rec[WARPS][TILE];
  __shared__ uint2 s_item[WARPS][MAXITEMS];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t nwarps = (uint64_t)gridDim.x * WARPS;
  const uint64_t ntiles = (n + TILE - 1) / TILE;
  const uint32_t* __restrict__ lane_base = arena + lane;
  RecDesc* __restrict__ recs = s_rec[warp];
  uint2* __restrict__ items = s_item[warp];

  uint64_t tile = blockIdx.x * (uint64_t)WARPS + warp;
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
    if (bad != 0u && lane == 0) atomicAdd(&tv.ctl->bad_records, (unsigned long long)__popc(bad));
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

// ---- tensor scan ---------------------------------------------------------------
template <uint32_t FMT>
struct TensorTraits;
template <>
struct TensorTraits<FPX_FP32> {
  static constexpr uint32_t V = 4;  // values per 16 B
};
template <>
struct TensorTraits<FPX_FP64> {
  static constexpr uint32_t V = 2;
};
template <>
struct TensorTraits<FPX_FP16> {
  static constexpr uint32_t V = 8;
};
template <>
struct TensorTraits<FPX_BF16> {
  static constexpr uint32_t V = 8;
};

// class of value e (0..V-1) of a 16-B vector
template <uint32_t FMT>
__device__ __forceinline__ uint32_t vec_cls(const uint4& q, uint32_t e) {
  const uint32_t w[4] = {q.x, q.y, q.z, q.w};
  if (FMT == FPX_FP32) return cls_fp32(w[e]);
  if (FMT == FPX_FP64) return cls_fp64(w[2 * e], w[2 * e + 1]);
  const uint32_t half = (w[e / 2] >> (16 * (e & 1))) & 0xFFFFu;
  return FMT == FPX_FP16 ? cls_fp16(half) : cls_bf16(half);
}

// Cheap "anything exceptional in this vector" witness update.
template <uint32_t FMT>
__device__ __forceinline__ void vec_witness(const uint4& q, uint32_t& mn, uint32_t& mx) {
  if (FMT == FPX_FP32) {
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint32_t a = w[k] & 0x7FFFFFFFu;
      mn = min(mn, a - 1u);
      mx = max(mx, a);
    }
  } else if (FMT == FPX_FP64) {
    const uint32_t lo[2] = {q.x, q.z}, hi[2] = {q.y, q.w};
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const uint32_t a2 = ((hi[k] & 0x7FFFFFFFu) << 1) | min(lo[k], 1u);
      mn = min(mn, a2 - 1u);
      mx = max(mx, a2);
    }
  } else {
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint32_t x = w[k] & 0x7FFF7FFFu;
      const uint32_t l = x & 0xFFFFu, h = x >> 16;
      mn = min(mn, min(l - 1u, h - 1u));
      mx = max(mx, max(l, h));
    }
  }
}
template <uint32_t FMT>
__device__ __forceinline__ bool witness_hit(uint32_t mn, uint32_t mx) {
  if (FMT == FPX_FP32) return mn < 0x007FFFFFu || mx > 0x7F7FFFFFu;
  if (FMT == FPX_FP64) return mn < 0x001FFFFFu || mx >= 0xFFE00000u;
  if (FMT == FPX_FP16) return mn < 0x03FFu || mx > 0x7BFFu;
  return mn < 0x007Fu || mx > 0x7F7Fu;
}

constexpr int TU = 4;  // vectors per thread per batch

// Exact per-warp reduction of per-lane kind counts and first offsets.
__device__ __forceinline__ void flush_kinds(const TableView& tv, uint32_t site, uint32_t fmt, const uint32_t cnt[3],
                                            const uint32_t first_off[3], uint64_t idx0) {
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const uint32_t tot = __reduce_add_sync(FULL, cnt[k]);
    if (tot) {
      const uint32_t f = __reduce_min_sync(FULL, first_off[k]);
      if ((threadIdx.x & 31) == 0) table_add(tv, make_key(site, fmt, (uint32_t)k), tot, idx0 + f);
    }
  }
}

static_assert(TU == 4, "tensor_exact takes four vectors");

// Exact classification of one hit batch (rare): offsets relative to the
// warp's lowest vector of the batch, reduced per warp.
template <uint32_t FMT>
__device__ __noinline__ void tensor_exact(uint4 q0, uint4 q1, uint4 q2, uint4 q3, uint64_t v0, uint64_t nthr,
                                          uint64_t nvec, int lane, uint64_t idx_base, uint32_t site,
                                          const TableView tv) {
  constexpr uint32_t V = TensorTraits<FMT>::V;
  const uint4 q[TU] = {q0, q1, q2, q3};
  const uint64_t wv0 = v0 - (uint64_t)lane;
  uint32_t cnt[3] = {0, 0, 0}, fo[3] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu};
#pragma unroll
  for (int u = 0; u < TU; ++u) {
    const uint64_t v = v0 + (uint64_t)u * nthr;
    if (v >= nvec) continue;
#pragma unroll
    for (uint32_t e = 0; e < V; ++e) {
      const int k = kind_of_cls(vec_cls<FMT>(q[u], e));
      const uint32_t off = (uint32_t)((v - wv0) * V + e);
#pragma unroll
      for (int kk = 0; kk < 3; ++kk)
        if (k == kk) { cnt[kk]++; fo[kk] = min(fo[kk], off); }
    }
  }
  flush_kinds(tv, site, FMT, cnt, fo, idx_base + wv0 * V);
}

template <uint32_t FMT>
__global__ void __launch_bounds__(256, 8)
k_scan_tensor(const uint4* __restrict__ body, uint64_t nvec, const uint8_t* __restrict__ scalars_lo,
              uint32_t n_head, const uint8_t* __restrict__ scalars_hi, uint32_t n_tail, uint64_t idx_body,
              uint64_t idx_tail, uint64_t base_index, uint32_t site, const TableView tv) {
  constexpr uint32_t V = TensorTraits<FMT>::V;
  constexpr uint32_t ES = 16 / V;
  const int lane = threadIdx.x & 31;
  const uint64_t nthr = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;

  // head / tail scalars (< one vector each): first warp of block 0, exact.
  if (blockIdx.x == 0 && threadIdx.x < 32) {
    auto one = [&](const uint8_t* q, uint32_t off, uint32_t cnt[3], uint32_t fo[3]) {
      uint32_t lo = 0, hi = 0;
      if (ES == 8) { lo = *(const uint32_t*)q; hi = *(const uint32_t*)(q + 4); }
      else if (ES == 4) lo = *(const uint32_t*)q;
      else lo = *(const uint16_t*)q;
      const int k = kind_of_cls(cls_val(FMT, lo, hi));
#pragma unroll
      for (int kk = 0; kk < 3; ++kk)
        if (k == kk) { cnt[kk]++; fo[kk] = min(fo[kk], off); }
    };
    uint32_t ch[3] = {0, 0, 0}, fh[3] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu};
    if ((uint32_t)lane < n_head) one(scalars_lo + (uint64_t)lane * ES, (uint32_t)lane, ch, fh);
    flush_kinds(tv, site, FMT, ch, fh, base_index);
    uint32_t ct[3] = {0, 0, 0}, ft[3] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu};
    if ((uint32_t)lane < n_tail) one(scalars_hi + (uint64_t)lane * ES, (uint32_t)lane, ct, ft);
    flush_kinds(tv, site, FMT, ct, ft, base_index + idx_tail);
  }

  // body: batches of TU vectors per thread, grid-stride
  for (uint64_t v0 = tid; v0 < nvec; v0 += nthr * TU) {
    uint4 q[TU];
#pragma unroll
    for (int u = 0; u < TU; ++u) {
      const uint64_t v = v0 + (uint64_t)u * nthr;
      q[u] = v < nvec ? ld_stream4(body + v) : make_uint4(0, 0, 0, 0);
    }
    uint32_t mn = 0xFFFFFFFFu, mx = 0u;
#pragma unroll
    for (int u = 0; u < TU; ++u) vec_witness<FMT>(q[u], mn, mx);
    if (__any_sync(FULL, witness_hit<FMT>(mn, mx)))
      tensor_exact<FMT>(q[0], q[1], q[2], q[3], v0, nthr, nvec, lane, base_index + idx_body, site, tv);
  }
}

template <int MODE>
cudaError_t launch_records_t(const fpx_rec_hdr* d_hdr, uint64_t n, const uint32_t* d_arena, uint64_t arena_planes,
                             uint64_t base_index, const TableView& tv, int num_sms, cudaStream_t s) {
  const uint64_t tiles = (n + TILE - 1) / TILE;
  uint64_t blocks = (tiles + WARPS - 1) / WARPS;
  const uint64_t cap = (uint64_t)num_sms * 4;
  if (blocks > cap) blocks = cap;
  k_scan_records<MODE><<<(unsigned)blocks, WARPS * 32, 0, s>>>(reinterpret_cast<const uint4*>(d_hdr), n, d_arena,
                                                               arena_planes, base_index, tv);
  return cudaGetLastError();
}

template <uint32_t FMT>
cudaError_t launch_tensor_t(const void* d_ptr, uint64_t n, uint32_t site, uint64_t base_index, const TableView& tv,
                            int num_sms, cudaStream_t s) {
  constexpr uint32_t V = TensorTraits<FMT>::V;
  constexpr uint32_t ES = 16 / V;
  const uintptr_t a = reinterpret_cast<uintptr_t>(d_ptr);
  uint64_t head = ((16u - (uint32_t)(a & 15u)) & 15u) / ES;
  if (head > n) head = n;
  const uint64_t nvec = (n - head) / V;
  const uint64_t tail = n - head - nvec * V;
  const uint8_t* p = static_cast<const uint8_t*>(d_ptr);
  const uint4* body = reinterpret_cast<const uint4*>(p + head * ES);
  const uint8_t* tailp = p + (head + nvec * V) * ES;
  uint64_t blocks = (nvec + 256 * TU - 1) / (256 * TU);
  const uint64_t cap = (uint64_t)num_sms * 8;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  k_scan_tensor<FMT><<<(unsigned)blocks, 256, 0, s>>>(body, nvec, p, (uint32_t)head, tailp, (uint32_t)tail, head,
                                                       head + nvec * V, base_index, site, tv);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_scan_records(const fpx_rec_hdr* d_hdr, uint64_t n, const uint32_t* d_arena, uint64_t arena_planes,
                                uint64_t base_index, uint32_t mode, const TableView& tv, int num_sms, cudaStream_t s) {
  if (mode == FPX_MODE_DEST)
    return launch_records_t<FPX_MODE_DEST>(d_hdr, n, d_arena, arena_planes, base_index, tv, num_sms, s);
  return launch_records_t<FPX_MODE_FLOW>(d_hdr, n, d_arena, arena_planes, base_index, tv, num_sms, s);
}

cudaError_t launch_scan_tensor(const void* d_ptr, uint64_t n, uint32_t fmt, uint32_t site, uint64_t base_index,
                               const TableView& tv, int num_sms, cudaStream_t s) {
  switch (fmt) {
    case FPX_FP32: return launch_tensor_t<FPX_FP32>(d_ptr, n, site, base_index, tv, num_sms, s);
    case FPX_FP64: return launch_tensor_t<FPX_FP64>(d_ptr, n, site, base_index, tv, num_sms, s);
    case FPX_FP16: return launch_tensor_t<FPX_FP16>(d_ptr, n, site, base_index, tv, num_sms, s);
    default: return launch_tensor_t<FPX_BF16>(d_ptr, n, site, base_index, tv, num_sms, s);
  }
}

}  // namespace fpx
