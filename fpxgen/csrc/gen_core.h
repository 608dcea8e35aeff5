// gen_core.h — counter-based synthetic record / tensor generator (inputs only).
//
// This module is the ONE piece shared by the oracle side (tests) and the CUDA
// side (bench, GPU tests): it produces seeded input bytes and the list of
// planted exceptional values.  It holds none of the method's arithmetic: it
// never classifies a value.  Clean values are *constructed* inside the normal
// range; exceptional values are *written* from fixed bit-pattern tables.
// Every value is a pure function of (seed, record, plane, lane), so any chunk
// can be regenerated on the host (C++) or on the device (CUDA) bit-identically.
//
// Recipe (shapes after the paper's workloads, SURVEY §8 d):
//   sites      Zipf(s) popularity over n_sites (kernels re-invoked many times)
//   formats    FP32/FP64 mixes, FP32 MUFU inside FP64 code, packed FP16/BF16
//   values     clean: random sign, exponent uniform in +-30 (FP32/BF16), +-300 (FP64),
//              +-10 (FP16), random mantissa; p_zero exact zeros
//   masks      90% full warps, p_partial random partial masks
//   inactive   lanes hold random garbage bits (may look exceptional; must be ignored)
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD inline
#endif

namespace fpxgen {

// Recipes.
enum : uint32_t {
  RECIPE_C1 = 0,      // tiny FP32 trace: FFMA / FADD / MUFU.RCP, dest only
  RECIPE_MIX = 1,     // FP32/FP64 mix of compute + MUFU + compare records, dest only (C2, C5)
  RECIPE_FLOW = 2,    // FP32/FP64 records with dest + 1..3 pre-execution sources (C3)
  RECIPE_PACKED = 3,  // HADD2/HFMA2/HMUL2 FP16x2/BF16x2 + HMMA (F16 and F32 accumulators) (C4a)
  RECIPE_STRESS = 4,  // FP32 FFMA only, dest only; dense NaN storms via dense_nan_ppm
  RECIPE_COUNT = 5
};

// Opcode-class and format codes (the record contract of include/fpx.h,
// restated here: this module may not include the product's headers).
enum : uint32_t {
  G_OP_FADD = 1, G_OP_FMUL = 2, G_OP_FFMA = 3, G_OP_RCP = 4, G_OP_RCP64H = 5, G_OP_MUFU = 6,
  G_OP_DADD = 7, G_OP_DMUL = 8, G_OP_DFMA = 9, G_OP_FSEL = 10, G_OP_FSETP = 12,
  G_OP_FMNMX = 13, G_OP_DSETP = 14, G_OP_HADD2 = 15, G_OP_HFMA2 = 16, G_OP_HMUL2 = 17,
  G_OP_HMMA = 18
};
enum : uint32_t { G_FP32 = 0, G_FP64 = 1, G_FP16 = 2, G_BF16 = 3 };

struct Params {
  uint64_t seed;
  uint64_t n_records;
  uint32_t n_sites;
  uint32_t recipe;
  uint32_t p_fp64_ppm;     // share of FP64 records (MIX / FLOW), parts per million
  uint32_t p_partial_ppm;  // share of records with a random partial active mask
  uint32_t p_zero_ppm;     // share of clean values that are +-0
  uint32_t dense_nan_ppm;  // STRESS: share of dest lane-values written as NaN (1e6 = all)
};

struct Hdr {
  uint32_t site, active_mask, meta, val_off;
};

// ---- counter-based hashing (splitmix64 finaliser) -------------------------
GEN_HD uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
GEN_HD uint64_t hash4(uint64_t seed, uint64_t a, uint64_t b, uint64_t tag) {
  return mix64(mix64(mix64(seed ^ (tag * 0xD6E8FEB86659FD93ull)) + a) + b);
}
// uniform in [0, 1) with 53 bits (exact in double on host and device)
GEN_HD double u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }

enum : uint64_t { TAG_HDR = 1, TAG_SITE = 2, TAG_MASK = 3, TAG_VAL = 4, TAG_ZERO = 5, TAG_DENSE = 6,
                  TAG_GARB = 7 };

GEN_HD uint32_t meta_of(uint32_t opclass, uint32_t fmt, uint32_t nsrc, uint32_t dwords) {
  return opclass | (fmt << 8) | (nsrc << 10) | (dwords << 12);
}
GEN_HD uint32_t src_words(uint32_t fmt) { return fmt == G_FP64 ? 2u : 1u; }
GEN_HD uint32_t planes_of(uint32_t meta) {
  uint32_t fmt = (meta >> 8) & 3, nsrc = (meta >> 10) & 3, dwords = (meta >> 12) & 7;
  return dwords + nsrc * src_words(fmt);
}

// Pick an opcode class / format / shape for record r from the recipe's mix.
// Percentages: MIX FP32: FFMA 45 FADD 20 FMUL 20 RCP 2 MUFU 3 FMNMX 2.5 FSEL 2.5 FSETP 5;
//              MIX FP64: DFMA 45 DADD 25 DMUL 20 RCP64H 2 DSETP 8.
GEN_HD uint32_t pick_meta(const Params& p, uint64_t h) {
  uint32_t u = (uint32_t)(h % 1000u);          // per-mille choice of opclass
  uint32_t fsel = (uint32_t)((h >> 20) % 1000000u);  // format choice
  switch (p.recipe) {
    case RECIPE_C1: {
      // "10^5 FFMA/FADD/MUFU.RCP records": 50 / 30 / 20
      uint32_t op = u < 500 ? G_OP_FFMA : u < 800 ? G_OP_FADD : G_OP_RCP;
      return meta_of(op, G_FP32, 0, 1);
    }
    case RECIPE_STRESS:
      return meta_of(G_OP_FFMA, G_FP32, 0, 1);
    case RECIPE_MIX:
    case RECIPE_FLOW: {
      const bool flow = p.recipe == RECIPE_FLOW;
      if (fsel < p.p_fp64_ppm) {
        uint32_t op, ns;
        if (u < 450) { op = G_OP_DFMA; ns = 3; }
        else if (u < 700) { op = G_OP_DADD; ns = 2; }
        else if (u < 900) { op = G_OP_DMUL; ns = 2; }
        else if (u < 920) { op = G_OP_RCP64H; ns = 1; }
        else { op = G_OP_DSETP; ns = 2; }
        uint32_t dw = op == G_OP_DSETP ? 0u : 2u;
        return meta_of(op, G_FP64, flow ? ns : 0u, dw);
      } else {
        uint32_t op, ns;
        if (u < 450) { op = G_OP_FFMA; ns = 3; }
        else if (u < 650) { op = G_OP_FADD; ns = 2; }
        else if (u < 850) { op = G_OP_FMUL; ns = 2; }
        else if (u < 870) { op = G_OP_RCP; ns = 1; }
        else if (u < 900) { op = G_OP_MUFU; ns = 1; }
        else if (u < 925) { op = G_OP_FMNMX; ns = 2; }
        else if (u < 950) { op = G_OP_FSEL; ns = 2; }
        else { op = G_OP_FSETP; ns = 2; }
        uint32_t dw = op == G_OP_FSETP ? 0u : 1u;
        return meta_of(op, G_FP32, flow ? ns : 0u, dw);
      }
    }
    default: {  // RECIPE_PACKED: HADD2 30 HFMA2 30 HMUL2 20 HMMA.F16 10 HMMA.F32 10
      uint32_t fmt = (fsel & 1) ? G_BF16 : G_FP16;
      if (u < 300) return meta_of(G_OP_HADD2, fmt, 0, 1);
      if (u < 600) return meta_of(G_OP_HFMA2, fmt, 0, 1);
      if (u < 800) return meta_of(G_OP_HMUL2, fmt, 0, 1);
      if (u < 900) return meta_of(G_OP_HMMA, G_FP16, 0, 2);
      return meta_of(G_OP_HMMA, G_FP32, 0, 4);
    }
  }
}

// Site of record r: inverse-CDF lookup of a Zipf(s) table (cdf[i] = P(site <= i)).
GEN_HD uint32_t pick_site(const double* cdf, uint32_t n_sites, uint64_t h) {
  double u = u01(h);
  uint32_t lo = 0, hi = n_sites - 1;  // first i with cdf[i] > u
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2;
    if (cdf[mid] > u) hi = mid; else lo = mid + 1;
  }
  return lo;
}

// Header of record r with val_off = number of planes (offsets are assigned by
// an exclusive prefix sum afterwards).
GEN_HD Hdr make_header(const Params& p, const double* cdf, uint64_t r) {
  Hdr h;
  uint64_t hh = hash4(p.seed, r, 0, TAG_HDR);
  h.meta = pick_meta(p, hh);
  h.site = pick_site(cdf, p.n_sites, hash4(p.seed, r, 0, TAG_SITE));
  uint64_t hm = hash4(p.seed, r, 0, TAG_MASK);
  bool partial = (uint32_t)(hm % 1000000u) < p.p_partial_ppm;
  h.active_mask = partial ? (uint32_t)(hm >> 32) : 0xFFFFFFFFu;
  h.val_off = planes_of(h.meta);
  return h;
}

// A clean FP32 word: sign | exponent in [127-30, 127+30] | random mantissa, or +-0.
GEN_HD uint32_t clean_fp32(uint64_t h, bool zero) {
  uint32_t sign = (uint32_t)(h >> 63) << 31;
  if (zero) return sign;
  uint32_t e = 97u + (uint32_t)((h >> 40) % 61u);
  return sign | (e << 23) | ((uint32_t)h & 0x7FFFFFu);
}
GEN_HD uint32_t clean_fp16(uint64_t h, bool zero) {
  uint32_t sign = (uint32_t)(h >> 15) & 1u;
  if (zero) return sign << 15;
  uint32_t e = 5u + (uint32_t)((h >> 16) % 21u);  // 15 +- 10
  return (sign << 15) | (e << 10) | ((uint32_t)h & 0x3FFu);
}
GEN_HD uint32_t clean_bf16(uint64_t h, bool zero) {
  uint32_t sign = (uint32_t)(h >> 15) & 1u;
  if (zero) return sign << 15;
  uint32_t e = 97u + (uint32_t)((h >> 16) % 61u);
  return (sign << 15) | (e << 7) | ((uint32_t)h & 0x7Fu);
}

// Word of plane `plane` (relative to the record), lane `lane`, of record r.
GEN_HD uint32_t plane_word(const Params& p, uint64_t r, const Hdr& h, uint32_t plane, uint32_t lane) {
  if (((h.active_mask >> lane) & 1u) == 0) {
    // inactive lane: garbage, deliberately including exceptional-looking bits
    return (uint32_t)hash4(p.seed, r, (uint64_t)plane * 32u + lane, TAG_GARB);
  }
  const uint32_t fmt = (h.meta >> 8) & 3, dwords = (h.meta >> 12) & 7;
  const uint32_t pz = p.p_zero_ppm;
  if (fmt == G_FP64) {
    // planes come in (lo, hi) pairs; both halves derive from the pair index
    uint32_t pair = plane / 2;
    uint64_t hv = hash4(p.seed, r, (uint64_t)pair * 32u + lane, TAG_VAL);
    bool zero = (uint32_t)(hash4(p.seed, r, (uint64_t)pair * 32u + lane, TAG_ZERO) % 1000000u) < pz;
    if ((plane & 1u) == 0) return zero ? 0u : (uint32_t)mix64(hv);  // low 32 mantissa bits
    uint32_t sign = (uint32_t)(hv >> 63) << 31;
    if (zero) return sign;
    uint32_t e = 723u + (uint32_t)((hv >> 32) % 601u);  // 1023 +- 300
    return sign | (e << 20) | ((uint32_t)hv & 0xFFFFFu);
  }
  uint64_t hv = hash4(p.seed, r, (uint64_t)plane * 32u + lane, TAG_VAL);
  uint64_t hz = hash4(p.seed, r, (uint64_t)plane * 32u + lane, TAG_ZERO);
  if (fmt == G_FP32) {
    if (p.dense_nan_ppm != 0 && plane < dwords) {
      uint64_t hd = hash4(p.seed, r, (uint64_t)plane * 32u + lane, TAG_DENSE);
      if ((uint32_t)(hd % 1000000u) < p.dense_nan_ppm) return 0x7FC00000u;  // planted qNaN
    }
    return clean_fp32(hv, (uint32_t)(hz % 1000000u) < pz);
  }
  bool z0 = (uint32_t)(hz % 1000000u) < pz, z1 = (uint32_t)((hz >> 32) % 1000000u) < pz;
  if (fmt == G_FP16) return clean_fp16(hv, z0) | (clean_fp16(hv >> 32, z1) << 16);
  return clean_bf16(hv, z0) | (clean_bf16(hv >> 32, z1) << 16);
}

// ---- planted exceptional bit patterns (IEEE-754 layouts, by construction) ---
// class codes for planting: 0 NaN, 1 INF, 2 SUB
struct PatternSet { const uint64_t* v; uint32_t n; };

}  // namespace fpxgen
