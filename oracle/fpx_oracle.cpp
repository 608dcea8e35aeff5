// fpx_oracle.cpp — plain, slow, single-threaded CPU oracle of the GPU-FPX
// exception scan.
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
// bench.py's cpu_baseline / --impl reference legs may load this library.  The
// product path (paper_conf_hpdc_lilfslg23_b200/, libfpx.so) never links,
// imports or calls it, and this file includes nothing from include/ or the
// package: every constant below is restated from the paper / SURVEY §8 on its
// own.  Built with plain -O2, no -ffast-math (std::isnan would be unreliable
// under it; classification here is by bit pattern anyway).
//
// What it computes (citations: P:<line> = /root/reference/PAPER.md line,
// R<n> = reading n listed in DESIGN.md §3):
//   classify()      the IEEE-754 special-value definitions of §2.1 P:140-145,
//                   written out per field (exponent all-ones / zero, mantissa
//                   zero / non-zero) for FP32, FP64, FP16 and BF16.
//   dest_kind()     Alg1's dispatch: MUFU.RCP(64H) -> DIV0
//                   iff the destination is NaN or INF; compares -> no dest;
//                   synthetic DIV -> IEEE divideByZero (R1); else the class.
//   scan_records()  Alg2's per-lane check in detector mode, and the
//                   Table 2 states in analyzer mode, aggregated
//                   into an ordered map key -> (count, first index): the plain
//                   definition of the deduplicated table GT with
//                   the widened key / value of R14, R15.
//   scan_tensor()   the same destination check over a plain buffer (R18).
// The loops follow the definition literally: record by record, lane by lane,
// value by value, one map update per exceptional lane-value.  No blocking, no
// warp aggregation, no hashing.
//
// Pins: tests/test_oracle_pins.py (exhaustive closed forms, numpy IEEE
// predicates, the paper's worked cases, brute force through real IEEE ops,
// planted-event aggregates).  Parity unpinned by the paper: the KILL kind
// when several sources are exceptional (severity order NaN > INF > SUB,
// reading R5) and per-half counting of packed FP16/BF16 values (R13) are
// conventions of DESIGN.md §3, pinned only to that text.

#include <cstdint>
#include <cstring>
#include <map>

namespace {

// ---- constants restated from the paper / SURVEY §8 ------------------------
// E_fp
constexpr uint32_t FMT_FP32 = 0, FMT_FP64 = 1, FMT_FP16 = 2, FMT_BF16 = 3;
// E_exce
constexpr uint32_t K_NAN = 0, K_INF = 1, K_SUB = 2, K_DIV0 = 3;
// Table 2 states: none (detector), Appearance, Propagation,
// Disappearance.
constexpr uint32_t F_NONE = 0, F_GEN = 1, F_PROP = 2, F_KILL = 3;
constexpr uint32_t MODE_DEST = 0, MODE_FLOW = 1, MODE_FLOW_DETAIL = 2;
// Opcode classes (Table 1 P:101-110 plus the packed / synthetic ones).
constexpr uint32_t OP_MUFU_RCP = 4, OP_MUFU_RCP64H = 5, OP_FSEL = 10, OP_FSET = 11, OP_FSETP = 12,
                   OP_FMNMX = 13, OP_DSETP = 14, OP_DIV = 19, OP_COUNT = 20;

// Value classes of §2.1.
enum Cls { CLEAN = 0, C_NAN = 1, C_INF = 2, C_SUB = 3 };

struct Hdr {  // one record header, 16 bytes (SURVEY §8 layout)
  uint32_t site, active_mask, meta, val_off;
};
static_assert(sizeof(Hdr) == 16, "header is 16 bytes");

struct Entry {  // fetched entry, 24 bytes
  uint32_t site;
  uint8_t kind, flow, fmt, detail;
  uint64_t count, first_index;
};
static_assert(sizeof(Entry) == 24, "entry is 24 bytes");

struct Val {  // the table value: count of lane-values and first index
  uint64_t count = 0;
  uint64_t first = UINT64_MAX;
};

// ---- §2.1 classification, field by field ----------------------------------
// "If the exponent is all ones: mantissa 0 -> INF, mantissa != 0 -> NaN.
//  If the exponent is 0 and the mantissa is non-zero -> subnormal."
Cls classify_fields(uint64_t exponent, uint64_t exp_all_ones, uint64_t mantissa) {
  if (exponent == exp_all_ones) return mantissa == 0 ? C_INF : C_NAN;
  if (exponent == 0 && mantissa != 0) return C_SUB;
  return CLEAN;
}

// bits holds the value's bit pattern in its low 16/32/64 bits.
Cls classify(uint32_t fmt, uint64_t bits) {
  switch (fmt) {
    case FMT_FP32:  // 1 sign, 8 exponent, 23 mantissa bits
      return classify_fields((bits >> 23) & 0xFF, 0xFF, bits & 0x7FFFFFull);
    case FMT_FP64:  // 1 sign, 11 exponent, 52 mantissa bits
      return classify_fields((bits >> 52) & 0x7FF, 0x7FF, bits & 0xFFFFFFFFFFFFFull);
    case FMT_FP16:  // 1 sign, 5 exponent, 10 mantissa bits
      return classify_fields((bits >> 10) & 0x1F, 0x1F, bits & 0x3FFull);
    default:        // BF16: 1 sign, 8 exponent, 7 mantissa bits
      return classify_fields((bits >> 7) & 0xFF, 0xFF, bits & 0x7Full);
  }
}

bool is_zero(uint32_t fmt, uint64_t bits) {  // +0 or -0: exponent 0 and mantissa 0
  switch (fmt) {
    case FMT_FP32: return (bits & 0x7FFFFFFFull) == 0;
    case FMT_FP64: return (bits & 0x7FFFFFFFFFFFFFFFull) == 0;
    case FMT_FP16: return (bits & 0x7FFFull) == 0;
    default: return (bits & 0x7FFFull) == 0;
  }
}

// Class -> E_exce code (only for non-clean classes).
uint32_t kind_of(Cls c) { return c == C_NAN ? K_NAN : c == C_INF ? K_INF : K_SUB; }

// Severity order for several exceptional sources of one lane: NaN > INF > SUB
// ("more serious" ordering; reading R5).
int severity(Cls c) { return c == C_NAN ? 3 : c == C_INF ? 2 : c == C_SUB ? 1 : 0; }

// Words per lane of one source operand (sw): 2 for FP64, 1 otherwise.
uint32_t source_words(uint32_t fmt) { return fmt == FMT_FP64 ? 2u : 1u; }

// Number of values held by `words` 32-bit words of format fmt.
uint32_t values_in(uint32_t fmt, uint32_t words) {
  if (fmt == FMT_FP64) return words / 2;
  if (fmt == FMT_FP32) return words;
  return 2 * words;  // FP16x2 / BF16x2 packed
}

// Value v of an operand whose 32-bit words (for one lane) are w[0..].
uint64_t value_bits(uint32_t fmt, const uint32_t* w, uint32_t v) {
  if (fmt == FMT_FP64) return ((uint64_t)w[2 * v + 1] << 32) | w[2 * v];  // (lo, hi)
  if (fmt == FMT_FP32) return w[v];
  uint32_t word = w[v / 2];
  return (v % 2 == 0) ? (word & 0xFFFFu) : (word >> 16);  // low half first
}

// "no destination kind" sentinel
constexpr uint32_t NO_KIND = 0xFFFFFFFFu;

// Alg1 dispatch + kind rule (readings R1, R2, R10, R11).
// src_vals[k] = value of source k at the same value position (if defined).
uint32_t dest_kind(uint32_t opclass, uint32_t fmt, uint64_t d,
                   const uint64_t* src_vals, uint32_t n_src_vals) {
  if (opclass == OP_MUFU_RCP || opclass == OP_MUFU_RCP64H) {
    // "the opcode is MUFU.RCP(64H) and the destination register holds a
    // NaN or INF value" -> division by zero.  RCP never reports SUB (R2).
    Cls c = classify(fmt, d);
    return (c == C_NAN || c == C_INF) ? K_DIV0 : NO_KIND;
  }
  if (opclass == OP_FSETP || opclass == OP_DSETP || opclass == OP_FSET) return NO_KIND;  // R10
  if (opclass == OP_DIV && n_src_vals >= 2) {
    // R1: IEEE divideByZero: divisor (src1) is +-0 and dividend (src0) finite, non-zero.
    uint64_t dividend = src_vals[0], divisor = src_vals[1];
    Cls cd = classify(fmt, dividend);
    bool dividend_finite_nonzero = (cd == CLEAN || cd == C_SUB) && !is_zero(fmt, dividend);
    if (is_zero(fmt, divisor) && dividend_finite_nonzero) return K_DIV0;
  }
  Cls c = classify(fmt, d);
  return c == CLEAN ? NO_KIND : kind_of(c);
}

uint64_t make_key(uint32_t site, uint32_t fmt, uint32_t flow, uint32_t kind, uint32_t detail = 0) {
  return ((uint64_t)site << 32) | ((uint64_t)detail << 6) | ((uint64_t)fmt << 4) | ((uint64_t)flow << 2) | kind;
}

// Control-flow opcodes of Table 1's right column.
bool is_control_flow(uint32_t op) {
  return op == OP_FSEL || op == OP_FSET || op == OP_FSETP || op == OP_FMNMX || op == OP_DSETP;
}

}  // namespace

struct orc_table {
  std::map<uint64_t, Val> gt;  // the deduplicated exception table GT
  uint64_t bad_records = 0;
  uint64_t lane_values = 0;    // lane-values classified (for throughput reporting)
};

namespace {

void record_event(orc_table* t, uint32_t site, uint32_t fmt, uint32_t flow, uint32_t kind,
                  uint64_t g, uint32_t detail = 0) {
  Val& e = t->gt[make_key(site, fmt, flow, kind, detail)];
  e.count += 1;
  if (g < e.first) e.first = g;
}

// Record validation (the header contract in SURVEY §8 / include/fpx.h prose).
bool record_valid(const Hdr& h, uint64_t arena_planes, uint32_t mode) {
  if (h.site == 0xFFFFFFFFu) return false;
  if ((h.meta >> 15) != 0) return false;
  uint32_t opclass = h.meta & 0xFF, fmt = (h.meta >> 8) & 3, nsrc = (h.meta >> 10) & 3,
           dwords = (h.meta >> 12) & 7;
  if (opclass >= OP_COUNT) return false;
  if (dwords > 4) return false;
  if (fmt == FMT_FP64 && (dwords % 2) != 0) return false;
  uint64_t planes = dwords + (uint64_t)nsrc * source_words(fmt);
  if ((uint64_t)h.val_off + planes > arena_planes) return false;
  if (mode != MODE_DEST) {
    // FLOW is defined for scalar FP32 / FP64 records only (R13).
    if (fmt != FMT_FP32 && fmt != FMT_FP64) return false;
    if (dwords != 0 && dwords != source_words(fmt)) return false;
  }
  return true;
}

}  // namespace

extern "C" {

orc_table* orc_new(void) { return new orc_table(); }
void orc_free(orc_table* t) { delete t; }
void orc_clear(orc_table* t) { t->gt.clear(); t->bad_records = 0; t->lane_values = 0; }

// Class code of one value: 0 clean, 1 NaN, 2 INF, 3 SUB.
int orc_classify(uint32_t fmt, uint64_t bits) { return (int)classify(fmt, bits); }

// Class histogram of every FP32 bit pattern in [lo, hi] (inclusive), for the
// exhaustive pin.  counts[0..3] += per class.
void orc_class_hist_fp32(uint32_t lo, uint32_t hi, uint64_t* counts) {
  uint64_t c[4] = {0, 0, 0, 0};
  for (uint64_t b = lo; b <= hi; ++b) c[classify(FMT_FP32, b)]++;
  for (int i = 0; i < 4; ++i) counts[i] += c[i];
}

// Kind of a destination value under the Alg1 dispatch, -1 when none.
// srcs may be NULL (nsrc = 0).
int orc_dest_kind(uint32_t opclass, uint32_t fmt, uint64_t d, const uint64_t* srcs, uint32_t nsrc) {
  uint32_t k = dest_kind(opclass, fmt, d, srcs, srcs ? nsrc : 0);
  return k == NO_KIND ? -1 : (int)k;
}

// The record scan: for r in 0..n-1 (global index g = base_index + r), for each
// active lane, for each destination value: kind rule, flow rule, table update.
void orc_scan_records(orc_table* t, const void* hdr_v, uint64_t n, const uint32_t* arena,
                      uint64_t arena_planes, uint64_t base_index, uint32_t mode) {
  const Hdr* hdr = static_cast<const Hdr*>(hdr_v);
  for (uint64_t r = 0; r < n; ++r) {
    const Hdr h = hdr[r];
    const uint64_t g = base_index + r;
    if (!record_valid(h, arena_planes, mode)) { t->bad_records++; continue; }
    const uint32_t opclass = h.meta & 0xFF, fmt = (h.meta >> 8) & 3, nsrc = (h.meta >> 10) & 3,
                   dwords = (h.meta >> 12) & 7;
    const uint32_t sw = source_words(fmt);
    const uint32_t n_dest = values_in(fmt, dwords);
    for (uint32_t lane = 0; lane < 32; ++lane) {
      if (((h.active_mask >> lane) & 1u) == 0) continue;  // inactive lanes ignored (R9)
      // This lane's words: plane p holds lane `lane` at word index p*32 + lane.
      uint32_t dw[4] = {0, 0, 0, 0};
      uint32_t sv[3][2] = {{0, 0}, {0, 0}, {0, 0}};
      for (uint32_t i = 0; i < dwords; ++i) dw[i] = arena[((uint64_t)h.val_off + i) * 32 + lane];
      for (uint32_t k = 0; k < nsrc; ++k)
        for (uint32_t i = 0; i < sw; ++i)
          sv[k][i] = arena[((uint64_t)h.val_off + dwords + (uint64_t)k * sw + i) * 32 + lane];

      // Source values at value position v; the kind rule of DIV uses them
      // when the destination is exactly one source-operand wide (R1).
      const bool src_aligned = (dwords == sw);
      uint64_t s[3] = {0, 0, 0};

      if (mode == MODE_DEST) {
        t->lane_values += n_dest;
        for (uint32_t v = 0; v < n_dest; ++v) {
          uint64_t d = value_bits(fmt, dw, v);
          for (uint32_t k = 0; k < nsrc; ++k) s[k] = value_bits(fmt, sv[k], v);
          uint32_t k = dest_kind(opclass, fmt, d, s, src_aligned ? nsrc : 0);
          if (k != NO_KIND) record_event(t, h.site, fmt, F_NONE, k, g);
        }
      } else {
        // Analyzer: S = most severe class among the PRE-execution source
        // values of this lane (R5); src = the lowest-index source
        // holding that class (R21).  Scalar records only (R13).
        t->lane_values += n_dest + nsrc;
        Cls S = CLEAN;
        uint32_t src = 0;
        for (uint32_t k = 0; k < nsrc; ++k) {
          s[k] = value_bits(fmt, sv[k], 0);
          Cls c = classify(fmt, s[k]);
          if (severity(c) > severity(S)) { S = c; src = k; }
        }
        uint32_t D = NO_KIND;
        if (n_dest == 1) D = dest_kind(opclass, fmt, value_bits(fmt, dw, 0), s, nsrc);
        // FLOW_DETAIL: which source, and Table 2's Comparison state (R22)
        uint32_t detail = 0;
        if (mode == MODE_FLOW_DETAIL && S != CLEAN) {
          detail = src + 1;
          if (is_control_flow(opclass)) detail |= 4;
        }
        // Table 2: Appearance (dest EV, no source EV), Propagation (dest EV,
        // source EV), Disappearance (no dest exception, source EV).
        if (D != NO_KIND && S == CLEAN) record_event(t, h.site, fmt, F_GEN, D, g, detail);
        else if (D != NO_KIND && S != CLEAN) record_event(t, h.site, fmt, F_PROP, D, g, detail);
        else if (D == NO_KIND && S != CLEAN) record_event(t, h.site, fmt, F_KILL, kind_of(S), g, detail);
      }
    }
  }
}

// Tensor scan: element i of a contiguous buffer, destination-only, site given.
void orc_scan_tensor(orc_table* t, const void* p, uint64_t n, uint32_t fmt, uint32_t site,
                     uint64_t base_index) {
  const unsigned char* b = static_cast<const unsigned char*>(p);
  const uint32_t esize = fmt == FMT_FP64 ? 8 : fmt == FMT_FP32 ? 4 : 2;
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t bits = 0;
    std::memcpy(&bits, b + i * esize, esize);  // little-endian host
    Cls c = classify(fmt, bits);
    if (c != CLEAN) record_event(t, site, fmt, F_NONE, kind_of(c), base_index + i);
  }
  t->lane_values += n;
}

uint64_t orc_size(const orc_table* t) { return t->gt.size(); }
uint64_t orc_bad_records(const orc_table* t) { return t->bad_records; }
uint64_t orc_lane_values(const orc_table* t) { return t->lane_values; }

// Entries in ascending key order (std::map order).  Returns the number
// written (<= cap).
uint64_t orc_fetch(const orc_table* t, void* out_v, uint64_t cap) {
  Entry* out = static_cast<Entry*>(out_v);
  uint64_t i = 0;
  for (const auto& kv : t->gt) {
    if (i >= cap) break;
    Entry e;
    std::memset(&e, 0, sizeof e);
    e.site = (uint32_t)(kv.first >> 32);
    e.fmt = (uint8_t)((kv.first >> 4) & 3);
    e.flow = (uint8_t)((kv.first >> 2) & 3);
    e.kind = (uint8_t)(kv.first & 3);
    e.detail = (uint8_t)((kv.first >> 6) & 7);
    e.count = kv.second.count;
    e.first_index = kv.second.first;
    out[i++] = e;
  }
  return i;
}

uint32_t orc_sizeof_hdr(void) { return (uint32_t)sizeof(Hdr); }
uint32_t orc_sizeof_entry(void) { return (uint32_t)sizeof(Entry); }
uint64_t orc_key(uint32_t site, uint32_t fmt, uint32_t flow, uint32_t kind) {
  return make_key(site, fmt, flow, kind);
}

}  // extern "C"
