// fpxgen.cu — host and device entry points of the synthetic input generator.
//
// Inputs only (see gen_core.h): headers, planes, planted exceptional values.
// The host path is plain sequential C++; the device path runs the same
// counter-based functions in CUDA kernels so that the benchmark can build
// 20+ GB traces directly in HBM.  Tests cross-check the two bit for bit.
#include <cuda_runtime.h>
#include <cub/device/device_scan.cuh>
#include <cmath>
#include <cstring>
#include <unordered_set>
#include <vector>

#include "gen_core.h"

using namespace fpxgen;

struct Write {  // one planted write: word = (word & and_mask) | or_bits on lanes in lanemask
  uint64_t record;  // relative to the generated chunk
  uint32_t plane, lanemask, and_mask, or_bits;
};
static_assert(sizeof(Write) == 24, "write is 24 B");

namespace {

// ---- planted bit patterns, per format and class (NaN, INF, SUB) -----------
// Chosen at the IEEE-754 field boundaries; FP64 ones include a NaN whose high
// word has a zero mantissa and subnormals whose low / high word is zero, so a
// check that looks at one word only is caught (SURVEY §7 hard part 6).
const uint64_t P32[3][5] = {
    {0x7FC00000ull, 0xFFC00000ull, 0x7F800001ull, 0x7FFFFFFFull, 0xFF800001ull},
    {0x7F800000ull, 0xFF800000ull, 0x7F800000ull, 0xFF800000ull, 0x7F800000ull},
    {0x00000001ull, 0x007FFFFFull, 0x80000001ull, 0x80400000ull, 0x00012345ull}};
const uint64_t P64[3][5] = {
    {0x7FF8000000000000ull, 0x7FF0000000000001ull, 0xFFF0000100000000ull, 0x7FFFFFFFFFFFFFFFull,
     0xFFF8000000000000ull},
    {0x7FF0000000000000ull, 0xFFF0000000000000ull, 0x7FF0000000000000ull, 0xFFF0000000000000ull,
     0x7FF0000000000000ull},
    {0x0000000000000001ull, 0x0000000100000000ull, 0x000FFFFFFFFFFFFFull, 0x8000000000000001ull,
     0x8000000100000000ull}};
const uint64_t P16[3][5] = {{0x7E00, 0x7C01, 0xFFFF, 0xFE00, 0x7D55},
                            {0x7C00, 0xFC00, 0x7C00, 0xFC00, 0x7C00},
                            {0x0001, 0x03FF, 0x8001, 0x8200, 0x0155}};
const uint64_t PB16[3][5] = {{0x7FC0, 0x7F81, 0xFFFF, 0xFFC0, 0x7FAA},
                             {0x7F80, 0xFF80, 0x7F80, 0xFF80, 0x7F80},
                             {0x0001, 0x007F, 0x8001, 0x8040, 0x0055}};

uint64_t pattern(uint32_t fmt, uint32_t pclass, uint64_t h) {
  uint32_t i = (uint32_t)(h % 5);
  switch (fmt) {
    case G_FP32: return P32[pclass][i];
    case G_FP64: return P64[pclass][i];
    case G_FP16: return P16[pclass][i];
    default: return PB16[pclass][i];
  }
}

uint32_t values_of(uint32_t fmt, uint32_t words) {
  return fmt == G_FP64 ? words / 2 : fmt == G_FP32 ? words : 2 * words;
}

// ---- device kernels ---------------------------------------------------------
__global__ void k_headers(Params p, const double* cdf, uint64_t r0, uint64_t n, Hdr* hdr,
                          uint64_t* planes) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    Hdr h = make_header(p, cdf, r0 + i);
    planes[i] = h.val_off;
    hdr[i] = h;
  }
}

__global__ void k_set_offsets(Hdr* hdr, const uint64_t* offs, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    hdr[i].val_off = (uint32_t)offs[i];
}

// one warp per record, lane = lane
__global__ void k_fill(Params p, uint64_t r0, const Hdr* hdr, uint64_t n, uint32_t* arena) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t w0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = w0; i < n; i += nw) {
    Hdr h = hdr[i];
    uint32_t np = planes_of(h.meta);
    for (uint32_t pl = 0; pl < np; ++pl)
      arena[((uint64_t)h.val_off + pl) * 32 + lane] = plane_word(p, r0 + i, h, pl, lane);
  }
}

__global__ void k_apply(const Write* w, uint64_t nw, const Hdr* hdr, uint32_t* arena) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t w0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t step = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t i = w0; i < nw; i += step) {
    Write e = w[i];
    if ((e.lanemask >> lane) & 1u) {
      uint64_t idx = ((uint64_t)hdr[e.record].val_off + e.plane) * 32 + lane;
      arena[idx] = (arena[idx] & e.and_mask) | e.or_bits;
    }
  }
}

thread_local char g_err[256];
int cuda_fail(cudaError_t e) {
  snprintf(g_err, sizeof g_err, "%s", cudaGetErrorString(e));
  return -2;
}
#define GCK(x) do { cudaError_t _e = (x); if (_e != cudaSuccess) return cuda_fail(_e); } while (0)

}  // namespace

extern "C" {

// Planted-event description returned to tests (closed-form expectation).
struct fpxgen_injection {
  uint64_t record;     // relative to the chunk
  uint32_t lanemask;   // lanes written (storms: all 32)
  uint8_t dest_class;  // 0 NaN, 1 INF, 2 SUB, 0xFF = destination untouched
  uint8_t src_class;   // same for the planted source value, 0xFF = none
  uint8_t flow_intent; // 0 none (dest-only recipe), 1 GEN, 2 PROP, 3 KILL
  uint8_t slot;        // destination value slot or source operand index
};

const char* fpxgen_last_error(void) { return g_err; }
uint32_t fpxgen_sizeof_hdr(void) { return sizeof(Hdr); }
uint32_t fpxgen_sizeof_write(void) { return sizeof(Write); }
uint32_t fpxgen_sizeof_injection(void) { return sizeof(fpxgen_injection); }

// Zipf(s) CDF over n sites: cdf[i] = sum_{j<=i} (j+1)^-s / H.
void fpxgen_zipf_cdf(uint32_t n, double s, double* cdf) {
  double acc = 0.0;
  for (uint32_t i = 0; i < n; ++i) { acc += std::pow((double)(i + 1), -s); cdf[i] = acc; }
  for (uint32_t i = 0; i < n; ++i) cdf[i] /= acc;
  cdf[n - 1] = 1.0;
}

// Headers of records [r0, r0+n) with chunk-relative val_off; returns the number
// of arena planes the chunk needs.  Host, sequential.
uint64_t fpxgen_headers_host(const Params* p, const double* cdf, uint64_t r0, uint64_t n, Hdr* out) {
  uint64_t off = 0;
  for (uint64_t i = 0; i < n; ++i) {
    Hdr h = make_header(*p, cdf, r0 + i);
    uint32_t np = h.val_off;
    h.val_off = (uint32_t)off;
    off += np;
    out[i] = h;
  }
  return off;
}

void fpxgen_fill_host(const Params* p, uint64_t r0, const Hdr* hdr, uint64_t n, uint32_t* arena) {
  for (uint64_t i = 0; i < n; ++i) {
    const Hdr h = hdr[i];
    const uint32_t np = planes_of(h.meta);
    for (uint32_t pl = 0; pl < np; ++pl)
      for (uint32_t lane = 0; lane < 32; ++lane)
        arena[((uint64_t)h.val_off + pl) * 32 + lane] = plane_word(*p, r0 + i, h, pl, lane);
  }
}

// Plan n_inj planted injections over records [r0, r0+n) (p->n_records is the
// chunk length here).  storm_ppm of them are storms: 1..64 consecutive records,
// all 32 lanes.  flow != 0: plant GEN / PROP / KILL shapes (needs sources).
// Two injections never touch the same record.  Returns the number of
// per-record injection entries; *n_writes receives the planned writes.
// Either output may be NULL to size the call (caps then ignored).
int64_t fpxgen_plan_injections(const Params* p, const double* cdf, uint64_t r0, uint64_t n_inj,
                               uint32_t storm_ppm, uint32_t flow, fpxgen_injection* inj,
                               uint64_t inj_cap, Write* writes, uint64_t w_cap, uint64_t* n_writes) {
  const uint64_t n = p->n_records;
  std::unordered_set<uint64_t> used;
  uint64_t ni = 0, nwr = 0;
  auto emit_write = [&](uint64_t rec, uint32_t plane, uint32_t lanes, uint32_t andm, uint32_t orb) {
    if (writes && nwr < w_cap) writes[nwr] = Write{rec, plane, lanes, andm, orb};
    nwr++;
  };
  // write value slot v (destination) or a source operand's first value
  auto plant_value = [&](uint64_t rec, uint32_t fmt, uint32_t plane_base, uint32_t v, uint32_t lanes,
                         uint64_t pat) {
    if (fmt == G_FP64) {
      emit_write(rec, plane_base + 2 * v, lanes, 0u, (uint32_t)pat);
      emit_write(rec, plane_base + 2 * v + 1, lanes, 0u, (uint32_t)(pat >> 32));
    } else if (fmt == G_FP32) {
      emit_write(rec, plane_base + v, lanes, 0u, (uint32_t)pat);
    } else {
      uint32_t sh = 16 * (v & 1);
      emit_write(rec, plane_base + v / 2, lanes, sh ? 0x0000FFFFu : 0xFFFF0000u, (uint32_t)pat << sh);
    }
  };
  if (n == 0) { if (n_writes) *n_writes = 0; return 0; }
  for (uint64_t i = 0; i < n_inj; ++i) {
    const uint64_t hi = hash4(p->seed, r0, i, 0x1A1Aull);
    const bool storm = (uint32_t)(hi % 1000000u) < storm_ppm;
    const uint64_t ra = (hi >> 20) % n;
    uint64_t len = storm ? 1 + ((hi >> 52) % 64) : 1;
    if (ra + len > n) len = n - ra;
    bool clash = false;
    for (uint64_t r = ra; r < ra + len; ++r) if (used.count(r)) { clash = true; break; }
    if (clash) continue;
    for (uint64_t r = ra; r < ra + len; ++r) used.insert(r);
    for (uint64_t r = ra; r < ra + len; ++r) {
      const uint64_t hr = hash4(p->seed, r0 + r, i, 0x2B2Bull);
      Hdr h = make_header(*p, cdf, r0 + r);
      const uint32_t op = h.meta & 0xFF, fmt = (h.meta >> 8) & 3, nsrc = (h.meta >> 10) & 3,
                     dwords = (h.meta >> 12) & 7;
      const uint32_t n_dest = values_of(fmt, dwords);
      const bool rcp = (op == G_OP_RCP || op == G_OP_RCP64H);
      uint32_t lanes;
      if (storm) {
        lanes = 0xFFFFFFFFu;
      } else {
        // one active lane, chosen uniformly among the active ones
        uint32_t m = h.active_mask;
        int pc = __builtin_popcount(m);
        if (pc == 0) continue;
        int k = (int)(hr % (uint64_t)pc);
        for (int j = 0; j < k; ++j) m &= m - 1;
        lanes = m & (~m + 1);
      }
      fpxgen_injection e;
      e.record = r; e.lanemask = lanes; e.dest_class = 0xFF; e.src_class = 0xFF;
      e.flow_intent = 0; e.slot = 0;
      // RCP destinations are planted with NaN / INF only: the paper's RCP check
      // reports DIV0 for those and never reports SUB (reading R2).
      const uint32_t dclass = rcp ? (uint32_t)((hr >> 8) % 2) : (uint32_t)((hr >> 8) % 3);
      const uint64_t dpat = pattern(fmt, dclass, hr >> 16);
      if (!flow) {
        if (n_dest == 0) continue;
        const uint32_t v = (uint32_t)((hr >> 40) % n_dest);
        plant_value(r, fmt, 0, v, lanes, dpat);
        e.dest_class = (uint8_t)dclass; e.slot = (uint8_t)v;
      } else {
        uint32_t type = 1 + (uint32_t)((hr >> 40) % 3);  // GEN, PROP, KILL
        if (nsrc == 0) type = 1;
        if (n_dest == 0) type = 3;
        if (n_dest == 0 && nsrc == 0) continue;
        const uint32_t k = nsrc ? (uint32_t)((hr >> 44) % nsrc) : 0;
        const uint32_t sclass = (uint32_t)((hr >> 48) % 3);
        const uint32_t sw = src_words(fmt);
        if (type == 1 || type == 2) {
          plant_value(r, fmt, 0, 0, lanes, dpat);
          e.dest_class = (uint8_t)dclass;
        }
        if (type == 2 || type == 3) {
          plant_value(r, fmt, dwords + k * sw, 0, lanes, pattern(fmt, sclass, hr >> 24));
          e.src_class = (uint8_t)sclass; e.slot = (uint8_t)k;
        }
        e.flow_intent = (uint8_t)type;
      }
      if (inj && ni < inj_cap) inj[ni] = e;
      ni++;
    }
  }
  if (n_writes) *n_writes = nwr;
  return (int64_t)ni;
}

void fpxgen_apply_host(const Write* w, uint64_t nw, const Hdr* hdr, uint32_t* arena) {
  for (uint64_t i = 0; i < nw; ++i)
    for (uint32_t lane = 0; lane < 32; ++lane)
      if ((w[i].lanemask >> lane) & 1u) {
        uint64_t idx = ((uint64_t)hdr[w[i].record].val_off + w[i].plane) * 32 + lane;
        arena[idx] = (arena[idx] & w[i].and_mask) | w[i].or_bits;
      }
}

// Device: headers of [r0, r0+n) with chunk-relative offsets; *total_planes is
// written after a stream synchronisation.  d_cdf is a device copy of the CDF.
int fpxgen_headers_device(const Params* p, const double* d_cdf, uint64_t r0, uint64_t n, Hdr* d_hdr,
                          uint64_t* total_planes, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (n == 0) { *total_planes = 0; return 0; }
  uint64_t* d_pl = nullptr;
  GCK(cudaMalloc(&d_pl, sizeof(uint64_t) * (n + 1)));
  k_headers<<<1184, 256, 0, s>>>(*p, d_cdf, r0, n, d_hdr, d_pl);
  GCK(cudaGetLastError());
  GCK(cudaMemsetAsync(d_pl + n, 0, sizeof(uint64_t), s));
  size_t tmp = 0;
  GCK(cub::DeviceScan::ExclusiveSum(nullptr, tmp, d_pl, d_pl, n + 1, s));
  void* d_tmp = nullptr;
  GCK(cudaMalloc(&d_tmp, tmp));
  GCK(cub::DeviceScan::ExclusiveSum(d_tmp, tmp, d_pl, d_pl, n + 1, s));
  k_set_offsets<<<1184, 256, 0, s>>>(d_hdr, d_pl, n);
  GCK(cudaGetLastError());
  GCK(cudaMemcpyAsync(total_planes, d_pl + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  GCK(cudaStreamSynchronize(s));
  GCK(cudaFree(d_tmp));
  GCK(cudaFree(d_pl));
  if (*total_planes >= (1ull << 32)) { snprintf(g_err, sizeof g_err, "chunk exceeds 2^32 planes"); return -1; }
  return 0;
}

int fpxgen_fill_device(const Params* p, uint64_t r0, const Hdr* d_hdr, uint64_t n, uint32_t* d_arena,
                       void* stream) {
  if (n == 0) return 0;
  k_fill<<<148 * 16, 256, 0, (cudaStream_t)stream>>>(*p, r0, d_hdr, n, d_arena);
  GCK(cudaGetLastError());
  return 0;
}

int fpxgen_apply_device(const Write* d_w, uint64_t nw, const Hdr* d_hdr, uint32_t* d_arena, void* stream) {
  if (nw == 0) return 0;
  unsigned blocks = (unsigned)((nw + 7) / 8);
  if (blocks > 148 * 16) blocks = 148 * 16;
  k_apply<<<blocks, 256, 0, (cudaStream_t)stream>>>(d_w, nw, d_hdr, d_arena);
  GCK(cudaGetLastError());
  return 0;
}

}  // extern "C"
