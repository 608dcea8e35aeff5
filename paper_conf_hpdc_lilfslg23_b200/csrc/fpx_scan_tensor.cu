// fpx_scan_tensor.cu — destination-only scan of a plain FP32/FP64/FP16/BF16
// buffer (the SRU case P:711-715 recast for model activations).
//
// 128-bit loads of the 16-B-aligned body, TU vectors in flight per thread,
// grid-stride over a persistent grid (8 CTAs x 256 threads per SM).  A few
// integer ops per value keep min / max witnesses of "subnormal" and
// "exponent all ones"; one vote per batch; exact classification, per-kind
// warp reduction and table update only for hit batches.  Misaligned heads and
// ragged tails (< one vector each) are classified by one warp.
#include <cuda_runtime.h>

#include "fpx_device.cuh"

namespace fpx {
namespace {

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
  // Exact witnesses (see witness_hit): FP32 a2 = |x| << 1 (x + x: FMA pipe);
  // FP64 a3 = |hi| | (lo != 0); packed halves per halfword.
  if (FMT == FPX_FP32) {
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint32_t a2 = w[k] + w[k];
      mn = min(mn, a2 - 2u);
      mx = max(mx, a2);
    }
  } else if (FMT == FPX_FP64) {
    const uint32_t lo[2] = {q.x, q.z}, hi[2] = {q.y, q.w};
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const uint32_t a3 = (hi[k] & 0x7FFFFFFFu) | min(lo[k], 1u);
      mn = min(mn, a3 - 1u);
      mx = max(mx, a3);
    }
  } else {
    // packed halves, doubled (x + x: FMA pipe): each half's exponent moves to
    // the top of its halfword and the signs drop out (the low half's sign
    // lands in bit 0 of the high half, below every threshold that matters);
    // then per-halfword DPX min / max (VIADDMNMX.U16x2, VIMNMX3.U16x2)
    const uint32_t a = q.x + q.x, b = q.y + q.y, c = q.z + q.z, d = q.w + q.w;
    mn = __viaddmin_u16x2(a, 0xFFFEFFFEu, mn);  // h - 2 per half (0, 1 -> 0xFFFE, 0xFFFF)
    mn = __viaddmin_u16x2(b, 0xFFFEFFFEu, mn);
    mn = __viaddmin_u16x2(c, 0xFFFEFFFEu, mn);
    mn = __viaddmin_u16x2(d, 0xFFFEFFFEu, mn);
    mx = __vimax3_u16x2(a, b, mx);
    mx = __vimax3_u16x2(c, d, mx);
  }
}
template <uint32_t FMT>
__device__ __forceinline__ bool witness_hit(uint32_t mn, uint32_t mx) {
  if (FMT == FPX_FP32) return mn < 0x00FFFFFEu || mx >= 0xFF000000u;  // subnormal | INF/NaN
  if (FMT == FPX_FP64) return mn < 0x000FFFFFu || mx >= 0x7FF00000u;
  const uint32_t lo = min(mn & 0xFFFFu, mn >> 16), hi = max(mx & 0xFFFFu, mx >> 16);
  // doubled halves h = 2|x| (+ 1 for a high half with a negative low half):
  // subnormal <=> 2 <= h <= 2 * max_mantissa + 1; INF/NaN <=> h >= 2 * exponent mask
  if (FMT == FPX_FP16) return lo < 0x07FEu || hi >= 0xF800u;
  return lo < 0x00FEu || hi >= 0xFF00u;
}

constexpr int TU = 4;  // vectors per thread per batch

// Exact per-warp reduction of per-lane kind counts and first offsets.
__device__ __forceinline__ void flush_kinds(const TableView& tv, uint32_t site, uint32_t fmt, const uint32_t cnt[3],
                                            const uint32_t first_off[3], uint64_t idx0) {
  PendingEvents pend;
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const uint32_t tot = __reduce_add_sync(FULL, cnt[k]);
    if (tot) {
      const uint32_t f = __reduce_min_sync(FULL, first_off[k]);
      pend.push(tv, make_key(site, fmt, (uint32_t)k), tot, idx0 + f);
    }
  }
  pend.flush(tv);  // the (at most 3) kinds update the table in parallel
}

static_assert(TU == 4, "tensor_exact takes four vectors");

// Exact classification of one thread's hit batch (rare), no warp collectives:
// only vectors whose own witness fires are classified (FP16 randn: ~5 % of
// batches hold a natural subnormal, ~0.04 % of vectors), and the per-kind
// (count, first body offset) go to the CTA's shared accumulators.  Every
// event of one tensor has the same site and format, so the table sees one
// update per kind per CTA, at the end of the kernel.
template <uint32_t FMT>
__device__ __noinline__ void tensor_exact(uint4 q0, uint4 q1, uint4 q2, uint4 q3, uint64_t v0, uint64_t nthr,
                                          uint64_t nvec, unsigned long long* s_cnt, unsigned long long* s_first) {
  constexpr uint32_t V = TensorTraits<FMT>::V;
  const uint4 q[TU] = {q0, q1, q2, q3};
  uint32_t cnt[3] = {0, 0, 0};
  unsigned long long fo[3] = {~0ull, ~0ull, ~0ull};
#pragma unroll
  for (int u = 0; u < TU; ++u) {
    const uint64_t v = v0 + (uint64_t)u * nthr;
    if (v >= nvec) continue;
    uint32_t mn = 0xFFFFFFFFu, mx = 0u;
    vec_witness<FMT>(q[u], mn, mx);
    if (!witness_hit<FMT>(mn, mx)) continue;
#pragma unroll
    for (uint32_t e = 0; e < V; ++e) {
      const int k = kind_of_cls(vec_cls<FMT>(q[u], e));
      const unsigned long long off = v * V + e;
#pragma unroll
      for (int kk = 0; kk < 3; ++kk)
        if (k == kk) { cnt[kk]++; fo[kk] = min(fo[kk], off); }
    }
  }
#pragma unroll
  for (int k = 0; k < 3; ++k)
    if (cnt[k]) {
      atomicAdd(&s_cnt[k], (unsigned long long)cnt[k]);
      atomicMin(&s_first[k], fo[k]);
    }
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

  // body: batches of TU vectors per thread, grid-stride; per-thread control
  // flow only (no collectives), events accumulate per CTA in shared memory
  __shared__ unsigned long long s_cnt[3], s_first[3];
  if (threadIdx.x < 3) {
    s_cnt[threadIdx.x] = 0ull;
    s_first[threadIdx.x] = ~0ull;
  }
  __syncthreads();
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
    if (witness_hit<FMT>(mn, mx)) tensor_exact<FMT>(q[0], q[1], q[2], q[3], v0, nthr, nvec, s_cnt, s_first);
  }
  __syncthreads();
  if (threadIdx.x < 3 && s_cnt[threadIdx.x] != 0ull)
    table_add(tv, make_key(site, FMT, threadIdx.x), s_cnt[threadIdx.x], base_index + idx_body + s_first[threadIdx.x]);
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


// ---- many tensors in one launch (fpx_scan_tensors) --------------------------
// Work items: every 16-B body vector of every tensor (prefix vbegin), then
// every misaligned-head / ragged-tail scalar (prefix sbegin).  A thread finds
// its tensor by binary search over the (L1-resident) entry table.  Lanes of a
// warp may belong to different tensors, so the rare exact path groups lanes by
// tensor before aggregating.
__device__ __forceinline__ uint32_t find_entry(const ListEntry* __restrict__ e, uint32_t n, uint64_t w, bool scalar) {
  uint32_t lo = 0, hi = n - 1;  // last entry whose begin <= w
  while (lo < hi) {
    const uint32_t mid = (lo + hi + 1) / 2;
    const uint64_t b = scalar ? e[mid].sbegin : e[mid].vbegin;
    if (b <= w) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ uint32_t any_cls(uint32_t fmt, uint32_t lo, uint32_t hi) { return cls_val(fmt, lo, hi); }

__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long t = __shfl_xor_sync(FULL, v, o);
    v = t < v ? t : v;
  }
  return v;
}

// Per-lane (count, first) for each kind -> grouped by tensor -> table.
__device__ __noinline__ void list_exact_flush(const ListEntry* __restrict__ ents, int ti, const uint32_t cnt[3],
                                              const unsigned long long first[3], const TableView tv) {
  PendingEvents pend;
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const int code = cnt[k] ? ti : -1;
    uint32_t pending = __ballot_sync(FULL, code >= 0);
    while (pending) {
      const int leader = __ffs(pending) - 1;
      const int t = __shfl_sync(FULL, code, leader);
      const bool mine = code == t;
      const uint32_t peers = __ballot_sync(FULL, mine);
      const uint32_t tot = __reduce_add_sync(FULL, mine ? cnt[k] : 0u);
      const unsigned long long f = warp_min_u64(mine ? first[k] : ~0ull);
      const ListEntry& e = ents[t];
      pend.push(tv, make_key(e.site, e.fmt, (uint32_t)k), tot, f);
      pending &= ~peers;
    }
  }
  pend.flush(tv);
}

__global__ void __launch_bounds__(256, 6)
k_scan_tensor_list(const ListEntry* __restrict__ ents, uint32_t n_ent, uint64_t total_vec, uint64_t total_scalar,
                   const TableView tv) {
  const uint64_t nthr = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  // body vectors (loop bound is warp-uniform so the exact path's collectives see the full warp)
  const uint64_t vtrips = (total_vec + nthr - 1) / nthr;
  for (uint64_t it = 0; it < vtrips; ++it) {
    const uint64_t w = it * nthr + tid;
    int ti = -1;
    uint32_t fmt = 0;
    uint4 q = make_uint4(0u, 0u, 0u, 0u);
    bool hit = false;
    if (w < total_vec) {
      ti = (int)find_entry(ents, n_ent, w, false);
      const ListEntry& e = ents[ti];
      fmt = e.fmt;
      const uint32_t es = fmt == FPX_FP64 ? 8u : fmt == FPX_FP32 ? 4u : 2u;
      q = ld_stream4(e.ptr + (uint64_t)e.head * es + (w - e.vbegin) * 16);
      uint32_t mn = 0xFFFFFFFFu, mx = 0u;
      switch (fmt) {
        case FPX_FP32: vec_witness<FPX_FP32>(q, mn, mx); hit = witness_hit<FPX_FP32>(mn, mx); break;
        case FPX_FP64: vec_witness<FPX_FP64>(q, mn, mx); hit = witness_hit<FPX_FP64>(mn, mx); break;
        case FPX_FP16: vec_witness<FPX_FP16>(q, mn, mx); hit = witness_hit<FPX_FP16>(mn, mx); break;
        default: vec_witness<FPX_BF16>(q, mn, mx); hit = witness_hit<FPX_BF16>(mn, mx); break;
      }
    }
    if (__any_sync(FULL, hit)) {
      uint32_t cnt[3] = {0, 0, 0};
      unsigned long long first[3] = {~0ull, ~0ull, ~0ull};
      if (hit) {
        const ListEntry& e = ents[ti];
        const uint32_t V = fmt == FPX_FP64 ? 2u : fmt == FPX_FP32 ? 4u : 8u;
        const uint64_t e0 = e.base + e.head + (w - e.vbegin) * V;  // global index of the vector's first value
        const uint32_t wd[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
        for (uint32_t v = 0; v < 8; ++v) {
          if (v >= V) break;
          uint32_t lo, hi = 0;
          if (fmt == FPX_FP64) { lo = wd[(2 * v) & 3]; hi = wd[(2 * v + 1) & 3]; }
          else if (fmt == FPX_FP32) lo = wd[v & 3];
          else lo = (wd[(v / 2) & 3] >> (16 * (v & 1))) & 0xFFFFu;
          const int k = kind_of_cls(any_cls(fmt, lo, hi));
#pragma unroll
          for (int kk = 0; kk < 3; ++kk)
            if (k == kk) { cnt[kk]++; first[kk] = min(first[kk], (unsigned long long)(e0 + v)); }
        }
      }
      list_exact_flush(ents, hit ? ti : -1, cnt, first, tv);
    }
  }
  // misaligned heads and ragged tails, one scalar per thread
  const uint64_t strips = (total_scalar + nthr - 1) / nthr;
  for (uint64_t it = 0; it < strips; ++it) {
    const uint64_t w = it * nthr + tid;
    int ti = -1;
    uint32_t cnt[3] = {0, 0, 0};
    unsigned long long first[3] = {~0ull, ~0ull, ~0ull};
    if (w < total_scalar) {
      ti = (int)find_entry(ents, n_ent, w, true);
      const ListEntry& e = ents[ti];
      const uint32_t es = e.fmt == FPX_FP64 ? 8u : e.fmt == FPX_FP32 ? 4u : 2u;
      const uint32_t V = 16u / es;
      const uint64_t r = w - e.sbegin;
      const uint64_t el = r < e.head ? r : e.head + e.nvec * V + (r - e.head);
      const uint8_t* a = e.ptr + el * es;
      uint32_t lo = 0, hi = 0;
      if (es == 8) { lo = *(const uint32_t*)a; hi = *(const uint32_t*)(a + 4); }
      else if (es == 4) lo = *(const uint32_t*)a;
      else lo = *(const uint16_t*)a;
      const int k = kind_of_cls(any_cls(e.fmt, lo, hi));
#pragma unroll
      for (int kk = 0; kk < 3; ++kk)
        if (k == kk) { cnt[kk] = 1; first[kk] = e.base + el; }
    }
    const bool any = cnt[0] | cnt[1] | cnt[2];
    if (__any_sync(FULL, any)) list_exact_flush(ents, any ? ti : -1, cnt, first, tv);
  }
}

}  // namespace

cudaError_t launch_scan_tensor_list(const ListEntry* d_entries, uint32_t n, uint64_t total_vec, uint64_t total_scalar,
                                    const TableView& tv, int num_sms, cudaStream_t s) {
  if (n == 0 || total_vec + total_scalar == 0) return cudaSuccess;
  uint64_t blocks = (total_vec + 1023) / 1024;
  const uint64_t cap = (uint64_t)num_sms * 8;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  k_scan_tensor_list<<<(unsigned)blocks, 256, 0, s>>>(d_entries, n, total_vec, total_scalar, tv);
  return cudaGetLastError();
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
