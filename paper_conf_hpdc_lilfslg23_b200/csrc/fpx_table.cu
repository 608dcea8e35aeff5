// fpx_table.cu — device table maintenance and the cold fetch path.
//
// reset      fill slots with {EMPTY, 0, UINT64_MAX, 0}
// compact    non-empty slots -> dense (key, count, first) arrays
// lookup     per key: count / first (0 / INT64_MAX when absent) — the dense
//            scatter step of the multi-GPU merge (SURVEY §8 e)
// merge      add (key, count, first) triples through the same insert path as
//            the scans (re-import of a fetched / merged table)
// sort / unique via CUB radix sort (a library primitive; off the hot path)
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include "fpx_device.cuh"

namespace fpx {
namespace {

__global__ void k_reset(Slot* slots, uint64_t n, Ctl* ctl, LiveSlot* live, uint32_t live_gen) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    Slot s;
    s.key = FPX_KEY_EMPTY;
    s.count = 0;
    s.first = ~0ull;
    s.pad = 0;
    slots[i] = s;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    Ctl c{};
    c.live = live;
    c.live_gen = live_gen;
    *ctl = c;
  }
}

__device__ __forceinline__ void clear_slot(Slot* slots, uint64_t i) {
  Slot s;
  s.key = FPX_KEY_EMPTY;
  s.count = 0;
  s.first = ~0ull;
  s.pad = 0;
  slots[i] = s;
}

// every occupied slot was logged at insert (unless the log overflowed)
__global__ void k_reset_touched(const TableView tv, uint64_t slots) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const unsigned long long tail = tv.ctl->newlog_tail;
  if (tv.ctl->newlog_overflow != 0 || tail > tv.newlog_cap) {
    for (uint64_t i = t0; i < slots; i += stride) clear_slot(tv.slots, i);
  } else {
    for (uint64_t i = t0; i < tail; i += stride) clear_slot(tv.slots, tv.newlog_slot[i]);
  }
}

// counters and padding (the whole block is copied to the host)
__global__ void k_reset_ctl(Ctl* ctl, LiveSlot* live, uint32_t live_gen) {
  Ctl c{};
  c.live = live;
  c.live_gen = live_gen;
  *ctl = c;
}

__global__ void k_compact(const Slot* slots, uint64_t n, uint64_t* keys, uint64_t* counts, uint64_t* firsts,
                          unsigned long long* d_n) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    const Slot s = slots[i];
    if (s.key != FPX_KEY_EMPTY) {
      const unsigned long long at = atomicAdd(d_n, 1ull);
      keys[at] = s.key;
      counts[at] = s.count;
      firsts[at] = s.first;
    }
  }
}

__device__ __forceinline__ const Slot* find(const TableView& tv, unsigned long long key) {
  if (key == FPX_KEY_EMPTY) return nullptr;
  unsigned long long i = hash_key(key) & tv.mask;
  for (unsigned long long probe = 0; probe <= tv.mask; ++probe) {
    const Slot* s = tv.slots + i;
    const unsigned long long k = s->key;
    if (k == key) return s;
    if (k == FPX_KEY_EMPTY) return nullptr;
    i = (i + 1) & tv.mask;
  }
  return nullptr;
}

__global__ void k_lookup(const TableView tv, const uint64_t* keys, uint64_t n, uint64_t* counts, uint64_t* firsts) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    const Slot* s = find(tv, keys[i]);
    counts[i] = s ? s->count : 0ull;
    firsts[i] = s ? s->first : 0x7FFFFFFFFFFFFFFFull;
  }
}

__global__ void k_merge(const TableView tv, const uint64_t* keys, const uint64_t* counts, const uint64_t* firsts,
                        uint64_t n) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    const uint64_t k = keys[i];
    if (k == FPX_KEY_EMPTY || counts[i] == 0) continue;
    table_add(tv, k, counts[i], firsts[i]);
  }
}

__global__ void k_iota(uint64_t* d, uint64_t n) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) d[i] = i;
}

__global__ void k_gather(const uint64_t* idx, uint64_t n, const uint64_t* c_in, const uint64_t* f_in, uint64_t* c_out,
                         uint64_t* f_out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    const uint64_t j = idx[i];
    c_out[i] = c_in[j];
    f_out[i] = f_in[j];
  }
}

unsigned grid_for(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  if (b > 148 * 16) b = 148 * 16;
  return (unsigned)(b ? b : 1);
}

}  // namespace

cudaError_t launch_table_reset(const TableView& tv, uint64_t slots, LiveSlot* live, uint32_t live_gen, cudaStream_t s) {
  k_reset<<<grid_for(slots), 256, 0, s>>>(tv.slots, slots, tv.ctl, live, live_gen);
  return cudaGetLastError();
}

cudaError_t launch_table_reset_touched(const TableView& tv, uint64_t slots, LiveSlot* live, uint32_t live_gen,
                                      cudaStream_t s) {
  k_reset_touched<<<148 * 4, 256, 0, s>>>(tv, slots);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  k_reset_ctl<<<1, 1, 0, s>>>(tv.ctl, live, live_gen);
  return cudaGetLastError();
}

cudaError_t launch_table_compact(const TableView& tv, uint64_t slots, uint64_t* d_keys, uint64_t* d_counts,
                                 uint64_t* d_first, unsigned long long* d_n, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(d_n, 0, sizeof(unsigned long long), s);
  if (e != cudaSuccess) return e;
  k_compact<<<grid_for(slots), 256, 0, s>>>(tv.slots, slots, d_keys, d_counts, d_first, d_n);
  return cudaGetLastError();
}

cudaError_t launch_table_lookup(const TableView& tv, const uint64_t* d_keys, uint64_t n, uint64_t* d_counts,
                                uint64_t* d_first, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_lookup<<<grid_for(n), 256, 0, s>>>(tv, d_keys, n, d_counts, d_first);
  return cudaGetLastError();
}

cudaError_t launch_table_merge(const TableView& tv, const uint64_t* d_keys, const uint64_t* d_counts,
                               const uint64_t* d_first, uint64_t n, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_merge<<<grid_for(n), 256, 0, s>>>(tv, d_keys, d_counts, d_first, n);
  return cudaGetLastError();
}

cudaError_t launch_iota(uint64_t* d, uint64_t n, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_iota<<<grid_for(n), 256, 0, s>>>(d, n);
  return cudaGetLastError();
}

cudaError_t launch_gather3(const uint64_t* d_idx, uint64_t n, const uint64_t* c_in, const uint64_t* f_in,
                           uint64_t* c_out, uint64_t* f_out, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_gather<<<grid_for(n), 256, 0, s>>>(d_idx, n, c_in, f_in, c_out, f_out);
  return cudaGetLastError();
}

cudaError_t sort_keys_with_index(void* d_temp, size_t* temp_bytes, const uint64_t* d_keys_in, uint64_t* d_keys_out,
                                 const uint64_t* d_idx_in, uint64_t* d_idx_out, uint64_t n, cudaStream_t s) {
  return cub::DeviceRadixSort::SortPairs(d_temp, *temp_bytes, d_keys_in, d_keys_out, d_idx_in, d_idx_out, (int)n, 0,
                                         64, s);
}

// Sort + unique + drop EMPTY.  d_out receives the unique keys; *d_nout their number.
// Temp layout: [sorted keys: n x 8][cub temp].
cudaError_t unique_keys(void* d_temp, size_t* temp_bytes, const uint64_t* d_in, uint64_t* d_out,
                        unsigned long long* d_nout, uint64_t n, cudaStream_t s) {
  size_t sort_b = 0, uniq_b = 0;
  cudaError_t e = cub::DeviceRadixSort::SortKeys(nullptr, sort_b, d_in, d_out, (int)n, 0, 64, s);
  if (e != cudaSuccess) return e;
  e = cub::DeviceSelect::Unique(nullptr, uniq_b, d_out, d_out, d_nout, (int)n, s);
  if (e != cudaSuccess) return e;
  const size_t keys_b = ((n * 8 + 255) / 256) * 256;
  const size_t need = keys_b + (sort_b > uniq_b ? sort_b : uniq_b);
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return cudaSuccess;
  }
  uint64_t* sorted = static_cast<uint64_t*>(d_temp);
  void* cub_tmp = static_cast<char*>(d_temp) + keys_b;
  size_t tb = need - keys_b;
  e = cub::DeviceRadixSort::SortKeys(cub_tmp, tb, d_in, sorted, (int)n, 0, 64, s);
  if (e != cudaSuccess) return e;
  tb = need - keys_b;
  // EMPTY (all ones) sorts last; unique keeps one copy of it, dropped by the caller's count fix-up
  return cub::DeviceSelect::Unique(cub_tmp, tb, sorted, d_out, d_nout, (int)n, s);
}

}  // namespace fpx
