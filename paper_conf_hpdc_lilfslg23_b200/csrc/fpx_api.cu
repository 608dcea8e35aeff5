// fpx_api.cu — the C ABI of include/fpx.h: argument checking, handle state,
// launches on the caller's stream, and the cold fetch path.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "fpx_internal.h"

using namespace fpx;

struct fpx_ctx {
  int device = 0;
  bool attached = false;  // table mapped from another process (fpx_open_attached)
  int num_sms = 148;
  uint32_t variant = 0;  // record-scan kernel: 0 TMA ring, 1 LDG (ablation)
  bool force_storm = false;  // FPX_OPT_STORM: always the storm instantiation
  uint64_t slots = 0;
  TableView tv{};
  uint64_t newlog_cursor = 0;  // FETCH_NEW position
  cudaStream_t last_stream = nullptr;
  // fetch scratch (lazily sized to `slots`)
  uint64_t* d_keys = nullptr;
  uint64_t* d_counts = nullptr;
  uint64_t* d_first = nullptr;
  uint64_t* d_keys2 = nullptr;
  uint64_t* d_idx = nullptr;
  uint64_t* d_idx2 = nullptr;
  unsigned long long* d_n = nullptr;
  void* d_temp = nullptr;
  size_t temp_bytes = 0;
  Ctl* h_ctl = nullptr;  // pinned mirror of the counters
  // fpx_scan_tensors: device entry table + pinned staging (reused once the
  // previous copy completed)
  ListEntry* d_list = nullptr;
  ListEntry* h_list = nullptr;
  uint32_t list_cap = 0;
  cudaEvent_t list_copied = nullptr;  // the last H2D copy out of h_list is done
  cudaEvent_t list_used = nullptr;    // the last launch reading d_list is done
  // record-scan chunk counters (fpx_scan_records.cu Sched): kSchedSlots
  // pairs, one per launch in turn, so that launches in flight on different
  // streams never share one
  unsigned int* d_sched = nullptr;
  uint32_t sched_seq = 0;
  // early notification (FPX_OPT_LIVE_NEW): mapped pinned ring + poll cursor
  LiveSlot* h_live = nullptr;
  LiveSlot* d_live = nullptr;  // device view of h_live
  // record-scan density feedback (storm kernel selection): mapped host struct
  // + device accumulator
  ScanFeedback* h_fb = nullptr;
  ScanFeedback* d_fb_view = nullptr;
  unsigned long long* d_fb_acc = nullptr;
  uint32_t live_gen = 1;       // bumped at every reset
  uint64_t live_cursor = 0;
};
constexpr uint32_t kSchedSlots = 64;

namespace {

char g_cuda_err[512] = "";
std::mutex g_err_mu;

fpx_status cuda_err(cudaError_t e, const char* where) {
  std::lock_guard<std::mutex> lk(g_err_mu);
  snprintf(g_cuda_err, sizeof g_cuda_err, "%s: %s", where, cudaGetErrorString(e));
  return FPX_ERR_CUDA;
}

// The record scan's zeroed chunk counters (see fpx_ctx::d_sched).
bool alloc_sched(fpx_ctx* h) {
  const size_t b = 2 * sizeof(unsigned int) * kSchedSlots;
  if (cudaMalloc(&h->d_sched, b) != cudaSuccess) {
    cudaGetLastError();
    h->d_sched = nullptr;
    return false;
  }
  return cudaMemsetAsync(h->d_sched, 0, b, nullptr) == cudaSuccess;
}

// The record scan's density feedback (fpx_internal.h ScanFeedback).
bool alloc_feedback(fpx_ctx* h) {
  if (cudaHostAlloc(&h->h_fb, sizeof(ScanFeedback), cudaHostAllocMapped) != cudaSuccess) {
    cudaGetLastError();
    h->h_fb = nullptr;
    return false;
  }
  std::memset(h->h_fb, 0, sizeof(ScanFeedback));
  if (cudaHostGetDevicePointer(&h->d_fb_view, h->h_fb, 0) != cudaSuccess ||
      cudaMalloc(&h->d_fb_acc, sizeof(unsigned long long)) != cudaSuccess ||
      cudaMemsetAsync(h->d_fb_acc, 0, sizeof(unsigned long long), nullptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return true;
}

#define CK(x)                                                  \
  do {                                                         \
    cudaError_t _e = (x);                                      \
    if (_e != cudaSuccess) return cuda_err(_e, #x);            \
  } while (0)

// Runs `fn` with the handle's device current and restores the caller's.
struct DeviceGuard {
  int prev = -1;
  bool ok = true;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) { ok = false; return; }
    if (prev != dev && cudaSetDevice(dev) != cudaSuccess) ok = false;
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

fpx_status ensure_scratch(fpx_ctx* h) {
  if (h->d_keys) return FPX_OK;
  // allocate into locals and commit only when every allocation succeeded, so
  // a failure leaves the handle without scratch (the next call retries)
  // instead of with a half-built set
  const size_t b = sizeof(uint64_t) * h->slots;
  void* p[7] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
  void* temp = nullptr;
  size_t t1 = 0, t2 = 0;
  cudaError_t e = cudaSuccess;
  for (int i = 0; i < 7 && e == cudaSuccess; ++i) e = cudaMalloc(&p[i], i < 6 ? b : sizeof(unsigned long long));
  if (e == cudaSuccess)
    e = sort_keys_with_index(nullptr, &t1, static_cast<uint64_t*>(p[0]), static_cast<uint64_t*>(p[3]),
                             static_cast<uint64_t*>(p[4]), static_cast<uint64_t*>(p[5]), h->slots, nullptr);
  if (e == cudaSuccess)
    e = unique_keys(nullptr, &t2, static_cast<uint64_t*>(p[0]), static_cast<uint64_t*>(p[3]),
                    static_cast<unsigned long long*>(p[6]), h->slots, nullptr);
  if (e == cudaSuccess) e = cudaMalloc(&temp, std::max(t1, t2));
  if (e != cudaSuccess) {
    for (void* q : p)
      if (q) cudaFree(q);
    return cuda_err(e, "ensure_scratch");
  }
  h->d_keys = static_cast<uint64_t*>(p[0]);
  h->d_counts = static_cast<uint64_t*>(p[1]);
  h->d_first = static_cast<uint64_t*>(p[2]);
  h->d_keys2 = static_cast<uint64_t*>(p[3]);
  h->d_idx = static_cast<uint64_t*>(p[4]);
  h->d_idx2 = static_cast<uint64_t*>(p[5]);
  h->d_n = static_cast<unsigned long long*>(p[6]);
  h->d_temp = temp;
  h->temp_bytes = std::max(t1, t2);
  return FPX_OK;
}

fpx_status ensure_temp(fpx_ctx* h, size_t need) {
  if (need <= h->temp_bytes) return FPX_OK;
  void* t = nullptr;
  CK(cudaMalloc(&t, need));
  if (h->d_temp) cudaFree(h->d_temp);
  h->d_temp = t;
  h->temp_bytes = need;
  return FPX_OK;
}

// Sorted (key, count, first) of either the whole table or a key list, into
// h->d_keys2 / d_counts / d_first (the latter two reused as outputs);
// returns the number of entries in *n.
fpx_status sorted_entries(fpx_ctx* h, cudaStream_t s, const uint64_t* d_key_list, uint64_t n_list, uint64_t* n) {
  uint64_t cnt = 0;
  if (d_key_list == nullptr) {
    CK(launch_table_compact(h->tv, h->slots, h->d_keys, h->d_counts, h->d_first, h->d_n, s));
    unsigned long long hn = 0;
    CK(cudaMemcpyAsync(&hn, h->d_n, sizeof hn, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    cnt = hn;
  } else {
    cnt = n_list;
    if (cnt) CK(cudaMemcpyAsync(h->d_keys, d_key_list, cnt * 8, cudaMemcpyDeviceToDevice, s));
    CK(launch_table_lookup(h->tv, h->d_keys, cnt, h->d_counts, h->d_first, s));
  }
  *n = cnt;
  if (cnt == 0) return FPX_OK;
  CK(launch_iota(h->d_idx, cnt, s));
  size_t tb = 0;
  CK(sort_keys_with_index(nullptr, &tb, h->d_keys, h->d_keys2, h->d_idx, h->d_idx2, cnt, s));
  fpx_status st = ensure_temp(h, tb);
  if (st != FPX_OK) return st;
  tb = h->temp_bytes;
  CK(sort_keys_with_index(h->d_temp, &tb, h->d_keys, h->d_keys2, h->d_idx, h->d_idx2, cnt, s));
  // gather counts / firsts by the permutation into d_keys (reused) / d_idx (reused)
  CK(launch_gather3(h->d_idx2, cnt, h->d_counts, h->d_first, h->d_keys, h->d_idx, s));
  return FPX_OK;
}

fpx_status sticky_status(fpx_ctx* h, cudaStream_t s) {
  CK(cudaMemcpyAsync(h->h_ctl, h->tv.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (h->h_ctl->dropped_events) return FPX_ERR_TABLE_FULL;
  if (h->h_ctl->bad_records) return FPX_ERR_BAD_RECORD;
  return FPX_OK;
}

}  // namespace

extern "C" {

uint32_t fpx_abi_version(void) { return 1u; }
uint32_t fpx_sizeof_rec_hdr(void) { return (uint32_t)sizeof(fpx_rec_hdr); }
uint32_t fpx_sizeof_entry(void) { return (uint32_t)sizeof(fpx_entry); }

const char* fpx_strerror(fpx_status s) {
  switch (s) {
    case FPX_OK: return "ok";
    case FPX_ERR_INVALID: return "invalid argument";
    case FPX_ERR_CUDA: return "CUDA error";
    case FPX_ERR_NOMEM: return "out of memory";
    case FPX_ERR_TABLE_FULL: return "exception table full: events dropped";
    case FPX_ERR_BAD_RECORD: return "bad record(s) skipped";
    case FPX_ERR_TRUNCATED: return "output truncated to capacity";
  }
  return "unknown status";
}

const char* fpx_last_cuda_error(void) { return g_cuda_err; }

fpx_status fpx_open(int device, const fpx_options* opt, fpx_handle* out) {
  if (!out) return FPX_ERR_INVALID;
  *out = nullptr;
  fpx_options o{};
  if (opt) o = *opt;
  if ((o.flags & ~(uint32_t)(FPX_OPT_SCAN_LDG | FPX_OPT_NO_WARP_AGG | FPX_OPT_LIVE_NEW | FPX_OPT_STORM)) != 0)
    return FPX_ERR_INVALID;
  if (o.table_log2_slots == 0) o.table_log2_slots = 20;
  if (o.table_log2_slots < 4 || o.table_log2_slots > 30) return FPX_ERR_INVALID;
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return FPX_ERR_INVALID;
  DeviceGuard g(device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  fpx_ctx* h = new (std::nothrow) fpx_ctx();
  if (!h) return FPX_ERR_NOMEM;
  h->device = device;
  h->variant = (o.flags & FPX_OPT_SCAN_LDG) ? 1u : 0u;
  h->force_storm = (o.flags & FPX_OPT_STORM) != 0;
  h->slots = 1ull << o.table_log2_slots;
  // every failure below releases what was built so far through fpx_close
  // (which tolerates the members still null)
  auto fail = [&](fpx_status st) {
    cudaGetLastError();
    fpx_close(h);
    return st;
  };
  cudaError_t e = cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return fail(cuda_err(e, "cudaDeviceGetAttribute"));
  // the log never holds more keys than the table has slots
  const uint64_t cap = o.newlog_capacity ? std::min<uint64_t>(o.newlog_capacity, h->slots) : h->slots;
  if (cudaMalloc(&h->tv.slots, sizeof(Slot) * h->slots) != cudaSuccess ||
      cudaMalloc(&h->tv.newlog, sizeof(unsigned long long) * cap) != cudaSuccess ||
      cudaMalloc(&h->tv.newlog_slot, sizeof(unsigned int) * cap) != cudaSuccess ||
      cudaMalloc(&h->tv.ctl, sizeof(Ctl)) != cudaSuccess || cudaMallocHost(&h->h_ctl, sizeof(Ctl)) != cudaSuccess)
    return fail(FPX_ERR_NOMEM);
  h->tv.mask = h->slots - 1;
  h->tv.newlog_cap = cap;
  h->tv.flags = o.flags & FPX_OPT_NO_WARP_AGG;
  if (o.flags & FPX_OPT_LIVE_NEW) {
    // one 32-B slot per log position in host memory the kernels write through
    // the mapping (inserts are rare: a few PCIe writes per new key)
    if (cudaHostAlloc(&h->h_live, sizeof(LiveSlot) * cap, cudaHostAllocMapped) != cudaSuccess)
      return fail(FPX_ERR_NOMEM);
    std::memset(h->h_live, 0, sizeof(LiveSlot) * cap);
    e = cudaHostGetDevicePointer(&h->d_live, h->h_live, 0);
    if (e != cudaSuccess) return fail(cuda_err(e, "cudaHostGetDevicePointer"));
    h->tv.flags |= TV_LIVE;
  }
  e = launch_table_reset(h->tv, h->slots, h->d_live, h->live_gen, nullptr);
  if (e != cudaSuccess) return fail(cuda_err(e, "launch_table_reset"));
  if (!alloc_sched(h) || !alloc_feedback(h)) return fail(FPX_ERR_NOMEM);
  e = cudaStreamSynchronize(nullptr);
  if (e != cudaSuccess) return fail(cuda_err(e, "cudaStreamSynchronize"));
  *out = h;
  return FPX_OK;
}

fpx_status fpx_scan_records(fpx_handle h, const fpx_rec_hdr* d_hdr, uint64_t n_records, const uint32_t* d_arena,
                            uint64_t arena_planes, uint64_t base_index, uint32_t mode, void* stream) {
  if (!h) return FPX_ERR_INVALID;
  if (mode != FPX_MODE_DEST && mode != FPX_MODE_FLOW && mode != FPX_MODE_FLOW_DETAIL) return FPX_ERR_INVALID;
  if (n_records == 0) return FPX_OK;
  if (!d_hdr || !aligned16(d_hdr)) return FPX_ERR_INVALID;
  if (arena_planes && (!d_arena || !aligned16(d_arena))) return FPX_ERR_INVALID;
  if (base_index + n_records < base_index) return FPX_ERR_INVALID;  // index overflow
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  unsigned int* sched = h->d_sched + 2 * (h->sched_seq++ % kSchedSlots);
  // storm kernel when forced, or when the handle's last published DEST launch
  // sent at least a quarter of its tiles (~records / 32) to the exact path;
  // read without synchronising (the value may be a launch or two old)
  bool storm = h->force_storm;
  if (!storm && h->h_fb != nullptr) {
    const volatile ScanFeedback* fb = h->h_fb;
    const uint64_t recs = fb->records, hits = fb->hit_tiles;
    storm = recs != 0 && hits * 128u >= recs;
  }
  const FeedbackPtrs fbp{mode == FPX_MODE_DEST ? h->d_fb_acc : nullptr, h->d_fb_view};
  CK(launch_scan_records(d_hdr, n_records, d_arena, arena_planes, base_index, mode, h->tv, h->num_sms, h->variant,
                         sched, fbp, storm, s));
  h->last_stream = s;
  return FPX_OK;
}

fpx_status fpx_scan_tensor(fpx_handle h, const void* d_ptr, uint64_t n_elems, uint32_t fmt, uint32_t site,
                           uint64_t base_index, void* stream) {
  if (!h || fmt > FPX_BF16) return FPX_ERR_INVALID;
  if (n_elems == 0) return FPX_OK;
  const uintptr_t es = fmt == FPX_FP64 ? 8 : fmt == FPX_FP32 ? 4 : 2;
  if (!d_ptr || (reinterpret_cast<uintptr_t>(d_ptr) % es) != 0) return FPX_ERR_INVALID;
  if (base_index + n_elems < base_index) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CK(launch_scan_tensor(d_ptr, n_elems, fmt, site, base_index, h->tv, h->num_sms, s));
  h->last_stream = s;
  return FPX_OK;
}

fpx_status fpx_scan_tensors(fpx_handle h, const fpx_tensor_desc* descs, uint32_t n, void* stream) {
  if (!h || (n && !descs)) return FPX_ERR_INVALID;
  // validate everything before enqueuing anything
  uint32_t m = 0;
  for (uint32_t i = 0; i < n; ++i) {
    const fpx_tensor_desc& d = descs[i];
    if (d.fmt > FPX_BF16) return FPX_ERR_INVALID;
    if (d.n_elems == 0) continue;
    const uintptr_t es = d.fmt == FPX_FP64 ? 8 : d.fmt == FPX_FP32 ? 4 : 2;
    if (!d.ptr || (reinterpret_cast<uintptr_t>(d.ptr) % es) != 0) return FPX_ERR_INVALID;
    if (d.base_index + d.n_elems < d.base_index) return FPX_ERR_INVALID;
    ++m;
  }
  if (m == 0) return FPX_OK;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (!h->list_copied) CK(cudaEventCreateWithFlags(&h->list_copied, cudaEventDisableTiming));
  if (!h->list_used) CK(cudaEventCreateWithFlags(&h->list_used, cudaEventDisableTiming));
  CK(cudaEventSynchronize(h->list_copied));  // the host staging buffer's previous copy is done
  if (m > h->list_cap) {
    if (h->d_list) {
      CK(cudaEventSynchronize(h->list_used));  // the launch reading the old table (any stream) is done
      CK(cudaFree(h->d_list));
    }
    if (h->h_list) CK(cudaFreeHost(h->h_list));
    h->d_list = nullptr;
    h->h_list = nullptr;
    uint32_t cap = 64;
    while (cap < m) cap *= 2;
    if (cudaMalloc(&h->d_list, sizeof(ListEntry) * cap) != cudaSuccess ||
        cudaMallocHost(&h->h_list, sizeof(ListEntry) * cap) != cudaSuccess) {
      cudaGetLastError();
      if (h->d_list) cudaFree(h->d_list);
      h->d_list = nullptr;
      h->h_list = nullptr;
      h->list_cap = 0;
      return FPX_ERR_NOMEM;
    }
    h->list_cap = cap;
  }
  uint64_t vsum = 0, ssum = 0;
  uint32_t j = 0;
  for (uint32_t i = 0; i < n; ++i) {
    const fpx_tensor_desc& d = descs[i];
    if (d.n_elems == 0) continue;
    const uint32_t es = d.fmt == FPX_FP64 ? 8u : d.fmt == FPX_FP32 ? 4u : 2u;
    const uint32_t V = 16u / es;
    const uintptr_t a = reinterpret_cast<uintptr_t>(d.ptr);
    uint64_t head = ((16u - (uint32_t)(a & 15u)) & 15u) / es;
    if (head > d.n_elems) head = d.n_elems;
    const uint64_t nvec = (d.n_elems - head) / V;
    const uint64_t tail = d.n_elems - head - nvec * V;
    ListEntry& e = h->h_list[j++];
    e.ptr = static_cast<const uint8_t*>(d.ptr);
    e.base = d.base_index;
    e.vbegin = vsum;
    e.sbegin = ssum;
    e.nvec = nvec;
    e.head = (uint32_t)head;
    e.tail = (uint32_t)tail;
    e.fmt = d.fmt;
    e.site = d.site;
    vsum += nvec;
    ssum += head + tail;
  }
  // the device table may still be read by the previous launch on another
  // stream: this stream waits for it before overwriting
  CK(cudaStreamWaitEvent(s, h->list_used, 0));
  CK(cudaMemcpyAsync(h->d_list, h->h_list, sizeof(ListEntry) * m, cudaMemcpyHostToDevice, s));
  CK(cudaEventRecord(h->list_copied, s));
  CK(launch_scan_tensor_list(h->d_list, m, vsum, ssum, h->tv, h->num_sms, s));
  CK(cudaEventRecord(h->list_used, s));
  h->last_stream = s;
  return FPX_OK;
}

fpx_status fpx_table_fetch(fpx_handle h, fpx_entry* host_out, uint64_t capacity, uint64_t* n_total, uint32_t flags) {
  if (!h || !n_total || (capacity && !host_out)) return FPX_ERR_INVALID;
  if (flags != FPX_FETCH_ALL && flags != FPX_FETCH_NEW) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = h->last_stream;
  CK(cudaStreamSynchronize(s));
  fpx_status st = ensure_scratch(h);
  if (st != FPX_OK) return st;
  uint64_t n = 0, new_total = 0;
  if (flags == FPX_FETCH_ALL) {
    st = sorted_entries(h, s, nullptr, 0, &n);
    new_total = n;
  } else {
    // keys inserted since the previous FETCH_NEW, read from the device log in
    // insertion order: a window of at most `capacity` of them (sorted by key
    // within it), and the cursor moves past exactly the keys returned, so a
    // truncated call loses nothing (the next call continues from there)
    CK(cudaMemcpyAsync(h->h_ctl, h->tv.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const uint64_t tail = std::min<uint64_t>(h->h_ctl->newlog_tail, h->tv.newlog_cap);
    const uint64_t from = std::min<uint64_t>(h->newlog_cursor, tail);
    new_total = tail - from;
    const uint64_t take = std::min<uint64_t>(new_total, capacity);
    st = sorted_entries(h, s, reinterpret_cast<const uint64_t*>(h->tv.newlog) + from, take, &n);
    if (st == FPX_OK) h->newlog_cursor = from + take;
  }
  if (st != FPX_OK) return st;
  *n_total = new_total;
  const uint64_t m = std::min(n, capacity);
  if (m) {
    std::vector<uint64_t> k(m), c(m), f(m);
    CK(cudaMemcpyAsync(k.data(), h->d_keys2, m * 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(c.data(), h->d_keys, m * 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(f.data(), h->d_idx, m * 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    for (uint64_t i = 0; i < m; ++i) {
      fpx_entry e;
      std::memset(&e, 0, sizeof e);
      e.site = (uint32_t)(k[i] >> 32);
      e.fmt = (uint8_t)((k[i] >> 4) & 3);
      e.flow = (uint8_t)((k[i] >> 2) & 3);
      e.kind = (uint8_t)(k[i] & 3);
      e.detail = (uint8_t)((k[i] >> 6) & 7);
      e.count = c[i];
      e.first_index = f[i];
      host_out[i] = e;
    }
  }
  if (capacity < new_total) return FPX_ERR_TRUNCATED;
  return sticky_status(h, s);
}

fpx_status fpx_table_fetch_device(fpx_handle h, uint64_t* d_keys, uint64_t* d_counts, uint64_t* d_first,
                                  uint64_t capacity, uint64_t* n_total, void* stream) {
  if (!h || !n_total || (capacity && (!d_keys || !d_counts || !d_first))) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->last_stream != s) CK(cudaStreamSynchronize(h->last_stream));
  fpx_status st = ensure_scratch(h);
  if (st != FPX_OK) return st;
  uint64_t n = 0;
  st = sorted_entries(h, s, nullptr, 0, &n);
  if (st != FPX_OK) return st;
  *n_total = n;
  const uint64_t m = std::min(n, capacity);
  if (m) {
    CK(cudaMemcpyAsync(d_keys, h->d_keys2, m * 8, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(d_counts, h->d_keys, m * 8, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(d_first, h->d_idx, m * 8, cudaMemcpyDeviceToDevice, s));
  }
  CK(cudaStreamSynchronize(s));
  if (capacity < n) return FPX_ERR_TRUNCATED;
  return sticky_status(h, s);
}

fpx_status fpx_table_lookup_device(fpx_handle h, const uint64_t* d_keys, uint64_t n, uint64_t* d_counts,
                                   uint64_t* d_first, void* stream) {
  if (!h || (n && (!d_keys || !d_counts || !d_first))) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->last_stream != s) CK(cudaStreamSynchronize(h->last_stream));
  CK(launch_table_lookup(h->tv, d_keys, n, d_counts, d_first, s));
  return FPX_OK;
}

fpx_status fpx_keys_unique_device(fpx_handle h, const uint64_t* d_keys, uint64_t n, uint64_t* d_out, uint64_t* n_out,
                                  void* stream) {
  if (!h || !n_out || (n && (!d_keys || !d_out))) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  *n_out = 0;
  if (n == 0) return FPX_OK;
  fpx_status st = ensure_scratch(h);
  if (st != FPX_OK) return st;
  size_t tb = 0;
  CK(unique_keys(nullptr, &tb, d_keys, d_out, h->d_n, n, s));
  st = ensure_temp(h, tb);
  if (st != FPX_OK) return st;
  tb = h->temp_bytes;
  CK(unique_keys(h->d_temp, &tb, d_keys, d_out, h->d_n, n, s));
  unsigned long long hn = 0;
  CK(cudaMemcpyAsync(&hn, h->d_n, sizeof hn, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (hn) {
    uint64_t last = 0;
    CK(cudaMemcpy(&last, d_out + hn - 1, 8, cudaMemcpyDeviceToHost));
    if (last == FPX_KEY_EMPTY) hn--;
  }
  *n_out = hn;
  return FPX_OK;
}

fpx_status fpx_table_merge_device(fpx_handle h, const uint64_t* d_keys, const uint64_t* d_counts,
                                  const uint64_t* d_first, uint64_t n, void* stream) {
  if (!h || (n && (!d_keys || !d_counts || !d_first))) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->last_stream != s) CK(cudaStreamSynchronize(h->last_stream));
  CK(launch_table_merge(h->tv, d_keys, d_counts, d_first, n, s));
  h->last_stream = s;
  return FPX_OK;
}

fpx_status fpx_table_reset(fpx_handle h, void* stream) {
  if (!h || h->attached) return FPX_ERR_INVALID;  // the home handle owns the shared table
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->last_stream != s) CK(cudaStreamSynchronize(h->last_stream));
  // scans ordered after this reset publish under a new generation; ring slots
  // of the previous table (even ones written later by scans still in flight
  // on other streams) never match the poll's expected seq again
  h->live_gen += 1;
  CK(launch_table_reset_touched(h->tv, h->slots, h->d_live, h->live_gen, s));
  h->newlog_cursor = 0;
  h->live_cursor = 0;
  h->last_stream = s;
  return FPX_OK;
}

fpx_status fpx_poll_new(fpx_handle h, fpx_entry* host_out, uint64_t capacity, uint64_t* n_out) {
  if (!h || !n_out || (capacity && !host_out)) return FPX_ERR_INVALID;
  *n_out = 0;
  if (!h->h_live) return FPX_ERR_INVALID;  // the handle was opened without FPX_OPT_LIVE_NEW
  // plain loads of mapped host memory: no CUDA call, no stream synchronised
  const unsigned long long gen = (unsigned long long)h->live_gen << 32;
  uint64_t n = 0;
  while (n < capacity && h->live_cursor < h->tv.newlog_cap) {
    const LiveSlot* l = h->h_live + h->live_cursor;
    const unsigned long long seq = __atomic_load_n(&l->seq, __ATOMIC_ACQUIRE);
    if (seq != (gen | (h->live_cursor + 1))) break;  // not published yet (log order)
    const unsigned long long k = l->key;
    fpx_entry e;
    std::memset(&e, 0, sizeof e);
    e.site = (uint32_t)(k >> 32);
    e.fmt = (uint8_t)((k >> 4) & 3);
    e.flow = (uint8_t)((k >> 2) & 3);
    e.kind = (uint8_t)(k & 3);
    e.detail = (uint8_t)((k >> 6) & 7);
    e.count = l->count;
    e.first_index = l->first;
    host_out[n++] = e;
    ++h->live_cursor;
  }
  *n_out = n;
  return FPX_OK;
}

fpx_status fpx_get_stats(fpx_handle h, fpx_stats* out) {
  if (!h || !out) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  CK(cudaStreamSynchronize(h->last_stream));
  CK(cudaMemcpy(h->h_ctl, h->tv.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost));
  out->bad_records = h->h_ctl->bad_records;
  out->dropped_events = h->h_ctl->dropped_events;
  out->table_entries = std::min<uint64_t>(h->h_ctl->newlog_tail, h->slots);
  out->newlog_overflow = h->h_ctl->newlog_overflow;
  return FPX_OK;
}

fpx_status fpx_table_export(fpx_handle h, fpx_ipc_table* out) {
  if (!h || !out || h->attached) return FPX_ERR_INVALID;
  DeviceGuard g(h->device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  std::memset(out, 0, sizeof *out);
  void* bases[4] = {h->tv.slots, h->tv.newlog, h->tv.newlog_slot, h->tv.ctl};
  for (int i = 0; i < 4; ++i) {
    cudaIpcMemHandle_t m;
    CK(cudaIpcGetMemHandle(&m, bases[i]));
    static_assert(sizeof(m) == 64, "cudaIpcMemHandle_t is 64 bytes");
    std::memcpy(out->ipc[i], &m, sizeof m);
  }
  uint32_t lg = 0;
  while ((1ull << lg) < h->slots) ++lg;
  out->table_log2_slots = lg;
  out->newlog_capacity = (uint32_t)h->tv.newlog_cap;
  out->home_device = h->device;
  out->magic = FPX_IPC_MAGIC;
  // other GPUs will update this table concurrently: the home's own scans
  // switch to system-scope atomics too
  h->tv.flags |= TV_SHARED;
  return FPX_OK;
}

fpx_status fpx_open_attached(int device, const fpx_ipc_table* t, fpx_handle* out) {
  if (!out || !t || t->magic != FPX_IPC_MAGIC) return FPX_ERR_INVALID;
  if (t->table_log2_slots < 4 || t->table_log2_slots > 30 || t->newlog_capacity == 0) return FPX_ERR_INVALID;
  *out = nullptr;
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return FPX_ERR_INVALID;
  DeviceGuard g(device);
  if (!g.ok) return cuda_err(cudaGetLastError(), "cudaSetDevice");
  fpx_ctx* h = new (std::nothrow) fpx_ctx();
  if (!h) return FPX_ERR_NOMEM;
  h->device = device;
  h->attached = true;
  cudaError_t ea = cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, device);
  if (ea != cudaSuccess) {
    delete h;
    return cuda_err(ea, "cudaDeviceGetAttribute");
  }
  h->slots = 1ull << t->table_log2_slots;
  void* ptrs[4] = {nullptr, nullptr, nullptr, nullptr};
  for (int i = 0; i < 4; ++i) {
    cudaIpcMemHandle_t m;
    std::memcpy(&m, t->ipc[i], sizeof m);
    cudaError_t e = cudaIpcOpenMemHandle(&ptrs[i], m, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      for (int j = 0; j < i; ++j) cudaIpcCloseMemHandle(ptrs[j]);
      delete h;
      return cuda_err(e, "cudaIpcOpenMemHandle");
    }
  }
  h->tv.slots = static_cast<Slot*>(ptrs[0]);
  h->tv.mask = h->slots - 1;
  h->tv.newlog = static_cast<unsigned long long*>(ptrs[1]);
  h->tv.newlog_slot = static_cast<unsigned int*>(ptrs[2]);
  h->tv.ctl = static_cast<Ctl*>(ptrs[3]);
  h->tv.newlog_cap = t->newlog_capacity;
  h->tv.flags = TV_SHARED;  // concurrent updates from several GPUs: system-scope atomics
  if (cudaMallocHost(&h->h_ctl, sizeof(Ctl)) != cudaSuccess) {
    for (int j = 0; j < 4; ++j) cudaIpcCloseMemHandle(ptrs[j]);
    delete h;
    return FPX_ERR_NOMEM;
  }
  if (!alloc_sched(h) || !alloc_feedback(h)) {
    fpx_close(h);
    return FPX_ERR_NOMEM;
  }
  ea = cudaStreamSynchronize(nullptr);
  if (ea != cudaSuccess) {
    fpx_close(h);
    return cuda_err(ea, "cudaStreamSynchronize");
  }
  *out = h;
  return FPX_OK;
}

fpx_status fpx_close(fpx_handle h) {
  if (!h) return FPX_ERR_INVALID;
  {
    DeviceGuard g(h->device);
    cudaDeviceSynchronize();
    if (h->attached) {
      cudaIpcCloseMemHandle(h->tv.slots);
      cudaIpcCloseMemHandle(h->tv.newlog);
      cudaIpcCloseMemHandle(h->tv.newlog_slot);
      cudaIpcCloseMemHandle(h->tv.ctl);
    } else {
      cudaFree(h->tv.slots);
      cudaFree(h->tv.newlog);
      cudaFree(h->tv.newlog_slot);
      cudaFree(h->tv.ctl);
    }
    cudaFreeHost(h->h_ctl);
    if (h->h_live) cudaFreeHost(h->h_live);
    if (h->h_fb) cudaFreeHost(h->h_fb);
    if (h->d_fb_acc) cudaFree(h->d_fb_acc);
    if (h->h_list) cudaFreeHost(h->h_list);
    if (h->d_list) cudaFree(h->d_list);
    if (h->list_copied) cudaEventDestroy(h->list_copied);
    if (h->list_used) cudaEventDestroy(h->list_used);
    for (void* p : {(void*)h->d_keys, (void*)h->d_counts, (void*)h->d_first, (void*)h->d_keys2, (void*)h->d_idx,
                    (void*)h->d_idx2, (void*)h->d_n, h->d_temp, (void*)h->d_sched})
      if (p) cudaFree(p);
  }
  delete h;
  return FPX_OK;
}

}  // extern "C"
