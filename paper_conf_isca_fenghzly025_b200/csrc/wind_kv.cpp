// wind_kv.cpp — host side of the C ABI (include/wind_kv.h): pools and peer mapping,
// argument checking, table validation, planners, tickets / layer waits, and the launch of
// the copy kernels (wind_kv_kernels.cu).  No allocation and no host synchronisation on the
// migrate / swap / compact path: everything an op needs (layer
// flags, arrival-counter ring) is allocated when a pool is created or imported.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <dlfcn.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges show up in ncu / nsys, free otherwise

#include "wind_kv_internal.h"

using namespace wkv;

// --------------------------------------------------------------------------- errors

namespace {

thread_local std::string g_last_error;
std::atomic<uint64_t> g_launches{0};

wind_status fail(wind_status code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

wind_status cuda_fail(cudaError_t e, const char* what) {
  return fail(WIND_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define WKV_CUDA(call, what)                        \
  do {                                              \
    cudaError_t _e = (call);                        \
    if (_e != cudaSuccess) return cuda_fail(_e, what); \
  } while (0)

// Restores the caller's current device on scope exit.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int now = -1;
    cudaGetDevice(&now);
    if (prev >= 0 && now != prev) cudaSetDevice(prev);
  }
};

// ------------------------------------------------------------- driver entry points

typedef CUresult (*PFN_waitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*PFN_getAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr);

template <typename F>
F driver_fn(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPointByVersion(name, &fn, 12000, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return nullptr;
  return reinterpret_cast<F>(fn);
}

// ------------------------------------------------------------ per-device context

struct DevCtx {
  std::mutex mu;
  bool ready = false;
  int sms = 0;
  uint8_t uuid[16] = {};
  uint32_t* counters = nullptr;  // kCounterSlots * WIND_KV_MAX_LAYERS, zeroed
  unsigned long long* stamps = nullptr;  // kCounterSlots: start time of a burst-paced op
  // Eager slot ownership (take_slot): after every eager op, done[s] is recorded on the op's
  // stream; slot s is free for another stream once done[s] has completed.
  std::mutex slot_mu;
  cudaEvent_t done[kEagerSlots] = {};
  bool used[kEagerSlots] = {};
  unsigned long long owner[kEagerSlots] = {};  // stream id of the slot's last op (0: unknown)
  std::unordered_map<unsigned long long, int> slot_of_stream;
  int cursor = 0;
  std::atomic<uint64_t> graph_seq{0};
  size_t tma_smem_set = 0;
  int32_t* err = nullptr;        // debug device-check word
  // debug table-check scratch, per counter slot: the op owning the slot is its only user
  // (two debug ops on different streams never share one)
  uint32_t* scratch[kCounterSlots] = {};
  int32_t scratch_n[kCounterSlots] = {};
};

constexpr int kMaxDevices = 64;
constexpr int kStageBufs = 3;  // staging buffers per host pool: a gather (scatter) may run
                               // two chunks ahead of the PCIe copies
DevCtx g_dev[kMaxDevices];

wind_status dev_ctx(int dev, DevCtx** out) {
  if (dev < 0 || dev >= kMaxDevices) return fail(WIND_ERR_INVALID_ARG, "device %d out of range", dev);
  DevCtx& c = g_dev[dev];
  std::lock_guard<std::mutex> lk(c.mu);
  if (!c.ready) {
    int n = 0;
    WKV_CUDA(cudaGetDeviceCount(&n), "cudaGetDeviceCount");
    if (dev >= n) return fail(WIND_ERR_INVALID_ARG, "device %d not present (%d devices)", dev, n);
    DeviceGuard g(dev);
    cudaDeviceProp prop;
    WKV_CUDA(cudaGetDeviceProperties(&prop, dev), "cudaGetDeviceProperties");
    c.sms = prop.multiProcessorCount;
    memcpy(c.uuid, &prop.uuid, 16);
    const size_t cbytes = sizeof(uint32_t) * kCounterSlots * WIND_KV_MAX_LAYERS;
    WKV_CUDA(cudaMalloc(&c.counters, cbytes), "cudaMalloc(counters)");
    WKV_CUDA(cudaMemset(c.counters, 0, cbytes), "cudaMemset(counters)");
    WKV_CUDA(cudaMalloc(&c.stamps, sizeof(unsigned long long) * kCounterSlots), "cudaMalloc(stamps)");
    for (int i = 0; i < kEagerSlots; ++i)
      WKV_CUDA(cudaEventCreateWithFlags(&c.done[i], cudaEventDisableTiming), "cudaEventCreate(slot)");
    WKV_CUDA(cudaMalloc(&c.err, sizeof(int32_t)), "cudaMalloc(err)");
    WKV_CUDA(cudaMemset(c.err, 0, sizeof(int32_t)), "cudaMemset(err)");
    const size_t max_smem = 227 * 1024;
    WKV_CUDA(prepare_kernels(dev, max_smem), "cudaFuncSetAttribute(tma smem)");
    c.tma_smem_set = max_smem;
    c.ready = true;
  }
  *out = &c;
  return WIND_OK;
}

// ------------------------------------------------------------------------- tuning

std::mutex g_tune_mu;
wind_kv_tuning g_tune[3] = {
    /* INTRA */ {kTma, 1, 49152, 4, 0, 0, 2, 0},  // sweep r01: 0.998 (C2) / 0.985 (C5) of HBM copy
    // PEER: SM stores over NVLink (the path the guide measures at 775 GB/s); 96 CTAs of 512
    // threads keep ~3 MiB of stores in flight (> 2 us x 900 GB/s) and leave SMs to the
    // co-running prefill / decode.  Not yet tuned on a multi-GPU box (one GPU per round-1 call).
    /* PEER  */ {kSimt, 1, 32768, 6, 96, 0, 0, 0},
    // HOST: PCIe-bound.  auto = the TMA kernel on mapped pinned memory (the staged copy-engine
    // path, staged_host_op, is opt-in: kernel 4).
    // max_ctas 0 = per-direction defaults (kHostCtas*): SM stores to host memory beyond
    // what PCIe drains back up into the GPU's memory system — 8 TMA CTAs writing at 52 GB/s
    // slowed a co-running decode kernel by 73 %, 2 CTAs at the same rate by 2 %
    /* HOST  */ {kAuto, 1, 49152, 4, 0, 0, 2, 0},
};

// HOST path defaults when the tuning's max_ctas is 0 (sweep r01: scripts/staged_sweep.py and
// the bench's c3_interference swap rows, profiles/r01/interference_swap_sweep*.json).  What
// matters is the bytes a grid keeps in flight (stages x work-unit bytes per CTA):
//  - SM stores into host memory: ~384 KiB in flight saturates PCIe (52 GB/s) and costs a
//    co-running decode kernel 2 %; 576 KiB 5 %, 768 KiB 7 %, 1.5 MiB 73 % (the writes PCIe
//    cannot drain back up into the GPU's memory system);
//  - SM loads from host memory: 8 CTAs (51 GB/s; fewer lose rate on small chunks);
//  - staged gather / scatter chunks hidden behind PCIe copies: ~768 KiB in flight keeps
//    them ahead of PCIe (56-57 / 55 GB/s) with 4-6 % victim cost (1.5 MiB+: no faster).
constexpr int64_t kHostToHostInFlight = 384 << 10;

// WIND_KV_PDL=0 launches the copy kernels without programmatic dependent launch (A/B).
bool pdl_enabled() {
  static const bool on = [] {
    const char* e = getenv("WIND_KV_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

// WIND_KV_BLOCKED_DEALING=0 turns the small-op contiguous dealing off (A/B measurements).
bool blocked_dealing_enabled() {
  static const bool on = [] {
    const char* e = getenv("WIND_KV_BLOCKED_DEALING");
    return !(e && e[0] == '0');
  }();
  return on;
}
// WIND_KV_FORCE_SYS_SCOPE=1 publishes every op's layer flags at system scope, as a peer
// (NVLink) destination requires: lets one-GPU tests run the peer publication path (the
// fences, the .sys reductions on device-memory flags) with the data on one device.
bool force_sys_scope() {
  static const bool on = [] {
    const char* e = getenv("WIND_KV_FORCE_SYS_SCOPE");
    return e && e[0] == '1';
  }();
  return on;
}

// WIND_KV_FORCE_PEER_ROUTE=1 routes an op between this process's pool and an IMPORTED pool
// of the same physical GPU (another process's pool, as under the N > 1 bench with every
// rank on one GPU) as a PEER op: the PEER tuning and system-scope publication, so one-GPU
// runs exercise the multi-GPU bench's peer-path choices.  Off by default.
bool force_peer_route() {
  static const bool on = [] {
    const char* e = getenv("WIND_KV_FORCE_PEER_ROUTE");
    return e && e[0] == '1';
  }();
  return on;
}

// WIND_KV_BURST_PACING=0: rate-limited device ops pace inside a small resident grid (the
// round-1 pacer) instead of in bursts (A/B measurements).
bool burst_pacing_enabled() {
  static const bool on = [] {
    const char* e = getenv("WIND_KV_BURST_PACING");
    return !(e && e[0] == '0');
  }();
  return on;
}
// A burst-paced op moves this many ns of its rate budget per burst (WIND_KV_BURST_PERIOD_US
// overrides it, for A/B measurements).
double burst_period_ns() {
  static const double ns = [] {
    const char* e = getenv("WIND_KV_BURST_PERIOD_US");
    const double us = e ? atof(e) : 0.0;
    return us >= 10.0 ? us * 1e3 : 2e6;
  }();
  return ns;
}

constexpr int kHostCtasFromHost = 8;
constexpr int64_t kStagedInFlight = 768 << 10;

// Work decomposition and TMA ring of an op copying CP bytes per (layer, kv, block) under a
// tuning (stage_bytes, stages, store_lag).  A chunk larger than a stage is split in `parts`
// equal 16-B-multiple pieces; smaller chunks are grouped `group` per unit (a warp-window of
// table entries).  For the TMA kernel the group is ROUNDED to the nearest count (C4's
// 32 KiB chunks in 48 KiB stages: 2 per unit, not 1 — per-unit overheads bound a CTA, and
// 32 KiB units ran C4 at 0.93 of HBM, 64 KiB units at 0.96) and the ring re-shaped to keep
// stages x stage_bytes bytes in flight (at least 3 stages, within shared memory), the
// store lag the same fraction of the ring.
struct Ring {
  int32_t parts = 1, part_bytes = 0, group = 1;  // decomposition
  int64_t unit = 0;                              // bytes per work unit
  int32_t stages = 0, stage_bytes = 0, lag = 0;  // TMA ring (the tuning's when unchanged)
};

Ring plan_ring(int64_t CP, const wind_kv_tuning& t, bool tma) {
  Ring r;
  r.stages = t.stages;
  r.stage_bytes = t.stage_bytes;
  r.lag = t.store_lag;
  const int64_t SB = t.stage_bytes;
  if (CP >= SB) {
    r.parts = static_cast<int32_t>((CP + SB - 1) / SB);
    r.part_bytes = static_cast<int32_t>((((CP + r.parts - 1) / r.parts) + 15) / 16 * 16);
    r.unit = r.part_bytes;
    return r;
  }
  r.part_bytes = static_cast<int32_t>(CP);
  int64_t g = std::min<int64_t>(kMaxSegs, SB / CP);
  r.group = static_cast<int32_t>(g);
  r.unit = g * CP;
  if (!tma) return r;
  const int64_t budget = static_cast<int64_t>(t.stages) * SB;
  const int64_t g2 = std::min<int64_t>(kMaxSegs, (SB + CP / 2) / CP);  // nearest
  const int64_t u2 = g2 * CP;
  if (u2 == SB) return r;
  const int64_t s2 = std::min<int64_t>(16, std::max<int64_t>(3, budget / u2));
  if (tma_smem_bytes(static_cast<int>(s2), static_cast<int>(u2)) > 227 * 1024) return r;
  r.group = static_cast<int32_t>(g2);
  r.unit = u2;
  r.stages = static_cast<int32_t>(s2);
  r.stage_bytes = static_cast<int32_t>(u2);
  if (t.store_lag > 0)
    r.lag = static_cast<int32_t>(std::min<int64_t>(s2 - 1, std::max<int64_t>(1, (t.store_lag * s2) / t.stages)));
  return r;
}

int ctas_for_in_flight(int64_t target, const Ring& r) {
  const int64_t per_cta = std::max<int64_t>(1, static_cast<int64_t>(r.stages) * r.unit);
  return static_cast<int>(std::max<int64_t>(1, (target + per_cta - 1) / per_cta));
}

int staged_hidden_ctas(int64_t chunk) {  // the staged path's hidden chunks: kStagedInFlight
  const wind_kv_tuning tg = {kTma, 1, 49152, 4, 0, 0, 2, 0};
  return ctas_for_in_flight(kStagedInFlight, plan_ring(chunk, tg, true));
}

}  // namespace

// ---------------------------------------------------------------------------- pool

// Streams of SM partitions (wind_kv_partition_sms, defined at the end of this file): the
// SM count an op on that stream may use, 0 for any other stream.
int32_t partition_sms_of(void* stream);

struct wind_kv_pool {
  wind_kv_pool_desc desc;
  uint8_t* base = nullptr;    // device-accessible data address
  size_t bytes = 0;
  int64_t chunk = 0;          // C
  uint32_t* flags = nullptr;  // layer_done[n_layers], device-accessible
  bool owns_data = false, owns_flags = false, imported = false;
  void* ipc_data_base = nullptr;   // imported: mapping to close
  void* ipc_flags_base = nullptr;
  uint8_t uuid[16] = {};           // physical GPU of the memory (device pools)
  std::atomic<uint32_t> enqueued{0};
  // Host pools: the staged copy-engine path (kernel 4, staged_host_op).  Three device buffers
  // on desc.device that SMs gather into / scatter from at HBM rate while the DMA engines
  // move the other buffer over PCIe, the side stream the DMA runs on, and the events of the
  // two-buffer pipeline.  Allocated at pool creation; dev < 0 if that failed.
  struct Staging {
    int dev = -1;
    uint8_t* buf[kStageBufs] = {};
    size_t buf_bytes = 0;
    int nbufs = 0;                    // buffers in use (kStageBufs; WIND_KV_STAGE_BUFS=2 for A/B)
    int32_t* iota = nullptr;          // 0, 1, ..., iota_n - 1: the staging side's block table
    int32_t iota_n = 0;
    uint32_t* dummy_flags = nullptr;  // layer flags of the internal gather / scatter ops
    cudaStream_t side[2] = {nullptr, nullptr};  // DMA streams (swap out uses both)
    cudaEvent_t fork = nullptr, done = nullptr, ready[kStageBufs] = {}, freed[kStageBufs] = {};
    bool has_done = false;            // `done` marks the end of the last uncaptured staged op
  } stg;
  // Host pools: ops INTO the pool update its layer flags by a plain read-modify-write over
  // PCIe (no PCIe atomics), so two of them must never overlap.  An op enqueued on another
  // stream than the pool's previous op first waits for that op's event (HostOrder in run_op);
  // ops on one stream are ordered anyway.  Not applied under graph capture.
  struct Order {
    std::mutex mu;
    cudaEvent_t ev[kMaxDevices] = {};  // recorded after the last op, on its executing device
    int last_dev = -1;
    unsigned long long last_sid = 0;
  } order;
};

namespace {

int64_t chunk_bytes_of(const wind_kv_pool_desc& d) {
  return static_cast<int64_t>(d.n_kv_heads) * d.block_size * d.head_dim * d.elem_bytes;
}

wind_status check_desc(const wind_kv_pool_desc* d) {
  if (!d) return fail(WIND_ERR_INVALID_ARG, "desc is NULL");
  if (d->n_layers < 1 || d->n_kv_heads < 1 || d->head_dim < 1 || d->block_size < 1 ||
      d->n_blocks < 1 || d->first_layer < 0)
    return fail(WIND_ERR_INVALID_ARG, "pool extents must be >= 1 (first_layer >= 0)");
  if (d->loc != WIND_LOC_DEVICE && d->loc != WIND_LOC_HOST)
    return fail(WIND_ERR_INVALID_ARG, "loc must be WIND_LOC_DEVICE or WIND_LOC_HOST");
  if (d->n_layers > WIND_KV_MAX_LAYERS)
    return fail(WIND_ERR_UNSUPPORTED, "n_layers %d > WIND_KV_MAX_LAYERS", d->n_layers);
  if (d->elem_bytes != 1 && d->elem_bytes != 2 && d->elem_bytes != 4)
    return fail(WIND_ERR_UNSUPPORTED, "elem_bytes must be 1, 2 or 4");
  if (chunk_bytes_of(*d) % 16 != 0)
    return fail(WIND_ERR_UNSUPPORTED, "chunk bytes H*bs*d*e_b = %lld not a multiple of 16",
                static_cast<long long>(chunk_bytes_of(*d)));
  return WIND_OK;
}

constexpr size_t kStagingMin = size_t(32) << 20;  // per buffer: >= 0.5 ms of PCIe Gen5 per chunk
constexpr int32_t kStagingMaxBlocks = 1 << 16;

void staging_free(wind_kv_pool::Staging& g) {
  if (g.dev < 0) return;
  DeviceGuard dg(g.dev);
  for (int b = 0; b < kStageBufs; ++b) {
    if (g.buf[b]) cudaFree(g.buf[b]);
    if (g.ready[b]) cudaEventDestroy(g.ready[b]);
    if (g.freed[b]) cudaEventDestroy(g.freed[b]);
  }
  if (g.iota) cudaFree(g.iota);
  if (g.dummy_flags) cudaFree(g.dummy_flags);
  if (g.fork) cudaEventDestroy(g.fork);
  if (g.done) cudaEventDestroy(g.done);
  for (int b = 0; b < 2; ++b)
    if (g.side[b]) cudaStreamDestroy(g.side[b]);
  cudaGetLastError();
  g = wind_kv_pool::Staging();
}

// Staging of a host pool on device `dev`: 3 buffers of max(32 MiB, 2 * L * C) bytes (so one
// block of every layer always fits), the identity table, dummy flags, a side stream and
// the pipeline events.  Best effort: on failure the pool has no staging and the HOST path
// uses the SM kernels (mapped pinned memory).
void staging_init(wind_kv_pool* p, int dev) {
  wind_kv_pool::Staging& g = p->stg;
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || dev < 0 || dev >= n) {
    cudaGetLastError();
    return;
  }
  DeviceGuard dg(dev);
  g.dev = dev;
  g.buf_bytes = std::max(kStagingMin, static_cast<size_t>(2) * p->desc.n_layers * p->chunk);
  g.iota_n = static_cast<int32_t>(std::min<int64_t>(kStagingMaxBlocks, g.buf_bytes / (2 * p->chunk)));
  std::vector<int32_t> iota(g.iota_n);
  for (int32_t i = 0; i < g.iota_n; ++i) iota[i] = i;
  g.nbufs = kStageBufs;
  if (const char* e = getenv("WIND_KV_STAGE_BUFS")) g.nbufs = std::max(2, std::min(kStageBufs, atoi(e)));
  bool ok = true;
  for (int b = 0; ok && b < g.nbufs; ++b) ok = cudaMalloc(&g.buf[b], g.buf_bytes) == cudaSuccess;
  ok = ok &&
            cudaMalloc(&g.iota, sizeof(int32_t) * g.iota_n) == cudaSuccess &&
            cudaMemcpy(g.iota, iota.data(), sizeof(int32_t) * g.iota_n, cudaMemcpyHostToDevice) == cudaSuccess &&
            cudaMalloc(&g.dummy_flags, sizeof(uint32_t) * WIND_KV_MAX_LAYERS) == cudaSuccess &&
            cudaMemset(g.dummy_flags, 0, sizeof(uint32_t) * WIND_KV_MAX_LAYERS) == cudaSuccess &&
            cudaStreamCreateWithFlags(&g.side[0], cudaStreamNonBlocking) == cudaSuccess &&
            cudaStreamCreateWithFlags(&g.side[1], cudaStreamNonBlocking) == cudaSuccess &&
            cudaEventCreateWithFlags(&g.fork, cudaEventDisableTiming) == cudaSuccess &&
            cudaEventCreateWithFlags(&g.done, cudaEventDisableTiming) == cudaSuccess;
  for (int b = 0; ok && b < kStageBufs; ++b)
    ok = cudaEventCreateWithFlags(&g.ready[b], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&g.freed[b], cudaEventDisableTiming) == cudaSuccess;
  if (!ok) staging_free(g);
  cudaGetLastError();
}

}  // namespace

extern "C" wind_status wind_kv_pool_create(const wind_kv_pool_desc* desc, void* external_base,
                                           wind_kv_pool** out) {
  if (!out) return fail(WIND_ERR_INVALID_ARG, "out is NULL");
  wind_status st = check_desc(desc);
  if (st != WIND_OK) return st;
  if (external_base && (reinterpret_cast<uintptr_t>(external_base) & 15))
    return fail(WIND_ERR_INVALID_ARG, "external_base must be 16-byte aligned");
  auto* p = new wind_kv_pool();
  p->desc = *desc;
  p->chunk = chunk_bytes_of(*desc);
  p->bytes = static_cast<size_t>(desc->n_layers) * 2 * desc->n_blocks * p->chunk;
  const size_t fbytes = sizeof(uint32_t) * desc->n_layers;
  cudaError_t e = cudaSuccess;
  if (desc->loc == WIND_LOC_DEVICE) {
    DevCtx* ctx;
    if ((st = dev_ctx(desc->device, &ctx)) != WIND_OK) { delete p; return st; }
    memcpy(p->uuid, ctx->uuid, 16);
    DeviceGuard g(desc->device);
    if (external_base) {
      cudaPointerAttributes a;
      if (cudaPointerGetAttributes(&a, external_base) != cudaSuccess || a.type != cudaMemoryTypeDevice ||
          a.device != desc->device) {
        cudaGetLastError();
        delete p;
        return fail(WIND_ERR_INVALID_ARG, "external_base is not device memory of device %d", desc->device);
      }
      p->base = static_cast<uint8_t*>(external_base);
    } else {
      e = cudaMalloc(&p->base, p->bytes);
      if (e != cudaSuccess) {
        cudaGetLastError();
        const size_t want = p->bytes;
        delete p;
        return fail(WIND_ERR_OOM, "cudaMalloc(%zu) failed: %s", want, cudaGetErrorString(e));
      }
      p->owns_data = true;
    }
    e = cudaMalloc(&p->flags, fbytes);
    if (e == cudaSuccess) e = cudaMemset(p->flags, 0, fbytes);
  } else {
    if (external_base) {
      void* dptr = nullptr;
      if (cudaHostGetDevicePointer(&dptr, external_base, 0) != cudaSuccess) {
        cudaGetLastError();
        delete p;
        return fail(WIND_ERR_INVALID_ARG, "external_base is not mapped pinned host memory");
      }
      p->base = static_cast<uint8_t*>(dptr);
    } else {
      void* h = nullptr;
      e = cudaHostAlloc(&h, p->bytes, cudaHostAllocMapped | cudaHostAllocPortable);
      if (e != cudaSuccess) {
        cudaGetLastError();
        const size_t want = p->bytes;
        delete p;
        return fail(WIND_ERR_OOM, "cudaHostAlloc(%zu) failed: %s", want, cudaGetErrorString(e));
      }
      void* dptr = nullptr;
      cudaHostGetDevicePointer(&dptr, h, 0);
      p->base = static_cast<uint8_t*>(dptr ? dptr : h);
      p->owns_data = true;
    }
    void* hf = nullptr;
    e = cudaHostAlloc(&hf, fbytes, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e == cudaSuccess) {
      memset(hf, 0, fbytes);
      void* df = nullptr;
      cudaHostGetDevicePointer(&df, hf, 0);
      p->flags = static_cast<uint32_t*>(df ? df : hf);
    }
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    p->owns_flags = false;
    wind_kv_pool_destroy(p);
    return fail(WIND_ERR_OOM, "layer flag allocation failed: %s", cudaGetErrorString(e));
  }
  p->owns_flags = true;
  if (desc->loc == WIND_LOC_HOST && !(desc->flags & WIND_POOL_NO_STAGING)) staging_init(p, desc->device);
  *out = p;
  return WIND_OK;
}

extern "C" wind_status wind_kv_pool_destroy(wind_kv_pool* p) {
  if (!p) return WIND_OK;
  if (p->imported) {
    DeviceGuard g(p->desc.device);
    if (p->ipc_data_base) cudaIpcCloseMemHandle(p->ipc_data_base);
    if (p->ipc_flags_base) cudaIpcCloseMemHandle(p->ipc_flags_base);
  } else if (p->desc.loc == WIND_LOC_DEVICE) {
    DeviceGuard g(p->desc.device);
    if (p->owns_data && p->base) cudaFree(p->base);
    if (p->owns_flags && p->flags) cudaFree(p->flags);
  } else {
    staging_free(p->stg);
    for (cudaEvent_t e : p->order.ev)
      if (e) cudaEventDestroy(e);
    if (p->owns_data && p->base) cudaFreeHost(p->base);
    if (p->owns_flags && p->flags) cudaFreeHost(p->flags);
  }
  cudaGetLastError();
  delete p;
  return WIND_OK;
}

extern "C" wind_status wind_kv_pool_info(const wind_kv_pool* p, void** base, size_t* bytes,
                                         wind_kv_pool_desc* desc) {
  if (!p) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  if (base) *base = p->base;
  if (bytes) *bytes = p->bytes;
  if (desc) *desc = p->desc;
  return WIND_OK;
}

extern "C" wind_status wind_kv_pool_flags(const wind_kv_pool* p, uint32_t** layer_done) {
  if (!p || !layer_done) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  *layer_done = p->flags;
  return WIND_OK;
}

// ----------------------------------------------------------------------------- IPC

namespace {

constexpr char kMagic[8] = {'W', 'I', 'N', 'D', 'K', 'V', '0', '1'};

struct IpcBlob {
  char magic[8];
  int32_t owner_pid;
  int32_t pad;
  wind_kv_pool_desc desc;
  cudaIpcMemHandle_t data;
  uint64_t data_off;
  cudaIpcMemHandle_t flags;
  uint64_t flags_off;
  uint64_t bytes;
  uint8_t uuid[16];
};
static_assert(sizeof(IpcBlob) <= WIND_KV_IPC_HANDLE_BYTES, "IPC blob too large");

wind_status alloc_base(void* p, void** base) {
  static PFN_getAddressRange fn = driver_fn<PFN_getAddressRange>("cuMemGetAddressRange");
  if (!fn) return fail(WIND_ERR_CUDA, "cuMemGetAddressRange entry point unavailable");
  CUdeviceptr b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, reinterpret_cast<CUdeviceptr>(p)) != CUDA_SUCCESS)
    return fail(WIND_ERR_CUDA, "cuMemGetAddressRange failed");
  *base = reinterpret_cast<void*>(b);
  return WIND_OK;
}

}  // namespace

extern "C" wind_status wind_kv_pool_export(const wind_kv_pool* p, wind_kv_ipc_handle* out) {
  if (!p || !out) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  if (p->desc.loc != WIND_LOC_DEVICE || p->imported)
    return fail(WIND_ERR_UNSUPPORTED, "only this process's device pools can be exported");
  DeviceGuard g(p->desc.device);
  IpcBlob b;
  memset(&b, 0, sizeof b);
  memcpy(b.magic, kMagic, 8);
  b.owner_pid = static_cast<int32_t>(getpid());
  b.desc = p->desc;
  b.bytes = p->bytes;
  memcpy(b.uuid, p->uuid, 16);
  void* db = nullptr;
  void* fb = nullptr;
  wind_status st;
  if ((st = alloc_base(p->base, &db)) != WIND_OK) return st;
  if ((st = alloc_base(p->flags, &fb)) != WIND_OK) return st;
  b.data_off = static_cast<uint64_t>(p->base - static_cast<uint8_t*>(db));
  b.flags_off = static_cast<uint64_t>(reinterpret_cast<uint8_t*>(p->flags) - static_cast<uint8_t*>(fb));
  WKV_CUDA(cudaIpcGetMemHandle(&b.data, db), "cudaIpcGetMemHandle(data)");
  WKV_CUDA(cudaIpcGetMemHandle(&b.flags, fb), "cudaIpcGetMemHandle(flags)");
  memset(out, 0, sizeof *out);
  memcpy(out->bytes, &b, sizeof b);
  return WIND_OK;
}

extern "C" wind_status wind_kv_pool_import(const wind_kv_ipc_handle* h, int32_t local_device,
                                           wind_kv_pool** out) {
  if (!h || !out) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  IpcBlob b;
  memcpy(&b, h->bytes, sizeof b);
  if (memcmp(b.magic, kMagic, 8) != 0) return fail(WIND_ERR_INVALID_ARG, "not a wind_kv IPC handle");
  if (b.owner_pid == static_cast<int32_t>(getpid()))
    return fail(WIND_ERR_UNSUPPORTED, "cannot import a pool in the process that exported it");
  DevCtx* ctx;
  wind_status st = dev_ctx(local_device, &ctx);
  if (st != WIND_OK) return st;
  DeviceGuard g(local_device);
  void* db = nullptr;
  void* fb = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&db, b.data, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    if (e == cudaErrorPeerAccessUnsupported || e == cudaErrorInvalidDevice)
      return fail(WIND_ERR_NO_PEER, "cannot map the peer pool on device %d: %s", local_device,
                  cudaGetErrorString(e));
    return cuda_fail(e, "cudaIpcOpenMemHandle(data)");
  }
  e = cudaIpcOpenMemHandle(&fb, b.flags, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    cudaIpcCloseMemHandle(db);
    return cuda_fail(e, "cudaIpcOpenMemHandle(flags)");
  }
  auto* p = new wind_kv_pool();
  p->desc = b.desc;
  p->desc.device = local_device;
  p->chunk = chunk_bytes_of(b.desc);
  p->bytes = b.bytes;
  p->base = static_cast<uint8_t*>(db) + b.data_off;
  p->flags = reinterpret_cast<uint32_t*>(static_cast<uint8_t*>(fb) + b.flags_off);
  p->imported = true;
  p->ipc_data_base = db;
  p->ipc_flags_base = fb;
  memcpy(p->uuid, b.uuid, 16);
  *out = p;
  return WIND_OK;
}

// ------------------------------------------------------------------ op validation

namespace {

bool same_geometry(const wind_kv_pool_desc& a, const wind_kv_pool_desc& b) {
  return a.n_kv_heads == b.n_kv_heads && a.head_dim == b.head_dim &&
         a.block_size == b.block_size && a.elem_bytes == b.elem_bytes;
}

bool layers_inside(const wind_kv_pool_desc& d, int32_t lo, int32_t hi) {
  return lo >= d.first_layer && hi <= d.first_layer + d.n_layers;
}

// Table content checks on host copies, O(n): BLOCK_RANGE > DUP_DST > ALIAS, each over the
// whole table (R4, R5).
wind_status check_tables_host(const wind_kv_pool* src, const int32_t* sbt,
                              const wind_kv_pool* dst, const int32_t* dbt, int32_t n) {
  const int32_t nbs = src->desc.n_blocks, nbd = dst->desc.n_blocks;
  for (int32_t i = 0; i < n; ++i)
    if (static_cast<uint32_t>(sbt[i]) >= static_cast<uint32_t>(nbs) ||
        static_cast<uint32_t>(dbt[i]) >= static_cast<uint32_t>(nbd))
      return fail(WIND_ERR_BLOCK_RANGE, "table entry %d out of range (src %d of %d, dst %d of %d)",
                  i, sbt[i], nbs, dbt[i], nbd);
  std::vector<uint8_t> hit(static_cast<size_t>(nbd), 0);
  for (int32_t i = 0; i < n; ++i) {
    if (hit[dbt[i]]) return fail(WIND_ERR_DUP_DST, "destination slot %d appears twice", dbt[i]);
    hit[dbt[i]] = 1;
  }
  if (src->base == dst->base) {
    // slot b is a source of some entry j and the destination of some entry i != j
    std::vector<int32_t> src_of(static_cast<size_t>(nbs), -1);  // an entry using b as source
    std::vector<uint8_t> multi(static_cast<size_t>(nbs), 0);    // >= 2 entries use it
    for (int32_t j = 0; j < n; ++j) {
      if (src_of[sbt[j]] >= 0) multi[sbt[j]] = 1;
      else src_of[sbt[j]] = j;
    }
    for (int32_t i = 0; i < n; ++i) {
      const int32_t b = dbt[i];
      if (src_of[b] < 0) continue;
      if (multi[b] || src_of[b] != i)
        return fail(WIND_ERR_ALIAS, "same pool: slot %d is written by entry %d and read by another entry", b, i);
    }
  }
  return WIND_OK;
}

// A head sub-range of every block (NEXT-3, TP reshard); n < 0 = whole chunks.
struct HeadRange {
  int32_t src_lo = 0, dst_lo = 0, n = -1;
};

// Argument checks, split by precedence class (S§8(b) "Errors": INVALID_ARG, then GEOMETRY,
// then LAYER_RANGE, then NO_PEER).  INVALID_ARG part of one (src, dst) pair: NULL pools,
// n < 0, NULL tables of a non-empty op, bad head-range arguments.
wind_status check_invalid(const wind_kv_pool* src, const wind_kv_pool* dst, int32_t n,
                          const int32_t* sbt, const int32_t* dbt, const HeadRange& hr = HeadRange()) {
  if (!src || !dst) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  if (n < 0) return fail(WIND_ERR_INVALID_ARG, "n_blocks < 0");
  if (n > 0 && (!sbt || !dbt)) return fail(WIND_ERR_INVALID_ARG, "block table is NULL");
  if (hr.n >= 0 && (hr.n < 1 || hr.src_lo < 0 || hr.dst_lo < 0))
    return fail(WIND_ERR_INVALID_ARG, "head range: n_heads >= 1 and offsets >= 0 required");
  return WIND_OK;
}

// GEOMETRY (and the head-tile UNSUPPORTED of a head range) of one pair.
wind_status check_geometry(const wind_kv_pool* src, const wind_kv_pool* dst,
                           const HeadRange& hr = HeadRange()) {
  if (hr.n < 0) {
    if (!same_geometry(src->desc, dst->desc))
      return fail(WIND_ERR_GEOMETRY, "pools differ in H/d/block_size/elem_bytes");
    return WIND_OK;
  }
  const wind_kv_pool_desc &a = src->desc, &b = dst->desc;
  if (a.head_dim != b.head_dim || a.block_size != b.block_size || a.elem_bytes != b.elem_bytes)
    return fail(WIND_ERR_GEOMETRY, "pools differ in d/block_size/elem_bytes");
  if (hr.src_lo + hr.n > a.n_kv_heads || hr.dst_lo + hr.n > b.n_kv_heads)
    return fail(WIND_ERR_GEOMETRY, "head range leaves a pool (src %d+%d of %d, dst %d+%d of %d)",
                hr.src_lo, hr.n, a.n_kv_heads, hr.dst_lo, hr.n, b.n_kv_heads);
  if ((static_cast<int64_t>(a.block_size) * a.head_dim * a.elem_bytes) % 16 != 0)
    return fail(WIND_ERR_UNSUPPORTED, "head tile bs*d*e_b must be a multiple of 16 bytes");
  return WIND_OK;
}

// LAYER_RANGE of one pair: lo <= hi, and a non-empty [lo, hi) inside both pools.
wind_status check_layers(const wind_kv_pool* src, const wind_kv_pool* dst, int32_t lo, int32_t hi) {
  if (lo > hi) return fail(WIND_ERR_LAYER_RANGE, "layer_lo %d > layer_hi %d", lo, hi);
  if (lo < hi && (!layers_inside(src->desc, lo, hi) || !layers_inside(dst->desc, lo, hi)))
    return fail(WIND_ERR_LAYER_RANGE, "layers [%d, %d) not inside both pools", lo, hi);
  return WIND_OK;
}

// All argument checks of one pair in precedence order (wind_kv_validate; no stream).
wind_status check_args(const wind_kv_pool* src, const wind_kv_pool* dst, int32_t n,
                       const int32_t* sbt, const int32_t* dbt, int32_t lo, int32_t hi,
                       const HeadRange& hr = HeadRange()) {
  wind_status st;
  if ((st = check_invalid(src, dst, n, sbt, dbt, hr)) != WIND_OK) return st;
  if ((st = check_geometry(src, dst, hr)) != WIND_OK) return st;
  return check_layers(src, dst, lo, hi);
}

// The device an op executes on (wind_kv.h, wind_kv_migrate): src's device if src is a
// device pool, else dst's; -1 for host -> host (no executing device: UNSUPPORTED in route).
int exec_device_of(const wind_kv_pool* src, const wind_kv_pool* dst) {
  if (src->desc.loc == WIND_LOC_DEVICE) return src->desc.device;
  if (dst->desc.loc == WIND_LOC_DEVICE) return dst->desc.device;
  return -1;
}

// Both pools are device pools whose data and flags every reader reaches through the
// executing GPU's L2 (same physical GPU), and the op is not forced onto the peer route.
bool local_pair(const wind_kv_pool* a, const wind_kv_pool* b) {
  return a->desc.loc == WIND_LOC_DEVICE && b->desc.loc == WIND_LOC_DEVICE &&
         memcmp(a->uuid, b->uuid, 16) == 0 && !(force_peer_route() && (a->imported || b->imported));
}

// Which device runs the op, and which tuning path applies.
wind_status route(const wind_kv_pool* src, const wind_kv_pool* dst, int* exec, int* path) {
  const bool sd = src->desc.loc == WIND_LOC_DEVICE, dd = dst->desc.loc == WIND_LOC_DEVICE;
  if (!sd && !dd) return fail(WIND_ERR_UNSUPPORTED, "host -> host migration has no executing device");
  *exec = sd ? src->desc.device : dst->desc.device;
  if (!sd || !dd) {
    *path = WIND_PATH_HOST;
    return WIND_OK;
  }
  *path = local_pair(src, dst) ? WIND_PATH_INTRA : WIND_PATH_PEER;
  if (src->imported && dst->imported)
    return fail(WIND_ERR_UNSUPPORTED, "at least one pool must be local to this process");
  // a local pool on another device of this process: enable peer access from the executing one
  const wind_kv_pool* other = (src->desc.device != *exec) ? src : dst;
  if (!other->imported && other->desc.device != *exec) {
    int can = 0;
    cudaDeviceCanAccessPeer(&can, *exec, other->desc.device);
    if (!can) return fail(WIND_ERR_NO_PEER, "device %d cannot access device %d", *exec, other->desc.device);
    DeviceGuard g(*exec);
    cudaError_t e = cudaDeviceEnablePeerAccess(other->desc.device, 0);  // once per pair
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(e, "cudaDeviceEnablePeerAccess");
    cudaGetLastError();
  }
  return WIND_OK;
}

wind_status check_stream(void* stream, int exec) {
  if (!stream) return WIND_OK;  // legacy default stream of the executing device
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(static_cast<cudaStream_t>(stream), &cap) == cudaSuccess &&
      cap != cudaStreamCaptureStatusNone)
    return WIND_OK;  // cudaStreamGetDevice is not permitted while capturing; trust the caller
  cudaGetLastError();
  int sd = -1;
  cudaError_t e = cudaStreamGetDevice(static_cast<cudaStream_t>(stream), &sd);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(WIND_ERR_INVALID_ARG, "invalid stream: %s", cudaGetErrorString(e));
  }
  if (sd != exec) return fail(WIND_ERR_INVALID_ARG, "stream belongs to device %d, op executes on %d", sd, exec);
  return WIND_OK;
}

struct OpItem {
  wind_kv_pool* dst;
  const int32_t* sbt;
  const int32_t* dbt;
  int32_t n;
};

// Debug pools: device-side table check (not on the release hot path; may allocate scratch).
// Runs in the op's stream with the scratch of the op's counter slot.
wind_status debug_check(DevCtx* ctx, int exec, int slot, const wind_kv_pool* src, const OpItem& it,
                        cudaStream_t s) {
  const int32_t need = std::max(src->desc.n_blocks, it.dst->desc.n_blocks);
  if (ctx->scratch_n[slot] < need) {
    DeviceGuard g(exec);
    if (ctx->scratch[slot]) cudaFree(ctx->scratch[slot]);  // synchronises: no launch still uses it
    ctx->scratch[slot] = nullptr;
    ctx->scratch_n[slot] = 0;
    WKV_CUDA(cudaMalloc(&ctx->scratch[slot], sizeof(uint32_t) * 2 * need), "cudaMalloc(debug scratch)");
    ctx->scratch_n[slot] = need;
  }
  WKV_CUDA(launch_table_check(it.sbt, it.dbt, it.n, src->desc.n_blocks, it.dst->desc.n_blocks,
                              src->base == it.dst->base, ctx->scratch[slot], ctx->scratch_n[slot], ctx->err, s),
           "table check launch");
  g_launches += 2;
  return WIND_OK;
}

bool host_readable(const void* ptr) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost || a.type == cudaMemoryTypeUnregistered ||
         a.type == cudaMemoryTypeManaged;
}

// Copy-engine path (tuning kernel = 3): the DMA engines move the bytes, no SM is used, so a
// co-running decode kernel keeps every SM (bench c3_interference).  One cudaMemcpy2DAsync
// per run of adjacent blocks covers all planes (rows = the 2 (hi - lo) planes, row pitch =
// each pool's plane stride).  The tables must be host-readable (the driver needs every
// address at enqueue time); the layer flags are published by one tiny kernel afterwards
// (stream order: after every copy), so per-layer streaming is not available on this path.
// The copy-engine path reads the tables on the CPU: check them before anything is enqueued
// (an entry out of range would make a DMA copy write outside both pools).
wind_status check_ce_tables(int32_t src_nb, const OpItem* items, int n_items) {
  for (int j = 0; j < n_items; ++j) {
    const OpItem& it = items[j];
    if (it.n == 0) continue;
    if (!host_readable(it.sbt) || !host_readable(it.dbt))
      return fail(WIND_ERR_UNSUPPORTED, "copy-engine path needs host-readable block tables");
    for (int32_t i = 0; i < it.n; ++i)
      if (static_cast<uint32_t>(it.sbt[i]) >= static_cast<uint32_t>(src_nb) ||
          static_cast<uint32_t>(it.dbt[i]) >= static_cast<uint32_t>(it.dst->desc.n_blocks))
        return fail(WIND_ERR_BLOCK_RANGE, "item %d: table entry %d out of range (src %d of %d, dst %d of %d)",
                    j, i, it.sbt[i], src_nb, it.dbt[i], it.dst->desc.n_blocks);
  }
  return WIND_OK;
}

// Counter-slot ownership (wind_kv_internal.h kEagerSlots).  An eager op takes the slot its
// stream's previous op used if that slot is still that stream's (stream order keeps the two
// apart), else a slot whose last op has completed (its done event).  No device work: the
// event is recorded after the op's launches (finish_slot).  Nothing is enqueued here;
// release_slot undoes a take when the op fails before launching.
struct Slot {
  int index = -1;
  bool eager = false;     // false: the stream is capturing (graph slot ring)
  bool prev_used = false;
  unsigned long long sid = 0, prev_owner = 0;
};

// The stream's unique id (0 if unavailable) and whether it is capturing.
void stream_identity(cudaStream_t s, unsigned long long* sid, bool* capturing) {
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &cap) != cudaSuccess) {
    cudaGetLastError();
    cap = cudaStreamCaptureStatusNone;
  }
  *capturing = cap != cudaStreamCaptureStatusNone;
  *sid = 0;
  if (!*capturing && cudaStreamGetId(s, sid) != cudaSuccess) {
    cudaGetLastError();
    *sid = 0;
  }
}

// Orders the ops INTO host pools (wind_kv_pool::Order): holds each host destination's lock
// from the wait to the record, so two threads cannot both slip in behind the same op.  A
// host SOURCE pool is only locked (its staging buffers and events, used by the staged path,
// are then enqueued by one thread at a time).
class HostOrder {
 public:
  HostOrder(const wind_kv_pool* src, const OpItem* items, int n_items, cudaStream_t s,
            unsigned long long sid, bool capturing)
      : s_(s), sid_(sid) {
    for (int j = 0; j < n_items; ++j)
      if (!capturing && items[j].dst->desc.loc == WIND_LOC_HOST &&
          std::find(pools_.begin(), pools_.end(), items[j].dst) == pools_.end())
        pools_.push_back(items[j].dst);
    locked_ = pools_;
    wind_kv_pool* hs = const_cast<wind_kv_pool*>(src);
    if (src->desc.loc == WIND_LOC_HOST && std::find(locked_.begin(), locked_.end(), hs) == locked_.end())
      locked_.push_back(hs);
    std::sort(locked_.begin(), locked_.end());  // one lock order for every thread
    for (wind_kv_pool* h : locked_) h->order.mu.lock();
  }
  ~HostOrder() {
    for (wind_kv_pool* h : locked_) h->order.mu.unlock();
  }
  HostOrder(const HostOrder&) = delete;
  HostOrder& operator=(const HostOrder&) = delete;
  // Before the op's first enqueue: wait for the previous op into each pool if it was
  // enqueued on another stream.
  wind_status wait() {
    for (wind_kv_pool* h : pools_) {
      const auto& o = h->order;
      if (o.last_dev >= 0 && (sid_ == 0 || o.last_sid != sid_))
        WKV_CUDA(cudaStreamWaitEvent(s_, o.ev[o.last_dev], 0), "cudaStreamWaitEvent(host pool order)");
    }
    return WIND_OK;
  }
  // After the op's last enqueue (current device = the executing one).
  wind_status commit(int exec) {
    for (wind_kv_pool* h : pools_) {
      auto& o = h->order;
      if (!o.ev[exec])
        WKV_CUDA(cudaEventCreateWithFlags(&o.ev[exec], cudaEventDisableTiming), "cudaEventCreate(host pool order)");
      WKV_CUDA(cudaEventRecord(o.ev[exec], s_), "cudaEventRecord(host pool order)");
      o.last_dev = exec;
      o.last_sid = sid_;
    }
    return WIND_OK;
  }

 private:
  cudaStream_t s_;
  unsigned long long sid_;
  std::vector<wind_kv_pool*> pools_;   // host destinations: ordered
  std::vector<wind_kv_pool*> locked_;  // pools_ plus a host source
};

wind_status take_slot(DevCtx* ctx, int exec, unsigned long long sid, bool capturing, Slot* out) {
  if (capturing) {  // a replay cannot be tracked here: round robin
    out->index = kEagerSlots + static_cast<int>(ctx->graph_seq.fetch_add(1) % kGraphSlots);
    out->eager = false;
    return WIND_OK;
  }
  std::lock_guard<std::mutex> lk(ctx->slot_mu);
  int idx = -1;
  if (sid) {
    auto it = ctx->slot_of_stream.find(sid);
    if (it != ctx->slot_of_stream.end() && ctx->owner[it->second] == sid) idx = it->second;
  }
  for (int probe = 0; idx < 0 && probe < kEagerSlots; ++probe) {
    const int i = (ctx->cursor + probe) % kEagerSlots;
    if (!ctx->used[i]) {
      idx = i;
    } else {
      const cudaError_t q = cudaEventQuery(ctx->done[i]);
      if (q == cudaSuccess) idx = i;
      else if (q != cudaErrorNotReady) cudaGetLastError();
    }
    if (idx >= 0) ctx->cursor = (i + 1) % kEagerSlots;
  }
  if (idx < 0)
    return fail(WIND_ERR_UNSUPPORTED, "ops of %d streams are in flight on device %d (the counter-slot "
                "limit); nothing enqueued", kEagerSlots, exec);
  out->index = idx;
  out->eager = true;
  out->sid = sid;
  out->prev_used = ctx->used[idx];
  out->prev_owner = ctx->owner[idx];
  if (ctx->owner[idx] && ctx->owner[idx] != sid) ctx->slot_of_stream.erase(ctx->owner[idx]);
  ctx->used[idx] = true;
  ctx->owner[idx] = sid;
  if (sid) ctx->slot_of_stream[sid] = idx;
  return WIND_OK;
}

// After the op's last launch: its slot is busy until the stream gets past this point.
wind_status finish_slot(DevCtx* ctx, const Slot& sl, cudaStream_t s) {
  if (!sl.eager) return WIND_OK;
  WKV_CUDA(cudaEventRecord(ctx->done[sl.index], s), "cudaEventRecord(slot)");
  return WIND_OK;
}

void release_slot(DevCtx* ctx, const Slot& sl) {
  if (!sl.eager) return;
  std::lock_guard<std::mutex> lk(ctx->slot_mu);
  if (ctx->owner[sl.index] != sl.sid) return;
  if (sl.sid && sl.sid != sl.prev_owner) ctx->slot_of_stream.erase(sl.sid);
  ctx->used[sl.index] = sl.prev_used;
  ctx->owner[sl.index] = sl.prev_owner;
  if (sl.prev_owner) ctx->slot_of_stream[sl.prev_owner] = sl.index;
}

wind_status copy_engine_op(const Params& p, int32_t src_nb, const OpItem* items, int n_items,
                           cudaStream_t s, int32_t rate_mbps) {
  const size_t rows = static_cast<size_t>(2) * p.n_layers;
  // rate limit: a pace kernel stamps the op start; after copies worth >= 20 us of the
  // budget, a pace kernel holds the stream until start + bytes_so_far / rate.  The stamp
  // lives in this op's (otherwise unused) arrival-counter slot.
  unsigned long long* t0 = reinterpret_cast<unsigned long long*>(p.counters + WIND_KV_MAX_LAYERS - 2);
  double sched_ns = 0, last_paced = 0;
  int launches = 0;
  (void)src_nb;  // the tables were range-checked by check_ce_tables before the slot was taken
  if (rate_mbps > 0) {
    WKV_CUDA(launch_pace(t0, 0, 1, s), "pace kernel launch");
    ++launches;
  }
  for (int j = 0; j < n_items; ++j) {
    const OpItem& it = items[j];
    if (it.n == 0) continue;
    const Item& q = p.items[j];
    const bool co = q.coalesce != 0;
    for (int32_t i = 0; i < it.n;) {
      int32_t k = 1;
      while (co && i + k < it.n && it.sbt[i + k] == it.sbt[i] + k && it.dbt[i + k] == it.dbt[i] + k) ++k;
      const uint8_t* sp = p.src_plane0 + static_cast<int64_t>(it.sbt[i]) * p.s_chunk;
      uint8_t* dp = q.dst_plane0 + static_cast<int64_t>(it.dbt[i]) * q.d_chunk;
      WKV_CUDA(cudaMemcpy2DAsync(dp, static_cast<size_t>(q.d_plane_stride), sp,
                                 static_cast<size_t>(p.s_plane_stride), static_cast<size_t>(p.copy) * k, rows,
                                 cudaMemcpyDefault, s),
               "cudaMemcpy2DAsync");
      if (rate_mbps > 0) {
        sched_ns += static_cast<double>(p.copy) * k * rows * 1e3 / rate_mbps;
        if (sched_ns - last_paced >= 20000) {
          WKV_CUDA(launch_pace(t0, static_cast<uint64_t>(sched_ns), 0, s), "pace kernel launch");
          last_paced = sched_ns;
          ++launches;
        }
      }
      i += k;
    }
  }
  if (rate_mbps > 0 && sched_ns > last_paced) {
    WKV_CUDA(launch_pace(t0, static_cast<uint64_t>(sched_ns), 0, s), "pace kernel launch");
    ++launches;
  }
  WKV_CUDA(launch_flag_bump(p, s), "flag kernel launch");
  g_launches += 1 + launches;
  return WIND_OK;
}

// Step-aligned pacing (wind_kv_migrate_stepped): slice k of the op waits until
// *counter >= first + k, the consumer's decode loop bumping the counter at each step start.
struct StepPacing {
  const uint32_t* counter;
  uint32_t first;
  uint64_t bytes_per_step;
};

wind_status run_op(const wind_kv_pool* src, const OpItem* items, int n_items, int32_t lo,
                   int32_t hi, void* stream, const HeadRange& hr, const wind_kv_tuning* override_tuning,
                   const StepPacing* step);

// Staged copy-engine host path (kernel 4, opt-in: the host-side block table is read on the
// CPU at enqueue, unlike every other op's tables).  PCIe is the bottleneck of a swap, and the DMA
// engines drive it harder than SM stores to mapped memory (full-size write packets: 57 vs
// 52 GB/s D2H on B200, profiles/r01/host_sweep.txt) while holding no SM; but a DMA engine
// needs every address at enqueue time and pays a setup per copy, so it cannot follow a
// shuffled device block table.  The op is therefore split by where each side's
// fragmentation lives:
//   device side (any table, device-resident): a TMA gather (swap out) / scatter (swap in)
//     kernel between the device pool and a contiguous staging buffer at HBM rate;
//   host side (table read on the CPU at enqueue): one cudaMemcpy2DAsync per run of adjacent
//     host slots, rows = the chunk's K/V planes, on side streams (a swap-out alternates its
//     chunks over two: two D2H copies in flight drive PCIe harder than one).
// Chunks are layer-major (A5): a chunk is a range of whole layers for all n blocks
// when they fit the buffer, else one layer for a range of blocks.  They alternate between
// three buffers, so gathers run up to two chunks ahead of the PCIe copies (fork / join
// with events: graph-capturable).  dst's layer flags are published as each layer's last
// chunk lands (after its PCIe copy on a side stream for a swap out, after its scatter on
// the op's stream for a swap in), so a consumer can start on layer 0 of a swap-in while
// later layers are still in flight.
wind_status staged_host_op(const wind_kv_pool* src, const OpItem& it, int32_t lo, int32_t hi,
                           cudaStream_t s, int32_t hidden_ctas) {
  const bool out = src->desc.loc == WIND_LOC_DEVICE;  // swap out: device -> host
  const wind_kv_pool* dev = out ? src : it.dst;
  const wind_kv_pool* host = out ? it.dst : src;
  wind_kv_pool::Staging& g = const_cast<wind_kv_pool*>(host)->stg;
  const int32_t* hbt = out ? it.dbt : it.sbt;       // read here, on the CPU
  const int32_t* dev_bt = out ? it.sbt : it.dbt;    // read by the gather / scatter kernel
  const int64_t C = dev->chunk;
  const int64_t layer_bytes = 2 * C * static_cast<int64_t>(it.n);  // one layer, all blocks
  // chunk shape: whole layers x all blocks when one layer fits, else 1 layer x m blocks
  int32_t lpc = 1, m = it.n;
  if (it.n <= g.iota_n && layer_bytes <= static_cast<int64_t>(g.buf_bytes)) {
    lpc = static_cast<int32_t>(std::min<int64_t>(hi - lo, static_cast<int64_t>(g.buf_bytes) / layer_bytes));
  } else {
    m = static_cast<int32_t>(std::min<int64_t>(g.iota_n, static_cast<int64_t>(g.buf_bytes) / (2 * C)));
    if (m < 1) return fail(WIND_ERR_UNSUPPORTED, "staging buffer smaller than one block of one layer");
  }
  for (int32_t i = 0; i < it.n; ++i)  // host-side range (the device side is the kernel's contract)
    if (hbt[i] < 0 || hbt[i] >= host->desc.n_blocks)
      return fail(WIND_ERR_BLOCK_RANGE, "host block table entry %d = %d out of [0, %d)", i, hbt[i],
                  host->desc.n_blocks);
  // the staging buffer seen as a device pool of m blocks over a chunk's layers, and a shadow
  // of the device pool: both publish into dummy flags (dst's real flags: flag_range below)
  wind_kv_pool stage;
  stage.desc = dev->desc;
  stage.desc.n_blocks = m;
  stage.desc.flags = 0;
  stage.chunk = C;
  stage.flags = g.dummy_flags;
  memcpy(stage.uuid, dev->uuid, 16);
  wind_kv_pool shadow;
  shadow.desc = dev->desc;
  shadow.desc.flags = 0;
  shadow.base = dev->base;
  shadow.chunk = C;
  shadow.bytes = dev->bytes;
  shadow.flags = g.dummy_flags;
  memcpy(shadow.uuid, dev->uuid, 16);
  // gather / scatter: the intra-device TMA kernel.  The one chunk whose gather (swap out:
  // the first) or scatter (swap in: the last) is not hidden behind a PCIe copy runs on every
  // SM (~10 us per 32 MiB); the hidden ones on `hidden_ctas` CTAs so they take few SMs and
  // little HBM burst from co-running work.
  const wind_kv_tuning t_exposed = {kTma, 1, 49152, 4, 0, 0, 2, 0};
  const wind_kv_tuning t_hidden = {kTma, 1, 49152, 4, std::max(1, hidden_ctas), 0, 2, 0};
  const int64_t hpitch = static_cast<int64_t>(host->desc.n_blocks) * C;
  const int64_t spitch = static_cast<int64_t>(m) * C;
  // +1 on dst's layer_done flags [a, b) (global ids), system scope, on stream `st`
  auto flag_range = [&](int32_t a, int32_t b, cudaStream_t st) -> wind_status {
    if (a >= b) return WIND_OK;
    Params fp;
    memset(&fp, 0, sizeof fp);
    fp.n_items = 1;
    fp.items[0].flags = it.dst->flags + (a - it.dst->desc.first_layer);
    fp.items[0].d_layers = b - a;
    fp.items[0].host_flags = it.dst->desc.loc == WIND_LOC_HOST;
    fp.items[0].sys_scope = 1;
    fp.sys_scope = 1;
    WKV_CUDA(launch_flag_bump(fp, st), "flag kernel launch");
    g_launches += 1;
    return WIND_OK;
  };
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &cap) != cudaSuccess) {
    cudaGetLastError();
    cap = cudaStreamCaptureStatusNone;
  }
  const bool capturing = cap != cudaStreamCaptureStatusNone;
  // staged ops on one host pool share its buffers: order after the previous one (outside
  // a graph capture; inside one, the graph's own order applies)
  if (!capturing && g.has_done) WKV_CUDA(cudaStreamWaitEvent(s, g.done, 0), "cudaStreamWaitEvent(done)");
  wind_status st;
  // dst layers outside [lo, hi): +1 at the start, as every op does (wind_kv_migrate)
  const int32_t f0 = it.dst->desc.first_layer, f1 = f0 + it.dst->desc.n_layers;
  if ((st = flag_range(f0, lo, s)) != WIND_OK) return st;
  if ((st = flag_range(hi, f1, s)) != WIND_OK) return st;
  const int32_t bchunks = (it.n + m - 1) / m;  // block chunks per layer group
  const int32_t lgroups = (hi - lo + lpc - 1) / lpc;
  const int32_t K = lgroups * bchunks;
  // DMA streams: a swap-out alternates chunks over two (two device-to-host copies in flight
  // drive PCIe ~3.5 % harder than one: 55.9 vs 54.0 GB/s, round-1 probe);
  // host-to-device gains nothing from a second stream, so a swap-in uses one
  const int nside = (out && K >= 2) ? 2 : 1;
  WKV_CUDA(cudaEventRecord(g.fork, s), "cudaEventRecord(fork)");
  for (int q = 0; q < nside; ++q)
    WKV_CUDA(cudaStreamWaitEvent(g.side[q], g.fork, 0), "cudaStreamWaitEvent(fork)");
  // one chunk's PCIe copies: runs of adjacent host slots among entries [i0, i0 + mk),
  // layers [la, lb), on DMA stream `ds`
  auto dma = [&](int32_t la, int32_t lb, int32_t i0, int32_t mk, uint8_t* buf, cudaStream_t ds) -> wind_status {
    uint8_t* hplane0 = host->base + static_cast<int64_t>(la - host->desc.first_layer) * 2 * hpitch;
    const size_t rows = static_cast<size_t>(2) * (lb - la);
    for (int32_t j = i0; j < i0 + mk;) {
      int32_t r = 1;
      while (j + r < i0 + mk && hbt[j + r] == hbt[j] + r) ++r;
      uint8_t* hp = hplane0 + static_cast<int64_t>(hbt[j]) * C;
      uint8_t* sp = buf + static_cast<int64_t>(j - i0) * C;
      WKV_CUDA(out ? cudaMemcpy2DAsync(hp, hpitch, sp, spitch, static_cast<size_t>(r * C), rows,
                                       cudaMemcpyDeviceToHost, ds)
                   : cudaMemcpy2DAsync(sp, spitch, hp, hpitch, static_cast<size_t>(r * C), rows,
                                       cudaMemcpyHostToDevice, ds),
               "cudaMemcpy2DAsync(staged)");
      j += r;
    }
    return WIND_OK;
  };
  for (int32_t k = 0; k < K; ++k) {
    const int32_t la = lo + (k / bchunks) * lpc, lb = std::min(hi, la + lpc);
    const int32_t i0 = (k % bchunks) * m, mk = std::min(m, it.n - i0), b = k % g.nbufs;
    const bool layers_done = k % bchunks == bchunks - 1;  // last block chunk of [la, lb)
    stage.base = g.buf[b];
    stage.desc.first_layer = la;
    stage.desc.n_layers = lb - la;
    stage.bytes = static_cast<size_t>(2 * (lb - la) * spitch);
    if (out) {
      if (k >= g.nbufs) WKV_CUDA(cudaStreamWaitEvent(s, g.freed[b], 0), "cudaStreamWaitEvent(freed)");
      OpItem gi{&stage, dev_bt + i0, g.iota, mk};
      if ((st = run_op(dev, &gi, 1, la, lb, s, HeadRange(), k == 0 ? &t_exposed : &t_hidden, nullptr)) != WIND_OK)
        return st;
      cudaStream_t ds = g.side[k % nside];
      WKV_CUDA(cudaEventRecord(g.ready[b], s), "cudaEventRecord(ready)");
      WKV_CUDA(cudaStreamWaitEvent(ds, g.ready[b], 0), "cudaStreamWaitEvent(ready)");
      if ((st = dma(la, lb, i0, mk, g.buf[b], ds)) != WIND_OK) return st;
      if (layers_done) {
        // the layers' earlier chunks may have gone over the other DMA stream
        if (nside == 2 && k >= 1)
          WKV_CUDA(cudaStreamWaitEvent(ds, g.freed[(k - 1) % g.nbufs], 0), "cudaStreamWaitEvent(other)");
        if ((st = flag_range(la, lb, ds)) != WIND_OK) return st;
      }
      WKV_CUDA(cudaEventRecord(g.freed[b], ds), "cudaEventRecord(freed)");
    } else {
      if (k >= g.nbufs) WKV_CUDA(cudaStreamWaitEvent(g.side[0], g.freed[b], 0), "cudaStreamWaitEvent(freed)");
      if ((st = dma(la, lb, i0, mk, g.buf[b], g.side[0])) != WIND_OK) return st;
      WKV_CUDA(cudaEventRecord(g.ready[b], g.side[0]), "cudaEventRecord(ready)");
      WKV_CUDA(cudaStreamWaitEvent(s, g.ready[b], 0), "cudaStreamWaitEvent(ready)");
      OpItem si{&shadow, g.iota, dev_bt + i0, mk};
      if ((st = run_op(&stage, &si, 1, la, lb, s, HeadRange(), k == K - 1 ? &t_exposed : &t_hidden, nullptr)) != WIND_OK)
        return st;
      if (layers_done && (st = flag_range(la, lb, s)) != WIND_OK) return st;
      WKV_CUDA(cudaEventRecord(g.freed[b], s), "cudaEventRecord(freed)");
    }
  }
  if (out)  // join: each DMA stream's last copy and flags (each runs its work in order)
    for (int q = 0; q < nside; ++q)
      WKV_CUDA(cudaStreamWaitEvent(s, g.freed[(K - 1 - q) % g.nbufs], 0), "cudaStreamWaitEvent(join)");
  if (!capturing) {
    WKV_CUDA(cudaEventRecord(g.done, s), "cudaEventRecord(done)");
    g.has_done = true;
  }
  it.dst->enqueued.fetch_add(1);
  return WIND_OK;
}

// The common op: src -> items[] over layers [lo, hi) on `stream`.
wind_status run_op(const wind_kv_pool* src, const OpItem* items, int n_items, int32_t lo,
                   int32_t hi, void* stream, const HeadRange& hr = HeadRange(),
                   const wind_kv_tuning* override_tuning = nullptr, const StepPacing* step = nullptr);
wind_status run_op(const wind_kv_pool* src, const OpItem* items, int n_items, int32_t lo,
                   int32_t hi, void* stream, const HeadRange& hr,
                   const wind_kv_tuning* override_tuning, const StepPacing* step) {
  if (!src) return fail(WIND_ERR_INVALID_ARG, "src pool is NULL");
  if (n_items < 1 || n_items > WIND_KV_MAX_BATCH) return fail(WIND_ERR_INVALID_ARG, "n_items out of range");
  struct NvtxRange {  // one NVTX range per op (the enqueue, on the host timeline)
    NvtxRange() { nvtxRangePushA("wind_kv op"); }
    ~NvtxRange() { nvtxRangePop(); }
  } nvtx_range;
  int exec = -1, path = 0;
  wind_status st;
  // (1) INVALID_ARG, every item: NULL pools / tables, n < 0, head-range arguments, repeated
  // batch destinations, items on different executing devices, an imported pool mapped for
  // another device, the stream's device (S§8(b) "Errors" precedence)
  for (int j = 0; j < n_items; ++j) {
    const OpItem& it = items[j];
    if ((st = check_invalid(src, it.dst, it.n, it.sbt, it.dbt, hr)) != WIND_OK) return st;
    for (int k = 0; k < j; ++k)
      if (items[k].dst == it.dst) return fail(WIND_ERR_INVALID_ARG, "batch destinations must be distinct");
    const int e2 = exec_device_of(src, it.dst);
    if (j == 0) exec = e2;
    else if (e2 != exec) return fail(WIND_ERR_INVALID_ARG, "batch items execute on different devices");
    // an imported pool is mapped for the device it was imported into: the op must run there
    const wind_kv_pool* imp = src->imported ? src : (it.dst->imported ? it.dst : nullptr);
    if (imp && exec >= 0 && imp->desc.device != exec)
      return fail(WIND_ERR_INVALID_ARG, "imported pool is mapped for device %d but the op executes on %d",
                  imp->desc.device, exec);
  }
  if (exec >= 0 && (st = check_stream(stream, exec)) != WIND_OK) return st;
  // (2) GEOMETRY, then (3) LAYER_RANGE, over every item
  for (int j = 0; j < n_items; ++j)
    if ((st = check_geometry(src, items[j].dst, hr)) != WIND_OK) return st;
  for (int j = 0; j < n_items; ++j)
    if ((st = check_layers(src, items[j].dst, lo, hi)) != WIND_OK) return st;
  // (4) reachability: NO_PEER (enables peer access as a side effect), UNSUPPORTED pairings
  for (int j = 0; j < n_items; ++j) {
    int e2 = -1, p2 = 0;
    if ((st = route(src, items[j].dst, &e2, &p2)) != WIND_OK) return st;
    path = j == 0 ? p2 : std::max(path, p2);
  }
  int64_t total_n = 0;
  for (int j = 0; j < n_items; ++j) total_n += items[j].n;
  if (lo == hi || total_n == 0) return WIND_OK;  // R19: successful no-op, no ticket

  DevCtx* ctx;
  if ((st = dev_ctx(exec, &ctx)) != WIND_OK) return st;
  wind_kv_tuning t;
  if (override_tuning) {
    t = *override_tuning;  // validated by wind_kv_migrate_ex
  } else {
    std::lock_guard<std::mutex> lk(g_tune_mu);
    t = g_tune[path];
  }
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  DeviceGuard g(exec);
  unsigned long long sid = 0;
  bool capturing = false;
  stream_identity(s, &sid, &capturing);
  HostOrder order(src, items, n_items, s, sid, capturing);  // ops into host pools never overlap

  if (step) {  // step-aligned slices: device pools (INTRA / PEER), SM kernels, no debug pools
    bool dbg = false;
    for (int j = 0; j < n_items; ++j) dbg = dbg || ((src->desc.flags | items[j].dst->desc.flags) & WIND_POOL_DEBUG);
    if (path == WIND_PATH_HOST || dbg || t.kernel == kCopyEngine || t.kernel == kStaged)
      return fail(WIND_ERR_UNSUPPORTED, "step-aligned ops need device pools, an SM kernel and no debug pool");
  }
  bool debug = false;  // the device-side table check is enqueued once the op's slot is taken
  for (int j = 0; j < n_items; ++j)
    debug = debug || (items[j].n > 0 && ((src->desc.flags | items[j].dst->desc.flags) & WIND_POOL_DEBUG));

  // HOST path: the staged copy-engine path only when the caller asks for it (kernel 4, via
  // wind_kv_set_tuning or a per-op wind_kv_migrate_ex override).  It reads the host-side
  // table on the CPU at enqueue, which is a different contract from every other op's
  // (tables borrowed and read when the op executes), so it is never chosen automatically:
  // kernel 0 on the HOST path is the TMA kernel over mapped pinned memory.
  if (path == WIND_PATH_HOST && t.kernel == kStaged) {
    const wind_kv_pool* host = src->desc.loc == WIND_LOC_HOST ? src : items[0].dst;
    const int32_t* hbt = host == src ? items[0].sbt : items[0].dbt;
    const bool staged = n_items == 1 && hr.n < 0 && !debug && host->stg.dev == exec &&
                        t.rate_mbps == 0 && host_readable(hbt);
    if (!staged)
      return fail(WIND_ERR_UNSUPPORTED, "staged path needs one item, whole chunks, no rate limit, a "
                  "host-readable host table and host-pool staging on device %d", exec);
    if ((st = order.wait()) != WIND_OK) return st;
    // hidden chunks run the staged kernel tuning (4 x 48 KiB stages)
    st = staged_host_op(src, items[0], lo, hi, s, t.max_ctas > 0 ? t.max_ctas : staged_hidden_ctas(src->chunk));
    return st == WIND_OK ? order.commit(exec) : st;
  }
  const int kernel = t.kernel == kAuto ? (path == WIND_PATH_PEER ? kSimt : kTma) : t.kernel;
  if (kernel == kStaged)
    return fail(WIND_ERR_UNSUPPORTED, "kernel 4 (staged copy engines) moves host pools only");
  // Read-once fan-out (backups; NEXT-3): when every item of a batch walks the SAME
  // source table (same pointer and length), the TMA kernel stages each source unit once and
  // stores it to every destination — (1 + k) x payload of DRAM traffic instead of 2k x.
  // Stores then outnumber loads k : 1, so unless the caller passed a per-op tuning the ring
  // keeps more stores in flight (sweep r01, k = 2 / 3: 0.957 / 0.905 -> 0.963 / 0.941 of HBM).
  int fan = 1;
  if (kernel == kTma && n_items > 1 && n_items <= kMaxFan && items[0].n > 0) {
    bool same = true;
    for (int j = 1; j < n_items; ++j)
      same = same && items[j].sbt == items[0].sbt && items[j].n == items[0].n;
    if (same) fan = n_items;
  }
  if (fan > 1 && !override_tuning) {
    t.stage_bytes = 32768;
    t.stages = 6;
    t.store_lag = 4;
  }

  Params p;
  memset(&p, 0, sizeof p);
  const int64_t CS = src->chunk;
  const int64_t tile = static_cast<int64_t>(src->desc.block_size) * src->desc.head_dim * src->desc.elem_bytes;
  const int64_t CP = hr.n < 0 ? CS : hr.n * tile;  // bytes copied per (layer, kv, block)
  const Ring ring = plan_ring(CP, t, kernel == kTma);
  p.s_chunk = CS;
  p.copy = CP;
  p.parts = ring.parts;
  p.part_bytes = ring.part_bytes;
  p.group = ring.group;
  p.layer_lo = lo;
  p.n_layers = hi - lo;
  p.src_plane0 = src->base + static_cast<int64_t>(lo - src->desc.first_layer) * 2 * src->desc.n_blocks * CS +
                 (hr.n < 0 ? 0 : hr.src_lo * tile);
  p.s_plane_stride = static_cast<int64_t>(src->desc.n_blocks) * CS;
  p.evict_first = t.evict_first;
  p.store_lag = ring.lag;
  p.stages = ring.stages;
  p.stage_bytes = ring.stage_bytes;
  int32_t base_units = 0;
  int ni = 0;
  for (int j = 0; j < n_items; ++j) {
    const OpItem& it = items[j];  // n == 0 items stay: they take a ticket, bump flags
    const wind_kv_pool* d = it.dst;
    Item& q = p.items[ni++];
    q.sbt = it.sbt;
    q.dbt = it.dbt;
    q.n = it.n;
    const int64_t CD = d->chunk;
    q.dst_plane0 = d->base + static_cast<int64_t>(lo - d->desc.first_layer) * 2 * d->desc.n_blocks * CD +
                   (hr.n < 0 ? 0 : hr.dst_lo * tile);
    q.d_plane_stride = static_cast<int64_t>(d->desc.n_blocks) * CD;
    q.d_chunk = CD;
    q.coalesce = (CP == CS && CP == CD) ? 1 : 0;
    q.flags = d->flags;
    q.d_flag_lo = lo - d->desc.first_layer;
    q.d_layers = d->desc.n_layers;
    q.host_flags = d->desc.loc == WIND_LOC_HOST;
    // GPU-scope publication only when both pools live on the executing GPU (same physical
    // device: every reader of the data and of the flags goes through this GPU's L2)
    q.sys_scope = force_sys_scope() || !local_pair(src, d);
    p.sys_scope |= q.sys_scope;
    const int64_t u = p.parts > 1 ? static_cast<int64_t>(it.n) * p.parts
                                  : (static_cast<int64_t>(it.n) + p.group - 1) / p.group;
    if (u + base_units > INT32_MAX) return fail(WIND_ERR_UNSUPPORTED, "too many work units");
    q.units = static_cast<int32_t>(u);
    q.unit_base = base_units;
    base_units += q.units;
  }
  p.n_items = ni;
  p.units_per_plane = base_units;
  p.total_units = static_cast<int64_t>(2) * p.n_layers * base_units;
  if (kernel == kCopyEngine && (st = check_ce_tables(src->desc.n_blocks, items, n_items)) != WIND_OK) return st;
  // the op's counter slot: the last step that may fail without enqueuing anything
  Slot sl;
  if ((st = take_slot(ctx, exec, sid, capturing, &sl)) != WIND_OK) return st;
  if ((st = order.wait()) != WIND_OK) {
    release_slot(ctx, sl);
    return st;
  }
  const int slot = sl.index;
  p.counters = ctx->counters + static_cast<size_t>(slot) * WIND_KV_MAX_LAYERS;
  p.abort_word = debug ? ctx->err : nullptr;
  if (debug)
    for (int j = 0; j < n_items; ++j)
      if (items[j].n > 0 && ((src->desc.flags | items[j].dst->desc.flags) & WIND_POOL_DEBUG))
        if ((st = debug_check(ctx, exec, slot, src, items[j], s)) != WIND_OK) {
          release_slot(ctx, sl);
          return st;
        }

  p.fan = fan;
  if (fan > 1) {  // every item walks items[0]'s units
    for (int j = 1; j < n_items; ++j) {
      p.items[0].coalesce &= p.items[j].coalesce;
      p.items[j].unit_base = 0;
    }
    p.units_per_plane = p.items[0].units;
    p.total_units = static_cast<int64_t>(2) * p.n_layers * p.units_per_plane;
  }
  if (kernel == kCopyEngine) {
    st = copy_engine_op(p, src->desc.n_blocks, items, n_items, s, t.rate_mbps);
    const wind_status fs = finish_slot(ctx, sl, s);  // whatever was enqueued holds the slot
    const wind_status os = order.commit(exec);
    if (st != WIND_OK) return st;
    if (fs != WIND_OK) return fs;
    if (os != WIND_OK) return os;
    for (int j = 0; j < n_items; ++j) items[j].dst->enqueued.fetch_add(1);
    return WIND_OK;
  }
  // a stream of an SM partition (wind_kv_partition_sms) only has that partition's SMs
  const int32_t part_sms = partition_sms_of(stream);
  int64_t grid = static_cast<int64_t>(part_sms > 0 ? part_sms : ctx->sms) * std::max(1, t.ctas_per_sm);
  if (t.max_ctas > 0)
    grid = std::min<int64_t>(grid, t.max_ctas);
  else if (path == WIND_PATH_HOST) {
    bool to_host = false;  // any store into host memory: the backpressure-prone direction
    for (int j = 0; j < n_items; ++j) to_host = to_host || items[j].dst->desc.loc == WIND_LOC_HOST;
    grid = std::min<int64_t>(grid, to_host ? ctas_for_in_flight(kHostToHostInFlight, ring) : kHostCtasFromHost);
  }
  // Rate limits.  Device ops (INTRA / PEER) with no CTA cap are BURST-paced: the op is cut
  // into slices of its units, each slice moved by half the grid at full rate and followed
  // by a 1-thread pace kernel that holds the stream until the rate schedule allows the next
  // one (2 ms of rate budget per slice).  Between bursts no copy CTA is resident, so a
  // co-running decode step keeps its SMs: at 150 GB/s a paced grid of sleeping CTAs (the
  // round-1 pacer, still used when max_ctas > 0 or on the HOST path) cost a decode step of
  // GEMMs + attention 19-29 %, the burst pacer ~7.5 %, and slices released on the
  // consumer's own steps (wind_kv_migrate_stepped, `step`, same code) ~4.5 %.
  const bool burst_paced = t.rate_mbps > 0 && t.max_ctas == 0 && path != WIND_PATH_HOST && !debug &&
                           burst_pacing_enabled();
  // in-kernel pacing: as few SMs as can sustain the rate (one CTA moves ~38 GB/s of payload
  // intra-device)
  if (t.rate_mbps > 0 && t.max_ctas == 0 && !burst_paced)
    grid = std::min<int64_t>(grid, std::max<int64_t>(1, (t.rate_mbps + kCtaMBps - 1) / kCtaMBps));
  grid = std::max<int64_t>(1, std::min<int64_t>(grid, p.total_units));
  // Work dealing.  Grid-stride (all CTAs sweep the layers together: each layer completes
  // early, A5 streaming) unless a plane has fewer units than the grid: then every CTA
  // would cross a layer boundary at almost every unit, and each crossing waits for its
  // older stores to be fully written before the arrival — a latency chain that dominates
  // small ops.  Those get contiguous unit ranges per CTA (a handful of crossings each).
  p.blocked = (p.units_per_plane < grid && t.rate_mbps == 0 && blocked_dealing_enabled()) ? 1 : 0;
  p.unit_lo = 0;
  p.unit_hi = p.total_units;
  p.first_slice = 1;
  if (burst_paced || step) {
    // source payload of the op (a fan-out reads each unit once)
    int64_t n_src = 0;
    for (int j = 0; j < (fan > 1 ? 1 : n_items); ++j) n_src += items[j].n;
    const double payload = 2.0 * p.n_layers * static_cast<double>(CP) * static_cast<double>(n_src);
    const double slice_bytes = step ? static_cast<double>(step->bytes_per_step)
                                    : t.rate_mbps * 1e6 * burst_period_ns() * 1e-9;
    int64_t slice_units = static_cast<int64_t>(p.total_units * slice_bytes / std::max(1.0, payload));
    // a burst runs on half the grid: nearly the full HBM rate (one CTA moves ~38 GB/s), and
    // half the SMs stay with the co-running work (sweep, profiles/r02/burst_pacer/: 74 CTAs
    // beat 148 / 37 / 16 next to both victims); WIND_KV_BURST_CTAS overrides it (A/B)
    grid = std::max<int64_t>(1, grid / 2);
    if (const char* e = getenv("WIND_KV_BURST_CTAS"))
      grid = std::max<int64_t>(1, atoi(e) > 0 ? atoi(e) : grid);
    grid = std::min<int64_t>(grid, p.total_units);
    slice_units = std::max<int64_t>(slice_units, grid);  // a burst keeps the whole grid busy
    unsigned long long* t0 = ctx->stamps + slot;
    p.ns_per_byte = 0.f;

    static PFN_waitValue32 wait_fn = driver_fn<PFN_waitValue32>("cuStreamWaitValue32");
    if (step && !wait_fn) return fail(WIND_ERR_CUDA, "cuStreamWaitValue32 entry point unavailable");
    int launches = 0;
    if (!step) {
      WKV_CUDA(launch_pace(t0, 0, 1, s), "pace kernel launch");
      ++launches;
    }
    uint32_t k = 0;
    for (int64_t u = 0; u < p.total_units; u += slice_units, ++k) {
      p.unit_lo = u;
      p.unit_hi = std::min<int64_t>(p.total_units, u + slice_units);
      p.first_slice = u == 0;
      if (step) {  // released by the consumer's step `first + k` (wrap-safe >=)
        CUresult r = wait_fn(static_cast<CUstream>(stream), reinterpret_cast<CUdeviceptr>(step->counter),
                             step->first + k, CU_STREAM_WAIT_VALUE_GEQ);
        if (r != CUDA_SUCCESS) return fail(WIND_ERR_CUDA, "cuStreamWaitValue32 failed (CUresult %d)", static_cast<int>(r));
      }
      cudaError_t e = launch_copy(p, kernel, static_cast<int>(std::min<int64_t>(grid, p.unit_hi - u)), s,
                                  pdl_enabled());
      if (e != cudaSuccess) return cuda_fail(e, "copy kernel launch");
      ++launches;
      if (step) continue;
      // hold the stream until the schedule reaches the bytes moved so far (after the last
      // slice too: the op then ends when its rate says, as the in-kernel pacer's ops do)
      const double done = payload * static_cast<double>(p.unit_hi) / static_cast<double>(p.total_units);
      WKV_CUDA(launch_pace(t0, static_cast<uint64_t>(done * 1e3 / t.rate_mbps), 0, s), "pace kernel launch");
      ++launches;
    }
    g_launches += launches;
    if ((st = finish_slot(ctx, sl, s)) != WIND_OK) return st;
    if ((st = order.commit(exec)) != WIND_OK) return st;
    for (int j = 0; j < n_items; ++j) items[j].dst->enqueued.fetch_add(1);
    return WIND_OK;
  }
  // rate limit: each of the `grid` CTAs gets rate / grid; ns per payload byte per CTA
  p.ns_per_byte = t.rate_mbps > 0 ? static_cast<float>(grid * 1e3 / t.rate_mbps) : 0.f;
  cudaError_t e = launch_copy(p, kernel, static_cast<int>(grid), s, pdl_enabled());
  if (e != cudaSuccess) {
    release_slot(ctx, sl);  // nothing of this op was enqueued (a debug check is harmless)
    return cuda_fail(e, "copy kernel launch");
  }
  g_launches += 1;
  if ((st = finish_slot(ctx, sl, s)) != WIND_OK) return st;
  if ((st = order.commit(exec)) != WIND_OK) return st;
  for (int j = 0; j < n_items; ++j) items[j].dst->enqueued.fetch_add(1);
  return WIND_OK;
}

}  // namespace

// ---------------------------------------------------------------- data-movement ABI

extern "C" wind_status wind_kv_migrate(const wind_kv_pool* src, const int32_t* src_bt,
                                       wind_kv_pool* dst, const int32_t* dst_bt, int32_t n_blocks,
                                       int32_t layer_lo, int32_t layer_hi, void* stream) {
  if (!dst) return fail(WIND_ERR_INVALID_ARG, "dst pool is NULL");
  OpItem it{dst, src_bt, dst_bt, n_blocks};
  return run_op(src, &it, 1, layer_lo, layer_hi, stream);
}

extern "C" wind_status wind_kv_migrate_heads(const wind_kv_pool* src, const int32_t* src_bt,
                                             wind_kv_pool* dst, const int32_t* dst_bt, int32_t n_blocks,
                                             int32_t layer_lo, int32_t layer_hi, int32_t src_head_lo,
                                             int32_t dst_head_lo, int32_t n_heads, void* stream) {
  if (!dst) return fail(WIND_ERR_INVALID_ARG, "dst pool is NULL");
  OpItem it{dst, src_bt, dst_bt, n_blocks};
  HeadRange hr;
  hr.src_lo = src_head_lo;
  hr.dst_lo = dst_head_lo;
  hr.n = n_heads < 0 ? 0 : n_heads;  // n_heads < 1 is rejected by check_args
  return run_op(src, &it, 1, layer_lo, layer_hi, stream, hr);
}

extern "C" wind_status wind_kv_migrate_batch(const wind_kv_pool* src, const wind_kv_migrate_item* items,
                                             int32_t n_items, int32_t layer_lo, int32_t layer_hi,
                                             void* stream) {
  if (!items || n_items < 1 || n_items > WIND_KV_MAX_BATCH)
    return fail(WIND_ERR_INVALID_ARG, "items NULL or n_items out of [1, %d]", WIND_KV_MAX_BATCH);
  OpItem its[WIND_KV_MAX_BATCH];
  for (int j = 0; j < n_items; ++j) {
    if (!items[j].dst) return fail(WIND_ERR_INVALID_ARG, "batch item %d has no dst", j);
    its[j] = OpItem{items[j].dst, items[j].src_bt, items[j].dst_bt, items[j].n_blocks};
  }
  return run_op(src, its, n_items, layer_lo, layer_hi, stream);
}

extern "C" wind_status wind_kv_swap_out(const wind_kv_pool* dev, const int32_t* dev_bt,
                                        wind_kv_pool* host, const int32_t* host_bt, int32_t n,
                                        void* stream) {
  if (!dev || !host) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  if (dev->desc.loc != WIND_LOC_DEVICE || host->desc.loc != WIND_LOC_HOST)
    return fail(WIND_ERR_INVALID_ARG, "swap_out needs a device source and a host destination");
  return wind_kv_migrate(dev, dev_bt, host, host_bt, n, dev->desc.first_layer,
                         dev->desc.first_layer + dev->desc.n_layers, stream);
}

extern "C" wind_status wind_kv_swap_in(const wind_kv_pool* host, const int32_t* host_bt,
                                       wind_kv_pool* dev, const int32_t* dev_bt, int32_t n,
                                       void* stream) {
  if (!dev || !host) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  if (dev->desc.loc != WIND_LOC_DEVICE || host->desc.loc != WIND_LOC_HOST)
    return fail(WIND_ERR_INVALID_ARG, "swap_in needs a host source and a device destination");
  return wind_kv_migrate(host, host_bt, dev, dev_bt, n, dev->desc.first_layer,
                         dev->desc.first_layer + dev->desc.n_layers, stream);
}

extern "C" wind_status wind_kv_compact(wind_kv_pool* pool, const int32_t* src_bt,
                                       const int32_t* dst_bt, int32_t n, void* stream) {
  if (!pool) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  return wind_kv_migrate(pool, src_bt, pool, dst_bt, n, pool->desc.first_layer,
                         pool->desc.first_layer + pool->desc.n_layers, stream);
}

// Which device and path an op from src to dst takes (tests and diagnostics: a green
// multi-device test must have run the PEER route, not INTRA).
extern "C" wind_status wind_kv_route(const wind_kv_pool* src, const wind_kv_pool* dst,
                                     int32_t* exec_device, int32_t* path, int32_t* sys_scope) {
  if (!src || !dst) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  int exec = -1, pth = 0;
  wind_status st = route(src, dst, &exec, &pth);
  if (st != WIND_OK) return st;
  if (exec_device) *exec_device = exec;
  if (path) *path = pth;
  // the publication scope run_op chooses: GPU scope only when both pools are device pools on
  // the executing GPU
  if (sys_scope)
    *sys_scope = force_sys_scope() || !local_pair(src, dst);
  return WIND_OK;
}

// ------------------------------------------------------------------- layer flags

extern "C" wind_status wind_kv_layer_ticket(const wind_kv_pool* dst, uint32_t* ticket) {
  if (!dst || !ticket) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  *ticket = dst->enqueued.load();
  return WIND_OK;
}

extern "C" wind_status wind_kv_layer_wait(const wind_kv_pool* dst, int32_t layer, uint32_t ticket,
                                          void* consumer) {
  if (!dst) return fail(WIND_ERR_INVALID_ARG, "dst is NULL");
  if (layer < dst->desc.first_layer || layer >= dst->desc.first_layer + dst->desc.n_layers)
    return fail(WIND_ERR_LAYER_RANGE, "layer %d not in pool", layer);
  static PFN_waitValue32 fn = driver_fn<PFN_waitValue32>("cuStreamWaitValue32");
  if (!fn) return fail(WIND_ERR_CUDA, "cuStreamWaitValue32 entry point unavailable");
  const uint32_t* f = dst->flags + (layer - dst->desc.first_layer);
  CUresult r = fn(static_cast<CUstream>(consumer), reinterpret_cast<CUdeviceptr>(f), ticket,
                  CU_STREAM_WAIT_VALUE_GEQ);
  if (r != CUDA_SUCCESS) return fail(WIND_ERR_CUDA, "cuStreamWaitValue32 failed (CUresult %d)", static_cast<int>(r));
  return WIND_OK;
}

extern "C" wind_status wind_kv_read_flags(const wind_kv_pool* p, uint32_t* out, void* stream) {
  if (!p || !out) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  if (p->desc.loc == WIND_LOC_DEVICE) {
    wind_status st = check_stream(stream, p->desc.device);
    if (st != WIND_OK) return st;
  }
  DeviceGuard g(p->desc.loc == WIND_LOC_DEVICE ? p->desc.device : 0);
  WKV_CUDA(cudaMemcpyAsync(out, p->flags, sizeof(uint32_t) * p->desc.n_layers, cudaMemcpyDefault,
                           static_cast<cudaStream_t>(stream)),
           "cudaMemcpyAsync(flags)");
  return WIND_OK;
}

extern "C" wind_status wind_kv_layer_count(const wind_kv_pool* dst, int32_t layer, uint32_t* value) {
  if (!dst || !value) return fail(WIND_ERR_INVALID_ARG, "NULL argument");
  if (layer < dst->desc.first_layer || layer >= dst->desc.first_layer + dst->desc.n_layers)
    return fail(WIND_ERR_LAYER_RANGE, "layer %d not in pool", layer);
  const uint32_t* f = dst->flags + (layer - dst->desc.first_layer);
  if (dst->desc.loc == WIND_LOC_HOST) {
    *value = *reinterpret_cast<const volatile uint32_t*>(f);
    return WIND_OK;
  }
  DeviceGuard g(dst->desc.device);
  WKV_CUDA(cudaMemcpy(value, f, sizeof(uint32_t), cudaMemcpyDeviceToHost), "cudaMemcpy(flag)");
  return WIND_OK;
}

// ------------------------------------------------------------------- host logic

extern "C" wind_status wind_kv_validate(const wind_kv_pool* src, const int32_t* sbt,
                                        const wind_kv_pool* dst, const int32_t* dbt, int32_t n,
                                        int32_t lo, int32_t hi) {
  wind_status st = check_args(src, dst, n, sbt, dbt, lo, hi);
  if (st != WIND_OK) return st;
  return check_tables_host(src, sbt, dst, dbt, n);
}

extern "C" wind_status wind_kv_plan_compact(const uint8_t* live, int32_t n_slots, int32_t* src_bt,
                                            int32_t* dst_bt, int32_t* n_moves) {
  if (!n_moves || n_slots < 0 || (n_slots > 0 && !live)) return fail(WIND_ERR_INVALID_ARG, "bad arguments");
  int32_t n_live = 0;
  for (int32_t b = 0; b < n_slots; ++b) n_live += live[b] != 0;
  // two fingers: `h` walks holes below n_live upward, `m` walks live slots at/above it upward
  int32_t k = 0, h = 0, m = n_live;
  for (;;) {
    while (h < n_live && live[h]) ++h;
    while (m < n_slots && !live[m]) ++m;
    if (h >= n_live || m >= n_slots) break;
    if (src_bt) src_bt[k] = m;
    if (dst_bt) dst_bt[k] = h;
    ++k, ++h, ++m;
  }
  *n_moves = k;
  return WIND_OK;
}

extern "C" wind_status wind_kv_plan_rebalance(int32_t G, int32_t R, const int32_t* req_gpu,
                                              const int32_t* req_blocks, int32_t* out_gpu,
                                              int32_t* n_moves) {
  if (G < 1 || R < 0 || !n_moves || (R > 0 && (!req_gpu || !req_blocks || !out_gpu)))
    return fail(WIND_ERR_INVALID_ARG, "bad arguments");
  std::vector<int64_t> load(G, 0);
  // per GPU: candidate requests sorted by (blocks desc, id asc); removed lazily
  std::vector<std::vector<int32_t>> by_gpu(G);
  int64_t total = 0;
  for (int32_t r = 0; r < R; ++r) {
    if (req_gpu[r] < 0 || req_gpu[r] >= G || req_blocks[r] < 0)
      return fail(WIND_ERR_INVALID_ARG, "request %d: bad gpu or block count", r);
    out_gpu[r] = req_gpu[r];
    load[req_gpu[r]] += req_blocks[r];
    total += req_blocks[r];
    if (req_blocks[r] > 0) by_gpu[req_gpu[r]].push_back(r);
  }
  for (auto& v : by_gpu)
    std::sort(v.begin(), v.end(), [&](int32_t a, int32_t b) {
      return req_blocks[a] != req_blocks[b] ? req_blocks[a] > req_blocks[b] : a < b;
    });
  const int64_t target = (total + G - 1) / G;
  int32_t moves = 0;
  for (;;) {
    const int src = static_cast<int>(std::max_element(load.begin(), load.end()) - load.begin());
    const int dst = static_cast<int>(std::min_element(load.begin(), load.end()) - load.begin());
    if (load[src] <= target || src == dst) break;
    const int64_t room = target - load[dst];
    auto& v = by_gpu[src];
    // first (longest, lowest id) request with blocks <= room: v is sorted by blocks desc
    auto itr = std::lower_bound(v.begin(), v.end(), room, [&](int32_t r, int64_t rm) {
      return req_blocks[r] > rm;
    });
    if (itr == v.end()) break;
    const int32_t r = *itr;
    v.erase(itr);
    out_gpu[r] = dst;
    load[src] -= req_blocks[r];
    load[dst] += req_blocks[r];
    ++moves;
    // r never moves again: dst stays <= target, so it never becomes the source
  }
  *n_moves = moves;
  return WIND_OK;
}

extern "C" wind_status wind_kv_check_device_error(const wind_kv_pool* p) {
  if (!p) return fail(WIND_ERR_INVALID_ARG, "pool is NULL");
  int32_t worst = 0;
  for (int d = 0; d < kMaxDevices; ++d) {
    DevCtx& c = g_dev[d];
    if (!c.ready) continue;
    if (p->desc.loc == WIND_LOC_DEVICE && d != p->desc.device) continue;
    DeviceGuard g(d);
    WKV_CUDA(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
    int32_t v = 0;
    WKV_CUDA(cudaMemcpy(&v, c.err, sizeof v, cudaMemcpyDeviceToHost), "cudaMemcpy(err)");
    WKV_CUDA(cudaMemset(c.err, 0, sizeof v), "cudaMemset(err)");
    worst = std::max(worst, v);
  }
  if (worst == 0) return WIND_OK;
  const char* what = worst == 4 ? "BLOCK_RANGE" : worst == 3 ? "DUP_DST" : "ALIAS";
  return fail(WIND_ERR_DEVICE_CHECK, "device table check recorded %s", what);
}

// -------------------------------------------------------------------- tuning/misc

extern "C" wind_status wind_kv_set_tuning(int32_t path, const wind_kv_tuning* t) {
  if (path < 0 || path > 2 || !t) return fail(WIND_ERR_INVALID_ARG, "bad path or NULL tuning");
  std::lock_guard<std::mutex> lk(g_tune_mu);
  wind_kv_tuning n = g_tune[path];
  if (t->kernel < 0 || t->kernel > 4) return fail(WIND_ERR_INVALID_ARG, "kernel must be 0 .. 4");
  if (t->kernel == kStaged && path != WIND_PATH_HOST)
    return fail(WIND_ERR_INVALID_ARG, "kernel 4 (staged copy engines) is a HOST-path kernel");
  n.kernel = t->kernel;
  if (t->ctas_per_sm) n.ctas_per_sm = t->ctas_per_sm;
  if (t->stage_bytes) n.stage_bytes = t->stage_bytes;
  if (t->stages) n.stages = t->stages;
  n.max_ctas = t->max_ctas;
  n.evict_first = t->evict_first;
  n.store_lag = t->store_lag;
  n.rate_mbps = t->rate_mbps;
  if (n.store_lag < 0 || n.store_lag >= n.stages) return fail(WIND_ERR_INVALID_ARG, "store_lag out of [0, stages)");
  if (n.rate_mbps < 0) return fail(WIND_ERR_INVALID_ARG, "rate_mbps < 0");
  if (n.ctas_per_sm < 1 || n.ctas_per_sm > 32) return fail(WIND_ERR_INVALID_ARG, "ctas_per_sm out of [1, 32]");
  if (n.stage_bytes < 16 || n.stage_bytes % 16) return fail(WIND_ERR_INVALID_ARG, "stage_bytes must be a positive multiple of 16");
  if (n.stages < 3 || n.stages > 16) return fail(WIND_ERR_INVALID_ARG, "stages out of [3, 16]");
  if (n.kernel != kSimt && tma_smem_bytes(n.stages, n.stage_bytes) > 227 * 1024)
    return fail(WIND_ERR_INVALID_ARG, "stages * stage_bytes exceeds shared memory");
  g_tune[path] = n;
  return WIND_OK;
}

extern "C" wind_status wind_kv_migrate_ex(const wind_kv_pool* src, const int32_t* src_bt,
                                          wind_kv_pool* dst, const int32_t* dst_bt, int32_t n_blocks,
                                          int32_t layer_lo, int32_t layer_hi, const wind_kv_tuning* tuning,
                                          void* stream) {
  if (!dst) return fail(WIND_ERR_INVALID_ARG, "dst pool is NULL");
  if (tuning) {  // validate the override like set_tuning would, then apply it to this op only
    if (tuning->kernel < 0 || tuning->kernel > 4) return fail(WIND_ERR_INVALID_ARG, "kernel must be 0..4");
    if (tuning->ctas_per_sm < 1 || tuning->ctas_per_sm > 32 || tuning->stage_bytes < 16 ||
        tuning->stage_bytes % 16 || tuning->stages < 3 || tuning->stages > 16 || tuning->store_lag < 0 ||
        tuning->store_lag >= tuning->stages || tuning->rate_mbps < 0 || tuning->max_ctas < 0)
      return fail(WIND_ERR_INVALID_ARG, "override tuning out of range (all fields explicit, see wind_kv.h)");
    if (tuning->kernel != kSimt && tma_smem_bytes(tuning->stages, tuning->stage_bytes) > 227 * 1024)
      return fail(WIND_ERR_INVALID_ARG, "stages * stage_bytes exceeds shared memory");
  }
  OpItem it{dst, src_bt, dst_bt, n_blocks};
  return run_op(src, &it, 1, layer_lo, layer_hi, stream, HeadRange(), tuning);
}

extern "C" wind_status wind_kv_migrate_stepped(const wind_kv_pool* src, const int32_t* src_bt,
                                               wind_kv_pool* dst, const int32_t* dst_bt, int32_t n_blocks,
                                               int32_t layer_lo, int32_t layer_hi,
                                               const uint32_t* step_counter, uint32_t first_step,
                                               uint64_t bytes_per_step, void* stream) {
  if (!dst) return fail(WIND_ERR_INVALID_ARG, "dst pool is NULL");
  if (!step_counter || bytes_per_step == 0)
    return fail(WIND_ERR_INVALID_ARG, "step_counter is NULL or bytes_per_step is 0");
  if (reinterpret_cast<uintptr_t>(step_counter) & 3) return fail(WIND_ERR_INVALID_ARG, "step_counter misaligned");
  OpItem it{dst, src_bt, dst_bt, n_blocks};
  const StepPacing sp{step_counter, first_step, bytes_per_step};
  return run_op(src, &it, 1, layer_lo, layer_hi, stream, HeadRange(), nullptr, &sp);
}

extern "C" wind_status wind_kv_step_signal(uint32_t* step_counter, void* stream) {
  if (!step_counter || (reinterpret_cast<uintptr_t>(step_counter) & 3))
    return fail(WIND_ERR_INVALID_ARG, "step_counter is NULL or misaligned");
  int d = -1;  // load the library's kernels on the stream's device first (no lazy loading later)
  if (!stream || cudaStreamGetDevice(static_cast<cudaStream_t>(stream), &d) != cudaSuccess) {
    cudaGetLastError();
    WKV_CUDA(cudaGetDevice(&d), "cudaGetDevice");
  }
  DevCtx* ctx;
  wind_status st = dev_ctx(d, &ctx);
  if (st != WIND_OK) return st;
  WKV_CUDA(launch_step_signal(step_counter, static_cast<cudaStream_t>(stream)), "step signal launch");
  g_launches += 1;
  return WIND_OK;
}

extern "C" wind_status wind_kv_get_tuning(int32_t path, wind_kv_tuning* t) {
  if (path < 0 || path > 2 || !t) return fail(WIND_ERR_INVALID_ARG, "bad path or NULL tuning");
  std::lock_guard<std::mutex> lk(g_tune_mu);
  *t = g_tune[path];
  return WIND_OK;
}

extern "C" uint64_t wind_kv_launch_count(void) { return g_launches.load(); }

extern "C" const char* wind_kv_status_string(wind_status s) {
  switch (s) {
    case WIND_OK: return "WIND_OK";
    case WIND_ERR_INVALID_ARG: return "WIND_ERR_INVALID_ARG";
    case WIND_ERR_GEOMETRY: return "WIND_ERR_GEOMETRY";
    case WIND_ERR_LAYER_RANGE: return "WIND_ERR_LAYER_RANGE";
    case WIND_ERR_BLOCK_RANGE: return "WIND_ERR_BLOCK_RANGE";
    case WIND_ERR_DUP_DST: return "WIND_ERR_DUP_DST";
    case WIND_ERR_ALIAS: return "WIND_ERR_ALIAS";
    case WIND_ERR_NO_PEER: return "WIND_ERR_NO_PEER";
    case WIND_ERR_CUDA: return "WIND_ERR_CUDA";
    case WIND_ERR_OOM: return "WIND_ERR_OOM";
    case WIND_ERR_UNSUPPORTED: return "WIND_ERR_UNSUPPORTED";
    case WIND_ERR_DEVICE_CHECK: return "WIND_ERR_DEVICE_CHECK";
    default: return "WIND_ERR_UNKNOWN";
  }
}

extern "C" const char* wind_kv_last_error(void) { return g_last_error.c_str(); }

// ------------------------------------------------------------------ SM partition

namespace {

typedef CUresult (*PFN_deviceGet)(CUdevice*, int);
typedef CUresult (*PFN_getDevResource)(CUdevice, CUdevResource*, CUdevResourceType);
typedef CUresult (*PFN_smSplit)(CUdevResource*, unsigned int*, const CUdevResource*, CUdevResource*,
                                unsigned int, unsigned int);
typedef CUresult (*PFN_genDesc)(CUdevResourceDesc*, CUdevResource*, unsigned int);
typedef CUresult (*PFN_greenCreate)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned int);
typedef CUresult (*PFN_greenDestroy)(CUgreenCtx);
typedef CUresult (*PFN_greenStream)(CUstream*, CUgreenCtx, unsigned int, int);
typedef CUresult (*PFN_streamDestroy)(CUstream);

// Driver entry points through the runtime's query, else straight from libcuda.so.1 (the
// library never links libcuda, so it still loads on a machine without a driver).
template <typename F>
F green_fn(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPointByVersion(name, &fn, 12080, cudaEnableDefault, &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess && fn)
    return reinterpret_cast<F>(fn);
  cudaGetLastError();
  static void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_NOLOAD);
  if (!h) h = dlopen("libcuda.so.1", RTLD_NOW);
  if (!h) return nullptr;
  return reinterpret_cast<F>(dlsym(h, name));
}

}  // namespace

// Streams created by wind_kv_partition_sms and the SM count of their partition (ops on them
// cap their grid to it; looked up by stream handle).
std::mutex g_part_mu;
std::vector<std::pair<void*, int32_t>> g_part_streams;

int32_t partition_sms_of(void* stream) {
  if (!stream) return 0;
  std::lock_guard<std::mutex> lk(g_part_mu);
  for (auto& e : g_part_streams)
    if (e.first == stream) return e.second;
  return 0;
}

extern "C" wind_status wind_kv_partition_sms(int32_t device, int32_t min_sms_migration,
                                             wind_kv_sm_partition* out) {
  if (!out || min_sms_migration < 1) return fail(WIND_ERR_INVALID_ARG, "NULL out or min_sms_migration < 1");
  memset(out, 0, sizeof *out);
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return fail(WIND_ERR_INVALID_ARG, "bad device %d", device);
  }
  auto dget = green_fn<PFN_deviceGet>("cuDeviceGet");
  auto gres = green_fn<PFN_getDevResource>("cuDeviceGetDevResource");
  auto split = green_fn<PFN_smSplit>("cuDevSmResourceSplitByCount");
  auto gdesc = green_fn<PFN_genDesc>("cuDevResourceGenerateDesc");
  auto gcreate = green_fn<PFN_greenCreate>("cuGreenCtxCreate");
  auto gdestroy = green_fn<PFN_greenDestroy>("cuGreenCtxDestroy");
  auto gstream = green_fn<PFN_greenStream>("cuGreenCtxStreamCreate");
  const char* missing = !dget ? "cuDeviceGet" : !gres ? "cuDeviceGetDevResource" : !split ? "cuDevSmResourceSplitByCount"
                       : !gdesc ? "cuDevResourceGenerateDesc" : !gcreate ? "cuGreenCtxCreate"
                       : !gdestroy ? "cuGreenCtxDestroy" : !gstream ? "cuGreenCtxStreamCreate" : nullptr;
  if (missing) return fail(WIND_ERR_UNSUPPORTED, "driver entry point %s unavailable", missing);
  DeviceGuard g(device);
  cudaFree(nullptr);  // the primary context exists (runtime initialised on this device)
  CUdevice dev;
  CUresult r = dget(&dev, device);
  CUdevResource all, grp, rest;
  memset(&grp, 0, sizeof grp);
  memset(&rest, 0, sizeof rest);
  unsigned int ng = 1;
  if (r == CUDA_SUCCESS) r = gres(dev, &all, CU_DEV_RESOURCE_TYPE_SM);
  if (r == CUDA_SUCCESS) r = split(&grp, &ng, &all, &rest, 0, static_cast<unsigned int>(min_sms_migration));
  if (r != CUDA_SUCCESS || ng != 1 || rest.sm.smCount == 0)
    return fail(WIND_ERR_INVALID_ARG, "cannot split %d SMs off device %d (CUresult %d)", min_sms_migration,
                device, static_cast<int>(r));
  CUdevResourceDesc dm, dc;
  CUgreenCtx gm = nullptr, gc = nullptr;
  CUstream sm = nullptr, sc = nullptr;
  r = gdesc(&dm, &grp, 1);
  if (r == CUDA_SUCCESS) r = gdesc(&dc, &rest, 1);
  if (r == CUDA_SUCCESS) r = gcreate(&gm, dm, dev, CU_GREEN_CTX_DEFAULT_STREAM);
  if (r == CUDA_SUCCESS) r = gcreate(&gc, dc, dev, CU_GREEN_CTX_DEFAULT_STREAM);
  int lo_pri = 0, hi_pri = 0;
  cudaDeviceGetStreamPriorityRange(&lo_pri, &hi_pri);
  if (r == CUDA_SUCCESS) r = gstream(&sm, gm, CU_STREAM_NON_BLOCKING, lo_pri);
  if (r == CUDA_SUCCESS) r = gstream(&sc, gc, CU_STREAM_NON_BLOCKING, hi_pri);
  if (r != CUDA_SUCCESS) {
    if (gm) gdestroy(gm);
    if (gc) gdestroy(gc);
    return fail(WIND_ERR_CUDA, "green context / stream creation failed (CUresult %d)", static_cast<int>(r));
  }
  out->migration_stream = sm;
  out->compute_stream = sc;
  out->sms_migration = static_cast<int32_t>(grp.sm.smCount);
  out->sms_compute = static_cast<int32_t>(rest.sm.smCount);
  out->_internal[0] = gm;
  out->_internal[1] = gc;
  std::lock_guard<std::mutex> lk(g_part_mu);
  g_part_streams.emplace_back(sm, out->sms_migration);
  g_part_streams.emplace_back(sc, out->sms_compute);
  return WIND_OK;
}

extern "C" wind_status wind_kv_partition_destroy(wind_kv_sm_partition* part) {
  if (!part) return fail(WIND_ERR_INVALID_ARG, "NULL partition");
  auto sdestroy = green_fn<PFN_streamDestroy>("cuStreamDestroy");
  auto gdestroy = green_fn<PFN_greenDestroy>("cuGreenCtxDestroy");
  if (!sdestroy || !gdestroy) return fail(WIND_ERR_UNSUPPORTED, "green-context entry points unavailable");
  {
    std::lock_guard<std::mutex> lk(g_part_mu);
    g_part_streams.erase(std::remove_if(g_part_streams.begin(), g_part_streams.end(),
                                        [&](const std::pair<void*, int32_t>& e) {
                                          return e.first == part->migration_stream ||
                                                 e.first == part->compute_stream;
                                        }),
                         g_part_streams.end());
  }
  if (part->migration_stream) sdestroy(static_cast<CUstream>(part->migration_stream));
  if (part->compute_stream) sdestroy(static_cast<CUstream>(part->compute_stream));
  for (void* gctx : part->_internal)
    if (gctx) gdestroy(static_cast<CUgreenCtx>(gctx));
  memset(part, 0, sizeof *part);
  return WIND_OK;
}

extern "C" const char* wind_kv_version(void) { return "wind_kv 0.1.0 (sm_100a)"; }
