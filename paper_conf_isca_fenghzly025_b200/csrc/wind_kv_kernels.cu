// wind_kv_kernels.cu — the sm_100a kernels of the paged KV-migration hot path.
//
// What they compute (include/wind_kv.h): for each (global layer
// l in [lo, hi), kv in {K, V}) "plane" and each table entry i,
//     dst[l][kv][dst_bt[i]] := src[l][kv][src_bt[i]]          (C contiguous bytes)
// with the pools laid out [L][2][NB][H][bs][d] (reading R2), so every (layer, kv, block)
// chunk is one contiguous C-byte span on both sides.  Pure data movement: no tensor
// cores, no arithmetic on the payload (R13).
//
// Work decomposition (shared by both kernels).  A *unit* is at most `unit` bytes:
//   C >= unit : one chunk split into `parts` pieces of part_bytes;
//   C <  unit : a window of `group` (<= 32) consecutive table entries.  One warp loads
//               the window, marks run heads where NOT (s_i = s_{i-1}+1 AND
//               d_i = d_{i-1}+1) with __ballot_sync, and gives each run its segment
//               index by prefix popcount (K3 run coalescer): a run of k
//               adjacent blocks becomes ONE k*C-byte copy on both sides.
// Units are numbered plane-major (layer ascending) and dealt to CTAs grid-stride,
// so all CTAs sweep the layers together and a layer completes early (A5 streaming).
//
// Layer completion (A5).  When a CTA leaves layer l (its next unit is in a later layer, or
// it is done) it makes its stores of l complete and visible, then adds the number of l's
// units it moved to this op's arrival counter for l; the CTA that brings the counter to
// the layer's unit total (2 planes x units_per_plane) publishes dst.layer_done[l] += 1
// behind a release fence — GPU scope when the data and the flags stay on this GPU, system
// scope for a peer (NVLink) or host destination — and resets the counter for the next op
// using the slot.  A CTA arrives only on layers it touched (a small op's CTAs touch one or
// two), so an op costs one counter atomic per (CTA, touched layer).  The TMA consumer
// defers the arrival until `lag` newer store groups are in flight, so the store pipeline
// never drains at a layer boundary.
//
// Kernels.
//   tma_copy_kernel  (K2): 2 warps per CTA.  Warp 0 = producer: decodes units and issues
//     cp.async.bulk global->shared loads into an S-stage ring (mbarrier complete_tx).
//     Warp 1 lane 0 = consumer: issues cp.async.bulk shared->global stores (bulk_group)
//     and frees a stage once the store issued two units later has read it.  One thread
//     keeps ~S*unit bytes in flight per CTA with a handful of instructions.
//   simt_copy_kernel (K1): 512 threads per CTA, 16-byte ld.global.nc.L1::no_allocate /
//     st.global vectors, 4 loads in flight per thread before the stores.
#include <cuda_runtime.h>
#include <stdint.h>

#include "wind_kv_internal.h"

namespace wkv {
namespace {

constexpr unsigned kFull = 0xffffffffu;

struct Seg {
  const uint8_t* src;
  uint8_t* dst;
  uint32_t len;   // bytes (multiple of 16)
  uint32_t soff;  // offset inside the unit's staging buffer
};

struct __align__(16) Desc {
  int32_t nseg;   // -1 = end of work
  int32_t plane;  // (l - lo) * 2 + kv
  Seg segs[kMaxSegs];
  uint8_t* fdst[kMaxFan - 1][kMaxSegs];  // fan-out: segment k's address in destination 1 + f
};

// ----------------------------------------------------------------------- PTX helpers

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WKV_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WKV_WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void bulk_load(void* sdst, const void* gsrc, uint32_t bytes,
                                          uint64_t* bar, bool ef, uint64_t pol) {
  if (ef)
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(sdst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
  else
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1], %2, [%3];" ::"r"(smem_u32(sdst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void bulk_store(void* gdst, const void* ssrc, uint32_t bytes,
                                           bool ef, uint64_t pol) {
  if (ef)
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
                 ::"l"(gdst), "r"(smem_u32(ssrc)), "r"(bytes), "l"(pol)
                 : "memory");
  else
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst),
                 "r"(smem_u32(ssrc)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;"); }

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void bulk_wait_all() {
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__device__ __forceinline__ void fence_sys() {
  asm volatile("fence.acq_rel.sys;" ::: "memory");
}

__device__ __forceinline__ void fence_gpu() {
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

__device__ __forceinline__ void fence_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

__device__ __forceinline__ int4 ld_stream(const int4* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ int4 ld_stream_ef(const int4* p, uint64_t pol) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p), "l"(pol));
  return r;
}

__device__ __forceinline__ void st_stream(int4* p, const int4& v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x),
               "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

__device__ __forceinline__ void st_stream_ef(int4* p, const int4& v, uint64_t pol) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.s32 [%0], {%1, %2, %3, %4}, %5;"
               ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol)
               : "memory");
}

// Programmatic dependent launch (PDL): a copy kernel launched right behind another one on
// its stream may start its prologue (shared-memory carve-out, mbarrier init) on SMs the
// previous grid has left, then waits here for that grid to complete and flush before it
// touches any global memory — data, flags or counters.  No-op without the launch attribute.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Rate limit (wind_kv_tuning.rate_mbps): a per-CTA pacer.  Before a unit of `bytes` is
// issued, wait until the CTA's schedule allows it, then push the schedule by
// bytes * ns_per_byte.  Bursts are bounded: a CTA that fell behind (slow memory) catches up
// at most one unit ahead of real time.
struct Pacer {
  uint64_t next = 0;
  __device__ __forceinline__ void wait(float ns_per_byte, uint32_t bytes) {
    if (ns_per_byte <= 0.f) return;
    uint64_t now = globaltimer_ns();
    if (next == 0 || next + 20000 < now) next = now;  // start, or behind by > 20 us
    while (now < next) {
      const uint64_t d = next - now;
      __nanosleep(d > 1000000 ? 1000000u : static_cast<unsigned>(d));
      now = globaltimer_ns();
    }
    next += static_cast<uint64_t>(static_cast<float>(bytes) * ns_per_byte);
  }
};

// --------------------------------------------------------------------- work decoding

// Decodes unit u into segments (called by a FULL warp; writes segs[] from the lanes that
// own a segment).  Returns the (warp-uniform) segment count; *plane_out, *bytes_out.
// Fan-out (p.fan > 1, fdst != nullptr): the units walk items[0]'s source table; a run must
// be adjacent in the source and in EVERY destination, and fdst[f][k] receives segment k's
// address in destination 1 + f.
// decode_unit_at takes the unit as (plane, r = its index inside the plane); the TMA producer
// keeps those incrementally (no 64-bit division per unit on its critical path).
__device__ __forceinline__ int decode_unit_at(const Params& p, int64_t plane, int32_t r, Seg* segs,
                                              uint8_t* (*fdst)[kMaxSegs], int32_t* plane_out,
                                              uint32_t* bytes_out) {
  const int lane = threadIdx.x & 31;
  int j = 0;
  if (p.fan <= 1)
    while (j + 1 < p.n_items && r >= p.items[j + 1].unit_base) ++j;
  const int fan = fdst ? p.fan : 1;
  const Item& it = p.items[j];
  r -= it.unit_base;
  const uint8_t* splane = p.src_plane0 + plane * p.s_plane_stride;
  uint8_t* dplane = it.dst_plane0 + plane * it.d_plane_stride;
  const int64_t CS = p.s_chunk, CD = it.d_chunk, CP = p.copy;  // CP == CS == CD unless a head range
  *plane_out = static_cast<int32_t>(plane);
  if (p.parts > 1) {  // one block's span, piece `part`
    const int32_t i = r / p.parts;
    const int32_t part = r - i * p.parts;
    const int64_t off = static_cast<int64_t>(part) * p.part_bytes;
    const int64_t rest = CP - off;
    const uint32_t len = static_cast<uint32_t>(rest < p.part_bytes ? rest : p.part_bytes);
    if (lane == 0) {
      const int32_t s = it.sbt[i], d = it.dbt[i];
      segs[0].src = splane + s * CS + off;
      segs[0].dst = dplane + d * CD + off;
      segs[0].len = len;
      segs[0].soff = 0;
    }
    if (lane > 0 && lane < fan) {  // lane f: destination f of the fan-out
      const Item& fi = p.items[lane];
      fdst[lane - 1][0] = fi.dst_plane0 + plane * fi.d_plane_stride + fi.dbt[i] * fi.d_chunk + off;
    }
    *bytes_out = len;
    return 1;
  }
  // a window of `group` entries: warp-ballot run coalescing (K3)
  const int32_t i0 = r * p.group;
  const int cnt = min(p.group, it.n - i0);
  int32_t s = 0, d = 0;
  int32_t df[kMaxFan - 1] = {0, 0, 0};
  if (lane < cnt) {
    s = it.sbt[i0 + lane];
    d = it.dbt[i0 + lane];
#pragma unroll
    for (int f = 1; f < kMaxFan; ++f)
      if (f < fan) df[f - 1] = p.items[f].dbt[i0 + lane];
  }
  const int32_t ps = __shfl_up_sync(kFull, s, 1);
  const int32_t pd = __shfl_up_sync(kFull, d, 1);
  bool adj = it.coalesce && s == ps + 1 && d == pd + 1;
#pragma unroll
  for (int f = 1; f < kMaxFan; ++f) {
    if (f < fan) {  // fan is warp-uniform
      const int32_t pf = __shfl_up_sync(kFull, df[f - 1], 1);
      adj = adj && df[f - 1] == pf + 1;
    }
  }
  const bool head = lane < cnt && (lane == 0 || !adj);
  const uint32_t heads = __ballot_sync(kFull, head);
  if (head) {
    const int k = __popc(heads & ((1u << lane) - 1u));       // prefix popcount
    const uint32_t later = heads & ~((2u << lane) - 1u);     // heads after this lane
    const int end = later ? __ffs(later) - 1 : cnt;
    segs[k].src = splane + s * CS;
    segs[k].dst = dplane + d * CD;
    segs[k].len = static_cast<uint32_t>((end - lane) * CP);
    segs[k].soff = static_cast<uint32_t>(lane * CP);
#pragma unroll
    for (int f = 1; f < kMaxFan; ++f) {
      if (f < fan) {
        const Item& fi = p.items[f];
        fdst[f - 1][k] = fi.dst_plane0 + plane * fi.d_plane_stride + df[f - 1] * fi.d_chunk;
      }
    }
  }
  *bytes_out = static_cast<uint32_t>(cnt * CP);
  return __popc(heads);
}

__device__ __forceinline__ int decode_unit(const Params& p, int64_t u, Seg* segs,
                                           uint8_t* (*fdst)[kMaxSegs], int32_t* plane_out,
                                           uint32_t* bytes_out) {
  const int64_t plane = u / p.units_per_plane;
  return decode_unit_at(p, plane, static_cast<int32_t>(u - plane * p.units_per_plane), segs, fdst,
                        plane_out, bytes_out);
}

// Adds 1 to a layer flag.  The caller has issued the release fence (fence.acq_rel at
// system scope when the item's data or flags leave this GPU, at GPU scope otherwise), so the
// increment itself is relaxed: one fence publishes every flag a thread bumps after it.
// Device-memory flags use a red reduction; flags of a host pool (mapped pinned memory, where
// PCIe may not carry atomics) a volatile read-modify-write — the executing device is then the
// only writer (wind_kv.h: one op at a time per host pool).
__device__ __forceinline__ void bump_flag(uint32_t* f, const Item& it) {
  if (it.host_flags) {
    const uint32_t v = *reinterpret_cast<volatile uint32_t*>(f);
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(f), "r"(v + 1u) : "memory");
  } else if (it.sys_scope) {
    asm volatile("red.relaxed.sys.global.add.u32 [%0], 1;" ::"l"(f) : "memory");
  } else {
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(f) : "memory");
  }
}

// Out-of-range layer flags: every op bumps every dst layer flag exactly once; the layers
// it does not move are bumped at the start (see wind_kv.h, wind_kv_migrate).  No data is
// published with them, so the bumps are relaxed (a release per flag costs a system-scope
// fence each, ~1 us); the caller is a thread off the copy's critical path.
__device__ void publish_untouched_layers(const Params& p) {
  for (int j = 0; j < p.n_items; ++j) {
    const Item& it = p.items[j];
    for (int f = 0; f < it.d_layers; ++f) {
      if (f >= it.d_flag_lo && f < it.d_flag_lo + p.n_layers) continue;
      uint32_t* fl = it.flags + f;
      if (!it.host_flags) {
        asm volatile("red.relaxed.sys.global.add.u32 [%0], 1;" ::"l"(fl) : "memory");
      } else {
        const uint32_t v = *reinterpret_cast<volatile uint32_t*>(fl);
        *reinterpret_cast<volatile uint32_t*>(fl) = v + 1u;
      }
    }
  }
}

// cp.async.bulk.wait_group.read needs an immediate: dispatch the runtime lag.
__device__ __forceinline__ void bulk_wait_read_n(int n) {
  switch (n) {
    case 0: bulk_wait_read<0>(); break;
    case 1: bulk_wait_read<1>(); break;
    case 2: bulk_wait_read<2>(); break;
    case 3: bulk_wait_read<3>(); break;
    case 4: bulk_wait_read<4>(); break;
    case 5: bulk_wait_read<5>(); break;
    case 6: bulk_wait_read<6>(); break;
    default: bulk_wait_read<7>(); break;
  }
}

// Same, but full completion (the stores' writes performed, not only their smem reads).
__device__ __forceinline__ void bulk_wait_done_n(int n) {
  switch (n) {
    case 0: asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); break;
    case 1: asm volatile("cp.async.bulk.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.bulk.wait_group 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.bulk.wait_group 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.bulk.wait_group 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.bulk.wait_group 5;" ::: "memory"); break;
    case 6: asm volatile("cp.async.bulk.wait_group 6;" ::: "memory"); break;
    default: asm volatile("cp.async.bulk.wait_group 7;" ::: "memory"); break;
  }
}

// Arrive on global layer `layer` with the `cnt` units of it this CTA moved; the arrival
// that completes the layer's 2 x units_per_plane units publishes.  Caller has made this
// CTA's stores of those units complete and ordered before this call.  Scope: when data and
// flags stay on this GPU (p.sys_scope == 0) every observer — the consumer stream's wait,
// the kernels it releases, another process's CTAs on this device — reads through this
// GPU's L2, so GPU-scope fences suffice; a fence.acq_rel.sys costs ~1 us.
__device__ void arrive_layer(const Params& p, int32_t layer, uint32_t cnt) {
  if (cnt == 0) return;
  if (p.sys_scope)
    fence_sys();
  else
    fence_gpu();
  uint32_t* c = p.counters + (layer - p.layer_lo);
  const uint32_t total = 2u * static_cast<uint32_t>(p.units_per_plane);
  if (atomicAdd(c, cnt) + cnt != total) return;
  if (p.sys_scope)  // acquire the other arrivals, release the flags below
    fence_sys();
  else
    fence_gpu();
  for (int j = 0; j < p.n_items; ++j)
    bump_flag(p.items[j].flags + p.items[j].d_flag_lo + (layer - p.layer_lo), p.items[j]);
  *reinterpret_cast<volatile uint32_t*>(c) = 0u;  // slot reusable
}

// Debug pools whose device table check fired: nothing is copied, but every layer flag of
// the op still moves once (a consumer waiting on a ticket must not hang).
__device__ void publish_aborted(const Params& p) {
  fence_sys();
  for (int32_t l = p.layer_lo; l < p.layer_lo + p.n_layers; ++l)
    for (int j = 0; j < p.n_items; ++j)
      bump_flag(p.items[j].flags + p.items[j].d_flag_lo + (l - p.layer_lo), p.items[j]);
}

// ------------------------------------------------------------------- K2: TMA staged

__global__ void __launch_bounds__(64, 1) tma_copy_kernel(const __grid_constant__ Params p) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int S = p.stages;
  const uint32_t SB = static_cast<uint32_t>(p.stage_bytes);
  uint8_t* buf = smem;
  Desc* desc = reinterpret_cast<Desc*>(smem + static_cast<size_t>(S) * SB);
  uint64_t* full = reinterpret_cast<uint64_t*>(desc + S);
  uint64_t* empty = full + S;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const bool ef = p.evict_first != 0;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 32);  // every producer lane arrives: each releases its own segment writes
      mbar_init(&empty[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  pdl_wait();  // everything below may see the previous grid's writes
  if (blockIdx.x == 0 && threadIdx.x == 33 && p.first_slice) publish_untouched_layers(p);  // an idle consumer lane
  if (p.abort_word && *reinterpret_cast<const volatile int32_t*>(p.abort_word)) {
    if (blockIdx.x == 0 && threadIdx.x == 0) publish_aborted(p);
    return;
  }

  if (warp == 0) {  // ------------------------------------------------ producer warp
    const uint64_t pol = ef ? evict_first_policy() : 0;
    const int64_t total = p.unit_hi;  // this launch's units: [unit_lo, unit_hi)
    int64_t u0 = p.unit_lo + blockIdx.x, ustep = gridDim.x, uend = total;
    if (p.blocked) {  // contiguous range: the CTA crosses few layer boundaries
      const int64_t per = (p.unit_hi - p.unit_lo + gridDim.x - 1) / gridDim.x;
      u0 = p.unit_lo + blockIdx.x * per;
      ustep = 1;
      uend = u0 + per < total ? u0 + per : total;
    }
    Pacer pacer;
    // unit u as (plane, index inside the plane), advanced by ustep without dividing
    const int64_t upp = p.units_per_plane;
    int64_t cur_plane = u0 / upp;
    int64_t cur_r = u0 - cur_plane * upp;
    const int64_t step_planes = ustep / upp, step_r = ustep - step_planes * upp;
    int it = 0;
    for (int64_t u = u0;; u += ustep, ++it) {
      const int st = it % S;
      if (it >= S) mbar_wait(&empty[st], ((it / S) & 1) ^ 1);
      if (u >= uend) {
        if (lane == 0) desc[st].nseg = -1;
        mbar_arrive(&full[st]);
        // every load of this CTA is issued: the next op on the stream may launch once all
        // CTAs got here (its CTAs then take SMs as ours exit and wait in pdl_wait) — never
        // earlier, so a paced op does not park the next op's CTAs on idle SMs
        pdl_launch_dependents();
        break;
      }
      int32_t plane;
      uint32_t bytes;
      const int nseg = decode_unit_at(p, cur_plane, static_cast<int32_t>(cur_r), desc[st].segs,
                                      desc[st].fdst, &plane, &bytes);
      cur_plane += step_planes;
      cur_r += step_r;
      if (cur_r >= upp) {
        cur_r -= upp;
        ++cur_plane;
      }
      __syncwarp();
      if (lane != 0) mbar_arrive(&full[st]);
      if (lane == 0) {
        pacer.wait(p.ns_per_byte, bytes);
        desc[st].nseg = nseg;
        desc[st].plane = plane;
        mbar_arrive_expect_tx(&full[st], bytes);
        uint8_t* sbuf = buf + static_cast<size_t>(st) * SB;
        for (int k = 0; k < nseg; ++k) {
          const Seg& g = desc[st].segs[k];
          bulk_load(sbuf + g.soff, g.src, g.len, &full[st], ef, pol);
        }
      }
      __syncwarp();
    }
  } else if (lane == 0) {  // ---------------------------------------- consumer thread
    const uint64_t pol = ef ? evict_first_policy() : 0;
    // stores allowed to be still reading their stage: half the ring (the other half is
    // the producer's load lookahead)
    const int lag = p.store_lag > 0 ? p.store_lag : (S / 2 > 0 ? S / 2 : 1);
    // Layer arrivals without draining the store pipeline: when unit `it` opens a later
    // layer, the stores of the layer just left are the bulk groups < it.  The arrival is
    // deferred until `lag` newer groups have been committed; then a full wait_group<lag>
    // (instead of this iteration's .read wait) makes exactly those groups complete.  A
    // second boundary while one is pending (< lag units per layer) resolves the first one
    // on the spot with a shallower wait.
    int32_t cur = -1;          // layer of the units being stored, and how many of them
    uint32_t cur_cnt = 0;
    int32_t pend = -1;         // pending arrival on layer `pend` (pend_cnt units) once the
    uint32_t pend_cnt = 0;     // groups < pend_it are done
    int pend_it = 0;
    for (int it = 0;; ++it) {
      const int st = it % S;
      mbar_wait(&full[st], (it / S) & 1);
      const int nseg = desc[st].nseg;
      if (nseg < 0) break;
      const int32_t layer = p.layer_lo + desc[st].plane / 2;
      if (cur >= 0 && layer != cur) {  // this CTA is done with layer `cur`
        if (pend >= 0) {
          bulk_wait_done_n(it - pend_it);  // the it - pend_it groups >= pend_it may stay pending
          fence_async_global();
          arrive_layer(p, pend, pend_cnt);
        }
        pend = cur;
        pend_cnt = cur_cnt;
        pend_it = it;
        cur_cnt = 0;
      }
      cur = layer;
      ++cur_cnt;
      const uint8_t* sbuf = buf + static_cast<size_t>(st) * SB;
      for (int k = 0; k < nseg; ++k) {
        const Seg& g = desc[st].segs[k];
        bulk_store(g.dst, sbuf + g.soff, g.len, ef, pol);
      }
      for (int f = 1; f < p.fan; ++f)  // read-once fan-out: the same staged bytes again
        for (int k = 0; k < nseg; ++k) {
          const Seg& g = desc[st].segs[k];
          bulk_store(desc[st].fdst[f - 1][k], sbuf + g.soff, g.len, ef, pol);
        }
      bulk_commit();
      if (pend >= 0 && it - pend_it + 1 >= lag) {
        bulk_wait_done_n(it - pend_it + 1);  // groups < pend_it complete (and <= it - lag read)
        fence_async_global();
        arrive_layer(p, pend, pend_cnt);
        pend = -1;
      } else {
        bulk_wait_read_n(lag);  // stores of units <= it - lag have read their stage
      }
      if (it >= lag) mbar_arrive(&empty[(it - lag) % S]);
    }
    bulk_wait_all();
    fence_async_global();
    if (pend >= 0) arrive_layer(p, pend, pend_cnt);
    if (cur >= 0) arrive_layer(p, cur, cur_cnt);
  }
}

// ------------------------------------------------------------------ K1: SIMT vectors

constexpr int kSimtThreads = 512;
constexpr int kSimtUnroll = 4;

__global__ void __launch_bounds__(kSimtThreads) simt_copy_kernel(const __grid_constant__ Params p) {
  __shared__ Seg segs[kMaxSegs];
  __shared__ int32_t s_nseg, s_plane;
  const int tid = threadIdx.x;
  const bool ef = p.evict_first != 0;
  const uint64_t pol = ef ? evict_first_policy() : 0;
  pdl_wait();
  if (blockIdx.x == 0 && tid == 32 && p.first_slice) publish_untouched_layers(p);  // not the decoding warp
  if (p.abort_word && *reinterpret_cast<const volatile int32_t*>(p.abort_word)) {
    if (blockIdx.x == 0 && tid == 0) publish_aborted(p);
    return;
  }
  int32_t cur = -1;  // layer of the units being copied, and how many of them
  uint32_t cur_cnt = 0;
  const int64_t total = p.unit_hi;  // this launch's units: [unit_lo, unit_hi)
  int64_t u0 = p.unit_lo + blockIdx.x, ustep = gridDim.x, uend = total;
  if (p.blocked) {
    const int64_t per = (p.unit_hi - p.unit_lo + gridDim.x - 1) / gridDim.x;
    u0 = p.unit_lo + blockIdx.x * per;
    ustep = 1;
    uend = u0 + per < total ? u0 + per : total;
  }
  Pacer pacer;
  for (int64_t u = u0; u < uend; u += ustep) {
    if (u + ustep >= uend) pdl_launch_dependents();  // this CTA's last unit (uniform)
    if (tid < 32) {
      int32_t plane;
      uint32_t bytes;
      const int n = decode_unit(p, u, segs, nullptr, &plane, &bytes);
      if (tid == 0) {
        pacer.wait(p.ns_per_byte, bytes);
        s_nseg = n;
        s_plane = plane;
      }
    }
    __syncthreads();
    const int32_t layer = p.layer_lo + s_plane / 2;
    if (cur >= 0 && layer != cur) {  // uniform: every thread of the CTA left layer `cur`
      if (tid == 0) arrive_layer(p, cur, cur_cnt);
      cur_cnt = 0;
    }
    cur = layer;
    ++cur_cnt;
    const int nseg = s_nseg;
    for (int k = 0; k < nseg; ++k) {
      const int4* s = reinterpret_cast<const int4*>(segs[k].src);
      int4* d = reinterpret_cast<int4*>(segs[k].dst);
      const int nv = static_cast<int>(segs[k].len >> 4);
      for (int v = tid; v < nv; v += kSimtUnroll * kSimtThreads) {
        int4 r[kSimtUnroll];
#pragma unroll
        for (int q = 0; q < kSimtUnroll; ++q) {
          const int vi = v + q * kSimtThreads;
          if (vi < nv) r[q] = ef ? ld_stream_ef(s + vi, pol) : ld_stream(s + vi);
        }
#pragma unroll
        for (int q = 0; q < kSimtUnroll; ++q) {
          const int vi = v + q * kSimtThreads;
          if (vi < nv) {
            if (ef)
              st_stream_ef(d + vi, r[q], pol);
            else
              st_stream(d + vi, r[q]);
          }
        }
      }
    }
    __syncthreads();  // all stores of this unit issued; segs may be overwritten
  }
  if (tid == 0 && cur >= 0) arrive_layer(p, cur, cur_cnt);
}

// ------------------------------------------------- copy-engine path: flag publication

__global__ void flag_bump_kernel(const __grid_constant__ Params p) {
  // the DMA copies before this kernel in stream order have completed; make that ordering
  // visible system-wide before the flags move
  fence_sys();
  for (int j = 0; j < p.n_items; ++j)
    for (int f = threadIdx.x; f < p.items[j].d_layers; f += blockDim.x)
      bump_flag(p.items[j].flags + f, p.items[j]);
}

// Copy-engine pacing: one thread (no SM resources worth mentioning, so a rate-limited DMA
// migration stays off the SMs).  The first launch of an op stamps the op's start time in
// *t0; every later launch sleeps until t0 + target_ns (the schedule of the bytes copied
// so far), so command overheads are absorbed and the average rate is exact.
__global__ void pace_kernel(unsigned long long* t0, uint64_t target_ns, int first) {
  if (first) {
    *t0 = globaltimer_ns();
    return;
  }
  const uint64_t until = *reinterpret_cast<volatile unsigned long long*>(t0) + target_ns;
  uint64_t now = globaltimer_ns();
  while (now < until) {
    const uint64_t d = until - now;
    __nanosleep(d > 1000000 ? 1000000u : static_cast<unsigned>(d));
    now = globaltimer_ns();
  }
}

// Step-aligned ops (wind_kv_migrate_stepped): the consumer's decode loop bumps its step
// counter at each step start; slices of a stepped op wait on it with cuStreamWaitValue32.
// A release reduction: the work before it on the stream is visible before the new count.
__global__ void step_signal_kernel(uint32_t* counter) {
  asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(counter) : "memory");
}

// -------------------------------------------------------- debug-pool device table check

__global__ void table_count_kernel(const int32_t* sbt, const int32_t* dbt, int32_t n,
                                   int32_t nb_src, int32_t nb_dst, uint32_t* dcnt,
                                   uint32_t* scnt, int32_t* err) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t s = sbt[i], d = dbt[i];
    if (s < 0 || s >= nb_src || d < 0 || d >= nb_dst) {
      atomicMax(reinterpret_cast<int*>(err), 4);  // 4 = BLOCK_RANGE (rank of precedence)
      continue;
    }
    atomicAdd(dcnt + d, 1u);
    atomicAdd(scnt + s, 1u);
  }
}

__global__ void table_judge_kernel(const int32_t* sbt, const int32_t* dbt, int32_t n,
                                   int32_t nb_src, int32_t nb_dst, int same_pool,
                                   const uint32_t* dcnt, const uint32_t* scnt, int32_t* err) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t s = sbt[i], d = dbt[i];
    if (s < 0 || s >= nb_src || d < 0 || d >= nb_dst) continue;
    if (dcnt[d] > 1) atomicMax(reinterpret_cast<int*>(err), 3);  // DUP_DST
    if (same_pool && scnt[d] > (s == d ? 1u : 0u)) atomicMax(reinterpret_cast<int*>(err), 2);  // ALIAS
  }
}

}  // namespace

size_t tma_smem_bytes(int stages, int stage_bytes) {
  return static_cast<size_t>(stages) * stage_bytes + static_cast<size_t>(stages) * sizeof(Desc) +
         2 * static_cast<size_t>(stages) * sizeof(uint64_t);
}

cudaError_t prepare_kernels(int device, size_t max_tma_smem) {
  (void)device;
  cudaError_t e = cudaFuncSetAttribute(tma_copy_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(max_tma_smem));
  if (e != cudaSuccess) return e;
  // Load every kernel now (pool creation): with CUDA's lazy module loading the first launch
  // of a kernel loads its code, which synchronises the whole device — an op must never do
  // that on the hot path.
  const void* fns[] = {reinterpret_cast<const void*>(simt_copy_kernel),
                       reinterpret_cast<const void*>(step_signal_kernel),
                       reinterpret_cast<const void*>(flag_bump_kernel),
                       reinterpret_cast<const void*>(pace_kernel),
                       reinterpret_cast<const void*>(table_count_kernel),
                       reinterpret_cast<const void*>(table_judge_kernel)};
  for (const void* f : fns) {
    cudaFuncAttributes a;
    if ((e = cudaFuncGetAttributes(&a, f)) != cudaSuccess) return e;
  }
  return cudaSuccess;
}

cudaError_t launch_copy(const Params& p, int kernel, int grid, cudaStream_t s, bool pdl) {
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.gridDim = dim3(static_cast<unsigned>(grid));
  cfg.stream = s;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  if (kernel == kTma) {
    cfg.blockDim = dim3(64);
    cfg.dynamicSmemBytes = tma_smem_bytes(p.stages, p.stage_bytes);
    return cudaLaunchKernelEx(&cfg, tma_copy_kernel, p);
  }
  cfg.blockDim = dim3(kSimtThreads);
  cfg.dynamicSmemBytes = 0;
  return cudaLaunchKernelEx(&cfg, simt_copy_kernel, p);
}

cudaError_t launch_pace(unsigned long long* t0, uint64_t target_ns, int first, cudaStream_t s) {
  pace_kernel<<<1, 1, 0, s>>>(t0, target_ns, first);
  return cudaGetLastError();
}

cudaError_t launch_step_signal(uint32_t* counter, cudaStream_t s) {
  step_signal_kernel<<<1, 1, 0, s>>>(counter);
  return cudaGetLastError();
}

cudaError_t launch_flag_bump(const Params& p, cudaStream_t s) {
  flag_bump_kernel<<<1, 128, 0, s>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_table_check(const int32_t* sbt, const int32_t* dbt, int32_t n,
                               int32_t nb_src, int32_t nb_dst, int same_pool,
                               uint32_t* scratch, int32_t nb_scratch, int32_t* err,
                               cudaStream_t s) {
  uint32_t* dcnt = scratch;
  uint32_t* scnt = scratch + nb_scratch;
  cudaError_t e = cudaMemsetAsync(scratch, 0, sizeof(uint32_t) * 2 * nb_scratch, s);
  if (e != cudaSuccess) return e;
  const int grid = n / 256 + 1 < 1024 ? n / 256 + 1 : 1024;
  table_count_kernel<<<grid, 256, 0, s>>>(sbt, dbt, n, nb_src, nb_dst, dcnt, scnt, err);
  table_judge_kernel<<<grid, 256, 0, s>>>(sbt, dbt, n, nb_src, nb_dst, same_pool, dcnt, scnt, err);
  return cudaGetLastError();
}

}  // namespace wkv
