// wind_kv_internal.h — internal structures shared by the host side (wind_kv.cpp) and the
// kernels (wind_kv_kernels.cu).  Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/wind_kv.h"

namespace wkv {

// Per-op, per-layer CTA-arrival counters on each executing device (A5): an op owns one slot
// of WIND_KV_MAX_LAYERS counters; the arrival completing a layer's units resets its counter.
// Eager ops take slots [0, kEagerSlots) (wind_kv.cpp take_slot): the slot of their stream's
// previous op (stream order keeps the two apart), else a slot whose last op has completed
// (a host event recorded after every eager op; no device-side bookkeeping).  So a
// long-pending op (a stepped migration waiting on decode steps, an op queued behind a
// layer_wait) keeps its slot however many ops other streams run meanwhile.  Ops captured
// into a CUDA graph take slots [kEagerSlots, kCounterSlots) round robin.
constexpr int kEagerSlots = 512;    // streams with ops in flight at once, per device
constexpr int kGraphSlots = 512;    // captured ops executing concurrently, per device
constexpr int kCounterSlots = kEagerSlots + kGraphSlots;  // 4 MiB of counters per device
constexpr int kMaxSegs = 32;  // segments (runs) per work unit = one warp's table window
constexpr int kMaxFan = 4;    // destinations of a read-once fan-out (TMA kernel)
constexpr int kCtaMBps = 30000;  // payload MB/s one copy CTA sustains with headroom (~38 measured)

// One destination of a (possibly batched) migrate launch.
struct Item {
  const int32_t* sbt;
  const int32_t* dbt;
  uint8_t* dst_plane0;     // dst chunk (layer lo, K, block 0) + head offset
  int64_t d_plane_stride;  // NB_dst * C_dst
  int64_t d_chunk;         // C_dst: block stride inside a dst plane
  int32_t coalesce;        // runs of adjacent blocks are contiguous on both sides
  uint32_t* flags;         // dst layer_done[0 .. d_layers)
  int32_t d_flag_lo;       // index of global layer lo in flags
  int32_t d_layers;        // dst n_layers (for the out-of-range increments)
  int32_t n;               // table entries
  int32_t units;           // work units per (layer, kv) plane for this item
  int32_t unit_base;       // prefix of `units` over previous items
  int32_t host_flags;      // flags live in mapped host memory: bump by plain RMW, not red.sys
  int32_t sys_scope;       // data or flags leave this GPU (peer / host pool): publish with
                           // system-scope fences; else GPU scope (a .sys fence costs ~1 us
                           // and stalls the copy stream, S DESIGN §6 publication cost)
};

struct Params {
  const uint8_t* src_plane0;  // src chunk (layer lo, K, block 0) + head offset
  int64_t s_plane_stride;     // NB_src * C_src
  int64_t s_chunk;            // C_src: block stride inside a src plane
  int64_t copy;               // bytes copied per (layer, kv, block): C, or n_heads * tile
  int64_t units_per_plane;    // sum of items' units
  int64_t total_units;        // planes * units_per_plane
  int64_t unit_lo, unit_hi;   // the units THIS launch moves (a burst-paced op launches
                              // slices of [0, total_units) on one counter slot)
  int32_t first_slice;        // 1: this launch also bumps the untouched layers' flags
  uint32_t* counters;         // this op's counter slot, [hi - lo]
  const int32_t* abort_word;  // debug pools: skip the copy if the device check fired
  int32_t layer_lo, n_layers; // global lo, hi - lo
  int32_t group;              // table entries per unit (>= 1; > 1 only when C < unit)
  int32_t parts;              // units per chunk (> 1 only when C > unit)
  int32_t part_bytes;         // bytes of a part (multiple of 16)
  int32_t n_items;
  int32_t evict_first;
  int32_t store_lag;          // TMA consumer: units whose stores may still read smem
  float ns_per_byte;          // per-CTA pacing (rate limit): 0 = unlimited
  int32_t stages;             // TMA ring depth
  int32_t stage_bytes;        // TMA stage size
  int32_t sys_scope;          // any item has sys_scope
  int32_t blocked;            // 1: CTA c takes the contiguous unit range [c*per, (c+1)*per)
                              // (small ops: fewer layer crossings per CTA); 0: grid-stride
  int32_t fan;                // > 1: read-once fan-out — every item shares items[0]'s source
                              // table and units; each staged unit is stored to all `fan`
                              // destinations (TMA kernel only; 1 otherwise)
  Item items[WIND_KV_MAX_BATCH];
};

enum Kernel { kAuto = 0, kTma = 1, kSimt = 2, kCopyEngine = 3, kStaged = 4 };

// Copy-engine path: after the DMA copies of an op (stream-ordered), one tiny kernel adds 1
// to every layer flag of every item (release, system scope).
cudaError_t launch_flag_bump(const Params& p, cudaStream_t s);
// Copy-engine rate limit: a 1-thread kernel; `first` stamps the op start in *t0, later
// launches sleep until *t0 + target_ns.
cudaError_t launch_pace(unsigned long long* t0, uint64_t target_ns, int first, cudaStream_t s);

// wind_kv_step_signal: +1 on a consumer's step counter (release, GPU scope), in stream order.
cudaError_t launch_step_signal(uint32_t* counter, cudaStream_t s);

// Launchers (wind_kv_kernels.cu).  Return cudaGetLastError() after the launch.
// pdl: launch with programmatic stream serialization (the kernel's prologue may overlap the
// previous kernel on the stream; it waits for it before touching global memory).
cudaError_t launch_copy(const Params& p, int kernel, int grid, cudaStream_t s, bool pdl);
size_t tma_smem_bytes(int stages, int stage_bytes);
cudaError_t prepare_kernels(int device, size_t max_tma_smem);

// Debug-pool device table check (wind_kv_kernels.cu): records error codes in *err.
cudaError_t launch_table_check(const int32_t* sbt, const int32_t* dbt, int32_t n,
                               int32_t nb_src, int32_t nb_dst, int same_pool,
                               uint32_t* scratch /* 2*max(nb) */, int32_t nb_scratch,
                               int32_t* err, cudaStream_t s);

}  // namespace wkv
