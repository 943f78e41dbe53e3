/* wind_kv.h — C ABI of the B200-native paged KV-cache migration library.
 *
 * The library implements the data-parallel hot path under WindServe's stall-free
 * rescheduling and KV-swap reduction (Feng et al., ISCA '25; PAPER.md = the paper text,
 * "P:n" = its line n): a request's K/V blocks are gathered, layer by layer, from a source
 * block pool through its block table and scattered into slots of a destination pool under
 * a new block table — within one GPU, to another GPU over NVLink, or to / from pinned
 * host memory.
 *
 *   - KV kept in fixed-size blocks with a per-instance KV manager: §2.1, §3.1
 *   - prefill->decode KV transfer, overlapped with prefill: §2.2, §1
 *   - KV swap GPU<->CPU under memory pressure: §2.2, §5.2, §5.4
 *   - decode->prefill migration of long-context requests (Dynamic Rescheduling) while
 *     decoding continues (stall-free): §3.2.2, §3.3
 *   - layers run in sequential order, so KV can be handed over layer by layer: P:219
 *   - no allocation / implicit stream sync on the hot path: §4
 * Everything the paper leaves open (layout, aliasing, slot choice, ...) follows the
 * readings R1-R21 listed in DESIGN.md (= SURVEY.md §8(c) A1-A21).
 *
 * Conventions
 *   - Every function returns wind_status: 0 = OK, < 0 = error.  Nothing throws or aborts
 *     across the ABI.  wind_kv_last_error() returns detail text (thread-local).
 *   - Argument errors are detected synchronously, before anything is enqueued, in this
 *     precedence: INVALID_ARG > GEOMETRY > LAYER_RANGE > NO_PEER.
 *   - Ops are asynchronous on the given stream, never allocate and never synchronise the
 *     host; they are CUDA-graph capturable.  Asynchronous CUDA faults surface at
 *     the caller's next synchronisation, as with any CUDA call.
 *   - Each kernel op owns one per-device arrival-counter slot from enqueue until it has
 *     completed (a host-side event recorded after it).  An op takes its stream's previous slot
 *     (ops on one stream run in order, so any number may be queued on one stream), else a
 *     slot whose op is done: ops of at most 512 STREAMS may be pending on one device at
 *     once; an op on a 513th stream fails with WIND_ERR_UNSUPPORTED, nothing enqueued.  A
 *     pending op (e.g. a stepped migration waiting on decode steps) keeps its slot however
 *     many ops other streams run meanwhile.  Ops captured into a CUDA graph take one of
 *     512 separate graph slots round robin, fixed at capture: at most 512 captured ops may
 *     execute concurrently on one device, and a graph must not run concurrently with
 *     itself (two replays of one captured op would share its slot).
 *   - `cudaStream_t` parameters are passed as `void*` (0 = the legacy default stream) so
 *     the header needs no CUDA include.
 *   - The copy kernels use programmatic dependent launch: each waits for the previous
 *     kernel on its stream to complete before touching global memory, and signals
 *     programmatic completion once all its loads are issued.  Ordinary launches after an
 *     op are unaffected; a kernel YOU launch after an op with programmatic stream
 *     serialization must call cudaGridDependencySynchronize() before reading the op's
 *     destination (the standard PDL contract).  WIND_KV_PDL=0 in the environment turns it
 *     off.
 *   - WIND_KV_FORCE_SYS_SCOPE=1 in the environment (tests): every op publishes its layer
 *     flags at system scope, as peer destinations always do (wind_kv_route reports it).
 *     WIND_KV_FORCE_PEER_ROUTE=1 (tests): an op between a local pool and a pool imported
 *     from another process on the SAME GPU takes the PEER route (PEER tuning, system scope),
 *     so one-GPU runs exercise the multi-GPU path's choices.
 */
#ifndef WIND_KV_H
#define WIND_KV_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t wind_status;

enum {
  WIND_OK = 0,
  WIND_ERR_INVALID_ARG = -1,   /* null handle, n < 0, wrong stream device, misaligned */
  WIND_ERR_GEOMETRY = -2,      /* H, d, block_size or elem_bytes differ between pools */
  WIND_ERR_LAYER_RANGE = -3,   /* lo > hi, or [lo, hi) not inside both pools */
  WIND_ERR_BLOCK_RANGE = -4,   /* a table entry outside [0, n_blocks) */
  WIND_ERR_DUP_DST = -5,       /* two entries of dst_bt name the same slot */
  WIND_ERR_ALIAS = -6,         /* same pool: a destination slot is another entry's source */
  WIND_ERR_NO_PEER = -7,       /* pools on devices that cannot reach each other */
  WIND_ERR_CUDA = -8,          /* a CUDA runtime / driver call failed (see last_error) */
  WIND_ERR_OOM = -9,           /* allocation failed (pool create / import only) */
  WIND_ERR_UNSUPPORTED = -10,  /* geometry the kernels do not support (C % 16 != 0, ...) */
  WIND_ERR_DEVICE_CHECK = -11  /* debug pools: the device-side table check fired */
};

typedef enum { WIND_LOC_DEVICE = 0, WIND_LOC_HOST = 1 /* pinned, mapped, portable */ } wind_loc;

/* Pool flags. */
#define WIND_POOL_DEBUG 0x1u /* ops into/out of this pool also run a device table check */
#define WIND_POOL_NO_STAGING 0x2u /* host pools: no copy-engine staging (saves 3 x max(32 MiB,
                                     2 L C) of device memory; swaps use the SM kernels) */

/* Pool descriptor.  Layout (reading R2): [L][2][NB][H][bs][d] elements of
 * elem_bytes, layer-major with K/V planes; chunk (layer l, kv, block b) is the C =
 * H*bs*d*elem_bytes contiguous bytes at offset (((l - first_layer)*2 + kv)*NB + b)*C, and
 * each head tile (H index h) is the contiguous bs*d*elem_bytes bytes inside it (HND).
 * Layers are GLOBAL ids [first_layer, first_layer + n_layers) (PP stages).
 * Requirements: every extent >= 1, n_layers <= WIND_KV_MAX_LAYERS, elem_bytes in {1,2,4}
 * (fp8 / fp16|bf16 / fp32 payloads are raw bytes, never interpreted: reading R13),
 * C % 16 == 0.  For a host pool, `device` names the GPU whose copy engines serve it: pool
 * creation also allocates there the staging of the staged swap path (3 buffers of
 * max(32 MiB, 2 * n_layers * C) bytes, a side stream, events; best effort — without a GPU
 * `device` the pool simply has no staging and swaps use the SM kernels). */
typedef struct {
  int32_t first_layer, n_layers;
  int32_t n_kv_heads, head_dim, block_size, elem_bytes;
  int32_t n_blocks;
  int32_t loc;    /* wind_loc */
  int32_t device; /* CUDA ordinal of a device pool */
  uint32_t flags; /* WIND_POOL_* */
} wind_kv_pool_desc;

#define WIND_KV_MAX_LAYERS 1024

typedef struct wind_kv_pool wind_kv_pool; /* opaque */

#define WIND_KV_IPC_HANDLE_BYTES 512
typedef struct {
  unsigned char bytes[WIND_KV_IPC_HANDLE_BYTES];
} wind_kv_ipc_handle;

/* ------------------------------------------------------------------- pools (§8(a) A1) */

/* Creates a pool.  external_base == NULL: the library allocates the data (cudaMalloc on
 * desc->device, or cudaHostAlloc(Mapped|Portable) for host pools) and frees it on
 * destroy.  external_base != NULL: the caller's memory (device memory on desc->device, or
 * mapped pinned host memory for host pools; >= pool bytes; 16-B aligned, else
 * INVALID_ARG) is used and never freed.  The pool's layer_done flags (one uint32 per
 * layer, zeroed) are always library-allocated: device memory for device pools, mapped
 * pinned memory for host pools.  Contents of library-allocated data are undefined.
 * Errors: INVALID_ARG, UNSUPPORTED, OOM, CUDA.  *out is set only on success. */
wind_status wind_kv_pool_create(const wind_kv_pool_desc* desc, void* external_base,
                                wind_kv_pool** out);

/* Destroys a pool handle.  Frees only library-allocated memory; imported pools are only
 * unmapped.  The caller guarantees no op using the pool is still in flight.  NULL is OK. */
wind_status wind_kv_pool_destroy(wind_kv_pool* pool);

/* Base address (device-accessible; for host pools the mapped pointer, valid on host and
 * device under UVA), size in bytes, and descriptor (for imported pools: the owner's
 * descriptor with `device` = the importing device).  Any out pointer may be NULL. */
wind_status wind_kv_pool_info(const wind_kv_pool* pool, void** base, size_t* bytes,
                              wind_kv_pool_desc* desc);

/* Address of the pool's layer_done[n_layers] uint32 flags (device-accessible), for
 * consumers that poll in their own kernels.  Flag i belongs to global layer
 * first_layer + i. */
wind_status wind_kv_pool_flags(const wind_kv_pool* pool, uint32_t** layer_done);

/* Exports a DEVICE pool (data + layer flags) for another process (CUDA IPC).  The handle
 * is plain bytes: send it over any channel (e.g. a torch process group).  Host pools:
 * UNSUPPORTED. */
wind_status wind_kv_pool_export(const wind_kv_pool* pool, wind_kv_ipc_handle* out);

/* Imports an exported pool into this process, mapped for `local_device` (peer access is
 * enabled from local_device to the owner's device when they differ; NO_PEER if it cannot
 * be).  The imported pool can be the destination (push, P:120 hand-off) or the source
 * (pull) of migrate.  Importing in the exporting process itself is UNSUPPORTED (CUDA IPC
 * restriction). */
wind_status wind_kv_pool_import(const wind_kv_ipc_handle* handle, int32_t local_device,
                                wind_kv_pool** out);

/* ------------------------------------------------------------ data movement (A2-A7) */

/* migrate (A2-A5): for every global layer l in [layer_lo, layer_hi), kv in {K, V} and
 * i in [0, n_blocks):   dst[l][kv][dst_bt[i]] := src_before[l][kv][src_bt[i]]
 * (C raw bytes).  All other bytes of dst are unchanged (R20).
 *   src_bt, dst_bt: BORROWED int32[n_blocks], device-accessible from the executing
 *     device (device memory or mapped pinned host memory); they must stay valid and
 *     unmodified until the op completes on `stream` (the cudaMemcpyAsync contract).
 *   Table contract (R4, R5): entries in range, dst_bt pairwise distinct, and if src and
 *     dst are the same pool, dst_bt[i] == src_bt[j] only for i == j.  Duplicate sources
 *     (fan-out) are allowed.  Release builds do not check table content on the hot path:
 *     an entry out of range is UNDEFINED BEHAVIOUR (the kernels read / write base + entry
 *     * C, like cudaMemcpyAsync with a bad pointer); duplicate or aliasing destinations
 *     leave the affected chunks of dst undefined.  Check tables with wind_kv_validate
 *     (host) or create the pools with WIND_POOL_DEBUG (a device-side check before every
 *     op; a violation aborts the op and is reported by wind_kv_check_device_error).  (A
 *     kernel-side range guard that skipped such entries was measured at ~1 % of the C2
 *     headline and not kept.)
 *   Executing device: src's device if src is a device pool (its own, or the device an
 *     imported src was mapped into), else dst's.  `stream` must belong to it
 *     (INVALID_ARG otherwise).  Cross-device ops push over NVLink peer stores (or pull
 *     when src is the remote one); host pools move over PCIe (mapped memory by default,
 *     staged copy engines on request: see wind_kv_swap_out).
 *   Argument errors, nothing enqueued, in this order: INVALID_ARG (NULL pool, n_blocks < 0,
 *     NULL table with n_blocks > 0, stream of another device, imported pool mapped for
 *     another device), then GEOMETRY, then LAYER_RANGE, then NO_PEER / UNSUPPORTED
 *     (unreachable pools, host -> host).
 *   Layer flags (A5): every call with n_blocks > 0 and lo < hi takes one ticket on dst
 *     (see wind_kv_layer_ticket) and, as each layer's bytes become visible, adds 1 to
 *     dst's layer_done flag of that layer with release semantics: at GPU scope when src
 *     and dst are device pools on the executing GPU (every reader of such a pool — the
 *     consumer stream's wait, the kernels it releases, another process's kernels on that
 *     GPU — goes through its L2; a system-scope fence per layer cost ~1.7 us),
 *     at system scope when dst is a peer or host pool.  An agent on another device that
 *     polls a LOCAL op's flags must order its reads through CUDA events / streams; flags of
 *     dst layers outside
 *     [lo, hi) are incremented at the start of the op, so "flag >= ticket" is meaningful
 *     for every layer.  Layers are processed in ascending order: every CTA walks
 *     its work units layer-major, so on ops with at least as many work units per (layer,
 *     K|V) plane as CTAs the flags complete layer by layer while the op runs; smaller ops
 *     give each CTA a contiguous unit range and their layers complete near the op's end,
 *     in no guaranteed order (a flag still never moves before its layer's bytes).
 *   n_blocks == 0 or layer_lo == layer_hi: WIND_OK, nothing enqueued, no ticket (R19). */
wind_status wind_kv_migrate(const wind_kv_pool* src, const int32_t* src_bt, wind_kv_pool* dst,
                            const int32_t* dst_bt, int32_t n_blocks, int32_t layer_lo,
                            int32_t layer_hi, void* stream);

/* swap_out / swap_in (A6): migrate over all layers of the device pool with a HOST pool as
 * destination / source.  The host pool must cover the device pool's
 * layers.  Executes on the device pool's GPU.  Two mechanisms:
 *   - default (HOST path, kernel 0 / 1 / 2): SM / TMA stores to and loads from mapped pinned
 *     memory over PCIe, tables borrowed and read when the op executes (the migrate
 *     contract), per-layer flags as in migrate.  Grids are sized by the bytes they keep in
 *     flight (wind_kv_tuning.max_ctas).
 *   - staged (kernel 4, OPT-IN via wind_kv_set_tuning(WIND_PATH_HOST) or a per-op
 *     wind_kv_migrate_ex override; UNSUPPORTED when it does not apply): the HOST-side table
 *     (host_bt) must be host-readable (e.g. pinned host memory) and the host pool must have
 *     staging on the executing GPU.  A TMA kernel gathers (scatters) the device blocks
 *     through the device table into a contiguous device staging buffer at HBM rate, and the
 *     copy engines move each chunk over PCIe, one cudaMemcpy2DAsync per run of adjacent host
 *     slots, triple-buffered on side streams (fork / join with events).  Chunks are
 *     layer-major and dst's layer flags move as each layer's last chunk lands.  CONTRACT
 *     DIFFERENCE: host_bt is READ ON THE CPU AT ENQUEUE (entries out of range: BLOCK_RANGE,
 *     nothing enqueued), so it must hold its final values when the call is made; inside a
 *     CUDA graph capture its contents are baked into the graph (a replay moves the slots
 *     the table held at capture).  Staged ops on one host pool serialise on its buffers
 *     automatically outside graph capture (inside a capture, order them yourself); ops on
 *     one host pool are enqueued under the pool's lock, so several host threads may issue
 *     them.
 * A host pool's layer flags live in mapped host memory and are updated without PCIe
 * atomics, so ops INTO one host pool must not overlap in time.  The library orders them:
 * an op into a host pool enqueued on another stream than the pool's previous op first
 * makes its stream wait (cudaStreamWaitEvent, nothing blocks the host) for that op; ops on
 * one stream are ordered anyway.  Under graph capture this is not done: order captured
 * ops into one host pool yourself.  The host observes swap_out progress by reading the
 * flags. */
wind_status wind_kv_swap_out(const wind_kv_pool* dev, const int32_t* dev_bt,
                             wind_kv_pool* host, const int32_t* host_bt, int32_t n_blocks,
                             void* stream);
wind_status wind_kv_swap_in(const wind_kv_pool* host, const int32_t* host_bt,
                            wind_kv_pool* dev, const int32_t* dev_bt, int32_t n_blocks,
                            void* stream);

/* compact (A7): migrate(pool, src_bt, pool, dst_bt, n, l0, l0 + L) — in-place moves of
 * live blocks into holes; tables typically from wind_kv_plan_compact. */
wind_status wind_kv_compact(wind_kv_pool* pool, const int32_t* src_bt, const int32_t* dst_bt,
                            int32_t n_blocks, void* stream);

/* Head-range migrate (NEXT-3, TP reshard): under tensor parallelism KV is sharded by head
 * (Table 3: every placement is TP-2) and prefill / decode placements may differ
 * ([TP-2, TP-1], Fig. 3).  For l in [lo, hi), kv, i, h in [0, n_heads):
 *   dst[l][kv][dst_bt[i]][dst_head_lo + h] := src_before[l][kv][src_bt[i]][src_head_lo + h]
 * (each head tile is bs*d*e_b contiguous bytes; H may differ between the pools).
 * Errors: INVALID_ARG (n_heads < 1, negative offsets) > GEOMETRY (d / bs / e_b differ, or a
 * head range leaves its pool) > LAYER_RANGE; UNSUPPORTED if bs*d*e_b % 16 != 0.  Same
 * execution, table contract, tickets and flags as wind_kv_migrate. */
wind_status wind_kv_migrate_heads(const wind_kv_pool* src, const int32_t* src_bt, wind_kv_pool* dst,
                                  const int32_t* dst_bt, int32_t n_blocks, int32_t layer_lo,
                                  int32_t layer_hi, int32_t src_head_lo, int32_t dst_head_lo,
                                  int32_t n_heads, void* stream);

/* One entry of a batched migrate: several (dst pool, tables) pairs from ONE source pool,
 * executed by one persistent launch (all-to-all rebalancing, A8: a GPU pushing to up to
 * 7 peers at once).  Each entry takes its own ticket on its dst. */
typedef struct {
  wind_kv_pool* dst;
  const int32_t* src_bt;
  const int32_t* dst_bt;
  int32_t n_blocks;
} wind_kv_migrate_item;

#define WIND_KV_MAX_BATCH 16

/* Batched migrate (A8): items[0..n_items) all read from `src`, layers [lo, hi), in one
 * launch on `stream`.  Destination pools must be pairwise distinct objects with
 * disjoint memory (the planner guarantees it).  n_items <= WIND_KV_MAX_BATCH.
 * Read-once fan-out (KV backups): when 2-4 items pass the SAME src_bt
 * pointer with the same n_blocks and the op runs on the TMA kernel, each source unit is
 * staged once and stored to every destination (DRAM traffic (1 + k) x payload instead of
 * 2k x); results are identical to the per-item path. */
wind_status wind_kv_migrate_batch(const wind_kv_pool* src, const wind_kv_migrate_item* items,
                                  int32_t n_items, int32_t layer_lo, int32_t layer_hi,
                                  void* stream);

/* Route query (diagnostics, tests): the device an op from src to dst executes on, its
 * tuning path (WIND_PATH_INTRA: both pools on one physical GPU; WIND_PATH_PEER: device pools
 * on different GPUs, NVLink peer stores / loads; WIND_PATH_HOST: one side is a host pool)
 * and whether its layer flags are published at system scope (1) or GPU scope (0).  Same
 * reachability checks as an op (NO_PEER, UNSUPPORTED for host -> host); enables peer access
 * like an op would.  Any out pointer may be NULL. */
wind_status wind_kv_route(const wind_kv_pool* src, const wind_kv_pool* dst, int32_t* exec_device,
                          int32_t* path, int32_t* sys_scope);

/* Step-aligned migrate (interference, S§8(d); DESIGN.md §6 "burst instead of trickle"):
 * the op of wind_kv_migrate, cut into slices of about `bytes_per_step` payload bytes (work
 * units in layer-ascending order); slice k waits on `stream` until *step_counter >=
 * first_step + k (wrap-safe, cuStreamWaitValue32 GEQ) and then runs at full rate on half
 * the grid.  The consumer's decode loop calls wind_kv_step_signal(step_counter, its
 * stream) at the start of every decode step, so each slice overlaps the beginning of one
 * decode step instead of trickling through all of them (next to an HBM-saturating decode
 * step: ~1.4 % at 50 GB/s and ~4.5 % at 150 GB/s average, against 4-5 % / 7-23 % for rate
 * limits).  `first_step` is the counter value of the step that releases slice 0 (the caller
 * knows its step count; inside a CUDA graph the waits are constants of the graph).
 * Results, tickets and layer flags are those of wind_kv_migrate (one op: a layer is
 * published when its last slice has landed).  step_counter: device-accessible uint32,
 * 4-byte aligned, owned by the caller.  Errors: as wind_kv_migrate, plus INVALID_ARG (NULL
 * or misaligned counter, bytes_per_step == 0) and UNSUPPORTED (host pools, debug pools,
 * copy-engine kernels).  The op never completes if the consumer stops signalling. */
wind_status wind_kv_migrate_stepped(const wind_kv_pool* src, const int32_t* src_bt, wind_kv_pool* dst,
                                    const int32_t* dst_bt, int32_t n_blocks, int32_t layer_lo,
                                    int32_t layer_hi, const uint32_t* step_counter, uint32_t first_step,
                                    uint64_t bytes_per_step, void* stream);

/* Adds 1 to *step_counter on `stream` (device side, release at GPU scope, in stream order):
 * the consumer's "a decode step starts here" for wind_kv_migrate_stepped. */
wind_status wind_kv_step_signal(uint32_t* step_counter, void* stream);

/* ------------------------------------------------------------- layer flags (A5) */

/* Number of ops this process has enqueued into `dst` so far (the ticket of the latest). */
wind_status wind_kv_layer_ticket(const wind_kv_pool* dst, uint32_t* ticket);

/* Makes `consumer` wait (device-side, no host sync) until dst's layer_done for global
 * `layer` reaches `ticket` (wrap-safe >=), i.e. until that many ops have landed that
 * layer.  Uses cuStreamWaitValue32(GEQ) on the flag, local to dst.  When ops into one
 * pool are issued on one stream, flag >= t means ops 1..t are complete for that layer.
 * Under CUDA graph capture the ticket is a constant of the graph: every replay waits for
 * the capture-time count, which the first replay's ops already reach — so a graph that
 * contains both the ops and their waits orders them correctly on its first replay only;
 * for repeated replays, wait outside the graph (or re-capture). */
wind_status wind_kv_layer_wait(const wind_kv_pool* dst, int32_t layer, uint32_t ticket,
                               void* consumer);

/* Asynchronous copy of all n_layers layer_done flags into caller memory `out` (pinned
 * host or device memory, n_layers uint32) on `stream` (a stream of the pool's local device;
 * for imported pools the flags are read over the peer mapping).  No host sync. */
wind_status wind_kv_read_flags(const wind_kv_pool* pool, uint32_t* out, void* stream);

/* Host read of layer_done[layer] (synchronous; tests and diagnostics). */
wind_status wind_kv_layer_count(const wind_kv_pool* dst, int32_t layer, uint32_t* value);

/* --------------------------------------------------------------- host-side logic */

/* Checks an op completely on HOST copies of the tables, O(n): the argument checks of
 * migrate, then BLOCK_RANGE > DUP_DST > ALIAS, each over the whole table (R4, R5). */
wind_status wind_kv_validate(const wind_kv_pool* src, const int32_t* src_bt_host,
                             const wind_kv_pool* dst, const int32_t* dst_bt_host, int32_t n,
                             int32_t layer_lo, int32_t layer_hi);

/* Compaction plan (A7, two-finger): live[n_slots] (0/1).  With n_live = sum(live):
 * holes = ascending b < n_live with !live[b]; movers = ascending b >= n_live with
 * live[b]; pair k moves movers[k] -> holes[k].  Writes n_moves entries to src_bt/dst_bt
 * (caller buffers of n_slots entries).  The pairs satisfy the same-pool table contract. */
wind_status wind_kv_plan_compact(const uint8_t* live, int32_t n_slots, int32_t* src_bt,
                                 int32_t* dst_bt, int32_t* n_moves);

/* Rebalance plan (A8, greedy; not in the paper — nearest P:219-227):
 * target = ceil(sum blocks / G); repeat { src = most loaded GPU, dst = least loaded
 * (lowest id on ties); stop if load[src] <= target; move the longest request of src that
 * keeps dst <= target (lowest id on ties; longest-first per P:227); stop if none }.
 * out_gpu[r] = final GPU of request r. */
wind_status wind_kv_plan_rebalance(int32_t n_gpus, int32_t n_requests, const int32_t* req_gpu,
                                   const int32_t* req_blocks, int32_t* out_gpu,
                                   int32_t* n_moves);

/* Debug pools: synchronises the pool's device and returns DEVICE_CHECK if a device-side
 * table check recorded an error (then clears it), else OK. */
wind_status wind_kv_check_device_error(const wind_kv_pool* pool);

/* ------------------------------------------------------------------ tuning & misc */

/* Kernel selection and launch shape, per path.  Defaults are the measured best on B200
 * (DESIGN.md §Kernels).  kernel: 3 = copy engines (DMA, zero SMs: the low-interference
 * background mode; needs host-readable block tables; one cudaMemcpy2DAsync per run of
 * adjacent blocks; flags published once after all layers; rate_mbps paces it with
 * 1-thread sleep kernels between copies — those hold the stream's hardware queue, so work
 * of another stream that CUDA maps onto the same queue waits behind them: raise
 * CUDA_DEVICE_MAX_CONNECTIONS (e.g. 32) and keep few streams; the TMA / SIMT kernels pace
 * inside the kernel and never hold a queue),
 * 4 = staged copy engines (HOST path only, opt-in: see wind_kv_swap_out; UNSUPPORTED when
 * it does not apply), 0 = auto (INTRA: TMA; PEER: SIMT; HOST: TMA on mapped pinned memory),
 * 1 = TMA bulk staged copy, 2 = SIMT 16-B vector copy.
 * ctas_per_sm, stage_bytes (TMA stage / SIMT unit bytes, multiple of 16), stages (TMA ring
 * depth); 0 keeps the current value. */
typedef enum { WIND_PATH_INTRA = 0, WIND_PATH_PEER = 1, WIND_PATH_HOST = 2 } wind_path;
typedef struct {
  int32_t kernel;
  int32_t ctas_per_sm;
  int32_t stage_bytes;
  int32_t stages;
  int32_t max_ctas; /* cap on the grid (e.g. to leave SMs to a decode stream); 0 = none,
                       except on the HOST path where 0 = per-direction defaults: SM kernel
                       into host memory with ~384 KiB of stores in flight (2-3 CTAs; more
                       back PCIe writes up into the GPU's memory system: 1.5 MiB in flight
                       slowed a co-running decode kernel by 73 %, 384 KiB by 2 %, same
                       52 GB/s), 8 CTAs from host memory; staged path: hidden gather /
                       scatter chunks with ~768 KiB in flight (4-6 CTAs).
                       PEER path: the same backpressure is expected when SM stores outrun
                       NVLink; for pushes next to latency-sensitive work on the SOURCE GPU,
                       cap the CTAs (or rate_mbps) so the link is not oversubscribed
                       (not measurable with one GPU per round-1 call) */
  int32_t evict_first; /* 1 = L2 evict-first policy on the copy's loads and stores */
  int32_t store_lag;   /* TMA: stores allowed in flight per CTA (0 = stages / 2) */
  int32_t rate_mbps;   /* payload rate limit of one op in MB/s (0 = unlimited): bounds the
                          HBM / link share a migration takes from co-running decode
                          (S§8(d) interference).  INTRA / PEER ops with max_ctas == 0 are
                          BURST-paced: slices of the op (2 ms of rate budget each) run on
                          half the grid at full rate, each followed by a 1-thread pace
                          kernel that holds the stream until the schedule allows the next,
                          so no copy CTA stays resident between bursts (1 + 2 x slices
                          launches; flags, tickets and results are one op's).  With
                          max_ctas > 0, and on the HOST path, the grid's CTAs pace
                          themselves with %globaltimer (one launch).  Either way the op ends
                          when its rate schedule says.  For background moves next to a
                          decode loop, one full-rate op per decode step is cheaper still
                          (DESIGN.md §6). */
} wind_kv_tuning;

wind_status wind_kv_set_tuning(int32_t path, const wind_kv_tuning* t);

/* wind_kv_migrate with a per-op tuning override (NULL = the path's current tuning): e.g.
 * the early stages of a stall-free migration on the copy engines with a rate budget and
 * its final stage on the TMA kernel at full rate.  Every field of the override is taken
 * literally (no "0 keeps" rule) and validated like set_tuning; kernel 0 = auto. */
wind_status wind_kv_migrate_ex(const wind_kv_pool* src, const int32_t* src_bt, wind_kv_pool* dst,
                               const int32_t* dst_bt, int32_t n_blocks, int32_t layer_lo,
                               int32_t layer_hi, const wind_kv_tuning* tuning, void* stream);
wind_status wind_kv_get_tuning(int32_t path, wind_kv_tuning* t);

/* SM partition (S§7 step 10, interference): two green contexts on `device` with disjoint
 * SM sets — one of at least `min_sms_migration` SMs (rounded up to the architecture's
 * granularity: 8 on sm_90+) for migrations, one with the remaining SMs for the co-running
 * prefill / decode work — and one stream in each (cudaStream_t; migration stream at low
 * priority, compute stream at high priority).  An op enqueued on the migration stream caps
 * its grid at that partition's SMs (x ctas_per_sm), and the compute stream's kernels never
 * share an SM (register file, shared memory, issue slots) with a migration CTA; they still
 * share HBM / L2 bandwidth.  Errors: INVALID_ARG (NULL out, bad device, min < 1),
 * UNSUPPORTED (no green-context support in the driver), CUDA.  The caller destroys the
 * partition after the work on both streams has completed. */
typedef struct {
  void* migration_stream;
  void* compute_stream;
  int32_t sms_migration;
  int32_t sms_compute;
  void* _internal[2];  /* the two green contexts */
} wind_kv_sm_partition;

wind_status wind_kv_partition_sms(int32_t device, int32_t min_sms_migration, wind_kv_sm_partition* out);
wind_status wind_kv_partition_destroy(wind_kv_sm_partition* part);

/* Number of kernels this process has launched through the library (all ops). */
uint64_t wind_kv_launch_count(void);

const char* wind_kv_status_string(wind_status s);
const char* wind_kv_last_error(void);
const char* wind_kv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* WIND_KV_H */
