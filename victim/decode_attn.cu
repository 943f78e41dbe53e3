// decode_attn.cu — BENCH HARNESS ONLY: the co-running decode-attention "victim" stream
// used to measure how much a migration slows decoding (S§8(d) "Interference",
// BJ:north_star "<5% slowdown of a co-running decode stream").  Not part of the product
// library and not on the migration path.
//
// Paged decode attention for one layer over a wind_kv pool (PagedAttention blocks,
// PAPER.md P:110; decode reads 4*SUM(L)*H bytes of KV per layer):
//   o[b][hq] = softmax(q[b][hq] . K[b][hkv]^T / sqrt(d)) V[b][hkv],  hkv = hq / (Hq/Hkv)
// K and V of layer l are the pool planes [NB][Hkv][bs][d] (HND), fp16; tables int32
// [B][max_blocks]; fp32 accumulation; split-K over blocks (flash-decoding style): kernel 1
// writes per-split (max, sum, acc[d]) partials, kernel 2 merges them.
// Layout assumptions: d == 128 (one warp lane holds 4 dims), bs == 16 (BJ:configs).
#include <cuda_fp16.h>
#include <stdint.h>

namespace {

constexpr int kD = 128;
constexpr int kWarps = 4;
constexpr int kBs = 16;

struct Partial {
  float m, s;
};

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// grid: (B * Hq, splits); block: kWarps warps.  Each warp walks blocks of its split
// round-robin, keeps an online softmax over its tokens, then the CTA merges its warps.
__global__ void __launch_bounds__(kWarps * 32) decode_split_kernel(
    const __half* __restrict__ q, const uint8_t* __restrict__ k_plane,
    const uint8_t* __restrict__ v_plane, const int32_t* __restrict__ bt, const int32_t* __restrict__ ctx,
    int max_blocks, int hq, int hkv, int bs, int blocks_per_split, float scale,
    float* __restrict__ part_acc, Partial* __restrict__ part_ms) {
  const int bh = blockIdx.x;
  const int b = bh / hq, h = bh % hq;
  const int hk = h / (hq / hkv);
  const int split = blockIdx.y, n_split = gridDim.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int len = ctx[b];
  const int nblk = (len + bs - 1) / bs;
  const int blk0 = split * blocks_per_split;
  const int blk1 = min(nblk, blk0 + blocks_per_split);
  const size_t tile = static_cast<size_t>(bs) * kD * sizeof(__half);  // one head tile
  const size_t chunk = static_cast<size_t>(hkv) * tile;               // one block chunk

  const __half2* qh = reinterpret_cast<const __half2*>(q + (static_cast<size_t>(b) * hq + h) * kD) + lane * 2;
  const float2 q01 = __half22float2(qh[0]);
  const float2 q23 = __half22float2(qh[1]);
  float m = -INFINITY, s = 0.f, a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;

  for (int blk = blk0 + warp; blk < blk1; blk += kWarps) {
    const int slot = bt[static_cast<size_t>(b) * max_blocks + blk];
    const uint8_t* kt = k_plane + slot * chunk + hk * tile;
    const uint8_t* vt = v_plane + slot * chunk + hk * tile;
    const int ntok = min(bs, len - blk * bs);
    uint2 kr[kBs], vr[kBs];
#pragma unroll
    for (int t = 0; t < kBs; ++t)
      if (t < ntok) kr[t] = *reinterpret_cast<const uint2*>(kt + t * kD * 2 + lane * 8);
#pragma unroll
    for (int t = 0; t < kBs; ++t)
      if (t < ntok) vr[t] = *reinterpret_cast<const uint2*>(vt + t * kD * 2 + lane * 8);
#pragma unroll
    for (int t = 0; t < kBs; ++t) {
      if (t >= ntok) break;
      const float2 k01 = __half22float2(*reinterpret_cast<const __half2*>(&kr[t].x));
      const float2 k23 = __half22float2(*reinterpret_cast<const __half2*>(&kr[t].y));
      const float x = warp_sum(q01.x * k01.x + q01.y * k01.y + q23.x * k23.x + q23.y * k23.y) * scale;
      const float mn = fmaxf(m, x);
      const float c = __expf(m - mn), p = __expf(x - mn);
      const float2 v01 = __half22float2(*reinterpret_cast<const __half2*>(&vr[t].x));
      const float2 v23 = __half22float2(*reinterpret_cast<const __half2*>(&vr[t].y));
      s = s * c + p;
      a0 = a0 * c + p * v01.x;
      a1 = a1 * c + p * v01.y;
      a2 = a2 * c + p * v23.x;
      a3 = a3 * c + p * v23.y;
      m = mn;
    }
  }
  // merge the CTA's warps
  __shared__ float sm_m[kWarps], sm_s[kWarps];
  __shared__ float sm_acc[kWarps][kD];
  if (lane == 0) {
    sm_m[warp] = m;
    sm_s[warp] = s;
  }
  sm_acc[warp][lane * 4 + 0] = a0;
  sm_acc[warp][lane * 4 + 1] = a1;
  sm_acc[warp][lane * 4 + 2] = a2;
  sm_acc[warp][lane * 4 + 3] = a3;
  __syncthreads();
  if (warp == 0) {
    float M = -INFINITY;
    for (int w = 0; w < kWarps; ++w) M = fmaxf(M, sm_m[w]);
    float S = 0.f, A[4] = {0.f, 0.f, 0.f, 0.f};
    for (int w = 0; w < kWarps; ++w) {
      const float c = (sm_m[w] == -INFINITY) ? 0.f : __expf(sm_m[w] - M);
      S += sm_s[w] * c;
      for (int j = 0; j < 4; ++j) A[j] += sm_acc[w][lane * 4 + j] * c;
    }
    const size_t pi = static_cast<size_t>(bh) * n_split + split;
    for (int j = 0; j < 4; ++j) part_acc[pi * kD + lane * 4 + j] = A[j];
    if (lane == 0) part_ms[pi] = Partial{M, S};
  }
}

// grid: B * Hq; block: 128 threads (one per dim)
__global__ void decode_merge_kernel(const float* __restrict__ part_acc, const Partial* __restrict__ part_ms,
                                    int n_split, float* __restrict__ out) {
  const int bh = blockIdx.x, j = threadIdx.x;
  float M = -INFINITY;
  for (int sp = 0; sp < n_split; ++sp) M = fmaxf(M, part_ms[static_cast<size_t>(bh) * n_split + sp].m);
  float S = 0.f, A = 0.f;
  for (int sp = 0; sp < n_split; ++sp) {
    const Partial pm = part_ms[static_cast<size_t>(bh) * n_split + sp];
    if (pm.m == -INFINITY) continue;
    const float c = __expf(pm.m - M);
    S += pm.s * c;
    A += part_acc[(static_cast<size_t>(bh) * n_split + sp) * kD + j] * c;
  }
  out[static_cast<size_t>(bh) * kD + j] = A / S;
}

}  // namespace

extern "C" {

// Scratch floats needed: B*Hq*splits*(kD + 2).
int victim_decode_attention(const void* q, const void* k_plane, const void* v_plane, const int32_t* bt,
                            const int32_t* ctx, int batch, int max_blocks, int hq, int hkv, int head_dim,
                            int bs, int blocks_per_split, float* scratch, float* out, void* stream) {
  if (head_dim != kD || bs != kBs || hq % hkv) return 1;
  const int splits = (max_blocks + blocks_per_split - 1) / blocks_per_split;
  float* part_acc = scratch;
  Partial* part_ms = reinterpret_cast<Partial*>(scratch + static_cast<size_t>(batch) * hq * splits * kD);
  dim3 g1(batch * hq, splits);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  decode_split_kernel<<<g1, kWarps * 32, 0, s>>>(
      static_cast<const __half*>(q), static_cast<const uint8_t*>(k_plane), static_cast<const uint8_t*>(v_plane),
      bt, ctx, max_blocks, hq, hkv, bs, blocks_per_split, 1.0f / sqrtf(static_cast<float>(head_dim)), part_acc,
      part_ms);
  decode_merge_kernel<<<batch * hq, kD, 0, s>>>(part_acc, part_ms, splits, out);
  return static_cast<int>(cudaGetLastError());
}

}  // extern "C"
