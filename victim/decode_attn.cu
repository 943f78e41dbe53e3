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

  // Lane layout: half-warp `hw` (= lane / 16) takes the tokens of parity hw; lane `dl` (=
  // lane % 16) holds dims [8 dl, 8 dl + 8) as one 16-B vector, so one warp-wide load moves
  // two adjacent 256-B token rows.  Each half-warp keeps its own online softmax; the two
  // are merged after the loop.
  const int hw = lane >> 4, dl = lane & 15;
  const uint4 qv = *reinterpret_cast<const uint4*>(q + (static_cast<size_t>(b) * hq + h) * kD + dl * 8);
  float qf[8];
  {
    const __half2* q2 = reinterpret_cast<const __half2*>(&qv);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float2 f = __half22float2(q2[j]);
      qf[2 * j] = f.x * scale;
      qf[2 * j + 1] = f.y * scale;
    }
  }
  float m = -INFINITY, s = 0.f, acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};

  for (int blk = blk0 + warp; blk < blk1; blk += kWarps) {
    const int slot = bt[static_cast<size_t>(b) * max_blocks + blk];
    const uint8_t* kt = k_plane + slot * chunk + hk * tile;
    const uint8_t* vt = v_plane + slot * chunk + hk * tile;
    const int ntok = min(bs, len - blk * bs);
    uint4 kr[kBs / 2], vr[kBs / 2];
#pragma unroll
    for (int t2 = 0; t2 < kBs / 2; ++t2) {
      const int t = 2 * t2 + hw;
      if (t < ntok) kr[t2] = *reinterpret_cast<const uint4*>(kt + t * kD * 2 + dl * 16);
    }
#pragma unroll
    for (int t2 = 0; t2 < kBs / 2; ++t2) {
      const int t = 2 * t2 + hw;
      if (t < ntok) vr[t2] = *reinterpret_cast<const uint4*>(vt + t * kD * 2 + dl * 16);
    }
#pragma unroll
    for (int t2 = 0; t2 < kBs / 2; ++t2) {
      const int t = 2 * t2 + hw;
      const __half2* k2 = reinterpret_cast<const __half2*>(&kr[t2]);
      float x = 0.f;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const float2 f = __half22float2(k2[j]);
        x += qf[2 * j] * f.x + qf[2 * j + 1] * f.y;
      }
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);  // within the half
      if (t < ntok) {
        const float mn = fmaxf(m, x);
        const float c = __expf(m - mn), p = __expf(x - mn);
        const __half2* v2 = reinterpret_cast<const __half2*>(&vr[t2]);
        s = s * c + p;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float2 f = __half22float2(v2[j]);
          acc[2 * j] = acc[2 * j] * c + p * f.x;
          acc[2 * j + 1] = acc[2 * j + 1] * c + p * f.y;
        }
        m = mn;
      }
    }
  }
  // merge the two half-warps (token parities): lane dl of half 0 with lane dl of half 1
  {
    const float mo = __shfl_xor_sync(0xffffffffu, m, 16);
    const float so = __shfl_xor_sync(0xffffffffu, s, 16);
    const float M = fmaxf(m, mo);
    const float c1 = (m == -INFINITY) ? 0.f : __expf(m - M);
    const float c2 = (mo == -INFINITY) ? 0.f : __expf(mo - M);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float ao = __shfl_xor_sync(0xffffffffu, acc[j], 16);
      acc[j] = acc[j] * c1 + ao * c2;
    }
    s = s * c1 + so * c2;
    m = M;
  }
  // lane dl of half 0 now holds dims [8 dl, 8 dl + 8); write as the 4-per-lane layout below
  float a0, a1, a2, a3;
  {
    // lane L needs dims [4L, 4L + 4) = half (L & 1) of lane (L >> 1)'s 8 dims
    const int srcl = lane >> 1;
    float g[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) g[j] = __shfl_sync(0xffffffffu, acc[j], srcl);
    const bool hi4 = lane & 1;
    a0 = hi4 ? g[4] : g[0];
    a1 = hi4 ? g[5] : g[1];
    a2 = hi4 ? g[6] : g[2];
    a3 = hi4 ? g[7] : g[3];
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
