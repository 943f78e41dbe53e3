// windgen_fill.cu — the O9 content generator, second implementation,
// for device memory.  TEST / BENCH INPUT INFRASTRUCTURE: it fills pools with the seeded
// splitmix64 byte pattern and checks chunks against that pattern.  It holds none of the
// migration method's arithmetic (no block addressing, no tables): callers pass byte
// offsets that the oracle computed.  The product library (paper_conf_isca_fenghzly025_b200)
// never links or calls this file, and this file includes nothing from it.
//
// Word w (the 8 bytes at pool byte offset 8*w) of pool (seed, tag) is
//   splitmix64(key ^ w),   key = seed*0x9E3779B97F4A7C15 ^ tag*0xD1B54A32D192ED03.
// windgen/__init__.py is the host implementation; tests/test_windgen.py pins both.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Fills nwords 8-byte words; word j of the buffer is pattern word (w0 + j).
__global__ void fill_kernel(uint64_t* __restrict__ dst, uint64_t nwords, uint64_t w0,
                            uint64_t key) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x * 2;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 2; j < nwords;
       j += stride) {
    if (j + 1 < nwords) {
      ulonglong2 v = make_ulonglong2(sm64(key ^ (w0 + j)), sm64(key ^ (w0 + j + 1)));
      *reinterpret_cast<ulonglong2*>(dst + j) = v;  // 16-B store (dst 16-B aligned)
    } else {
      dst[j] = sm64(key ^ (w0 + j));
    }
  }
}

// One CTA per chunk (grid-stride over chunks): compare chunk at base+dst_off[c] with the
// pattern of key[c] starting at word exp_off[c]/8.  Counts mismatching chunks and
// records the lowest mismatching chunk index.
__global__ void check_kernel(const uint8_t* __restrict__ base, uint64_t chunk_bytes,
                             const int64_t* __restrict__ dst_off,
                             const int64_t* __restrict__ exp_off,
                             const uint64_t* __restrict__ keys, int64_t n_chunks,
                             unsigned long long* __restrict__ out /* [0]=count [1]=first */) {
  __shared__ int bad;
  uint64_t nwords = chunk_bytes / 8;
  for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
    if (threadIdx.x == 0) bad = 0;
    __syncthreads();
    const uint64_t* p = reinterpret_cast<const uint64_t*>(base + dst_off[c]);
    uint64_t w0 = (uint64_t)exp_off[c] / 8;
    uint64_t key = keys[c];
    int mine = 0;
    for (uint64_t j = threadIdx.x; j < nwords; j += blockDim.x)
      mine |= (p[j] != sm64(key ^ (w0 + j)));
    if (mine) bad = 1;
    __syncthreads();
    if (threadIdx.x == 0 && bad) {
      atomicAdd(&out[0], 1ull);
      atomicMin(&out[1], (unsigned long long)c);
    }
    __syncthreads();
  }
}

}  // namespace

extern "C" {

// Fills [dptr, dptr+nbytes) with pattern bytes [byte_offset, byte_offset+nbytes) of pool
// (seed, tag).  dptr 16-B aligned; byte_offset and nbytes multiples of 8.  Returns a
// cudaError_t value (0 = success).  Asynchronous on `stream`.
int windgen_fill(void* dptr, uint64_t nbytes, uint64_t byte_offset, uint64_t seed,
                 uint64_t tag, void* stream) {
  if ((reinterpret_cast<uintptr_t>(dptr) & 15) || (nbytes & 7) || (byte_offset & 7))
    return (int)cudaErrorInvalidValue;
  if (nbytes == 0) return 0;
  uint64_t key = (seed * 0x9E3779B97F4A7C15ull) ^ (tag * 0xD1B54A32D192ED03ull);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  fill_kernel<<<sms * 8, 256, 0, (cudaStream_t)stream>>>((uint64_t*)dptr, nbytes / 8,
                                                          byte_offset / 8, key);
  return (int)cudaGetLastError();
}

// Compares n_chunks chunks (all device arrays).  out: 2 device uint64 (count, first);
// the caller initialises out = {0, UINT64_MAX}.
int windgen_check_chunks(const void* base, uint64_t chunk_bytes, const int64_t* dst_off,
                         const int64_t* exp_off, const uint64_t* keys, int64_t n_chunks,
                         unsigned long long* out, void* stream) {
  if ((chunk_bytes & 7) || (reinterpret_cast<uintptr_t>(base) & 7))
    return (int)cudaErrorInvalidValue;
  if (n_chunks <= 0) return 0;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int64_t grid = n_chunks < (int64_t)sms * 16 ? n_chunks : (int64_t)sms * 16;
  check_kernel<<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>(
      (const uint8_t*)base, chunk_bytes, dst_off, exp_off, keys, n_chunks, out);
  return (int)cudaGetLastError();
}

}  // extern "C"
