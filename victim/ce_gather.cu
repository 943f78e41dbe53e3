// ce_gather.cu — BENCH HARNESS ONLY: copy-engine comparators for the paged gather/scatter
// (copy-engine comparators "to learn the practical ceilings").  It moves exactly what wind_kv_migrate moves —
// dst[plane][dst_bt[i]] := src[plane][src_bt[i]], C bytes per (plane, i) — but with the
// DMA engines instead of SM kernels:
//   ce_gather_loop  : one cudaMemcpyAsync per chunk (the classic per-block swap loop).
// Tables are HOST arrays (the driver needs every address at enqueue time).  Not part of
// the product library.
#include <cuda_runtime.h>
#include <stdint.h>

extern "C" {

int ce_gather_loop(const uint8_t* src_plane0, int64_t s_stride, uint8_t* dst_plane0, int64_t d_stride,
                   int64_t chunk, const int32_t* sbt, const int32_t* dbt, int32_t n, int32_t planes,
                   void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  for (int32_t p = 0; p < planes; ++p)
    for (int32_t i = 0; i < n; ++i) {
      cudaError_t e = cudaMemcpyAsync(dst_plane0 + p * d_stride + static_cast<int64_t>(dbt[i]) * chunk,
                                      src_plane0 + p * s_stride + static_cast<int64_t>(sbt[i]) * chunk,
                                      chunk, cudaMemcpyDefault, s);
      if (e != cudaSuccess) return static_cast<int>(e);
    }
  return 0;
}

}  // extern "C"
