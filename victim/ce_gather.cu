// ce_gather.cu — BENCH HARNESS ONLY: copy-engine comparators for the paged gather/scatter
// ("Copy-engine comparators (cudaMemcpyAsync / cudaMemcpyBatchAsync) to
// learn the practical ceilings").  They move exactly what wind_kv_migrate moves —
// dst[plane][dst_bt[i]] := src[plane][src_bt[i]], C bytes per (plane, i) — but with the
// DMA engines instead of SM kernels:
//   ce_gather_loop  : one cudaMemcpyAsync per chunk (the classic per-block swap loop);
//   ce_gather_batch : cudaMemcpyBatchAsync (CUDA 12.8+), up to 64 Ki copies per call.
// Tables are HOST arrays (the driver needs every address at enqueue time).  Not part of
// the product library.
#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

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

int ce_gather_batch(const uint8_t* src_plane0, int64_t s_stride, uint8_t* dst_plane0, int64_t d_stride,
                    int64_t chunk, const int32_t* sbt, const int32_t* dbt, int32_t n, int32_t planes,
                    void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const size_t total = static_cast<size_t>(n) * planes;
  const size_t per_call = 65536;
  std::vector<void*> dsts(per_call), srcs(per_call);
  std::vector<size_t> sizes(per_call, static_cast<size_t>(chunk));
  cudaMemcpyAttributes attr = {};
  attr.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
  size_t attr_idx = 0;
  for (size_t base = 0; base < total; base += per_call) {
    const size_t cnt = total - base < per_call ? total - base : per_call;
    for (size_t k = 0; k < cnt; ++k) {
      const size_t c = base + k;
      const int64_t p = static_cast<int64_t>(c / n), i = static_cast<int64_t>(c % n);
      dsts[k] = dst_plane0 + p * d_stride + static_cast<int64_t>(dbt[i]) * chunk;
      srcs[k] = const_cast<uint8_t*>(src_plane0 + p * s_stride + static_cast<int64_t>(sbt[i]) * chunk);
    }
    size_t fail = 0;
    cudaError_t e = cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), cnt, &attr, &attr_idx, 1,
                                         &fail, s);
    if (e != cudaSuccess) return static_cast<int>(e);
  }
  return 0;
}

}  // extern "C"
