// Development probe (round 2): what a single small kernel launch costs between two CUDA
// events after an L2-flushing kernel, by parameter-block size and dynamic shared memory —
// the fixed cost that bounds a small migrate / compaction op (bench c1_intra).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/launch_probe scripts/launch_probe.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>

#include <algorithm>
#include <vector>

template <int BYTES>
struct Blob {
  uint8_t b[BYTES];
};

template <int BYTES>
__global__ void empty_kernel(const __grid_constant__ Blob<BYTES> p, int* sink) {
  extern __shared__ uint8_t smem[];
  if (threadIdx.x == 0 && p.b[BYTES - 1] == 7) sink[blockIdx.x] = smem[0];
}

// one global load + one dependent store per CTA (the "table read then copy" chain)
template <int BYTES>
__global__ void chain_kernel(const __grid_constant__ Blob<BYTES> p, const int* table, int* out) {
  if (threadIdx.x == 0) {
    int v = table[blockIdx.x * 32];
    out[v & 1023] = v + p.b[0];
  }
}

__global__ void flush_kernel(const int4* buf, size_t n, int* sink) {
  int4 acc = {0, 0, 0, 0};
  for (size_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    int4 v = buf[i];
    acc.x ^= v.x;
  }
  if (acc.x == 12345) sink[0] = acc.y;
}

template <typename F>
float timed(F launch, const int4* fbuf, size_t fn, int* sink, bool flush, int reps = 50) {
  cudaStream_t s;
  cudaStreamCreate(&s);
  std::vector<float> t;
  for (int r = 0; r < reps + 3; ++r) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    if (flush) flush_kernel<<<592, 512, 0, s>>>(fbuf, fn, sink);
    cudaEventRecord(a, s);
    launch(s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r >= 3) t.push_back(ms * 1e3f);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
  }
  cudaStreamDestroy(s);
  std::sort(t.begin(), t.end());
  return t[t.size() / 2];
}

int main() {
  size_t fbytes = size_t(256) << 20;
  int4* fbuf;
  int* sink;
  int* table;
  cudaMalloc(&fbuf, fbytes);
  cudaMemset(fbuf, 1, fbytes);
  cudaMalloc(&sink, 1 << 20);
  cudaMalloc(&table, 1 << 20);
  cudaMemset(table, 0, 1 << 20);
  const size_t fn = fbytes / 16;
  cudaFuncSetAttribute(empty_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(empty_kernel<2432>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int flush = 0; flush < 2; ++flush) {
    for (int grid : {24, 148}) {
      for (int smem : {0, 196 * 1024}) {
        Blob<64> p64 = {};
        Blob<2432> p2k = {};
        float a = timed([&](cudaStream_t s) { empty_kernel<64><<<grid, 64, smem, s>>>(p64, sink); }, fbuf, fn, sink, flush);
        float b = timed([&](cudaStream_t s) { empty_kernel<2432><<<grid, 64, smem, s>>>(p2k, sink); }, fbuf, fn, sink, flush);
        printf("flush=%d grid=%3d smem=%6d  empty: params 64 B %.2f us, params 2432 B %.2f us\n", flush, grid, smem, a, b);
      }
      Blob<64> p64 = {};
      float c = timed([&](cudaStream_t s) { chain_kernel<64><<<grid, 64, 0, s>>>(p64, table, sink); }, fbuf, fn, sink, flush);
      printf("flush=%d grid=%3d  load->store chain kernel: %.2f us\n", flush, grid, c);
    }
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
