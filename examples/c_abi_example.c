/* c_abi_example.c — using libwind_kv.so from plain C (no Python, no torch).
 *
 * Two device pools on GPU 0 (OPT-125M-shaped KV: 12 layers, 12 heads, d 64, fp16, 16-token
 * blocks), a shuffled hand-off of 64 blocks with per-layer flags, then a check that every
 * destination chunk holds its source chunk and every other chunk kept its bytes.
 *
 * Build (done by __graft_entry__.build()):
 *   gcc -O2 -I include examples/c_abi_example.c -L paper_conf_isca_fenghzly025_b200 \
 *       -lwind_kv -L /usr/local/cuda/lib64 -lcudart -Wl,-rpath,... -o examples/c_abi_example
 * Exit code 0 = success. */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "wind_kv.h"

#define CHECK(x)                                                                        \
  do {                                                                                  \
    wind_status s_ = (x);                                                               \
    if (s_ != WIND_OK) {                                                                \
      fprintf(stderr, "%s failed: %s (%s)\n", #x, wind_kv_status_string(s_),            \
              wind_kv_last_error());                                                    \
      return 1;                                                                         \
    }                                                                                   \
  } while (0)

static uint8_t pattern(uint64_t pool, uint64_t off) {
  uint64_t z = pool * 0x9E3779B97F4A7C15ull ^ off;
  z ^= z >> 29;
  z *= 0xBF58476D1CE4E5B9ull;
  return (uint8_t)(z >> 56);
}

int main(void) {
  const int L = 12, H = 12, D = 64, BS = 16, EB = 2, NB_SRC = 100, NB_DST = 120, N = 64;
  wind_kv_pool_desc d = {0, L, H, D, BS, EB, NB_SRC, WIND_LOC_DEVICE, 0, 0};
  wind_kv_pool *src = NULL, *dst = NULL;
  CHECK(wind_kv_pool_create(&d, NULL, &src));
  d.n_blocks = NB_DST;
  CHECK(wind_kv_pool_create(&d, NULL, &dst));
  void *sb, *db;
  size_t sbytes, dbytes;
  CHECK(wind_kv_pool_info(src, &sb, &sbytes, NULL));
  CHECK(wind_kv_pool_info(dst, &db, &dbytes, NULL));
  uint8_t* hs = (uint8_t*)malloc(sbytes);
  uint8_t* hd = (uint8_t*)malloc(dbytes);
  uint8_t* out = (uint8_t*)malloc(dbytes);
  for (size_t i = 0; i < sbytes; ++i) hs[i] = pattern(1, i);
  for (size_t i = 0; i < dbytes; ++i) hd[i] = pattern(2, i);
  cudaMemcpy(sb, hs, sbytes, cudaMemcpyHostToDevice);
  cudaMemcpy(db, hd, dbytes, cudaMemcpyHostToDevice);

  int32_t sbt[64], dbt[64];
  for (int i = 0; i < N; ++i) {
    sbt[i] = (i * 37 + 11) % NB_SRC; /* a permutation slice (37 coprime with 100) */
    dbt[i] = (i * 7 + 3) % NB_DST;   /* distinct: 7 coprime with 120 */
  }
  CHECK(wind_kv_validate(src, sbt, dst, dbt, N, 0, L));
  int32_t *dsbt, *ddbt;
  cudaMalloc((void**)&dsbt, sizeof sbt);
  cudaMalloc((void**)&ddbt, sizeof dbt);
  cudaMemcpy(dsbt, sbt, sizeof sbt, cudaMemcpyHostToDevice);
  cudaMemcpy(ddbt, dbt, sizeof dbt, cudaMemcpyHostToDevice);

  cudaStream_t mover, consumer;
  cudaStreamCreateWithFlags(&mover, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&consumer, cudaStreamNonBlocking);
  CHECK(wind_kv_migrate(src, dsbt, dst, ddbt, N, 0, L, mover));
  uint32_t ticket = 0;
  CHECK(wind_kv_layer_ticket(dst, &ticket));
  for (int l = 0; l < L; ++l) CHECK(wind_kv_layer_wait(dst, l, ticket, consumer));
  cudaStreamSynchronize(consumer); /* every layer has landed */
  cudaMemcpy(out, db, dbytes, cudaMemcpyDeviceToHost);

  /* expected: chunk (l, kv, dbt[i]) = source chunk (l, kv, sbt[i]); others unchanged */
  const size_t C = (size_t)H * BS * D * EB;
  for (int l = 0; l < L; ++l)
    for (int kv = 0; kv < 2; ++kv)
      for (int i = 0; i < N; ++i)
        memcpy(hd + (((size_t)l * 2 + kv) * NB_DST + dbt[i]) * C,
               hs + (((size_t)l * 2 + kv) * NB_SRC + sbt[i]) * C, C);
  if (memcmp(out, hd, dbytes) != 0) {
    fprintf(stderr, "mismatch\n");
    return 2;
  }
  printf("c_abi_example OK: %d blocks x %d layers, ticket %u, %s\n", N, L, ticket, wind_kv_version());
  CHECK(wind_kv_pool_destroy(src));
  CHECK(wind_kv_pool_destroy(dst));
  free(hs);
  free(hd);
  free(out);
  return 0;
}
