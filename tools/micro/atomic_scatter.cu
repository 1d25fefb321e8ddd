// Microbenchmark: throughput of random global atomicAdd cursors (L2 atomics)
// and of the full one-pass "atomic cursor" scatter of 16-byte payloads into
// B buckets -- the candidate non-stable partition for NOWILD_UNORDERED.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t bkt(uint64_t h, int nb) { return (uint32_t)((h * 0x9E3779B97F4A7C15ull) >> (64 - nb)); }
__global__ void k_count(const uint64_t* h, int64_t n, int nb, uint32_t* cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&cnt[bkt(h[i], nb)], 1u);
}
__global__ void k_scatter(const uint64_t* h, int64_t n, int nb, uint32_t* cur, uint4* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t x = h[i];
    const uint32_t p = atomicAdd(&cur[bkt(x, nb)], 1u);
    out[p] = make_uint4((uint32_t)x, (uint32_t)(x >> 32), (uint32_t)i, 0u);
  }
}
__global__ void k_init(uint64_t* h, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    h[i] = (uint64_t)i * 0xD6E8FEB86659FD93ull ^ ((uint64_t)i << 17);
}
__global__ void k_starts(const uint32_t* cnt, uint32_t* cur, int B) {  // naive serial scan (setup only)
  if (threadIdx.x == 0 && blockIdx.x == 0) { uint32_t s = 0; for (int b = 0; b < B; b++) { cur[b] = s; s += cnt[b]; } }
}
int main() {
  const int64_t n = 1 << 25;
  uint64_t* h; uint32_t *cnt, *cur; uint4* out;
  cudaMalloc(&h, n * 8); cudaMalloc(&out, n * 16);
  cudaMalloc(&cnt, (1 << 20) * 4); cudaMalloc(&cur, (1 << 20) * 4);
  k_init<<<148 * 8, 256>>>(h, n);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int nb = 8; nb <= 18; nb += 2) {
    const int B = 1 << nb;
    float tc = 0, ts = 0;
    for (int rep = 0; rep < 3; rep++) {
      cudaMemset(cnt, 0, B * 4);
      cudaEventRecord(a); k_count<<<148 * 16, 256>>>(h, n, nb, cnt); cudaEventRecord(b); cudaEventSynchronize(b);
      cudaEventElapsedTime(&tc, a, b);
      k_starts<<<1, 32>>>(cnt, cur, B);
      cudaEventRecord(a); k_scatter<<<148 * 16, 256>>>(h, n, nb, cur, out); cudaEventRecord(b); cudaEventSynchronize(b);
      cudaEventElapsedTime(&ts, a, b);
    }
    printf("B=2^%d  count %.1f us (%.1f G atomics/s)  scatter %.1f us (%.1f G/s, %.0f GB/s moved)\n", nb, tc * 1e3,
           n / (tc * 1e-3) / 1e9, ts * 1e3, n / (ts * 1e-3) / 1e9, n * 24.0 / (ts * 1e-3) / 1e9);
  }
  return 0;
}
