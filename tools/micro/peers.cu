// Microbenchmark: peer masks of 32 lanes' keys -- match.any vs one ballot per key bit.
#include <cstdio>
#include <cstdint>
__global__ void k_peers(int iters, int mode, int nkeys, unsigned long long* out, uint32_t* sink) {
  const int lane = threadIdx.x & 31;
  uint32_t acc = 0, key = (lane * 2654435761u + blockIdx.x) % nkeys;
  const int nbits = 32 - __clz(nkeys | 1);
  long long t0 = clock64();
  for (int t = 0; t < iters; t++) {
    uint32_t m;
    if (mode == 0) {
      m = __match_any_sync(0xFFFFFFFFu, key);
    } else {
      m = 0xFFFFFFFFu;
      for (int b = 0; b < nbits; b++) {
        const bool bit = (key >> b) & 1u;
        const uint32_t bb = __ballot_sync(0xFFFFFFFFu, bit);
        m &= bit ? bb : ~bb;
      }
    }
    acc += __popc(m);
    key = (key * 1103515245u + 12345u + m) % nkeys;
  }
  long long t1 = clock64();
  if (lane == 0) out[blockIdx.x * 2 + (threadIdx.x >> 5)] = (unsigned long long)(t1 - t0);
  sink[blockIdx.x * 64 + threadIdx.x] = acc;
}
int main() {
  unsigned long long* d; uint32_t* s;
  cudaMalloc(&d, 8 * 148 * 64); cudaMalloc(&s, 4 * 148 * 64 * 64);
  for (int nk : {8, 64, 1024}) for (int mode = 0; mode < 2; mode++) for (int warps : {1, 16}) {
    int iters = 20000;
    k_peers<<<148, 32 * warps>>>(iters, mode, nk, d, s);
    cudaDeviceSynchronize();
    unsigned long long h[2];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    printf("nkeys %5d %-10s warps/SM %2d: %.1f cycles/op per warp\n", nk, mode == 0 ? "match.any" : "ballots", warps, (double)h[0] / iters);
  }
  return 0;
}
