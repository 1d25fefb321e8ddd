// Microbenchmark: latency of one step of a dependent warp chain
// (LDS -> redux.sync.min -> compare -> select), one warp per SM.
#include <cstdio>
#include <cstdint>
__global__ void k_chain(int iters, int mode, unsigned long long* out, uint32_t* sink) {
  __shared__ uint16_t buf[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) buf[i] = (uint16_t)((i * 37 + threadIdx.x) & 1023);
  __syncwarp();
  const int lane = threadIdx.x & 31;
  uint32_t c = lane, acc = 0;
  long long t0 = clock64();
  for (int t = 0; t < iters; t++) {
    uint32_t cand;
    if (mode == 0) cand = buf[(c + t) & 4095];           // LDS + redux
    else if (mode == 1) cand = (c * 2654435761u + t) >> 20;  // ALU + redux
    else cand = buf[(c + t) & 4095];                     // LDS only (dependent), no redux
    uint32_t win;
    if (mode == 2) win = cand;
    else win = __reduce_min_sync(0xFFFFFFFFu, cand);
    if (cand == win) c++;
    acc += win;
  }
  long long t1 = clock64();
  if (lane == 0) out[blockIdx.x] = (unsigned long long)(t1 - t0);
  sink[blockIdx.x * 32 + lane] = acc + c;
}
int main() {
  unsigned long long* d; uint32_t* s;
  cudaMalloc(&d, 8 * 148); cudaMalloc(&s, 4 * 148 * 32);
  for (int mode = 0; mode < 3; mode++) {
    int iters = 10000;
    k_chain<<<148, 32>>>(iters, mode, d, s);
    cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, 8 * 148, cudaMemcpyDeviceToHost);
    printf("mode %d (%s): %.1f cycles/step\n", mode, mode == 0 ? "LDS+redux" : mode == 1 ? "ALU+redux" : "LDS only", (double)h[0] / iters);
  }
  return 0;
}
