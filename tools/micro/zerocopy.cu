// Zero-copy PCIe bandwidth of kernels reading / writing pinned host memory
// directly (mapped through UVA), against cudaMemcpyAsync of the same bytes.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o zerocopy zerocopy.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void rd8(const uint64_t* __restrict__ src, uint64_t* __restrict__ dst, size_t n) {
  uint64_t acc = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) acc ^= src[i];
  if (acc == 0x123456789ull) dst[0] = acc;
}
__global__ void rd8x4(const uint64_t* __restrict__ src, uint64_t* __restrict__ dst, size_t n) {
  uint64_t acc = 0;
  const size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += 4 * st) {
    uint64_t v[4];
#pragma unroll
    for (int u = 0; u < 4; u++) v[u] = i + u * st < n ? src[i + u * st] : 0;
#pragma unroll
    for (int u = 0; u < 4; u++) acc ^= v[u];
  }
  if (acc == 0x123456789ull) dst[0] = acc;
}
__global__ void wr8(uint64_t* __restrict__ dst, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) dst[i] = i;
}
__global__ void rw8(const uint64_t* __restrict__ src, uint64_t* __restrict__ dst, size_t n) {
  const size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += 4 * st) {
    uint64_t v[4];
#pragma unroll
    for (int u = 0; u < 4; u++) v[u] = i + u * st < n ? src[i + u * st] : 0;
#pragma unroll
    for (int u = 0; u < 4; u++)
      if (i + u * st < n) dst[i + u * st] = v[u] + 1;
  }
}

int main() {
  const size_t n = 67108864 / 8;  // 64 MB
  uint64_t *hs, *hd, *ds, *dd;
  cudaHostAlloc(&hs, n * 8, cudaHostAllocDefault);
  cudaHostAlloc(&hd, n * 8, cudaHostAllocDefault);
  cudaMalloc(&ds, n * 8);
  cudaMalloc(&dd, n * 8);
  for (size_t i = 0; i < n; i++) hs[i] = i * 7;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto tm = [&](auto f) {
    for (int w = 0; w < 2; w++) f();
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    for (int r = 0; r < 5; r++) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / 5;
  };
  int grids[] = {148, 296, 592, 1184, 2368};
  for (int g : grids) {
    float t1 = tm([&] { rd8<<<g, 256>>>(hs, dd, n); });
    float t2 = tm([&] { rd8x4<<<g, 256>>>(hs, dd, n); });
    float t3 = tm([&] { wr8<<<g, 256>>>(hd, n); });
    float t4 = tm([&] { rw8<<<g, 256>>>(hs, hd, n); });
    printf("grid %5d  read %.1f GB/s  read x4 %.1f GB/s  write %.1f GB/s  read+write %.1f GB/s each way\n", g,
           n * 8 / t1 / 1e6, n * 8 / t2 / 1e6, n * 8 / t3 / 1e6, n * 8 / t4 / 1e6);
  }
  float c1 = tm([&] { cudaMemcpyAsync(ds, hs, n * 8, cudaMemcpyHostToDevice); });
  float c2 = tm([&] { cudaMemcpyAsync(hd, dd, n * 8, cudaMemcpyDeviceToHost); });
  printf("memcpy H2D %.1f GB/s  D2H %.1f GB/s\n", n * 8 / c1 / 1e6, n * 8 / c2 / 1e6);
  cudaStream_t s1, s2;
  cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  uint64_t *hs2, *hd2;
  cudaHostAlloc(&hs2, n * 8, cudaHostAllocDefault);
  cudaHostAlloc(&hd2, n * 8, cudaHostAllocDefault);
  auto both = [&](auto f1, auto f2) {
    return tm([&] {
      cudaEvent_t e0;
      cudaEventCreateWithFlags(&e0, cudaEventDisableTiming);
      cudaEventRecord(e0, 0);
      cudaStreamWaitEvent(s1, e0, 0);
      cudaStreamWaitEvent(s2, e0, 0);
      f1(s1);
      f2(s2);
      cudaEvent_t e1, e2;
      cudaEventCreateWithFlags(&e1, cudaEventDisableTiming);
      cudaEventCreateWithFlags(&e2, cudaEventDisableTiming);
      cudaEventRecord(e1, s1);
      cudaEventRecord(e2, s2);
      cudaStreamWaitEvent(0, e1, 0);
      cudaStreamWaitEvent(0, e2, 0);
    });
  };
  float x1 = both([&](cudaStream_t s) { cudaMemcpyAsync(ds, hs, n * 8, cudaMemcpyHostToDevice, s); },
                  [&](cudaStream_t s) { cudaMemcpyAsync(hd, dd, n * 8, cudaMemcpyDeviceToHost, s); });
  float x2 = both([&](cudaStream_t s) { cudaMemcpyAsync(ds, hs, n * 8, cudaMemcpyHostToDevice, s); },
                  [&](cudaStream_t s) { wr8<<<592, 256, 0, s>>>(hd, n); });
  float x3 = both([&](cudaStream_t s) { rd8x4<<<592, 256, 0, s>>>(hs, dd, n); },
                  [&](cudaStream_t s) { cudaMemcpyAsync(hd, dd, n * 8, cudaMemcpyDeviceToHost, s); });
  float x4 = both([&](cudaStream_t s) { rd8x4<<<296, 256, 0, s>>>(hs, dd, n); },
                  [&](cudaStream_t s) { wr8<<<296, 256, 0, s>>>(hd, n); });
  printf("64 MB each way, concurrent: memcpy+memcpy %.3f ms, memcpy H2D + kernel writes %.3f ms, kernel reads + memcpy D2H %.3f ms, kernel reads + kernel writes %.3f ms\n", x1, x2, x3, x4);
  // H2D of 64 MB in 12 copies on one stream: with and without an event
  // record after each copy (does a record drain the copy pipeline?)
  {
    cudaEvent_t ev[12];
    for (int j = 0; j < 12; j++) cudaEventCreateWithFlags(&ev[j], cudaEventDisableTiming);
    for (int rep = 0; rep < 3; rep++) {
      float t0 = tm([&] { for (int j = 0; j < 12; j++) cudaMemcpyAsync(ds + j * (n / 12), hs + j * (n / 12), (n / 12) * 8, cudaMemcpyHostToDevice); });
      float t1 = tm([&] { for (int j = 0; j < 12; j++) { cudaMemcpyAsync(ds + j * (n / 12), hs + j * (n / 12), (n / 12) * 8, cudaMemcpyHostToDevice); cudaEventRecord(ev[j], 0); } });
      float t2 = tm([&] { cudaMemcpyAsync(ds, hs, n * 8, cudaMemcpyHostToDevice); });
      printf("H2D 64 MB: 12 copies %.3f ms, 12 copies + event records %.3f ms, 1 copy %.3f ms\n", t0, t1, t2);
    }
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
