// Microbenchmark: achievable HBM throughput of random row gathers on B200 (the access
// pattern of MTTKRP's factor gathers).  Not part of the library.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void init_idx(uint32_t *idx, uint64_t n, uint32_t rows, uint64_t seed) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = (i + seed) * 0x9E3779B97F4A7C15ull;
    z ^= z >> 31; z *= 0xbf58476d1ce4e5b9ull; z ^= z >> 29;
    idx[i] = (uint32_t)(z % rows);
  }
}

__global__ void copy_k(const float4 *__restrict__ a, float4 *__restrict__ b, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) b[i] = a[i];
}

// LPN lanes per row, each lane loads 16 B; U rows per group in flight.
template <int LPN, int U>
__global__ void __launch_bounds__(256) gather_k(const float *__restrict__ tab, const uint32_t *__restrict__ idx,
                                                uint64_t n, float *__restrict__ sink) {
  constexpr int G = 32 / LPN;
  int lane = threadIdx.x & 31, g = lane / LPN, l = lane % LPN;
  uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * G * U; base < n; base += nw * G * U) {
    uint32_t r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { uint64_t j = base + u * G + g; r[u] = j < n ? __ldg(idx + j) : 0; }
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = __ldg(reinterpret_cast<const float4 *>(tab + (uint64_t)r[u] * (LPN * 4)) + l);
#pragma unroll
    for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

template <int LPN, int U>
void run_gather(const char *name, const float *tab, const uint32_t *idx, uint64_t n, float *sink, int sms, int blocks_per_sm) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int grid = sms * blocks_per_sm;
  gather_k<LPN, U><<<grid, 256>>>(tab, idx, n, sink);
  cudaEventRecord(a);
  for (int it = 0; it < 5; ++it) gather_k<LPN, U><<<grid, 256>>>(tab, idx, n, sink);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
  double bytes = (double)n * LPN * 16 + (double)n * 4;
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, gather_k<LPN, U>);
  printf("%-28s bpsm=%d regs=%d  %.3f ms  %.1f GB/s (row bytes %d)\n", name, blocks_per_sm, fa.numRegs, ms, bytes / ms / 1e6, LPN * 16);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint64_t rows = 1ull << 23;
  uint64_t n = 200000000ull;  // gathers
  float *tab; uint32_t *idx; float *sink;
  cudaMalloc(&tab, rows * 32 * 4 * 2); cudaMalloc(&idx, n * 4); cudaMalloc(&sink, 64);
  cudaMemset(tab, 0, rows * 32 * 4 * 2);
  init_idx<<<4096, 256>>>(idx, n, (uint32_t)rows, 1);
  // stream copy
  {
    uint64_t m = (1ull << 30) / 16;
    float4 *x, *y; cudaMalloc(&x, m * 16); cudaMalloc(&y, m * 16);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    copy_k<<<sms * 8, 256>>>(x, y, m);
    cudaEventRecord(a); for (int i = 0; i < 5; ++i) copy_k<<<sms * 8, 256>>>(x, y, m); cudaEventRecord(b);
    cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
    printf("stream copy 1 GiB: %.1f GB/s (r+w)\n", 2.0 * m * 16 / ms / 1e6);
    cudaFree(x); cudaFree(y);
  }
  for (int bpsm : {2, 4, 8}) {
    run_gather<4, 1>("gather 64B U=1", tab, idx, n, sink, sms, bpsm);
    run_gather<4, 2>("gather 64B U=2", tab, idx, n, sink, sms, bpsm);
    run_gather<4, 4>("gather 64B U=4", tab, idx, n, sink, sms, bpsm);
    run_gather<4, 8>("gather 64B U=8", tab, idx, n, sink, sms, bpsm);
  }
  run_gather<2, 8>("gather 32B U=8", tab, idx, n, sink, sms, 8);
  run_gather<8, 4>("gather 128B U=4", tab, idx, n, sink, sms, 8);
  run_gather<8, 8>("gather 128B U=8", tab, idx, n, sink, sms, 4);
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
