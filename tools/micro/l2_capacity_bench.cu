// Microbenchmark: effective L2 capacity for random 64-B row gathers from all SMs (working-set
// sweep).  Not part of the library.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void init_idx(uint32_t *idx, uint64_t n, uint32_t rows, uint64_t seed) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = (i + seed) * 0x9E3779B97F4A7C15ull;
    z ^= z >> 31; z *= 0xbf58476d1ce4e5b9ull; z ^= z >> 29;
    idx[i] = (uint32_t)(z % rows);
  }
}

__global__ void __launch_bounds__(256) gather_k(const float *__restrict__ tab, const uint32_t *__restrict__ idx,
                                                uint64_t n, float *__restrict__ sink) {
  int lane = threadIdx.x & 31, g = lane / 4, l = lane % 4;
  uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * 32; base < n; base += nw * 32) {
    uint32_t r[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) r[u] = __ldg(idx + base + u * 8 + g);
    float4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = __ldg(reinterpret_cast<const float4 *>(tab + (uint64_t)r[u] * 16) + l);
#pragma unroll
    for (int u = 0; u < 4; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint64_t n = 200000000ull;
  float *tab; uint32_t *idx; float *sink;
  cudaMalloc(&tab, 512ull << 20); cudaMalloc(&idx, n * 4); cudaMalloc(&sink, 64);
  cudaMemset(tab, 0, 512ull << 20);
  for (int mb : {4, 8, 16, 24, 32, 40, 48, 56, 64, 80, 96, 112, 128, 192, 256, 512}) {
    uint32_t rows = (uint32_t)((uint64_t(mb) << 20) / 64);
    init_idx<<<4096, 256>>>(idx, n, rows, 7);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    gather_k<<<sms * 8, 256>>>(tab, idx, n, sink);
    cudaEventRecord(a);
    for (int it = 0; it < 3; ++it) gather_k<<<sms * 8, 256>>>(tab, idx, n, sink);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); ms /= 3;
    printf("table %4d MB: %.3f ms  %.1f G rows/s  %.1f GB/s useful\n", mb, ms, n / ms / 1e6, n * 64.0 / ms / 1e6);
  }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
