// Microbenchmark: does splitting a random-gather working set between the two dies' SMs
// double the effective L2 capacity?  Each warp maps its row into half f(smid) of the table;
// with the right SM -> die map f, each die's L2 only has to hold half the table.  Not part of
// the library.
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

__device__ __forceinline__ uint32_t smid() { uint32_t s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s)); return s; }

__device__ __forceinline__ int side(int map, uint32_t s, uint32_t nsm) {
  switch (map) {
    case 0: return 0;                      // no split: everything into half 0 (table/2 working set)
    case 1: return s < nsm / 2;            // low / high SM ids
    case 2: return s & 1;                  // parity
    case 3: return (s >> 1) & 1;
    case 4: return (s >> 2) & 1;
    case 5: return (s >> 3) & 1;
    case 6: return (s >> 4) & 1;
    case 7: return (s >> 5) & 1;
    case 8: return (s >> 6) & 1;
    default: return -1;                    // -1: no split, full table
  }
}

__global__ void __launch_bounds__(256) gather_k(const float *__restrict__ tab, const uint32_t *__restrict__ idx,
                                                uint64_t n, uint32_t half, int map, float *__restrict__ sink) {
  int lane = threadIdx.x & 31, g = lane / 4, l = lane % 4;
  uint32_t nsm; asm volatile("mov.u32 %0, %%nsmid;" : "=r"(nsm));
  int sd = side(map, smid(), nsm);
  uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * 32; base < n; base += nw * 32) {
    uint32_t r[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      r[u] = __ldg(idx + base + u * 8 + g);
      if (sd >= 0) r[u] = r[u] % half + (uint32_t)sd * half;
    }
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
  const char *names[] = {"half only", "smid<n/2", "smid&1", "smid>>1&1", "smid>>2&1", "smid>>3&1",
                         "smid>>4&1", "smid>>5&1", "smid>>6&1", "full table"};
  for (int mb : {64, 96, 128, 160}) {
    uint32_t rows = (uint32_t)((uint64_t(mb) << 20) / 64);
    init_idx<<<4096, 256>>>(idx, n, rows, 7);
    for (int map = -1; map <= 8; ++map) {
      cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
      gather_k<<<sms * 8, 256>>>(tab, idx, n, rows / 2, map, sink);
      cudaEventRecord(a);
      for (int it = 0; it < 3; ++it) gather_k<<<sms * 8, 256>>>(tab, idx, n, rows / 2, map, sink);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); ms /= 3;
      printf("table %4d MB  %-11s: %.3f ms  %.1f G rows/s\n", mb, names[map < 0 ? 9 : map], ms, n / ms / 1e6);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
