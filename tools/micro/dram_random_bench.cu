// Microbenchmark (not part of the library): the random-access ceiling of B200 HBM3e for row
// gathers, with a table far larger than L2 (8 GiB) so that almost every gather is a DRAM
// access.  Reports rows/s and row bytes/s for 32-, 64- and 128-B rows at several degrees of
// memory-level parallelism (blocks per SM x rows in flight per lane group).  The index stream
// (4 B per gather, sequential) is read with evict_first and is not counted in the row bytes.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/dram_random_bench tools/micro/dram_random_bench.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void init_idx(uint32_t *idx, uint64_t n, uint64_t rows, uint64_t seed) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = (i + seed) * 0x9E3779B97F4A7C15ull;
    z ^= z >> 31; z *= 0xbf58476d1ce4e5b9ull; z ^= z >> 29;
    idx[i] = (uint32_t)(z % rows);
  }
}

__device__ __forceinline__ uint32_t ld_ef(const uint32_t *p) {
  uint32_t r;
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
               "ld.global.nc.L2::cache_hint.u32 %0, [%1], pol;\n\t}" : "=r"(r) : "l"(p));
  return r;
}

// LPN lanes per row (16 B each), U rows per group in flight
template <int LPN, int U>
__global__ void __launch_bounds__(256) gather_k(const float4 *__restrict__ tab, const uint32_t *__restrict__ idx,
                                                uint64_t n, float *__restrict__ sink) {
  constexpr int G = 32 / LPN;
  const int lane = threadIdx.x & 31, g = lane / LPN, l = lane % LPN;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * G * U; base < n; base += nw * G * U) {
    uint32_t r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t j = base + u * G + g;
      r[u] = j < n ? ld_ef(idx + j) : 0u;
    }
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = __ldg(tab + (uint64_t)r[u] * LPN + l);
#pragma unroll
    for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

template <int LPN, int U>
void run(const float4 *tab, uint64_t tab_rows64, const uint32_t *idx, uint64_t n, float *sink, int sms, int bpsm) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int grid = sms * bpsm;
  gather_k<LPN, U><<<grid, 256>>>(tab, idx, n, sink);
  cudaEventRecord(a);
  for (int it = 0; it < 3; ++it) gather_k<LPN, U><<<grid, 256>>>(tab, idx, n, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  ms /= 3;
  printf("row %3d B  U=%2d  blocks/SM=%2d  %.3f ms  %.1f G rows/s  %.1f GB/s of rows\n", LPN * 16, U, bpsm, ms,
         n / ms / 1e6, double(n) * LPN * 16 / ms / 1e6);
  (void)tab_rows64;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const uint64_t bytes = 8ull << 30;  // 8 GiB table
  const uint64_t n = 200000000ull;    // gathers per launch
  float4 *tab;
  uint32_t *idx;
  float *sink;
  if (cudaMalloc(&tab, bytes) != cudaSuccess || cudaMalloc(&idx, n * 4) != cudaSuccess ||
      cudaMalloc(&sink, 64) != cudaSuccess) {
    printf("alloc failed\n");
    return 1;
  }
  cudaMemset(tab, 0, bytes);
  printf("# table %.1f GiB, %llu random gathers per launch, %d SMs\n", bytes / 1073741824.0, (unsigned long long)n, sms);
  for (int lpn : {2, 4, 8}) {
    const uint64_t rows = bytes / (lpn * 16);
    init_idx<<<4096, 256>>>(idx, n, rows, 7 + lpn);
    cudaDeviceSynchronize();
    for (int bpsm : {4, 8}) {
      if (lpn == 2) { run<2, 4>(tab, rows, idx, n, sink, sms, bpsm); run<2, 8>(tab, rows, idx, n, sink, sms, bpsm); run<2, 16>(tab, rows, idx, n, sink, sms, bpsm); }
      if (lpn == 4) { run<4, 4>(tab, rows, idx, n, sink, sms, bpsm); run<4, 8>(tab, rows, idx, n, sink, sms, bpsm); run<4, 16>(tab, rows, idx, n, sink, sms, bpsm); }
      if (lpn == 8) { run<8, 4>(tab, rows, idx, n, sink, sms, bpsm); run<8, 8>(tab, rows, idx, n, sink, sms, bpsm); run<8, 16>(tab, rows, idx, n, sink, sms, bpsm); }
    }
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s\n", cudaGetErrorString(e));
  return e == cudaSuccess ? 0 : 1;
}
