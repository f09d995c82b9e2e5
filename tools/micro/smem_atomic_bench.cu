// Microbenchmark: shared-memory fp32 atomicAdd throughput on B200 (HiCOO output-tile
// accumulation design decision).  Not part of the library.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void k(float *sink, int iters, int rows) {
  __shared__ float tile[128 * 32];
  for (int i = threadIdx.x; i < 128 * 32; i += blockDim.x) tile[i] = 0.f;
  __syncthreads();
  uint32_t s = threadIdx.x * 2654435761u + blockIdx.x;
  int lane = threadIdx.x & 31;
  for (int it = 0; it < iters; ++it) {
    s = s * 1664525u + 1013904223u;
    // rows: a group of 4 lanes (MODE 0: 16 cols each lane 4 floats) hits one row
    int row = (__shfl_sync(0xffffffff, s, lane & ~3) >> 8) % rows;
    float *p = tile + row * 16 + (lane & 3) * 4;
    if (MODE == 0) {
      atomicAdd(p + 0, 1.f); atomicAdd(p + 1, 1.f); atomicAdd(p + 2, 1.f); atomicAdd(p + 3, 1.f);
    } else {
      p[0] += 1.f; p[1] += 1.f; p[2] += 1.f; p[3] += 1.f;  // racy plain RMW (reference cost)
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) sink[blockIdx.x] = tile[0];
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float *sink; cudaMalloc(&sink, 1 << 20);
  int iters = 4096;
  for (int rows : {128, 8}) {
    for (int bpsm : {2, 4, 8}) {
      cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
      for (int mode = 0; mode < 2; ++mode) {
        auto kern = mode == 0 ? k<0> : k<1>;
        kern<<<sms * bpsm, 256>>>(sink, iters, rows);
        cudaEventRecord(a);
        kern<<<sms * bpsm, 256>>>(sink, iters, rows);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double nnz = (double)sms * bpsm * 256 / 4 * iters;  // one "nonzero" = 4 lanes x 4 floats
        printf("rows=%3d bpsm=%d %s: %.3f ms  %.2f G nnz-updates/s (R=16), %.2f cyc/nnz/SM @1.9GHz\n", rows, bpsm,
               mode == 0 ? "atomicAdd smem" : "plain RMW smem", ms, nnz / ms / 1e6,
               (ms * 1e-3 * 1.9e9 * sms) / nnz);
      }
    }
  }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
