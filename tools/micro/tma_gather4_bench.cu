// Microbenchmark (not part of the library): random 64-B row gathers with register loads
// (LDG.128, 4 lanes per row, as the COO MTTKRP kernel does) against TMA tile::gather4 into
// shared memory (cp.async.bulk.tensor.2d ... tile::gather4: one instruction fetches 4 rows,
// completion on an mbarrier, no registers held while in flight).  Tables of 32 MB .. 1 GB.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t hash32(uint64_t z) {
  z *= 0x9E3779B97F4A7C15ull; z ^= z >> 31; z *= 0xbf58476d1ce4e5b9ull; z ^= z >> 29;
  return uint32_t(z);
}

// register gathers: 8 groups of 4 lanes, U rows in flight per group
template <int U>
__global__ void __launch_bounds__(256) ldg_k(const float *__restrict__ tab, uint32_t rows, uint64_t ngath, float *sink) {
  const int lane = threadIdx.x & 31, g = lane / 4, l = lane % 4;
  const uint64_t warp = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * 8 * U; base < ngath; base += nw * 8 * U) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t r = hash32(base + u * 8 + g) % rows;
      v[u] = __ldg(reinterpret_cast<const float4 *>(tab + uint64_t(r) * 16) + l);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return uint32_t(__cvta_generic_to_shared(p)); }

// TMA gathers: each warp owns a ring of S stages x ROWS rows (64 B each); lane 0 issues ROWS/4
// gather4 ops per stage on the stage's mbarrier; the warp consumes the stage S-1 stages later
template <int S, int ROWS>
__global__ void __launch_bounds__(128) tma_k(const __grid_constant__ CUtensorMap map, uint32_t rows, uint64_t ngath,
                                             float *sink) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bars[4][S];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  float4 *ring = reinterpret_cast<float4 *>(smem + size_t(warp) * S * ROWS * 64);
  if (lane == 0)
    for (int s = 0; s < S; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[warp][s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const uint64_t gw = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  const uint64_t nbatch = ngath / ROWS;
  auto issue = [&](uint64_t b, int s) {
    if (lane == 0) {
      const uint32_t bar = smem_u32(&bars[warp][s]);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(ROWS * 64) : "memory");
      for (int q = 0; q < ROWS / 4; ++q) {
        int32_t r[4];
        for (int i = 0; i < 4; ++i) r[i] = int32_t(hash32(b * ROWS + q * 4 + i) % rows);
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(ring + (size_t(s) * ROWS + q * 4) * 4)),
            "l"(&map), "r"(0), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(bar)
            : "memory");
      }
    }
  };
  float4 acc = make_float4(0, 0, 0, 0);
  uint32_t phase[S] = {};
  uint64_t it = 0;
  for (uint64_t b = gw; b < nbatch + uint64_t(S - 1) * nw; b += nw, ++it) {
    const int s = int(it % S);
    if (b < nbatch) issue(b, s);
    if (it >= uint64_t(S - 1)) {  // consume the stage issued S-1 iterations ago
      const int sc = int((it - (S - 1)) % S);
      const uint32_t bar = smem_u32(&bars[warp][sc]);
      uint32_t done = 0;
      while (!done)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done) : "r"(bar), "r"(phase[sc]) : "memory");
      phase[sc] ^= 1u;
      for (int i = lane; i < ROWS * 4; i += 32) {
        const float4 v = ring[size_t(sc) * ROWS * 4 + i];
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
      __syncwarp();
    }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

typedef CUresult (*EncodeFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                             const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  EncodeFn encode = reinterpret_cast<EncodeFn>(fn);
  const size_t max_bytes = size_t(1) << 30;
  float *tab, *sink;
  CK(cudaMalloc(&tab, max_bytes));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(tab, 0, max_bytes));
  const uint64_t ngath = 200000000ull;
  for (size_t mb : {32, 64, 128, 256, 1024}) {
    const uint32_t rows = uint32_t((mb << 20) / 64);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    float ms;
    ldg_k<8><<<sms * 8, 256>>>(tab, rows, ngath, sink);
    cudaEventRecord(e0);
    ldg_k<8><<<sms * 8, 256>>>(tab, rows, ngath, sink);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    printf("table %4zu MB  LDG.128 x8     : %.3f ms  %6.1f G rows/s  %6.1f GB/s\n", mb, ms, ngath / ms / 1e6,
           ngath * 64.0 / ms / 1e6);
    CUtensorMap map;
    cuuint64_t dims[2] = {16, rows};
    cuuint64_t strides[1] = {64};
    cuuint32_t box[2] = {16, 1};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = encode(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, dims, strides, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("encode failed %d\n", int(r)); return 1; }
    auto run = [&](auto kern, int S, int ROWS, int cpsm, const char *name) {
      const int smem = 4 * S * ROWS * 64;
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
      kern<<<sms * cpsm, 128, smem>>>(map, rows, ngath, sink);
      CK(cudaGetLastError());
      cudaEventRecord(e0);
      kern<<<sms * cpsm, 128, smem>>>(map, rows, ngath, sink);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float t;
      cudaEventElapsedTime(&t, e0, e1);
      printf("table %4zu MB  %-14s: %.3f ms  %6.1f G rows/s  %6.1f GB/s\n", mb, name, t, ngath / t / 1e6,
             ngath * 64.0 / t / 1e6);
    };
    run(tma_k<4, 32>, 4, 32, 4, "TMA g4 4x32 c4");
    run(tma_k<4, 64>, 4, 64, 2, "TMA g4 4x64 c2");
    run(tma_k<8, 64>, 8, 64, 1, "TMA g4 8x64 c1");
  }
  CK(cudaDeviceSynchronize());
  printf("ok\n");
}
