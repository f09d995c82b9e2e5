// Microbenchmark (not part of the library): is B200's ~64 MB effective L2 for random gathers
// the two dies' L2 halves each keeping a copy of lines their own SMs read?  If so, gathers in
// which the SMs of die d touch only lines HOMED on die d should see ~126 MB.
//
// 1. SM -> die: every SM times coherent (ld.global.cv, served by the home L2 slice) loads to
//    the same 256 2-KB chunks; SMs of one die share the near/far pattern (B300_MICROARCH.md:
//    near 234 / far 262 cycles, address -> die at 2 KB grain).  Group = sign of the
//    correlation with SM 0's pattern.
// 2. chunk -> home die: one SM per die times every 2-KB chunk of the table; near on its die.
// 3. random 64-B row gathers (4 lanes x 16 B, 8 in flight per group) over tables of 48..192 MB:
//      full   : every SM over every chunk
//      va     : SMs of die d over the d-th half of the table by address
//      home   : SMs of die d over the chunks homed on die d
//      cross  : SMs of die d over the chunks homed on the other die
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t smid() { uint32_t s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s)); return s; }

__device__ __forceinline__ uint32_t ld_cv(const uint32_t *p) {
  uint32_t v; asm volatile("ld.global.cv.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}

// every line of a 2-KB chunk holds (in word 0) the chunk-relative word offset of the next line
__global__ void init_chase(uint32_t *buf, uint64_t nchunks) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < nchunks * 16;
       i += uint64_t(gridDim.x) * blockDim.x)
    buf[i * 32] = uint32_t(((i + 1) % 16) * 32);
}

// dependent chase of `len` coherent loads through the lines of chunk c: cycles per load.  The
// chain's result is stored to shared memory (a side effect waiting on the last load) before
// the second clock read, which ptxas otherwise hoists above the loads.
__device__ __forceinline__ uint32_t chase(const uint32_t *chunk, int len, volatile uint32_t *sink) {
  uint32_t off = 0;
  const long long t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < len; ++i) off = ld_cv(chunk + off);
  *sink = off;
  __syncwarp();
  const long long t1 = clock64();
  return uint32_t((t1 - t0) / len);
}

// one CTA per SM (forced by shared memory); thread 0 times NC chunks (64-load chase, min of 2)
__global__ void sm_pattern(const uint32_t *buf, int nc, uint32_t *lat, uint32_t *sm_of_cta) {
  extern __shared__ uint32_t pad[];
  if (threadIdx.x != 0) return;
  sm_of_cta[blockIdx.x] = smid();
  for (int c = 0; c < nc; ++c) {
    const uint32_t *ch = buf + size_t(c) * 512;
    lat[size_t(blockIdx.x) * nc + c] = chase(ch, 64, pad);
  }
}

// chunk latencies from one chosen SM (CTAs on other SMs exit); thread t chases chunks t, t+256..
__global__ void chunk_home(const uint32_t *buf, uint64_t nchunks, uint32_t want_sm, uint32_t *lat, int *ran) {
  extern __shared__ uint32_t pad[];
  if (smid() != want_sm) return;
  if (threadIdx.x == 0) *ran = 1;
  for (uint64_t c = threadIdx.x; c < nchunks; c += blockDim.x) lat[c] = chase(buf + c * 512, 16, pad + threadIdx.x);
}

__device__ __forceinline__ uint32_t hash32(uint64_t z) {
  z *= 0x9E3779B97F4A7C15ull; z ^= z >> 31; z *= 0xbf58476d1ce4e5b9ull; z ^= z >> 29;
  return uint32_t(z);
}

// chunks: [die][n_d] chunk ids; die_of[smid]; mode 0 = full list (die 0 list = all chunks)
__global__ void __launch_bounds__(256) gather_k(const float *__restrict__ tab, const uint32_t *__restrict__ list0,
                                                uint32_t n0, const uint32_t *__restrict__ list1, uint32_t n1,
                                                const int8_t *__restrict__ die_of, uint64_t ngath, float *sink) {
  const int lane = threadIdx.x & 31, g = lane / 4, l = lane % 4;
  const int d = die_of[smid()];
  const uint32_t *list = d ? list1 : list0;
  const uint32_t n = d ? n1 : n0;
  const uint64_t warp = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint64_t base = warp * 64; base < ngath; base += nw * 64) {
    uint32_t r[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t h = hash32(base + u * 8 + g);
      r[u] = __ldg(list + (h % n)) * 32u + (h >> 27);  // 32 rows of 64 B per 2-KB chunk
    }
    float4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldg(reinterpret_cast<const float4 *>(tab + uint64_t(r[u]) * 16) + l);
#pragma unroll
    for (int u = 0; u < 8; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 1234.5f) sink[0] = acc.y + acc.z + acc.w;
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const size_t max_mb = 192;
  const size_t bytes = max_mb << 20;
  uint32_t *buf; float *sink;
  CK(cudaMalloc(&buf, bytes));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(buf, 0, bytes));
  // ---- 1. SM -> die
  const int NC = 256;
  uint32_t *lat, *smof;
  CK(cudaMalloc(&lat, size_t(sms) * NC * 4));
  CK(cudaMalloc(&smof, sms * 4));
  const int big = 200 * 1024;
  CK(cudaFuncSetAttribute(sm_pattern, cudaFuncAttributeMaxDynamicSharedMemorySize, big));
  CK(cudaFuncSetAttribute(chunk_home, cudaFuncAttributeMaxDynamicSharedMemorySize, big));
  init_chase<<<4096, 256>>>(buf, bytes / 2048);
  CK(cudaGetLastError());
  sm_pattern<<<sms, 32, big>>>(buf, NC, lat, smof);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  std::vector<uint32_t> hl(size_t(sms) * NC), hsm(sms);
  CK(cudaMemcpy(hl.data(), lat, hl.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hsm.data(), smof, sms * 4, cudaMemcpyDeviceToHost));
  // per CTA: centred pattern; correlation with CTA 0's
  std::vector<double> mean(sms, 0);
  for (int b = 0; b < sms; ++b) {
    for (int c = 0; c < NC; ++c) mean[b] += hl[size_t(b) * NC + c];
    mean[b] /= NC;
  }
  std::vector<int8_t> die(1024, -1);
  int cnt[2] = {0, 0};
  double minabs = 1e9;
  uint32_t lo_lat = 1e9, hi_lat = 0;
  for (int b = 0; b < sms; ++b) {
    double cov = 0, v0 = 0, vb = 0;
    for (int c = 0; c < NC; ++c) {
      double a = hl[c] - mean[0], x = hl[size_t(b) * NC + c] - mean[b];
      cov += a * x; v0 += a * a; vb += x * x;
      lo_lat = std::min(lo_lat, hl[size_t(b) * NC + c]);
      hi_lat = std::max(hi_lat, hl[size_t(b) * NC + c]);
    }
    double r = cov / std::sqrt(v0 * vb + 1e-30);
    minabs = std::min(minabs, std::fabs(r));
    int d = r > 0 ? 0 : 1;
    die[hsm[b]] = d;
    cnt[d]++;
  }
  printf("SM->die: %d / %d SMs, min |corr| %.3f, cv latency range %u..%u cycles\n", cnt[0], cnt[1], minabs, lo_lat,
         hi_lat);
  printf("die map:");
  for (int s = 0; s < sms; ++s) printf("%d", die[s]);
  printf("\nCTA0 pattern (first 64 chunks):");
  for (int c = 0; c < 64; ++c) printf(" %u", hl[c]);
  printf("\n");
  // ---- 2. chunk -> home die (times from one SM of die 0 and one of die 1)
  const uint64_t nchunks = bytes / 2048;
  uint32_t *clat0, *clat1; int *ran;
  CK(cudaMalloc(&clat0, nchunks * 4));
  CK(cudaMalloc(&clat1, nchunks * 4));
  CK(cudaMalloc(&ran, 4));
  if (cnt[0] == 0 || cnt[1] == 0) { printf("no two SM groups found; stopping\n"); return 0; }
  int ref[2] = {-1, -1};
  for (int s = 0; s < sms; ++s) if (ref[die[s]] < 0) ref[die[s]] = s;
  std::vector<uint32_t> c0(nchunks), c1(nchunks);
  for (int d = 0; d < 2; ++d) {
    CK(cudaMemset(ran, 0, 4));
    chunk_home<<<sms, 256, big>>>(buf, nchunks, uint32_t(ref[d]), d ? clat1 : clat0, ran);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
  }
  CK(cudaMemcpy(c0.data(), clat0, nchunks * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(c1.data(), clat1, nchunks * 4, cudaMemcpyDeviceToHost));
  std::vector<uint8_t> home(nchunks);
  uint64_t nh[2] = {0, 0}, ambiguous = 0;
  for (uint64_t c = 0; c < nchunks; ++c) {
    home[c] = c0[c] <= c1[c] ? 0 : 1;
    if (c0[c] == c1[c]) ambiguous++;
    nh[home[c]]++;
  }
  printf("chunk homes: %llu on die 0, %llu on die 1, %llu ties; first 64: ", (unsigned long long)nh[0],
         (unsigned long long)nh[1], (unsigned long long)ambiguous);
  for (int c = 0; c < 64; ++c) printf("%d", home[c]);
  printf("\n");
  // ---- 3. gathers
  int8_t *ddie;
  CK(cudaMalloc(&ddie, 1024));
  CK(cudaMemcpy(ddie, die.data(), 1024, cudaMemcpyHostToDevice));
  uint32_t *l0, *l1;
  CK(cudaMalloc(&l0, nchunks * 4));
  CK(cudaMalloc(&l1, nchunks * 4));
  const uint64_t ngath = 200000000ull;
  for (size_t mb : {32, 48, 64, 80, 96, 112, 128, 160, 192}) {
    const uint64_t nc = (mb << 20) / 2048;
    for (int mode = 0; mode < 4; ++mode) {
      std::vector<uint32_t> a, b;
      for (uint64_t c = 0; c < nc; ++c) {
        if (mode == 0) { a.push_back(c); b.push_back(c); }
        else if (mode == 1) (c < nc / 2 ? a : b).push_back(c);
        else if (mode == 2) (home[c] == 0 ? a : b).push_back(c);
        else (home[c] == 1 ? a : b).push_back(c);
      }
      CK(cudaMemcpy(l0, a.data(), a.size() * 4, cudaMemcpyHostToDevice));
      CK(cudaMemcpy(l1, b.data(), b.size() * 4, cudaMemcpyHostToDevice));
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0); cudaEventCreate(&e1);
      gather_k<<<sms * 8, 256>>>((const float *)buf, l0, a.size(), l1, b.size(), ddie, ngath, sink);
      cudaEventRecord(e0);
      for (int it = 0; it < 3; ++it)
        gather_k<<<sms * 8, 256>>>((const float *)buf, l0, a.size(), l1, b.size(), ddie, ngath, sink);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= 3;
      const char *names[] = {"full ", "va   ", "home ", "cross"};
      printf("table %3zu MB %s: %.3f ms  %.1f G rows/s  (%zu / %zu chunks)\n", mb, names[mode], ms, ngath / ms / 1e6,
             a.size(), b.size());
    }
  }
  CK(cudaDeviceSynchronize());
  printf("ok\n");
}
