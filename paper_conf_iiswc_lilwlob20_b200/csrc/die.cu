// die.cu -- which of the B200's two dies each SM sits on (for the die-split COO MTTKRP).
//
// Why: B200's L2 is split across its two dies and a die's L2 keeps the lines its own SMs
// read, so data gathered by SMs of both dies is held twice.  Measured with random 64-B row
// gathers (tools/micro/l2_home_bench.cu, profiles/r02_l2_home_bench.txt): the effective
// capacity knee sits at ~64 MB when every SM gathers from the whole table, and moves to
// ~120 MB when the SMs of each die gather from their own half.  The die-split MTTKRP
// (coo_mark_hot / coo_staged_kernel) uses this map to give each die a disjoint half of the
// hot factor rows.
//
// How: the SM -> die map is yield-dependent (B300_MICROARCH.md: "per-GPU", a 70/78 split on
// this part) and %smid carries no die bit, so it is measured once per device: every SM times
// dependent coherent loads (ld.global.cv, served by the line's home L2 slice) to the same 256
// 2-KB chunks; the home of a chunk is on one die (2-KB grain), so the SMs of one die see the
// same near/far latency pattern.  SMs are clustered into two groups by the correlation of
// their centred patterns (2-means, seeded with SM 0).
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kCalChunks = 256;
constexpr int kCalLoads = 64;

__device__ __forceinline__ uint32_t cal_smid() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

// every line of a 2-KB chunk holds (in word 0) the chunk-relative word offset of the next line
__global__ void die_cal_init(uint32_t *buf, uint64_t nlines) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < nlines; i += uint64_t(gridDim.x) * blockDim.x)
    buf[i * 32] = uint32_t(((i + 1) % 16) * 32);
}

// one CTA per SM (the dynamic shared memory admits one); thread 0 chases kCalLoads coherent
// loads through each chunk.  The chain's result is stored to shared memory before the second
// clock read, which ptxas would otherwise hoist above the loads.
__global__ void die_cal_kernel(const uint32_t *buf, uint32_t *lat, uint32_t *sm_of_cta) {
  extern __shared__ uint32_t die_cal_pad[];
  if (threadIdx.x != 0) return;
  sm_of_cta[blockIdx.x] = cal_smid();
  volatile uint32_t *sink = die_cal_pad;
  for (int c = 0; c < kCalChunks; ++c) {
    const uint32_t *chunk = buf + size_t(c) * 512;
    uint32_t off = 0;
    const long long t0 = clock64();
#pragma unroll 1
    for (int i = 0; i < kCalLoads; ++i) asm volatile("ld.global.cv.u32 %0, [%1];" : "=r"(off) : "l"(chunk + off) : "memory");
    *sink = off;
    __syncwarp();
    const long long t1 = clock64();
    lat[size_t(blockIdx.x) * kCalChunks + c] = uint32_t((t1 - t0) / kCalLoads);
  }
}

DieMap calibrate(int dev) {
  DieMap m;
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0 ||
      sms > kMaxSms)
    return m;
  const size_t bytes = size_t(kCalChunks) * 2048;
  uint32_t *buf = nullptr, *lat = nullptr, *smof = nullptr;
  const int big = 200 * 1024;
  bool ok = cudaMalloc(&buf, bytes) == cudaSuccess && cudaMalloc(&lat, size_t(sms) * kCalChunks * 4) == cudaSuccess &&
            cudaMalloc(&smof, size_t(sms) * 4) == cudaSuccess &&
            cudaFuncSetAttribute(die_cal_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, big) == cudaSuccess;
  std::vector<uint32_t> hl(size_t(sms) * kCalChunks), hs(sms, 0xFFFFFFFFu);
  if (ok) {
    cudaMemset(buf, 0, bytes);
    die_cal_init<<<64, 256>>>(buf, bytes / 128);
    die_cal_kernel<<<sms, 32, big>>>(buf, lat, smof);
    count_launch();
    count_launch();
    ok = cudaDeviceSynchronize() == cudaSuccess &&
         cudaMemcpy(hl.data(), lat, hl.size() * 4, cudaMemcpyDeviceToHost) == cudaSuccess &&
         cudaMemcpy(hs.data(), smof, size_t(sms) * 4, cudaMemcpyDeviceToHost) == cudaSuccess;
  }
  cudaFree(buf);
  cudaFree(lat);
  cudaFree(smof);
  cudaGetLastError();
  if (!ok) return m;
  // every SM measured exactly once (one CTA per SM), else no map
  std::vector<int> cta_of(sms, -1);
  for (int b = 0; b < sms; ++b) {
    if (hs[b] >= uint32_t(sms) || cta_of[hs[b]] >= 0) return m;
    cta_of[hs[b]] = b;
  }
  // centred, normalised patterns; 2-means on the correlation, seeded by SM 0
  std::vector<double> z(size_t(sms) * kCalChunks);
  for (int s = 0; s < sms; ++s) {
    const uint32_t *v = hl.data() + size_t(cta_of[s]) * kCalChunks;
    double mean = 0, var = 0;
    for (int c = 0; c < kCalChunks; ++c) mean += v[c];
    mean /= kCalChunks;
    for (int c = 0; c < kCalChunks; ++c) var += (v[c] - mean) * (v[c] - mean);
    const double inv = var > 0 ? 1.0 / std::sqrt(var) : 0.0;
    for (int c = 0; c < kCalChunks; ++c) z[size_t(s) * kCalChunks + c] = (v[c] - mean) * inv;
  }
  std::vector<int> g(sms, 0);
  std::vector<double> cen(kCalChunks);
  for (int c = 0; c < kCalChunks; ++c) cen[c] = z[c];  // seed: SM 0's pattern
  for (int it = 0; it < 8; ++it) {
    for (int s = 0; s < sms; ++s) {
      double r = 0;
      for (int c = 0; c < kCalChunks; ++c) r += z[size_t(s) * kCalChunks + c] * cen[c];
      g[s] = r >= 0 ? 0 : 1;
    }
    // centroid direction = mean of group 0 minus mean of group 1
    std::vector<double> m0(kCalChunks, 0), m1(kCalChunks, 0);
    int n0 = 0, n1 = 0;
    for (int s = 0; s < sms; ++s) {
      std::vector<double> &t = g[s] ? m1 : m0;
      (g[s] ? n1 : n0)++;
      for (int c = 0; c < kCalChunks; ++c) t[c] += z[size_t(s) * kCalChunks + c];
    }
    if (n0 == 0 || n1 == 0) return m;
    for (int c = 0; c < kCalChunks; ++c) cen[c] = m0[c] / n0 - m1[c] / n1;
  }
  m.n[0] = m.n[1] = 0;
  for (int s = 0; s < sms; ++s) {
    m.die[s] = int8_t(g[s]);
    m.n[g[s]]++;
  }
  m.sms = sms;
  // a plausible two-die split (B200: 70 / 78); anything else -> no die split
  m.ok = m.n[0] >= sms / 3 && m.n[1] >= sms / 3;
  return m;
}

}  // namespace

const DieMap &die_map() {
  static DieMap maps[16];
  static bool done[16] = {};
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 16) {
    static DieMap none;
    return none;
  }
  if (!done[dev]) {
    const char *e = getenv("PASTA_DIE_SPLIT");
    if (!(e && *e == '0')) maps[dev] = calibrate(dev);
    if (maps[dev].ok) {
      PASTA_CUDA(cudaMalloc(&maps[dev].d_die, kMaxSms));
      PASTA_CUDA(cudaMemcpy(maps[dev].d_die, maps[dev].die, kMaxSms, cudaMemcpyHostToDevice));
    }
    if (getenv("PASTA_DEBUG")) {
      fprintf(stderr, "[pasta] die map dev %d: ok %d, %d / %d SMs: ", dev, int(maps[dev].ok), maps[dev].n[0],
              maps[dev].n[1]);
      for (int s = 0; s < maps[dev].sms; ++s) fprintf(stderr, "%d", int(maps[dev].die[s]));
      fprintf(stderr, "\n");
    }
    done[dev] = true;
  }
  return maps[dev];
}

}  // namespace pasta
