// capi.cu -- the extern "C" boundary of libpasta (include/pasta.h): validation, handles,
// errors, host-side IO / partitioning and measurement hooks.  Every compute step runs in
// the kernels of gen.cu, sort.cu, hicoo.cu and mttkrp.cu.
#include <cerrno>
#include <cinttypes>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <memory>
#include <new>

#include "internal.cuh"

namespace pasta {

// ----------------------------------------------------------------------------- errors
static thread_local std::string t_last_error;

void set_last_error(pasta_status code, const std::string &msg) {
  (void)code;
  t_last_error = msg;
}

static std::atomic<uint64_t> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

// ----------------------------------------------------------------------------- memory
static std::mutex g_alloc_mu;
static pasta_allocator g_alloc{nullptr, nullptr, nullptr};
static bool g_alloc_set = false;

void *dev_alloc(size_t bytes, cudaStream_t s) {
  pasta_allocator a;
  bool set;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    a = g_alloc;
    set = g_alloc_set;
  }
  void *p = nullptr;
  if (set) {
    p = a.alloc(bytes, reinterpret_cast<void *>(s), a.ctx);
    if (!p) fail(PASTA_ENOMEM, "device allocation of " + std::to_string(bytes) + " bytes failed (hook)");
    return p;
  }
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    fail(e == cudaErrorMemoryAllocation ? PASTA_ENOMEM : PASTA_ECUDA,
         "cudaMalloc(" + std::to_string(bytes) + "): " + cudaGetErrorString(e));
  }
  return p;
}

void dev_free(void *p, cudaStream_t s) {
  if (!p) return;
  pasta_allocator a;
  bool set;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    a = g_alloc;
    set = g_alloc_set;
  }
  if (set) {
    a.free(p, reinterpret_cast<void *>(s), a.ctx);
  } else {
    cudaFree(p);
  }
}

// ----------------------------------------------------------------------------- profiling
static std::mutex g_prof_mu;
static std::atomic<bool> g_prof_on{false};
struct ProfRec {
  cudaEvent_t a, b;
};
static std::vector<ProfRec> g_prof[kProfKinds];

ProfScope::ProfScope(int k, cudaStream_t st) : kind(k), s(st) {
  if (!g_prof_on.load(std::memory_order_relaxed)) return;
  if (cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) {
    cudaGetLastError();
    a = b = nullptr;
    return;
  }
  cudaEventRecord(a, s);
}
ProfScope::~ProfScope() {
  if (!a) return;
  cudaEventRecord(b, s);
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_prof[kind].push_back({a, b});
}

}  // namespace pasta

using namespace pasta;

#define API_BEGIN try {
#define API_END                                                            \
  return PASTA_OK;                                                         \
  }                                                                        \
  catch (const pasta::Error &e) {                                          \
    set_last_error(e.code, e.msg);                                         \
    return e.code;                                                         \
  }                                                                        \
  catch (const std::bad_alloc &) {                                         \
    set_last_error(PASTA_ENOMEM, "host allocation failed");                \
    return PASTA_ENOMEM;                                                   \
  }                                                                        \
  catch (...) {                                                            \
    set_last_error(PASTA_EINVAL, "unexpected internal exception");         \
    return PASTA_EINVAL;                                                   \
  }

static void require(bool cond, const char *msg) {
  if (!cond) fail(PASTA_EINVAL, msg);
}

static cudaStream_t as_stream(void *s) { return reinterpret_cast<cudaStream_t>(s); }

static void check_device(int dev) {
  int cur = -1;
  PASTA_CUDA(cudaGetDevice(&cur));
  if (cur != dev)
    fail(PASTA_EINVAL, "handle lives on device " + std::to_string(dev) + " but device " +
                           std::to_string(cur) + " is current");
}

static int current_device() {
  int d = 0;
  PASTA_CUDA(cudaGetDevice(&d));
  return d;
}

static void validate_dims(uint32_t order, const uint32_t *dims) {
  require(order >= 1 && order <= kMaxOrder, "order must be in 1..PASTA_MAX_ORDER");
  require(dims != nullptr, "dims is NULL");
  for (uint32_t k = 0; k < order; ++k) require(dims[k] >= 1, "every dimension must be >= 1");
}

// Upload host arrays into a fresh handle (indices already validated).
static std::unique_ptr<pasta_coo> coo_upload(uint32_t order, const uint32_t *dims, uint64_t nnz,
                                             const uint32_t *const *inds, const float *vals,
                                             cudaStream_t s) {
  auto x = std::make_unique<pasta_coo>();
  x->order = order;
  for (uint32_t k = 0; k < order; ++k) x->dims[k] = dims[k];
  x->nnz = nnz;
  x->device = current_device();
  for (uint32_t k = 0; k < order; ++k) {
    x->inds[k].alloc(nnz, s);
    if (nnz)
      PASTA_CUDA(cudaMemcpyAsync(x->inds[k].p, inds[k], nnz * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
  }
  x->val.alloc(nnz, s);
  if (nnz) PASTA_CUDA(cudaMemcpyAsync(x->val.p, vals, nnz * sizeof(float), cudaMemcpyHostToDevice, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  const uint32_t *ip[kMaxOrder];
  for (uint32_t k = 0; k < order; ++k) ip[k] = x->inds[k].p;
  x->lex_sorted = is_lex_sorted_device(ip, order, nnz, s);
  return x;
}

pasta_coo::~pasta_coo() {
  for (auto *f : fib) delete f;
}

namespace pasta {

void coo_prepare_mode(pasta_coo *x, uint32_t mode, cudaStream_t s) {
  CooModeCopy &mc = x->mc[mode];
  if (mc.ready) return;
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  if (mode == 0 && x->lex_sorted) {  // canonical order already is the mode-0 order
    for (uint32_t k = 0; k < N; ++k) mc.inds[k] = x->inds[k].p;
    mc.val = x->val.p;
    mc.ready = true;
    return;
  }
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  const uint32_t *comps[kMaxOrder];
  uint32_t bits[kMaxOrder];
  for (uint32_t j = 0; j < N; ++j) {
    uint32_t k = (mode + j) % N;
    comps[j] = x->inds[k].p;
    bits[j] = ceil_log2(x->dims[k]);
  }
  lexsort(comps, bits, int(N), perm, M, s);
  for (uint32_t k = 0; k < N; ++k) {
    mc.own_inds[k].alloc(M, s);
    gather_u32(x->inds[k].p, perm.p, mc.own_inds[k].p, M, s);
    mc.inds[k] = mc.own_inds[k].p;
  }
  mc.own_val.alloc(M, s);
  gather_f32(x->val.p, perm.p, mc.own_val.p, M, s);
  mc.val = mc.own_val.p;
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.ready = true;
}

}  // namespace pasta

// ================================================================== extern "C" ABI ======
extern "C" {

const char *pasta_last_error(void) { return t_last_error.c_str(); }

const char *pasta_version(void) { return "pasta-b200 0.1 sm_100a"; }

pasta_status pasta_set_allocator(const pasta_allocator *alloc) {
  API_BEGIN
  std::lock_guard<std::mutex> lk(g_alloc_mu);
  if (alloc) {
    require(alloc->alloc && alloc->free, "allocator hook needs both alloc and free");
    g_alloc = *alloc;
    g_alloc_set = true;
  } else {
    g_alloc = pasta_allocator{nullptr, nullptr, nullptr};
    g_alloc_set = false;
  }
  API_END
}

// ---------------------------------------------------------------------------- ingest
// Binary tensor cache (.pbin, R#17): little-endian "PASTAB01", u32 order, u32 0, u64 nnz,
// u32 dims[order], then order x nnz u32 indices (0-based, mode after mode), nnz f32 values.
static const char kPbinMagic[8] = {'P', 'A', 'S', 'T', 'A', 'B', '0', '1'};

static std::unique_ptr<pasta_coo> load_pbin(FILE *f, const char *path) {
  struct Closer { FILE *f; ~Closer() { std::fclose(f); } } closer{f};
  uint32_t head[2];
  uint64_t nnz = 0;
  if (std::fread(head, 4, 2, f) != 2 || std::fread(&nnz, 8, 1, f) != 1)
    fail(PASTA_EFORMAT, std::string("truncated .pbin header in ") + path);
  const uint32_t order = head[0];
  if (order < 1 || order > kMaxOrder || head[1] != 0) fail(PASTA_EFORMAT, "bad .pbin header (order / flags)");
  if (nnz > 0xFFFFFFFEull) fail(PASTA_ERANGE, "more than 2^32-2 nonzeros");
  uint32_t dims[kMaxOrder];
  if (std::fread(dims, 4, order, f) != order) fail(PASTA_EFORMAT, "truncated .pbin dims");
  validate_dims(order, dims);
  // the file must hold exactly the arrays the header announces
  const long here = std::ftell(f);
  std::fseek(f, 0, SEEK_END);
  const uint64_t size = uint64_t(std::ftell(f));
  std::fseek(f, here, SEEK_SET);
  if (size != uint64_t(here) + (uint64_t(order) + 1) * 4 * nnz)
    fail(PASTA_EFORMAT, std::string(".pbin size does not match its header: ") + path);
  std::vector<std::vector<uint32_t>> inds(order, std::vector<uint32_t>(nnz));
  std::vector<float> vals(nnz);
  for (uint32_t k = 0; k < order; ++k) {
    if (std::fread(inds[k].data(), 4, nnz, f) != nnz) fail(PASTA_EIO, std::string("read error on ") + path);
    for (uint64_t i = 0; i < nnz; ++i)
      if (inds[k][i] >= dims[k])
        fail(PASTA_ERANGE, "index " + std::to_string(inds[k][i]) + " >= dims[" + std::to_string(k) + "]");
  }
  if (std::fread(vals.data(), 4, nnz, f) != nnz) fail(PASTA_EIO, std::string("read error on ") + path);
  const uint32_t *ip[kMaxOrder];
  for (uint32_t k = 0; k < order; ++k) ip[k] = inds[k].data();
  return coo_upload(order, dims, nnz, ip, vals.data(), nullptr);
}

pasta_status pasta_load_coo(const char *path, pasta_coo **out) {
  API_BEGIN
  require(path && out, "path/out is NULL");
  *out = nullptr;
  FILE *f = std::fopen(path, "rb");
  if (!f) fail(PASTA_EIO, std::string("cannot open ") + path);
  {
    char magic[8] = {};
    const size_t got = std::fread(magic, 1, 8, f);
    if (got == 8 && std::memcmp(magic, kPbinMagic, 8) == 0) {
      *out = load_pbin(f, path).release();
      return PASTA_OK;
    }
    std::rewind(f);
  }
  std::string text;
  {
    char buf[1 << 16];
    size_t got;
    while ((got = std::fread(buf, 1, sizeof(buf), f)) > 0) text.append(buf, got);
    bool err = std::ferror(f);
    std::fclose(f);
    if (err) fail(PASTA_EIO, std::string("read error on ") + path);
  }
  std::vector<std::vector<uint32_t>> inds;
  std::vector<float> vals;
  uint32_t order = 0;
  std::vector<uint32_t> dims;
  size_t pos = 0, line_no = 0;
  std::vector<std::string> tok;
  while (pos < text.size()) {
    size_t eol = text.find('\n', pos);
    if (eol == std::string::npos) eol = text.size();
    ++line_no;
    const char *p = text.c_str() + pos, *end = text.c_str() + eol;
    pos = eol + 1;
    while (p < end && (*p == ' ' || *p == '\t' || *p == '\r')) ++p;
    if (p == end || *p == '#') continue;
    tok.clear();
    while (p < end) {
      const char *q = p;
      while (q < end && *q != ' ' && *q != '\t' && *q != '\r') ++q;
      tok.emplace_back(p, q);
      p = q;
      while (p < end && (*p == ' ' || *p == '\t' || *p == '\r')) ++p;
    }
    if (order == 0) {
      if (tok.size() < 2 || tok.size() - 1 > kMaxOrder)
        fail(PASTA_EFORMAT, "line " + std::to_string(line_no) + ": expected 2..9 tokens");
      order = uint32_t(tok.size() - 1);
      inds.resize(order);
      dims.assign(order, 0);
    }
    if (tok.size() != order + 1)
      fail(PASTA_EFORMAT, "line " + std::to_string(line_no) + ": ragged line");
    for (uint32_t k = 0; k < order; ++k) {
      errno = 0;
      char *e = nullptr;
      unsigned long long v = std::strtoull(tok[k].c_str(), &e, 10);
      if (errno || !e || *e != '\0' || tok[k][0] == '-')
        fail(PASTA_EFORMAT, "line " + std::to_string(line_no) + ": bad index '" + tok[k] + "'");
      if (v == 0) fail(PASTA_EFORMAT, "line " + std::to_string(line_no) + ": indices are 1-based");
      if (v > 0xFFFFFFFFull) fail(PASTA_ERANGE, "line " + std::to_string(line_no) + ": index too large");
      inds[k].push_back(uint32_t(v - 1));
      if (uint32_t(v) > dims[k]) dims[k] = uint32_t(v);
    }
    errno = 0;
    char *e = nullptr;
    float fv = std::strtof(tok[order].c_str(), &e);
    if (!e || *e != '\0') fail(PASTA_EFORMAT, "line " + std::to_string(line_no) + ": bad value");
    vals.push_back(fv);
    if (vals.size() > 0xFFFFFFFEull) fail(PASTA_ERANGE, "more than 2^32-2 nonzeros");
  }
  if (order == 0) fail(PASTA_EFORMAT, std::string("no nonzeros in ") + path);
  const uint32_t *ip[kMaxOrder];
  for (uint32_t k = 0; k < order; ++k) ip[k] = inds[k].data();
  auto x = coo_upload(order, dims.data(), vals.size(), ip, vals.data(), nullptr);
  *out = x.release();
  API_END
}

pasta_status pasta_save_coo(const pasta_coo *x, const char *path) {
  API_BEGIN
  require(x && path, "x/path is NULL");
  check_device(x->device);
  std::vector<std::vector<uint32_t>> h(x->order, std::vector<uint32_t>(x->nnz));
  std::vector<float> v(x->nnz);
  for (uint32_t k = 0; k < x->order; ++k)
    if (x->nnz) PASTA_CUDA(cudaMemcpy(h[k].data(), x->inds[k].p, x->nnz * 4, cudaMemcpyDeviceToHost));
  if (x->nnz) PASTA_CUDA(cudaMemcpy(v.data(), x->val.p, x->nnz * 4, cudaMemcpyDeviceToHost));
  FILE *f = std::fopen(path, "wb");
  if (!f) fail(PASTA_EIO, std::string("cannot create ") + path);
  const size_t plen = std::strlen(path);
  if (plen >= 5 && std::strcmp(path + plen - 5, ".pbin") == 0) {  // binary cache
    const uint32_t head[2] = {x->order, 0};
    const uint64_t nnz = x->nnz;
    bool ok = std::fwrite(kPbinMagic, 1, 8, f) == 8 && std::fwrite(head, 4, 2, f) == 2 &&
              std::fwrite(&nnz, 8, 1, f) == 1 && std::fwrite(x->dims, 4, x->order, f) == x->order;
    for (uint32_t k = 0; k < x->order && ok; ++k) ok = std::fwrite(h[k].data(), 4, nnz, f) == nnz;
    ok = ok && std::fwrite(v.data(), 4, nnz, f) == nnz;
    ok = (std::fclose(f) == 0) && ok;
    if (!ok) fail(PASTA_EIO, std::string("write error on ") + path);
    return PASTA_OK;
  }
  bool ok = true;
  for (uint64_t i = 0; i < x->nnz && ok; ++i) {
    for (uint32_t k = 0; k < x->order; ++k) ok &= std::fprintf(f, "%u ", h[k][i] + 1) > 0;
    ok &= std::fprintf(f, "%.9g\n", double(v[i])) > 0;
  }
  ok &= std::fclose(f) == 0;
  if (!ok) fail(PASTA_EIO, std::string("write error on ") + path);
  API_END
}

pasta_status pasta_coo_from_arrays(uint32_t order, const uint32_t *dims, uint64_t nnz,
                                   const uint32_t *const *inds, const float *vals, pasta_coo **out) {
  API_BEGIN
  require(out != nullptr, "out is NULL");
  *out = nullptr;
  validate_dims(order, dims);
  require(nnz == 0 || (inds && vals), "inds/vals is NULL");
  if (nnz > 0xFFFFFFFEull) fail(PASTA_ERANGE, "more than 2^32-2 nonzeros");
  for (uint32_t k = 0; k < order && nnz; ++k) {
    require(inds[k] != nullptr, "inds[k] is NULL");
    for (uint64_t i = 0; i < nnz; ++i)
      if (inds[k][i] >= dims[k])
        fail(PASTA_ERANGE, "index " + std::to_string(inds[k][i]) + " >= dims[" + std::to_string(k) + "]");
  }
  auto x = coo_upload(order, dims, nnz, inds, vals, nullptr);
  *out = x.release();
  API_END
}

pasta_status pasta_gen_powerlaw(uint32_t order, const uint32_t *dims, uint64_t nnz, uint64_t seed,
                                const pasta_gen_params *params, pasta_coo **out) {
  API_BEGIN
  require(out != nullptr, "out is NULL");
  *out = nullptr;
  validate_dims(order, dims);
  pasta_gen_params p{1, nullptr, 0.0, 0, 0.f, 0.f, 0.0};
  if (params) p = *params;
  require(p.kind <= 2, "unknown generator kind");
  require(p.permute <= 1, "permute must be 0 or 1");
  double cells = 1.0;
  for (uint32_t k = 0; k < order; ++k) cells *= double(dims[k]);
  require(double(nnz) <= cells, "nnz exceeds the number of cells");
  if (nnz > 0xFFFFFFFEull) fail(PASTA_ERANGE, "more than 2^32-2 nonzeros");
  if (p.kind == 2) {
    const double alpha = p.alpha == 0.0 ? 1.0 : p.alpha;
    require(alpha > 0.0 && alpha <= 8.0, "alpha must be in (0, 8] (0 selects the default 1.0)");
    for (uint32_t k = 0; k < order; ++k)
      if (dims[k] > (1u << 27)) fail(PASTA_ERANGE, "slice power law: dims above 2^27 (weight table)");
    float lo = p.val_lo, hi = p.val_hi;
    if (lo == 0.f && hi == 0.f) { lo = -1.f; hi = 1.f; }
    require(lo < hi, "val_lo must be < val_hi");
    auto x = std::make_unique<pasta_coo>();
    x->order = order;
    for (uint32_t k = 0; k < order; ++k) x->dims[k] = dims[k];
    x->nnz = nnz;
    x->device = current_device();
    gen_powerlaw_device(x.get(), seed, nullptr, 0, lo, hi, nullptr, alpha);
    if (p.permute) relabel_device(x.get(), seed, nullptr);
    x->lex_sorted = true;
    *out = x.release();
    return PASTA_OK;
  }
  const uint32_t ncell = 1u << order;
  double table[1 << kMaxOrder];
  if (p.kind == 0) {
    for (uint32_t c = 0; c < ncell; ++c) {
      double v = 1.0;
      for (uint32_t k = 0; k < order; ++k) v = v * 0.5;
      table[c] = v;
    }
  } else if (p.initiator) {
    double sum = 0.0;
    for (uint32_t c = 0; c < ncell; ++c) {
      require(p.initiator[c] >= 0.0 && std::isfinite(p.initiator[c]), "initiator weights must be >= 0");
      table[c] = p.initiator[c];
      sum += table[c];
    }
    require(sum > 0.0, "initiator weights sum to zero");
  } else {
    double q = (p.q > 0.0 && p.q < 1.0) ? p.q : 0.75;
    require(p.q == 0.0 || (p.q > 0.0 && p.q < 1.0), "q must be in (0, 1)");
    for (uint32_t c = 0; c < ncell; ++c) {
      double v = 1.0;
      for (uint32_t k = 0; k < order; ++k) v = v * (((c >> k) & 1u) ? (1.0 - q) : q);
      table[c] = v;
    }
  }
  float lo = p.val_lo, hi = p.val_hi;
  if (lo == 0.f && hi == 0.f) { lo = -1.f; hi = 1.f; }
  require(lo < hi, "val_lo must be < val_hi");
  auto x = std::make_unique<pasta_coo>();
  x->order = order;
  for (uint32_t k = 0; k < order; ++k) x->dims[k] = dims[k];
  x->nnz = nnz;
  x->device = current_device();
  gen_powerlaw_device(x.get(), seed, table, ncell, lo, hi, nullptr);
  if (p.permute) relabel_device(x.get(), seed, nullptr);
  x->lex_sorted = true;
  *out = x.release();
  API_END
}

// ---------------------------------------------------------------------------- formats
pasta_status pasta_coo_to_hicoo(const pasta_coo *x, uint32_t block_bits, pasta_hicoo **out) {
  API_BEGIN
  require(x && out, "x/out is NULL");
  *out = nullptr;
  require(block_bits >= 1 && block_bits <= 8, "block_bits must be in 1..8 (8-bit element indices, P:181)");
  check_device(x->device);
  auto h = std::make_unique<pasta_hicoo>();
  h->order = x->order;
  for (uint32_t k = 0; k < x->order; ++k) h->dims[k] = x->dims[k];
  h->block_bits = block_bits;
  h->cmask = (1u << x->order) - 1u;
  h->device = x->device;
  coo_to_hicoo_device(x, h.get(), nullptr);
  *out = h.release();
  API_END
}

// gHiCOO storage in bytes (R#29): per nonzero 1 B per compressed mode, 4 B per uncompressed
// mode, 4 B value; per block 8 B bptr + 4 B binds per compressed mode.
static uint64_t ghicoo_bytes(uint32_t order, uint32_t cmask, uint64_t M, uint64_t nb) {
  uint32_t nc = uint32_t(__builtin_popcount(cmask)), nu = order - nc;
  return (uint64_t(nc) + 4ull * nu + 4ull) * M + (8ull + 4ull * nc) * nb;
}

static uint32_t choose_ghicoo_mask(const pasta_coo *x, uint32_t block_bits, uint64_t *bytes) {
  const uint32_t N = x->order;
  const uint32_t full = (1u << N) - 1u;
  uint32_t best = full;
  uint64_t best_b = ~0ull;
  auto cost = [&](uint32_t m) {
    return ghicoo_bytes(N, m, x->nnz, count_blocks_device(x, block_bits, m, nullptr));
  };
  if (N <= 4) {  // exhaustive, ascending mask value; strict improvement keeps the smallest mask
    for (uint32_t m = 1; m <= full; ++m) {
      uint64_t c = cost(m);
      if (c < best_b) { best_b = c; best = m; }
    }
  } else {  // greedy forward selection from the best single mode
    for (uint32_t k = 0; k < N; ++k) {
      uint64_t c = cost(1u << k);
      if (c < best_b) { best_b = c; best = 1u << k; }
    }
    for (bool grew = true; grew;) {
      grew = false;
      uint32_t cand = best;
      uint64_t cand_b = best_b;
      for (uint32_t k = 0; k < N; ++k) {
        if ((best >> k) & 1u) continue;
        uint64_t c = cost(best | (1u << k));
        if (c < cand_b) { cand_b = c; cand = best | (1u << k); }
      }
      if (cand != best) { best = cand; best_b = cand_b; grew = true; }
    }
  }
  if (bytes) *bytes = best_b;
  return best;
}

pasta_status pasta_ghicoo_auto_mask(const pasta_coo *x, uint32_t block_bits, uint32_t *cmask,
                                    uint64_t *bytes) {
  API_BEGIN
  require(x && cmask, "x/cmask is NULL");
  require(block_bits >= 1 && block_bits <= 8, "block_bits must be in 1..8 (8-bit element indices, P:181)");
  check_device(x->device);
  *cmask = choose_ghicoo_mask(x, block_bits, bytes);
  API_END
}

pasta_status pasta_coo_to_ghicoo(const pasta_coo *x, uint32_t block_bits, uint32_t cmask,
                                 pasta_hicoo **out) {
  API_BEGIN
  require(x && out, "x/out is NULL");
  *out = nullptr;
  require(block_bits >= 1 && block_bits <= 8, "block_bits must be in 1..8 (8-bit element indices, P:181)");
  require((cmask >> x->order) == 0, "cmask has bits >= order");
  check_device(x->device);
  if (cmask == 0) cmask = choose_ghicoo_mask(x, block_bits, nullptr);
  auto h = std::make_unique<pasta_hicoo>();
  h->order = x->order;
  for (uint32_t k = 0; k < x->order; ++k) h->dims[k] = x->dims[k];
  h->block_bits = block_bits;
  h->cmask = cmask;
  h->device = x->device;
  coo_to_hicoo_device(x, h.get(), nullptr);
  *out = h.release();
  API_END
}

pasta_status pasta_coo_prepare(pasta_coo *x, uint32_t mode, void *stream) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  std::lock_guard<std::mutex> lk(x->mu);
  coo_prepare_mode(x, mode, as_stream(stream));
  API_END
}

pasta_status pasta_coo_release_mode(pasta_coo *x, uint32_t mode) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  std::lock_guard<std::mutex> lk(x->mu);
  CooModeCopy &mc = x->mc[mode];
  if (mc.fence.e) PASTA_CUDA(cudaEventSynchronize(mc.fence.e));  // launches still reading it
  for (uint32_t k = 0; k < kMaxOrder; ++k) {
    mc.own_inds[k].reset();
    mc.hot_inds[k].reset();
    mc.inds[k] = nullptr;
  }
  mc.own_val.reset();
  mc.val = nullptr;
  mc.hot_rows.reset();
  mc.hot_buf.reset();
  mc.hs_rows.reset();
  mc.split_irow.reset();
  mc.split_val.reset();
  mc.claim.reset();
  mc.hot_R = 0;
  mc.hot_total = mc.hs_total = 0;
  mc.split = false;
  mc.ready = false;
  API_END
}

pasta_status pasta_hicoo_prepare(pasta_hicoo *h, uint32_t mode, void *stream) {
  API_BEGIN
  require(h != nullptr, "h is NULL");
  require(mode < h->order, "mode >= order");
  check_device(h->device);
  std::lock_guard<std::mutex> lk(h->mu);
  hicoo_prepare_mode(h, mode, as_stream(stream));
  API_END
}

// ---------------------------------------------------------------------------- MTTKRP
static void validate_mttkrp(uint32_t order, uint32_t mode, const float *const *factors, uint32_t R,
                            const float *out) {
  require(mode < order, "mode >= order");
  require(R >= 1, "R must be >= 1");
  require(factors != nullptr, "factors is NULL");
  require(out != nullptr, "out is NULL");
  for (uint32_t k = 0; k < order; ++k)
    if (k != mode) require(factors[k] != nullptr, "factors[k] is NULL for a mode k != mode");
}

pasta_status pasta_mttkrp_coo(pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                              float *out, void *stream) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  validate_mttkrp(x->order, mode, factors, R, out);
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  // the handle's per-mode caches (sorted copy, hot-row tiers) are built / refilled under the
  // handle's lock; the launches are only enqueued while it is held
  std::lock_guard<std::mutex> lk(x->mu);
  if (!x->mc[mode].ready) coo_prepare_mode(x, mode, s);
  uint64_t lo = 0, hi = x->dims[mode];
  if (x->shard_mode == int(mode)) { lo = x->row_lo; hi = x->row_hi; }
  launch_zero_rows(out, lo, hi, R, s);
  launch_coo_mttkrp(x, mode, factors, R, out, s);
  API_END
}

pasta_status pasta_mttkrp_coo_bcast(pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                                    float *const *outs, uint32_t nout, void *stream) {
  API_BEGIN
  require(x != nullptr && outs != nullptr, "x/outs is NULL");
  require(nout >= 1 && nout <= kMaxOrder, "nout must be 1..8");
  for (uint32_t d = 0; d < nout; ++d) {
    require(outs[d] != nullptr, "outs[d] is NULL");
    require((reinterpret_cast<uintptr_t>(outs[d]) & 15) == 0, "outs[d] must be 16-byte aligned");
  }
  validate_mttkrp(x->order, mode, factors, R, outs[0]);
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  std::lock_guard<std::mutex> lk(x->mu);
  if (!x->mc[mode].ready) coo_prepare_mode(x, mode, s);
  uint64_t lo = 0, hi = x->dims[mode];
  if (x->shard_mode == int(mode)) { lo = x->row_lo; hi = x->row_hi; }
  for (uint32_t d = 0; d < nout; ++d) launch_zero_rows(outs[d], lo, hi, R, s);  // owned rows, every replica
  launch_coo_mttkrp_bcast(x, mode, factors, R, outs, nout, s);
  API_END
}

pasta_status pasta_mttkrp_hicoo(pasta_hicoo *h, uint32_t mode, const float *const *factors, uint32_t R,
                                float *out, void *stream) {
  API_BEGIN
  require(h != nullptr, "h is NULL");
  validate_mttkrp(h->order, mode, factors, R, out);
  check_device(h->device);
  cudaStream_t s = as_stream(stream);
  std::lock_guard<std::mutex> lk(h->mu);
  if (!h->mc[mode].ready) hicoo_prepare_mode(h, mode, s);
  uint64_t lo = 0, hi = h->dims[mode];
  if (h->shard_mode == int(mode)) { lo = h->row_lo; hi = h->row_hi; }
  launch_zero_rows(out, lo, hi, R, s);
  launch_hicoo_mttkrp(h, mode, factors, R, out, s);
  API_END
}

// nsteps independent all-modes steps from/to host buffers (step i: host_factors[i*N + k],
// host_out[i*N + m]).  Pipelined: factors go up on a copy stream in the order the modes need
// them (U1..U_{N-1}, then U0), mode m's kernel starts as soon as its factors have landed, its
// result goes down on a second copy stream while later modes compute (PCIe/C2C is full
// duplex), and with nsteps > 1 step i+1's uploads (slot (i+1) & 1) overlap step i's
// downloads.  Returns after the last result is in host memory.
static void allmodes_host_steps(pasta_coo *x, uint32_t nsteps, const float *const *host_factors,
                                uint32_t R, float *const *host_out, cudaStream_t s) {
  const uint32_t N = x->order;
  for (uint32_t k = 0; k < N; ++k) coo_prepare_mode(x, k, s);
  const int nslots = nsteps > 1 ? 2 : 1;
  for (int b = 0; b < nslots; ++b) {
    if (x->stage_R[b] == R) continue;
    for (uint32_t k = 0; k < N; ++k) {
      x->stage_f[b][k].alloc(uint64_t(x->dims[k]) * R, s);
      x->stage_o[b][k].alloc(uint64_t(x->dims[k]) * R, s);
    }
    x->stage_R[b] = R;
  }
  E2EStreams &e = x->e2e;
  e.init();
  PASTA_CUDA(cudaEventRecord(e.start, s));
  PASTA_CUDA(cudaStreamWaitEvent(e.h2d, e.start, 0));
  PASTA_CUDA(cudaStreamWaitEvent(e.d2h, e.start, 0));
  for (uint32_t i = 0; i < nsteps; ++i) {
    const int b = int(i & 1u);
    const float *const *hf = host_factors + size_t(i) * N;
    float *const *ho = host_out + size_t(i) * N;
    const float *dfac[kMaxOrder];
    if (i >= 2) PASTA_CUDA(cudaStreamWaitEvent(e.h2d, e.kd[b], 0));  // step i-2 done reading
    for (uint32_t j = 0; j < N; ++j) {
      const uint32_t k = (j + 1) % N;  // 1, 2, ..., N-1, 0
      PASTA_CUDA(cudaMemcpyAsync(x->stage_f[b][k].p, hf[k], uint64_t(x->dims[k]) * R * sizeof(float),
                                 cudaMemcpyHostToDevice, e.h2d));
      PASTA_CUDA(cudaEventRecord(e.f[b][k], e.h2d));
      dfac[k] = x->stage_f[b][k].p;
    }
    for (uint32_t m = 0; m < N; ++m) {
      for (uint32_t k = 0; k < N; ++k)
        if (k != m) PASTA_CUDA(cudaStreamWaitEvent(s, e.f[b][k], 0));
      if (i >= 2) PASTA_CUDA(cudaStreamWaitEvent(s, e.od[b][m], 0));  // step i-2's result is out
      uint64_t lo = 0, hi = x->dims[m];
      if (x->shard_mode == int(m)) { lo = x->row_lo; hi = x->row_hi; }
      launch_zero_rows(x->stage_o[b][m].p, lo, hi, R, s);
      launch_coo_mttkrp(x, m, dfac, R, x->stage_o[b][m].p, s);
      PASTA_CUDA(cudaEventRecord(e.o[b][m], s));
      PASTA_CUDA(cudaStreamWaitEvent(e.d2h, e.o[b][m], 0));
      // only the rows this handle owns go down (a shard leaves the host's other rows alone)
      PASTA_CUDA(cudaMemcpyAsync(ho[m] + lo * R, x->stage_o[b][m].p + lo * R, (hi - lo) * R * sizeof(float),
                                 cudaMemcpyDeviceToHost, e.d2h));
      PASTA_CUDA(cudaEventRecord(e.od[b][m], e.d2h));
    }
    PASTA_CUDA(cudaEventRecord(e.kd[b], s));
  }
  PASTA_CUDA(cudaStreamSynchronize(e.d2h));
  PASTA_CUDA(cudaStreamSynchronize(e.h2d));
  PASTA_CUDA(cudaStreamSynchronize(s));
}

pasta_status pasta_mttkrp_coo_allmodes_host(pasta_coo *x, const float *const *host_factors, uint32_t R,
                                            float *const *host_out, void *stream) {
  API_BEGIN
  require(x && host_factors && host_out, "x/host_factors/host_out is NULL");
  require(R >= 1, "R must be >= 1");
  for (uint32_t k = 0; k < x->order; ++k)
    require(host_factors[k] && host_out[k], "host_factors[k]/host_out[k] is NULL");
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  std::lock_guard<std::mutex> lk(x->mu);
  allmodes_host_steps(x, 1, host_factors, R, host_out, s);
  API_END
}

pasta_status pasta_mttkrp_coo_allmodes_host_batch(pasta_coo *x, uint32_t nsteps, const float *const *host_factors,
                                                  uint32_t R, float *const *host_out, void *stream) {
  API_BEGIN
  require(x && host_factors && host_out, "x/host_factors/host_out is NULL");
  require(R >= 1, "R must be >= 1");
  for (uint64_t k = 0; k < uint64_t(nsteps) * x->order; ++k)
    require(host_factors[k] && host_out[k], "host_factors[i*order+k]/host_out[i*order+k] is NULL");
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  std::lock_guard<std::mutex> lk(x->mu);
  if (nsteps) allmodes_host_steps(x, nsteps, host_factors, R, host_out, s);
  API_END
}

pasta_status pasta_coo_release_staging(pasta_coo *x) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  check_device(x->device);
  std::lock_guard<std::mutex> lk(x->mu);
  if (x->e2e.ready) {
    for (int b = 0; b < 2; ++b)
      for (uint32_t m = 0; m < x->order; ++m) PASTA_CUDA(cudaEventSynchronize(x->e2e.od[b][m]));
  }
  for (int b = 0; b < 2; ++b) {
    for (uint32_t k = 0; k < pasta::kMaxOrder; ++k) {
      x->stage_f[b][k].reset();
      x->stage_o[b][k].reset();
    }
    x->stage_R[b] = 0;
  }
  API_END
}

// ---------------------------------------------------------------------------- multi-GPU
pasta_status pasta_coo_row_counts(const pasta_coo *x, uint32_t mode, uint64_t *counts) {
  API_BEGIN
  require(x && counts, "x/counts is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  row_counts_device(x->inds[mode].p, x->nnz, x->dims[mode], counts, nullptr);
  API_END
}

pasta_status pasta_row_partition(uint32_t nrows, const uint64_t *counts, uint32_t nparts,
                                 uint32_t *bounds) {
  API_BEGIN
  require(nparts >= 1, "nparts must be >= 1");
  require(bounds != nullptr && (nrows == 0 || counts != nullptr), "counts/bounds is NULL");
  // S(r) = sum_{i<r} counts[i];  bounds[p] = min{r : S(r) * nparts >= p * T}
  unsigned __int128 T = 0;
  for (uint32_t r = 0; r < nrows; ++r) T += counts[r];
  bounds[0] = 0;
  uint32_t p = 1;
  unsigned __int128 S = 0;
  for (uint32_t r = 0; r <= nrows && p < nparts; ++r) {
    while (p < nparts && S * nparts >= T * p) bounds[p++] = r;
    if (r < nrows) S += counts[r];
  }
  while (p < nparts) bounds[p++] = nrows;
  bounds[nparts] = nrows;
  API_END
}

pasta_status pasta_coo_partition(const pasta_coo *x, uint32_t mode, uint32_t nparts, uint32_t *bounds) {
  API_BEGIN
  require(x && bounds, "x/bounds is NULL");
  require(mode < x->order, "mode >= order");
  std::vector<uint64_t> counts(x->dims[mode]);
  pasta_status st = pasta_coo_row_counts(x, mode, counts.data());
  if (st != PASTA_OK) fail(st, t_last_error);
  st = pasta_row_partition(x->dims[mode], counts.data(), nparts, bounds);
  if (st != PASTA_OK) fail(st, t_last_error);
  API_END
}

pasta_status pasta_hicoo_shard(const pasta_hicoo *h, uint32_t mode, uint32_t row_lo, uint32_t row_hi,
                              pasta_hicoo **out) {
  API_BEGIN
  require(h && out, "h/out is NULL");
  *out = nullptr;
  require(mode < h->order, "mode >= order");
  require(row_lo <= row_hi && row_hi <= h->dims[mode], "need row_lo <= row_hi <= dims[mode]");
  check_device(h->device);
  auto y = std::make_unique<pasta_hicoo>();
  hicoo_shard_device(h, mode, row_lo, row_hi, y.get(), nullptr);
  *out = y.release();
  API_END
}

pasta_status pasta_coo_shard(pasta_coo *x, uint32_t mode, uint32_t row_lo, uint32_t row_hi,
                             pasta_coo **out) {
  API_BEGIN
  require(x && out, "x/out is NULL");
  *out = nullptr;
  require(mode < x->order, "mode >= order");
  require(row_lo <= row_hi && row_hi <= x->dims[mode], "need row_lo <= row_hi <= dims[mode]");
  check_device(x->device);
  cudaStream_t s = nullptr;
  {
    std::lock_guard<std::mutex> lk(x->mu);
    coo_prepare_mode(x, mode, s);
  }
  const CooModeCopy &mc = x->mc[mode];
  uint64_t a = lower_bound_device(mc.inds[mode], x->nnz, row_lo, s);
  uint64_t b = row_hi >= x->dims[mode] ? x->nnz : lower_bound_device(mc.inds[mode], x->nnz, row_hi, s);
  auto y = std::make_unique<pasta_coo>();
  y->order = x->order;
  for (uint32_t k = 0; k < x->order; ++k) y->dims[k] = x->dims[k];
  y->nnz = b - a;
  y->device = x->device;
  for (uint32_t k = 0; k < x->order; ++k) {
    y->inds[k].alloc(y->nnz, s);
    if (y->nnz)
      PASTA_CUDA(cudaMemcpyAsync(y->inds[k].p, mc.inds[k] + a, y->nnz * 4, cudaMemcpyDeviceToDevice, s));
  }
  y->val.alloc(y->nnz, s);
  if (y->nnz) PASTA_CUDA(cudaMemcpyAsync(y->val.p, mc.val + a, y->nnz * 4, cudaMemcpyDeviceToDevice, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  y->lex_sorted = (mode == 0) ? true : false;
  CooModeCopy &ym = y->mc[mode];
  for (uint32_t k = 0; k < y->order; ++k) ym.inds[k] = y->inds[k].p;
  ym.val = y->val.p;
  ym.ready = true;
  y->shard_mode = int(mode);
  y->row_lo = row_lo;
  y->row_hi = row_hi;
  *out = y.release();
  API_END
}

// ---------------------------------------------------------------------------- CP-ALS
static void require_R64(uint32_t R) {
  require(R >= 1, "R must be >= 1");
  if (R > 64) fail(PASTA_EUNSUPPORTED, "CP-ALS supports R <= 64");
}

pasta_status pasta_gram(const float *U, uint64_t rows, uint32_t R, double *G, void *stream) {
  API_BEGIN
  require((U || !rows) && G, "U/G is NULL");
  require_R64(R);
  launch_gram(U, rows, R, G, as_stream(stream));
  API_END
}

pasta_status pasta_cpals_solve(const float *M, uint64_t rows, uint32_t R, const double *const *grams,
                               uint32_t ngrams, float *U, double *colsq, void *stream) {
  API_BEGIN
  require((M && U) || !rows, "M/U is NULL");
  require(colsq && (grams || !ngrams), "colsq/grams is NULL");
  require_R64(R);
  for (uint32_t k = 0; k < ngrams; ++k) require(grams[k] != nullptr, "grams[k] is NULL");
  launch_solve(M, rows, R, grams, ngrams, U, colsq, as_stream(stream));
  API_END
}

pasta_status pasta_cpals_prepare(const double *GM, const double *const *grams, uint32_t ngrams, uint32_t R,
                                 float *Wn, double *Gn, double *lambda, void *stream) {
  API_BEGIN
  require_R64(R);
  require(GM && Wn && Gn && lambda && (grams || ngrams == 0), "NULL argument");
  for (uint32_t k = 0; k < ngrams; ++k) require(grams[k] != nullptr, "grams[k] is NULL");
  launch_cpals_prep(GM, grams, ngrams, R, Wn, Gn, lambda, as_stream(stream));
  API_END
}

pasta_status pasta_cpals_fit(const double *const *grams, uint32_t ngrams, uint32_t R, const double *lambda,
                             const double *inner, double normx2, double *fit, void *stream) {
  API_BEGIN
  require_R64(R);
  require(grams && lambda && inner && fit, "NULL argument");
  for (uint32_t k = 0; k < ngrams; ++k) require(grams[k] != nullptr, "grams[k] is NULL");
  cudaStream_t s = as_stream(stream);
  DevArray<double> out(2, s);
  launch_cpals_fit(grams, ngrams, R, lambda, inner, normx2, out.p, s);
  PASTA_CUDA(cudaMemcpyAsync(fit, out.p, sizeof(double), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  API_END
}

pasta_status pasta_rows_times(const float *M, uint64_t rows, uint32_t R, const float *Wn, float *U,
                              void *stream) {
  API_BEGIN
  require_R64(R);
  require((M && U && Wn) || rows == 0, "NULL argument");
  if (rows) launch_apply(M, rows, R, Wn, U, as_stream(stream));
  API_END
}

pasta_status pasta_rows_times_bcast(const float *M, uint64_t row_lo, uint64_t row_hi, uint32_t R,
                                    const float *Wn, float *const *dsts, uint32_t ndst, void *stream) {
  API_BEGIN
  require(M && Wn && dsts, "NULL argument");
  require(row_lo <= row_hi, "row_lo > row_hi");
  for (uint32_t k = 0; k < ndst; ++k) require(dsts[k] != nullptr, "dsts[k] is NULL");
  launch_apply_bcast(M, row_lo, row_hi, R, Wn, dsts, ndst, as_stream(stream));
  API_END
}

// ---------------------------------------------------------------------------- peer memory
pasta_status pasta_bcast_f32(const float *src, uint64_t n, float *const *dsts, uint32_t ndst, void *stream) {
  API_BEGIN
  require((src && dsts) || n == 0, "NULL argument");
  for (uint32_t k = 0; k < ndst && dsts; ++k) require(dsts[k] != nullptr, "dsts[k] is NULL");
  launch_bcast(src, n, dsts, ndst, as_stream(stream));
  API_END
}


pasta_status pasta_dev_alloc(uint64_t bytes, void **ptr) {
  API_BEGIN
  require(ptr != nullptr, "ptr is NULL");
  *ptr = nullptr;
  PASTA_CUDA(cudaMalloc(ptr, bytes ? bytes : 1));
  API_END
}

pasta_status pasta_dev_free(void *ptr) {
  API_BEGIN
  if (ptr) PASTA_CUDA(cudaFree(ptr));
  API_END
}

pasta_status pasta_ipc_get_handle(void *base, void *handle) {
  API_BEGIN
  require(base && handle, "NULL argument");
  static_assert(sizeof(cudaIpcMemHandle_t) == PASTA_IPC_HANDLE_BYTES, "IPC handle size");
  cudaIpcMemHandle_t h;
  PASTA_CUDA(cudaIpcGetMemHandle(&h, base));
  std::memcpy(handle, &h, sizeof(h));
  API_END
}

pasta_status pasta_ipc_open(const void *handle, void **ptr) {
  API_BEGIN
  require(handle && ptr, "NULL argument");
  *ptr = nullptr;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  PASTA_CUDA(cudaIpcOpenMemHandle(ptr, h, cudaIpcMemLazyEnablePeerAccess));
  API_END
}

pasta_status pasta_ipc_close(void *ptr) {
  API_BEGIN
  if (ptr) PASTA_CUDA(cudaIpcCloseMemHandle(ptr));
  API_END
}

pasta_status pasta_normalize_columns(float *U, uint64_t rows, uint32_t R, const double *colsq,
                                     double *lambda, void *stream) {
  API_BEGIN
  require((U || !rows) && colsq && lambda, "U/colsq/lambda is NULL");
  require_R64(R);
  launch_normalize(U, rows, R, colsq, lambda, as_stream(stream));
  API_END
}

pasta_status pasta_weighted_inner(const float *A, const float *B, uint64_t rows, uint32_t R,
                                  const double *lambda, double *out, void *stream) {
  API_BEGIN
  require(((A && B) || !rows) && lambda && out, "A/B/lambda/out is NULL");
  require_R64(R);
  launch_inner(A, B, rows, R, lambda, out, as_stream(stream));
  API_END
}

pasta_status pasta_coo_norm2(const pasta_coo *x, double *out) {
  API_BEGIN
  require(x && out, "x/out is NULL");
  check_device(x->device);
  DevArray<double> d(1);
  PASTA_CUDA(cudaMemset(d.p, 0, sizeof(double)));
  launch_sumsq(x->val.p, x->nnz, d.p, nullptr);
  PASTA_CUDA(cudaMemcpy(out, d.p, sizeof(double), cudaMemcpyDeviceToHost));
  API_END
}

pasta_status pasta_cpals_coo(pasta_coo *x, uint32_t R, uint32_t max_iters, double tol,
                             float *const *factors, double *lambda, double *fit_history,
                             uint32_t *iters, void *stream) {
  API_BEGIN
  require(x && factors && lambda && (fit_history || !max_iters) && iters, "NULL argument");
  require_R64(R);
  const uint32_t N = x->order;
  for (uint32_t k = 0; k < N; ++k) require(factors[k] != nullptr, "factors[k] is NULL");
  require(N >= 2, "CP-ALS needs order >= 2");
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  std::lock_guard<std::mutex> lk(x->mu);  // the MTTKRPs below use the handle's caches
  for (uint32_t k = 0; k < N; ++k) coo_prepare_mode(x, k, s);
  uint64_t maxd = 0;
  for (uint32_t k = 0; k < N; ++k) maxd = x->dims[k] > maxd ? x->dims[k] : maxd;
  DevArray<float> Mbuf(maxd * R, s);
  DevArray<double> grams(uint64_t(N) * R * R, s), colsq(R, s), lam(R, s), scal(2, s), GM(uint64_t(R) * R, s);
  DevArray<float> Wn(uint64_t(R) * R, s);
  DevArray<double> fitbuf(2, s);
  // fused epilogue (default): gram of M, R x R algebra, one pass U = M Wn; PASTA_CPALS_FUSED=0
  // runs the unfused solve -> normalise -> gram sequence
  const char *fz = getenv("PASTA_CPALS_FUSED");
  const bool fused = !(fz && *fz == '0');
  auto G = [&](uint32_t k) { return grams.p + uint64_t(k) * R * R; };
  PASTA_CUDA(cudaMemsetAsync(grams.p, 0, grams.bytes(), s));
  for (uint32_t k = 0; k < N; ++k) launch_gram(factors[k], x->dims[k], R, G(k), s);
  PASTA_CUDA(cudaMemsetAsync(scal.p, 0, scal.bytes(), s));
  launch_sumsq(x->val.p, x->nnz, scal.p, s);
  double normx2 = 0.0;
  PASTA_CUDA(cudaMemcpyAsync(&normx2, scal.p, sizeof(double), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  double prev = 0.0;
  uint32_t it = 0;
  const float *cf[kMaxOrder];
  for (uint32_t k = 0; k < N; ++k) cf[k] = factors[k];
  for (; it < max_iters; ++it) {
    for (uint32_t n = 0; n < N; ++n) {
      launch_zero_rows(Mbuf.p, 0, x->dims[n], R, s);
      launch_coo_mttkrp(x, n, cf, R, Mbuf.p, s);
      const double *gl[kMaxOrder];
      uint32_t ng = 0;
      for (uint32_t k = 0; k < N; ++k)
        if (k != n) gl[ng++] = G(k);
      if (fused) {
        PASTA_CUDA(cudaMemsetAsync(GM.p, 0, GM.bytes(), s));
        launch_gram(Mbuf.p, x->dims[n], R, GM.p, s);
        launch_cpals_prep(GM.p, gl, ng, R, Wn.p, G(n), lam.p, s);
        launch_apply(Mbuf.p, x->dims[n], R, Wn.p, factors[n], s);
        continue;
      }
      PASTA_CUDA(cudaMemsetAsync(colsq.p, 0, colsq.bytes(), s));
      launch_solve(Mbuf.p, x->dims[n], R, gl, ng, factors[n], colsq.p, s);
      launch_normalize(factors[n], x->dims[n], R, colsq.p, lam.p, s);
      PASTA_CUDA(cudaMemsetAsync(G(n), 0, sizeof(double) * R * R, s));
      launch_gram(factors[n], x->dims[n], R, G(n), s);
    }
    // fit from the last mode's MTTKRP (still in Mbuf) and the normalised factors, in a kernel
    PASTA_CUDA(cudaMemsetAsync(scal.p + 1, 0, sizeof(double), s));
    launch_inner(Mbuf.p, factors[N - 1], x->dims[N - 1], R, lam.p, scal.p + 1, s);
    const double *gall[kMaxOrder];
    for (uint32_t k = 0; k < N; ++k) gall[k] = G(k);
    launch_cpals_fit(gall, N, R, lam.p, scal.p + 1, normx2, fitbuf.p, s);
    double fit = 0.0;
    PASTA_CUDA(cudaMemcpyAsync(&fit, fitbuf.p, sizeof(double), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    fit_history[it] = fit;
    const bool done = it > 0 && std::fabs(fit - prev) < tol;
    prev = fit;
    if (done) { ++it; break; }
  }
  PASTA_CUDA(cudaMemcpyAsync(lambda, lam.p, R * sizeof(double), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  *iters = it;
  API_END
}

// ---------------------------------------------------------------------------- TTV / TTM
pasta_status pasta_coo_fibers(pasta_coo *x, uint32_t mode, uint64_t *nfibers, void *stream) {
  API_BEGIN
  require(x && nfibers, "x/nfibers is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  std::lock_guard<std::mutex> lk(x->mu);
  coo_build_fibers(x, mode, as_stream(stream));
  *nfibers = x->fib[mode]->nf;
  API_END
}

pasta_status pasta_coo_fiber_export(pasta_coo *x, uint32_t mode, uint32_t *const *inds) {
  API_BEGIN
  require(x && inds, "x/inds is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  {
    std::lock_guard<std::mutex> lk(x->mu);
    coo_build_fibers(x, mode, nullptr);
  }
  const FiberCopy &f = *x->fib[mode];
  for (uint32_t k = 0; k < x->order; ++k) {
    if (k == mode || !f.nf) continue;
    require(inds[k] != nullptr, "inds[k] is NULL for a mode k != mode");
    PASTA_CUDA(cudaMemcpy(inds[k], f.finds[k].p, f.nf * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  }
  API_END
}

pasta_status pasta_ttm_coo(pasta_coo *x, uint32_t mode, const float *U, uint32_t R, float *out,
                           void *stream) {
  API_BEGIN
  require(x && U && out, "x/U/out is NULL");
  require(mode < x->order, "mode >= order");
  require(R >= 1, "R must be >= 1");
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  if (!x->fib[mode]) {
    std::lock_guard<std::mutex> lk(x->mu);
    coo_build_fibers(x, mode, s);
  }
  FiberCopy &f = *x->fib[mode];
  if (!f.mat.mc[0].ready) {
    std::lock_guard<std::mutex> lk(f.mat.mu);
    coo_prepare_mode(&f.mat, 0, s);
  }
  launch_zero_rows(out, 0, f.nf, R, s);
  const float *fac[2] = {nullptr, U};
  launch_coo_mttkrp(&f.mat, 0, fac, R, out, s);
  API_END
}

pasta_status pasta_ttv_coo(pasta_coo *x, uint32_t mode, const float *v, float *out, void *stream) {
  API_BEGIN
  require(x && v && out, "x/v/out is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  cudaStream_t s = as_stream(stream);
  if (!x->fib[mode]) {
    std::lock_guard<std::mutex> lk(x->mu);
    coo_build_fibers(x, mode, s);
  }
  FiberCopy &f = *x->fib[mode];
  if (!f.mat.mc[0].ready) {
    std::lock_guard<std::mutex> lk(f.mat.mu);
    coo_prepare_mode(&f.mat, 0, s);
  }
  launch_zero_rows(out, 0, f.nf, 1, s);
  // PASTA_TTV_SEGSUM=0: the R = 1 MTTKRP path of pasta_ttm_coo instead of the segmented sum
  const char *e = getenv("PASTA_TTV_SEGSUM");
  if (e && *e == '0') {
    const float *fac[2] = {nullptr, v};
    launch_coo_mttkrp(&f.mat, 0, fac, 1, out, s);
  } else {
    launch_ttv(f.mat, v, out, s);
  }
  API_END
}

// ---------------------------------------------------------------------------- introspection
// ---------------------------------------------------------------------------- TEW / TS
pasta_status pasta_ts(const float *vals, uint64_t n, uint32_t op, float s, float *out, void *stream) {
  API_BEGIN
  require(op <= PASTA_OP_DIV, "op must be PASTA_OP_ADD/SUB/MUL/DIV");
  require(n == 0 || (vals && out), "vals/out is NULL");
  launch_ts(op, vals, s, out, n, as_stream(stream));
  API_END
}

pasta_status pasta_tew(const float *a, const float *b, uint64_t n, uint32_t op, float *out, void *stream) {
  API_BEGIN
  require(op <= PASTA_OP_DIV, "op must be PASTA_OP_ADD/SUB/MUL/DIV");
  require(n == 0 || (a && b && out), "a/b/out is NULL");
  launch_tew(op, a, b, out, n, as_stream(stream));
  API_END
}

pasta_status pasta_coo_values(const pasta_coo *x, float **vals) {
  API_BEGIN
  require(x && vals, "x/vals is NULL");
  *vals = x->val.p;
  API_END
}

pasta_status pasta_coo_ts(const pasta_coo *x, uint32_t op, float s, pasta_coo **out) {
  API_BEGIN
  require(x && out, "x/out is NULL");
  *out = nullptr;
  require(op <= PASTA_OP_DIV, "op must be PASTA_OP_ADD/SUB/MUL/DIV");
  check_device(x->device);
  auto y = std::make_unique<pasta_coo>();
  copy_pattern_device(x, y.get(), nullptr);  // pre-processing: output indices
  launch_ts(op, x->val.p, s, y->val.p, x->nnz, nullptr);
  PASTA_CUDA(cudaStreamSynchronize(nullptr));
  *out = y.release();
  API_END
}

pasta_status pasta_coo_tew(pasta_coo *x, pasta_coo *y, uint32_t op, pasta_coo **out) {
  API_BEGIN
  require(x && y && out, "x/y/out is NULL");
  *out = nullptr;
  require(op <= PASTA_OP_DIV, "op must be PASTA_OP_ADD/SUB/MUL/DIV");
  require(x->order == y->order, "tew: tensors of different orders");
  for (uint32_t k = 0; k < x->order; ++k) require(x->dims[k] == y->dims[k], "tew: tensors of different shapes");
  check_device(x->device);
  check_device(y->device);
  auto z = std::make_unique<pasta_coo>();
  if (same_pattern_device(x, y, nullptr)) {
    copy_pattern_device(x, z.get(), nullptr);
    launch_tew(op, x->val.p, y->val.p, z->val.p, x->nnz, nullptr);
    PASTA_CUDA(cudaStreamSynchronize(nullptr));
  } else {
    {
      std::lock_guard<std::mutex> lk(x->mu);
      coo_prepare_mode(x, 0, nullptr);
    }
    if (y != x) {
      std::lock_guard<std::mutex> lk(y->mu);
      coo_prepare_mode(y, 0, nullptr);
    }
    tew_merge_device(x, y, op, z.get(), nullptr);
  }
  *out = z.release();
  API_END
}

pasta_status pasta_coo_info(const pasta_coo *x, uint32_t *order, uint32_t *dims, uint64_t *nnz) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  if (order) *order = x->order;
  if (dims)
    for (uint32_t k = 0; k < x->order; ++k) dims[k] = x->dims[k];
  if (nnz) *nnz = x->nnz;
  API_END
}

static void export_arrays(uint32_t order, uint64_t nnz, const uint32_t *const *dinds, const float *dval,
                          uint32_t *const *inds, float *vals) {
  for (uint32_t k = 0; k < order; ++k) {
    require(!inds || inds[k] || !nnz, "inds[k] is NULL");
    if (inds && inds[k] && nnz)
      PASTA_CUDA(cudaMemcpy(inds[k], dinds[k], nnz * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  }
  if (vals && nnz) PASTA_CUDA(cudaMemcpy(vals, dval, nnz * sizeof(float), cudaMemcpyDeviceToHost));
}

pasta_status pasta_coo_export(const pasta_coo *x, uint32_t *const *inds, float *vals) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  check_device(x->device);
  const uint32_t *di[kMaxOrder];
  for (uint32_t k = 0; k < x->order; ++k) di[k] = x->inds[k].p;
  export_arrays(x->order, x->nnz, di, x->val.p, inds, vals);
  API_END
}

pasta_status pasta_coo_export_mode(pasta_coo *x, uint32_t mode, uint32_t *const *inds, float *vals) {
  API_BEGIN
  require(x != nullptr, "x is NULL");
  require(mode < x->order, "mode >= order");
  check_device(x->device);
  {
    std::lock_guard<std::mutex> lk(x->mu);
    coo_prepare_mode(x, mode, nullptr);
  }
  export_arrays(x->order, x->nnz, x->mc[mode].inds, x->mc[mode].val, inds, vals);
  API_END
}

pasta_status pasta_hicoo_info(const pasta_hicoo *h, uint32_t *order, uint32_t *dims, uint32_t *block_bits,
                              uint64_t *nblocks, uint64_t *nnz) {
  API_BEGIN
  require(h != nullptr, "h is NULL");
  if (order) *order = h->order;
  if (dims)
    for (uint32_t k = 0; k < h->order; ++k) dims[k] = h->dims[k];
  if (block_bits) *block_bits = h->block_bits;
  if (nblocks) *nblocks = h->nblocks;
  if (nnz) *nnz = h->nnz;
  API_END
}

pasta_status pasta_ghicoo_info(const pasta_hicoo *h, uint32_t *cmask) {
  API_BEGIN
  require(h && cmask, "h/cmask is NULL");
  *cmask = h->cmask;
  API_END
}

pasta_status pasta_ghicoo_export(const pasta_hicoo *h, uint64_t *bptr, uint32_t *const *binds,
                                 uint8_t *const *einds, uint32_t *const *uinds, float *vals) {
  API_BEGIN
  require(h != nullptr, "h is NULL");
  check_device(h->device);
  if (bptr) PASTA_CUDA(cudaMemcpy(bptr, h->bptr.p, (h->nblocks + 1) * 8, cudaMemcpyDeviceToHost));
  for (uint32_t k = 0; k < h->order; ++k) {
    if ((h->cmask >> k) & 1u) {
      if (binds && binds[k] && h->nblocks)
        PASTA_CUDA(cudaMemcpy(binds[k], h->binds[k].p, h->nblocks * 4, cudaMemcpyDeviceToHost));
      if (einds && einds[k] && h->nnz)
        PASTA_CUDA(cudaMemcpy(einds[k], h->einds[k].p, h->nnz, cudaMemcpyDeviceToHost));
    } else if (uinds && uinds[k] && h->nnz) {
      PASTA_CUDA(cudaMemcpy(uinds[k], h->uinds[k].p, h->nnz * 4, cudaMemcpyDeviceToHost));
    }
  }
  if (vals && h->nnz) PASTA_CUDA(cudaMemcpy(vals, h->val.p, h->nnz * 4, cudaMemcpyDeviceToHost));
  API_END
}

pasta_status pasta_hicoo_export(const pasta_hicoo *h, uint64_t *bptr, uint32_t *const *binds,
                                uint8_t *const *einds, float *vals) {
  API_BEGIN
  require(h != nullptr, "h is NULL");
  require(h->cmask == (1u << h->order) - 1u, "gHiCOO handle: use pasta_ghicoo_export");
  check_device(h->device);
  if (bptr) PASTA_CUDA(cudaMemcpy(bptr, h->bptr.p, (h->nblocks + 1) * 8, cudaMemcpyDeviceToHost));
  for (uint32_t k = 0; k < h->order; ++k) {
    if (binds && binds[k] && h->nblocks)
      PASTA_CUDA(cudaMemcpy(binds[k], h->binds[k].p, h->nblocks * 4, cudaMemcpyDeviceToHost));
    if (einds && einds[k] && h->nnz)
      PASTA_CUDA(cudaMemcpy(einds[k], h->einds[k].p, h->nnz, cudaMemcpyDeviceToHost));
  }
  if (vals && h->nnz) PASTA_CUDA(cudaMemcpy(vals, h->val.p, h->nnz * 4, cudaMemcpyDeviceToHost));
  API_END
}

void pasta_coo_free(pasta_coo *x) { delete x; }
void pasta_hicoo_free(pasta_hicoo *h) { delete h; }

// ---------------------------------------------------------------------------- measurement
uint64_t pasta_launch_count(void) { return g_launches.load(); }

pasta_status pasta_die_map(uint32_t *nsms, int8_t *die_of_sm, uint32_t *n_die) {
  API_BEGIN
  require(nsms != nullptr, "nsms is NULL");
  const DieMap &m = die_map();
  *nsms = m.ok ? uint32_t(m.sms) : 0u;
  if (m.ok && die_of_sm) memcpy(die_of_sm, m.die, size_t(m.sms));
  if (n_die) {
    n_die[0] = m.ok ? uint32_t(m.n[0]) : 0u;
    n_die[1] = m.ok ? uint32_t(m.n[1]) : 0u;
  }
  API_END
}

pasta_status pasta_profile_enable(int on) {
  API_BEGIN
  g_prof_on.store(on != 0);
  API_END
}

pasta_status pasta_profile_read(uint32_t which, double *total_ms, uint64_t *launches, int reset) {
  API_BEGIN
  require(which < kProfKinds, "which must be 0 (COO), 1 (HiCOO), 2 (zero-fill) or 3 (TEW/TS)");
  std::lock_guard<std::mutex> lk(g_prof_mu);
  double sum = 0.0;
  for (auto &r : g_prof[which]) {
    PASTA_CUDA(cudaEventSynchronize(r.b));
    float ms = 0.f;
    PASTA_CUDA(cudaEventElapsedTime(&ms, r.a, r.b));
    sum += ms;
  }
  if (total_ms) *total_ms = sum;
  if (launches) *launches = g_prof[which].size();
  if (reset) {
    for (auto &r : g_prof[which]) {
      cudaEventDestroy(r.a);
      cudaEventDestroy(r.b);
    }
    g_prof[which].clear();
  }
  API_END
}

}  // extern "C"
