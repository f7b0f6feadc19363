// wdgen.cu — device-side copy of the counter-based input generator of wdgen/__init__.py.
// Generator only (no hashing/probing/partitioning of the method): used by the bench and
// the large GPU tests to create inputs in HBM without a host round trip; never timed
// ("test data generation ... omitted").  tests/test_gen_gpu.py checks it equals
// the numpy version element by element.
#include <cstdint>
#include <cuda_runtime.h>

namespace {
constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr uint64_t TAG_PERM = 0x5045524D, TAG_VAL = 0x56414C55, TAG_UNI = 0x554E4946,
                   TAG_MIX = 0x4D495851, TAG_ZIPF = 0x5A495046;

__host__ __device__ inline uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ inline uint64_t stream_key(uint64_t seed, uint64_t tag) {
  return splitmix64(seed ^ (tag << 32));
}
struct RK { uint64_t k[4]; };
RK round_keys(uint64_t seed) {
  RK r;
  const uint64_t base = stream_key(seed, TAG_PERM);
  for (int i = 0; i < 4; ++i) r.k[i] = splitmix64(base + i);
  return r;
}
__device__ inline uint32_t feistel(uint32_t x, const RK& rk) {
  uint64_t L = x >> 16, R = x & 0xFFFF;
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const uint64_t F = splitmix64(R ^ rk.k[r]) & 0xFFFF;
    const uint64_t nl = R;
    R = L ^ F;
    L = nl;
  }
  return uint32_t((L << 16) | R);
}
__device__ inline uint32_t perm32(uint32_t x, const RK& rk) {
  uint32_t y = feistel(x, rk);
  if (y == kEmpty) y = feistel(kEmpty, rk);
  return y;
}

__global__ void k_unique(uint32_t* out, uint64_t start, uint64_t n, RK rk) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    out[i] = perm32(uint32_t(start + i), rk);
}
__global__ void k_values(uint32_t* out, uint64_t start, uint64_t n, uint64_t sk) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    out[i] = uint32_t(splitmix64(start + i + sk));
}
__global__ void k_uniform(uint32_t* out, uint64_t start, uint64_t n, uint64_t sk) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t z = splitmix64(start + i + sk);
    uint32_t k = uint32_t(z);
    if (k == kEmpty) k = uint32_t(z >> 32);
    if (k == kEmpty) k = 0;
    out[i] = k;
  }
}
__global__ void k_interleaved(uint32_t* out, uint64_t n_present, uint64_t start, uint64_t count, RK rk) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < count; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t j = start + i;
    const uint64_t idx = (j >> 1) + (j & 1) * n_present;
    out[i] = perm32(uint32_t(idx), rk);
  }
}
__global__ void k_mixed(uint32_t* out, uint8_t* hit_out, uint64_t n_table, uint64_t start, uint64_t count,
                        uint64_t thr, uint64_t sk, RK rk) {
  const uint64_t n_abs = uint64_t(kEmpty) - n_table;
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < count; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t z = splitmix64(start + i + sk);
    const uint64_t lo = z & 0xFFFFFFFFull, r = z >> 32;
    const bool hit = lo < thr;
    const uint64_t idx = hit ? r % (n_table ? n_table : 1) : n_table + r % n_abs;
    out[i] = perm32(uint32_t(idx), rk);
    if (hit_out) hit_out[i] = hit;
  }
}
// ---- closed-form checker (test harness; generator arithmetic only, none of the method's):
// a key k is present iff its generator index pi_s^-1(k) < n_present, and then its value is
// values(pi_s^-1(k)) — the same closed form as oracle.expected_unique, evaluated on the
// device so full-size runs can check EVERY query.  res[0] += mismatches, res[1] = min
// mismatching position, res[2] += found count.
__device__ inline uint32_t feistel_inv(uint32_t y, const RK& rk) {
  uint64_t L = y >> 16, R = y & 0xFFFF;
#pragma unroll
  for (int r = 3; r >= 0; --r) {
    const uint64_t F = splitmix64(L ^ rk.k[r]) & 0xFFFF;
    const uint64_t nl = R ^ F;
    R = L;
    L = nl;
  }
  return uint32_t((L << 16) | R);
}
__device__ inline uint32_t perm32_inv(uint32_t y, const RK& rk) {
  uint32_t x = feistel_inv(y, rk);
  if (x == kEmpty) x = feistel_inv(kEmpty, rk);
  return x;
}
__global__ void k_check_unique(const uint32_t* q, const uint32_t* vout, const uint8_t* fout,
                               uint64_t count, uint64_t n_present, uint64_t vsk, RK rk,
                               unsigned long long* res) {
  unsigned long long bad = 0, found = 0, first = ~0ull;
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < count; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t k = q[i];
    bool present = false;
    uint32_t ev = 0xFFFFFFFFu;
    if (k != kEmpty) {
      const uint64_t idx = perm32_inv(k, rk);
      present = idx < n_present;
      if (present) ev = uint32_t(splitmix64(idx + vsk));
    }
    bool ok = true;
    if (fout) {
      ok = ok && (fout[i] == (present ? 1 : 0));
      found += fout[i] == 1;
    }
    if (vout) ok = ok && vout[i] == ev;
    if (!ok) {
      ++bad;
      if (i < first) first = i;
    }
  }
  for (int o = 16; o; o >>= 1) {
    bad += __shfl_xor_sync(0xFFFFFFFFu, bad, o);
    found += __shfl_xor_sync(0xFFFFFFFFu, found, o);
    const unsigned long long f2 = __shfl_xor_sync(0xFFFFFFFFu, first, o);
    first = f2 < first ? f2 : first;
  }
  if ((threadIdx.x & 31) == 0) {
    if (bad) { atomicAdd(res, bad); atomicMin(res + 1, first); }
    if (found) atomicAdd(res + 2, found);
  }
}

// exact Zipf by rejection-inversion — the same computation as wdgen.zipf_ranks
struct ZipfC { double expo, c1, cn, sq, universe; };
__host__ __device__ inline double zh1(double x) {
  return fabs(x) > 1e-8 ? log1p(x) / x : 1 - x * (0.5 - x * (1.0 / 3 - 0.25 * x));
}
__host__ __device__ inline double zh2(double x) {
  return fabs(x) > 1e-8 ? expm1(x) / x : 1 + x * 0.5 * (1 + x * (1.0 / 3) * (1 + 0.25 * x));
}
__host__ __device__ inline double zh(double x, double e) { return exp(-e * log(x)); }
__host__ __device__ inline double zhi(double x, double e) { return zh2((1.0 - e) * log(x)) * log(x); }
__host__ __device__ inline double zhinv(double x, double e) {
  double t = x * (1.0 - e);
  if (t < -1.0) t = -1.0;
  return exp(zh1(t) * x);
}
ZipfC zipf_consts(uint64_t universe, double e) {
  ZipfC c;
  c.expo = e;
  c.universe = double(universe);
  c.c1 = zhi(1.5, e) - 1.0;
  c.cn = zhi(double(universe) + 0.5, e);
  c.sq = 2.0 - zhinv(zhi(2.5, e) - zh(2.0, e), e);
  return c;
}
__global__ void k_zipf(uint32_t* out, uint64_t start, uint64_t n, uint64_t sk, ZipfC c, RK rk) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
    double k = 1.0;
    for (int j = 0; j < 8; ++j) {
      const uint64_t z = splitmix64((start + i) * 8 + j + sk);
      const double uu = double(z >> 11) * (1.0 / 9007199254740992.0);
      const double u = c.cn + uu * (c.c1 - c.cn);
      const double x = zhinv(u, c.expo);
      k = floor(x + 0.5);
      if (k < 1.0) k = 1.0;
      if (k > c.universe) k = c.universe;
      if (k - x <= c.sq || u >= zhi(k + 0.5, c.expo) - zh(k, c.expo)) break;
    }
    out[i] = perm32(uint32_t(uint64_t(k) - 1), rk);
  }
}
int grid_for(uint64_t n) {
  uint64_t g = (n + 255) / 256;
  return int(g < 148 * 16 ? (g ? g : 1) : 148 * 16);
}
}  // namespace

extern "C" {
int wdgen_unique_keys(uint32_t* out, uint64_t start, uint64_t n, uint64_t seed, cudaStream_t st) {
  // pi_s is a bijection on [0, 2^32 - 1) only (the sentinel is cycle-walked out, C14):
  // index 2^32 - 1 would alias another key
  if (start > uint64_t(kEmpty) || n > uint64_t(kEmpty) - start) return int(cudaErrorInvalidValue);
  if (n) k_unique<<<grid_for(n), 256, 0, st>>>(out, start, n, round_keys(seed));
  return int(cudaGetLastError());
}
int wdgen_values(uint32_t* out, uint64_t start, uint64_t n, uint64_t seed, cudaStream_t st) {
  if (n) k_values<<<grid_for(n), 256, 0, st>>>(out, start, n, stream_key(seed, TAG_VAL));
  return int(cudaGetLastError());
}
int wdgen_uniform_keys(uint32_t* out, uint64_t start, uint64_t n, uint64_t seed, cudaStream_t st) {
  if (n) k_uniform<<<grid_for(n), 256, 0, st>>>(out, start, n, stream_key(seed, TAG_UNI));
  return int(cudaGetLastError());
}
int wdgen_interleaved_queries(uint32_t* out, uint64_t n_present, uint64_t start, uint64_t count,
                              uint64_t seed, cudaStream_t st) {
  const uint64_t jmax = start + count;   // largest index used: (jmax - 1) / 2 + n_present
  if (count && (count > (1ull << 33) || (jmax - 1) / 2 + n_present >= uint64_t(kEmpty)))
    return int(cudaErrorInvalidValue);
  if (count) k_interleaved<<<grid_for(count), 256, 0, st>>>(out, n_present, start, count, round_keys(seed));
  return int(cudaGetLastError());
}
int wdgen_zipf_keys(uint32_t* out, uint64_t start, uint64_t n, uint64_t universe, uint64_t seed,
                    cudaStream_t st) {
  if (n) k_zipf<<<grid_for(n), 256, 0, st>>>(out, start, n, stream_key(seed, TAG_ZIPF),
                                             zipf_consts(universe, 1.0 + 1e-6), round_keys(seed));
  return int(cudaGetLastError());
}
int wdgen_check_unique(const uint32_t* q, const uint32_t* vout, const uint8_t* fout, uint64_t count,
                       uint64_t n_present, uint64_t key_seed, uint64_t val_seed,
                       unsigned long long* res, cudaStream_t st) {
  if (count)
    k_check_unique<<<grid_for(count), 256, 0, st>>>(q, vout, fout, count, n_present,
                                                    stream_key(val_seed, TAG_VAL), round_keys(key_seed), res);
  return int(cudaGetLastError());
}
int wdgen_mixed_queries(uint32_t* out, uint8_t* hit_out, uint64_t n_table, uint64_t start, uint64_t count,
                        double hit_frac, uint64_t seed, cudaStream_t st) {
  double t = hit_frac * 4294967296.0;
  uint64_t thr = t >= 4294967296.0 ? 4294967296ull : (t <= 0 ? 0ull : uint64_t(t));
  if (count)
    k_mixed<<<grid_for(count), 256, 0, st>>>(out, hit_out, n_table, start, count, thr,
                                             stream_key(seed, TAG_MIX), round_keys(seed));
  return int(cudaGetLastError());
}
}
