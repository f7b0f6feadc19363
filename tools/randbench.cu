// randbench.cu — measurement tool (not product): the random-access ceiling of a B200 for
// the hash table's access pattern.  Every "probe" reads one random window of WB bytes
// aligned to AB bytes inside a large buffer, fetched by WB/8 lanes x 8 B (the coalesced
// group pattern, |g| = WB/8).  Each lane keeps D independent windows in flight.  Variants:
//   read : window read only (a query)
//   cas  : window read, then a 64-bit CAS on the window's first slot that FAILS (no write)
//   casw : ... a CAS that SUCCEEDS (dirty sector, written back later: an insert)
// Reports windows/s and useful GB/s for the buffer sizes given (GB; default 2.26 = config 2's
// table and 36 = config 3's; 0.0088 = config 1's L2-resident table).
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/randbench tools/randbench.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
  return x;
}
__device__ __forceinline__ unsigned long long ldr(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

template <int D, int MODE, int WB, int AB>
__global__ void __launch_bounds__(256) gather(unsigned long long* buf, uint64_t nwin, int iters,
                                              uint32_t salt, unsigned long long* sink) {
  constexpr int L = WB / 8;  // lanes per window
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t g = tid / L, r = tid % L;
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    unsigned long long v[D];
    const unsigned long long* p[D];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const uint32_t h = hash32(g * 2654435761u + (it * D + d) * 40503u + salt);
      const uint64_t w = (uint64_t(h) * nwin) >> 32;         // window start = w * AB bytes
      p[d] = buf + w * (AB / 8) + r;
      v[d] = ldr(p[d]);
    }
#pragma unroll
    for (int d = 0; d < D; ++d) {
      acc += v[d];
      if (MODE != 0 && r == 0) {
        if (MODE == 1) acc += atomicCAS((unsigned long long*)p[d], 0x1234567812345678ull, 1ull);
        else acc += atomicCAS((unsigned long long*)p[d], v[d], v[d] ^ 1ull);
      }
    }
  }
  if (acc == 42) sink[0] = acc;
}

// dependent chains: each lane follows D independent chains; the next window of a chain is
// derived from the data just loaded (as in probing), so only D windows per lane are ever
// in flight.  WB = window bytes loaded by ONE lane with vector loads (8/16/32).
template <int D, int WB>
__global__ void __launch_bounds__(256) chase(unsigned long long* buf, uint64_t nwin, int iters,
                                             unsigned long long* sink) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t cur[D];
  unsigned long long acc = 0;
#pragma unroll
  for (int d = 0; d < D; ++d) cur[d] = hash32(tid * 2654435761u + d * 97u + 5u);
  for (int it = 0; it < iters; ++it) {
    unsigned long long v[D];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const uint64_t w = (uint64_t(cur[d]) * nwin) >> 32;
      const unsigned long long* p = buf + w * 4;
      if (WB == 32) {
        unsigned long long a, b, c, e;
        asm volatile("ld.global.cg.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a), "=l"(b), "=l"(c), "=l"(e) : "l"(p));
        v[d] = a ^ b ^ c ^ e;
      } else {
        v[d] = ldr(p);
      }
    }
#pragma unroll
    for (int d = 0; d < D; ++d) {
      acc += v[d];
      cur[d] = hash32(cur[d] ^ uint32_t(v[d]) ^ uint32_t(it));   // next address depends on data
    }
  }
  if (acc == 42) sink[0] = acc;
}

template <int D, int WB>
void run_chase(unsigned long long* buf, uint64_t bytes, int grid, int iters, unsigned long long* sink,
               const char* tag) {
  const uint64_t nwin = (bytes - 256) / 32;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  chase<D, WB><<<grid, 256>>>(buf, nwin, 2, sink);
  cudaEventRecord(a);
  chase<D, WB><<<grid, 256>>>(buf, nwin, iters, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  const double windows = double(grid) * 256 * D * iters;
  printf("%.2fGB chase W=%2dB D=%d %s: %6.1f Gwin/s  (%d thr/SM x %d chains)\n", bytes / 1e9, WB, D, tag,
         windows / (ms * 1e-3) / 1e9, grid * 256 / 148, D);
}

// chase2: probe-like chains.  Each chain works on "keys": a key starts at a random
// 32-B-aligned window and continues with the ADJACENT window with probability ~1/2 (so
// ~2 windows per key, like alpha = 0.95, |g| = 4).  Variants add the probe kernel's other
// traffic: V&1: read a 4-byte input key per key (sequential per lane); V&2: write a 4-byte
// + 1-byte output per key (scattered by key index); V&4: CAS the last window (insert-like,
// succeeds -> dirty line).
template <int D, int V>
__global__ void __launch_bounds__(256) chase2(unsigned long long* buf, uint64_t nwin, int keys_per_chain,
                                              const uint32_t* in, uint32_t* out_v, uint8_t* out_f,
                                              unsigned long long* sink) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t nthr = gridDim.x * blockDim.x;
  uint32_t cur[D], kidx[D];
  uint64_t w[D];
  unsigned long long acc = 0;
#pragma unroll
  for (int d = 0; d < D; ++d) {
    kidx[d] = 0;
    cur[d] = hash32(tid * 2654435761u + d * 97u + 5u);
    w[d] = (uint64_t(cur[d]) * nwin) >> 32;
  }
  int done_keys = 0;
  const int total = keys_per_chain * D;
  while (done_keys < total) {
    unsigned long long v[D];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const unsigned long long* p = buf + w[d] * 4;
      unsigned long long a, b, c, e;
      asm volatile("ld.global.cg.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a), "=l"(b), "=l"(c), "=l"(e) : "l"(p));
      v[d] = a ^ b ^ c ^ e;
    }
#pragma unroll
    for (int d = 0; d < D; ++d) {
      acc += v[d];
      cur[d] = hash32(cur[d] ^ uint32_t(v[d]) ^ 0x9e37u);
      const bool cont = (cur[d] & 1u) && w[d] + 1 < nwin;          // adjacent next window
      if (cont) { w[d] += 1; continue; }
      // key finished
      const uint64_t item = uint64_t(kidx[d]) * nthr * D + uint64_t(tid) * D + d;
      if (V & 4) acc += atomicCAS(buf + w[d] * 4, v[d], v[d] ^ 1ull);
      if (V & 2) { out_v[item] = uint32_t(v[d]); out_f[item] = 1; }
      ++kidx[d];
      ++done_keys;
      uint32_t nk = cur[d];
      if (V & 1) nk ^= __ldg(in + item);
      w[d] = (uint64_t(hash32(nk)) * nwin) >> 32;
    }
  }
  if (acc == 42) sink[0] = acc;
}

template <int D, int V>
void run_chase2(unsigned long long* buf, uint64_t bytes, int grid, int kpc, uint32_t* in, uint32_t* ov,
                uint8_t* of, unsigned long long* sink) {
  const uint64_t nwin = (bytes - 256) / 32;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  chase2<D, V><<<grid, 256>>>(buf, nwin, 2, in, ov, of, sink);
  cudaEventRecord(a);
  chase2<D, V><<<grid, 256>>>(buf, nwin, kpc, in, ov, of, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  const double keys = double(grid) * 256 * D * kpc;
  printf("%.2fGB chase2 V=%d D=%d (%d thr/SM): %6.2f G keys/s  (~%.1f G windows/s)\n", bytes / 1e9, V, D,
         grid * 256 / 148, keys / (ms * 1e-3) / 1e9, 2 * keys / (ms * 1e-3) / 1e9);
}

// atomics only: every lane issues D independent 64-bit CAS (succeeding: the expected value is
// read first by the same lane... no — plain CAS on random slots, alternating values so each
// succeeds or fails with ~1/2), or atomicAdd, on random 8-B slots of the buffer: the L2's
// random atomic throughput, the floor of an insert's claim (one CAS per new key).
template <int D, int OP>
__global__ void __launch_bounds__(256) atom_only(unsigned long long* buf, uint64_t nslot, int iters,
                                                 unsigned long long* sink) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    unsigned long long r[D];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const uint32_t h = hash32(tid * 2654435761u + (it * D + d) * 40503u + 17u);
      unsigned long long* p = buf + ((uint64_t(h) * nslot) >> 32);
      if (OP == 0) r[d] = atomicCAS(p, 0xFFFFFFFFFFFFFFFFull, uint64_t(tid));
      else r[d] = atomicAdd(p, 1ull);
    }
#pragma unroll
    for (int d = 0; d < D; ++d) acc += r[d];
  }
  if (acc == 42) sink[0] = acc;
}
template <int D, int OP>
void run_atom(unsigned long long* buf, uint64_t bytes, int grid, int iters, unsigned long long* sink) {
  const uint64_t nslot = bytes / 8;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  atom_only<D, OP><<<grid, 256>>>(buf, nslot, 2, sink);
  cudaEventRecord(a);
  atom_only<D, OP><<<grid, 256>>>(buf, nslot, iters, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  const double ops = double(grid) * 256 * D * iters;
  printf("%.4fGB %s-only D=%d (%d thr/SM): %6.1f G atomics/s\n", bytes / 1e9, OP == 0 ? "cas" : "add",
         D, grid * 256 / 148, ops / (ms * 1e-3) / 1e9);
}

template <int D, int MODE, int WB, int AB>
void run(const char* name, unsigned long long* buf, uint64_t bytes, int grid, int iters,
         unsigned long long* sink) {
  const uint64_t nwin = (bytes - 256) / AB;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  gather<D, MODE, WB, AB><<<grid, 256>>>(buf, nwin, 2, 1, sink);
  cudaEventRecord(a);
  gather<D, MODE, WB, AB><<<grid, 256>>>(buf, nwin, iters, 7, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  const double windows = double(grid) * 256 / (WB / 8) * D * iters;
  printf("%.2fGB %-5s W=%3dB align=%3dB D=%d : %6.1f Gwin/s  %6.0f GB/s useful\n", bytes / 1e9, name,
         WB, AB, D, windows / (ms * 1e-3) / 1e9, windows * WB / (ms * 1e-3) / 1e9);
}

int main(int argc, char** argv) {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* sink; cudaMalloc(&sink, 8);
  cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, 32);
  // buffer sizes in GB from the command line (default: the config-2 table and config 3);
  // 0.0088 = config 1's 8.8 MB table, L2-resident: its ceiling is the L2's random rate
  std::vector<double> sizes;
  for (int i = 1; i < argc; ++i) sizes.push_back(atof(argv[i]));
  if (sizes.empty()) sizes = {2.26, 36.0};
  for (double gb : sizes) {
    const uint64_t bytes = uint64_t(gb * 1e9) / 256 * 256;
    unsigned long long* buf;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) { printf("alloc %.1f GB failed\n", gb); continue; }
    cudaMemset(buf, 0xff, bytes);
    const int grid = sms * 8;
    const int it = 32;
    run_atom<4, 0>(buf, bytes, grid, it, sink);
    run_atom<8, 0>(buf, bytes, grid, it, sink);
    run_atom<8, 1>(buf, bytes, grid, it, sink);
    run_atom<8, 0>(buf, bytes, sms * 4, it, sink);
    if (getenv("RB_ATOM_ONLY")) { cudaFree(buf); continue; }
    run<8, 0, 8, 32>("read", buf, bytes, grid, it, sink);
    run<8, 0, 32, 32>("read", buf, bytes, grid, it, sink);
    run<8, 0, 32, 64>("read", buf, bytes, grid, it, sink);
    run<8, 0, 64, 32>("read", buf, bytes, grid, it, sink);
    run<8, 0, 64, 64>("read", buf, bytes, grid, it, sink);
    run<8, 0, 128, 32>("read", buf, bytes, grid, it, sink);
    run<8, 0, 128, 128>("read", buf, bytes, grid, it, sink);
    run<8, 0, 256, 32>("read", buf, bytes, grid, it, sink);
    run<8, 0, 256, 256>("read", buf, bytes, grid, it, sink);
    run<8, 1, 32, 32>("cas", buf, bytes, grid, it, sink);
    run<8, 2, 32, 32>("casw", buf, bytes, grid, it, sink);
    run<8, 1, 64, 64>("cas", buf, bytes, grid, it, sink);
    run<8, 2, 64, 64>("casw", buf, bytes, grid, it, sink);
    run<8, 1, 128, 128>("cas", buf, bytes, grid, it, sink);
    run<8, 2, 128, 128>("casw", buf, bytes, grid, it, sink);
    {
      const int grid = sms * 4, kpc = 32;
      const size_t nk = size_t(grid) * 256 * 8 * kpc;
      uint32_t *in, *ov; uint8_t* of;
      cudaMalloc(&in, nk * 4); cudaMalloc(&ov, nk * 4); cudaMalloc(&of, nk);
      cudaMemset(in, 1, nk * 4);
      run_chase2<4, 0>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<4, 1>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<4, 2>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<4, 3>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<4, 4>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<4, 7>(buf, bytes, grid, kpc, in, ov, of, sink);
      run_chase2<8, 0>(buf, bytes, grid, kpc / 2, in, ov, of, sink);
      run_chase2<8, 3>(buf, bytes, grid, kpc / 2, in, ov, of, sink);
      cudaMemset(buf, 0xff, bytes);
      cudaFree(in); cudaFree(ov); cudaFree(of);
    }
    for (int occ : {2, 4, 8}) {
      run_chase<1, 32>(buf, bytes, sms * occ, 64, sink, "");
      run_chase<2, 32>(buf, bytes, sms * occ, 64, sink, "");
      run_chase<4, 32>(buf, bytes, sms * occ, 64, sink, "");
      run_chase<8, 32>(buf, bytes, sms * occ, 32, sink, "");
      run_chase<4, 8>(buf, bytes, sms * occ, 64, sink, "");
    }
    cudaFree(buf);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
