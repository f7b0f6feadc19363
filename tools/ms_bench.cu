// ms_bench.cu — measurement tool (not product): the slice grouping / cascade multisplit in
// isolation.  Times wd::multisplit_kernel (round 1) against wd::multisplit_kernel (round 2,
// ballot ranking, no shared-memory atomics) on 2^n random keys, and a plain interleave copy
// (read 4 + 4 B, write 8 B per pair) as the streaming speed of light.  Every output is
// checked on the host: each slice's range holds only keys of that slice, and the values
// (= input indices) form a permutation.
// Build (compile-time variants via -DWD_MS2_IPT=.. -DWD_MS2_MINB=.., cursor mode -DWD_MS2_IPTC/MINBC):
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -Iinclude \
//        -o tools/ms_bench tools/ms_bench.cu
// Run: tools/ms_bench [log2 n = 28] [reps = 10]
#include "../paper_conf_ipps_junger0s18_b200/csrc/wd_device.cuh"

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__global__ void gen(uint32_t* k, uint32_t* v, uint64_t n) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t x = uint32_t(i) * 0x9E3779B1u + 0x1234567u;
    x ^= x >> 15; x *= 0x2c1b3c6du; x ^= x >> 12; x *= 0x297a2d39u; x ^= x >> 15;
    k[i] = x == 0xFFFFFFFFu ? 0u : x;
    v[i] = uint32_t(i);
  }
}
__global__ void interleave(const uint32_t* __restrict__ k, const uint32_t* __restrict__ v, uint64_t n,
                           unsigned long long* __restrict__ out) {
  const uint64_t n4 = n / 4;
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n4; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(k) + i), b = __ldg(reinterpret_cast<const uint4*>(v) + i);
    ulonglong2* o = reinterpret_cast<ulonglong2*>(out) + 2 * i;
    o[0] = make_ulonglong2((uint64_t(b.x) << 32) | a.x, (uint64_t(b.y) << 32) | a.y);
    o[1] = make_ulonglong2((uint64_t(b.z) << 32) | a.z, (uint64_t(b.w) << 32) | a.w);
  }
}

static uint32_t h_fmix32(uint32_t x) {
  x ^= x >> 16; x *= 0x85ebca6bu; x ^= x >> 13; x *= 0xc2b2ae35u; x ^= x >> 16;
  return x;
}

template <class F>
static float time_ms(F f, int reps) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  std::vector<float> t;
  for (int r = 0; r < reps + 2; ++r) {
    CK(cudaEventRecord(a));
    f();
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    if (r >= 2) t.push_back(ms);
  }
  std::sort(t.begin(), t.end());
  return t[t.size() / 2];
}

template <class K>
static int occ(K kern) {
  int b = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kern, wd::kBlock, 0));
  return b;
}

int main(int argc, char** argv) {
  const int lg = argc > 1 ? atoi(argv[1]) : 28;
  const int reps = argc > 2 ? atoi(argv[2]) : 10;
  const uint64_t n = 1ull << lg;
  int sms = 0; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  uint32_t *k, *v; unsigned long long *out, *meta, *ctr;
  CK(cudaMalloc(&k, n * 4)); CK(cudaMalloc(&v, n * 4)); CK(cudaMalloc(&out, n * 8));
  CK(cudaMalloc(&meta, 3 * 256 * 8 + 8)); CK(cudaMalloc(&ctr, 16 * 8));
  CK(cudaMemset(ctr, 0, 16 * 8));
  gen<<<sms * 8, 256>>>(k, v, n);
  CK(cudaDeviceSynchronize());
  const uint32_t seed = 0x5bd1e995u;
  unsigned long long *bounds = meta + 256, *cursor = meta + 2 * 256 + 1;
  unsigned int* segc; unsigned long long* sego;           // segment mode: counts, offsets
  CK(cudaMalloc(&segc, 4096 * 128 * 4)); CK(cudaMalloc(&sego, 4096 * 128 * 8));
  const double gb = n * 16.0 / 1e9;

  const float tcopy = time_ms([&] { interleave<<<sms * 8, 256>>>(k, v, n, out); }, reps);
  printf("{\"kernel\": \"interleave\", \"n\": %llu, \"ms\": %.4f, \"GBps\": %.1f}\n",
         (unsigned long long)n, tcopy, gb / tcopy * 1e3);

  std::vector<unsigned long long> hb(257), ho(n);
  std::vector<uint32_t> hk(n);
  CK(cudaMemcpy(hk.data(), k, n * 4, cudaMemcpyDeviceToHost));
  auto check = [&](int nbk, const char* name) {
    CK(cudaMemcpy(hb.data(), bounds, (nbk + 1) * 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(ho.data(), out, n * 8, cudaMemcpyDeviceToHost));
    std::vector<uint8_t> seen(n, 0);
    uint64_t bad = 0;
    for (int j = 0; j < nbk; ++j)
      for (uint64_t o = hb[j]; o < hb[j + 1]; ++o) {
        const uint32_t key = uint32_t(ho[o]), idx = uint32_t(ho[o] >> 32);
        const uint32_t sl = uint32_t((uint64_t(h_fmix32(key + seed)) * nbk) >> 32);
        if (sl != uint32_t(j) || idx >= n || seen[idx] || hk[idx] != key) ++bad;
        else seen[idx] = 1;
      }
    if (hb[nbk] != n) ++bad;
    printf("{\"check\": \"%s\", \"nbk\": %d, \"bad\": %llu}\n", name, nbk, (unsigned long long)bad);
    return bad == 0;
  };
  wd::DstPtrs dst{};
  dst.p[0] = out;
  bool ok = true;
  for (int nbk : {32, 64, 128}) {
    auto k2 = nbk <= 32 ? wd::multisplit_kernel<true, 1, true, true> : nbk <= 64 ? wd::multisplit_kernel<true, 2, true, true>
                                                                                 : wd::multisplit_kernel<true, 4, true, true>;
    const int S = sms * occ(k2);
    const uint64_t L = ((n + S - 1) / S + wd::kMs2Tile - 1) / wd::kMs2Tile * wd::kMs2Tile;
    auto seg_prep = [&] {
      wd::seg_hist_kernel<<<S, wd::kBlock>>>(k, n, L, nbk, seed, segc);
      wd::seg_scan_kernel<<<1, 1024>>>(segc, S, nbk, bounds, cursor, sego);
    };
    const float th = time_ms([&] { wd::seg_hist_kernel<<<S, wd::kBlock>>>(k, n, L, nbk, seed, segc); }, reps);
    const float tsh = time_ms(seg_prep, reps);
    const float t2 = time_ms([&] {
      k2<<<S, wd::kBlock>>>(k, v, n, dst, nullptr, sego, L, nullptr, nbk, seed, n, ctr);
    }, reps);
    ok &= check(nbk, "multisplit");
    const float t2all = time_ms([&] {
      seg_prep();
      k2<<<S, wd::kBlock>>>(k, v, n, dst, nullptr, sego, L, nullptr, nbk, seed, n, ctr);
    }, reps);
    printf("{\"nbk\": %d, \"seg_hist_ms\": %.4f, \"seg_hist_scan_ms\": %.4f, \"multisplit_ms\": %.4f, "
           "\"group_ms\": %.4f, \"occ\": %d, \"S\": %d, \"ipt\": %d, \"GBps\": %.1f, \"frac_copy\": %.3f}\n",
           nbk, th, tsh, t2, t2all, occ(k2), S, wd::kMs2IPT, gb / t2 * 1e3, tcopy / t2);
  }
  // the cascade form (cursor mode): m owners, separate buffers, pairs and keys + pos; timed
  // at 2^n / 8 owners, checked also on small batches with partial tiles
  auto cascade = [&](uint64_t nc, int m, bool timed, int mis = 0) {
    const uint64_t B = nc / m + 4096 + nc / 16;
    unsigned long long* rbuf; uint32_t* posb;
    CK(cudaMalloc(&rbuf, B * m * 8)); CK(cudaMalloc(&posb, nc * 4 + 4));
    wd::DstPtrs dd{};
    for (int d = 0; d < m; ++d) dd.p[d] = rbuf + d * B;
    auto run2 = [&](bool pairs) {
      CK(cudaMemsetAsync(cursor, 0, m * 8));
      const int g = std::min<uint64_t>((nc + wd::kMs2TileC - 1) / wd::kMs2TileC,
                                       uint64_t(sms) * occ(wd::multisplit_kernel<true, 1, false, false, 0>));
      if (pairs) wd::multisplit_kernel<true, 1, false, false, 0><<<g, wd::kBlock>>>(k + mis, v + mis, nc, dd, cursor, nullptr, 0, nullptr, m, seed, B, ctr);
      else wd::multisplit_kernel<false, 1, false, false, 0><<<g, wd::kBlock>>>(k + mis, nullptr, nc, dd, cursor, nullptr, 0, posb, m, seed, B, ctr);
    };
    for (bool pairs : {true, false}) {
      const float b = timed ? time_ms([&] { run2(pairs); }, reps) : 0.f;
      run2(pairs);
      CK(cudaDeviceSynchronize());
      std::vector<unsigned long long> cur(m);
      CK(cudaMemcpy(cur.data(), cursor, m * 8, cudaMemcpyDeviceToHost));
      uint64_t bad = 0, tot = 0;
      std::vector<uint32_t> hp;
      if (!pairs) { hp.resize(nc); CK(cudaMemcpy(hp.data(), posb, nc * 4, cudaMemcpyDeviceToHost)); }
      for (int d = 0; d < m; ++d) {
        tot += cur[d];
        if (cur[d] > B) { ++bad; continue; }
        if (pairs) {
          std::vector<unsigned long long> r(cur[d]);
          CK(cudaMemcpy(r.data(), rbuf + d * B, cur[d] * 8, cudaMemcpyDeviceToHost));
          for (auto x : r) {
            const uint32_t key = uint32_t(x), idx = uint32_t(x >> 32);
            if (idx < uint32_t(mis) || idx >= nc + mis || hk[idx] != key || ((uint64_t(h_fmix32(key + seed)) * m) >> 32) != uint64_t(d)) ++bad;
          }
        } else {
          std::vector<uint32_t> r(cur[d]);
          CK(cudaMemcpy(r.data(), reinterpret_cast<uint32_t*>(rbuf + d * B), cur[d] * 4, cudaMemcpyDeviceToHost));
          for (uint64_t i = 0; i < nc; ++i) {
            if ((hp[i] >> wd::kPosShift) != uint32_t(d)) continue;
            const uint32_t o = hp[i] & ((1u << wd::kPosShift) - 1);
            if (o >= cur[d] || r[o] != hk[i + mis]) ++bad;
          }
        }
      }
      if (tot != nc) ++bad;
      ok &= bad == 0;
      printf("{\"cascade_m\": %d, \"n\": %llu, \"misaligned\": %d, \"pairs\": %d, \"ms\": %.4f, \"ipt\": %d, \"bad\": %llu}\n", m,
             (unsigned long long)nc, mis, int(pairs), b, WD_MS2_IPTC, (unsigned long long)bad);
    }
    CK(cudaFree(rbuf)); CK(cudaFree(posb));
  };
  cascade(n, 8, true);
  cascade(n / 2, 2, true);   // pos offsets hold 27 bits: batches of <= 2^27 items per owner
  for (int mis : {0, 1})
    for (int mm : {2, 3})
      for (uint64_t nc : {1ull, 100ull, 3656ull, 4096ull, 8192ull, 9000ull, 60000ull, 1000003ull}) cascade(nc, mm, false, mis);
  unsigned long long hc[16];
  CK(cudaMemcpy(hc, ctr, sizeof hc, cudaMemcpyDeviceToHost));
  printf("{\"xerr\": %llu, \"ok\": %d}\n", hc[wd::CNT_XERR], int(ok));
  return ok ? 0 : 1;
}
