// =====================================================================================
// wd_host.cuh — internal host-side header of libwarpdrive.so (not installed, not part of
// the C-ABI): the table / shard state and the probe-kernel dispatch templates.
//
// The probe dispatch (launch_probe_g<G, INSERT, In, Out>) is explicitly instantiated once
// per group size in probe_g{1,2,4,8,16,32}.cu, so the six template-heavy translation units
// compile in parallel; warpdrive.cu sees them through the extern declarations below.
// =====================================================================================
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <type_traits>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "../../include/warpdrive.h"
#include "wd_device.cuh"

namespace wdi {

// last error of this thread (defined in warpdrive.cu)
extern thread_local wd_status_t g_last;
extern thread_local char g_msg[1024];
wd_status_t fail(wd_status_t s, const char* fmt, ...);

#define CK(x)                                                                            \
  do {                                                                                   \
    cudaError_t e_ = (x);                                                                \
    if (e_ != cudaSuccess)                                                               \
      return fail(e_ == cudaErrorMemoryAllocation ? WD_ERR_OUT_OF_MEMORY : WD_ERR_CUDA,  \
                  "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__);     \
  } while (0)
#define TRY(x)                          \
  do {                                  \
    wd_status_t s_ = (x);               \
    if (s_ != WD_OK) return s_;         \
  } while (0)

enum Mode { MODE_SINGLE = 0, MODE_LOOPBACK = 1, MODE_MULTI = 2, MODE_RANK = 3 };
enum Flag { FLAG_READY = 0, FLAG_DONE = 1, FLAG_RESC = 2, FLAG_N = 3 };
enum PtrKind { PK_DEVICE = 0, PK_PINNED = 1, PK_PAGEABLE = 2 };

constexpr unsigned long long kWaitTimeoutNs = 30ull * 1000 * 1000 * 1000;  // 30 s

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    cudaGetDevice(&prev);
    if (prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    int cur;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

// pointers into one shard's exchange arena, valid in this process (own or peer-mapped)
struct PeerView {
  unsigned long long* recv[2] = {nullptr, nullptr};        // [m][B] items written by senders
  unsigned long long* res[2] = {nullptr, nullptr};         // [m][B] packed query results, region d pushed by owner d
  unsigned long long* recv_count[2] = {nullptr, nullptr};  // [m] column of T
  unsigned long long* flags = nullptr;                     // [FLAG_N][m]
};

// Out-of-core staging depth (Fig. 5).  Three slots: a query batch's slot is busy for
// H2D + probe + D2H, so with two slots the pipeline runs at half that cycle, ~10 % slower
// than the D2H stream alone; with three the slowest copy direction sets the pace.
constexpr int kStage = 3;

struct Shard {
  int id = 0;        // global shard index (= owner id of p(k))
  int device = 0;
  uint64_t cap = 0, nb = 0;
  uint32_t hseed = 0;            // hash seed of the current table (changes on rebuild)
  unsigned long long* slots = nullptr;
  unsigned long long* counters = nullptr;
  // slice-grouped bulk insert (slice_insert): packed-pair scratch for one chunk, and
  // counts[32] | bounds[33] | cursor[32]; sl_done orders reuse across streams
  unsigned long long* sl_buf[2] = {nullptr, nullptr};   // double buffer: group c+1 || probe c
  uint64_t sl_cap[2] = {0, 0};
  unsigned long long* sl_meta = nullptr;
  cudaEvent_t sl_done = nullptr, sl_fork = nullptr;
  cudaEvent_t sl_grouped[2] = {}, sl_probed[2] = {};
  cudaStream_t s_group = nullptr;
  bool sl_used = false;
  cudaStream_t s_main = nullptr, s_h2d = nullptr, s_d2h = nullptr;
  cudaStream_t s_probe = nullptr;   // phase B of the cascade (own stream unless loopback)
  bool own_main = true;
  // exchange arena (one allocation: IPC-exportable)
  void* arena = nullptr;
  size_t arena_bytes = 0;
  PeerView self;
  unsigned long long* cursor[2] = {nullptr, nullptr};  // [m] local send counters
  uint32_t* pos[2] = {nullptr, nullptr};               // [B] query positions
  // staging for host input / output: kStage slots, batch b in slot b % kStage
  uint64_t st_batch = 0;
  uint32_t *st_keys[kStage] = {}, *st_vals[kStage] = {}, *st_vout[kStage] = {};
  uint8_t* st_fout[kStage] = {};
  uint64_t pin_batch = 0;
  uint32_t *pin_keys[kStage] = {}, *pin_vals[kStage] = {}, *pin_vout[kStage] = {};
  uint8_t* pin_fout[kStage] = {};
  cudaEvent_t ev_h2d[kStage] = {}, ev_free[kStage] = {}, ev_kdone[kStage] = {}, ev_d2h[kStage] = {};
  cudaEvent_t ev_join_main = nullptr, ev_join_h2d = nullptr, ev_join_d2h = nullptr;
  cudaEvent_t ev_join_probe = nullptr;
  cudaEvent_t ev_fork = nullptr;   // _sharded calls: this shard's caller stream
  bool h2d_pending[kStage] = {};   // the slot's staging buffers have a pending release (ev_free)
  // staged exchange (WD_OPT_EXCHANGE = 1 copy engine, 2 NCCL): the multisplit writes the
  // batch into a local send buffer [m][B]; query results are staged in res_stage [m][B]
  // before the reverse transfer.  hrow / hcol: pinned host copies of this shard's row /
  // column of T per exchange slot; Tdev: the gathered T (NCCL rank mode)
  void* send = nullptr;
  unsigned long long* res_stage = nullptr;
  uint64_t staged_B = 0;
  unsigned long long* hrow[2] = {nullptr, nullptr};
  unsigned long long* hcol[2] = {nullptr, nullptr};
  unsigned long long* hT[2] = {nullptr, nullptr};
  unsigned long long* Tdev[2] = {nullptr, nullptr};
  cudaEvent_t ev_row = nullptr, ev_col = nullptr;
  cudaEvent_t ev_ready[2] = {}, ev_pdone[2] = {}, ev_done[2] = {}, ev_unperm[2] = {};
  bool pdone_rec[2] = {}, unperm_rec[2] = {};
  unsigned long long* fail_list = nullptr;    // inserts that hit Line 26 (WD_OPT_AUTO_REBUILD)
  unsigned long long* fail_count = nullptr;
  void* comm_fwd = nullptr;        // ncclComm_t of the forward / reverse transpositions
  void* comm_rev = nullptr;
  bool l2_held = false;            // holds the device's L2 fetch-granularity setting
};

}  // namespace wdi

struct wd_table {
  int mode = wdi::MODE_SINGLE;
  int m = 1;          // number of shards (= GPUs, or virtual shards in loopback)
  int rank = 0;       // rank mode: this process's shard id
  int G = 4;          // |g|, or 0 = dynamic by load
  int G_used = 4;     // |g| of the current / last call
  int G_ins = 4;      // |g| of the last insert (dynamic |g|: by load)
  int qg = -1;        // |g| of query / erase calls (WD_OPT_QUERY_GROUP_SIZE; -1 auto, 0 table's)
  int ig = -1;        // |g| of insert calls (WD_OPT_INSERT_GROUP_SIZE; -1 auto, 0 table's)
  uint32_t align = 4; // A of reading C2': 16 for tables created with |g| >= 16, else 4
  uint64_t est_size = 0;   // host-side upper estimate of the stored keys (no sync needed)
  int pmax = 0;      // 0: p_max = nb (full period, C4'), else explicit
  int kif = 0;        // keys in flight per group (0 = default)
  int probe_mode = 0; // 0: auto, 1: cooperative groups (Fig. 3), 2: lane-window (|g| <= 8)
  int spl = 0;        // slots per lane V (WD_OPT_SLOTS_PER_LANE; 0 = from probe mode)
  int span = 0;       // windows per lane load S (WD_OPT_SPAN; 0 = auto)
  int slices = 0;     // table slices of a grouped bulk insert (WD_OPT_SLICES; 0 = auto)
  // wd::kF_* kernel variants (WD_OPT_KERNEL_FLAGS).  Default all three: atom.exch value
  // updates take hot (Zipf) keys from 0.5 to 6-8 G inserts/s (tools/flags_bench.py),
  // L1-allowed probe loads add ~15 % there; the scrambled query chunk order adds 22-40 % to
  // queries issued in insert order (profiles/r01_query_order.md).
  uint32_t kflags = wd::kF_L1 | wd::kF_XCHG | wd::kF_QSCR;
  uint64_t batch = 1ull << 24;
  bool batch_set = false;  // WD_OPT_BATCH given: the single-shard pipeline uses it as is
  int serial = 0;
  uint32_t pseed = 0x9E3779B9u;
  int pmode = 0;
  unsigned long long epoch = 0;
  unsigned long long res_used[2] = {0, 0};  // last (query) epoch that filled result slot i
  uint64_t launches = 0;
  uint64_t xbatch = 0;  // batch size the exchange arenas were built for
  int sm_count = 148;
  std::vector<wdi::Shard> local;
  std::vector<wdi::PeerView> peers;  // size m
  std::vector<void*> opened;    // IPC-mapped peer arenas (rank mode)
  // rank mode: host collective supplied by the caller (torch.distributed), connected peers
  wd_allreduce_fn allreduce = nullptr;
  void* allreduce_ctx = nullptr;
  bool connected = false;
  cudaStream_t loop_stream = nullptr;       // loopback: one stream for all shards
  // a8 / a10 transport (WD_OPT_EXCHANGE): 0 fused peer stores in the multisplit / probe
  // kernels, 1 staged buffers + copy engine (cudaMemcpyAsync of exact counts, the paper's
  // "asynchronous inter-GPU copies"), 2 staged buffers + NCCL send/recv (all-to-all(v) of
  // exact counts after an all-gather of T; the north star's NCCL path)
  int exchange = 0;
  bool auto_rebuild = false;  // WD_OPT_AUTO_REBUILD
  uint32_t rebuilds = 0;      // automatic rebuilds so far (new seeds are derived from it)
  // per-phase CUDA-event timing (WD_OPT_PHASE_TIMING, wd_phase_times): begin/end event pairs
  // recorded on the stream each phase runs on; events are pooled per device
  bool phase_on = false;
  struct PhaseRec { int phase, device; cudaEvent_t a, b; };
  std::vector<PhaseRec> ph_recs;
  std::unordered_map<int, std::vector<cudaEvent_t>> ph_pool;
  bool nccl_ready = false;
  unsigned char nccl_id[128] = {};           // rank mode: rank 0's ncclUniqueId (wd_rank_connect)
  bool have_nccl_id = false;
};

namespace wdi {

// ------------------------------------------------------------------ helpers
inline uint64_t round_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

inline PtrKind classify(const void* p, int* dev) {
  if (!p) return PK_DEVICE;
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return PK_PAGEABLE;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
    if (dev) *dev = a.device;
    return PK_DEVICE;
  }
  if (a.type == cudaMemoryTypeHost) return PK_PINNED;
  return PK_PAGEABLE;
}

// resident blocks per SM of a kernel (occupancy API), cached; tables may be used from
// several host threads (one thread per table), so the cache is guarded
template <class K>
int blocks_per_sm(K kern) {
  static std::unordered_map<const void*, int> cache;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find((const void*)kern);
  if (it != cache.end()) return it->second;
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, wd::kBlock, 0) != cudaSuccess) {
    cudaGetLastError();
    nb = 1;
  }
  nb = std::max(nb, 1);
  cache[(const void*)kern] = nb;
  return nb;
}

// ------------------------------------------------------------------ probe dispatch
constexpr uint32_t kFailCap = 1u << 20;   // failed-insert list per shard (8 MB, auto rebuild)

template <int G, int V, int K, bool INSERT, class In, class Out, int S = 1>
wd_status_t launch_probe_k(wd_table* t, Shard& s, const In& in, const Out& out, uint64_t n_hint,
                           cudaStream_t st) {
  auto kern = wd::probe_kernel<G, V, K, INSERT, In, Out, S>;
  // C4': default p_max = nb — eq. 3 then visits every region, so an insert fails only when
  // no slot is free (a fixed 1024 is exceeded at alpha = 0.999 even sequentially).
  const uint32_t pmax = t->pmax > 0 ? static_cast<uint32_t>(t->pmax) : static_cast<uint32_t>(s.nb);
  wd::TableView tv{s.slots, static_cast<uint32_t>(s.nb), pmax, t->kflags, s.hseed, t->align,
                   INSERT && t->auto_rebuild ? s.fail_list : nullptr, s.fail_count, kFailCap};
  int grid = 1, block = 32;
  if (!t->serial) {
    block = wd::kBlock;
    const uint64_t keys_per_block = uint64_t(wd::kBlock / 32) * K * (32 / (G / V));
    const uint64_t need = std::max<uint64_t>(1, (n_hint + keys_per_block - 1) / keys_per_block);
    grid = static_cast<int>(std::min<uint64_t>(need, uint64_t(t->sm_count) * blocks_per_sm(kern)));
    static const int cap_env = getenv("WD_MAX_BLOCKS") ? atoi(getenv("WD_MAX_BLOCKS")) : 0;
    if (cap_env > 0) grid = std::min(grid, cap_env);   // measurement hook (tools/)
  }
  kern<<<grid, block, 0, st>>>(tv, in, out, s.counters, t->serial);
  CK(cudaGetLastError());
  t->launches++;
  return WD_OK;
}

// instantiated (|g|, V, K) combinations: V = slots per lane (1: the paper's cooperative
// group of |g| lanes; |g|: one lane per window), K = keys in flight per group
// windows per lane load S (span read-ahead, one lane per window): 2 for L2-resident tables
// with |g| <= 4 — calls on them are bound by the longest probe chain, not by bandwidth
// (profiles/r01_small_calls.md), and S = 2 halves its round trips — and for |g| = 1 at any
// size (7 windows per insert at alpha 0.95).  Measured (tools/span_bench.py,
// profiles/r01_span.txt): config 1 (2^20 keys, |g| = 4) 5.4 -> 9.1 G inserts/s and
// 5.9 -> 8.8 G queries/s; |g| = 1 at 2^26 keys 3.9 -> 7.3 G inserts/s (queries equal).
// Single-shard input only.
inline int choose_span(const wd_table* t, const Shard& s, int G, int V) {
  if (V != G || G > 4 || t->span == 1) return 1;
  if (t->span == 2 || G == 1) return 2;
  return s.cap * sizeof(unsigned long long) <= (64ull << 20) ? 2 : 1;
}

template <int G, int V, bool INSERT, class In, class Out>
wd_status_t launch_gv(wd_table* t, Shard& s, const In& in, const Out& out, uint64_t n_hint,
                      cudaStream_t st, int k) {
  if constexpr (V == G && G <= 4 && std::is_same_v<In, wd::InSoA>) {
    // span read-ahead variants, at the K the auto choice uses for these (G, V)
    constexpr int KS = G == 1 ? 8 : G == 2 ? 4 : 2;
    if (k == KS && choose_span(t, s, G, V) == 2)
      return launch_probe_k<G, V, KS, INSERT, In, Out, 2>(t, s, in, out, n_hint, st);
  }
  if constexpr (V == 16) {          // one lane reads a whole 128-byte window
    if (k <= 1) return launch_probe_k<G, 16, 1, INSERT>(t, s, in, out, n_hint, st);
    return launch_probe_k<G, 16, 2, INSERT>(t, s, in, out, n_hint, st);
  } else if constexpr (V == 1) {
    if (k == 2) return launch_probe_k<G, 1, 2, INSERT>(t, s, in, out, n_hint, st);
    if (k == 4) return launch_probe_k<G, 1, 4, INSERT>(t, s, in, out, n_hint, st);
    return launch_probe_k<G, 1, 8, INSERT>(t, s, in, out, n_hint, st);
  } else if constexpr (V == 2) {
    if (k <= 4) return launch_probe_k<G, 2, 4, INSERT>(t, s, in, out, n_hint, st);
    return launch_probe_k<G, 2, 8, INSERT>(t, s, in, out, n_hint, st);
  } else if constexpr (V == 4) {
    if (k <= 2) return launch_probe_k<G, 4, 2, INSERT>(t, s, in, out, n_hint, st);
    return launch_probe_k<G, 4, 4, INSERT>(t, s, in, out, n_hint, st);
  } else {
    return launch_probe_k<G, 8, 2, INSERT>(t, s, in, out, n_hint, st);
  }
}

// Slots per lane V (window read by |g|/V lanes) and keys in flight K for this call.
// Explicit WD_OPT_SLOTS_PER_LANE / WD_OPT_KEYS_IN_FLIGHT win; probe mode 1 forces the
// paper's cooperative group (V = 1), mode 2 one lane per window (V = |g| <= 8).  Auto,
// from measurements on B200 (tools/kbench.py split, profiles/r01_split.txt):
//  * shard in half the L2 (<= 64 MB): one lane per window, K = 2 for 32/64-byte windows —
//    instruction-lean (e.g. |g| = 8: 18 G inserts/s, 32 G queries/s at 2^22 keys);
//  * from HBM: two lanes per window (V = |g|/2), K = 2-4 — a warp step then waits for
//    the slowest of 16 loads, not 32, with half the instructions of V = 1
//    (|g| = 8, alpha 0.95, 2^28: 12.9 G inserts/s, 23.4 G queries/s vs 9.8 / 12.1 at V = 1).
//    Lanes load at most 64 B (V <= 8), inserts on 32-B-aligned tables at most 32 B (V <= 4):
//    |g| = 16 queries 24.3 G/s at V = 8 vs 18.6 at V = 4 (profiles/r01_query_order.md);
//    on line-aligned tables (A = 16, reading C2') inserts too: |g| = 16 14.3 -> 15.0 G/s,
//    |g| = 32 10.9 -> 12.9 G/s at V = 8, while |g| = 8 (A = 4) drops 12.9 -> 8.3
//    (tools/kbench.py cfg, profiles/r01_ab_insert_v8.txt).
inline int choose_v(const wd_table* t, const Shard& s, int G, bool insert) {
  int v = t->spl;
  if (v == 0) {
    const bool small = s.cap * sizeof(unsigned long long) <= (64ull << 20);
    if (t->probe_mode == 1) v = 1;
    else if (t->probe_mode == 2 || small) v = G;
    else v = G >= 2 ? std::max(1, std::min(G / 2, insert && t->align < 16 ? 4 : 8)) : 1;
    if (G == 2 && t->probe_mode == 0) v = 2;
    // |g| = 32 queries from HBM: two lanes of one 128-B line each (19.4 vs 18.3 G/s at 2^28)
    if (G == 32 && !insert && !small && t->probe_mode == 0 && t->align == 16) v = 16;
  }
  v = std::min(v, std::min(G, (t->spl == 16 || v == 16) ? 16 : 8));
  return v;
}
inline int choose_k(const wd_table* t, const Shard& s, int G, int V, bool insert) {
  if (t->kif) return t->kif;
  // |g| = 1 inserts into tables > 1 GB run slice-grouped (no span read-ahead): K = 4
  // (2^28, alpha 0.95: 7.5 -> 9.7 G/s); queries and smaller tables keep K = 8 with the span.
  if (V == 1) return (G == 1 && insert && double(s.cap) * 8 > 1.0e9) ? 4 : (G <= 4 ? 8 : 4);
  // V = 2: K = 4 everywhere (K = 8 spills: |g| = 2 from HBM 10.1 -> 14.3 G inserts/s and
  // 7.0 -> 10.4 G queries/s, tools/rates.py, profiles/r02/small_g.jsonl)
  if (V == 2) return 4;
  // V = 4: K = 2 (4 blocks/SM for inserts).  Judged on the whole step (tools/ab_retrieve.py,
  // |g| = 8, 2^28): insert/retrieve K = 2/2 -> 13.7 / 22.6 G/s (17.1 G ops/s combined),
  // 4/4 -> 12.9 / 23.5 (16.7), 2/4 -> 13.7 / 21.9 (16.8).
  (void)insert;
  if (V == 4) return 2;
  if (V == 16) return 1;
  return 2;
}

template <int G, bool INSERT, class In, class Out>
wd_status_t launch_probe_g(wd_table* t, Shard& s, const In& in, const Out& out, uint64_t n_hint,
                           cudaStream_t st) {
  // sliced bulk inserts (InBucket) on line-aligned tables: one lane reads the whole 128-B
  // window (V = 16, K = 1; tools/gpu_vk_sweep.sh: 2^28 pairs 18.8 -> 19.7 G inserts/s, 2^24
  // 20.5 -> 22.8) while the projected load stays <= 0.975 — above it, with longer chains, two
  // lanes of 64 B and two keys in flight win (alpha 0.97 / 0.98 / 0.99: 17.7 / 15.9 / 13.4
  // vs 17.1 / 16.2 / 14.9 G/s).  Not for queries from HBM: one lane per 128-B line drops them
  // to 9 G/s.
  // The same holds for every |g| >= 4 in the sliced launches (a good part of each slice is in
  // L2, where one lane per window is the instruction-lean choice, as for small tables):
  // |g| = 4 V = 4, K = 2: 16.4 -> 19.9; |g| = 8 V = 8, K = 2: 18.8 -> 21.1; |g| = 32 V = 16,
  // K = 1 (two lanes of one line each): 12.9 -> 14.1 G inserts/s (tools/gpu_vk_all.sh,
  // profiles/r02/vk_all.jsonl, 2^28, alpha 0.95).
  if constexpr (G >= 4 && INSERT && std::is_same_v<In, wd::InBucket>)
    if (t->spl == 0 && t->kif == 0 && t->probe_mode == 0 &&
        double(t->est_size) <= 0.975 * double(s.cap)) {
      if constexpr (G >= 16) {
        if (t->align == 16) return launch_gv<G, 16, INSERT>(t, s, in, out, n_hint, st, 1);
      } else {
        return launch_gv<G, G, INSERT>(t, s, in, out, n_hint, st, 2);
      }
    }
  const int v = choose_v(t, s, G, INSERT), k = choose_k(t, s, G, v, INSERT);
  if constexpr (G >= 16)
    if (v == 16) return launch_gv<G, 16, INSERT>(t, s, in, out, n_hint, st, k);
  if constexpr (G >= 8)
    if (v == 8) return launch_gv<G, 8, INSERT>(t, s, in, out, n_hint, st, k);
  if constexpr (G >= 4)
    if (v == 4) return launch_gv<G, 4, INSERT>(t, s, in, out, n_hint, st, k);
  if constexpr (G >= 2)
    if (v == 2) return launch_gv<G, 2, INSERT>(t, s, in, out, n_hint, st, k);
  return launch_gv<G, 1, INSERT>(t, s, in, out, n_hint, st, k);
}

// (In, Out) combinations the library launches; each is instantiated for every |g| in
// probe_g<G>.cu and declared extern everywhere else
#define WD_PROBE_COMBOS(X, G)                                 \
  X(G, true, wd::InSoA, wd::OutNone)                          \
  X(G, true, wd::InBucket, wd::OutNone)                       \
  X(G, true, wd::InSeg<true>, wd::OutNone)                    \
  X(G, false, wd::InSoA, wd::OutSoA)                          \
  X(G, false, wd::InSoA, wd::OutErase<wd::OutSoA>)            \
  X(G, false, wd::InSeg<false>, wd::OutPacked)                \
  X(G, false, wd::InSeg<false>, wd::OutErase<wd::OutPacked>) \
  X(G, false, wd::InSeg<false>, wd::OutLocalPacked)          \
  X(G, false, wd::InSeg<false>, wd::OutErase<wd::OutLocalPacked>)
#define WD_PROBE_SIG(G, I, IN, OUT) \
  launch_probe_g<G, I, IN, OUT>(wd_table*, Shard&, const IN&, const OUT&, uint64_t, cudaStream_t)
#define WD_PROBE_EXTERN(G, I, IN, OUT) extern template wd_status_t WD_PROBE_SIG(G, I, IN, OUT);
#define WD_PROBE_INST(G, I, IN, OUT) template wd_status_t WD_PROBE_SIG(G, I, IN, OUT);
#ifndef WD_PROBE_TU
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 1)
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 2)
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 4)
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 8)
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 16)
WD_PROBE_COMBOS(WD_PROBE_EXTERN, 32)
#endif

template <bool INSERT, class In, class Out>
wd_status_t launch_probe(wd_table* t, Shard& s, const In& in, const Out& out, uint64_t n_hint,
                         cudaStream_t st) {
  // inserts (including rebuild re-inserts) with the inserts' |g|; queries / erases with the
  // |g| pick_group_size chose for the call
  const int G = INSERT ? t->G_ins : t->G_used;
  switch (G) {
    case 1: return launch_probe_g<1, INSERT>(t, s, in, out, n_hint, st);
    case 2: return launch_probe_g<2, INSERT>(t, s, in, out, n_hint, st);
    case 4: return launch_probe_g<4, INSERT>(t, s, in, out, n_hint, st);
    case 8: return launch_probe_g<8, INSERT>(t, s, in, out, n_hint, st);
    case 16: return launch_probe_g<16, INSERT>(t, s, in, out, n_hint, st);
    case 32: return launch_probe_g<32, INSERT>(t, s, in, out, n_hint, st);
  }
  return fail(WD_ERR_INVALID_ARG, "group size %d not in {1,2,4,8,16,32}", G);
}

}  // namespace wdi
