// =====================================================================================
// warpdrive.cu — host side of libwarpdrive.so: the C-ABI of include/warpdrive.h.
//
//   wd_table ........ m shards ("GPU i exclusively holds keys where p(k) = i"),
//                     of which this process owns 1 (single / rank mode) or all
//                     (loopback: m virtual shards on one device; multi: one per device).
//   single path ..... device input: one probe kernel on the caller's stream.
//                     host input: out-of-core pipeline H2D(b+1) || probe(b) || D2H(b-1)
//                     on three streams with double-buffered staging (Fig. 5).
//   cascade (m > 1) . per batch: multisplit fused with the push into the owners'
//                     receive regions -> publish T row + ready flags -> owner waits for its
//                     T column -> local insert / query, results pushed back into the
//                     origins' result regions -> done flags -> (query) origin unpermutes
//                     from its own memory -> consumed flags.  All signalling
//                     is device-side (no host synchronisation per batch); receive and
//                     result regions are double-buffered by epoch parity.
// =====================================================================================
#include "wd_host.cuh"

#include <dlfcn.h>
#include <nvtx3/nvToolsExt.h>

#include <mutex>

namespace wdi {

thread_local wd_status_t g_last = WD_OK;
thread_local char g_msg[1024] = "";

wd_status_t fail(wd_status_t s, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_msg, sizeof g_msg, fmt, ap);
  va_end(ap);
  g_last = s;
  return s;
}

// ------------------------------------------------------------------ NCCL (WD_OPT_EXCHANGE = 2)
// Loaded at run time (dlopen), so the library needs NCCL only when the NCCL exchange is
// selected: the copy already in the process (torch's), else libnccl.so.2 from the loader
// path.  Only ABI-stable NCCL 2.x types are used (ncclUniqueId = 128 bytes, ncclUint8 = 1,
// ncclUint64 = 5).
struct NcclUid { char internal[128]; };
constexpr int kNcclUint8 = 1, kNcclUint64 = 5;
struct NcclApi {
  bool tried = false, ok = false;
  char why[256] = "";
  int (*GetUniqueId)(NcclUid*) = nullptr;
  int (*CommInitRank)(void**, int, NcclUid, int) = nullptr;
  int (*CommInitAll)(void**, int, const int*) = nullptr;
  int (*CommSplit)(void*, int, int, void**, void*) = nullptr;
  int (*CommDestroy)(void*) = nullptr;
  int (*GroupStart)() = nullptr;
  int (*GroupEnd)() = nullptr;
  int (*Send)(const void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*Recv)(void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*AllGather)(const void*, void*, size_t, int, void*, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(int) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

const NcclApi* nccl_api() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  NcclApi& a = g_nccl;
  if (a.tried) return a.ok ? &a : nullptr;
  a.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    snprintf(a.why, sizeof a.why, "libnccl.so.2 not loadable: %s", dlerror());
    return nullptr;
  }
#define WD_NCCL_SYM(f, name)                                                        \
  a.f = reinterpret_cast<decltype(a.f)>(dlsym(h, name));                            \
  if (!a.f) { snprintf(a.why, sizeof a.why, "NCCL symbol %s missing", name); return nullptr; }
  WD_NCCL_SYM(GetUniqueId, "ncclGetUniqueId")
  WD_NCCL_SYM(CommInitRank, "ncclCommInitRank")
  WD_NCCL_SYM(CommInitAll, "ncclCommInitAll")
  WD_NCCL_SYM(CommSplit, "ncclCommSplit")
  WD_NCCL_SYM(CommDestroy, "ncclCommDestroy")
  WD_NCCL_SYM(GroupStart, "ncclGroupStart")
  WD_NCCL_SYM(GroupEnd, "ncclGroupEnd")
  WD_NCCL_SYM(Send, "ncclSend")
  WD_NCCL_SYM(Recv, "ncclRecv")
  WD_NCCL_SYM(AllGather, "ncclAllGather")
  WD_NCCL_SYM(GetErrorString, "ncclGetErrorString")
#undef WD_NCCL_SYM
  a.ok = true;
  return &a;
}
#define NK(x)                                                                              \
  do {                                                                                     \
    const int r_ = (x);                                                                    \
    if (r_ != 0)                                                                           \
      return fail(WD_ERR_NCCL, "%s: %s (%s:%d)", #x, g_nccl.GetErrorString(r_), __FILE__, \
                  __LINE__);                                                               \
  } while (0)

// ------------------------------------------------------------------ phases: events + NVTX
// WD_OPT_PHASE_TIMING = 1 records a CUDA-event pair around every phase of every batch, on
// the stream the phase runs on (the decomposition of Fig. 11); wd_phase_times
// sums them.  NVTX ranges mark the host-side issue of every call and phase (for nsys /
// ncu --nvtx; no-ops without a tool attached).
struct Nvtx {
  explicit Nvtx(const char* name) { nvtxRangePushA(name); }
  ~Nvtx() { nvtxRangePop(); }
};
struct Ph { cudaEvent_t a = nullptr; int phase = 0, device = 0; cudaStream_t st = nullptr; };
cudaEvent_t ph_event(wd_table* t, int device) {
  auto& pool = t->ph_pool[device];
  if (!pool.empty()) {
    cudaEvent_t e = pool.back();
    pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  if (cudaEventCreate(&e) != cudaSuccess) { cudaGetLastError(); return nullptr; }
  return e;
}
Ph ph_begin(wd_table* t, int phase, int device, cudaStream_t st) {
  Ph p;
  if (!t->phase_on) return p;
  p.a = ph_event(t, device);
  if (p.a && cudaEventRecord(p.a, st) != cudaSuccess) { cudaGetLastError(); p.a = nullptr; }
  p.phase = phase; p.device = device; p.st = st;
  return p;
}
void ph_end(wd_table* t, const Ph& p) {
  if (!p.a) return;
  cudaEvent_t b = ph_event(t, p.device);
  if (!b || cudaEventRecord(b, p.st) != cudaSuccess) { cudaGetLastError(); return; }
  t->ph_recs.push_back({p.phase, p.device, p.a, b});
}

// ------------------------------------------------------------------ L2 fetch granularity
// Random 32-byte windows: do not let L2 promote a sector miss to a 64/128-byte DRAM fetch
// (measured: 6.7 DRAM sectors per |g| = 4 insert with the default, 2.4 needed).  The limit
// is device-wide, so it is scoped to the tables' lifetime: the first live shard on a device
// records the caller's value and sets 32 B; the last one destroyed restores it
// (include/warpdrive.h, wd_create).  WD_L2_FETCH_BYTES=<bytes> overrides, 0 leaves it alone.
struct L2Hold { int users = 0; size_t saved = 0; bool set = false; };
L2Hold g_l2[64];
std::mutex g_l2_mu;

wd_status_t l2_fetch_acquire(int device) {
  std::lock_guard<std::mutex> lk(g_l2_mu);
  if (device < 0 || device >= 64) return WD_OK;
  L2Hold& h = g_l2[device];
  if (h.users++ > 0) return WD_OK;
  size_t want = 32;
  if (const char* e = getenv("WD_L2_FETCH_BYTES")) want = size_t(atoi(e));
  h.set = false;
  if (want == 0) return WD_OK;
  CK(cudaDeviceGetLimit(&h.saved, cudaLimitMaxL2FetchGranularity));
  CK(cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, want));
  h.set = true;
  return WD_OK;
}
void l2_fetch_release(int device) {
  std::lock_guard<std::mutex> lk(g_l2_mu);
  if (device < 0 || device >= 64) return;
  L2Hold& h = g_l2[device];
  if (h.users <= 0 || --h.users > 0) return;
  if (h.set && cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, h.saved) != cudaSuccess)
    cudaGetLastError();
  h.set = false;
}

// ------------------------------------------------------------------ shard lifetime
wd_status_t shard_init(wd_table* t, Shard& s, int id, int device, uint64_t cap,
                       cudaStream_t shared_main) {
  DeviceGuard g(device);
  TRY(l2_fetch_acquire(device));
  s.l2_held = true;
  s.id = id;
  s.device = device;
  if (cap == 0) return fail(WD_ERR_INVALID_ARG, "capacity per shard exceeds 4 * 2^32 slots");
  s.cap = cap;
  s.nb = (cap - 32) / t->align + 1;
  CK(cudaMalloc(&s.slots, cap * sizeof(unsigned long long)));
  CK(cudaMalloc(&s.counters, wd::CNT_N * sizeof(unsigned long long)));
  if (shared_main) {
    s.s_main = s.s_probe = shared_main;   // loopback: one stream, phases in issue order
    s.own_main = false;
  } else {
    CK(cudaStreamCreateWithFlags(&s.s_main, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&s.s_probe, cudaStreamNonBlocking));
  }
  CK(cudaStreamCreateWithFlags(&s.s_h2d, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s.s_d2h, cudaStreamNonBlocking));
  for (int i = 0; i < kStage; ++i) {
    CK(cudaEventCreateWithFlags(&s.ev_h2d[i], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&s.ev_free[i], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&s.ev_kdone[i], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&s.ev_d2h[i], cudaEventDisableTiming));
  }
  CK(cudaEventCreateWithFlags(&s.ev_join_main, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_join_h2d, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_join_d2h, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_join_probe, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_fork, cudaEventDisableTiming));
  // a1: fresh table
  const int grid = t->sm_count * 4;
  wd::fill_kernel<<<grid, wd::kBlock, 0, s.s_main>>>(s.slots, s.cap, s.counters, wd::CNT_N);
  CK(cudaGetLastError());
  t->launches++;
  CK(cudaStreamSynchronize(s.s_main));  // device-path calls use the caller's stream
  return WD_OK;
}

void free_exchange(Shard& s) {
  DeviceGuard g(s.device);
  if (s.arena) cudaFree(s.arena);
  s.arena = nullptr;
  s.self = PeerView{};
  for (int i = 0; i < 2; ++i) {
    if (s.cursor[i]) cudaFree(s.cursor[i]);
    if (s.pos[i]) cudaFree(s.pos[i]);
    s.cursor[i] = nullptr;
    s.pos[i] = nullptr;
  }
}

void free_staging(Shard& s) {
  DeviceGuard g(s.device);
  for (int i = 0; i < kStage; ++i) {
    if (s.st_keys[i]) cudaFree(s.st_keys[i]);
    if (s.st_vals[i]) cudaFree(s.st_vals[i]);
    if (s.st_vout[i]) cudaFree(s.st_vout[i]);
    if (s.st_fout[i]) cudaFree(s.st_fout[i]);
    if (s.pin_keys[i]) cudaFreeHost(s.pin_keys[i]);
    if (s.pin_vals[i]) cudaFreeHost(s.pin_vals[i]);
    if (s.pin_vout[i]) cudaFreeHost(s.pin_vout[i]);
    if (s.pin_fout[i]) cudaFreeHost(s.pin_fout[i]);
    s.st_keys[i] = s.st_vals[i] = s.st_vout[i] = nullptr;
    s.st_fout[i] = nullptr;
    s.pin_keys[i] = s.pin_vals[i] = s.pin_vout[i] = nullptr;
    s.pin_fout[i] = nullptr;
  }
  s.st_batch = s.pin_batch = 0;
}

void shard_free(Shard& s) {
  DeviceGuard g(s.device);
  if (s.s_main) cudaStreamSynchronize(s.s_main);
  if (s.s_probe) cudaStreamSynchronize(s.s_probe);
  if (s.s_h2d) cudaStreamSynchronize(s.s_h2d);
  if (s.s_d2h) cudaStreamSynchronize(s.s_d2h);
  free_exchange(s);
  free_staging(s);
  for (int b = 0; b < 2; ++b) {
    if (s.sl_buf[b]) cudaFree(s.sl_buf[b]);
    if (s.sl_grouped[b]) cudaEventDestroy(s.sl_grouped[b]);
    if (s.sl_probed[b]) cudaEventDestroy(s.sl_probed[b]);
  }
  if (s.sl_meta) cudaFree(s.sl_meta);
  if (s.sl_done) cudaEventDestroy(s.sl_done);
  if (s.sl_fork) cudaEventDestroy(s.sl_fork);
  if (s.s_group) {
    cudaStreamSynchronize(s.s_group);
    cudaStreamDestroy(s.s_group);
  }
  if (s.slots) cudaFree(s.slots);
  if (s.counters) cudaFree(s.counters);
  if (s.fail_list) cudaFree(s.fail_list);
  if (s.fail_count) cudaFree(s.fail_count);
  for (int i = 0; i < kStage; ++i) {
    if (s.ev_h2d[i]) cudaEventDestroy(s.ev_h2d[i]);
    if (s.ev_free[i]) cudaEventDestroy(s.ev_free[i]);
    if (s.ev_kdone[i]) cudaEventDestroy(s.ev_kdone[i]);
    if (s.ev_d2h[i]) cudaEventDestroy(s.ev_d2h[i]);
  }
  if (s.ev_join_main) cudaEventDestroy(s.ev_join_main);
  if (s.ev_join_h2d) cudaEventDestroy(s.ev_join_h2d);
  if (s.ev_join_d2h) cudaEventDestroy(s.ev_join_d2h);
  if (s.ev_join_probe) cudaEventDestroy(s.ev_join_probe);
  if (s.ev_fork) cudaEventDestroy(s.ev_fork);
  if (s.l2_held) l2_fetch_release(s.device);
  if (s.own_main && s.s_main) cudaStreamDestroy(s.s_main);
  if (s.own_main && s.s_probe) cudaStreamDestroy(s.s_probe);
  if (s.s_h2d) cudaStreamDestroy(s.s_h2d);
  if (s.s_d2h) cudaStreamDestroy(s.s_d2h);
  s = Shard{};
}

wd_status_t ensure_staging(Shard& s, uint64_t B, bool pageable) {
  DeviceGuard g(s.device);
  if (s.st_batch < B) {
    for (int i = 0; i < kStage; ++i) {
      if (s.st_keys[i]) cudaFree(s.st_keys[i]);
      if (s.st_vals[i]) cudaFree(s.st_vals[i]);
      if (s.st_vout[i]) cudaFree(s.st_vout[i]);
      if (s.st_fout[i]) cudaFree(s.st_fout[i]);
      CK(cudaMalloc(&s.st_keys[i], B * 4));
      CK(cudaMalloc(&s.st_vals[i], B * 4));
      CK(cudaMalloc(&s.st_vout[i], B * 4));
      CK(cudaMalloc(&s.st_fout[i], B));
    }
    s.st_batch = B;
  }
  if (pageable && s.pin_batch < B) {
    for (int i = 0; i < kStage; ++i) {
      if (s.pin_keys[i]) cudaFreeHost(s.pin_keys[i]);
      if (s.pin_vals[i]) cudaFreeHost(s.pin_vals[i]);
      if (s.pin_vout[i]) cudaFreeHost(s.pin_vout[i]);
      if (s.pin_fout[i]) cudaFreeHost(s.pin_fout[i]);
      CK(cudaMallocHost(&s.pin_keys[i], B * 4));
      CK(cudaMallocHost(&s.pin_vals[i], B * 4));
      CK(cudaMallocHost(&s.pin_vout[i], B * 4));
      CK(cudaMallocHost(&s.pin_fout[i], B));
    }
    s.pin_batch = B;
  }
  return WD_OK;
}

// arena layout: recv[2] | res[2] | recv_count[2] | flags
PeerView arena_view(void* base, int m, uint64_t B) {
  PeerView v;
  char* p = static_cast<char*>(base);
  const size_t region = size_t(m) * B * 8;
  for (int i = 0; i < 2; ++i) v.recv[i] = reinterpret_cast<unsigned long long*>(p + i * region);
  p += 2 * region;
  for (int i = 0; i < 2; ++i) v.res[i] = reinterpret_cast<unsigned long long*>(p + i * region);
  p += 2 * region;
  for (int i = 0; i < 2; ++i) v.recv_count[i] = reinterpret_cast<unsigned long long*>(p + i * m * 8);
  p += 2 * m * 8;
  v.flags = reinterpret_cast<unsigned long long*>(p);
  return v;
}
size_t arena_size(int m, uint64_t B) {
  return 4 * size_t(m) * B * 8 + 2 * size_t(m) * 8 + size_t(FLAG_N) * m * 8 + 256;
}

wd_status_t exchange_init_shard(wd_table* t, Shard& s, uint64_t B) {
  DeviceGuard g(s.device);
  s.arena_bytes = arena_size(t->m, B);
  CK(cudaMalloc(&s.arena, s.arena_bytes));
  s.self = arena_view(s.arena, t->m, B);
  // counts and flags start at 0: epochs are >= 1
  CK(cudaMemsetAsync(s.self.recv_count[0], 0, 2 * t->m * 8 + FLAG_N * t->m * 8, s.s_main));
  for (int i = 0; i < 2; ++i) {
    CK(cudaMalloc(&s.cursor[i], t->m * 8));
    CK(cudaMemsetAsync(s.cursor[i], 0, t->m * 8, s.s_main));
    CK(cudaMalloc(&s.pos[i], B * 4));
  }
  CK(cudaStreamSynchronize(s.s_main));
  return WD_OK;
}

wd_status_t rank_allgather_views(wd_table* t, uint64_t B);

// Items per shard per cascade batch: WD_OPT_BATCH rounded up to a power of two, so the
// exchange regions sit a power of two apart and the owner's result push (OutPacked) finds
// its target region with a shift.
uint64_t xchg_batch(const wd_table* t) {
  uint64_t b = 1;
  while (b < t->batch) b <<= 1;
  return b;
}

// (re)build the exchange arenas for batch size B (collective in rank mode)
wd_status_t ensure_exchange(wd_table* t) {
  if (t->m == 1) return WD_OK;
  if (t->xbatch == xchg_batch(t)) return WD_OK;
  if (t->mode == MODE_RANK && t->connected)
    return fail(WD_ERR_INVALID_ARG, "rank mode: batch size fixed after wd_rank_connect");
  const uint64_t B = xchg_batch(t);
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    CK(cudaStreamSynchronize(s.s_main));
    CK(cudaStreamSynchronize(s.s_probe));
  }
  for (void* p : t->opened) cudaIpcCloseMemHandle(p);
  t->opened.clear();
  for (auto& s : t->local) free_exchange(s);
  for (auto& s : t->local) TRY(exchange_init_shard(t, s, B));
  t->peers.assign(t->m, PeerView{});
  if (t->mode == MODE_RANK) {
    if (t->connected) return fail(WD_ERR_INVALID_ARG, "rank mode: batch size fixed after wd_rank_connect");
    t->peers[t->rank] = t->local[0].self;   // peers mapped by wd_rank_connect
  } else {
    for (auto& s : t->local) t->peers[s.id] = s.self;
  }
  t->xbatch = B;
  t->epoch = 0;  // fresh flags
  t->res_used[0] = t->res_used[1] = 0;
  return WD_OK;
}

// rank-mode handle blob: IPC handle of the exchange arena + its geometry
struct RankHandle {
  char ipc[64];
  uint64_t magic, batch, arena_bytes;
  uint32_t world, rank;
  uint32_t exchange, has_nccl_id;       // rank 0: an ncclUniqueId follows (WD_OPT_EXCHANGE = 2)
  char nccl_id[128];
  char pad[WD_RANK_HANDLE_BYTES - 64 - 3 * 8 - 4 * 4 - 128];
};
static_assert(sizeof(RankHandle) == WD_RANK_HANDLE_BYTES, "rank handle size");
constexpr uint64_t kHandleMagic = 0x5744524B48444C32ull;  // "WDRKHDL2"

wd_status_t host_allreduce(wd_table* t, uint64_t* v, int op) {
  if (t->mode != MODE_RANK) return WD_OK;
  if (!t->allreduce) return fail(WD_ERR_INVALID_ARG, "rank mode: not connected (wd_rank_connect)");
  if (t->allreduce(v, op, t->allreduce_ctx) != 0)
    return fail(WD_ERR_EXCHANGE, "rank mode: host allreduce callback failed");
  return WD_OK;
}

// ------------------------------------------------------------------ join helpers
// make the shard's internal streams wait for `stream` (per != nullptr: shard r waits for
// per[r], the _sharded calls)
wd_status_t fork_from(wd_table* t, cudaStream_t stream, cudaEvent_t* ev_tmp,
                      const cudaStream_t* per = nullptr) {
  *ev_tmp = nullptr;
  if (!per) {
    CK(cudaEventCreateWithFlags(ev_tmp, cudaEventDisableTiming));
    CK(cudaEventRecord(*ev_tmp, stream));
  }
  for (size_t r = 0; r < t->local.size(); ++r) {
    Shard& s = t->local[r];
    DeviceGuard g(s.device);
    cudaEvent_t ev = *ev_tmp;
    if (per) {
      CK(cudaEventRecord(s.ev_fork, per[r]));
      ev = s.ev_fork;
    }
    CK(cudaStreamWaitEvent(s.s_main, ev, 0));
    if (s.s_probe != s.s_main) CK(cudaStreamWaitEvent(s.s_probe, ev, 0));
    CK(cudaStreamWaitEvent(s.s_h2d, ev, 0));
    CK(cudaStreamWaitEvent(s.s_d2h, ev, 0));
  }
  return WD_OK;
}
// make `stream` (or per[r] for shard r) wait for all internal streams
wd_status_t join_into(wd_table* t, cudaStream_t stream, cudaEvent_t ev_tmp,
                      const cudaStream_t* per = nullptr) {
  for (size_t r = 0; r < t->local.size(); ++r) {
    Shard& s = t->local[r];
    DeviceGuard g(s.device);
    const cudaStream_t out = per ? per[r] : stream;
    CK(cudaEventRecord(s.ev_join_main, s.s_main));
    if (s.s_probe != s.s_main) {
      CK(cudaEventRecord(s.ev_join_probe, s.s_probe));
      CK(cudaStreamWaitEvent(out, s.ev_join_probe, 0));
    }
    CK(cudaEventRecord(s.ev_join_h2d, s.s_h2d));
    CK(cudaEventRecord(s.ev_join_d2h, s.s_d2h));
    CK(cudaStreamWaitEvent(out, s.ev_join_main, 0));
    CK(cudaStreamWaitEvent(out, s.ev_join_h2d, 0));
    CK(cudaStreamWaitEvent(out, s.ev_join_d2h, 0));
  }
  if (ev_tmp) cudaEventDestroy(ev_tmp);
  return WD_OK;
}

// ------------------------------------------------------------------ per-shard IO chunk
struct IO {
  const uint32_t* keys = nullptr;
  const uint32_t* vals = nullptr;
  uint32_t* vout = nullptr;
  uint8_t* fout = nullptr;
  uint64_t n = 0;
  PtrKind kin = PK_DEVICE, kout = PK_DEVICE;
};

// stage batch b's input of `io` into device memory; returns device pointers
wd_status_t stage_in(wd_table* t, Shard& s, const IO& io, uint64_t off, uint64_t cnt, int slot,
                     bool with_vals, const uint32_t** dk, const uint32_t** dv) {
  DeviceGuard g(s.device);
  // the slot's staging buffers (input and output) may still be used by an earlier batch —
  // of this call or of an earlier call on any stream: both the copy-in and the kernel that
  // writes the slot's outputs wait for its release
  if (s.h2d_pending[slot]) {
    CK(cudaStreamWaitEvent(s.s_h2d, s.ev_free[slot], 0));
    CK(cudaStreamWaitEvent(s.s_main, s.ev_free[slot], 0));
    s.h2d_pending[slot] = false;
  }
  if (io.kin == PK_DEVICE) {
    *dk = io.keys + off;
    *dv = with_vals ? io.vals + off : nullptr;
    return WD_OK;
  }
  const uint32_t* hk = io.keys + off;
  const uint32_t* hv = with_vals ? io.vals + off : nullptr;
  if (io.kin == PK_PAGEABLE && cnt) {
    // the pinned bounce buffer of this slot must not be read by an in-flight copy
    CK(cudaEventSynchronize(s.ev_h2d[slot]));
    memcpy(s.pin_keys[slot], hk, cnt * 4);
    if (hv) memcpy(s.pin_vals[slot], hv, cnt * 4);
    hk = s.pin_keys[slot];
    hv = hv ? s.pin_vals[slot] : nullptr;
  }
  if (cnt) {
    const Ph ph = ph_begin(t, wd::PH_H2D, s.device, s.s_h2d);
    CK(cudaMemcpyAsync(s.st_keys[slot], hk, cnt * 4, cudaMemcpyHostToDevice, s.s_h2d));
    if (hv) CK(cudaMemcpyAsync(s.st_vals[slot], hv, cnt * 4, cudaMemcpyHostToDevice, s.s_h2d));
    ph_end(t, ph);
  }
  CK(cudaEventRecord(s.ev_h2d[slot], s.s_h2d));
  CK(cudaStreamWaitEvent(s.s_main, s.ev_h2d[slot], 0));
  *dk = s.st_keys[slot];
  *dv = with_vals ? s.st_vals[slot] : nullptr;
  return WD_OK;
}

// device output pointers for batch b
void out_ptrs(Shard& s, const IO& io, uint64_t off, int slot, uint32_t** dv, uint8_t** df) {
  if (io.kout == PK_DEVICE) {
    *dv = io.vout ? io.vout + off : nullptr;
    *df = io.fout ? io.fout + off : nullptr;
  } else {
    *dv = io.vout ? s.st_vout[slot] : nullptr;
    *df = io.fout ? s.st_fout[slot] : nullptr;
  }
}

// after the kernel that consumed slot `slot` (recorded on s_main): release staging;
// for host outputs copy results back (pageable: through the pinned bounce, synchronously)
wd_status_t stage_out(wd_table* t, Shard& s, const IO& io, uint64_t off, uint64_t cnt, int slot, bool query) {
  DeviceGuard g(s.device);
  CK(cudaEventRecord(s.ev_kdone[slot], s.s_main));
  if (!query || io.kout == PK_DEVICE) {
    if (io.kin != PK_DEVICE) {
      CK(cudaEventRecord(s.ev_free[slot], s.s_main));
      s.h2d_pending[slot] = true;
    }
    return WD_OK;
  }
  CK(cudaStreamWaitEvent(s.s_d2h, s.ev_kdone[slot], 0));
  const Ph ph = ph_begin(t, wd::PH_D2H, s.device, s.s_d2h);
  if (io.kout == PK_PINNED) {
    if (io.vout && cnt) CK(cudaMemcpyAsync(io.vout + off, s.st_vout[slot], cnt * 4, cudaMemcpyDeviceToHost, s.s_d2h));
    if (io.fout && cnt) CK(cudaMemcpyAsync(io.fout + off, s.st_fout[slot], cnt, cudaMemcpyDeviceToHost, s.s_d2h));
    ph_end(t, ph);
    CK(cudaEventRecord(s.ev_free[slot], s.s_d2h));
    s.h2d_pending[slot] = true;
  } else {
    if (io.vout && cnt) CK(cudaMemcpyAsync(s.pin_vout[slot], s.st_vout[slot], cnt * 4, cudaMemcpyDeviceToHost, s.s_d2h));
    if (io.fout && cnt) CK(cudaMemcpyAsync(s.pin_fout[slot], s.st_fout[slot], cnt, cudaMemcpyDeviceToHost, s.s_d2h));
    ph_end(t, ph);
    CK(cudaEventRecord(s.ev_free[slot], s.s_d2h));
    s.h2d_pending[slot] = true;
    CK(cudaEventSynchronize(s.ev_free[slot]));
    if (io.vout) memcpy(io.vout + off, s.pin_vout[slot], cnt * 4);
    if (io.fout) memcpy(io.fout + off, s.pin_fout[slot], cnt);
  }
  return WD_OK;
}

bool needs_staging(const IO& io) { return io.kin != PK_DEVICE || io.kout != PK_DEVICE; }

// ------------------------------------------------------------------ single-shard path
enum Op { OP_INSERT = 0, OP_RETRIEVE = 1, OP_ERASE = 2 };

// the probe kernel of one call on a plain (SoA) input
// (the probe kernels index one launch's input with 32 bits: device calls of >= 2^32 pairs
// are launched in pieces of 2^31)
wd_status_t probe_soa(wd_table* t, Shard& s, int op, const wd::InSoA& in, uint32_t* ov, uint8_t* of,
                      uint64_t n, cudaStream_t st) {
  constexpr uint64_t kPiece = 1ull << 31;
  if (n >= (1ull << 32)) {
    for (uint64_t off = 0; off < n; off += kPiece) {
      const uint64_t c = std::min(kPiece, n - off);
      const wd::InSoA p{in.keys + off, in.vals ? in.vals + off : nullptr, c};
      TRY(probe_soa(t, s, op, p, ov ? ov + off : nullptr, of ? of + off : nullptr, c, st));
    }
    return WD_OK;
  }
  if (op == OP_INSERT) return launch_probe<true>(t, s, in, wd::OutNone{}, n, st);
  if (op == OP_ERASE) return launch_probe<false>(t, s, in, wd::OutErase<wd::OutSoA>{{nullptr, of}}, n, st);
  return launch_probe<false>(t, s, in, wd::OutSoA{ov, of}, n, st);
}

// Table slices for a bulk insert of n device-resident pairs (WD_OPT_SLICES): 16 when the
// table is HBM-sized (> 512 MB) and the call has >= 2^22 pairs, else 1 (plain launch).
// Auto only where it was measured to pay (profiles/r01_slices.txt: 2^28 pairs into 2.3 GB;
// 16 slices over 2^24-pair chunks were SLOWER than one launch): calls of >= 2^26 pairs, so
// each slice launch gets >= 2^22 keys, and not where the plain launch uses the span
// read-ahead (|g| = 1), whose gain the sliced launches (InBucket) do not have.  The slice
// count follows the table: slices of ~128-280 MB pay, slices of ~540 MB are SLOWER than no
// slicing (profiles/r02/capacity_knee.md, 2^29 pairs at alpha 0.5 into 8.6 GB: 16 slices
// 9.9, none 17.1, 32 slices 22.1 G inserts/s); slices of <= 80 MB where possible (2^28 pairs
// into 2.3 GB: 8 / 16 / 32 slices -> 16.7 / 19.65 / 19.86 G/s — the probes gain more than
// the 32-way multisplit loses); at most 32 slices, so tables above ~9.6 GB are not sliced.
int choose_slices(const wd_table* t, const Shard& s, int op, uint64_t n) {
  if (op != OP_INSERT || t->serial || t->slices == 1) return 1;
  if (t->slices > 1) return t->slices;
  const double tb = double(s.cap) * sizeof(unsigned long long);
  if (tb <= double(512ull << 20) || n < (1ull << 26)) return 1;
  // the plain launch's span read-ahead (|g| = 1) wins up to ~1 GB, slicing beyond it
  // (|g| = 1, alpha 0.95: 2^26 pairs 7.5 vs 7.45, 2^27 5.7 vs 7.5, 2^28 5.2 vs 7.5 G/s)
  const int v = choose_v(t, s, t->G_used, true);
  if (choose_span(t, s, t->G_used, v) == 2 && tb <= 1.0e9) return 1;
  // <= 80 MB slices where the launches read one line per lane (|g| = 16 on a line-aligned
  // table: 16 -> 32 slices 19.65 -> 19.86 G/s at alpha 0.95, 12.5 -> 13.3 at 0.99); <= 160 MB
  // otherwise (|g| = 4: 16 slices 15.5, 32 slices 13.4 G/s)
  const double target = (t->G_used == 16 && t->align == 16) ? 80e6 : 160e6;
  int nbk = 2;
  while (nbk < wd::kMaxSlices && tb / nbk > target) nbk *= 2;
  if (tb / nbk > 300e6) return 1;
  return nbk;
}

// Slice-grouped bulk insert.  Each chunk of <= 2^28 pairs is grouped by the table slice of
// its keys' first region (Line 5: h(k) is monotone in fmix32(k + seed), so slice j of nbk
// holds the region starts [j nb / nbk, (j + 1) nb / nbk)): a histogram, a scan and the
// multisplit kernel write the pairs slice by slice into a scratch buffer; then one probe
// launch per slice inserts them.  Each launch works on 1/nbk of the table, which the L2
// holds a good part of: dirty lines take several inserts before they are written back and
// fewer window loads go to DRAM.  Measured on B200 (tools/slice_probe.py,
// profiles/r01_slices.txt): 2^28 pairs, |g| = 16, alpha 0.95: 15.0 -> 20.9 G inserts/s
// for the probe launches.  Results are those of one launch: the probing of every key is
// Fig. 3's; only the order in which the keys of one call are inserted changes (C20: any of
// a call's duplicate values may win).
// Round 2: the grouping of chunk c + 1 runs on a side stream while chunk c is probed (two
// scratch buffers, event-ordered), so only the first chunk's grouping is exposed; chunks of
// 2^28 (tools/gpu_chunk_sweep.sh, 2^28 pairs: 2^25 / 2^26 / 2^27 / 2^28 -> 17.2 / 18.8 /
// 19.6 / 19.7 G inserts/s; 2^29 pairs into 8.6 GB: 2^27 / 2^28 / 2^29 -> 21.2 / 22.1 / 22.6:
// fewer, longer probe launches; WD_SLICE_CHUNK_LOG2 overrides).
wd_status_t slice_insert(wd_table* t, Shard& s, const IO& io, int nbk, cudaStream_t st) {
  static const int chunk_log2 = getenv("WD_SLICE_CHUNK_LOG2") ? atoi(getenv("WD_SLICE_CHUNK_LOG2")) : 28;
  const uint64_t kChunkPairs = 1ull << chunk_log2;
  const uint64_t cap = std::min<uint64_t>(io.n, kChunkPairs);
  const int nbuf = io.n > kChunkPairs ? 2 : 1;
  if (!s.sl_done) {
    CK(cudaEventCreateWithFlags(&s.sl_done, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&s.sl_fork, cudaEventDisableTiming));
    for (int b = 0; b < 2; ++b) {
      CK(cudaEventCreateWithFlags(&s.sl_grouped[b], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&s.sl_probed[b], cudaEventDisableTiming));
    }
    CK(cudaStreamCreateWithFlags(&s.s_group, cudaStreamNonBlocking));
  }
  if (s.sl_used) CK(cudaStreamWaitEvent(st, s.sl_done, 0));   // scratch of an earlier call
  for (int b = 0; b < nbuf; ++b) {
    if (s.sl_cap[b] >= cap) continue;
    // stream-ordered (no device synchronisation): the old scratch is released after its
    // last use (st waits on sl_done above), the new one is allocated in st's order.  The
    // scratch (8 B per pair, <= 2 x 2 GB) is kept for the table's lifetime.
    if (s.sl_buf[b]) CK(cudaFreeAsync(s.sl_buf[b], st));
    s.sl_buf[b] = nullptr;
    s.sl_cap[b] = 0;
    const cudaError_t e = cudaMallocAsync(&s.sl_buf[b], cap * sizeof(unsigned long long), st);
    if (e != cudaSuccess) {
      cudaGetLastError();
      s.sl_buf[b] = nullptr;
      if (t->slices == 0) {        // auto: the optimisation steps back, the call still runs
        const wd::InSoA in{io.keys, io.vals, io.n};
        return probe_soa(t, s, OP_INSERT, in, nullptr, nullptr, io.n, st);
      }
      return fail(e == cudaErrorMemoryAllocation ? WD_ERR_OUT_OF_MEMORY : WD_ERR_CUDA,
                  "slice scratch of %llu pairs: %s", (unsigned long long)cap, cudaGetErrorString(e));
    }
    s.sl_cap[b] = cap;
  }
  // the multisplit instance with the fewest destination slots that fits nbk, in segment
  // mode: grid = one block per SM slot, block b groups the contiguous segment
  // [b L, (b + 1) L) of the chunk (L a multiple of the tile)
  auto ms_kern = nbk <= 32 ? wd::multisplit_kernel<true, 1, true, true>
                           : nbk <= 64 ? wd::multisplit_kernel<true, 2, true, true>
                                       : wd::multisplit_kernel<true, wd::kMaxSlices / 32, true, true>;
  const int S = t->sm_count * blocks_per_sm(ms_kern);
  const int S_max = t->sm_count * std::max({blocks_per_sm(wd::multisplit_kernel<true, 1, true, true>),
                                            blocks_per_sm(wd::multisplit_kernel<true, 2, true, true>),
                                            blocks_per_sm(wd::multisplit_kernel<true, wd::kMaxSlices / 32, true, true>)});
  // per buffer: bounds (kMaxSlices + 1) | cursor (kMaxSlices) | seg_off (S_max x kMaxSlices)
  // | seg counts (S_max x kMaxSlices u32, in u64 words)
  const uint64_t kMeta = 2 * wd::kMaxSlices + 1 + uint64_t(S_max) * wd::kMaxSlices * 3 / 2 + 1;
  if (!s.sl_meta) CK(cudaMalloc(&s.sl_meta, 2 * kMeta * sizeof(unsigned long long)));
  // the grouping stream starts after everything st has so far (inputs, scratch allocation)
  CK(cudaEventRecord(s.sl_fork, st));
  CK(cudaStreamWaitEvent(s.s_group, s.sl_fork, 0));
  const uint64_t nchunks = (io.n + kChunkPairs - 1) / kChunkPairs;
  auto group = [&](uint64_t c) -> wd_status_t {   // on s_group, into buffer c % 2
    const int b = int(c % 2);
    const uint64_t off = c * kChunkPairs, cnt = std::min(kChunkPairs, io.n - off);
    unsigned long long* bounds = s.sl_meta + b * kMeta;
    unsigned long long* cursor = bounds + wd::kMaxSlices + 1;
    unsigned long long* seg_off = cursor + wd::kMaxSlices;
    unsigned int* seg_cnt = reinterpret_cast<unsigned int*>(seg_off + uint64_t(S_max) * wd::kMaxSlices);
    if (c >= 2) CK(cudaStreamWaitEvent(s.s_group, s.sl_probed[b], 0));   // probes of c - 2 done
    const Ph pg = ph_begin(t, wd::PH_GROUP, s.device, s.s_group);
    const uint64_t L = ((cnt + S - 1) / S + wd::kMs2Tile - 1) / wd::kMs2Tile * wd::kMs2Tile;
    wd::seg_hist_kernel<<<S, wd::kBlock, 0, s.s_group>>>(io.keys + off, cnt, L, nbk, s.hseed, seg_cnt);
    wd::seg_scan_kernel<<<1, 1024, 0, s.s_group>>>(seg_cnt, S, nbk, bounds, cursor, seg_off);
    wd::DstPtrs dst{};                               // one buffer, slice j at bounds[j]
    dst.p[0] = s.sl_buf[b];
    ms_kern<<<S, wd::kBlock, 0, s.s_group>>>(io.keys + off, io.vals + off, cnt, dst, nullptr, seg_off, L,
                                             nullptr, nbk, s.hseed, cnt, s.counters);
    CK(cudaGetLastError());
    t->launches += 3;
    ph_end(t, pg);
    CK(cudaEventRecord(s.sl_grouped[b], s.s_group));
    return WD_OK;
  };
  auto probe = [&](uint64_t c) -> wd_status_t {   // on st
    const int b = int(c % 2);
    const uint64_t off = c * kChunkPairs, cnt = std::min(kChunkPairs, io.n - off);
    const unsigned long long* bounds = s.sl_meta + b * kMeta;
    CK(cudaStreamWaitEvent(st, s.sl_grouped[b], 0));
    const Ph pp = ph_begin(t, wd::PH_PROBE, s.device, st);
    // (programmatic dependent launch of slice j + 1 into slice j's tail was measured slower:
    // 10.4 -> 11.1 ms for the 32 launches, two slices' working sets share the L2 —
    // profiles/r02/pdl_negative.md)
    for (int j = 0; j < nbk; ++j)
      TRY(launch_probe<true>(t, s, wd::InBucket{s.sl_buf[b], bounds, j, j + 1}, wd::OutNone{},
                             cnt / nbk + 1, st));
    ph_end(t, pp);
    CK(cudaEventRecord(s.sl_probed[b], st));
    return WD_OK;
  };
  TRY(group(0));
  for (uint64_t c = 0; c < nchunks; ++c) {
    if (c + 1 < nchunks) TRY(group(c + 1));
    TRY(probe(c));
  }
  CK(cudaEventRecord(s.sl_done, st));
  s.sl_used = true;
  return WD_OK;
}

wd_status_t single_op(wd_table* t, int op, const IO& io, cudaStream_t stream) {
  const bool insert = op == OP_INSERT;
  Shard& s = t->local[0];
  DeviceGuard g(s.device);
  if (!needs_staging(io)) {  // device-resident: one kernel on the caller's stream
    if (io.n == 0) return WD_OK;
    const int nbk = choose_slices(t, s, op, io.n);
    if (nbk > 1) return slice_insert(t, s, io, nbk, stream);
    const wd::InSoA in{io.keys, io.vals, io.n};
    const Ph pp = ph_begin(t, op == OP_INSERT ? wd::PH_PROBE : wd::PH_PROBE_QUERY, s.device, stream);
    TRY(probe_soa(t, s, op, in, io.vout, io.fout, io.n, stream));
    ph_end(t, pp);
    return WD_OK;
  }
  // out-of-core pipeline (Fig. 5): H2D(b+1) || probe(b) || D2H(b-1).  Default
  // batch here 2^22 (not P:197's 2^24): shorter pipeline fill and drain; the bench's e2e
  // step (2^28 pairs, pinned) took 67.7 / 68.0 / 69.7 / 72.5 ms at 2^22 / 2^23 / 2^24 /
  // 2^25 (tools/e2e_batch.py, profiles/r01_e2e_batch.txt)
  const uint64_t B = t->batch_set ? t->batch : std::min<uint64_t>(t->batch, 1ull << 22);
  TRY(ensure_staging(s, B, io.kin == PK_PAGEABLE || io.kout == PK_PAGEABLE));
  cudaEvent_t ev0;
  TRY(fork_from(t, stream, &ev0));
  const uint64_t nbt = (io.n + B - 1) / B;
  for (uint64_t b = 0; b < nbt; ++b) {
    const int slot = int(b % kStage);
    const uint64_t off = b * B, cnt = std::min(B, io.n - off);
    const uint32_t *dk, *dv;
    TRY(stage_in(t, s, io, off, cnt, slot, insert, &dk, &dv));
    const wd::InSoA in{dk, dv, cnt};
    uint32_t* ov = nullptr; uint8_t* of = nullptr;
    if (!insert) out_ptrs(s, io, off, slot, &ov, &of);
    const Ph pp = ph_begin(t, insert ? wd::PH_PROBE : wd::PH_PROBE_QUERY, s.device, s.s_main);
    TRY(probe_soa(t, s, op, in, ov, of, cnt, s.s_main));
    ph_end(t, pp);
    TRY(stage_out(t, s, io, off, cnt, slot, !insert));
  }
  return join_into(t, stream, ev0);
}

// ------------------------------------------------------------------ multi-shard cascade
wd::FlagPtrs flag_ptrs(wd_table* t, int flag, int who) {
  wd::FlagPtrs f{};
  for (int d = 0; d < t->m; ++d) f.p[d] = t->peers[d].flags + flag * t->m + who;
  return f;
}

wd_status_t launch_wait(wd_table* t, Shard& s, cudaStream_t st, int flag, unsigned long long target) {
  wd::wait_kernel<<<1, 32, 0, st>>>(s.self.flags + flag * t->m, t->m, target, kWaitTimeoutNs,
                                    s.counters);
  CK(cudaGetLastError());
  t->launches++;
  return WD_OK;
}
wd_status_t launch_signal(wd_table* t, Shard& s, cudaStream_t st, int flag, unsigned long long epoch) {
  wd::signal_kernel<<<1, 32, 0, st>>>(flag_ptrs(t, flag, s.id), t->m, epoch);
  CK(cudaGetLastError());
  t->launches++;
  return WD_OK;
}

wd_status_t agree_batches(wd_table* t, uint64_t local_nbt, uint64_t* global_nbt) {
  uint64_t v = local_nbt;
  TRY(host_allreduce(t, &v, WD_REDUCE_MAX));   // every rank runs the same batch sequence
  *global_nbt = v;
  return WD_OK;
}

// ------------------------------------------------------------------ staged exchange
void free_staged(Shard& s) {
  DeviceGuard g(s.device);
  if (s.send) cudaFree(s.send);
  if (s.res_stage) cudaFree(s.res_stage);
  s.send = nullptr;
  s.res_stage = nullptr;
  for (int i = 0; i < 2; ++i) {
    if (s.hrow[i]) cudaFreeHost(s.hrow[i]);
    if (s.hcol[i]) cudaFreeHost(s.hcol[i]);
    if (s.hT[i]) cudaFreeHost(s.hT[i]);
    if (s.Tdev[i]) cudaFree(s.Tdev[i]);
    s.hrow[i] = s.hcol[i] = s.hT[i] = s.Tdev[i] = nullptr;
    for (cudaEvent_t* e : {&s.ev_ready[i], &s.ev_pdone[i], &s.ev_done[i], &s.ev_unperm[i]}) {
      if (*e) cudaEventDestroy(*e);
      *e = nullptr;
    }
    s.pdone_rec[i] = s.unperm_rec[i] = false;
  }
  if (s.ev_row) cudaEventDestroy(s.ev_row);
  if (s.ev_col) cudaEventDestroy(s.ev_col);
  s.ev_row = s.ev_col = nullptr;
  s.staged_B = 0;
}

void free_nccl(wd_table* t) {
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    if (s.comm_rev) g_nccl.CommDestroy(s.comm_rev);
    if (s.comm_fwd) g_nccl.CommDestroy(s.comm_fwd);
    s.comm_fwd = s.comm_rev = nullptr;
  }
  t->nccl_ready = false;
}

// the staged transport's buffers for batch size B: send [m][B] items (u64 pairs or u32 keys),
// res_stage [m][B] packed results, pinned rows / columns of T per exchange slot
wd_status_t ensure_staged(wd_table* t, Shard& s, uint64_t B) {
  if (s.staged_B == B) return WD_OK;
  free_staged(s);
  DeviceGuard g(s.device);
  const int m = t->m;
  CK(cudaMalloc(&s.send, size_t(m) * B * 8));
  CK(cudaMalloc(&s.res_stage, size_t(m) * B * 8));
  for (int i = 0; i < 2; ++i) {
    CK(cudaMallocHost(&s.hrow[i], m * 8));
    CK(cudaMallocHost(&s.hcol[i], m * 8));
    CK(cudaMallocHost(&s.hT[i], size_t(m) * m * 8));
    CK(cudaMalloc(&s.Tdev[i], size_t(m) * m * 8));
    for (cudaEvent_t* e : {&s.ev_ready[i], &s.ev_pdone[i], &s.ev_done[i], &s.ev_unperm[i]})
      CK(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
  }
  CK(cudaEventCreateWithFlags(&s.ev_row, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_col, cudaEventDisableTiming));
  s.staged_B = B;
  return WD_OK;
}

// NCCL communicators of the forward and the reverse transposition (collective: every rank
// calls it at its first NCCL-exchange operation, in the same order)
wd_status_t ensure_nccl(wd_table* t) {
  if (t->nccl_ready) return WD_OK;
  const NcclApi* a = nccl_api();
  if (!a) return fail(WD_ERR_NCCL, "%s", g_nccl.why);
  if (t->mode == MODE_MULTI) {
    std::vector<void*> c(t->m, nullptr);
    std::vector<int> devs(t->m);
    for (int r = 0; r < t->m; ++r) devs[r] = t->local[r].device;
    NK(a->CommInitAll(c.data(), t->m, devs.data()));
    for (int r = 0; r < t->m; ++r) t->local[r].comm_fwd = c[r];
    NK(a->CommInitAll(c.data(), t->m, devs.data()));
    for (int r = 0; r < t->m; ++r) t->local[r].comm_rev = c[r];
  } else if (t->mode == MODE_RANK) {
    if (!t->have_nccl_id)
      return fail(WD_ERR_NCCL, "rank mode: set WD_OPT_EXCHANGE = 2 before wd_rank_handle / "
                               "wd_rank_connect (rank 0's NCCL id travels in the handles)");
    Shard& s = t->local[0];
    DeviceGuard g(s.device);
    NcclUid id;
    memcpy(&id, t->nccl_id, sizeof id);
    NK(a->CommInitRank(&s.comm_fwd, t->m, id, t->rank));
    NK(a->CommSplit(s.comm_fwd, 0, t->rank, &s.comm_rev, nullptr));
  } else {
    return fail(WD_ERR_UNSUPPORTED, "the NCCL exchange needs one GPU per shard (wd_create with "
                                    "n_gpus > 1, or rank mode); loopback shards share a device");
  }
  t->nccl_ready = true;
  return WD_OK;
}

wd_status_t cascade_op(wd_table* t, int op, std::vector<IO>& ios, cudaStream_t stream,
                       const cudaStream_t* per = nullptr) {
  const bool insert = op == OP_INSERT;
  TRY(ensure_exchange(t));
  const uint64_t B = t->xbatch;   // a power of two (xchg_batch)
  const int m = t->m;
  const int X = t->exchange;      // 0 fused, 1 staged + copy engine, 2 staged + NCCL
  if (X == 2) TRY(ensure_nccl(t));
  uint64_t local_nbt = 0;
  for (size_t r = 0; r < t->local.size(); ++r) {
    local_nbt = std::max(local_nbt, (ios[r].n + B - 1) / B);
    if (needs_staging(ios[r]))
      TRY(ensure_staging(t->local[r], B,
                         ios[r].kin == PK_PAGEABLE || ios[r].kout == PK_PAGEABLE));
    if (X) TRY(ensure_staged(t, t->local[r], B));
  }
  uint64_t nbt = 0;
  TRY(agree_batches(t, local_nbt, &nbt));
  if (nbt == 0) return WD_OK;
  cudaEvent_t ev0;
  TRY(fork_from(t, stream, &ev0, per));
  const size_t isz = insert ? 8 : 4;          // bytes per exchanged item (pair / key)
  const bool all_local = t->mode != MODE_RANK;  // this process holds every row of T

  // Three phases per batch b (epoch e = epoch0 + 1 + b, exchange slot e % 2):
  //   A (s_main):  multisplit; fused (X = 0): straight into the owners' receive regions,
  //                then publish the row of T and the READY flags.  Staged (X = 1, 2): into
  //                the local send buffer, then the transposition proper (phase T below).
  //   B (s_probe): wait for the column of T, probe (insert / retrieve); queries send their
  //                results back (fused: peer stores in the probe kernel; staged: res_stage,
  //                then copy engine / NCCL), DONE flags / events
  //   C (s_main):  queries only — unpermute the results that arrived in this shard's result
  //                slot (local gather), RESC flags / events (the slot may be reused)
  // Issued as A(0), then A(b+1), B(b), C(b): the multisplit and transposition of batch b+1
  // overlap the probing of batch b (Fig. 5's MST || INS), and the query's unpermute of
  // batch b never blocks the next multisplit.  Fused and copy-engine: cross-shard ordering by
  // epoch flags only; NCCL: by the collective's own completion, recorded in events.
  const unsigned long long e0 = t->epoch;
  auto multisplit = [&](Shard& s, const uint32_t* dk, const uint32_t* dv, uint64_t cnt,
                        int slot) -> wd_status_t {
    wd::DstPtrs dst{};
    for (int d = 0; d < m; ++d) {
      if (X) dst.p[d] = static_cast<char*>(s.send) + uint64_t(d) * B * isz;   // local buckets
      else if (insert) dst.p[d] = t->peers[d].recv[slot] + uint64_t(s.id) * B;
      else dst.p[d] = reinterpret_cast<uint32_t*>(t->peers[d].recv[slot]) + uint64_t(s.id) * B;
    }
    // every resident block of the SM (occupancy API): more tiles in flight per SM
    // cursor mode (the owners read their column of T from the cursors), p(k) of C15 or
    // Fig. 4's k mod m (WD_OPT_PART_MODE)
    auto kern = insert ? (t->pmode == 1 ? wd::multisplit_kernel<true, 1, false, false, 1>
                                        : wd::multisplit_kernel<true, 1, false, false, 0>)
                       : (t->pmode == 1 ? wd::multisplit_kernel<false, 1, false, false, 1>
                                        : wd::multisplit_kernel<false, 1, false, false, 0>);
    const uint64_t tiles = (cnt + wd::kMs2TileC - 1) / wd::kMs2TileC;
    const int grid = int(std::min<uint64_t>(tiles, uint64_t(t->sm_count) * blocks_per_sm(kern)));
    kern<<<grid, wd::kBlock, 0, s.s_main>>>(dk, insert ? dv : nullptr, cnt, dst, s.cursor[slot], nullptr, 0,
                                             insert ? nullptr : s.pos[slot], m, t->pseed, B, s.counters);
    CK(cudaGetLastError());
    t->launches++;
    return WD_OK;
  };
  auto publish = [&](Shard& s, int slot, unsigned long long e) -> wd_status_t {
    wd::FlagPtrs cnt_dst{};
    for (int d = 0; d < m; ++d) cnt_dst.p[d] = t->peers[d].recv_count[slot] + s.id;
    wd::publish_kernel<<<1, 32, 0, s.s_main>>>(s.cursor[slot], cnt_dst,
                                               flag_ptrs(t, FLAG_READY, s.id), m, e);
    CK(cudaGetLastError());
    t->launches++;
    return WD_OK;
  };
  auto phaseA = [&](uint64_t b) -> wd_status_t {
    Nvtx nv("wd:A multisplit");
    const unsigned long long e = e0 + 1 + b;
    const int slot = int(e & 1);
    for (size_t r = 0; r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      const IO& io = ios[r];
      DeviceGuard g(s.device);
      const uint64_t off = std::min(io.n, b * B), cnt = std::min(B, io.n - off);
      const uint32_t *dk = nullptr, *dv = nullptr;
      TRY(stage_in(t, s, io, off, cnt, int(b % kStage), insert, &dk, &dv));
      if (X == 0 && e > 2) TRY(launch_wait(t, s, s.s_main, FLAG_DONE, e - 2));  // owners released e-2
      if (cnt) {
        const Ph pm = ph_begin(t, wd::PH_MULTISPLIT, s.device, s.s_main);
        TRY(multisplit(s, dk, dv, cnt, slot));
        ph_end(t, pm);
      }
      if (insert) TRY(stage_out(t, s, io, off, cnt, int(b % kStage), false));  // input slot free
      if (X == 0) {
        TRY(publish(s, slot, e));
      } else {                          // this shard's row of T to the host
        CK(cudaMemcpyAsync(s.hrow[slot], s.cursor[slot], m * 8, cudaMemcpyDeviceToHost, s.s_main));
        CK(cudaEventRecord(s.ev_row, s.s_main));
      }
    }
    return WD_OK;
  };
  // T (staged only): the transposition of P:117 with exact counts — the copy engine pushes
  // each bucket into its owner's receive region and publishes the counts with the READY
  // flags; NCCL all-gathers T (rank mode), then one grouped send/recv per peer (an
  // all-to-all(v)).  The host waits for this batch's row(s) of T first.
  auto phaseT = [&](uint64_t b) -> wd_status_t {
    Nvtx nv("wd:T transposition");
    const unsigned long long e = e0 + 1 + b;
    const int slot = int(e & 1);
    for (auto& s : t->local) {
      DeviceGuard g(s.device);
      CK(cudaEventSynchronize(s.ev_row));
    }
    if (X == 1) {
      for (auto& s : t->local) {
        DeviceGuard g(s.device);
        if (e > 2) TRY(launch_wait(t, s, s.s_main, FLAG_DONE, e - 2));   // owners released e-2
        const Ph px = ph_begin(t, wd::PH_EXCHANGE, s.device, s.s_main);
        for (int d = 0; d < m; ++d) {
          const uint64_t c = std::min<uint64_t>(s.hrow[slot][d], B);
          if (c)
            CK(cudaMemcpyAsync(reinterpret_cast<char*>(t->peers[d].recv[slot]) + uint64_t(s.id) * B * isz,
                               static_cast<char*>(s.send) + uint64_t(d) * B * isz, c * isz,
                               cudaMemcpyDefault, s.s_main));
        }
        ph_end(t, px);
        TRY(publish(s, slot, e));       // counts + READY after the copies (stream order)
      }
      return WD_OK;
    }
    // X == 2: the whole T on the host
    unsigned long long* T = t->local[0].hT[slot];
    if (all_local) {
      for (auto& s : t->local)
        for (int d = 0; d < m; ++d) T[size_t(s.id) * m + d] = s.hrow[slot][d];
    } else {
      Shard& s = t->local[0];
      DeviceGuard g(s.device);
      NK(g_nccl.AllGather(s.cursor[slot], s.Tdev[slot], m, kNcclUint64, s.comm_fwd, s.s_main));
      CK(cudaMemcpyAsync(T, s.Tdev[slot], size_t(m) * m * 8, cudaMemcpyDeviceToHost, s.s_main));
      CK(cudaStreamSynchronize(s.s_main));
    }
    for (auto& s : t->local) {          // the receive region must be free: own probe of e-2
      DeviceGuard g(s.device);
      if (s.pdone_rec[slot]) CK(cudaStreamWaitEvent(s.s_main, s.ev_pdone[slot], 0));
    }
    std::vector<Ph> px;
    for (auto& s : t->local) {
      DeviceGuard g(s.device);
      px.push_back(ph_begin(t, wd::PH_EXCHANGE, s.device, s.s_main));
    }
    NK(g_nccl.GroupStart());
    for (auto& s : t->local) {
      DeviceGuard g(s.device);
      for (int d = 0; d < m; ++d) {
        const uint64_t cs = std::min<uint64_t>(T[size_t(s.id) * m + d], B);   // s -> d
        const uint64_t cr = std::min<uint64_t>(T[size_t(d) * m + s.id], B);   // d -> s
        if (cs) NK(g_nccl.Send(static_cast<char*>(s.send) + uint64_t(d) * B * isz, cs * isz,
                               kNcclUint8, d, s.comm_fwd, s.s_main));
        if (cr) NK(g_nccl.Recv(reinterpret_cast<char*>(s.self.recv[slot]) + uint64_t(d) * B * isz,
                               cr * isz, kNcclUint8, d, s.comm_fwd, s.s_main));
      }
    }
    NK(g_nccl.GroupEnd());
    for (size_t r = 0; r < t->local.size(); ++r) {
      DeviceGuard g(t->local[r].device);
      ph_end(t, px[r]);
    }
    for (auto& s : t->local) {          // my column of T -> recv_count (InSeg), cursor reset
      DeviceGuard g(s.device);
      for (int d = 0; d < m; ++d) s.hcol[slot][d] = T[size_t(d) * m + s.id];
      CK(cudaMemcpyAsync(s.self.recv_count[slot], s.hcol[slot], m * 8, cudaMemcpyHostToDevice, s.s_main));
      CK(cudaMemsetAsync(s.cursor[slot], 0, m * 8, s.s_main));
      CK(cudaEventRecord(s.ev_ready[slot], s.s_main));
    }
    return WD_OK;
  };
  auto phaseB = [&](uint64_t b) -> wd_status_t {
    Nvtx nv("wd:B probe");
    const unsigned long long e = e0 + 1 + b;
    const int slot = int(e & 1);
    for (auto& s : t->local) {
      DeviceGuard g(s.device);
      if (X == 2) CK(cudaStreamWaitEvent(s.s_probe, s.ev_ready[slot], 0));
      else TRY(launch_wait(t, s, s.s_probe, FLAG_READY, e));
      if (X == 0 && !insert && t->res_used[slot])   // origins consumed this result slot
        TRY(launch_wait(t, s, s.s_probe, FLAG_RESC, t->res_used[slot]));
      const Ph pp = ph_begin(t, insert ? wd::PH_PROBE : wd::PH_PROBE_QUERY, s.device, s.s_probe);
      if (insert) {
        const wd::InSeg<true> in{s.self.recv[slot], s.self.recv_count[slot], B, m};
        TRY(launch_probe<true>(t, s, in, wd::OutNone{}, B, s.s_probe));
      } else {
        const wd::InSeg<false> in{s.self.recv[slot], s.self.recv_count[slot], B, m};
        if (X == 0) {
          // reverse transposition: results go straight to their origins' result
          // slots (region s.id of origin d's slot), coalesced remote stores
          wd::OutPacked out{};
          out.stride = B;
          out.shift = __builtin_ctzll(B);
          for (int d = 0; d < m; ++d) out.seg[d] = t->peers[d].res[slot] + uint64_t(s.id) * B;
          if (op == OP_ERASE)
            TRY(launch_probe<false>(t, s, in, wd::OutErase<wd::OutPacked>{out}, B, s.s_probe));
          else
            TRY(launch_probe<false>(t, s, in, out, B, s.s_probe));
        } else {
          // staged: results at their receive location in res_stage, then transferred back
          const wd::OutLocalPacked out{s.res_stage};
          if (op == OP_ERASE)
            TRY(launch_probe<false>(t, s, in, wd::OutErase<wd::OutLocalPacked>{out}, B, s.s_probe));
          else
            TRY(launch_probe<false>(t, s, in, out, B, s.s_probe));
        }
      }
      ph_end(t, pp);
      if (X == 2) {
        CK(cudaEventRecord(s.ev_pdone[slot], s.s_probe));   // recv[slot] may be refilled
        s.pdone_rec[slot] = true;
      }
    }
    if (!insert && X == 1) {            // reverse transposition with the copy engine
      for (auto& s : t->local) {
        DeviceGuard g(s.device);
        const unsigned long long* col = s.hcol[slot];
        if (all_local) {
          for (int d = 0; d < m; ++d) s.hcol[slot][d] = t->local[d].hrow[slot][s.id];
        } else {                       // my column of T: the counts the senders published
          CK(cudaMemcpyAsync(s.hcol[slot], s.self.recv_count[slot], m * 8, cudaMemcpyDeviceToHost, s.s_probe));
          CK(cudaEventRecord(s.ev_col, s.s_probe));
          CK(cudaEventSynchronize(s.ev_col));
        }
        if (t->res_used[slot]) TRY(launch_wait(t, s, s.s_probe, FLAG_RESC, t->res_used[slot]));
        const Ph pr = ph_begin(t, wd::PH_REVERSE, s.device, s.s_probe);
        for (int d = 0; d < m; ++d) {
          const uint64_t c = std::min<uint64_t>(col[d], B);
          if (c)
            CK(cudaMemcpyAsync(t->peers[d].res[slot] + uint64_t(s.id) * B,
                               s.res_stage + uint64_t(d) * B, c * 8, cudaMemcpyDefault, s.s_probe));
        }
        ph_end(t, pr);
      }
    }
    if (!insert && X == 2) {            // reverse transposition with NCCL
      const unsigned long long* T = t->local[0].hT[slot];
      for (auto& s : t->local) {        // own result slot free: own unpermute of e-2
        DeviceGuard g(s.device);
        if (s.unperm_rec[slot]) CK(cudaStreamWaitEvent(s.s_probe, s.ev_unperm[slot], 0));
      }
      std::vector<Ph> pr;
      for (auto& s : t->local) {
        DeviceGuard g(s.device);
        pr.push_back(ph_begin(t, wd::PH_REVERSE, s.device, s.s_probe));
      }
      NK(g_nccl.GroupStart());
      for (auto& s : t->local) {
        DeviceGuard g(s.device);
        for (int d = 0; d < m; ++d) {
          const uint64_t cs = std::min<uint64_t>(T[size_t(d) * m + s.id], B);  // answers to d
          const uint64_t cr = std::min<uint64_t>(T[size_t(s.id) * m + d], B);  // from d
          if (cs) NK(g_nccl.Send(s.res_stage + uint64_t(d) * B, cs * 8, kNcclUint8, d, s.comm_rev, s.s_probe));
          if (cr) NK(g_nccl.Recv(s.self.res[slot] + uint64_t(d) * B, cr * 8, kNcclUint8, d, s.comm_rev, s.s_probe));
        }
      }
      NK(g_nccl.GroupEnd());
      for (size_t r = 0; r < t->local.size(); ++r) {
        DeviceGuard g(t->local[r].device);
        ph_end(t, pr[r]);
      }
    }
    for (auto& s : t->local) {
      DeviceGuard g(s.device);
      if (X == 2) CK(cudaEventRecord(s.ev_done[slot], s.s_probe));
      else TRY(launch_signal(t, s, s.s_probe, FLAG_DONE, e));
    }
    if (!insert) t->res_used[slot] = e;
    return WD_OK;
  };
  auto phaseC = [&](uint64_t b) -> wd_status_t {
    Nvtx nv("wd:C unpermute");
    const unsigned long long e = e0 + 1 + b;
    const int slot = int(e & 1);
    for (size_t r = 0; r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      const IO& io = ios[r];
      DeviceGuard g(s.device);
      const uint64_t off = std::min(io.n, b * B), cnt = std::min(B, io.n - off);
      if (X == 2) CK(cudaStreamWaitEvent(s.s_main, s.ev_done[slot], 0));
      else TRY(launch_wait(t, s, s.s_main, FLAG_DONE, e));
      if (cnt) {
        wd::DstPtrs src{};
        for (int d = 0; d < m; ++d) src.p[d] = s.self.res[slot] + uint64_t(d) * B;   // local
        uint32_t* ov; uint8_t* of;
        out_ptrs(s, io, off, int(b % kStage), &ov, &of);
        const int grid = int(std::min<uint64_t>((cnt + wd::kBlock - 1) / wd::kBlock,
                                                uint64_t(t->sm_count) * 8));
        const Ph pu = ph_begin(t, wd::PH_UNPERMUTE, s.device, s.s_main);
        wd::unpermute_kernel<<<grid, wd::kBlock, 0, s.s_main>>>(s.pos[slot], cnt, src, ov, of);
        CK(cudaGetLastError());
        ph_end(t, pu);
        t->launches++;
      }
      if (X == 2) {
        CK(cudaEventRecord(s.ev_unperm[slot], s.s_main));
        s.unperm_rec[slot] = true;
      } else {
        TRY(launch_signal(t, s, s.s_main, FLAG_RESC, e));
      }
      TRY(stage_out(t, s, io, off, cnt, int(b % kStage), true));
    }
    return WD_OK;
  };

  TRY(phaseA(0));
  if (X) TRY(phaseT(0));
  for (uint64_t b = 0; b < nbt; ++b) {
    if (b + 1 < nbt) {
      TRY(phaseA(b + 1));
      if (X) TRY(phaseT(b + 1));
    }
    TRY(phaseB(b));
    if (!insert) TRY(phaseC(b));
  }
  t->epoch += nbt;
  return join_into(t, stream, ev0, per);
}

// split a host/device array over the local shards ("split into portions of
// approximately equal size"); in rank mode the whole call is this rank's portion.
void split_io(wd_table* t, const IO& all, std::vector<IO>& ios) {
  const size_t L = t->local.size();
  ios.assign(L, all);
  for (size_t r = 0; r < L; ++r) {
    const uint64_t lo = all.n * r / L, hi = all.n * (r + 1) / L;
    ios[r].n = hi - lo;
    if (all.keys) ios[r].keys = all.keys + lo;
    if (all.vals) ios[r].vals = all.vals + lo;
    if (all.vout) ios[r].vout = all.vout + lo;
    if (all.fout) ios[r].fout = all.fout + lo;
  }
}

// shard < 0: a whole-table call (device memory only for single-device tables); else the
// pointer of local shard `shard` in a _sharded call (device memory on that shard's device)
wd_status_t check_ptr(wd_table* t, const void* p, PtrKind* kind, int shard = -1) {
  int dev = -1;
  *kind = classify(p, &dev);
  if (*kind == PK_DEVICE && p) {
    if (shard < 0 && t->mode == MODE_MULTI)
      return fail(WD_ERR_INVALID_ARG,
                  "device pointers with n_gpus > 1 in one process: pass host memory or use "
                  "wd_insert_sharded / wd_retrieve_sharded");
    const int want = t->local[shard < 0 ? 0 : shard].device;
    if (dev != want)
      return fail(WD_ERR_INVALID_ARG, "device pointer on device %d, shard on device %d", dev, want);
  }
  return WD_OK;
}

// pointer kinds of one call's buffers (same rules for whole-table and per-shard calls)
wd_status_t classify_io(wd_table* t, bool insert, IO& io, int shard) {
  if (!io.n) return WD_OK;
  if (!io.keys) return fail(WD_ERR_INVALID_ARG, "keys == NULL with n > 0");
  if (insert && !io.vals) return fail(WD_ERR_INVALID_ARG, "vals == NULL with n > 0");
  PtrKind k1, k2 = PK_DEVICE, k3 = PK_DEVICE;
  TRY(check_ptr(t, io.keys, &k1, shard));
  if (insert) TRY(check_ptr(t, io.vals, &k2, shard));
  else {
    if (io.vout) TRY(check_ptr(t, io.vout, &k2, shard));
    if (io.fout) TRY(check_ptr(t, io.fout, &k3, shard));
  }
  if (insert && (k1 == PK_DEVICE) != (k2 == PK_DEVICE))
    return fail(WD_ERR_INVALID_ARG, "keys and vals must both be host or both device");
  if (!insert && io.vout && io.fout && (k2 == PK_DEVICE) != (k3 == PK_DEVICE))
    return fail(WD_ERR_INVALID_ARG, "vals_out and found_out must both be host or device");
  io.kin = (k1 == PK_PAGEABLE || k2 == PK_PAGEABLE) && insert ? PK_PAGEABLE : k1;
  io.kout = insert ? PK_DEVICE : (io.vout ? k2 : k3);
  if (!insert && !io.vout && !io.fout) io.kout = PK_DEVICE;
  return WD_OK;
}

// P:245 future work, built: "a heuristic which dynamically scales the group size |g| with
// the current load factor".  P:89 makes switching |g| between calls safe (same probe
// sequence).  Measured on B200 (profiles/r01_sweep.jsonl, 2^28 keys, insert + retrieve
// step): |g| = 8 is fastest up to alpha 0.9, |g| = 16 from 0.95 on (and for misses at any
// load).  The load used is the projected one after this call, from a host-side upper
// estimate of the size (no synchronisation).
// Calls probe with their own |g| (reading C24): P:89 gives every |g| the same probe sequence,
// and an insert's slot — the leftmost empty slot of the sequence — does not depend on the
// window size, so the layout, hence the cost of every call, depends only on the load and on
// the region alignment A fixed at creation.  Auto (default), measured on B200
// (profiles/r02/sweep_r02o.jsonl, 2^28 keys; the table's |g| rows are the paper's setting):
//  * inserts: 16-slot windows on line-aligned tables (A = 16: |g| 32 tables 15.9 -> 23.5 G/s
//    at alpha 0.95) and on shards of <= 64 MB (L2-resident: 2^20 / 2^22 keys 6.9 / 19.8 ->
//    11.0 / 23.9 G/s against 8-slot windows), 8-slot windows on larger A = 4 tables (|g| 1 /
//    2 / 4: 9.7 / 14.4 / 20.7 -> 22.1 G/s; 16-slot windows there: 15.4, they straddle two
//    lines; profiles/r02/insert_group.jsonl) up to 24 GB shards (2^29 / 2^30 / 2^31 keys at
//    |g| 4: 20.7 / 20.2 / 19.0 -> 22.0 / 20.8 / 20.0 G/s); above, where a slice no longer
//    fits the L2 (config 3's 36 GB: 282 MB slices), the table's |g|, at least 4 (|g| 4:
//    21.9 against 20.0 G/s with 8-slot windows; profiles/r02/insert_group_large.jsonl);
//    tables created with |g| = 0 keep the dynamic choice by load;
//  * queries / erases: 16-slot windows on A = 16 tables and above a projected load of 0.93,
//    else 8 (alpha 0.8 / 0.9 on A = 4: 32.2 / 28.0 G/s against 27.1 / 26.1 with 16-slot
//    windows, which straddle two lines there; 0.95 / 0.99: 24.3 / 20.2 against 24.0 / 18.2;
//    misses favour 16 at any load).
// Option value 0 restores the paper's setting (the table's |g|), > 0 forces a |g|.
void pick_group_size(wd_table* t, int op, uint64_t n) {
  const double cap = double(wd_capacity(t));
  const double est = double(t->est_size) + (op == OP_INSERT ? double(n) : 0.0);
  const bool high = est / cap > 0.93;
  const int table_g = t->G ? t->G : (high ? 16 : 8);        // the paper's |g| (0: P:245 by load)
  if (t->ig == 0 || (t->ig < 0 && t->G == 0)) t->G_ins = table_g;
  else if (t->ig > 0) t->G_ins = t->ig;
  else if (t->align >= 16 || t->local[0].cap * 8 <= (64ull << 20)) t->G_ins = 16;
  else t->G_ins = double(t->local[0].cap) * 8 > 24e9 ? std::max(t->G, 4) : 8;
  if (op == OP_INSERT) t->G_used = t->G_ins;
  else if (t->qg == 0) t->G_used = table_g;
  else if (t->qg > 0) t->G_used = t->qg;
  else t->G_used = (t->align >= 16 || high) ? 16 : 8;
  if (op == OP_INSERT) t->est_size = std::min<uint64_t>(t->est_size + n, wd_capacity(t));
}

const char* op_name(int op) {
  return op == OP_INSERT ? "wd_insert" : op == OP_RETRIEVE ? "wd_retrieve" : "wd_erase";
}

wd_status_t do_op_plain(wd_table* t, int op, const IO& io, cudaStream_t stream) {
  if (t->m == 1) {
    if (io.n == 0) return WD_OK;
    return single_op(t, op, io, stream);
  }
  std::vector<IO> ios;
  split_io(t, io, ios);
  return cascade_op(t, op, ios, stream);
}

extern "C" wd_status_t wd_rebuild(wd_table_t* t, uint32_t seed, wd_stream_t stream);

// "In the unlikely case that the probing scheme cannot determine an empty slot for
// n < c the whole data structure is invalidated followed by a subsequent reconstruction with
// a distinct hash function."  With WD_OPT_AUTO_REBUILD an insert call that left keys behind
// (Line 26) while the table still has room — e.g. tombstones of earlier deletions fill the
// probe sequences (reading C9') — is followed, synchronously, by wd_rebuild with a new seed
// (the tombstones go) and a re-insert of the keys recorded at Line 26.
wd_status_t insert_auto_rebuild(wd_table* t, const IO& io, cudaStream_t stream) {
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    if (!s.fail_list) {
      CK(cudaMalloc(&s.fail_list, size_t(kFailCap) * sizeof(unsigned long long)));
      CK(cudaMalloc(&s.fail_count, sizeof(unsigned long long)));
    }
    CK(cudaStreamSynchronize(stream));
    CK(cudaMemset(s.fail_count, 0, sizeof(unsigned long long)));
  }
  TRY(do_op_plain(t, OP_INSERT, io, stream));
  for (int attempt = 0; attempt < 4; ++attempt) {
    // how many keys were left behind, and were they all recorded?
    uint64_t failed = 0, live = 0;
    bool recorded = true;
    std::vector<unsigned long long> nfail(t->local.size(), 0);
    for (size_t r = 0; r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      DeviceGuard g(s.device);
      CK(cudaStreamSynchronize(stream));
      CK(cudaDeviceSynchronize());
      unsigned long long c[wd::CNT_N], fc = 0;
      CK(cudaMemcpy(c, s.counters, sizeof c, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(&fc, s.fail_count, sizeof fc, cudaMemcpyDeviceToHost));
      failed += c[wd::CNT_FAIL];
      live += c[wd::CNT_NEW] - c[wd::CNT_ERASED];
      nfail[r] = fc;
      recorded = recorded && fc == c[wd::CNT_FAIL] && fc <= kFailCap;
    }
    if (failed == 0) return WD_OK;
    if (!recorded || live + failed > wd_capacity(t))   // truly full: keep the sticky error
      return fail(WD_ERR_TABLE_FULL, "%llu inserts exhausted p_max with %llu of %llu slots live",
                  (unsigned long long)failed, (unsigned long long)live,
                  (unsigned long long)wd_capacity(t));
    // set the recorded pairs aside, rebuild with a distinct hash, re-insert them
    std::vector<unsigned long long*> keep(t->local.size(), nullptr), kcnt(t->local.size(), nullptr);
    auto release = [&]() {
      for (size_t r = 0; r < t->local.size(); ++r) {
        DeviceGuard g(t->local[r].device);
        if (keep[r]) cudaFree(keep[r]);
        if (kcnt[r]) cudaFree(kcnt[r]);
      }
    };
    for (size_t r = 0; r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      DeviceGuard g(s.device);
      cudaError_t e = cudaMalloc(&keep[r], std::max<uint64_t>(nfail[r], 1) * 8);
      if (e == cudaSuccess) e = cudaMalloc(&kcnt[r], 8);
      if (e == cudaSuccess && nfail[r])
        e = cudaMemcpy(keep[r], s.fail_list, nfail[r] * 8, cudaMemcpyDeviceToDevice);
      if (e == cudaSuccess) e = cudaMemcpy(kcnt[r], &nfail[r], 8, cudaMemcpyHostToDevice);
      if (e != cudaSuccess) {
        cudaGetLastError();
        release();
        return fail(WD_ERR_OUT_OF_MEMORY, "auto rebuild: %s", cudaGetErrorString(e));
      }
    }
    // the failure record restarts: failures of the rebuild's own re-insert and of the
    // re-insert below are recorded again and handled by the next attempt
    wd_status_t st = WD_OK;
    for (size_t r = 0; st == WD_OK && r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      DeviceGuard g(s.device);
      if (cudaMemset(s.counters + wd::CNT_FAIL, 0, 8) != cudaSuccess ||
          cudaMemset(s.fail_count, 0, 8) != cudaSuccess)
        st = fail(WD_ERR_CUDA, "auto rebuild: counter reset");
    }
    ++t->rebuilds;
    const uint32_t seed = t->local[0].hseed + 0x9E3779B9u * t->rebuilds;
    if (st == WD_OK) st = wd_rebuild(t, seed, reinterpret_cast<wd_stream_t>(stream));
    for (size_t r = 0; st == WD_OK && r < t->local.size(); ++r) {
      Shard& s = t->local[r];
      DeviceGuard g(s.device);
      if (nfail[r]) {
        const wd::InSeg<true> in{keep[r], kcnt[r], nfail[r], 1};
        st = launch_probe<true>(t, s, in, wd::OutNone{}, nfail[r], s.s_main);
      }
      if (st == WD_OK && cudaStreamSynchronize(s.s_main) != cudaSuccess)
        st = fail(WD_ERR_CUDA, "auto rebuild: re-insert");
    }
    release();
    TRY(st);
  }
  return fail(WD_ERR_TABLE_FULL, "auto rebuild: inserts still fail after 4 reconstructions");
}

wd_status_t do_op(wd_table* t, int op, const uint32_t* keys, const uint32_t* vals,
                  uint32_t* vout, uint8_t* fout, uint64_t n, cudaStream_t stream) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  Nvtx nv(op_name(op));
  IO io;
  io.keys = keys; io.vals = vals; io.vout = vout; io.fout = fout; io.n = n;
  TRY(classify_io(t, op == OP_INSERT, io, -1));
  pick_group_size(t, op, n);
  if (op == OP_INSERT && t->auto_rebuild && n) return insert_auto_rebuild(t, io, stream);
  return do_op_plain(t, op, io, stream);
}

// The paper's device-sided cascades: every local shard brings its own
// device-resident portion ("split into portions"), on its own stream.
wd_status_t do_op_sharded(wd_table* t, int op, const uint32_t* const* keys,
                          const uint32_t* const* vals, uint32_t* const* vout, uint8_t* const* fout,
                          const uint64_t* n, const wd_stream_t* streams) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  Nvtx nv(op == OP_INSERT ? "wd_insert_sharded" : "wd_retrieve_sharded");
  if (!keys || !n || (op == OP_INSERT && !vals))
    return fail(WD_ERR_INVALID_ARG, "_sharded: NULL array argument");
  const size_t L = t->local.size();
  std::vector<IO> ios(L);
  std::vector<cudaStream_t> per(L, nullptr);
  uint64_t total = 0;
  for (size_t r = 0; r < L; ++r) {
    IO& io = ios[r];
    io.keys = keys[r];
    io.vals = vals ? vals[r] : nullptr;
    io.vout = vout ? vout[r] : nullptr;
    io.fout = fout ? fout[r] : nullptr;
    io.n = n[r];
    if (streams) per[r] = reinterpret_cast<cudaStream_t>(streams[r]);
    TRY(classify_io(t, op == OP_INSERT, io, int(r)));
    total += n[r];
  }
  pick_group_size(t, op, total);
  if (t->m == 1) {
    if (ios[0].n == 0) return WD_OK;
    return single_op(t, op, ios[0], per[0]);
  }
  return cascade_op(t, op, ios, nullptr, per.data());
}

wd_table* create_common(uint64_t capacity, int mode, int m, int group_size) {
  if (capacity < 1) { fail(WD_ERR_INVALID_ARG, "capacity must be >= 1"); return nullptr; }
  if (group_size != 0 && group_size != 1 && group_size != 2 && group_size != 4 &&
      group_size != 8 && group_size != 16 && group_size != 32) {
    fail(WD_ERR_INVALID_ARG, "group_size %d not in {0 (auto),1,2,4,8,16,32}", group_size);
    return nullptr;
  }
  if (m < 1 || m > wd::kMaxShards) {
    fail(WD_ERR_INVALID_ARG, "number of shards %d not in [1, %d]", m, wd::kMaxShards);
    return nullptr;
  }
  wd_table* t = new wd_table();
  t->mode = mode;
  t->m = m;
  t->G = group_size;
  t->G_used = t->G_ins = group_size ? group_size : 8;
  t->align = wd::region_align_for(group_size);   // reading C2': fixed for the table's life
  return t;
}

bool is_prime(uint64_t x) {
  if (x < 2) return false;
  if (x % 2 == 0) return x == 2;
  for (uint64_t d = 3; d * d <= x; d += 2)
    if (x % d == 0) return false;
  return true;
}

// Reading C13': ceil(c/m) slots, rounded up to a multiple of A (C2') and
// >= 32, then up until the number of region starts nb = (c-32)/A + 1 is prime, so eq. 3's
// double hashing visits every region before repeating.  0 if nb would not fit 32 bits.
uint64_t shard_cap(uint64_t capacity, int m, uint64_t A) {
  uint64_t c = (capacity + m - 1) / m;
  c = round_up(std::max<uint64_t>(c, 32), A);
  uint64_t nb = (c - 32) / A + 1;
  if (nb > 1)
    while (!is_prime(nb)) ++nb;
  if (nb >= (1ull << 32)) return 0;
  return A * (nb - 1) + 32;
}

wd_status_t sticky_status(wd_table* t) {
  unsigned long long agg[wd::CNT_N] = {};
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    unsigned long long c[wd::CNT_N];
    CK(cudaStreamSynchronize(s.s_main));
    CK(cudaStreamSynchronize(s.s_probe));
    CK(cudaStreamSynchronize(s.s_h2d));
    CK(cudaStreamSynchronize(s.s_d2h));
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(c, s.counters, sizeof c, cudaMemcpyDeviceToHost));
    for (int i = 0; i < wd::CNT_N; ++i) agg[i] += c[i];
  }
  if (agg[wd::CNT_XERR]) return fail(WD_ERR_EXCHANGE, "%llu exchange errors (overflow/timeout)", agg[wd::CNT_XERR]);
  if (agg[wd::CNT_FAIL]) return fail(WD_ERR_TABLE_FULL, "%llu inserts exhausted p_max", agg[wd::CNT_FAIL]);
  if (agg[wd::CNT_RSV]) return fail(WD_ERR_RESERVED_KEY, "%llu reserved keys (0xFFFFFFFF) seen", agg[wd::CNT_RSV]);
  return WD_OK;
}

}  // namespace wdi

using namespace wdi;

// ===================================================================== C-ABI
extern "C" {

wd_table_t* wd_create(uint64_t capacity, int n_gpus, int group_size) {
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
    cudaGetLastError();
    fail(WD_ERR_CUDA, "no CUDA device");
    return nullptr;
  }
  // test hook (tests/test_gpu_multi_samedev.py): every shard of a multi-GPU table on the
  // current device, so the single-process multi-GPU code (per-device streams, host-input
  // split, _sharded calls, device-pointer rules) runs on a one-GPU box
  const bool same_dev = getenv("WD_MULTI_SAME_DEVICE") != nullptr;
  if (n_gpus < 1 || (n_gpus > ndev && !same_dev)) {
    fail(WD_ERR_INVALID_ARG, "n_gpus %d not in [1, %d visible]", n_gpus, ndev);
    return nullptr;
  }
  wd_table* t = create_common(capacity, n_gpus == 1 ? MODE_SINGLE : MODE_MULTI, n_gpus, group_size);
  if (!t) return nullptr;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaDeviceGetAttribute(&t->sm_count, cudaDevAttrMultiProcessorCount, n_gpus == 1 || same_dev ? cur : 0);
  const uint64_t c = shard_cap(capacity, n_gpus, t->align);
  t->local.resize(n_gpus);
  for (int d = 0; d < n_gpus; ++d) {
    const int dev = n_gpus == 1 || same_dev ? cur : d;
    if (n_gpus > 1 && !same_dev) {
      DeviceGuard g(dev);
      for (int p = 0; p < n_gpus; ++p)
        if (p != dev) {
          int ok = 0;
          cudaDeviceCanAccessPeer(&ok, dev, p);
          if (ok && cudaDeviceEnablePeerAccess(p, 0) != cudaSuccess) cudaGetLastError();
        }
    }
    if (shard_init(t, t->local[d], d, dev, c, nullptr) != WD_OK) {
      wd_destroy(t);
      return nullptr;
    }
  }
  g_last = WD_OK;
  return t;
}

wd_table_t* wd_create_loopback(uint64_t capacity, int n_shards, int group_size) {
  wd_table* t = create_common(capacity, MODE_LOOPBACK, n_shards, group_size);
  if (!t) return nullptr;
  int cur = 0;
  if (cudaGetDevice(&cur) != cudaSuccess) {
    fail(WD_ERR_CUDA, "no CUDA device");
    delete t;
    return nullptr;
  }
  cudaDeviceGetAttribute(&t->sm_count, cudaDevAttrMultiProcessorCount, cur);
  if (cudaStreamCreateWithFlags(&t->loop_stream, cudaStreamNonBlocking) != cudaSuccess) {
    fail(WD_ERR_CUDA, "stream creation failed");
    delete t;
    return nullptr;
  }
  const uint64_t c = shard_cap(capacity, n_shards, t->align);
  t->local.resize(n_shards);
  for (int d = 0; d < n_shards; ++d)
    if (shard_init(t, t->local[d], d, cur, c, t->loop_stream) != WD_OK) {
      wd_destroy(t);
      return nullptr;
    }
  g_last = WD_OK;
  return t;
}

wd_table_t* wd_create_rank(uint64_t capacity, int rank, int world, int group_size) {
  if (world < 1 || rank < 0 || rank >= world) {
    fail(WD_ERR_INVALID_ARG, "rank %d / world %d", rank, world);
    return nullptr;
  }
  wd_table* t = create_common(capacity, world == 1 ? MODE_SINGLE : MODE_RANK, world, group_size);
  if (!t) return nullptr;
  t->rank = rank;
  int cur = 0;
  if (cudaGetDevice(&cur) != cudaSuccess) {
    fail(WD_ERR_CUDA, "no CUDA device");
    delete t;
    return nullptr;
  }
  cudaDeviceGetAttribute(&t->sm_count, cudaDevAttrMultiProcessorCount, cur);
  t->local.resize(1);
  if (shard_init(t, t->local[0], rank, cur, shard_cap(capacity, world, t->align), nullptr) != WD_OK) {
    wd_destroy(t);
    return nullptr;
  }
  g_last = WD_OK;
  return t;
}

wd_status_t wd_rank_handle(wd_table_t* t, uint8_t out[WD_RANK_HANDLE_BYTES]) {
  if (!t || !out) return fail(WD_ERR_INVALID_ARG, "wd_rank_handle arguments");
  RankHandle h;
  memset(&h, 0, sizeof h);
  h.magic = kHandleMagic;
  h.world = uint32_t(t->m);
  h.rank = uint32_t(t->rank);
  if (t->mode == MODE_RANK) {
    TRY(ensure_exchange(t));                  // arena for the current batch size
    Shard& s = t->local[0];
    DeviceGuard g(s.device);
    cudaIpcMemHandle_t ipc;
    CK(cudaIpcGetMemHandle(&ipc, s.arena));
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "ipc handle size");
    memcpy(h.ipc, &ipc, 64);
    h.batch = t->xbatch;
    h.arena_bytes = s.arena_bytes;
    h.exchange = uint32_t(t->exchange);
    if (t->exchange == 2 && t->rank == 0) {   // NCCL bootstrap id, only when asked for
      const NcclApi* a = nccl_api();
      if (!a) return fail(WD_ERR_NCCL, "%s", g_nccl.why);
      NcclUid id;
      NK(a->GetUniqueId(&id));
      memcpy(h.nccl_id, &id, sizeof id);
      h.has_nccl_id = 1;
    }
  }
  memcpy(out, &h, sizeof h);
  return WD_OK;
}

wd_status_t wd_rank_connect(wd_table_t* t, const uint8_t* handles, wd_allreduce_fn fn, void* ctx) {
  if (!t || !handles || !fn) return fail(WD_ERR_INVALID_ARG, "wd_rank_connect arguments");
  t->allreduce = fn;
  t->allreduce_ctx = ctx;
  if (t->mode != MODE_RANK) { t->connected = true; return WD_OK; }
  if (t->connected) return fail(WD_ERR_INVALID_ARG, "already connected");
  TRY(ensure_exchange(t));
  Shard& s = t->local[0];
  DeviceGuard g(s.device);
  for (int d = 0; d < t->m; ++d) {
    RankHandle h;
    memcpy(&h, handles + size_t(d) * WD_RANK_HANDLE_BYTES, sizeof h);
    if (h.magic != kHandleMagic || int(h.world) != t->m || int(h.rank) != d)
      return fail(WD_ERR_INVALID_ARG, "handle %d: bad magic/world/rank order", d);
    if (h.batch != t->xbatch || h.arena_bytes != s.arena_bytes)
      return fail(WD_ERR_INVALID_ARG, "handle %d: batch size differs between ranks", d);
    if (int(h.exchange) != t->exchange)
      return fail(WD_ERR_INVALID_ARG, "handle %d: WD_OPT_EXCHANGE differs between ranks", d);
    if (d == 0 && h.has_nccl_id) {
      memcpy(t->nccl_id, h.nccl_id, sizeof t->nccl_id);
      t->have_nccl_id = true;
    }
    if (d == t->rank) continue;
    cudaIpcMemHandle_t ipc;
    memcpy(&ipc, h.ipc, 64);
    void* base = nullptr;
    CK(cudaIpcOpenMemHandle(&base, ipc, cudaIpcMemLazyEnablePeerAccess));
    t->opened.push_back(base);
    t->peers[d] = arena_view(base, t->m, t->xbatch);
  }
  t->connected = true;
  uint64_t one = 1;                            // every rank mapped every peer before use
  TRY(host_allreduce(t, &one, WD_REDUCE_SUM));
  if (one != uint64_t(t->m)) return fail(WD_ERR_EXCHANGE, "connect barrier: %llu of %d ranks",
                                         (unsigned long long)one, t->m);
  return WD_OK;
}

void wd_destroy(wd_table_t* t) {
  if (!t) return;
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    cudaDeviceSynchronize();
  }
  if (t->mode == MODE_RANK && t->connected) {  // no rank unmaps before every rank is done
    uint64_t one = 1;
    host_allreduce(t, &one, WD_REDUCE_SUM);
  }
  for (void* p : t->opened) cudaIpcCloseMemHandle(p);
  if (t->nccl_ready) free_nccl(t);
  for (auto& kv : t->ph_pool) {
    DeviceGuard g(kv.first);
    for (cudaEvent_t e : kv.second) cudaEventDestroy(e);
  }
  for (auto& r : t->ph_recs) {
    DeviceGuard g(r.device);
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  for (auto& s : t->local) free_staged(s);
  for (auto& s : t->local) shard_free(s);
  if (t->loop_stream) cudaStreamDestroy(t->loop_stream);
  delete t;
}

wd_status_t wd_clear(wd_table_t* t, wd_stream_t stream) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  t->est_size = 0;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (t->mode == MODE_SINGLE) {
    Shard& s = t->local[0];
    DeviceGuard g(s.device);
    wd::fill_kernel<<<t->sm_count * 4, wd::kBlock, 0, st>>>(s.slots, s.cap, s.counters, wd::CNT_N);
    CK(cudaGetLastError());
    t->launches++;
    return WD_OK;
  }
  cudaEvent_t ev0;
  TRY(fork_from(t, st, &ev0));
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    wd::fill_kernel<<<t->sm_count * 4, wd::kBlock, 0, s.s_main>>>(s.slots, s.cap, s.counters,
                                                                  wd::CNT_N);
    CK(cudaGetLastError());
    t->launches++;
  }
  return join_into(t, st, ev0);
}

wd_status_t wd_insert(wd_table_t* t, const uint32_t* keys, const uint32_t* vals, uint64_t n,
                      wd_stream_t stream) {
  return do_op(t, OP_INSERT, keys, vals, nullptr, nullptr, n, reinterpret_cast<cudaStream_t>(stream));
}

wd_status_t wd_retrieve(wd_table_t* t, const uint32_t* keys, uint32_t* vals_out, uint8_t* found_out,
                        uint64_t n, wd_stream_t stream) {
  return do_op(t, OP_RETRIEVE, keys, nullptr, vals_out, found_out, n,
               reinterpret_cast<cudaStream_t>(stream));
}

wd_status_t wd_insert_sharded(wd_table_t* t, const uint32_t* const keys[], const uint32_t* const vals[],
                              const uint64_t n[], const wd_stream_t streams[]) {
  return do_op_sharded(t, OP_INSERT, keys, vals, nullptr, nullptr, n, streams);
}

wd_status_t wd_retrieve_sharded(wd_table_t* t, const uint32_t* const keys[], uint32_t* const vals_out[],
                                uint8_t* const found_out[], const uint64_t n[],
                                const wd_stream_t streams[]) {
  return do_op_sharded(t, OP_RETRIEVE, keys, nullptr, vals_out, found_out, n, streams);
}

wd_status_t wd_erase(wd_table_t* t, const uint32_t* keys, uint8_t* found_out, uint64_t n,
                     wd_stream_t stream) {
  return do_op(t, OP_ERASE, keys, nullptr, nullptr, found_out, n,
               reinterpret_cast<cudaStream_t>(stream));
}

wd_status_t wd_rebuild(wd_table_t* t, uint32_t seed, wd_stream_t stream) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    CK(cudaStreamSynchronize(st));
    CK(cudaStreamSynchronize(s.s_main));
    CK(cudaStreamSynchronize(s.s_probe));
    // live entries = new keys - erased keys (counters: the contents survive, the
    // tombstones do not)
    unsigned long long c[wd::CNT_N];
    CK(cudaMemcpy(c, s.counters, sizeof c, cudaMemcpyDeviceToHost));
    const uint64_t n_live = c[wd::CNT_NEW] - c[wd::CNT_ERASED];
    unsigned long long *live = nullptr, *cnt = nullptr, *fresh = nullptr;
    auto release = [&]() {
      if (live) cudaFree(live);
      if (cnt) cudaFree(cnt);
      if (fresh) cudaFree(fresh);
    };
    cudaError_t e = cudaMalloc(&live, std::max<uint64_t>(n_live, 1) * sizeof(unsigned long long));
    if (e == cudaSuccess) e = cudaMalloc(&cnt, sizeof(unsigned long long));
    if (e == cudaSuccess) e = cudaMalloc(&fresh, s.cap * sizeof(unsigned long long));
    if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, sizeof(unsigned long long), s.s_main);
    if (e != cudaSuccess) {
      cudaGetLastError();
      release();
      return fail(e == cudaErrorMemoryAllocation ? WD_ERR_OUT_OF_MEMORY : WD_ERR_CUDA,
                  "wd_rebuild: %s", cudaGetErrorString(e));
    }
    // 1. gather the live slots; 2. a fresh table with the distinct hash (translated variant,
    // P:161).  The sticky error counters are kept; only new / erased restart.
    const int cgrid = t->serial ? 1 : t->sm_count * 8;
    wd::compact_kernel<<<cgrid, t->serial ? 32 : wd::kBlock, 0, s.s_main>>>(s.slots, s.cap, live, n_live, cnt);
    wd::fill_kernel<<<t->sm_count * 4, wd::kBlock, 0, s.s_main>>>(fresh, s.cap, s.counters, 0);
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemsetAsync(s.counters + wd::CNT_NEW, 0, sizeof(unsigned long long), s.s_main);
    if (e == cudaSuccess) e = cudaMemsetAsync(s.counters + wd::CNT_ERASED, 0, sizeof(unsigned long long), s.s_main);
    if (e != cudaSuccess) {
      cudaStreamSynchronize(s.s_main);
      release();
      return fail(WD_ERR_CUDA, "wd_rebuild: %s", cudaGetErrorString(e));
    }
    t->launches += 2;
    // 3. re-insert (Fig. 3) from the gathered pairs into the fresh slots
    unsigned long long* old = s.slots;
    const uint32_t old_seed = s.hseed;
    s.slots = fresh;
    s.hseed = seed;
    const wd::InSeg<true> in{live, cnt, std::max<uint64_t>(n_live, 1), 1};
    wd_status_t r = launch_probe<true>(t, s, in, wd::OutNone{}, n_live, s.s_main);
    e = cudaStreamSynchronize(s.s_main);
    if (r != WD_OK || e != cudaSuccess) {   // keep the old table
      s.slots = old;
      s.hseed = old_seed;
      release();
      if (r == WD_OK) r = fail(WD_ERR_CUDA, "wd_rebuild: %s", cudaGetErrorString(e));
      return r;
    }
    fresh = nullptr;                         // now the table
    cudaFree(old);
    release();
  }
  return WD_OK;
}

wd_status_t wd_sync(wd_table_t* t) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  return sticky_status(t);
}

uint64_t wd_size(wd_table_t* t) {
  if (!t) { fail(WD_ERR_INVALID_ARG, "null table"); return UINT64_MAX; }
  unsigned long long total = 0;
  for (auto& s : t->local) {
    DeviceGuard g(s.device);
    unsigned long long c[wd::CNT_N];
    if (cudaDeviceSynchronize() != cudaSuccess ||
        cudaMemcpy(c, s.counters, sizeof c, cudaMemcpyDeviceToHost) != cudaSuccess) {
      fail(WD_ERR_CUDA, "wd_size: %s", cudaGetErrorString(cudaGetLastError()));
      return UINT64_MAX;
    }
    total += c[wd::CNT_NEW] - c[wd::CNT_ERASED];
  }
  if (t->mode == MODE_RANK) {
    uint64_t v = total;
    if (host_allreduce(t, &v, WD_REDUCE_SUM) != WD_OK) return UINT64_MAX;
    total = v;
  }
  t->est_size = total;
  return total;
}

uint64_t wd_capacity(wd_table_t* t) {
  if (!t) return 0;
  return t->local[0].cap * uint64_t(t->m);
}

wd_status_t wd_set_option(wd_table_t* t, wd_option_t opt, int64_t v) {
  if (!t) return fail(WD_ERR_INVALID_ARG, "null table");
  switch (opt) {
    case WD_OPT_GROUP_SIZE:
      if (v != 0 && v != 1 && v != 2 && v != 4 && v != 8 && v != 16 && v != 32)
        return fail(WD_ERR_INVALID_ARG, "group size %lld", (long long)v);
      t->G = int(v);
      if (v) t->G_used = t->G_ins = int(v);
      return WD_OK;
    case WD_OPT_QUERY_GROUP_SIZE:
      if (v != -1 && v != 0 && v != 1 && v != 2 && v != 4 && v != 8 && v != 16 && v != 32)
        return fail(WD_ERR_INVALID_ARG, "query group size %lld", (long long)v);
      t->qg = int(v);
      return WD_OK;
    case WD_OPT_INSERT_GROUP_SIZE:
      if (v != -1 && v != 0 && v != 1 && v != 2 && v != 4 && v != 8 && v != 16 && v != 32)
        return fail(WD_ERR_INVALID_ARG, "insert group size %lld", (long long)v);
      t->ig = int(v);
      return WD_OK;
    case WD_OPT_P_MAX:
      if (v < 0 || v > (1 << 26)) return fail(WD_ERR_INVALID_ARG, "p_max %lld", (long long)v);
      t->pmax = int(v);
      return WD_OK;
    case WD_OPT_BATCH:
      if (v < 1 || v > (1ll << wd::kPosShift)) return fail(WD_ERR_INVALID_ARG, "batch %lld", (long long)v);
      t->batch = uint64_t(v);
      t->batch_set = true;
      return WD_OK;
    case WD_OPT_SERIAL: t->serial = v ? 1 : 0; return WD_OK;
    case WD_OPT_KEYS_IN_FLIGHT:
      if (v != 0 && v != 1 && v != 2 && v != 4 && v != 8) return fail(WD_ERR_INVALID_ARG, "keys in flight %lld", (long long)v);
      t->kif = int(v);
      return WD_OK;
    case WD_OPT_PART_SEED: t->pseed = uint32_t(v); return WD_OK;
    case WD_OPT_SLOTS_PER_LANE:
      if (v != 0 && v != 1 && v != 2 && v != 4 && v != 8 && v != 16)
        return fail(WD_ERR_INVALID_ARG, "slots per lane %lld", (long long)v);
      t->spl = int(v);
      return WD_OK;
    case WD_OPT_KERNEL_FLAGS:
      if (v < 0 || (uint32_t(v) & ~wd::kF_ALL) != 0) return fail(WD_ERR_INVALID_ARG, "kernel flags %lld", (long long)v);
      t->kflags = uint32_t(v);
      return WD_OK;
    case WD_OPT_PROBE_MODE:
      if (v < 0 || v > 2) return fail(WD_ERR_INVALID_ARG, "probe mode %lld", (long long)v);
      t->probe_mode = int(v);
      return WD_OK;
    case WD_OPT_PART_MODE:
      if (v != 0 && v != 1) return fail(WD_ERR_INVALID_ARG, "partition mode %lld", (long long)v);
      t->pmode = int(v);
      return WD_OK;
    case WD_OPT_SPAN:
      if (v < 0 || v > 2) return fail(WD_ERR_INVALID_ARG, "span %lld", (long long)v);
      t->span = int(v);
      return WD_OK;
    case WD_OPT_SLICES:
      if (v < 0 || v > wd::kMaxSlices) return fail(WD_ERR_INVALID_ARG, "slices %lld", (long long)v);
      t->slices = int(v);
      return WD_OK;
    case WD_OPT_PHASE_TIMING:
      t->phase_on = v != 0;
      return WD_OK;
    case WD_OPT_AUTO_REBUILD:
      if (v && t->mode == MODE_RANK)
        return fail(WD_ERR_UNSUPPORTED, "automatic rebuild is single-process only");
      t->auto_rebuild = v != 0;
      return WD_OK;
    case WD_OPT_EXCHANGE:
      if (v < 0 || v > 2) return fail(WD_ERR_INVALID_ARG, "exchange %lld", (long long)v);
      if (v == 2 && t->mode == MODE_LOOPBACK)
        return fail(WD_ERR_UNSUPPORTED, "the NCCL exchange needs one GPU per shard; loopback "
                                        "shards share a device (use 1, the copy engine)");
      if (t->mode == MODE_RANK && t->connected && int(v) != t->exchange)
        return fail(WD_ERR_INVALID_ARG, "rank mode: WD_OPT_EXCHANGE is fixed by wd_rank_connect");
      t->exchange = int(v);
      return WD_OK;
    default: return fail(WD_ERR_INVALID_ARG, "option %d is read-only or unknown", int(opt));
  }
}

int64_t wd_get_option(wd_table_t* t, wd_option_t opt) {
  if (!t) { fail(WD_ERR_INVALID_ARG, "null table"); return INT64_MIN; }
  switch (opt) {
    case WD_OPT_GROUP_SIZE: return t->G;
    case WD_OPT_GROUP_SIZE_USED: return t->G_used;
    case WD_OPT_QUERY_GROUP_SIZE: return t->qg;
    case WD_OPT_INSERT_GROUP_SIZE: return t->ig;
    case WD_OPT_REGION_ALIGN: return t->align;
    case WD_OPT_P_MAX: return t->pmax;
    case WD_OPT_BATCH: return int64_t(t->batch);
    case WD_OPT_SERIAL: return t->serial;
    case WD_OPT_KEYS_IN_FLIGHT: return t->kif;
    case WD_OPT_PART_SEED: return t->pseed;
    case WD_OPT_PROBE_MODE: return t->probe_mode;
    case WD_OPT_KERNEL_FLAGS: return t->kflags;
    case WD_OPT_SLOTS_PER_LANE: return t->spl;
    case WD_OPT_PART_MODE: return t->pmode;
    case WD_OPT_SPAN: return t->span;
    case WD_OPT_SLICES: return t->slices;
    case WD_OPT_EXCHANGE: return t->exchange;
    case WD_OPT_PHASE_TIMING: return t->phase_on ? 1 : 0;
    case WD_OPT_AUTO_REBUILD: return t->auto_rebuild ? 1 : 0;
    case WD_OPT_N_SHARDS: return t->m;
    case WD_OPT_RANK: return t->rank;
    case WD_OPT_LOCAL_SHARDS: return int64_t(t->local.size());
    case WD_OPT_LAUNCHES: return int64_t(t->launches);
  }
  fail(WD_ERR_INVALID_ARG, "unknown option %d", int(opt));
  return INT64_MIN;
}

wd_status_t wd_phase_times(wd_table_t* t, double ms_out[WD_N_PHASES], uint64_t count_out[WD_N_PHASES]) {
  if (!t || !ms_out) return fail(WD_ERR_INVALID_ARG, "wd_phase_times arguments");
  for (int i = 0; i < WD_N_PHASES; ++i) {
    ms_out[i] = 0.0;
    if (count_out) count_out[i] = 0;
  }
  wd_status_t st = WD_OK;
  for (auto& r : t->ph_recs) {
    DeviceGuard g(r.device);
    float ms = 0.f;
    if (st == WD_OK) {
      const cudaError_t e1 = cudaEventSynchronize(r.b);
      const cudaError_t e2 = e1 == cudaSuccess ? cudaEventElapsedTime(&ms, r.a, r.b) : e1;
      if (e2 != cudaSuccess) st = fail(WD_ERR_CUDA, "wd_phase_times: %s", cudaGetErrorString(e2));
    }
    if (r.phase >= 0 && r.phase < WD_N_PHASES) {
      ms_out[r.phase] += ms;
      if (count_out) count_out[r.phase] += 1;
    }
    t->ph_pool[r.device].push_back(r.a);
    t->ph_pool[r.device].push_back(r.b);
  }
  t->ph_recs.clear();
  return st;
}

wd_status_t wd_probe_counts(wd_table_t* t, int shard, uint64_t out[5]) {
  if (!t || shard < 0 || shard >= int(t->local.size()) || !out)
    return fail(WD_ERR_INVALID_ARG, "wd_probe_counts arguments");
#ifndef WD_COUNT_PROBES
  return fail(WD_ERR_UNSUPPORTED, "probe accounting needs a -DWD_COUNT_PROBES build of the library");
#else
  Shard& s = t->local[shard];
  DeviceGuard g(s.device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(out, s.counters + wd::CNT_WIN, 5 * 8, cudaMemcpyDeviceToHost));
  CK(cudaMemset(s.counters + wd::CNT_WIN, 0, 5 * 8));
  return WD_OK;
#endif
}

wd_status_t wd_last_error(void) { return g_last; }

const char* wd_error_string(wd_status_t s) {
  switch (s) {
    case WD_OK: return "WD_OK";
    case WD_ERR_INVALID_ARG: return "WD_ERR_INVALID_ARG";
    case WD_ERR_OUT_OF_MEMORY: return "WD_ERR_OUT_OF_MEMORY";
    case WD_ERR_CUDA: return "WD_ERR_CUDA";
    case WD_ERR_NCCL: return "WD_ERR_NCCL";
    case WD_ERR_TABLE_FULL: return "WD_ERR_TABLE_FULL";
    case WD_ERR_RESERVED_KEY: return "WD_ERR_RESERVED_KEY";
    case WD_ERR_EXCHANGE: return "WD_ERR_EXCHANGE";
    case WD_ERR_UNSUPPORTED: return "WD_ERR_UNSUPPORTED";
  }
  return "WD_ERR_UNKNOWN";
}

const char* wd_last_error_message(void) { return g_msg; }

uint64_t wd_shard_capacity(wd_table_t* t, int shard) {
  if (!t || shard < 0 || shard >= int(t->local.size())) return 0;
  return t->local[shard].cap;
}

wd_status_t wd_dump(wd_table_t* t, int shard, uint64_t* host_out) {
  if (!t || shard < 0 || shard >= int(t->local.size()) || !host_out)
    return fail(WD_ERR_INVALID_ARG, "wd_dump arguments");
  Shard& s = t->local[shard];
  DeviceGuard g(s.device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(host_out, s.slots, s.cap * 8, cudaMemcpyDeviceToHost));
  return WD_OK;
}

wd_status_t wd_counters(wd_table_t* t, int shard, uint64_t out[6]) {
  if (!t || shard < 0 || shard >= int(t->local.size()) || !out)
    return fail(WD_ERR_INVALID_ARG, "wd_counters arguments");
  Shard& s = t->local[shard];
  DeviceGuard g(s.device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(out, s.counters, 6 * 8, cudaMemcpyDeviceToHost));   // the ABI's six (probe counts: wd_probe_counts)
  return WD_OK;
}

}  // extern "C"
