/* =====================================================================================
 * warpdrive.h — C-ABI of the B200-native WarpDrive hot path (libwarpdrive.so).
 *
 * Bulk insert / retrieve of 32-bit keys and 32-bit values in an open-addressing GPU hash
 * table with subwarp window probing (D. Jünger, C. Hundt, B. Schmidt, "WarpDrive:
 * Massively Parallel Hashing on Multi-GPU Nodes", IPDPS 2018; P:N = line N of PAPER.md).
 *
 *   problem statement ...... exact map f: K -> V, k -> v
 *   data layout ............ 4-byte key + 4-byte value packed in one 64-bit slot
 *   load factor ............ alpha = n / c, fixed capacity
 *   probing ................ Fig. 3 INSERT with a coalesced group of |g| lanes
 *   duplicates ............. an existing key's value is updated
 *   multi-GPU .............. multisplit -> transposition -> insert / query
 *   out-of-core ............ host batches overlapped with the device cascade   (Fig. 5)
 *
 * No C++ or torch type crosses this boundary: plain pointers (host or device), sizes and
 * cudaStream_t.  Everything behind wd_table_t is owned by the library.
 *
 * Conventions (apply to every call unless stated otherwise)
 * ---------------------------------------------------------
 * Errors   Argument/allocation errors are returned synchronously.  Device-side conditions
 *          (WD_ERR_TABLE_FULL, WD_ERR_RESERVED_KEY, WD_ERR_EXCHANGE) are STICKY: they are
 *          reported by the next call, by wd_sync() or wd_size(), and cleared by wd_clear().
 *          wd_last_error_message() returns a thread-local human-readable description.
 * Async    Calls enqueue work ordered after `stream` and return; `stream` is made to wait
 *          for the call's completion, so completion is observed through `stream`.  Buffers
 *          passed in must stay valid and unmodified until `stream` passes the call.
 *          stream may be 0 (legacy default stream) or any stream of the table's device.
 * Pointers Host pointers (pinned or pageable) are accepted by every mode and are streamed
 *          in batches; pageable memory is staged through internal pinned buffers.
 *          Device pointers must be on the table's device (single / rank / loopback modes).
 * Threads  A handle is not thread-safe: one host thread uses it at a time.
 * ===================================================================================== */
#ifndef WARPDRIVE_H
#define WARPDRIVE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* wd_stream_t;   /* == cudaStream_t, without including CUDA */
typedef struct wd_table wd_table_t;        /* opaque */

typedef enum {
    WD_OK = 0,
    WD_ERR_INVALID_ARG = 1,
    WD_ERR_OUT_OF_MEMORY = 2,
    WD_ERR_CUDA = 3,
    WD_ERR_NCCL = 4,           /* NCCL exchange (WD_OPT_EXCHANGE = 2): NCCL not loadable or an
                                  NCCL call failed (text: wd_last_error_message) */
    WD_ERR_TABLE_FULL = 5,     /* >=1 insert exhausted p_max regions (Fig. 3 Line 26);
                                  that pair was dropped */
    WD_ERR_RESERVED_KEY = 6,   /* >=1 input key == WD_EMPTY_KEY; those pairs were skipped
                                  (inserts) or reported not-found (queries) */
    WD_ERR_EXCHANGE = 7,       /* multi-GPU exchange: receive-region overflow or a peer
                                  signal timed out */
    WD_ERR_UNSUPPORTED = 8
} wd_status_t;

/* "empty placeholder".  Reading C8: all-ones key; never stored. */
#define WD_EMPTY_KEY 0xFFFFFFFFu
/* value written to vals_out[i] when found_out[i] == 0 (found_out is authoritative:
 * stored values may legitimately equal 0xFFFFFFFF, "arbitrary 4-byte values"). */
#define WD_NOT_FOUND 0xFFFFFFFFu

/* ------------------------------------------------------------------ creation ------- */

/* Single process.  n_gpus == 1: one table on the current CUDA device.
 * Side effect: while any table lives on a device, that device's L2 fetch granularity
 * (cudaLimitMaxL2FetchGranularity, device-wide) is 32 B so random 32-B windows do not pull
 * whole lines; the caller's value is restored when the last table on the device is
 * destroyed (environment WD_L2_FETCH_BYTES=<bytes> overrides, 0 = leave it alone).
 * n_gpus > 1: one shard per device 0..n_gpus-1, keys owned by shard p(k),
 * peer access over NVLink; host input is split into n_gpus contiguous chunks.
 * (Test hook: with environment WD_MULTI_SAME_DEVICE set, all shards live on the current
 * device, so this mode's code runs on a one-GPU box; n_gpus may then exceed the count.)
 * capacity: total slots c (alpha = n / c).  Each shard gets ceil(c / m) slots,
 * rounded up to a multiple of A and to at least 32 (the 32-slot region, Fig. 3 Line 6), then
 * until the region count is prime (C13').  A = the region-start alignment (C2'):
 * 16 slots (one 128-byte line) if group_size >= 16, else 4 (one sector).
 * group_size: |g| in {1,2,4,8,16,32}, or 0 = dynamic by load (see
 * WD_OPT_GROUP_SIZE).  Returns NULL on error (see wd_last_error). */
wd_table_t* wd_create(uint64_t capacity, int n_gpus, int group_size);

/* Test backend: m virtual shards on the CURRENT device, running the full multi-GPU
 * cascade (multisplit -> transposition -> insert/query -> reverse) with peer pointers
 * that happen to be local.  Semantics identical to wd_create(capacity, m, g). */
wd_table_t* wd_create_loopback(uint64_t capacity, int n_shards, int group_size);

/* One process per GPU (torchrun).  Collective: every rank calls every wd_insert /
 * wd_retrieve / wd_clear / wd_size / wd_destroy in the same order (each with its own
 * local n >= 0).  Bootstrap, on each rank's current device:
 *   t = wd_create_rank(capacity, rank, world, g);      capacity = total slots, all ranks
 *   wd_rank_handle(t, blob);                           IPC handle of the exchange arena
 *   (caller all-gathers the world blobs in rank order, e.g. torch.distributed)
 *   wd_rank_connect(t, blobs, allreduce, ctx);         maps every peer's arena (NVLink)
 * `allreduce` is a HOST collective over the same ranks (sum or max of one uint64, in
 * place, returns 0 on success); it is called synchronously, in the same order on every
 * rank, for control only (batch-count agreement, wd_size, barriers) — the data path is
 * peer-memory stores/loads inside the kernels.  WD_OPT_BATCH is fixed once connected. */
#define WD_RANK_HANDLE_BYTES 256
#define WD_REDUCE_SUM 0
#define WD_REDUCE_MAX 1
typedef int (*wd_allreduce_fn)(uint64_t* value, int op, void* ctx);
wd_table_t* wd_create_rank(uint64_t capacity, int rank, int world, int group_size);
wd_status_t wd_rank_handle(wd_table_t* t, uint8_t out[WD_RANK_HANDLE_BYTES]);
wd_status_t wd_rank_connect(wd_table_t* t, const uint8_t* handles, wd_allreduce_fn allreduce,
                            void* ctx);

/* Resource release (no passage of the paper: its table lives for the whole run).
 * NULL-safe.  Synchronizes the table's devices, then frees the table, staging and scratch
 * buffers, peer mappings and communicators; in rank mode it is collective (a barrier
 * before unmapping).  Errors are ignored. */
void wd_destroy(wd_table_t* t);

/* ------------------------------------------------------------------ the hot path --- */

/* a1: re-fill every slot with EMPTY and zero the counters (a fresh table). */
wd_status_t wd_clear(wd_table_t* t, wd_stream_t stream);

/* a2+a3 (and a6-a9 when m > 1, a11 for host pointers): bulk upsert of n pairs
 * keys[i] -> vals[i] (SoA uint32 arrays).  Duplicate keys: the stored value is one of
 * the values inserted for that key; across stream-ordered calls the later call
 * wins.  Reserved key WD_EMPTY_KEY: skipped, sticky WD_ERR_RESERVED_KEY. */
wd_status_t wd_insert(wd_table_t* t, const uint32_t* keys, const uint32_t* vals, uint64_t n,
                      wd_stream_t stream);

/* a4 — retrieval "in a similar way" to the insertion: the same windows of the same
 * region sequence; a query stops at the first window holding its key (found) or an empty
 * slot (absent, reading C10).  With m > 1 also a6-a10: multisplit -> transposition ->
 * local query -> reverse transposition; with host pointers a11.
 * For each i: found_out[i] = 1 and vals_out[i] = the stored value if keys[i] is present,
 * else found_out[i] = 0 and vals_out[i] = WD_NOT_FOUND (C11).  keys: uint32[n];
 * vals_out: uint32[n] or NULL (presence only); found_out: uint8[n] or NULL.  Results in
 * input order.  The reserved key reports not-found (sticky WD_ERR_RESERVED_KEY). */
wd_status_t wd_retrieve(wd_table_t* t, const uint32_t* keys, uint32_t* vals_out,
                        uint8_t* found_out, uint64_t n, wd_stream_t stream);

/* The paper's device-sided cascades: the call's pairs are
 * already split into per-GPU portions in device memory.  Arrays have one entry per
 * LOCAL shard (wd_get_option(WD_OPT_LOCAL_SHARDS): n_gpus for wd_create / loopback tables,
 * 1 in rank mode); keys[r] / vals[r] (uint32[n[r]]) live on shard r's device (host memory is
 * also accepted and streamed, a11); streams[r] is a stream of that device (NULL array: the
 * legacy stream everywhere).  Each portion is multisplit and sent to its owners exactly like
 * the whole-table calls; completion of shard r's part (its table's inserts, or the results of
 * its portion's queries) is ordered on streams[r].  Same semantics and errors as
 * wd_insert / wd_retrieve. */
wd_status_t wd_insert_sharded(wd_table_t* t, const uint32_t* const keys[],
                              const uint32_t* const vals[], const uint64_t n[],
                              const wd_stream_t streams[]);
wd_status_t wd_retrieve_sharded(wd_table_t* t, const uint32_t* const keys[],
                                uint32_t* const vals_out[], uint8_t* const found_out[],
                                const uint64_t n[], const wd_stream_t streams[]);

/* P:91 deletion (NEXT #3; barrier-separated from inserts, i.e. not concurrent with a
 * wd_insert on the same table): every present key in keys[0..n) is removed — its slot
 * becomes a tombstone (reading C9': probed past by queries, not reused by inserts until
 * wd_rebuild).  found_out[i] (may be NULL) = 1 for exactly one occurrence of each key this
 * call removed.  Same pointer kinds and asynchrony as wd_retrieve. */
wd_status_t wd_erase(wd_table_t* t, const uint32_t* keys, uint8_t* found_out, uint64_t n,
                     wd_stream_t stream);

/* P:63 reconstruction: re-insert every live entry into a fresh table of the same capacity
 * with the hash seed `seed` (translated variants h(k + seed)); tombstones are dropped.
 * Synchronizes.  Needs, transiently, a second table's worth of device memory plus 8 B per
 * live entry; on any failure the old table is kept and nothing leaks.  Sticky error
 * counters (TABLE_FULL / RESERVED_KEY / EXCHANGE) survive the rebuild. */
wd_status_t wd_rebuild(wd_table_t* t, uint32_t seed, wd_stream_t stream);

/* a5: number of distinct keys stored (summed over shards and ranks) — the n of the load
 * factor alpha = n / c.  Synchronizes (collective in rank mode).  UINT64_MAX on
 * error (wd_last_error). */
uint64_t wd_size(wd_table_t* t);

/* physical slots summed over all shards (load = wd_size / wd_capacity). */
uint64_t wd_capacity(wd_table_t* t);

/* Wait for all enqueued work; returns (and keeps) sticky device-side errors. */
wd_status_t wd_sync(wd_table_t* t);

/* ------------------------------------------------------------------ options -------- */
typedef enum {
    WD_OPT_GROUP_SIZE = 0,   /* |g|; the probe sequence does not depend on it.
                                0 = dynamic by load: 8, or 16 above a projected
                                load of 0.93 (measured on B200) */
    WD_OPT_P_MAX = 1,        /* outer probing bound p_max (Fig. 3 Line 4); 0 (default) = the
                                number of regions nb, i.e. fail only when the table is full (C4') */
    WD_OPT_BATCH = 2,        /* items per shard per pipeline batch; multi-shard calls round it
                                up to a power of two.  Default: 2^24 for the multi-shard
                                cascade, 2^22 for single-shard host streaming (shorter
                                pipeline fill/drain, measured) unless set explicitly */
    WD_OPT_SERIAL = 3,       /* 1: one probing group, one key at a time (deterministic
                                layout, test hook for the Fig. 3 replay) */
    WD_OPT_KEYS_IN_FLIGHT = 4, /* 0 = default; else keys per group in flight (1,2,4,8) */
    WD_OPT_PART_SEED = 5,    /* seed of the partition function p(k) (C15) */
    WD_OPT_PART_MODE = 6,    /* 0: p(k) = fmix32(k+seed)*m >> 32; 1: k mod m (Fig. 4) */
    WD_OPT_PROBE_MODE = 7,   /* 0 (default): auto — lane-window when the shard fits in half
                                the L2 (<= 64 MB) and |g| <= 8, else cooperative group;
                                1: cooperative group of |g| lanes per window (Fig. 3);
                                2: lane-window — one lane loads the whole |g|-slot window with
                                one sm_100 vector load (|g| <= 8; same windows, same result) */
    WD_OPT_KERNEL_FLAGS = 8, /* bit 0: probe loads may hit L1 (safe: keys never change once
                                written; a lost CAS reloads from L2); bit 1: value updates
                                of existing keys as atomic exchange; bit 2: reserved
                                (rejected); bit 3: a query call visits its input chunks in a scrambled
                                order (keys inserted together are not queried together;
                                results land in the same positions).  Default 11. */
    WD_OPT_SLOTS_PER_LANE = 9, /* V: each lane of a window loads V consecutive slots with one
                                vector load, so a window is read by |g|/V lanes (1: the
                                paper's cooperative group; |g|: one lane).  0 = from
                                WD_OPT_PROBE_MODE.  V in {1,2,4,8}, V <= |g|. */
    WD_OPT_SPAN = 10,        /* S: windows one lane loads per round trip in the one-lane-per-
                                window mode (V = |g| <= 4, single-shard calls): the lane decides
                                on the first of the S windows holding a match or an empty slot
                                (Fig. 3 order), so results and layout do not depend on S.
                                0 (default): 2 for tables of <= 64 MB and for |g| = 1, else 1;
                                1: off; 2: on. */
    WD_OPT_SLICES = 11,      /* a bulk insert of device-resident pairs into a single-shard table
                                is grouped by table slice of the keys' first region (Line 5) and
                                inserted with one probe launch per slice (better L2 reuse); the
                                probing of each key is unchanged.  0 (default): for tables > 512 MB
                                (> 1 GB where the span read-ahead applies) and calls of
                                >= 2^26 pairs, the power of two that makes a slice <= 80 MB
                                for |g| = 16 on line-aligned tables (32 for config 2's
                                2.3 GB) or <= 160 MB otherwise, at most 128, and off when a
                                slice would exceed 300 MB (measured slower);
                                1: off; 2..128: that many slices.  Uses 8 B of scratch per pair,
                                two buffers of at most 2^28 pairs (grouping of the next chunk
                                overlaps the probing of this one), kept for the table's lifetime
                                (stream-ordered allocation); in auto mode a failed scratch
                                allocation falls back to the plain launch. */
    WD_OPT_EXCHANGE = 12,    /* how the transposition of P:117 (a8) and its reverse (a10) move
                                data between shards (m > 1):
                                0 (default): fused — the multisplit kernel stores every item
                                  straight into its owner's receive region and the owner's
                                  probe kernel stores every answer straight into its origin's
                                  result region (peer memory over NVLink, epoch flags, no
                                  host synchronisation);
                                1: staged + copy engine — local per-destination send buckets,
                                  then one cudaMemcpyAsync of the exact count per peer (the
                                  paper's asynchronous inter-GPU copies), results back
                                  the same way; the host reads its row of T per batch;
                                2: staged + NCCL — T all-gathered with ncclAllGather, then an
                                  all-to-all(v) of the exact counts as grouped ncclSend /
                                  ncclRecv (forward and reverse on two communicators).  Needs
                                  one GPU per shard (wd_create with n_gpus > 1, or rank mode;
                                  rank mode: set before wd_rank_handle).  NCCL is loaded at
                                  run time (libnccl.so.2).
                                Results are identical in all three modes. */
    WD_OPT_PHASE_TIMING = 13, /* 1: record CUDA events around every phase of every call (see
                                wd_phase_times); 0 (default): off */
    /* 14: reserved (a |g| = 32 launch for long probe chains was measured slower and removed,
       profiles/r02/tail_launch.md) */
    WD_OPT_AUTO_REBUILD = 15, /* P:63 "the whole data structure is invalidated followed by a
                                subsequent reconstruction with a distinct hash function":
                                1 = after an insert call that left keys behind (Line 26) while
                                live keys + those keys still fit the capacity (e.g. tombstones
                                fill the probe sequences), rebuild with a new seed and re-insert
                                them (up to 4 times).  Makes wd_insert synchronous; applies
                                to whole-table wd_insert calls (not the _sharded ones).  0
                                (default): off, the sticky WD_ERR_TABLE_FULL is reported.
                                Single-process tables only (not rank mode). */
    WD_OPT_QUERY_GROUP_SIZE = 16, /* |g| of wd_retrieve / wd_erase calls.  P:89: the probe
                                sequence, hence every result, is the same for any |g| (a key
                                sits at the leftmost empty slot of its sequence, so no empty
                                slot precedes it for any window size).  -1 (default): auto,
                                by region alignment and load: 16 (one 128-byte line) on A = 16
                                tables and above a projected load of 0.93, else 8.  Measured
                                on B200 (profiles/r02/sweep_r02o.jsonl, query_group.jsonl;
                                2^28 keys): alpha 0.95 hits on |g| = 1 / 2 / 4 / 32 tables
                                7.0 / 10.4 / 17.6 / 19.0 -> 24.2 / 24.2 / 24.3 / 26.6 G/s,
                                misses on |g| = 4 2.9 -> 7.9 G/s.  0: the table's |g| (the
                                paper's setting); else 1..32. */
    WD_OPT_INSERT_GROUP_SIZE = 17, /* |g| of wd_insert calls.  The slot an insert takes (the
                                leftmost empty slot of its sequence, or its key's slot) is the
                                same for any |g|, so the layout is too.  -1 (default):
                                auto, 16 on A = 16 tables and on shards of <= 64 MB, else 8
                                up to 24 GB shards and the table's |g| (at least 4) above
                                (tables created with |g| = 0 keep the choice by load).  Measured (2^28 keys,
                                alpha 0.95): |g| 1 / 2 / 4 / 32 tables 9.7 / 14.4 / 20.7 / 15.9
                                -> 22.1 / 22.1 / 22.1 / 23.5 G inserts/s.  0: the table's |g|
                                (the paper's setting); else 1..32. */
    WD_OPT_N_SHARDS = 100,   /* read-only: m */
    WD_OPT_RANK = 101,       /* read-only: this process's rank (0 unless rank mode) */
    WD_OPT_LOCAL_SHARDS = 102, /* read-only: shards owned by this process */
    WD_OPT_LAUNCHES = 103,   /* read-only: kernels launched by the library so far */
    WD_OPT_GROUP_SIZE_USED = 104, /* read-only: |g| used by the last call */
    WD_OPT_REGION_ALIGN = 105  /* read-only: A, region starts are multiples of A slots
                                  (reading C2'): 16 (one 128-byte line) when the table was
                                  created with group_size >= 16, else 4 (one sector); fixed
                                  for the table's life, so every |g| later used on it probes
                                  the same sequence */
} wd_option_t;

wd_status_t wd_set_option(wd_table_t* t, wd_option_t opt, int64_t value);
int64_t     wd_get_option(wd_table_t* t, wd_option_t opt);   /* INT64_MIN on error */

/* ------------------------------------------------------------------ phase timing --- */
/* The per-phase decomposition of Fig. 11.  With WD_OPT_PHASE_TIMING = 1 every
 * phase of every batch is bracketed by CUDA events on the stream it runs on; this call
 * synchronizes, writes the summed milliseconds (and the number of intervals) per phase
 * since the last call, and resets.  Phases on different streams overlap, so the sum is
 * not the wall time.  Indices: */
#define WD_PHASE_H2D 0         /* a11: host -> device copies of the input */
#define WD_PHASE_GROUP 1       /* slice grouping of a bulk insert (histogram, scan, multisplit) */
#define WD_PHASE_MULTISPLIT 2  /* a6 (fused mode: includes the transposition a8) */
#define WD_PHASE_EXCHANGE 3    /* a8 staged: copy engine / NCCL send+recv */
#define WD_PHASE_PROBE 4       /* a3 / a9 insert probe kernels */
#define WD_PHASE_REVERSE 5     /* a10 staged: results back to their origins */
#define WD_PHASE_UNPERMUTE 6   /* a10: gather into input order */
#define WD_PHASE_D2H 7         /* a11: device -> host copies of the results */
#define WD_PHASE_PROBE_QUERY 8 /* a4 / a9 retrieve / erase probe kernels (fused mode: includes
                                  a10's push of the answers) */
#define WD_N_PHASES 9
wd_status_t wd_phase_times(wd_table_t* t, double ms_out[WD_N_PHASES], uint64_t count_out[WD_N_PHASES]);

/* ------------------------------------------------------------------ diagnostics ---- */
wd_status_t wd_last_error(void);
const char* wd_error_string(wd_status_t s);
const char* wd_last_error_message(void);

/* Probe accounting under concurrency (SURVEY §8(d) "replaced by the measured values from the
 * WD_COUNT_PROBES build"): windows examined, distinct 128-byte lines touched, CAS attempts,
 * CAS lost to a concurrent insert, keys probed — summed since the last call over the probe
 * launches of local shard `shard`, then reset.  Synchronizes.  WD_ERR_UNSUPPORTED unless the
 * library was built with -DWD_COUNT_PROBES (a measurement build: tools/probe_counts.py). */
wd_status_t wd_probe_counts(wd_table_t* t, int shard, uint64_t out[5]);

/* slots of local shard `shard` (0-based among this process's shards) */
uint64_t    wd_shard_capacity(wd_table_t* t, int shard);
/* copy the raw 64-bit slots of a local shard to host memory (debug / layout tests);
 * word = key | (uint64_t)value << 32, empty = all ones.  Synchronizes. */
wd_status_t wd_dump(wd_table_t* t, int shard, uint64_t* host_out);
/* per-shard device counters: [0] new keys, [1] failed inserts, [2] reserved keys,
 * [3] exchange errors, [4] key of the most recent failed insert, [5] keys erased.
 * Synchronizes. */
wd_status_t wd_counters(wd_table_t* t, int shard, uint64_t out[6]);

#ifdef __cplusplus
}
#endif
#endif /* WARPDRIVE_H */
