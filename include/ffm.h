/*
 * ffm.h -- C ABI of the B200-native duplicate memory-transfer detector
 * (the transfer hot path of Diogenes' feed-forward measurement model,
 * Welton & Miller, SC'19; /root/reference/PAPER.md, cited as P:<line>).
 *
 * The operation (Sec. 3.3.2 "Identifying Problematic Memory
 * Transfers"): every recorded CPU<->GPU transfer payload is content-hashed and
 * compared with the stored hashes of prior transfers; a match -- confirmed
 * byte-by-byte here (reading R2) -- marks the transfer a duplicate of
 * "the first transfer of the duplicated data".  The expected benefit of
 * removing a duplicate is its transfer call's duration (Fig. 5
 * RemoveMemoryTransfer), summed per call site
 * ("single point" grouping).
 *
 *   duplicate_of[i] = gid of min{ j < i : size_j == size_i && bytes_j == bytes_i }, or -1
 *   benefit_ns[s]   = sum_{i : site_i == s, duplicate_of[i] >= 0} duration_ns_i   (mod 2^64)
 *
 * Every function returns FFM_OK (0) or a negative ffm_status unless stated.
 * No C++ exception crosses this boundary.  A handle is externally synchronised
 * (one thread at a time).  After a CUDA error the handle is poisoned: every
 * call except ffm_log_destroy / ffm_last_error returns FFM_E_STATE.
 */
#ifndef FFM_H
#define FFM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum ffm_status {
    FFM_OK = 0,
    FFM_E_INVAL = -1,   /* NULL handle/argument, bad config, NULL payload with size > 0 */
    FFM_E_RANGE = -2,   /* call_site >= n_sites; gids not strictly increasing */
    FFM_E_NOMEM = -3,   /* host or device allocation failed */
    FFM_E_CUDA  = -4,   /* a CUDA runtime call failed (handle is now poisoned) */
    FFM_E_COMM  = -5,   /* shard exchange inconsistent (multi-rank) */
    FFM_E_STATE = -6,   /* poisoned handle, or call out of order */
    FFM_E_NODEV = -7    /* no CUDA device / driver (there is no CPU fallback) */
} ffm_status;

/* Opaque, library-owned log handle. */
typedef struct ffm_log ffm_log;

/* payload_kind for ffm_log_append_batch */
enum { FFM_PAYLOAD_AUTO = 0,        /* detected per pointer (cudaPointerGetAttributes) */
       FFM_PAYLOAD_HOST = 1,        /* pageable host memory: copied through a pinned staging ring */
       FFM_PAYLOAD_DEVICE = 2,      /* device memory on cfg->device: gathered by a kernel / D2D */
       FFM_PAYLOAD_HOST_PINNED = 3  /* page-locked (cudaHostAlloc / cudaHostRegister) host memory:
                                       read over PCIe by the gather kernel or the copy engines */ };

/* ffm_config.flags */
enum { FFM_FLAG_TIMING = 1u,     /* record per-stage CUDA events (ffm_last_run_stats); such runs
                                    launch their kernels directly (no graph replay) */
       FFM_FLAG_PREFILTER = 2u,  /* S8(f) #4: ffm_dedup_run hashes only the first chunk of a large
                                    payload whose (size, first-chunk digest, channel) is unique in the
                                    log -- it cannot equal any other payload.  Same results, fewer bytes.
                                    Ignored by ffm_shard_* and ffm_online_step (uniqueness within one
                                    shard / window says nothing about the others). */
       FFM_FLAG_TWO_PASS = 4u,   /* round 0 of H1-H3 as two passes: hash every payload fully, group by
                                    the full digest, then byte-verify members (chunk-major per class).
                                    Default is fused: group large payloads by their first chunk and hash
                                    + compare in one pass -- fewer bytes when duplicates are exact, more
                                    when most candidates are near-duplicates (BASELINE config 3).  Same
                                    results either way.  With neither flag the mode is adaptive: a log
                                    whose fused run found more than half of its candidates to mismatch
                                    uses two-pass on later runs. */
       FFM_FLAG_FUSED = 8u,      /* force the fused round 0 (no adaptation) */
       FFM_FLAG_NO_GRAPH = 16u,  /* launch every kernel directly instead of replaying the captured
                                    CUDA graph of a run (default: graph while the log is unchanged) */
       FFM_FLAG_ONLINE = 32u,    /* online mode (S8(f) #2): every append uploads its records' metadata
                                    right away (staging stream), so ffm_online_step starts from a
                                    device-resident window; the step runs the fused round 0 on its
                                    window (each byte read once) */
       FFM_FLAG_APPEND_HASH = 64u /* with FFM_FLAG_ONLINE: every append also hashes its records on a
                                    hashing stream that follows the staging copies (the next
                                    append's staging overlaps it); the step then groups by the full
                                    digests and re-reads the members to verify them (two-pass) */ };

/* Caller-provided exchange transport of a sharded log (world > 1), used instead of the
   library's own NCCL communicator when NCCL cannot connect the ranks (e.g. several ranks
   sharing one GPU in tests).  Both functions are collective over the world, take HOST
   buffers and return 0 on success (anything else fails the run with FFM_E_COMM).
     allgather:     recv[world * bytes] = every rank's send[bytes], rank-major
     allreduce_u64: buf[n] = elementwise sum over ranks, mod 2^64, in place
   The struct is copied at ffm_log_create; ctx and the functions must stay valid until
   ffm_log_destroy. */
typedef struct ffm_comm_ops {
    void* ctx;
    int (*allgather)(void* ctx, const void* send, void* recv, uint64_t bytes);
    int (*allreduce_u64)(void* ctx, uint64_t* buf, uint64_t n);
} ffm_comm_ops;

typedef struct ffm_config {
    uint32_t n_sites;      /* call_site must be < n_sites.  Sites are caller-interned stack
                              traces, matched by instruction address. */
    int32_t  device;       /* CUDA ordinal this log lives on */
    int32_t  rank, world;  /* shard id / count; 0, 1 for one GPU.  world > 1 makes ffm_log_create
                              and ffm_dedup_run collective (see "Sharded logs" below) */
    uint64_t arena_bytes;  /* initial HBM payload arena capacity (bytes); grows x2 on demand */
    uint64_t max_records;  /* initial record capacity hint; grows on demand (within it the host
                              copy of the metadata is page-locked: its uploads are async DMA) */
    uint32_t digest_bits;  /* 64 normally.  < 64 truncates the group-by digest to FORCE
                              collisions (test / verify-stress knob, BASELINE config 3);
                              results never change.  0 => group by size alone. */
    uint32_t refine_bits;  /* 64 normally; < 64 weakens the first collision-resolution
                              re-key (test knob for the worst-case resolve path). */
    uint32_t chunk_bytes;  /* large-payload work unit, multiple of 1024; 0 => 32768.
                              Results never change. */
    uint32_t small_bytes;  /* payloads <= this are hashed/verified one per 8-lane group;
                              multiple of 128; 0 => 4096.  Results never change. */
    uint32_t flags;        /* FFM_FLAG_* */
    uint32_t reserved0;
    void*    stream;       /* cudaStream_t to run on, or NULL: the log creates its own */
    const void* nccl_id;   /* world > 1: the 128-byte ncclUniqueId of the world (ffm_nccl_unique_id on
                              one rank, broadcast by the caller); the log owns the communicator.
                              Also allowed with world == 1: a world of one runs the collective
                              path (NCCL included) on its own */
    const ffm_comm_ops* comm;  /* instead of nccl_id: caller transport (copied) */
} ffm_config;

/* Fill *cfg with defaults: n_sites 1, device 0, rank 0, world 1, digest_bits 64,
   refine_bits 64, everything else 0 / NULL. */
void ffm_config_init(ffm_config* cfg);

/* Create a log on cfg->device.  *out is owned by the library until ffm_log_destroy.
   With world > 1 this is collective: every rank calls it with the same nccl_id (the
   library's NCCL communicator is created here) or with its comm transport.
   Errors: FFM_E_INVAL (NULL, n_sites == 0, bad chunk/small bytes, digest_bits > 64,
   world > 1 without exactly one of nccl_id / comm), FFM_E_NODEV, FFM_E_NOMEM, FFM_E_CUDA,
   FFM_E_COMM (NCCL unavailable or its init failed). */
int ffm_log_create(const ffm_config* cfg, ffm_log** out);

/* Append one transfer record (the intercepted call's payload location
   and size; its call site and time in the driver call).
   gid = the record's local append index (program order).
   payload_ptr is BORROWED for the call: the bytes as of this call are snapshotted
   into HBM before return (reading R11; PAPER.md P:1459-1463 shows bytes may change
   later), so the caller may reuse the buffer afterwards.  Host (pageable or pinned)
   or device pointers are accepted (detected with cudaPointerGetAttributes).
   payload_ptr may be NULL only if size == 0.  A failed append leaves the log
   unchanged.  Errors: FFM_E_INVAL, FFM_E_RANGE (call_site >= n_sites), FFM_E_NOMEM,
   FFM_E_CUDA, FFM_E_STATE. */
int ffm_log_append(ffm_log* log, uint32_t call_site, uint64_t size,
                   const void* payload_ptr, uint64_t duration_ns);

/* Append n records at once (host arrays of length n).  payloads[i] follows the
   rules of ffm_log_append; payload_kind says whether they are all HOST, all DEVICE,
   or AUTO (detected per pointer).  gids may be NULL (local append order) or give
   each record's GLOBAL gid, strictly increasing across all appends to this log and
   < 2^63 (sharded logs: records of one global program order split over ranks; there
   gids are REQUIRED -- every rank numbering from 0 would repeat gids across ranks).
   A device payload on another GPU is copied by the copy engines (cudaMemcpyDefault).
   Device payloads are read on the library's staging stream after it waits on the log's
   stream (cfg->stream) and on the legacy default stream; a producer on any other stream
   must synchronize before the append.
   All-or-nothing: on error the log is unchanged.  Errors as ffm_log_append, plus
   FFM_E_RANGE (gids not increasing, or >= 2^63), FFM_E_INVAL (world > 1 and gids NULL). */
int ffm_log_append_batch(ffm_log* log, uint64_t n, const uint32_t* call_sites,
                         const uint64_t* sizes, const void* const* payloads,
                         const uint64_t* durations_ns, const uint64_t* gids,
                         int payload_kind);

/* ffm_log_append_batch with an optional per-record channel id (S8(f) #3, the
   destination-aware variant: "retransfer the same data to the same destination",
   P:1194-1197; direction "to and from the GPU").  A record then
   duplicates only an earlier record with equal size, bytes AND channel.  channels
   NULL (or all equal) is the content-only reading R5. */
int ffm_log_append_batch_ex(ffm_log* log, uint64_t n, const uint32_t* call_sites,
                            const uint64_t* sizes, const void* const* payloads,
                            const uint64_t* durations_ns, const uint64_t* gids,
                            const uint64_t* channels, int payload_kind);

/* Run the hot path over the whole log (H1 hash, H2 group-by, H3 verify,
   H4 collision resolve, H5 label, H6 per-site benefit, H7 return):
     duplicate_of[n_local]  int64  gid of the earliest byte-identical record, or -1
     benefit_ns[n_sites]    uint64 per-site sum of duplicate durations
   Either array may be host or device memory (caller-owned; device arrays must be
   on cfg->device).  benefit_ns may be NULL.  Idempotent: re-running over an
   unchanged log gives identical outputs; appends after a run are allowed.
   Synchronous: returns when the outputs are written.
   world > 1: COLLECTIVE -- every rank calls it; duplicate_of[n_local] receives GLOBAL
   gids (the earliest byte-identical record on any rank) and benefit_ns the global
   per-site sums, identical on every rank (see "Sharded logs"). */
int ffm_dedup_run(ffm_log* log, int64_t* duplicate_of, uint64_t* benefit_ns);

/* Number of records appended (local) / payload bytes appended. */
uint64_t ffm_log_count(const ffm_log* log);
uint64_t ffm_log_payload_bytes(const ffm_log* log);

/* The cudaStream_t the log runs its kernels on (for CUDA-event timing). */
void* ffm_log_stream(const ffm_log* log);

typedef struct ffm_run_stats {
    double   ms_total;          /* CUDA-event time of the last run (FFM_FLAG_TIMING) */
    double   ms_hash;           /* H1: hash kernels */
    double   ms_group;          /* H2: table insert + leader lookup */
    double   ms_verify;         /* H3: verify planning + verify kernels */
    double   ms_resolve;        /* H4: collision-resolution rounds */
    double   ms_label;          /* H5+H6: label + benefit */
    double   ms_output;         /* H7: output copies */
    double   ms_hash_large;     /* the large-payload prefix-pass kernel alone (first chunks) */
    double   ms_hash_small;     /* the small-payload hash kernel alone */
    uint64_t n_records;
    uint64_t payload_bytes;     /* sum of sizes */
    uint64_t n_members;         /* records whose group candidate is an earlier record */
    uint64_t n_residual;        /* members that failed byte verification (collisions) */
    uint64_t resolve_rounds;
    uint64_t kernel_launches;   /* kernels this library launched in the last run */
    uint64_t hash_items;        /* large-payload hash work units */
    uint64_t verify_items;      /* large-payload verify work units */
    uint64_t prefilter_rest_bytes; /* bytes hashed beyond first chunks by the fused pass */
    double   ms_fused;          /* the fused hash + compare kernel alone (large payloads) */
    uint64_t two_pass;          /* 1 if the last run used the two-pass round 0 */
    uint64_t n_reread;          /* residual members whose bytes were compared again; after a fused
                                   round 0 the others are settled exactly through their difference
                                   lists against the group head */
    /* sharded runs (world > 1); 0 otherwise */
    uint64_t n_reps_local;      /* exact local classes exported by this rank */
    uint64_t n_reps_global;     /* representatives of all ranks */
    uint64_t exchange_bytes;    /* bytes this rank received through the collectives of the run */
    uint64_t remote_verify_bytes; /* B_x: payload bytes this rank compared against peer arenas over
                                   NVLink */
    uint64_t n_slow;            /* representatives resolved by the same-key segment scan */
    uint64_t host_syncs;        /* host synchronisations of the run's stream */
    double   ms_exchange;       /* CUDA-event time from the end of the local pass to the outputs */
} ffm_run_stats;

/* Statistics of the last ffm_dedup_run. */
int ffm_last_run_stats(const ffm_log* log, ffm_run_stats* out);

/* Number of duplicates per call site in the last run ("Number of Transfer Issues",
   Fig. 6), [n_sites] uint64, host or device.  For a sharded log these are
   the global counts (all-reduced with the benefit). */
int ffm_site_duplicate_counts(ffm_log* log, uint64_t* counts_out);

/* Folded grouping: group_values_out[g] = sum of site_values[s] over the
   sites s with site_to_group[s] == g (uint64, mod 2^64), computed by a kernel on the
   log's device.  site_values [n_sites] and site_to_group [n_sites] (host or device),
   group_values_out [n_groups] (host or device).  The caller builds site_to_group by
   folding each site's stack-trace function name: demangled, template parameters
   discarded (paper_conf_sc_weltonm19_b200/report.py).  Errors: FFM_E_INVAL,
   FFM_E_RANGE (a group id >= n_groups). */
int ffm_fold_sites(ffm_log* log, const uint64_t* site_values, const uint32_t* site_to_group, uint32_t n_groups,
                   uint64_t* group_values_out);

/* ---------------------------------------------------------------------------
 * Online (streaming) mode -- the paper's per-call semantics: each new
 * transfer is "hashed and then compared to the stored hashes from prior transfers".
 * The stored hashes are a persistent, insert-only device table of every exact class
 * seen so far (key of the full digest, size and channel -> the classes' representatives,
 * whose bytes stay in the HBM arena).  ffm_online_step labels every record appended since
 * the previous step (a window): H1..H4 on the window alone -- by default the batch run's
 * fused round 0 on the window in its batch record order (built on the device: every byte
 * read once, leaders hashed, members compared); with FFM_FLAG_APPEND_HASH the appends hash
 * their records and the step verifies two-pass -- then each window class looks its key up
 * in the table and is byte-verified against the stored classes there; classes with no
 * equal stored class are inserted.  A window of <= 8 small records is labelled by one warp,
 * record by record in gid order, directly against the table (one launch per step).  A step's work is O(window), never O(prior records) (the table is
 * rehashed only when its capacity doubles).  Labels of earlier records never change, so
 * the concatenated windows equal ffm_dedup_run over the whole log, bit for bit.
 *   duplicate_of [window records] (host or device): gids, or -1
 *   benefit_ns   [n_sites] (may be NULL): cumulative per-site benefit so far
 *   *n_window    (may be NULL): records labelled by this step
 * Single-log only (world == 1). */
int ffm_online_step(ffm_log* log, int64_t* duplicate_of, uint64_t* benefit_ns, uint64_t* n_window);

/* Records labelled by online steps so far. */
uint64_t ffm_online_done(const ffm_log* log);

/* Debug / conformance: copy the last run's 64-bit payload digests (host array [n]).
   The digest is specified in DESIGN.md "Digest"; it is an implementation detail
   and never part of the result. */
int ffm_debug_digests(ffm_log* log, uint64_t* digests_out);

/* ---------------------------------------------------------------------------
 * Sharded logs (world > 1).  One process per GPU; the
 * caller assigns records to ranks (ffm_shard_plan) and appends each rank's records with
 * their GLOBAL gids.  Exact byte equality is transitive, so per-rank results merge
 * through one exchange of class representatives.  ffm_dedup_run on every rank:
 *   1. H1..H4 on this rank's records -> exact local classes, one representative each
 *      (key of the full digest, size, gid, arena offset, channel);
 *   2. all-gather of the representatives (NCCL over NVLink / NVSwitch on the log's
 *      stream, or the caller's ffm_comm_ops);
 *   3. every rank builds the same global group-by over all representatives; a rank's
 *      representative whose candidate lives on another rank is byte-verified by a
 *      kernel that loads the candidate's bytes straight from the peer GPU's arena
 *      (CUDA-IPC mapping, exchanged by the library whenever an arena was reallocated);
 *      digest collisions take a scan of the key's segment;
 *   4. labels (global gids), per-site partial sums, and an all-reduce of the sums.
 * Two host synchronisations per run when no rank has digest collisions.  When the run
 * returns, no peer reads this rank's arena any more (the all-reduce orders every rank's
 * compare kernels before it), so appends / reset may follow.
 * ------------------------------------------------------------------------- */

/* The 128-byte ncclUniqueId for a new world (call on one rank, broadcast it).
   Errors: FFM_E_INVAL (NULL), FFM_E_COMM (libnccl.so.2 unavailable). */
int ffm_nccl_unique_id(void* id_out);

enum { FFM_SHARD_SITE_LPT = 0,     /* whole call sites, bin-packed by bytes (largest first) */
       FFM_SHARD_CONTIGUOUS = 1 }; /* contiguous gid ranges of ~equal bytes */

/* Host-only shard planner: rank_out[i] in [0, world) for each of n records.
   SITE_LPT keeps every re-upload of a call site (the dominant duplicate pattern,
   P:1194-1197) on one rank.  Errors: FFM_E_INVAL, FFM_E_RANGE (site >= n_sites). */
int ffm_shard_plan(uint64_t n, const uint32_t* call_sites, const uint64_t* sizes, uint32_t n_sites,
                   int32_t world, int policy, int32_t* rank_out);

/* Replace cfg.flags of a live log (e.g. toggle FFM_FLAG_TIMING between measured and
   instrumented runs).  Takes effect at the next run. */
int ffm_log_set_flags(ffm_log* log, uint32_t flags);

/* Empty the log (records, online state) but keep every allocation (HBM arena, work
   buffers, staging ring): the next batch of transfers reuses them. */
int ffm_log_reset(ffm_log* log);

/* Destroy the log and release its memory.  NULL is a no-op (returns FFM_OK). */
int ffm_log_destroy(ffm_log* log);

/* Static text for a status code. */
const char* ffm_strerror(int status);

/* Detail of the last error on this handle (including CUDA error text); "" if none.
   Valid until the next call on the handle. */
const char* ffm_last_error(const ffm_log* log);

/* Library build identification, e.g. "ffm 0.1 sm_100a". */
const char* ffm_version(void);

#ifdef __cplusplus
}
#endif

#endif /* FFM_H */
