// ffm_internal.h -- internal structures of libffm (product path).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/ffm.h"
#include "ffm_comm.h"

namespace ffm {

constexpr uint32_t kArenaAlign = 32;         // record slots in the HBM arena (consecutive small records are contiguous)
constexpr uint64_t kEmptyKey = ~0ull;         // group-by table: empty slot
constexpr uint32_t kNoRecord = 0xFFFFFFFFu;
constexpr uint32_t kDiffK = 4;                // difference-list entries kept per large member

// Device-side views handed to the kernel launchers.
struct DevLog {
    const uint8_t* arena;
    const uint64_t* off;     // [n] arena offset of record i (32-B aligned)
    const uint64_t* size;    // [n]
    const uint32_t* site;    // [n]
    const uint64_t* dur;     // [n]
    const uint64_t* gid;     // [n]
    const uint64_t* chan;    // [n] channel (direction / destination) id, 0 = content only
    uint32_t n;
    const uint32_t* small_order;  // records <= small_bytes, sorted by block count (descending)
    const uint32_t* order_pos;    // inverse of small_order (+ large_order): position of record r
    uint32_t n_small;
    const uint32_t* large_order;  // records > small_bytes, ascending
    uint32_t n_large;
};

// Scratch of one run (grown on demand, reused across runs).
struct Work {
    uint64_t* accA = nullptr;      // [n] NH accumulator A
    uint64_t* accB = nullptr;      // [n] NH accumulator B
    uint64_t* key = nullptr;       // [n] group key (chained through resolve rounds)
    uint64_t* digest = nullptr;    // [n] 64-bit digest (debug / conformance)
    uint32_t* slot = nullptr;      // [n] table slot
    uint32_t* leader = nullptr;    // [n] local index of the candidate / final leader
    uint32_t* eq = nullptr;        // [n] 1 = verified equal so far (members)
    uint64_t* mis = nullptr;       // [n] first mismatching 16-B word vs leader
    uint32_t* res[2] = {nullptr, nullptr};  // residual lists (double buffer)
    uint32_t* lcount = nullptr;    // [n+1] per-leader verify chunk counts
    uint32_t* lstart = nullptr;    // [n+1] exclusive scan of lcount: group base of each leader
    uint32_t* gcount = nullptr;    // [n+1] large members per leader (chunk-major stride)
    uint32_t* pos = nullptr;       // [n] position of a large record within its fused / verify group
    uint32_t* fhead = nullptr;     // [n] round 0: head (leader) of a large record's fused group
    uint2* hitems = nullptr;       // large-payload hash work units (record, chunk)
    uint4* sdesc = nullptr;        // [2 * n] fused round 0: compare descriptors of small records (order position)
    uint4* fitems = nullptr;       // pipelined fused pass stage descriptors (2 x uint4 each)
    uint32_t* dcnt = nullptr;      // [n] fused round 0: words where a large member differs from its group head
    uint32_t* dq = nullptr;        // [n * kDiffK] their 16-B word indices (the first kDiffK recorded)
    uint4* dv = nullptr;           // [n * kDiffK] the member's values of those words
    uint32_t* hcount = nullptr;    // [n+1] per-record hash chunk counts
    uint32_t* hstart = nullptr;    // [n+1] exclusive scan of hcount
    uint64_t* hpart = nullptr;     // [2 * hitem_cap] per-unit partial NH sums (A, B)
    uint64_t* tkey = nullptr;      // [cap] group-by table: (32-bit key fingerprint << 32 | min local index)
    int64_t* dup = nullptr;        // [n] output staging
    uint64_t* ben = nullptr;       // [n_sites]
    uint64_t* label_part = nullptr; // [label_hist_rows * n_sites] per-block benefit partials
    uint32_t* label_cpart = nullptr; // [label_hist_rows * n_sites] per-block duplicate counts
    uint64_t* cnt = nullptr;       // [n_sites] duplicates per site (last run)
    uint32_t* counters = nullptr;  // device counters: [0] nres, [1] n_members, [2..] misc
    void* cub_tmp = nullptr;
    size_t cub_tmp_bytes = 0;
    uint64_t n_cap = 0, t_cap = 0, hitem_cap = 0, vitem_cap = 0, site_cap = 0, fitem_cap = 0;
};

// A pageable payload (or a piece of one) to stage: source, arena offset (or offset in a
// ring half), bytes.
struct PageablePiece {
    const uint8_t* src;
    uint64_t off, size;
};

// One representative per exact local class, exported for the cross-shard merge.
struct RepTuple {
    uint64_t key;    // group key of the full digest (same function on every rank)
    uint64_t size;
    uint64_t gid;    // global gid of the class's first local record
    uint64_t off;    // arena offset on the owning rank
    uint64_t chan;   // channel id (destination-aware variant), 0 = content only
    uint64_t dig;    // full 64-bit digest (prunes the slow path; a function of the bytes)
};

struct ShardWork {
    uint32_t* flag = nullptr;        // [n+1]
    uint32_t* rep_idx = nullptr;     // [n+1] exclusive scan of flag: tuple index of each local rep
    uint64_t* tkey = nullptr;        // [cap] global table over all representatives
    uint64_t* tgid = nullptr;        // [cap]
    uint32_t* tidx = nullptr;        // [cap]
    uint32_t* need = nullptr;        // [cap] slow path: key has a slow representative (zero between runs)
    uint32_t* scnt = nullptr;        // [cap] its segment length (zero between runs)
    uint32_t* sbase = nullptr;       // [cap] its segment start
    uint32_t* sfill = nullptr;       // [cap]
    uint32_t* tslot = nullptr;       // [M]
    uint32_t* seg = nullptr;         // [M] tuple indices, grouped by key segment
    uint32_t* state = nullptr;       // [nloc]
    uint32_t* cand = nullptr;        // [nloc]
    uint32_t* vcount = nullptr;      // [nloc+1]
    uint32_t* vstart = nullptr;      // [nloc+1]
    uint64_t* G = nullptr;           // [nloc] global leader gid of each local representative
    uint32_t* slow_list = nullptr;   // [nloc]
    uint2* vitems = nullptr;         // merge verify work units
    uint32_t* rank_lo = nullptr;     // [world] first tuple index of each rank
    const uint8_t** bases = nullptr; // [world] arena base of each rank (peer ones IPC-mapped)
    unsigned long long* sctr = nullptr;  // [4] n_slow, segment cursor, remote verify bytes (B_x)
    uint64_t n_cap = 0, m_cap = 0, t_cap = 0, l_cap = 0, v_cap = 0, w_cap = 0;
};

// Online mode: stored class representatives (insert-only pool) and the table over them.
struct OnlineRep {
    uint64_t gid, off, size, chan, dig;   // dig: full 64-bit digest
    uint32_t next, pad;                   // chain of the key (kNoRep-terminated)
};

struct OnlineTable {
    uint64_t* key = nullptr;     // [mask + 1] group key, kEmptyKey = free
    uint32_t* head = nullptr;    // [mask + 1] first pool entry of the key's chain
    OnlineRep* pool = nullptr;   // [pool_cap]
    uint32_t* count = nullptr;   // device: pool entries used
    uint64_t mask = 0;
};

// The metadata of an online window, gathered into fixed buffers (so that the captured
// step of a window replays for the next window of the same size).
struct WinMeta {
    uint64_t* off = nullptr;
    uint64_t* size = nullptr;
    uint64_t* dur = nullptr;
    uint64_t* gid = nullptr;
    uint64_t* chan = nullptr;
    uint32_t* site = nullptr;
};

struct Params {
    uint64_t digest_mask;
    uint64_t refine_mask;
    uint32_t chunk_bytes;
    uint32_t small_bytes;
    int num_sms;
    int max_smem;      // opt-in dynamic shared memory per block (bytes)
    uint32_t prefix_bytes;  // fused round 0: large payloads are grouped by the NH of their first prefix_bytes
};

// ---- kernel launchers (kernels.cu).  All asynchronous on `st`; each returns the
// number of kernels it launched (for the launch count), or -1 on launch error.
int launch_hash_small(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_fused_small(const DevLog& L, Work& W, const Params& P, uint32_t* res_out, cudaStream_t st);
int launch_hash_plan(const DevLog& L, Work& W, const Params& P, bool units, cudaStream_t st);
int launch_hash_large(const DevLog& L, Work& W, const Params& P, uint64_t n_items, cudaStream_t st);
int launch_prefix(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_combine(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_fused(const DevLog& L, Work& W, const Params& P, uint64_t n_units, bool prefilter, uint32_t* res_out,
                 cudaStream_t st, cudaEvent_t ev_a, cudaEvent_t ev_b);
// round 0 with label_sites != 0 (label_fused_ok): the leader lookup also writes the
// speculative labels (label_dup, if non-null) and the per-site sums (W.ben / W.cnt)
int launch_group(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                 uint64_t cap, int round, uint32_t* res_out, cudaStream_t st, bool use_diff = false,
                 uint32_t label_sites = 0, int64_t* label_dup = nullptr);
bool label_fused_ok(const Work& W, const Params& P, uint32_t n_sites);
int launch_verify(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                  uint32_t* res_out, uint64_t vitem_cap, cudaStream_t st, cudaStream_t side, cudaEvent_t ev_fork,
                  cudaEvent_t ev_join);
int launch_label(const DevLog& L, Work& W, const Params& P, uint32_t n_sites, int64_t* dup_out, cudaStream_t st);
size_t label_smem_bytes(uint32_t n_sites);
int launch_fold(const uint64_t* site_vals, const uint32_t* site_to_group, uint32_t n_sites, uint64_t* group_vals,
                uint32_t n_groups, cudaStream_t st);
uint32_t label_hist_rows(int num_sms);
int launch_site_reduce(const uint64_t* part, const uint32_t* cpart, uint32_t rows, uint32_t n_sites, uint64_t* ben,
                       uint64_t* cnt, cudaStream_t st);
// shard.cu
int launch_rep_export(const DevLog& L, Work& W, ShardWork& S, const Params& P, RepTuple* out, cudaStream_t st);
int launch_merge(const DevLog& L, Work& W, ShardWork& S, const Params& P, const RepTuple* T, uint32_t M,
                 uint32_t lo, uint32_t nloc, int world, int rank, uint64_t cap, cudaStream_t st);
// online.cu
int launch_online_rehash(OnlineTable& T, uint32_t np, uint64_t digest_mask, cudaStream_t st);
int launch_online_window(const DevLog& L, const Work& W, const uint64_t* accA, const uint64_t* accB,
                         OnlineTable& T, const Params& P, uint32_t n_sites, uint64_t* G, int64_t* dup_out,
                         uint64_t* ben, uint64_t* cnt, cudaStream_t st);
// tiny windows: one warp labels the records in order against the table (ffm_online_step)
constexpr uint32_t kTinyWindow = 8;
int launch_online_tiny(const DevLog& L, OnlineTable& T, const Params& P, int64_t* dup_out, uint64_t* ben,
                       uint64_t* cnt, cudaStream_t st);
int launch_online_fix(const DevLog& L, const Work& W, const uint64_t* accA, const uint64_t* accB, OnlineTable& T,
                      const Params& P, const uint32_t* list, uint32_t n_list, uint64_t* G, int64_t* dup_out,
                      uint64_t* ben, uint64_t* cnt, cudaStream_t st);
int launch_merge_label(const DevLog& L, Work& W, ShardWork& S, const Params& P, uint32_t n_sites, int64_t* dup_out,
                       cudaStream_t st);
int launch_shard_header(const uint32_t* rep_count, const uint32_t* counters, uint64_t gen, uint64_t n,
                        uint64_t* hdr, cudaStream_t st);
int launch_gather(const uint64_t* d_desc, uint32_t n, uint8_t* arena, cudaStream_t st);
int launch_zero_counters(Work& W, cudaStream_t st);
int launch_invert(const uint32_t* order, uint32_t n, uint32_t* inv, cudaStream_t st);
// The window [*d_a, *d_a + n) of the log L: its metadata gathered into wm, and its batch
// record order (small records grouped by 32-byte block count, largest first; then the
// large ones) and inverse.  bins: [3 * window_bins(small_bytes)] words, zero between calls.
__host__ __device__ uint32_t window_bins(uint32_t small_bytes);
int launch_window_order(const DevLog& L, const uint64_t* d_a, uint32_t n, const WinMeta& wm, uint32_t small_bytes,
                        uint32_t* bins, uint32_t* order, uint32_t* inv, cudaStream_t st);
int launch_iota(uint32_t* a, uint32_t n, cudaStream_t st);
int launch_spec_label(const DevLog& L, Work& W, int64_t* dup_out, cudaStream_t st);
int launch_digest_fill(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_hash_small_list(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                           cudaStream_t st);
size_t cub_scan_bytes(uint64_t n);
uint64_t fx_entry_cap(uint64_t n_large_chunks, uint32_t chunk_bytes);
uint32_t blocks_for(uint64_t threads, uint32_t bs = 256);
uint32_t resident_grid(const void* kernel, int num_sms, int block = 256);
bool smem_configured(const void* kernel, int bytes);

}  // namespace ffm

// What a captured run graph depends on.
struct GraphKey {
    uint64_t epoch = ~0ull;
    const void* dup = nullptr;
    const void* hdup = nullptr;   // pinned host duplicate_of of the speculative D2H (or null)
    bool two_pass = false, prefilter = false, timing = false;
    static constexpr int kExtra = 6;
    uint64_t extra[kExtra] = {0, 0, 0, 0, 0, 0};   // online windows: what else the captured step depends on
    bool operator==(const GraphKey& o) const {
        bool same = epoch == o.epoch && dup == o.dup && hdup == o.hdup && two_pass == o.two_pass &&
                    prefilter == o.prefilter && timing == o.timing;
        for (int i = 0; i < kExtra; ++i) same = same && extra[i] == o.extra[i];
        return same;
    }
};

// A captured CUDA graph and what it was captured for.
struct GraphSlot {
    cudaGraphExec_t exec = nullptr;
    GraphKey key;
    uint64_t launches = 0;
};


// The opaque handle.
struct ffm_log {
    ffm_config cfg{};
    int device = 0;
    cudaStream_t stream = nullptr;
    cudaStream_t stage_stream = nullptr;
    cudaStream_t side_stream = nullptr;   // small-payload kernels run concurrently here
    cudaStream_t hash_stream = nullptr;   // append-time hashing (online mode)
    cudaStream_t copy_stream = nullptr;   // speculative D2H of duplicate_of during H3
    cudaEvent_t copy_ev[2] = {};
    cudaEvent_t hash_ev = nullptr;        // the last append-time hashing
    cudaEvent_t fork_ev[4] = {};
    bool own_stream = false;
    bool poisoned = false;
    bool host_ptr_ok = false;      // kernels may dereference registered host pointers
    bool prefer_two_pass = false;  // adaptive round 0 (see run_local)
    uint64_t epoch = 0;            // bumped whenever records or device buffers change
    GraphSlot graph;           // captured run segment A (see run_local)
    GraphSlot wgraph;          // captured online window step (fused windows)
    uint64_t bufgen = 0;            // bumped whenever a device buffer a captured graph uses moves
    uint64_t gather_max = 0;       // payloads up to this are gathered by k_gather, above: DMA
    std::string last_error;

    // host metadata (authoritative), program order
    std::vector<uint32_t> h_site;
    std::vector<uint64_t> h_size, h_off, h_dur, h_gid, h_chan;
    uint64_t payload_bytes = 0;
    uint64_t n_large_chunks = 0;   // sum over size > small of ceil(size / chunk)
    uint64_t last_gid = 0;
    bool any_gid = false;

    // device metadata mirrors
    uint64_t* d_off = nullptr;
    uint64_t* d_size = nullptr;
    uint32_t* d_site = nullptr;
    uint64_t* d_dur = nullptr;
    uint64_t* d_gid = nullptr;
    uint64_t* d_chan = nullptr;
    uint64_t d_meta_cap = 0;       // records
    uint64_t d_meta_n = 0;         // records uploaded
    uint64_t d_order_n = 0;        // records covered by d_small_order
    uint32_t* d_small_order = nullptr;   // small records by size class (built at upload)
    uint64_t d_small_cap = 0, n_small = 0, n_large_rec = 0;

    // HBM arena
    uint8_t* arena = nullptr;
    uint64_t arena_cap = 0, arena_used = 0;

    // pinned staging ring for host payloads
    uint8_t* ring[2] = {nullptr, nullptr};
    cudaEvent_t ring_ev[2] = {nullptr, nullptr};
    uint64_t ring_bytes = 0;
    int ring_cur = 0;
    uint64_t ring_arena_start = 0;  // arena offset corresponding to ring[cur][0]
    uint64_t ring_fill = 0;         // bytes used in ring[cur]
    bool ring_pending = false;
    std::vector<ffm::PageablePiece> stage_jobs;   // copy jobs of one ring window (reused)

    // sharded runs (world > 1, or a transport given: collective ffm_dedup_run)
    bool collective = false;
    ffm::Comm comm;
    ffm::ShardWork shard;
    uint64_t arena_gen = 0;         // bumped whenever the arena is reallocated (peers re-map it)
    std::vector<uint64_t> xgen;     // every rank's arena generation at the last handle exchange
    std::vector<uint8_t> xhandles;  // the IPC handles of that exchange (64 B per rank)
    std::vector<uint64_t> peer_gen; // generation of each mapped peer arena
    std::vector<void*> peer_ptr;    // IPC-mapped peer arenas (index = rank)
    ffm::RepTuple* d_send = nullptr;   // this rank's representatives (padded to the max count)
    ffm::RepTuple* d_recv = nullptr;   // all-gathered, world x max count
    ffm::RepTuple* d_T = nullptr;      // compacted, rank-major
    uint64_t send_cap = 0, recv_cap = 0, T_cap = 0;
    uint64_t* d_hdr = nullptr;         // [4] this rank's header; [4 + 4 * world] all headers
    uint8_t* d_ipc = nullptr;          // [64 * (world + 1)] IPC handle exchange
    uint64_t* h_hdr = nullptr;         // pinned mirror of all headers (+ run counters)

    // online (streaming) mode: the persistent table of every class seen so far
    uint64_t online_done = 0;        // records already labelled online
    uint64_t online_hashed = 0;      // records whose NH sums are in on_A / on_B
    ffm::OnlineTable otab;
    uint64_t online_np = 0;          // stored representatives (read back after each step)
    uint64_t pool_cap = 0;
    uint64_t* on_A = nullptr;        // [records] NH sums (global record index)
    uint64_t* on_B = nullptr;
    uint64_t on_cap = 0;
    uint64_t* on_G = nullptr;        // [window] global leader gid of each window class
    uint32_t* on_res = nullptr;      // [window] the step's round-0 residuals (speculative labels fix-up)
    uint64_t on_G_cap = 0;
    uint64_t* online_ben = nullptr;  // [2 * n_sites] cumulative per-site benefit | duplicate counts
    uint64_t* online_cnt = nullptr;  //   (= online_ben + n_sites)
    uint32_t* d_iota = nullptr;      // identity record order of online windows (0, 1, 2, ...)
    uint64_t iota_cap = 0;
    // fused online windows: the window's batch record order (small by size class, then
    // large), built on the device -- [order | inverse] and the sort's key / temp space
    uint32_t* d_word = nullptr;
    ffm::WinMeta wmeta;               // [cap] the window's metadata (fixed buffers)
    uint64_t* d_wa = nullptr;         // device: first record of the window
    uint64_t* h_wa = nullptr;         // pinned mirror
    uint32_t* d_wbins = nullptr;      // window order: class counts | cursors | done (zero between steps)
    uint64_t word_cap = 0;
    uint64_t last_window = 0;         // size of the previous online window
    uint64_t n_small_recs = 0;        // records <= small_bytes appended so far
    uint64_t online_small0 = 0;       // n_small_recs / n_large_chunks at online_done
    uint64_t online_chunks0 = 0;

    // folded grouping scratch
    void* fold_buf = nullptr;
    uint64_t fold_cap = 0;

    // gather descriptors for device payloads
    uint64_t* d_desc = nullptr;
    uint64_t desc_cap = 0;
    uint64_t* h_desc = nullptr;     // page-locked staging of the descriptors
    uint64_t h_desc_cap = 0;
    bool meta_pinned = false;       // h_site .. h_chan page-locked (within the reserved capacity)

    // run state
    ffm::Work work;
    ffm::Params params{};
    uint32_t* h_counters = nullptr;   // pinned mirror
    cudaEvent_t ev[20] = {};
    ffm_run_stats stats{};
    uint64_t n_syncs = 0;             // host synchronisations of the run stream (this run)
    bool digests_valid = false;
};
