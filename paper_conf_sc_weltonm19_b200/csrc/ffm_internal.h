// ffm_internal.h -- internal structures of libffm (product path).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/ffm.h"

namespace ffm {

constexpr uint32_t kArenaAlign = 128;        // record slots in the HBM arena
constexpr uint64_t kEmptyKey = ~0ull;         // group-by table: empty slot
constexpr uint32_t kNoRecord = 0xFFFFFFFFu;

// Device-side views handed to the kernel launchers.
struct DevLog {
    const uint8_t* arena;
    const uint64_t* off;     // [n] arena offset of record i (128-B aligned)
    const uint64_t* size;    // [n]
    const uint32_t* site;    // [n]
    const uint64_t* dur;     // [n]
    const uint64_t* gid;     // [n]
    uint32_t n;
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
    uint32_t* pos = nullptr;       // [n] position of a large member within its leader's group
    uint2* hitems = nullptr;       // large-payload hash work units (record, chunk)
    uint2* vitems = nullptr;       // large-payload verify work units (member, chunk)
    uint32_t* hcount = nullptr;    // [n+1] per-record hash chunk counts
    uint32_t* hstart = nullptr;    // [n+1] exclusive scan of hcount
    uint64_t* hpart = nullptr;     // [2 * hitem_cap] per-unit partial NH sums (A, B)
    uint64_t* tkey = nullptr;      // [cap] table keys
    uint32_t* tval = nullptr;      // [cap] table min local index
    int64_t* dup = nullptr;        // [n] output staging
    uint64_t* ben = nullptr;       // [n_sites]
    uint64_t* label_part = nullptr; // [label_hist_rows * n_sites] per-block benefit partials
    uint32_t* counters = nullptr;  // device counters: [0] nres, [1] n_members, [2..] misc
    void* cub_tmp = nullptr;
    size_t cub_tmp_bytes = 0;
    uint64_t n_cap = 0, t_cap = 0, hitem_cap = 0, vitem_cap = 0, site_cap = 0;
};

struct Params {
    uint64_t digest_mask;
    uint64_t refine_mask;
    uint32_t chunk_bytes;
    uint32_t small_bytes;
    int num_sms;
    int max_smem;      // opt-in dynamic shared memory per block (bytes)
};

// ---- kernel launchers (kernels.cu).  All asynchronous on `st`; each returns the
// number of kernels it launched (for the launch count), or -1 on launch error.
int launch_hash_small(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_hash_plan(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_hash_large(const DevLog& L, Work& W, const Params& P, uint64_t n_items, cudaStream_t st);
int launch_hash_combine(const DevLog& L, Work& W, const Params& P, cudaStream_t st);
int launch_group(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                 uint64_t cap, int round, cudaStream_t st);
int launch_verify(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                  uint32_t* res_out, uint64_t vitem_cap, cudaStream_t st, cudaStream_t side, cudaEvent_t ev_fork,
                  cudaEvent_t ev_join);
int launch_label(const DevLog& L, Work& W, const Params& P, uint32_t n_sites, int64_t* dup_out,
                 uint64_t* ben_out, cudaStream_t st);
uint32_t label_hist_rows(int num_sms);
int launch_gather(const uint64_t* d_desc, uint32_t n, uint8_t* arena, cudaStream_t st);
int launch_zero_counters(Work& W, cudaStream_t st);
size_t cub_scan_bytes(uint64_t n);

}  // namespace ffm

// The opaque handle.
struct ffm_log {
    ffm_config cfg{};
    int device = 0;
    cudaStream_t stream = nullptr;
    cudaStream_t stage_stream = nullptr;
    cudaStream_t side_stream = nullptr;   // small-payload kernels run concurrently here
    cudaEvent_t fork_ev[4] = {};
    bool own_stream = false;
    bool poisoned = false;
    std::string last_error;

    // host metadata (authoritative), program order
    std::vector<uint32_t> h_site;
    std::vector<uint64_t> h_size, h_off, h_dur, h_gid;
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
    uint64_t d_meta_cap = 0;       // records
    uint64_t d_meta_n = 0;         // records uploaded

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

    // gather descriptors for device payloads
    uint64_t* d_desc = nullptr;
    uint64_t desc_cap = 0;

    // run state
    ffm::Work work;
    ffm::Params params{};
    uint32_t* h_counters = nullptr;   // pinned mirror
    cudaEvent_t ev[16] = {};
    ffm_run_stats stats{};
    bool digests_valid = false;
};
