// ffm_api.cu -- the C ABI (include/ffm.h): log management, HBM staging (H0) and the
// run pipeline (H1..H7).  No C++ exception crosses the boundary; every CUDA error
// poisons the handle.  There is no CPU fallback: without a device, create fails.
#include <cuda_runtime.h>
#include <omp.h>
#include <stdio.h>

#include <chrono>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <functional>
#include <new>
#include <string>
#include <iterator>
#include <vector>

#include "ffm_internal.h"

using namespace ffm;

namespace {

constexpr uint64_t kRingBytes = 32ull << 20;      // per half of the pinned staging ring
constexpr uint64_t kDirectCopy = 4ull << 20;      // host payloads above this bypass the ring
constexpr uint64_t kGatherMax = 1ull << 20;   // device / pinned payloads up to this use k_gather (not DMA)

struct LocalRun {
    uint64_t n_members, n_res_total, rounds, prefilter_rest;
    uint64_t n_res0;     // round-0 residuals (kept in keep_res when asked)
    uint64_t n_reread;   // residual members whose bytes were compared again (not settled by difference lists)
    uint64_t n_overflow; // round-0 residuals whose difference list against their head overflowed
    bool two_pass;
    bool spec_stale;     // the speculative host labels need the final copy (residuals)
};

struct CudaFail {
    cudaError_t e;
    const char* what;
};

struct CommFail {   // an exchange error of a sharded run (FFM_E_COMM), or a range error
    int code;
    std::string what;
};

inline void ck(cudaError_t e, const char* what) {
    if (e != cudaSuccess) throw CudaFail{e, what};
}

inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

inline uint64_t pow2_at_least(uint64_t x) {
    uint64_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

int fail_cuda(ffm_log* log, const CudaFail& f) {
    log->poisoned = true;
    log->last_error = std::string(f.what) + ": " + cudaGetErrorString(f.e);
    cudaGetLastError();
    return FFM_E_CUDA;
}

int set_err(ffm_log* log, int code, const std::string& msg) {
    if (log) log->last_error = msg;
    return code;
}

template <class T>
void dev_grow(T*& p, uint64_t& cap, uint64_t need, uint64_t keep, cudaStream_t st) {
    if (need <= cap) return;
    uint64_t nc = std::max<uint64_t>(need, cap * 2);
    T* np = nullptr;
    ck(cudaMalloc(&np, nc * sizeof(T)), "cudaMalloc(metadata)");
    if (p && keep) ck(cudaMemcpyAsync(np, p, keep * sizeof(T), cudaMemcpyDeviceToDevice, st), "grow copy");
    ck(cudaStreamSynchronize(st), "grow sync");
    if (p) ck(cudaFree(p), "cudaFree");
    p = np;
    cap = nc;
}

template <class T>
void dev_alloc(T*& p, uint64_t count) {
    if (p) cudaFree(p);
    p = nullptr;
    ck(cudaMalloc(&p, std::max<uint64_t>(count, 1) * sizeof(T)), "cudaMalloc(work)");
}

// ---------------------------------------------------------------- staging (H0)
void ring_flush(ffm_log* L) {
    if (!L->ring_fill) return;
    int c = L->ring_cur;
    ck(cudaMemcpyAsync(L->arena + L->ring_arena_start, L->ring[c], L->ring_fill, cudaMemcpyHostToDevice,
                       L->stage_stream),
       "ring H2D");
    ck(cudaEventRecord(L->ring_ev[c], L->stage_stream), "ring event");
    L->ring_cur = c ^ 1;
    ck(cudaEventSynchronize(L->ring_ev[L->ring_cur]), "ring wait");   // other half free again
    L->ring_fill = 0;
}

void ensure_arena(ffm_log* L, uint64_t need) {
    // slack: kernels load a record's last, partial 32-byte block whole (and mask it in
    // registers), so the allocation must extend to the 32-byte boundary past the end
    need = align_up(need, kArenaAlign) + 64;
    if (need <= L->arena_cap) return;
    ring_flush(L);
    ck(cudaStreamSynchronize(L->stage_stream), "arena sync");
    ck(cudaStreamSynchronize(L->stream), "arena sync");
    uint64_t nc = std::max<uint64_t>(need, std::max<uint64_t>(L->arena_cap * 2, 64ull << 20));
    uint8_t* na = nullptr;
    if (cudaMalloc(&na, nc) != cudaSuccess) {
        cudaGetLastError();
        nc = need;   // retry exact
        ck(cudaMalloc(&na, nc), "cudaMalloc(arena)");
    }
    if (L->arena && L->arena_used)
        ck(cudaMemcpyAsync(na, L->arena, L->arena_used, cudaMemcpyDeviceToDevice, L->stage_stream), "arena copy");
    ck(cudaStreamSynchronize(L->stage_stream), "arena copy sync");
    if (L->arena) ck(cudaFree(L->arena), "cudaFree(arena)");
    L->arena = na;
    L->arena_cap = nc;
    ++L->epoch;
    ++L->bufgen;
    ++L->arena_gen;   // peers of a sharded log re-map it at their next run
}

void stage_host(ffm_log* L, const void* src, uint64_t size, uint64_t off) {
    if (size > kDirectCopy) {
        // pageable source: cudaMemcpyAsync returns once the bytes are in the driver's
        // staging memory, so the snapshot is taken before return without a sync
        ring_flush(L);
        ck(cudaMemcpyAsync(L->arena + off, src, size, cudaMemcpyHostToDevice, L->stage_stream), "H2D");
        return;
    }
    if (L->ring_fill && (off < L->ring_arena_start || off + size - L->ring_arena_start > L->ring_bytes))
        ring_flush(L);
    if (!L->ring_fill) L->ring_arena_start = off;
    memcpy(L->ring[L->ring_cur] + (off - L->ring_arena_start), src, size);
    L->ring_fill = off + size - L->ring_arena_start;
}

// Pageable payloads of one batch, staged in parallel: the arena range they cover is cut
// into ring-sized windows; for each window the host threads copy every record piece that
// falls in it into one half of the pinned ring (OpenMP), then that half goes to HBM
// asynchronously while the next window fills the other half.  The bytes are snapshotted
// (in the ring, or already in HBM) before the append returns (reading R11).
// host threads of the pageable staging copies (at most 8: several ranks may share a node)
[[maybe_unused]] int stage_threads() {   // (used in an OpenMP pragma)
    static const int t = std::max(1, std::min(8, omp_get_max_threads()));
    return t;
}

void stage_pageable(ffm_log* L, const std::vector<PageablePiece>& recs) {
    if (recs.empty()) return;
    ring_flush(L);
    const uint64_t R = L->ring_bytes;
    const uint64_t a0 = recs.front().off, a1 = recs.back().off + recs.back().size;
    size_t first = 0;   // first record that may reach into the current window
    for (uint64_t w0 = a0; w0 < a1; w0 += R) {
        const uint64_t w1 = std::min(a1, w0 + R);
        while (first < recs.size() && recs[first].off + recs[first].size <= w0) ++first;
        size_t last = first;
        while (last < recs.size() && recs[last].off < w1) ++last;
        const int c = L->ring_cur;
        uint8_t* ring = L->ring[c];
        // copy jobs of at most 1 MiB (a large record is split across the threads)
        std::vector<PageablePiece>& jobs = L->stage_jobs;
        jobs.clear();
        for (size_t k = first; k < last; ++k) {
            const PageablePiece& p = recs[k];
            for (uint64_t lo = std::max(p.off, w0), hi = std::min(p.off + p.size, w1); lo < hi; lo += (1ull << 20))
                jobs.push_back({p.src + (lo - p.off), lo - w0, std::min<uint64_t>(hi - lo, 1ull << 20)});
        }
        const long nj = (long)jobs.size();
        uint64_t bytes = 0;
        for (const PageablePiece& j : jobs) bytes += j.size;
#pragma omp parallel for schedule(dynamic, 1) num_threads(stage_threads()) if (bytes > (1ull << 20))
        for (long k = 0; k < nj; ++k) memcpy(ring + jobs[(size_t)k].off, jobs[(size_t)k].src, jobs[(size_t)k].size);
        ck(cudaMemcpyAsync(L->arena + w0, ring, w1 - w0, cudaMemcpyHostToDevice, L->stage_stream), "ring H2D");
        ck(cudaEventRecord(L->ring_ev[c], L->stage_stream), "ring event");
        L->ring_cur = c ^ 1;
        ck(cudaEventSynchronize(L->ring_ev[L->ring_cur]), "ring wait");   // the other half is free again
    }
}

// FFM_PAYLOAD_DEVICE / _HOST_PINNED / _HOST (pageable) of one pointer; *dev = the
// device a device pointer lives on (-1 for host memory).
int pointer_kind(const void* p, int* dev) {
    *dev = -1;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return FFM_PAYLOAD_HOST;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
        *dev = a.device;
        return FFM_PAYLOAD_DEVICE;
    }
    if (a.type == cudaMemoryTypeHost) return FFM_PAYLOAD_HOST_PINNED;
    return FFM_PAYLOAD_HOST;
}

// Kind / device of many payload pointers: one attribute query per allocation (the
// driver's address range of a device or pinned allocation is cached), not per record.
struct PtrCache {
    uintptr_t lo = 0, hi = 0;
    int kind = FFM_PAYLOAD_HOST, dev = -1;
    int (*get_attr)(void*, int, uintptr_t) = nullptr;   // cuPointerGetAttribute
    bool tried = false;

    int classify(const void* p, int* dev_out) {
        const uintptr_t a = (uintptr_t)p;
        if (a >= lo && a < hi) {
            *dev_out = dev;
            return kind;
        }
        const int k = pointer_kind(p, dev_out);
        if (k == FFM_PAYLOAD_HOST) return k;   // pageable: no range to cache
        if (!tried) {
            tried = true;
            void* fn = nullptr;
            if (cudaGetDriverEntryPoint("cuPointerGetAttribute", &fn, cudaEnableDefault, nullptr) == cudaSuccess)
                get_attr = (int (*)(void*, int, uintptr_t))fn;
            else
                cudaGetLastError();
        }
        uintptr_t start = 0;
        size_t size = 0;
        if (get_attr && get_attr(&start, 11 /* RANGE_START_ADDR */, a) == 0 &&
            get_attr(&size, 12 /* RANGE_SIZE */, a) == 0 && size) {
            lo = start;
            hi = start + size;
            kind = k;
            dev = *dev_out;
        }
        return k;
    }
};

bool is_pinned_host(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeHost;
}

bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Records in [begin, end) as indices relative to begin: first those with size <=
// small_bytes, ordered by 32-byte block count, largest first (stable counting sort);
// then the large ones in index order (one warp per large record in the planning
// kernels).  Returns the number of small records.
uint64_t build_small_order(const ffm_log* L, uint64_t begin, uint64_t end, std::vector<uint32_t>& order) {
    const uint32_t nb = (L->params.small_bytes + 31) / 32 + 1;
    std::vector<uint32_t> start(nb + 1, 0);
    uint64_t ns = 0;
    for (uint64_t i = begin; i < end; ++i)
        if (L->h_size[i] <= L->params.small_bytes) {
            start[nb - (uint32_t)((L->h_size[i] + 31) / 32)]++;
            ++ns;
        }
    for (uint32_t b = 1; b <= nb; ++b) start[b] += start[b - 1];
    // start[c] now counts classes < c; class c = nb-1-blocks  ->  cursor = start[c]
    std::vector<uint32_t> cur(nb, 0);
    for (uint32_t c = 0; c < nb; ++c) cur[c] = c ? start[c] : 0;
    order.assign(ns, 0);
    for (uint64_t i = begin; i < end; ++i)
        if (L->h_size[i] <= L->params.small_bytes)
            order[cur[nb - 1 - (uint32_t)((L->h_size[i] + 31) / 32)]++] = (uint32_t)(i - begin);
    for (uint64_t i = begin; i < end; ++i)
        if (L->h_size[i] > L->params.small_bytes) order.push_back((uint32_t)(i - begin));
    return ns;
}

void upload_order(ffm_log* L, const std::vector<uint32_t>& order, uint32_t*& dptr, uint64_t& cap, cudaStream_t s) {
    uint64_t ns = order.size();
    if (ns > cap || !dptr) {
        if (dptr) ck(cudaFree(dptr), "cudaFree");
        dptr = nullptr;
        cap = std::max<uint64_t>(std::max<uint64_t>(ns, 2 * cap), 1024);
        ck(cudaMalloc(&dptr, 2 * cap * sizeof(uint32_t)), "cudaMalloc(order)");   // order, then its inverse
    }
    if (ns) {
        ck(cudaMemcpyAsync(dptr, order.data(), ns * 4, cudaMemcpyHostToDevice, s), "order H2D");
        if (launch_invert(dptr, (uint32_t)ns, dptr + cap, s) < 0) throw CudaFail{cudaGetLastError(), "invert order"};
    }
}

// H0 tail: the metadata SoA of records appended since the last upload (incremental;
// pageable-source copies are staged before the call returns, no sync needed).
void upload_meta_arrays(ffm_log* L) {
    uint64_t n = L->h_size.size();
    if (L->d_meta_n == n) return;
    uint64_t c0 = L->d_meta_cap, keep = L->d_meta_n;
    uint64_t cap = c0;
    dev_grow(L->d_off, cap, n, keep, L->stage_stream);
    cap = c0;
    dev_grow(L->d_size, cap, n, keep, L->stage_stream);
    cap = c0;
    dev_grow(L->d_site, cap, n, keep, L->stage_stream);
    cap = c0;
    dev_grow(L->d_dur, cap, n, keep, L->stage_stream);
    cap = c0;
    dev_grow(L->d_gid, cap, n, keep, L->stage_stream);
    cap = c0;
    dev_grow(L->d_chan, cap, n, keep, L->stage_stream);
    if (cap != L->d_meta_cap) ++L->bufgen;
    L->d_meta_cap = cap;
    uint64_t a = L->d_meta_n, k = n - a;
    cudaStream_t s = L->stage_stream;
    ck(cudaMemcpyAsync(L->d_off + a, L->h_off.data() + a, k * 8, cudaMemcpyHostToDevice, s), "meta H2D");
    ck(cudaMemcpyAsync(L->d_size + a, L->h_size.data() + a, k * 8, cudaMemcpyHostToDevice, s), "meta H2D");
    ck(cudaMemcpyAsync(L->d_site + a, L->h_site.data() + a, k * 4, cudaMemcpyHostToDevice, s), "meta H2D");
    ck(cudaMemcpyAsync(L->d_dur + a, L->h_dur.data() + a, k * 8, cudaMemcpyHostToDevice, s), "meta H2D");
    ck(cudaMemcpyAsync(L->d_gid + a, L->h_gid.data() + a, k * 8, cudaMemcpyHostToDevice, s), "meta H2D");
    ck(cudaMemcpyAsync(L->d_chan + a, L->h_chan.data() + a, k * 8, cudaMemcpyHostToDevice, s), "meta H2D");
    L->d_meta_n = n;
}

// The whole log's record order of the batch passes: small records by size class
// (largest first: the four 8-lane groups of a warp then get payloads of near-equal
// length), then the large ones.  Rebuilt only when records were appended since.
void upload_meta(ffm_log* L) {
    upload_meta_arrays(L);
    const uint64_t n = L->h_size.size();
    if (L->d_order_n == n && L->d_small_order) return;
    std::vector<uint32_t> order;
    L->n_small = build_small_order(L, 0, n, order);
    L->n_large_rec = order.size() - L->n_small;
    upload_order(L, order, L->d_small_order, L->d_small_cap, L->stage_stream);
    L->d_order_n = n;
}

uint64_t large_chunks(const ffm_log* L, uint64_t size) {
    uint64_t cb = L->params.chunk_bytes;
    return size > L->params.small_bytes ? (size + cb - 1) / cb : 0;
}

int check_state(ffm_log* L) {
    if (!L) return FFM_E_INVAL;
    if (L->poisoned) return FFM_E_STATE;
    return FFM_OK;
}

// Validate + assign arena offsets for a batch; returns FFM_OK or an error without
// touching the log.  Slots are 32-byte aligned, so offs[i] = base + sum over earlier
// records of align_up(size, 32): a prefix sum, split over the host threads for a large
// batch (each thread's chunk checked and summed, then offset by the chunks before it); an
// error is reported for the first offending record, as the serial check would.
int plan_batch(ffm_log* L, uint64_t n, const uint32_t* sites, const uint64_t* sizes, const void* const* payloads,
               const uint64_t* gids, std::vector<uint64_t>& offs, uint64_t& arena_end) {
    const bool any0 = L->any_gid || !L->h_gid.empty();
    const uint64_t last0 = L->last_gid;
    uint64_t base_n = L->h_size.size();
    if (base_n + n >= 0xFFFFFFFFull) return set_err(L, FFM_E_RANGE, "too many records for one log (2^32-1)");
    if (L->cfg.world > 1 && !gids)
        return set_err(L, FFM_E_INVAL, "a sharded log needs the records' global gids (gids == NULL)");
    offs.resize(n);
    // record i's problem (0: none), independent of the others but for the gid order
    auto check = [&](uint64_t i) -> int {
        if (sites[i] >= L->cfg.n_sites) return 1;
        if (sizes[i] > 0 && payloads[i] == nullptr) return 2;
        if (gids) {
            if ((i > 0 || any0) && gids[i] <= (i > 0 ? gids[i - 1] : last0)) return 3;
            if (gids[i] >> 63) return 4;
        } else if (((any0 ? last0 + 1 : 0) + i) >> 63) {
            return 4;
        }
        return 0;
    };
    const uint64_t base = align_up(L->arena_used, kArenaAlign);
    const int T = n >= 65536 ? stage_threads() : 1;
    std::vector<uint64_t> part(T + 1, 0), bad(T, ~0ull);
    int used = 1;
#pragma omp parallel num_threads(T) if (T > 1)
    {
        const int t = omp_get_thread_num(), nt = omp_get_num_threads();
        const uint64_t lo = n * t / nt, hi = n * (t + 1) / nt;
        uint64_t sum = 0;
        for (uint64_t i = lo; i < hi; ++i) {
            if (bad[t] == ~0ull && check(i)) bad[t] = i;
            offs[i] = sum;
            sum += align_up(sizes[i], kArenaAlign);
        }
        part[t + 1] = sum;
#pragma omp barrier
#pragma omp single
        {
            used = nt;
            for (int k = 0; k < nt; ++k) part[k + 1] += part[k];
        }
        for (uint64_t i = lo; i < hi; ++i) offs[i] += base + part[t];
    }
    uint64_t first = ~0ull;
    for (int t = 0; t < used; ++t) first = std::min(first, bad[t]);
    if (first != ~0ull) {
        switch (check(first)) {
            case 1: return set_err(L, FFM_E_RANGE, "call_site >= n_sites");
            case 2: return set_err(L, FFM_E_INVAL, "NULL payload with size > 0");
            case 3: return set_err(L, FFM_E_RANGE, "gids must be strictly increasing");
            default: return set_err(L, FFM_E_RANGE, "gid >= 2^63 (duplicate_of is int64)");
        }
    }
    arena_end = n ? offs[n - 1] + sizes[n - 1] : L->arena_used;
    return FFM_OK;
}

// The host metadata vectors are page-locked while they stay within the capacity reserved
// at create (cfg.max_records): their uploads are then plain asynchronous DMA.  Growing past
// it reallocates them -- unregistered first, pageable from then on.
void pin_meta(ffm_log* L, bool on) {
    void* ptrs[] = {L->h_site.data(), L->h_size.data(), L->h_off.data(), L->h_dur.data(), L->h_gid.data(),
                    L->h_chan.data()};
    const size_t bytes[] = {L->h_site.capacity() * 4, L->h_size.capacity() * 8, L->h_off.capacity() * 8,
                            L->h_dur.capacity() * 8, L->h_gid.capacity() * 8, L->h_chan.capacity() * 8};
    if (on && !L->meta_pinned) {
        bool ok = true;
        for (int i = 0; i < 6; ++i) ok = ok && bytes[i] && cudaHostRegister(ptrs[i], bytes[i], cudaHostRegisterDefault) == cudaSuccess;
        cudaGetLastError();
        L->meta_pinned = ok;
        if (!ok)
            for (int i = 0; i < 6; ++i) cudaHostUnregister(ptrs[i]);   // (the ones that did register)
        cudaGetLastError();
    } else if (!on && L->meta_pinned) {
        ck(cudaStreamSynchronize(L->stage_stream), "unpin sync");   // no upload still reads them
        for (int i = 0; i < 6; ++i) cudaHostUnregister(ptrs[i]);
        cudaGetLastError();
        L->meta_pinned = false;
    }
}

// gids g, g + 1, ... as an iterator range (no temporary, no zero-fill pass)
struct CountIt {
    using iterator_category = std::forward_iterator_tag;
    using value_type = uint64_t;
    using difference_type = std::ptrdiff_t;
    using pointer = const uint64_t*;
    using reference = uint64_t;
    uint64_t v;
    uint64_t operator*() const { return v; }
    CountIt& operator++() {
        ++v;
        return *this;
    }
    bool operator!=(const CountIt& o) const { return v != o.v; }
};

// Appends the batch's metadata to the host copies: the six arrays copied concurrently and
// the running sums reduced in parallel for large batches (the append's host cost).
void push_meta(ffm_log* L, uint64_t n, const uint32_t* sites, const uint64_t* sizes, const uint64_t* durs,
               const uint64_t* gids, const uint64_t* chans, const std::vector<uint64_t>& offs, uint64_t arena_end) {
    const uint64_t base = L->h_size.size();
    const bool any = base > 0;
    if (L->meta_pinned && base + n > L->h_size.capacity()) pin_meta(L, false);   // about to reallocate
    const uint64_t g0 = gids ? 0 : (any ? L->last_gid + 1 : 0);
    [[maybe_unused]] const bool par = n >= 65536;   // (used in the OpenMP clauses)
#pragma omp parallel sections num_threads(6) if (par)
    {
#pragma omp section
        L->h_site.insert(L->h_site.end(), sites, sites + n);
#pragma omp section
        L->h_size.insert(L->h_size.end(), sizes, sizes + n);
#pragma omp section
        L->h_off.insert(L->h_off.end(), offs.begin(), offs.begin() + n);
#pragma omp section
        L->h_dur.insert(L->h_dur.end(), durs, durs + n);
#pragma omp section
        {
            if (chans)
                L->h_chan.insert(L->h_chan.end(), chans, chans + n);
            else
                L->h_chan.resize(base + n, 0);
        }
#pragma omp section
        {
            if (gids)
                L->h_gid.insert(L->h_gid.end(), gids, gids + n);
            else
                L->h_gid.insert(L->h_gid.end(), CountIt{g0}, CountIt{g0 + n});
        }
    }
    if (gids) L->any_gid = true;
    if (n) L->last_gid = L->h_gid.back();
    uint64_t pb = 0, nlc = 0, nsr = 0;
    const uint64_t cb = L->params.chunk_bytes, sb = L->params.small_bytes;
#pragma omp parallel for reduction(+ : pb, nlc, nsr) num_threads(8) if (par)
    for (uint64_t i = 0; i < n; ++i) {
        const uint64_t z = sizes[i];
        pb += z;
        nlc += z > sb ? (z + cb - 1) / cb : 0;
        nsr += z <= sb;
    }
    L->payload_bytes += pb;
    L->n_large_chunks += nlc;
    L->n_small_recs += nsr;
    L->arena_used = arena_end;
    ++L->epoch;
}

// ---------------------------------------------------------------- work buffers
void ensure_work(ffm_log* L, uint64_t n) {
    Work& W = L->work;
    uint64_t tcap = std::max<uint64_t>(1024, pow2_at_least(2 * std::max<uint64_t>(n, 1)));
    const uint64_t fcap0 = fx_entry_cap(L->n_large_chunks, L->params.chunk_bytes);
    if (n > W.n_cap || W.accA == nullptr || tcap > W.t_cap || L->n_large_chunks > W.hitem_cap ||
        fcap0 > W.fitem_cap || L->cfg.n_sites > W.site_cap) {
        // growing frees buffers that append-time hashing (staging stream) may still read
        ck(cudaStreamSynchronize(L->stage_stream), "work sync");
        ck(cudaStreamSynchronize(L->hash_stream), "work sync");
        ck(cudaStreamSynchronize(L->stream), "work sync");
    }
    if (n > W.n_cap || W.accA == nullptr) {
        ++L->epoch;
        ++L->bufgen;
        uint64_t c = std::max<uint64_t>(n, 1024);
        dev_alloc(W.accA, c);
        dev_alloc(W.accB, c);
        dev_alloc(W.key, c);
        dev_alloc(W.digest, c);
        dev_alloc(W.slot, c);
        dev_alloc(W.leader, c);
        dev_alloc(W.eq, c);
        dev_alloc(W.mis, c);
        dev_alloc(W.res[0], c);
        dev_alloc(W.res[1], c);
        dev_alloc(W.lcount, c + 1);
        dev_alloc(W.lstart, c + 1);
        dev_alloc(W.gcount, c + 1);
        dev_alloc(W.pos, c);
        dev_alloc(W.fhead, c);
        dev_alloc(W.dcnt, c);
        dev_alloc(W.dq, (uint64_t)kDiffK * c);
        dev_alloc(W.dv, (uint64_t)kDiffK * c);
        dev_alloc(W.sdesc, 2 * c);
        dev_alloc(W.hcount, c + 1);
        dev_alloc(W.hstart, c + 1);
        dev_alloc(W.dup, c);
        if (!W.counters) dev_alloc(W.counters, 16);
        size_t cb = cub_scan_bytes(c + 1);
        if (W.cub_tmp) cudaFree(W.cub_tmp);
        W.cub_tmp = nullptr;
        ck(cudaMalloc(&W.cub_tmp, std::max<size_t>(cb, 256)), "cudaMalloc(cub)");
        W.cub_tmp_bytes = std::max<size_t>(cb, 256);
        W.n_cap = c;
    }
    if (tcap > W.t_cap) {
        ++L->epoch;
        ++L->bufgen;
        dev_alloc(W.tkey, tcap);
        W.t_cap = tcap;
    }
    if (L->n_large_chunks > W.hitem_cap) {
        ++L->epoch;
        ++L->bufgen;
        uint64_t c = L->n_large_chunks + L->n_large_chunks / 4 + 64;
        dev_alloc(W.hitems, c);
        dev_alloc(W.hpart, 2 * c);
        W.hitem_cap = W.vitem_cap = c;   // vitem_cap: non-zero enables the large verify
    }
    const uint64_t fcap = fx_entry_cap(L->n_large_chunks, L->params.chunk_bytes);
    if (fcap > W.fitem_cap) {
        ++L->epoch;
        ++L->bufgen;
        const uint64_t c = fcap + fcap / 4;
        dev_alloc(W.fitems, 2 * c);   // 32-byte descriptors
        W.fitem_cap = c;
    }
    if (L->cfg.n_sites > W.site_cap) {
        ++L->epoch;
        ++L->bufgen;
        dev_alloc(W.ben, 2 * (uint64_t)L->cfg.n_sites);   // [benefit | duplicate counts]: one all-reduce
        W.cnt = W.ben + L->cfg.n_sites;
        if (label_smem_bytes(L->cfg.n_sites) <= (uint64_t)L->params.max_smem) {
            dev_alloc(W.label_part, (uint64_t)label_hist_rows(L->params.num_sms) * L->cfg.n_sites);
            dev_alloc(W.label_cpart, (uint64_t)label_hist_rows(L->params.num_sms) * L->cfg.n_sites);
        }
        W.site_cap = L->cfg.n_sites;
    }
}

DevLog dev_view(const ffm_log* L) {
    DevLog d;
    d.arena = L->arena;
    d.off = L->d_off;
    d.size = L->d_size;
    d.site = L->d_site;
    d.dur = L->d_dur;
    d.gid = L->d_gid;
    d.chan = L->d_chan;
    d.n = (uint32_t)L->h_size.size();
    d.small_order = L->d_small_order;
    d.order_pos = L->d_small_order ? L->d_small_order + L->d_small_cap : nullptr;
    d.n_small = (uint32_t)L->n_small;
    d.large_order = L->d_small_order ? L->d_small_order + L->n_small : nullptr;
    d.n_large = (uint32_t)L->n_large_rec;
    return d;
}

float ev_ms(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return 0.f;
    }
    return ms;
}

#define LCHK(x)                                                                \
    do {                                                                       \
        int _k = (x);                                                          \
        if (_k < 0) throw CudaFail{cudaGetLastError(), "kernel launch " #x};   \
        launches += (uint64_t)_k;                                              \
    } while (0)


// ---------------------------------------------------------------- run pipeline
// A host synchronisation of the run's stream (counted: ffm_run_stats.host_syncs).
void sync_run(ffm_log* L, const char* what) {
    ++L->n_syncs;
    ck(cudaStreamSynchronize(L->stream), what);
}

void run_prologue(ffm_log* L) {
    ck(cudaSetDevice(L->device), "cudaSetDevice");
    // H0 tail: flush staged payloads and metadata, order the run after them
    ring_flush(L);
    if (L->collective) ensure_arena(L, 1);   // peers map it: it exists before the header exchange
    upload_meta(L);
    ck(cudaEventRecord(L->ring_ev[L->ring_cur], L->stage_stream), "event");
    ck(cudaStreamWaitEvent(L->stream, L->ring_ev[L->ring_cur], 0), "wait staging");
    ck(cudaStreamWaitEvent(L->stream, L->hash_ev, 0), "wait append-time hashing");
    ensure_work(L, L->h_size.size());
}

// An online window [a, b) of the log as a log of its own (indices relative to a) in the
// identity record order: no host-side order build per window -- the small / large
// kernels skip records of the other kind by size (two-pass round 0, hashing).
DevLog window_view(ffm_log* L, uint64_t a, uint64_t b, bool has_large, cudaStream_t st) {
    const uint64_t nw = b - a;
    if (nw > L->iota_cap) {
        if (L->d_iota) ck(cudaFree(L->d_iota), "cudaFree");
        L->d_iota = nullptr;
        const uint64_t c = std::max<uint64_t>(std::max<uint64_t>(nw, 2 * L->iota_cap), 4096);
        ck(cudaMalloc(&L->d_iota, c * sizeof(uint32_t)), "cudaMalloc(iota)");
        if (launch_iota(L->d_iota, (uint32_t)c, st) < 0) throw CudaFail{cudaGetLastError(), "iota"};
        L->iota_cap = c;
        ++L->bufgen;
    }
    DevLog D = dev_view(L);
    D.off += a;
    D.size += a;
    D.site += a;
    D.dur += a;
    D.gid += a;
    D.chan += a;
    D.n = (uint32_t)nw;
    D.small_order = L->d_iota;
    D.order_pos = L->d_iota;
    D.n_small = (uint32_t)nw;
    D.large_order = L->d_iota;
    D.n_large = has_large ? (uint32_t)nw : 0u;   // (no large-record kernels for a window without any)
    return D;
}

// An online window [a, b) in the batch record order (small records by size class, then
// the large ones), its metadata gathered into fixed buffers: window_view_sorted sizes the
// buffers and returns the view; queue_window_order queues the gather and the order build
// (a counting sort by size class: 2 kernels).  n_small: small records in it.
DevLog window_view_sorted(ffm_log* L, uint64_t a, uint64_t b, uint64_t n_small, cudaStream_t st) {
    DevLog D = window_view(L, a, b, true, st);   // (iota of >= b - a entries)
    const uint64_t nw = b - a;
    if (nw > L->word_cap) {
        ck(cudaStreamSynchronize(st), "window buffers");
        for (void* p : {(void*)L->d_word, (void*)L->wmeta.off, (void*)L->wmeta.size, (void*)L->wmeta.dur,
                        (void*)L->wmeta.gid, (void*)L->wmeta.chan, (void*)L->wmeta.site})
            if (p) ck(cudaFree(p), "cudaFree");
        L->d_word = nullptr;
        L->wmeta = WinMeta{};
        const uint64_t c = std::max<uint64_t>(std::max<uint64_t>(nw, 2 * L->word_cap), 4096);
        ck(cudaMalloc(&L->d_word, 2 * c * sizeof(uint32_t)), "cudaMalloc(window order)");
        ck(cudaMalloc(&L->wmeta.off, c * sizeof(uint64_t)), "cudaMalloc(window meta)");
        ck(cudaMalloc(&L->wmeta.size, c * sizeof(uint64_t)), "cudaMalloc(window meta)");
        ck(cudaMalloc(&L->wmeta.dur, c * sizeof(uint64_t)), "cudaMalloc(window meta)");
        ck(cudaMalloc(&L->wmeta.gid, c * sizeof(uint64_t)), "cudaMalloc(window meta)");
        ck(cudaMalloc(&L->wmeta.chan, c * sizeof(uint64_t)), "cudaMalloc(window meta)");
        ck(cudaMalloc(&L->wmeta.site, c * sizeof(uint32_t)), "cudaMalloc(window meta)");
        if (!L->d_wbins) {
            const uint64_t nb = 3ull * window_bins(L->params.small_bytes);
            ck(cudaMalloc(&L->d_wbins, nb * sizeof(uint32_t)), "cudaMalloc(window bins)");
            ck(cudaMemsetAsync(L->d_wbins, 0, nb * sizeof(uint32_t), st), "memset");
        }
        L->word_cap = c;
        ++L->bufgen;
    }
    if (!L->d_wa) {
        ck(cudaMalloc(&L->d_wa, sizeof(uint64_t)), "cudaMalloc(window start)");
        ck(cudaMallocHost(&L->h_wa, sizeof(uint64_t)), "cudaMallocHost(window start)");
    }
    D.off = L->wmeta.off;
    D.size = L->wmeta.size;
    D.site = L->wmeta.site;
    D.dur = L->wmeta.dur;
    D.gid = L->wmeta.gid;
    D.chan = L->wmeta.chan;
    D.small_order = L->d_word;
    D.order_pos = L->d_word + L->word_cap;
    D.n_small = (uint32_t)n_small;
    D.large_order = L->d_word + n_small;
    D.n_large = (uint32_t)(nw - n_small);
    return D;
}

void queue_window_order(ffm_log* L, const DevLog& D, cudaStream_t st, uint64_t& launches) {
    const int k = launch_window_order(dev_view(L), L->d_wa, D.n, L->wmeta, L->params.small_bytes, L->d_wbins,
                                      const_cast<uint32_t*>(D.small_order), const_cast<uint32_t*>(D.order_pos), st);
    if (k < 0) throw CudaFail{cudaGetLastError(), "window order"};
    launches += (uint64_t)k;
}

// Online mode (S8(f) #2): the NH sums of records [a, b) into on_A / on_B (global record
// index), on stream st -- at append time on the hashing stream (FFM_FLAG_APPEND_HASH), else
// at the start of a step.
void online_hash(ffm_log* L, uint64_t a, uint64_t b, cudaStream_t st, uint64_t& launches) {
    if (a >= b) return;
    if (b > L->on_cap) {
        uint64_t c0 = L->on_cap, cap = c0;
        const uint64_t need = std::max<uint64_t>(b, 2 * c0);
        dev_grow(L->on_A, cap, need, a, st);
        cap = c0;
        dev_grow(L->on_B, cap, need, a, st);
        L->on_cap = cap;
    }
    uint64_t n_large = 0;
    for (uint64_t i = a; i < b; ++i) n_large += large_chunks(L, L->h_size[i]);
    const DevLog D = window_view(L, a, b, n_large != 0, st);
    Work W2 = L->work;
    W2.accA = L->on_A + a;
    W2.accB = L->on_B + a;
    LCHK(launch_hash_small(D, W2, L->params, st));
    if (n_large) {
        LCHK(launch_hash_plan(D, W2, L->params, true, st));
        LCHK(launch_hash_large(D, W2, L->params, n_large, st));
        LCHK(launch_combine(D, W2, L->params, st));
    }
}

// Capacity of the persistent online table for nw more representatives (the table is
// rehashed only when it has to grow: never by a step that fits).
void ensure_online(ffm_log* L, uint64_t nw) {
    OnlineTable& T = L->otab;
    cudaStream_t s = L->stream;
    if (!T.count) {
        ck(cudaMalloc(&T.count, sizeof(uint32_t)), "cudaMalloc(online)");
        ck(cudaMemsetAsync(T.count, 0, sizeof(uint32_t), s), "memset");
    }
    const uint64_t need = L->online_np + nw;
    if (need > L->pool_cap) {
        const uint64_t c = std::max<uint64_t>(std::max<uint64_t>(need, 1024), 2 * L->pool_cap);
        OnlineRep* np = nullptr;
        ck(cudaMalloc(&np, c * sizeof(OnlineRep)), "cudaMalloc(online pool)");
        if (L->online_np)
            ck(cudaMemcpyAsync(np, T.pool, L->online_np * sizeof(OnlineRep), cudaMemcpyDeviceToDevice, s), "copy");
        ck(cudaStreamSynchronize(s), "pool sync");
        if (T.pool) ck(cudaFree(T.pool), "cudaFree");
        T.pool = np;
        L->pool_cap = c;
        ++L->bufgen;
    }
    if (2 * need > T.mask + 1 || !T.key) {
        const uint64_t cap = std::max<uint64_t>(1024, pow2_at_least(4 * need));
        ck(cudaStreamSynchronize(s), "table sync");
        if (T.key) ck(cudaFree(T.key), "cudaFree");
        if (T.head) ck(cudaFree(T.head), "cudaFree");
        T.key = nullptr;
        T.head = nullptr;
        ck(cudaMalloc(&T.key, cap * sizeof(uint64_t)), "cudaMalloc(online table)");
        ck(cudaMalloc(&T.head, cap * sizeof(uint32_t)), "cudaMalloc(online table)");
        T.mask = cap - 1;
        ++L->bufgen;
        if (launch_online_rehash(T, (uint32_t)L->online_np, L->params.digest_mask, s) < 0)
            throw CudaFail{cudaGetLastError(), "online rehash"};
    }
    if (nw > L->on_G_cap) {
        dev_alloc(L->on_G, nw);
        dev_alloc(L->on_res, nw);
        L->on_G_cap = nw;
        ++L->bufgen;
    }
}

// H1..H4 over the local log: on return W.leader holds every record's final local
// leader (the min local index of its exact byte class).  With `label` the H5/H6
// kernels are queued before the first sync (single-GPU fast path: one sync when
// there are no digest collisions) and re-run after collision resolution.
// pre_sync: more stream work queued after segment A, before its host sync (a sharded
// run's representative export and header exchange).
// prehashed: the NH sums are already in W.accA / W.accB (online windows): two-pass
// round 0 without H1.
// h_spec: pinned host duplicate_of: the labels are written speculatively after the
// round-0 group-by and copied there while H3 runs (R.spec_stale: residuals changed some;
// the caller copies again).
LocalRun run_local(ffm_log* L, const DevLog& D, uint64_t n_large, uint64_t& launches, bool label, int64_t* d_dup,
                   bool prefilter = false, const std::function<void()>* pre_sync = nullptr, bool prehashed = false,
                   int64_t* h_spec = nullptr, bool window = false, uint32_t* keep_res = nullptr,
                   GraphSlot* wslot = nullptr, const uint64_t* wextra = nullptr,
                   const std::function<void()>* pre_a = nullptr) {
    const bool timing = (L->cfg.flags & FFM_FLAG_TIMING) != 0;
    const uint64_t n = D.n;
    Work& W = L->work;
    cudaStream_t s = L->stream;
    const uint32_t ns = L->cfg.n_sites;
    LocalRun R{};
    cudaStream_t side = L->side_stream;
    // round-0 mode: forced by a flag, else adaptive -- a log whose fused run found most
    // large candidates to be near-duplicate mismatches uses the two-pass round 0 next time
    const bool two_pass = prehashed || (L->cfg.flags & FFM_FLAG_TWO_PASS) != 0 ||
                          (!(L->cfg.flags & FFM_FLAG_FUSED) && L->prefer_two_pass);
    // segment A: everything up to the first host sync (H1, H2, H3, speculative H5/H6 and
    // the counters read-back) -- ~30 launches on two streams, no host dependency
    auto segment_a = [&]() {
        if (timing) ck(cudaEventRecord(L->ev[0], s), "event");
        if (launch_zero_counters(W, s) < 0) throw CudaFail{cudaGetLastError(), "zero counters"};
        // two-pass H1 of small payloads on the side stream, concurrently with the large path
        // (fused: small payloads are grouped by their first 32 bytes, hashed after H2)
        if (two_pass && !prehashed) {
            ck(cudaEventRecord(L->fork_ev[0], s), "event");
            ck(cudaStreamWaitEvent(side, L->fork_ev[0], 0), "fork");
            if (timing) ck(cudaEventRecord(L->ev[12], side), "event");
            LCHK(launch_hash_small(D, W, L->params, side));
            if (timing) ck(cudaEventRecord(L->ev[8], side), "event");
            ck(cudaEventRecord(L->fork_ev[1], side), "event");
        }
        if (n_large && !prehashed) {
            LCHK(launch_hash_plan(D, W, L->params, two_pass, s));
            if (timing) ck(cudaEventRecord(L->ev[10], s), "event");
            // fused: the prefix pass (first prefix_bytes); two-pass: every chunk, then the combine
            if (two_pass) LCHK(launch_hash_large(D, W, L->params, n_large, s));
            else LCHK(launch_prefix(D, W, L->params, s));
            if (timing) ck(cudaEventRecord(L->ev[11], s), "event");
            if (two_pass) LCHK(launch_combine(D, W, L->params, s));
        }
        if (two_pass && !prehashed) ck(cudaStreamWaitEvent(s, L->fork_ev[1], 0), "join");
        if (timing) ck(cudaEventRecord(L->ev[1], s), "event");
        // H2 group-by (round 0): two-pass -- every payload by its full digest; fused -- small
        // payloads by their first 32 bytes, large ones by their first-chunk digest
        uint64_t cap = std::max<uint64_t>(1024, pow2_at_least(2 * std::max<uint64_t>(n, 1)));
        // fused round 0 with labels: the lookup also writes the speculative labels and the
        // per-site sums (H5 + H6 need no pass after H3 unless H3 finds residuals)
        const bool lab0 = label && !two_pass && D.n && label_fused_ok(W, L->params, ns);
        LCHK(launch_group(D, W, L->params, nullptr, D.n, cap, two_pass ? -1 : 0, W.res[0], s, false, lab0 ? ns : 0,
                          lab0 ? d_dup : nullptr));
        if (h_spec) {
            // speculative labels, copied to the host on the copy stream during H3
            if (!lab0) LCHK(launch_spec_label(D, W, d_dup, s));
            ck(cudaEventRecord(L->copy_ev[0], s), "event");
            ck(cudaStreamWaitEvent(L->copy_stream, L->copy_ev[0], 0), "fork copy");
            ck(cudaMemcpyAsync(h_spec, d_dup, (uint64_t)D.n * sizeof(int64_t), cudaMemcpyDeviceToHost,
                               L->copy_stream),
               "D2H dup (speculative)");
            ck(cudaEventRecord(L->copy_ev[1], L->copy_stream), "event");
        }
        if (timing) ck(cudaEventRecord(L->ev[2], s), "event");
        if (two_pass) {
            // H3 (two-pass): every member byte-verified against its full-digest candidate
            if (timing) ck(cudaEventRecord(L->ev[16], s), "event");
            LCHK(launch_verify(D, W, L->params, nullptr, D.n, W.res[0], n_large ? W.vitem_cap : 0, s, side,
                               L->fork_ev[2], L->fork_ev[3]));
            if (timing) ck(cudaEventRecord(L->ev[17], s), "event");
        } else {
            // H1 + H3 of small payloads on the side stream (hash each, byte-compare members
            // with their prefix-group leader) while the fused pass hashes the rest of every
            // large payload and byte-compares each large member with its group leader
            ck(cudaEventRecord(L->fork_ev[2], s), "event");
            ck(cudaStreamWaitEvent(side, L->fork_ev[2], 0), "fork");
            if (timing) ck(cudaEventRecord(L->ev[12], side), "event");
            LCHK(launch_fused_small(D, W, L->params, W.res[0], side));
            if (timing) ck(cudaEventRecord(L->ev[8], side), "event");
            ck(cudaEventRecord(L->fork_ev[3], side), "event");
            // per-site sums of the lookup's block rows, off the small pass's critical path
            if (lab0)
                LCHK(launch_site_reduce(W.label_part, W.label_cpart, label_hist_rows(L->params.num_sms), ns, W.ben,
                                        W.cnt, s));
            if (n_large)
                LCHK(launch_fused(D, W, L->params, n_large, prefilter, W.res[0], s, timing ? L->ev[16] : nullptr,
                                  timing ? L->ev[17] : nullptr));
            ck(cudaStreamWaitEvent(s, L->fork_ev[3], 0), "join");
        }
        if (timing) ck(cudaEventRecord(L->ev[3], s), "event");
        // H5 + H6 (speculative: valid unless H3 found residuals)
        if (label && !lab0) LCHK(launch_label(D, W, L->params, ns, h_spec ? nullptr : d_dup, s));
        if (h_spec) ck(cudaStreamWaitEvent(s, L->copy_ev[1], 0), "join copy");
        if (timing) ck(cudaEventRecord(L->ev[4], s), "event");
        ck(cudaMemcpyAsync(L->h_counters, W.counters, 16 * sizeof(uint32_t), cudaMemcpyDeviceToHost, s), "D2H");
    };
    // (per-stage timing needs directly recorded events: FFM_FLAG_TIMING runs launch directly)
    // An online window (window) is captured only with a slot of its own (wslot): the
    // captured step then spans pre_a (the window's metadata gather and order build),
    // segment A and pre_sync (the match against the stored classes); its key is the
    // caller's (wextra: buffer generation, window size, outputs), not the log's epoch.
    const bool graph = !prehashed && (!window || wslot) && !(L->cfg.flags & FFM_FLAG_NO_GRAPH) && !timing;
    const bool in_graph_sync = graph && window;
    auto body = [&]() {
        if (pre_a) (*pre_a)();
        segment_a();
        if (in_graph_sync && pre_sync) (*pre_sync)();
    };
    if (graph) {
        // replay a CUDA graph of segment A while the log, its buffers and the run mode are
        // unchanged: one launch instead of ~30 (launch-bound small logs)
        GraphSlot& G = window ? *wslot : L->graph;
        GraphKey key{window ? ~0ull : L->epoch, d_dup, h_spec, two_pass, prefilter, timing};
        if (wextra)
            for (int i = 0; i < GraphKey::kExtra; ++i) key.extra[i] = wextra[i];
        if (!G.exec || !(key == G.key)) {
            uint64_t before = launches;
            ck(cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed), "begin capture");
            try {
                body();
            } catch (...) {
                cudaGraph_t g = nullptr;
                cudaStreamEndCapture(s, &g);
                if (g) cudaGraphDestroy(g);
                cudaGetLastError();
                throw;
            }
            cudaGraph_t g = nullptr;
            ck(cudaStreamEndCapture(s, &g), "end capture");
            // same topology (e.g. the next window of another size): update the executable
            // graph in place, much cheaper than instantiating it again
            cudaGraphExecUpdateResultInfo info;
            cudaError_t e = cudaErrorUnknown;
            if (G.exec) {
                e = cudaGraphExecUpdate(G.exec, g, &info);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    cudaGraphExecDestroy(G.exec);
                    G.exec = nullptr;
                }
            }
            if (!G.exec) e = cudaGraphInstantiate(&G.exec, g, 0);
            cudaGraphDestroy(g);
            ck(e, "graph instantiate");
            G.key = key;
            G.launches = launches - before;
            launches = before;
        }
        ck(cudaGraphLaunch(G.exec, s), "graph launch");
        launches += G.launches;
    } else {
        body();
    }
    if (pre_sync && !in_graph_sync) (*pre_sync)();
    sync_run(L, "run sync");
    R.n_members = L->h_counters[1];
    R.two_pass = two_pass;
    R.prefilter_rest = (uint64_t)L->h_counters[4] | ((uint64_t)L->h_counters[5] << 32);
    uint64_t nres = L->h_counters[0];
    R.n_res_total = nres;
    R.n_res0 = nres;
    // (the caller fixes up work it queued on the speculative labels: keep the list, the
    // resolve rounds reuse the residual buffers)
    if (nres && keep_res)
        ck(cudaMemcpyAsync(keep_res, W.res[0], nres * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s), "keep residuals");
    if (nres) {
        // H4 collision resolution: exact classes among the residual members
        if (timing) ck(cudaEventRecord(L->ev[6], s), "event");
        // a fused round 0 hashed no small member: the residual ones are hashed now
        if (!two_pass && D.n_small) LCHK(launch_hash_small_list(D, W, L->params, W.res[0], (uint32_t)nres, s));
        int cur = 0;
        while (nres) {
            ++R.rounds;
            if (R.rounds > n + 2) throw CudaFail{cudaErrorUnknown, "collision resolution did not converge"};
            ck(cudaMemsetAsync(W.counters, 0, 16 * sizeof(uint32_t), s), "memset");
            uint64_t capr = std::max<uint64_t>(1024, pow2_at_least(2 * nres));
            // after a fused round 0 a large residual is first matched against its new
            // leader through their difference lists (exact, no payload bytes re-read)
            LCHK(launch_group(D, W, L->params, W.res[cur], (uint32_t)nres, capr, (int)R.rounds, W.res[cur ^ 1], s,
                              !two_pass));
            LCHK(launch_verify(D, W, L->params, W.res[cur], (uint32_t)nres, W.res[cur ^ 1],
                               n_large ? W.vitem_cap : 0, s, nullptr, nullptr, nullptr));
            ck(cudaMemcpyAsync(L->h_counters, W.counters, 16 * sizeof(uint32_t), cudaMemcpyDeviceToHost, s), "D2H");
            sync_run(L, "round sync");
            nres = L->h_counters[0];
            R.n_reread += L->h_counters[10];
            if (R.rounds == 1) R.n_overflow = L->h_counters[11];
            R.n_res_total += nres;
            cur ^= 1;
        }
        if (label) LCHK(launch_label(D, W, L->params, ns, d_dup, s));
        if (timing) ck(cudaEventRecord(L->ev[7], s), "event");
        R.spec_stale = h_spec != nullptr;
    }
    return R;
}

void fill_stats(ffm_log* L, const LocalRun& R, uint64_t launches, bool single) {
    const bool timing = (L->cfg.flags & FFM_FLAG_TIMING) != 0;
    ffm_run_stats& S = L->stats;
    memset(&S, 0, sizeof(S));
    S.n_records = L->h_size.size();
    S.payload_bytes = L->payload_bytes;
    S.n_members = R.n_members;
    S.n_residual = R.n_res_total;
    S.resolve_rounds = R.rounds;
    S.kernel_launches = launches;
    S.hash_items = L->n_large_chunks;
    S.prefilter_rest_bytes = R.prefilter_rest;
    S.two_pass = R.two_pass ? 1 : 0;
    S.n_reread = R.n_reread;
    if (timing) {
        S.ms_hash_small = ev_ms(L->ev[12], L->ev[8]);
        S.ms_hash_large = L->n_large_chunks ? ev_ms(L->ev[10], L->ev[11]) : 0.0;
        S.ms_fused = L->n_large_chunks ? ev_ms(L->ev[16], L->ev[17]) : 0.0;
        S.ms_hash = ev_ms(L->ev[0], L->ev[1]);
        S.ms_group = ev_ms(L->ev[1], L->ev[2]);
        S.ms_verify = ev_ms(L->ev[2], L->ev[3]);
        S.ms_label = single ? ev_ms(L->ev[3], L->ev[4]) : 0.0;
        S.ms_resolve = R.rounds ? ev_ms(L->ev[6], L->ev[7]) : 0.0;
        if (single) {
            S.ms_output = ev_ms(L->ev[9], L->ev[5]);
            S.ms_total = ev_ms(L->ev[0], L->ev[5]);
        }
    }
    L->digests_valid = true;
}


// ---------------------------------------------------------------- sharded runs
// (zeroed on the run stream: the legacy-stream cudaMemset does not order before kernels
// on the library's non-blocking streams)
template <class T>
void dev_alloc_zero(T*& p, uint64_t count, cudaStream_t st) {
    dev_alloc(p, count);
    ck(cudaMemsetAsync(p, 0, std::max<uint64_t>(count, 1) * sizeof(T), st), "memset");
}

void ensure_cub(ffm_log* L, uint64_t n) {
    size_t cb = cub_scan_bytes(n);
    if (cb > L->work.cub_tmp_bytes) {
        if (L->work.cub_tmp) cudaFree(L->work.cub_tmp);
        L->work.cub_tmp = nullptr;
        ck(cudaMalloc(&L->work.cub_tmp, cb), "cudaMalloc(cub)");
        L->work.cub_tmp_bytes = cb;
    }
}

// Buffers of the merge: n local records, M representatives of all ranks, nloc of them
// this rank's, vcap verify work units.
void ensure_shard(ffm_log* L, uint64_t n, uint64_t M, uint64_t nloc, uint64_t vcap, int world) {
    ShardWork& S = L->shard;
    if (n + 1 > S.n_cap || !S.flag) {
        uint64_t c = std::max<uint64_t>(n + 1, 1024);
        dev_alloc(S.flag, c);
        dev_alloc(S.rep_idx, c);
        S.n_cap = c;
        ensure_cub(L, c);
    }
    uint64_t cap = std::max<uint64_t>(1024, pow2_at_least(2 * std::max<uint64_t>(M, 1)));
    if (cap > S.t_cap) {
        dev_alloc(S.tkey, cap);
        dev_alloc(S.tgid, cap);
        dev_alloc(S.tidx, cap);
        dev_alloc_zero(S.need, cap, L->stream);   // zero between runs (k_seg_clear)
        dev_alloc_zero(S.scnt, cap, L->stream);
        dev_alloc(S.sbase, cap);
        dev_alloc(S.sfill, cap);
        S.t_cap = cap;
    }
    if (M > S.m_cap || !S.tslot) {
        uint64_t c = std::max<uint64_t>(M, 1024);
        dev_alloc(S.tslot, c);
        dev_alloc(S.seg, c);
        S.m_cap = c;
    }
    if (nloc + 1 > S.l_cap || !S.state) {
        uint64_t c = std::max<uint64_t>(nloc + 1, 1024);
        dev_alloc(S.state, c);
        dev_alloc(S.cand, c);
        dev_alloc(S.vcount, c);
        dev_alloc(S.vstart, c);
        dev_alloc(S.G, c);
        dev_alloc(S.slow_list, c);
        S.l_cap = c;
        ensure_cub(L, c);
    }
    if (vcap > S.v_cap || !S.vitems) {
        uint64_t c = std::max<uint64_t>(vcap, 1024);
        dev_alloc(S.vitems, c);
        S.v_cap = c;
    }
    if ((uint64_t)world > S.w_cap || !S.rank_lo) {
        dev_alloc(S.rank_lo, world);
        dev_alloc(S.bases, world);
        if (!S.sctr) dev_alloc(S.sctr, 4);
        S.w_cap = world;
    }
}

void free_shard(ShardWork& S) {
    void* ptrs[] = {S.flag, S.rep_idx, S.tkey, S.tgid, S.tidx, S.need, S.scnt, S.sbase, S.sfill, S.tslot, S.seg,
                    S.state, S.cand, S.vcount, S.vstart, S.G, S.slow_list, S.vitems, S.rank_lo, (void*)S.bases, S.sctr};
    for (void* p : ptrs)
        if (p) cudaFree(p);
}

void comm_ck(ffm_log* L, int rc) {
    if (rc == FFM_OK) return;
    if (rc == FFM_E_CUDA) throw CudaFail{cudaErrorUnknown, L->comm.err.c_str()};
    throw CommFail{rc, L->comm.err};
}

// grow a tuple buffer keeping its first `keep` entries (stream-ordered copy)
void grow_tuples(ffm_log* L, RepTuple*& p, uint64_t& cap, uint64_t need, uint64_t keep) {
    if (need <= cap && p) return;
    RepTuple* np = nullptr;
    const uint64_t c = std::max<uint64_t>(std::max<uint64_t>(need, 1024), cap + cap / 2);
    ck(cudaMalloc(&np, c * sizeof(RepTuple)), "cudaMalloc(reps)");
    if (p && keep) ck(cudaMemcpyAsync(np, p, keep * sizeof(RepTuple), cudaMemcpyDeviceToDevice, L->stream), "copy");
    ck(cudaStreamSynchronize(L->stream), "grow sync");
    if (p) ck(cudaFree(p), "cudaFree");
    p = np;
    cap = c;
}

// Peer arenas (CUDA IPC).  The handles travel through the exchange transport whenever
// some rank's arena generation changed since the last exchange -- a decision every rank
// takes identically from the all-gathered headers (collective).  A peer's arena is
// mapped only while it has representatives (a rank with none is never read).
void map_peers(ffm_log* L, const std::vector<uint64_t>& gens, const std::vector<uint64_t>& counts) {
    const int world = L->cfg.world, rank = L->cfg.rank;
    if (L->xgen != gens) {
        cudaIpcMemHandle_t h;
        static_assert(sizeof(h) == 64, "IPC handle size");
        ck(cudaIpcGetMemHandle(&h, L->arena), "cudaIpcGetMemHandle");
        uint8_t* hh = reinterpret_cast<uint8_t*>(L->h_hdr + 8 + 4 * (uint64_t)world);   // pinned scratch
        memcpy(hh, &h, 64);
        ck(cudaMemcpyAsync(L->d_ipc, hh, 64, cudaMemcpyHostToDevice, L->stream), "H2D");
        comm_ck(L, comm_allgather(L->comm, L->d_ipc, L->d_ipc + 64, 64, L->stream));
        ck(cudaMemcpyAsync(hh, L->d_ipc + 64, 64 * (uint64_t)world, cudaMemcpyDeviceToHost, L->stream), "D2H");
        sync_run(L, "handle exchange sync");
        L->xhandles.assign(hh, hh + 64 * (size_t)world);
        L->xgen = gens;
    }
    L->peer_ptr.resize(world, nullptr);
    L->peer_gen.resize(world, ~0ull);
    for (int r = 0; r < world; ++r) {
        if (r == rank || counts[r] == 0 || (L->peer_ptr[r] && L->peer_gen[r] == gens[r])) continue;
        if (L->peer_ptr[r]) ck(cudaIpcCloseMemHandle(L->peer_ptr[r]), "cudaIpcCloseMemHandle");
        L->peer_ptr[r] = nullptr;
        cudaIpcMemHandle_t ph;
        memcpy(&ph, L->xhandles.data() + 64ull * r, 64);
        void* p = nullptr;
        ck(cudaIpcOpenMemHandle(&p, ph, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
        L->peer_ptr[r] = p;
        L->peer_gen[r] = gens[r];
    }
}

// One collective run of a sharded log (include/ffm.h "Sharded logs"): local H1..H4 with
// the representative export and the header exchange queued before the first sync; then
// the representative all-gather, the merge (global group-by, peer-memory verify, slow
// segments decided on the device), labels, the all-reduce of the per-site sums and the
// outputs before the second.
void run_sharded(ffm_log* L, int64_t* dup_out, uint64_t* ben_out, bool dup_dev, bool ben_dev, LocalRun& R,
                 uint64_t& launches) {
    const int world = L->cfg.world, rank = L->cfg.rank;
    const uint64_t n = L->h_size.size();
    const uint32_t ns = L->cfg.n_sites;
    Work& W = L->work;
    ShardWork& S = L->shard;
    cudaStream_t s = L->stream;
    const bool timing = (L->cfg.flags & FFM_FLAG_TIMING) != 0;
    ensure_shard(L, n, 1, 1, 1, world);
    grow_tuples(L, L->d_send, L->send_cap, std::max<uint64_t>(n, 1), 0);
    const DevLog D = dev_view(L);
    const std::function<void()> exchange_header = [&]() {
        LCHK(launch_rep_export(D, W, S, L->params, L->d_send, s));
        LCHK(launch_shard_header(S.rep_idx + n, W.counters, L->arena_gen, n, L->d_hdr, s));
        comm_ck(L, comm_allgather(L->comm, L->d_hdr, L->d_hdr + 4, 4 * sizeof(uint64_t), s));
        ck(cudaMemcpyAsync(L->h_hdr, L->d_hdr + 4, 32 * (uint64_t)world, cudaMemcpyDeviceToHost, s), "D2H");
    };
    // sync 1: local classes (speculative export: valid unless some rank had residuals)
    R = run_local(L, D, L->n_large_chunks, launches, false, nullptr, false, &exchange_header);
    bool any_res = false;
    for (int r = 0; r < world; ++r) any_res |= L->h_hdr[4 * r + 1] != 0;
    if (any_res) {   // every rank re-exports its final classes (collective)
        exchange_header();
        sync_run(L, "header sync");
    }
    if (timing) ck(cudaEventRecord(L->ev[13], s), "event");
    std::vector<uint64_t> counts(world), gens(world);
    std::vector<uint32_t> rank_lo(world);
    uint64_t M = 0, maxc = 0;
    for (int r = 0; r < world; ++r) {
        counts[r] = L->h_hdr[4 * r];
        gens[r] = L->h_hdr[4 * r + 2];
        rank_lo[r] = (uint32_t)M;
        M += counts[r];
        maxc = std::max(maxc, counts[r]);
    }
    if (M >= 0xFFFFFFFFull) throw CommFail{FFM_E_RANGE, "too many representatives"};
    map_peers(L, gens, counts);
    const uint64_t nloc = counts[rank], lo = rank_lo[rank];
    ensure_shard(L, n, M, nloc, nloc + L->n_large_chunks + 64, world);
    // all-gather of the representatives (padded to the largest count), compacted rank-major
    grow_tuples(L, L->d_send, L->send_cap, std::max<uint64_t>(maxc, 1), nloc);
    grow_tuples(L, L->d_recv, L->recv_cap, std::max<uint64_t>(maxc * world, 1), 0);
    grow_tuples(L, L->d_T, L->T_cap, std::max<uint64_t>(M, 1), 0);
    if (maxc) comm_ck(L, comm_allgather(L->comm, L->d_send, L->d_recv, maxc * sizeof(RepTuple), s));
    for (int r = 0; r < world; ++r)
        if (counts[r])
            ck(cudaMemcpyAsync(L->d_T + rank_lo[r], L->d_recv + maxc * r, counts[r] * sizeof(RepTuple),
                               cudaMemcpyDeviceToDevice, s),
               "compact reps");
    // rank tables (pinned staging: the copies stay asynchronous)
    uint32_t* h_lo = reinterpret_cast<uint32_t*>(L->h_hdr + 8 + 4 * (uint64_t)world + 8 * (uint64_t)world);
    const uint8_t** h_bases = reinterpret_cast<const uint8_t**>(h_lo + world + (world & 1));
    for (int r = 0; r < world; ++r) {
        h_lo[r] = rank_lo[r];
        h_bases[r] = r == rank ? L->arena : (const uint8_t*)L->peer_ptr[r];
    }
    ck(cudaMemcpyAsync(S.rank_lo, h_lo, world * sizeof(uint32_t), cudaMemcpyHostToDevice, s), "H2D");
    ck(cudaMemcpyAsync((void*)S.bases, h_bases, world * sizeof(void*), cudaMemcpyHostToDevice, s), "H2D");
    const uint64_t cap = std::max<uint64_t>(1024, pow2_at_least(2 * std::max<uint64_t>(M, 1)));
    LCHK(launch_merge(D, W, S, L->params, L->d_T, (uint32_t)M, (uint32_t)lo, (uint32_t)nloc, world, rank, cap, s));
    int64_t* d_dup = dup_dev ? dup_out : W.dup;
    LCHK(launch_merge_label(D, W, S, L->params, ns, d_dup, s));
    // per-site benefit and duplicate counts ([ben | cnt], contiguous) summed over ranks
    comm_ck(L, comm_allreduce_u64(L->comm, W.ben, 2 * (uint64_t)ns, s));
    if (!dup_dev && n)
        ck(cudaMemcpyAsync(dup_out, d_dup, n * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "D2H dup");
    if (ben_out)
        ck(cudaMemcpyAsync(ben_out, W.ben, ns * sizeof(uint64_t),
                           ben_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s),
           "copy ben");
    ck(cudaMemcpyAsync(L->h_hdr + 4 * (uint64_t)world, S.sctr, 4 * sizeof(uint64_t), cudaMemcpyDeviceToHost, s),
       "D2H");
    if (timing) ck(cudaEventRecord(L->ev[14], s), "event");
    // sync 2: outputs written; every peer finished reading this rank's arena (its
    // compare kernels precede its part of the all-reduce)
    sync_run(L, "sharded output sync");
    ck(cudaGetLastError(), "sharded run");
    fill_stats(L, R, launches, false);
    L->stats.n_reps_local = nloc;
    L->stats.n_reps_global = M;
    L->stats.n_slow = L->h_hdr[4 * world];
    L->stats.remote_verify_bytes = L->h_hdr[4 * world + 2];
    L->stats.n_residual += L->stats.n_slow;
    L->stats.exchange_bytes = L->comm.bytes_moved;
    if (timing) {
        L->stats.ms_exchange = ev_ms(L->ev[13], L->ev[14]);
        L->stats.ms_total = ev_ms(L->ev[0], L->ev[14]);
    }
}

}  // namespace

// ======================================================================== ABI
extern "C" {

void ffm_config_init(ffm_config* cfg) {
    if (!cfg) return;
    memset(cfg, 0, sizeof(*cfg));
    cfg->n_sites = 1;
    cfg->world = 1;
    cfg->digest_bits = 64;
    cfg->refine_bits = 64;
}

const char* ffm_version(void) { return "ffm 0.1 sm_100a"; }

const char* ffm_strerror(int s) {
    switch (s) {
        case FFM_OK: return "ok";
        case FFM_E_INVAL: return "invalid argument";
        case FFM_E_RANGE: return "argument out of range";
        case FFM_E_NOMEM: return "out of memory";
        case FFM_E_CUDA: return "CUDA error";
        case FFM_E_COMM: return "shard exchange error";
        case FFM_E_STATE: return "invalid state (poisoned handle)";
        case FFM_E_NODEV: return "no CUDA device";
        default: return "unknown status";
    }
}

const char* ffm_last_error(const ffm_log* log) { return log ? log->last_error.c_str() : ""; }

int ffm_log_create(const ffm_config* cfg, ffm_log** out) {
    if (!cfg || !out) return FFM_E_INVAL;
    *out = nullptr;
    if (cfg->n_sites == 0 || cfg->digest_bits > 64 || cfg->refine_bits > 64 || cfg->world < 1 ||
        cfg->rank < 0 || cfg->rank >= cfg->world)
        return FFM_E_INVAL;
    if ((cfg->world > 1 && (cfg->nccl_id == nullptr) == (cfg->comm == nullptr)) || (cfg->nccl_id && cfg->comm))
        return FFM_E_INVAL;   // a sharded log needs exactly one exchange transport
    uint32_t chunk = cfg->chunk_bytes ? cfg->chunk_bytes : 32768;
    uint32_t small = cfg->small_bytes ? cfg->small_bytes : 4096;
    if (chunk % 1024 || small % 128 || chunk == 0) return FFM_E_INVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return FFM_E_NODEV;
    }
    if (cfg->device < 0 || cfg->device >= ndev) return FFM_E_INVAL;
    ffm_log* L = new (std::nothrow) ffm_log();
    if (!L) return FFM_E_NOMEM;
    L->cfg = *cfg;
    L->device = cfg->device;
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        int prop_major = 0;
        ck(cudaDeviceGetAttribute(&prop_major, cudaDevAttrComputeCapabilityMajor, L->device), "attr");
        if (prop_major < 10) {
            delete L;
            return FFM_E_NODEV;   // built for sm_100a only
        }
        ck(cudaDeviceGetAttribute(&L->params.num_sms, cudaDevAttrMultiProcessorCount, L->device), "attr");
        ck(cudaDeviceGetAttribute(&L->params.max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, L->device), "attr");
        int hp = 0;
        ck(cudaDeviceGetAttribute(&hp, cudaDevAttrCanUseHostPointerForRegisteredMem, L->device), "attr");
        L->host_ptr_ok = hp != 0;
        L->gather_max = kGatherMax;
        L->params.prefix_bytes = std::min<uint32_t>(4096, chunk);   // a multiple of 256 (chunk: of 1024)
        L->params.chunk_bytes = chunk;
        L->params.small_bytes = small;
        L->params.digest_mask = cfg->digest_bits >= 64 ? ~0ull : ((1ull << cfg->digest_bits) - 1);
        L->params.refine_mask = cfg->refine_bits >= 64 ? ~0ull : ((1ull << cfg->refine_bits) - 1);
        if (cfg->stream) {
            L->stream = (cudaStream_t)cfg->stream;
        } else {
            ck(cudaStreamCreateWithFlags(&L->stream, cudaStreamNonBlocking), "stream");
            L->own_stream = true;
        }
        ck(cudaStreamCreateWithFlags(&L->stage_stream, cudaStreamNonBlocking), "stream");
        ck(cudaStreamCreateWithFlags(&L->side_stream, cudaStreamNonBlocking), "stream");
        ck(cudaStreamCreateWithFlags(&L->hash_stream, cudaStreamNonBlocking), "stream");
        ck(cudaStreamCreateWithFlags(&L->copy_stream, cudaStreamNonBlocking), "stream");
        for (auto& e : L->copy_ev) ck(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
        ck(cudaEventCreateWithFlags(&L->hash_ev, cudaEventDisableTiming), "event");
        ck(cudaEventRecord(L->hash_ev, L->hash_stream), "event");
        for (auto& e : L->fork_ev) ck(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
        L->ring_bytes = kRingBytes;
        for (int i = 0; i < 2; ++i) {
            ck(cudaHostAlloc((void**)&L->ring[i], kRingBytes, cudaHostAllocDefault), "cudaHostAlloc(ring)");
            ck(cudaEventCreateWithFlags(&L->ring_ev[i], cudaEventDisableTiming), "event");
            ck(cudaEventRecord(L->ring_ev[i], L->stage_stream), "event");
        }
        for (auto& e : L->ev) ck(cudaEventCreate(&e), "event");
        ck(cudaHostAlloc((void**)&L->h_counters, 16 * sizeof(uint32_t), cudaHostAllocDefault), "cudaHostAlloc");
        // a transport makes the log collective -- also a world of one (the whole collective
        // path, NCCL included, then runs on a single GPU)
        L->collective = cfg->world > 1 || cfg->nccl_id || cfg->comm;
        if (L->collective) {
            const uint64_t w = (uint64_t)cfg->world;
            ck(cudaMalloc(&L->d_hdr, (4 + 4 * w) * sizeof(uint64_t)), "cudaMalloc(hdr)");
            ck(cudaMalloc(&L->d_ipc, 64 * (w + 1)), "cudaMalloc(ipc)");
            // headers [4w] | run counters [8] | IPC handles [8w] | rank table [w u32] | bases [w]
            ck(cudaHostAlloc((void**)&L->h_hdr, (16 + 16 * w) * sizeof(uint64_t), cudaHostAllocDefault),
               "cudaHostAlloc(hdr)");
            const int rc = comm_init(L->comm, cfg->world, cfg->rank, cfg->nccl_id, cfg->comm);
            if (rc != FFM_OK) {
                ffm_log_destroy(L);
                return rc;
            }
        }
        if (cfg->arena_bytes) ensure_arena(L, cfg->arena_bytes);
        if (cfg->max_records) {
            L->h_site.reserve(cfg->max_records);
            L->h_size.reserve(cfg->max_records);
            L->h_off.reserve(cfg->max_records);
            L->h_dur.reserve(cfg->max_records);
            L->h_gid.reserve(cfg->max_records);
            L->h_chan.reserve(cfg->max_records);
            pin_meta(L, true);
        }
    } catch (const CudaFail& f) {
        int code = (f.e == cudaErrorMemoryAllocation) ? FFM_E_NOMEM : FFM_E_CUDA;
        cudaGetLastError();
        ffm_log_destroy(L);
        return code;
    } catch (const std::bad_alloc&) {
        ffm_log_destroy(L);
        return FFM_E_NOMEM;
    }
    *out = L;
    return FFM_OK;
}

int ffm_log_append_batch(ffm_log* L, uint64_t n, const uint32_t* sites, const uint64_t* sizes,
                         const void* const* payloads, const uint64_t* durs, const uint64_t* gids, int kind) {
    return ffm_log_append_batch_ex(L, n, sites, sizes, payloads, durs, gids, nullptr, kind);
}

#ifdef FFM_APPEND_TIMES
#define FFM_AT(tag) fprintf(stderr, "[append] %s %.3f ms\n", tag, std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - at0).count())
#else
#define FFM_AT(tag)
#endif
int ffm_log_append_batch_ex(ffm_log* L, uint64_t n, const uint32_t* sites, const uint64_t* sizes,
                            const void* const* payloads, const uint64_t* durs, const uint64_t* gids,
                            const uint64_t* channels, int kind) {
#ifdef FFM_APPEND_TIMES
    const auto at0 = std::chrono::steady_clock::now();
#endif
    int st = check_state(L);
    if (st) return st;
    if (n == 0) return FFM_OK;
    if (!sites || !sizes || !payloads || !durs) return set_err(L, FFM_E_INVAL, "NULL array");
    if (kind < FFM_PAYLOAD_AUTO || kind > FFM_PAYLOAD_HOST_PINNED) return set_err(L, FFM_E_INVAL, "bad payload_kind");
    std::vector<uint64_t> offs;
    uint64_t end = 0;
    int rc = plan_batch(L, n, sites, sizes, payloads, gids, offs, end);
    if (rc) return rc;
    FFM_AT("plan");
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        ensure_arena(L, end);
        // k_gather descriptors (source, arena offset, bytes), written into page-locked
        // staging (the previous append's copy of it completed: appends sync before return)
        if (3 * n > L->h_desc_cap) {
            if (L->h_desc) ck(cudaFreeHost(L->h_desc), "cudaFreeHost");
            L->h_desc = nullptr;
            const uint64_t c = std::max<uint64_t>(3 * n, 2 * L->h_desc_cap);
            ck(cudaMallocHost(&L->h_desc, c * sizeof(uint64_t)), "cudaMallocHost(desc)");
            L->h_desc_cap = c;
        }
        uint64_t nde = 0;   // descriptor words written
        bool need_sync = false, ordered = false;
        PtrCache pc;
        std::vector<PageablePiece> pageable;   // consecutive pageable records, staged together
        // a large batch of device or page-locked payloads: classified and its descriptors
        // written by the host threads in parallel (no ring staging can occur)
        const bool par = (kind == FFM_PAYLOAD_DEVICE || kind == FFM_PAYLOAD_HOST_PINNED) && n >= 65536;
        if (par) {
            if (kind == FFM_PAYLOAD_DEVICE) {
                // device payloads may still be being produced (see below)
                ordered = true;
                ck(cudaEventRecord(L->fork_ev[0], cudaStreamLegacy), "event");
                ck(cudaStreamWaitEvent(L->stage_stream, L->fork_ev[0], 0), "wait producer");
                if (L->stream != cudaStreamLegacy) {
                    ck(cudaEventRecord(L->fork_ev[1], L->stream), "event");
                    ck(cudaStreamWaitEvent(L->stage_stream, L->fork_ev[1], 0), "wait producer");
                }
            }
            if (L->ring_fill) ring_flush(L);
            std::vector<uint8_t> act(n);   // 0: nothing (empty), 1: k_gather, 2: copy engine
            const int T = stage_threads();
            std::vector<uint64_t> cnt(T + 1, 0);
            int used = 1;
            const uint64_t gmax = L->gather_max;
            const bool hp_ok = L->host_ptr_ok;
            const int mydev = L->device;
#pragma omp parallel num_threads(T)
            {
                const int t = omp_get_thread_num(), nt = omp_get_num_threads();
                const uint64_t lo = n * t / nt, hi = n * (t + 1) / nt;
                PtrCache pct;
                uint64_t c = 0;
                for (uint64_t i = lo; i < hi; ++i) {
                    if (sizes[i] == 0) {
                        act[i] = 0;
                        continue;
                    }
                    int pdev = mydev;
                    if (kind == FFM_PAYLOAD_DEVICE) {
                        int d = -1;   // (a peer GPU's memory is never dereferenced by k_gather)
                        if (pct.classify(payloads[i], &d) == FFM_PAYLOAD_DEVICE) pdev = d;
                    }
                    const bool dma = sizes[i] > gmax || (kind == FFM_PAYLOAD_HOST_PINNED && !hp_ok) ||
                                     (kind == FFM_PAYLOAD_DEVICE && pdev != mydev);
                    act[i] = dma ? 2 : 1;
                    c += !dma;
                }
                cnt[t + 1] = c;
#pragma omp barrier
#pragma omp single
                {
                    used = nt;
                    for (int k = 0; k < nt; ++k) cnt[k + 1] += cnt[k];
                }
                uint64_t k = 3 * cnt[t];
                for (uint64_t i = lo; i < hi; ++i) {
                    if (act[i] != 1) continue;
                    L->h_desc[k++] = (uint64_t)(uintptr_t)payloads[i];
                    L->h_desc[k++] = offs[i];
                    L->h_desc[k++] = sizes[i];
                }
            }
            nde = 3 * cnt[used];
            need_sync = nde != 0;
            for (uint64_t i = 0; i < n; ++i) {
                if (act[i] != 2) continue;
                need_sync = true;   // async copy engine from caller memory: sync before return
                ck(cudaMemcpyAsync(L->arena + offs[i], payloads[i], sizes[i], cudaMemcpyDefault, L->stage_stream),
                   "copy");
            }
        }
        for (uint64_t i = 0; i < (par ? 0 : n); ++i) {
            if (sizes[i] == 0) continue;
            int src = kind, pdev = L->device;
            if (kind == FFM_PAYLOAD_AUTO) {
                src = pc.classify(payloads[i], &pdev);
            } else if (kind == FFM_PAYLOAD_DEVICE) {
                int d = -1;   // which GPU (a peer GPU's memory is never dereferenced by k_gather)
                if (pc.classify(payloads[i], &d) == FFM_PAYLOAD_DEVICE) pdev = d;
            }
            const bool ring = src == FFM_PAYLOAD_HOST;        // pageable host: via the pinned ring
            if (src == FFM_PAYLOAD_DEVICE && !ordered) {
                // device payloads may still be being produced: the staging stream waits for
                // the log's stream and the legacy default stream first (ffm.h)
                ordered = true;
                ck(cudaEventRecord(L->fork_ev[0], cudaStreamLegacy), "event");
                ck(cudaStreamWaitEvent(L->stage_stream, L->fork_ev[0], 0), "wait producer");
                if (L->stream != cudaStreamLegacy) {
                    ck(cudaEventRecord(L->fork_ev[1], L->stream), "event");
                    ck(cudaStreamWaitEvent(L->stage_stream, L->fork_ev[1], 0), "wait producer");
                }
            }
            // the ring uploads one contiguous arena range: close it before a record that
            // is written into the arena by another path
            if (!ring) {
                stage_pageable(L, pageable);
                pageable.clear();
                if (L->ring_fill) ring_flush(L);
            }
            if (ring) {
                if (n == 1) stage_host(L, payloads[i], sizes[i], offs[i]);   // single appends: the ring
                else pageable.push_back({(const uint8_t*)payloads[i], offs[i], sizes[i]});
            } else if (sizes[i] > L->gather_max || (src == FFM_PAYLOAD_HOST_PINNED && !L->host_ptr_ok) ||
                       (src == FFM_PAYLOAD_DEVICE && pdev != L->device)) {
                // (a payload on another GPU: the copy engines, never a kernel dereference)
                need_sync = true;     // async copy engine from caller memory: sync before return
                ck(cudaMemcpyAsync(L->arena + offs[i], payloads[i], sizes[i], cudaMemcpyDefault, L->stage_stream),
                   "copy");
            } else {
                need_sync = true;     // k_gather reads caller memory (HBM, or pinned host over PCIe)
                L->h_desc[nde++] = (uint64_t)(uintptr_t)payloads[i];
                L->h_desc[nde++] = offs[i];
                L->h_desc[nde++] = sizes[i];
            }
        }
        stage_pageable(L, pageable);
        FFM_AT("staging loop");
        if (nde) {
            uint64_t nd = nde / 3;
            uint64_t cap = L->desc_cap;
            if (nde > cap) {
                ck(cudaStreamSynchronize(L->stage_stream), "desc grow");
                if (L->d_desc) ck(cudaFree(L->d_desc), "cudaFree");
                L->d_desc = nullptr;
                cap = std::max<uint64_t>(nde, 2 * cap);
                ck(cudaMalloc(&L->d_desc, cap * sizeof(uint64_t)), "cudaMalloc(desc)");
                L->desc_cap = cap;
            }
            ck(cudaMemcpyAsync(L->d_desc, L->h_desc, nde * 8, cudaMemcpyHostToDevice, L->stage_stream), "desc H2D");
            if (launch_gather(L->d_desc, (uint32_t)nd, L->arena, L->stage_stream) < 0)
                throw CudaFail{cudaGetLastError(), "k_gather"};
        }
        FFM_AT("desc + gather queued");
        push_meta(L, n, sites, sizes, durs, gids, channels, offs, end);
        FFM_AT("push_meta");
        L->digests_valid = false;
        if (L->cfg.flags & FFM_FLAG_ONLINE) {
            // online mode: the new records' metadata goes to the device now, overlapping
            // the payload gather (the step starts from a resident window)
            ring_flush(L);
            upload_meta_arrays(L);
            need_sync = true;
        }
        FFM_AT("meta upload queued");
        if (need_sync) ck(cudaStreamSynchronize(L->stage_stream), "append sync");   // snapshot before return
        FFM_AT("synced");
        if ((L->cfg.flags & FFM_FLAG_ONLINE) && (L->cfg.flags & FFM_FLAG_APPEND_HASH)) {
            // append-time hashing: hash the new records now, on the hashing stream after
            // their staging copies -- the next append's staging overlaps this hashing
            ensure_work(L, L->h_size.size());
            ck(cudaEventRecord(L->fork_ev[2], L->stage_stream), "event");
            ck(cudaStreamWaitEvent(L->hash_stream, L->fork_ev[2], 0), "wait staging");
            uint64_t launches = 0;
            const uint64_t a = std::max(L->online_hashed, L->online_done), b = L->h_size.size();
            online_hash(L, a, b, L->hash_stream, launches);
            ck(cudaEventRecord(L->hash_ev, L->hash_stream), "event");
            L->online_hashed = b;
        }
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    } catch (const std::bad_alloc&) {
        return set_err(L, FFM_E_NOMEM, "host allocation failed");
    }
    return FFM_OK;
}

int ffm_log_append(ffm_log* L, uint32_t site, uint64_t size, const void* payload, uint64_t dur) {
    const void* p[1] = {payload};
    return ffm_log_append_batch(L, 1, &site, &size, p, &dur, nullptr, FFM_PAYLOAD_AUTO);
}

uint64_t ffm_log_count(const ffm_log* L) { return L ? (uint64_t)L->h_size.size() : 0; }
uint64_t ffm_log_payload_bytes(const ffm_log* L) { return L ? L->payload_bytes : 0; }
void* ffm_log_stream(const ffm_log* L) { return L ? (void*)L->stream : nullptr; }

int ffm_last_run_stats(const ffm_log* L, ffm_run_stats* out) {
    if (!L || !out) return FFM_E_INVAL;
    *out = L->stats;
    return FFM_OK;
}

int ffm_dedup_run(ffm_log* L, int64_t* dup_out, uint64_t* ben_out) {
    int st = check_state(L);
    if (st) return st;
    uint64_t n = L->h_size.size();
    if (n > 0 && !dup_out) return set_err(L, FFM_E_INVAL, "duplicate_of is NULL");
    try {
        L->n_syncs = 0;
        L->comm.bytes_moved = 0;
        run_prologue(L);
        Work& W = L->work;
        cudaStream_t s = L->stream;
        const uint32_t ns = L->cfg.n_sites;
        bool dup_dev = dup_out && is_device_ptr(dup_out);
        bool ben_dev = ben_out && is_device_ptr(ben_out);
        int64_t* d_dup = dup_dev ? dup_out : W.dup;
        uint64_t launches = 0;
        if (L->collective) {
            LocalRun R{};
            run_sharded(L, dup_out, ben_out, dup_dev, ben_dev, R, launches);
            L->stats.host_syncs = L->n_syncs;
            return FFM_OK;
        }
        const bool prefilter = (L->cfg.flags & FFM_FLAG_PREFILTER) != 0;
        // pinned host output: the labels travel over PCIe while H3 streams HBM
        const bool spec = !dup_dev && n && is_pinned_host(dup_out);
        LocalRun R = run_local(L, dev_view(L), L->n_large_chunks, launches, true, d_dup, prefilter, nullptr, false,
                               spec ? dup_out : nullptr);
        // H7 return
        const bool timing = (L->cfg.flags & FFM_FLAG_TIMING) != 0;
        if (timing) ck(cudaEventRecord(L->ev[9], s), "event");
        if (!dup_dev && n && (!spec || R.spec_stale))
            ck(cudaMemcpyAsync(dup_out, d_dup, n * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "D2H dup");
        if (ben_out)
            ck(cudaMemcpyAsync(ben_out, W.ben, ns * sizeof(uint64_t),
                               ben_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s),
               "copy ben");
        if (timing) ck(cudaEventRecord(L->ev[5], s), "event");
        sync_run(L, "output sync");
        ck(cudaGetLastError(), "run");
        fill_stats(L, R, launches, true);
        L->stats.host_syncs = L->n_syncs;
        // adaptive round 0: more than half of the candidates failed the fused compare
        // (near-duplicates sharing first chunks) -> hash-all-then-verify is cheaper
        // (residuals settled through difference lists cost no re-read: what counts are the
        // members compared again, or residuals that differ from their head in many words --
        // each of those pays the fused pass's mismatch path on every piece)
        if (!R.two_pass && R.n_members >= 64 && 2 * std::max(R.n_reread, R.n_overflow) > R.n_members)
            L->prefer_two_pass = true;
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    } catch (const CommFail& f) {
        // an exchange failed part-way through a collective: the ranks are out of step
        L->poisoned = true;
        return set_err(L, f.code, f.what);
    } catch (const std::bad_alloc&) {
        return set_err(L, FFM_E_NOMEM, "host allocation failed");
    }
    return FFM_OK;
}

int ffm_nccl_unique_id(void* id_out) {
    if (!id_out) return FFM_E_INVAL;
    return comm_unique_id(id_out);
}

int ffm_site_duplicate_counts(ffm_log* L, uint64_t* counts_out) {
    int st = check_state(L);
    if (st) return st;
    if (!counts_out) return FFM_E_INVAL;
    if (!L->digests_valid || !L->work.cnt) return set_err(L, FFM_E_STATE, "no run since the last append");
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        ck(cudaMemcpyAsync(counts_out, L->work.cnt, L->cfg.n_sites * sizeof(uint64_t), cudaMemcpyDefault,
                           L->stream),
           "copy counts");
        ck(cudaStreamSynchronize(L->stream), "sync");
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    }
    return FFM_OK;
}

int ffm_fold_sites(ffm_log* L, const uint64_t* site_values, const uint32_t* site_to_group, uint32_t n_groups,
                   uint64_t* group_values_out) {
    int st = check_state(L);
    if (st) return st;
    const uint32_t ns = L->cfg.n_sites;
    if (!site_values || !site_to_group || !group_values_out || n_groups == 0) return FFM_E_INVAL;
    std::vector<uint32_t> map(ns);
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        cudaStream_t s = L->stream;
        ck(cudaMemcpy(map.data(), site_to_group, ns * sizeof(uint32_t), cudaMemcpyDefault), "copy map");
        for (uint32_t i = 0; i < ns; ++i)
            if (map[i] >= n_groups) return set_err(L, FFM_E_RANGE, "site_to_group[s] >= n_groups");
        uint64_t need = (uint64_t)ns * 8 + (uint64_t)ns * 4 + (uint64_t)n_groups * 8;
        if (need > L->fold_cap) {
            if (L->fold_buf) ck(cudaFree(L->fold_buf), "cudaFree");
            L->fold_buf = nullptr;
            ck(cudaMalloc(&L->fold_buf, need), "cudaMalloc(fold)");
            L->fold_cap = need;
        }
        uint64_t* d_vals = (uint64_t*)L->fold_buf;
        uint64_t* d_out = d_vals + ns;
        uint32_t* d_map = (uint32_t*)(d_out + n_groups);
        ck(cudaMemcpyAsync(d_vals, site_values, ns * 8, cudaMemcpyDefault, s), "copy vals");
        ck(cudaMemcpyAsync(d_map, map.data(), ns * 4, cudaMemcpyHostToDevice, s), "copy map");
        if (launch_fold(d_vals, d_map, ns, d_out, n_groups, s) < 0) throw CudaFail{cudaGetLastError(), "k_fold"};
        ck(cudaMemcpyAsync(group_values_out, d_out, (uint64_t)n_groups * 8, cudaMemcpyDefault, s), "copy out");
        ck(cudaStreamSynchronize(s), "fold sync");
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    } catch (const std::bad_alloc&) {
        return set_err(L, FFM_E_NOMEM, "host allocation failed");
    }
    return FFM_OK;
}

uint64_t ffm_online_done(const ffm_log* L) { return L ? L->online_done : 0; }

int ffm_online_step(ffm_log* L, int64_t* dup_out, uint64_t* ben_out, uint64_t* n_out) {
    int st = check_state(L);
    if (st) return st;
    if (L->collective) return set_err(L, FFM_E_STATE, "online mode is single-log (no exchange transport)");
    const uint64_t n = L->h_size.size(), w0 = L->online_done, nw = n - w0;
    if (nw && !dup_out) return set_err(L, FFM_E_INVAL, "duplicate_of is NULL");
    const uint32_t ns = L->cfg.n_sites;
    try {
        L->n_syncs = 0;
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        Work& W = L->work;
        cudaStream_t s = L->stream;
        // H0 tail for the window only (no whole-log order: O(window) host work per step)
        ring_flush(L);
        upload_meta_arrays(L);
        ck(cudaEventRecord(L->ring_ev[L->ring_cur], L->stage_stream), "event");
        ck(cudaStreamWaitEvent(s, L->ring_ev[L->ring_cur], 0), "wait staging");
        ck(cudaStreamWaitEvent(s, L->hash_ev, 0), "wait append-time hashing");
        ensure_work(L, n);
        if (!L->online_ben) {
            ck(cudaMalloc(&L->online_ben, 2 * (uint64_t)ns * sizeof(uint64_t)), "cudaMalloc(online)");
            ck(cudaMemsetAsync(L->online_ben, 0, 2 * (uint64_t)ns * sizeof(uint64_t), s), "memset");
            L->online_cnt = L->online_ben + ns;
        }
        uint64_t launches = 0;
        LocalRun R{};
        const uint64_t n_large_w = L->n_large_chunks - L->online_chunks0;
        if (nw && nw <= kTinyWindow && !n_large_w && L->online_hashed <= w0) {
            // a tiny window (a few small records, e.g. one intercepted call): one warp labels
            // them in order against the table -- one launch, one sync
            ensure_online(L, nw);
            const bool dup_dev = is_device_ptr(dup_out);
            int64_t* d_dup = dup_dev ? dup_out : W.dup;
            const DevLog D = window_view(L, w0, n, false, s);
            LCHK(launch_online_tiny(D, L->otab, L->params, d_dup, L->online_ben, L->online_cnt, s));
            if (!dup_dev) ck(cudaMemcpyAsync(dup_out, d_dup, nw * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "D2H dup");
            ck(cudaMemcpyAsync(L->h_counters + 2, L->otab.count, sizeof(uint32_t), cudaMemcpyDeviceToHost, s), "D2H");
            if (ben_out)
                ck(cudaMemcpyAsync(ben_out, L->online_ben, ns * sizeof(uint64_t), cudaMemcpyDefault, s), "copy ben");
            sync_run(L, "online sync");
        } else if (nw) {
            const uint64_t n_small_w = L->n_small_recs - L->online_small0;
            const uint64_t n_large = n_large_w;
            const bool fused = L->online_hashed <= w0;
            ensure_online(L, nw);
            const bool dup_dev = is_device_ptr(dup_out);
            int64_t* d_dup = dup_dev ? dup_out : W.dup;
            const uint64_t* wA = fused ? W.accA : L->on_A + w0;
            const uint64_t* wB = fused ? W.accB : L->on_B + w0;
            DevLog D;
            // the window's classes against the stored classes of all earlier windows
            // ("compared to the stored hashes from prior transfers"), queued on
            // the round-0 (speculative) labels before run_local's host sync: one sync per
            // step unless H4 finds residuals (then the fix-up below)
            const std::function<void()> match = [&]() {
                LCHK(launch_online_window(D, W, wA, wB, L->otab, L->params, ns, L->on_G, d_dup, L->online_ben,
                                          L->online_cnt, s));
                if (!dup_dev)
                    ck(cudaMemcpyAsync(dup_out, d_dup, nw * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "D2H dup");
                ck(cudaMemcpyAsync(L->h_counters + 2, L->otab.count, sizeof(uint32_t), cudaMemcpyDeviceToHost, s),
                   "D2H");
                if (ben_out)
                    ck(cudaMemcpyAsync(ben_out, L->online_ben, ns * sizeof(uint64_t), cudaMemcpyDefault, s),
                       "copy ben");
            };
            if (fused) {
                // fused window (default): the batch round 0 on the window in its batch
                // record order -- each byte read once (leaders hashed, members compared with
                // their prefix-group leader), full digests for the class representatives.
                // The whole step (gather + order, segment A, match) is one captured CUDA
                // graph, replayed for the next window of the same size while no buffer
                // moved; the window's start reaches it through a device word.
                D = window_view_sorted(L, w0, n, n_small_w, s);
                *L->h_wa = w0;
                ck(cudaMemcpyAsync(L->d_wa, L->h_wa, sizeof(uint64_t), cudaMemcpyHostToDevice, s), "window start");
                const std::function<void()> order = [&]() { queue_window_order(L, D, s, launches); };
                // (captured copies need device or pinned host outputs; a window size is
                // captured the second time in a row it occurs -- a one-off size, e.g. the
                // tail of a stream, launches directly instead of paying a capture)
                const bool capt = (dup_dev || is_pinned_host(dup_out)) &&
                                  (!ben_out || is_device_ptr(ben_out) || is_pinned_host(ben_out)) &&
                                  (nw == L->last_window || (L->wgraph.exec && L->wgraph.key.extra[1] == nw));
                L->last_window = nw;
                const uint64_t extra[GraphKey::kExtra] = {L->bufgen, nw, n_small_w, n_large,
                                                          (uint64_t)(uintptr_t)dup_out, (uint64_t)(uintptr_t)ben_out};
                R = run_local(L, D, n_large, launches, false, nullptr, false, &match, false, nullptr, true, L->on_res,
                              capt ? &L->wgraph : nullptr, extra, &order);
            } else {
                // hashed at append time (FFM_FLAG_APPEND_HASH): H2..H4 from the window's NH
                // sums (the slice of on_A / on_B), two-pass, every member byte-verified
                const uint64_t h0 = std::max(L->online_hashed, w0);
                if (h0 < n) online_hash(L, h0, n, s, launches);
                L->online_hashed = n;
                D = window_view(L, w0, n, n_large != 0, s);
                uint64_t* keepA = W.accA;
                uint64_t* keepB = W.accB;
                W.accA = L->on_A + w0;
                W.accB = L->on_B + w0;
                try {
                    R = run_local(L, D, n_large, launches, false, nullptr, false, &match, true, nullptr, true,
                                  L->on_res);
                } catch (...) {
                    W.accA = keepA;
                    W.accB = keepB;
                    throw;
                }
                W.accA = keepA;
                W.accB = keepB;
            }
            if (R.n_res0) {
                // H4 changed the labels of the round-0 residuals: match their classes and
                // correct their labels and the cumulative sums
                LCHK(launch_online_fix(D, W, wA, wB, L->otab, L->params, L->on_res, (uint32_t)R.n_res0, L->on_G,
                                       d_dup, L->online_ben, L->online_cnt, s));
                if (!dup_dev)
                    ck(cudaMemcpyAsync(dup_out, d_dup, nw * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "D2H dup");
                ck(cudaMemcpyAsync(L->h_counters + 2, L->otab.count, sizeof(uint32_t), cudaMemcpyDeviceToHost, s),
                   "D2H");
                if (ben_out)
                    ck(cudaMemcpyAsync(ben_out, L->online_ben, ns * sizeof(uint64_t), cudaMemcpyDefault, s),
                       "copy ben");
                sync_run(L, "online fix-up sync");
            }
        } else {
            if (ben_out)
                ck(cudaMemcpyAsync(ben_out, L->online_ben, ns * sizeof(uint64_t), cudaMemcpyDefault, s), "copy ben");
            sync_run(L, "online sync");
        }
        ck(cudaGetLastError(), "online step");
        if (nw) L->online_np = L->h_counters[2];
        L->online_done = n;
        L->online_small0 = L->n_small_recs;
        L->online_chunks0 = L->n_large_chunks;
        fill_stats(L, R, launches, false);
        L->stats.n_records = nw;
        L->stats.host_syncs = L->n_syncs;
        L->digests_valid = false;
        if (n_out) *n_out = nw;
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    } catch (const std::bad_alloc&) {
        return set_err(L, FFM_E_NOMEM, "host allocation failed");
    }
    return FFM_OK;
}

int ffm_debug_digests(ffm_log* L, uint64_t* out) {
    int st = check_state(L);
    if (st) return st;
    if (!out) return FFM_E_INVAL;
    if (!L->digests_valid) return set_err(L, FFM_E_STATE, "no run since the last append");
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        uint64_t n = L->h_size.size();
        if (n && launch_digest_fill(dev_view(L), L->work, L->params, L->stream) < 0)
            throw CudaFail{cudaGetLastError(), "digest fill"};
        if (n) ck(cudaMemcpyAsync(out, L->work.digest, n * 8, cudaMemcpyDeviceToHost, L->stream), "D2H digests");
        ck(cudaStreamSynchronize(L->stream), "digests sync");
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    }
    return FFM_OK;
}

int ffm_log_set_flags(ffm_log* L, uint32_t flags) {
    int st = check_state(L);
    if (st) return st;
    L->cfg.flags = flags;
    return FFM_OK;
}

int ffm_log_reset(ffm_log* L) {
    int st = check_state(L);
    if (st) return st;
    try {
        ck(cudaSetDevice(L->device), "cudaSetDevice");
        ck(cudaStreamSynchronize(L->stage_stream), "reset sync");
        ck(cudaStreamSynchronize(L->hash_stream), "reset sync");
        ck(cudaStreamSynchronize(L->stream), "reset sync");
    } catch (const CudaFail& f) {
        return fail_cuda(L, f);
    }
    L->h_site.clear();
    L->h_size.clear();
    L->h_off.clear();
    L->h_dur.clear();
    L->h_gid.clear();
    L->h_chan.clear();
    L->payload_bytes = L->n_large_chunks = L->last_gid = 0;
    L->n_small_recs = L->online_small0 = L->online_chunks0 = 0;
    L->last_window = 0;   // (a new stream: its first window of a size launches directly)
    L->any_gid = false;
    L->d_meta_n = 0;
    L->d_order_n = 0;
    L->n_small = 0;
    L->n_large_rec = 0;
    L->arena_used = 0;
    L->ring_fill = 0;
    L->online_done = L->online_np = L->online_hashed = 0;
    if (L->online_ben) cudaMemsetAsync(L->online_ben, 0, 2 * (uint64_t)L->cfg.n_sites * sizeof(uint64_t), L->stream);
    if (L->otab.count) {   // an empty table (keeps its capacity)
        cudaMemsetAsync(L->otab.count, 0, sizeof(uint32_t), L->stream);
        cudaMemsetAsync(L->otab.key, 0xFF, (L->otab.mask + 1) * sizeof(uint64_t), L->stream);
        cudaMemsetAsync(L->otab.head, 0xFF, (L->otab.mask + 1) * sizeof(uint32_t), L->stream);
    }
    if (cudaStreamSynchronize(L->stream) != cudaSuccess) {
        L->poisoned = true;
        L->last_error = "reset sync failed";
        return FFM_E_CUDA;
    }
    L->digests_valid = false;
    L->prefer_two_pass = false;
    ++L->epoch;   // (no buffer moved: bufgen stays, captured window steps stay valid)
    memset(&L->stats, 0, sizeof(L->stats));
    return FFM_OK;
}

int ffm_log_destroy(ffm_log* L) {
    if (!L) return FFM_OK;
    cudaSetDevice(L->device);
    if (L->stream) cudaStreamSynchronize(L->stream);
    if (L->stage_stream) cudaStreamSynchronize(L->stage_stream);
    Work& W = L->work;
    void* ptrs[] = {W.accA, W.accB, W.key, W.digest, W.slot, W.leader, W.eq, W.mis, W.res[0], W.res[1],
                    W.lcount, W.lstart, W.gcount, W.pos, W.fhead, W.hitems, W.fitems, W.sdesc, W.hcount, W.hstart, W.hpart, W.tkey,
                    W.dup, W.ben, W.label_part, W.label_cpart, W.counters, W.cub_tmp, L->d_off, L->d_size, L->d_site, L->d_dur, L->d_gid, L->d_chan,
                    L->arena, L->d_desc, L->d_small_order};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    free_shard(L->shard);
    if (L->fold_buf) cudaFree(L->fold_buf);
    void* op[] = {L->otab.key, L->otab.head, L->otab.pool, L->otab.count, L->on_A, L->on_B, L->on_G,
                  L->on_res, L->online_ben, L->d_iota, L->d_word, L->d_wbins, L->d_wa, L->wmeta.off,
                  L->wmeta.size, L->wmeta.dur, L->wmeta.gid, L->wmeta.chan, L->wmeta.site};
    for (void* p : op)
        if (p) cudaFree(p);
    for (void* p : L->peer_ptr)
        if (p) cudaIpcCloseMemHandle(p);
    void* sp[] = {L->d_send, L->d_recv, L->d_T, L->d_hdr, L->d_ipc};
    for (void* p : sp)
        if (p) cudaFree(p);
    if (L->h_hdr) cudaFreeHost(L->h_hdr);
    comm_destroy(L->comm);
    for (int i = 0; i < 2; ++i) {
        if (L->ring[i]) cudaFreeHost(L->ring[i]);
        if (L->ring_ev[i]) cudaEventDestroy(L->ring_ev[i]);
    }
    for (auto e : L->ev)
        if (e) cudaEventDestroy(e);
    if (L->h_counters) cudaFreeHost(L->h_counters);
    if (L->h_wa) cudaFreeHost(L->h_wa);
    if (L->h_desc) cudaFreeHost(L->h_desc);
    if (L->meta_pinned) {
        void* mp[] = {L->h_site.data(), L->h_size.data(), L->h_off.data(), L->h_dur.data(), L->h_gid.data(),
                      L->h_chan.data()};
        for (void* p : mp) cudaHostUnregister(p);
    }
    if (L->stage_stream) cudaStreamDestroy(L->stage_stream);
    if (L->side_stream) cudaStreamDestroy(L->side_stream);
    if (L->hash_stream) {
        cudaStreamSynchronize(L->hash_stream);
        cudaStreamDestroy(L->hash_stream);
    }
    if (L->hash_ev) cudaEventDestroy(L->hash_ev);
    if (L->copy_stream) cudaStreamDestroy(L->copy_stream);
    for (auto e : L->copy_ev)
        if (e) cudaEventDestroy(e);
    for (auto e : L->fork_ev)
        if (e) cudaEventDestroy(e);
    if (L->graph.exec) cudaGraphExecDestroy(L->graph.exec);
    if (L->wgraph.exec) cudaGraphExecDestroy(L->wgraph.exec);
    if (L->own_stream && L->stream) cudaStreamDestroy(L->stream);
    cudaGetLastError();
    delete L;
    return FFM_OK;
}

}  // extern "C"
