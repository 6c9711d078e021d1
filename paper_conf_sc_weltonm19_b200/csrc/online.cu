// online.cu -- online (streaming) mode, SURVEY.md 8(f) #2 / DESIGN.md §10: the paper's
// per-call semantics (Sec. 3.3.2): "The data being transferred is hashed and
// then compared to the stored hashes from prior transfers."
//
// The stored hashes are a persistent device table of every exact class seen so far:
// open addressing on the group key of (full digest, size, channel) -> a chain of class
// representatives in an insert-only pool (gid, arena offset, size, channel, digest).
// A step labels one window of new records:
//   1-2. H1-H4 on the window alone -> exact window classes: by default the batch run's fused
//      round 0 on the window in its batch record order (built on the device by
//      launch_window_order); with FFM_FLAG_APPEND_HASH the NH sums were computed at append time
//      on the hashing stream and the step runs the two-pass round 0 without H1;
//   3. k_online_probe (thread per record): each window class representative looks its key
//      up in the table -- absent: the class is new and stored at once; present:
//      k_online_cmp (8 lanes per listed class) byte-compares the chained prior
//      representatives of its size / channel / digest (their bytes stay resident in the
//      HBM arena) -- at most one prior class can be equal, so the chain order does not
//      matter; a class with no equal stored class is stored by the same kernel;
//   4. k_online_label: labels (gids) and the cumulative per-site benefit / counts.
// The table is never rebuilt by a step; it is rehashed only when its capacity doubles.
#include "digest.cuh"
#include "ffm_internal.h"

namespace ffm {

constexpr uint32_t kNoRep = 0xFFFFFFFFu;

// slot of `key` in the table (probing), or the empty slot where it would go
__device__ __forceinline__ uint64_t online_probe(const OnlineTable& T, uint64_t key) {
    uint64_t h = key & T.mask;
    while (true) {
        const uint64_t k = T.key[h];
        if (k == key || k == kEmptyKey) return h;
        h = (h + 1) & T.mask;
    }
}

__device__ __forceinline__ void online_link(OnlineTable& T, uint64_t key, uint32_t idx) {
    uint64_t h = key & T.mask;
    while (true) {
        unsigned long long prev =
            atomicCAS((unsigned long long*)&T.key[h], (unsigned long long)kEmptyKey, (unsigned long long)key);
        if (prev == kEmptyKey || prev == key) break;
        h = (h + 1) & T.mask;
    }
    T.pool[idx].next = atomicExch(&T.head[h], idx);
}

// Store window class r as a new class (its entry is complete before the CAS that
// publishes it on its key's chain).
// kFence: chain walkers may run concurrently (k_online_cmp) -- the entry must be visible
// before the head CAS; k_online_probe has no concurrent walkers (the kernel boundary orders
// its stores before any walk).
// ni: the entry's pool index (atomicAdd on T.count, warp-aggregated by the caller)
template <bool kFence>
__device__ __forceinline__ void online_store(OnlineTable& T, const DevLog& L, uint32_t r, uint64_t key, uint64_t dig,
                                             uint32_t ni) {
    OnlineRep e;
    e.gid = L.gid[r];
    e.off = L.off[r];
    e.size = L.size[r];
    e.chan = L.chan[r];
    e.dig = dig;
    e.pad = 0;
    uint64_t hh = key & T.mask;
    while (true) {
        unsigned long long prev =
            atomicCAS((unsigned long long*)&T.key[hh], (unsigned long long)kEmptyKey, (unsigned long long)key);
        if (prev == kEmptyKey || prev == key) break;
        hh = (hh + 1) & T.mask;
    }
    uint32_t old = *reinterpret_cast<volatile uint32_t*>(&T.head[hh]);
    while (true) {
        e.next = old;
        T.pool[ni] = e;
        if (kFence) __threadfence();
        const uint32_t seen = atomicCAS(&T.head[hh], old, ni);
        if (seen == old) break;
        old = seen;
    }
}

// Thread per window record: a window class representative r (leader[r] == r) looks its
// key up; with the key absent from the table no stored class can equal it and r's class
// is stored right away (G[r] = its own gid); with the key present r goes to the compare
// list for k_online_cmp.  Concurrent stores are safe: a window's classes are pairwise
// distinct, so a class that finds a key stored by another window class of the same
// step only pays a compare that fails.
// (list != nullptr: only the listed records -- the residual fix-up of a step)
__global__ void __launch_bounds__(256) k_online_probe(DevLog L, const uint32_t* __restrict__ leader,
                                                      const uint64_t* __restrict__ accA,
                                                      const uint64_t* __restrict__ accB, OnlineTable T,
                                                      uint64_t digest_mask, uint64_t* __restrict__ G,
                                                      uint32_t* __restrict__ cmp_list, uint32_t* __restrict__ n_cmp,
                                                      const uint32_t* __restrict__ list, uint32_t n_list) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    uint32_t r = 0;
    bool rep = false;
    if (i < n_list) {
        r = list ? list[i] : i;
        rep = leader[r] == r;
    }
    uint64_t key = 0, dig = 0;
    bool present = false;
    if (rep) {
        const uint64_t n = L.size[r];
        dig = finalize_digest(accA[r], accB[r], n);
        key = group_key(dig, n, digest_mask, L.chan[r]);
        present = T.key[online_probe(T, key)] == key;
    }
    // one atomic per warp for each of the two appends (list / pool)
    const unsigned below = (1u << lane) - 1u;
    const unsigned mp = __ballot_sync(0xFFFFFFFFu, present);
    const unsigned ms = __ballot_sync(0xFFFFFFFFu, rep && !present);
    uint32_t bp = 0, bs = 0;
    if (lane == 0) {
        if (mp) bp = atomicAdd(n_cmp, (uint32_t)__popc(mp));
        if (ms) bs = atomicAdd(T.count, (uint32_t)__popc(ms));
    }
    bp = __shfl_sync(0xFFFFFFFFu, bp, 0);
    bs = __shfl_sync(0xFFFFFFFFu, bs, 0);
    if (present) {
        cmp_list[bp + __popc(mp & below)] = r;
    } else if (rep) {
        G[r] = L.gid[r];
        online_store<false>(T, L, r, key, dig, bs + __popc(ms & below));
    }
}

// One 8-lane group per listed window class r, grid-stride: byte-compare the chained
// stored classes of its size / channel / digest (32-byte blocks per lane, stopping at the
// first differing step) -- at most one can be equal; with none, r's class is stored.
__global__ void __launch_bounds__(256) k_online_cmp(DevLog L, const uint64_t* __restrict__ accA,
                                                    const uint64_t* __restrict__ accB, OnlineTable T,
                                                    uint64_t digest_mask, uint64_t refine_mask,
                                                    uint64_t* __restrict__ G, const uint32_t* __restrict__ cmp_list,
                                                    const uint32_t* __restrict__ n_cmp) {
    const int g = threadIdx.x & 7;
    const unsigned omask = 0xFFu << (threadIdx.x & 24);
    const uint32_t noct = (gridDim.x * blockDim.x) >> 3;
    const uint32_t m = *n_cmp;
    for (uint32_t i = (blockIdx.x * blockDim.x + threadIdx.x) >> 3; i < m; i += noct) {
        const uint32_t r = cmp_list[i];
        const uint64_t n = L.size[r], chan = L.chan[r];
        const uint64_t dig = finalize_digest(accA[r], accB[r], n);
        const uint64_t key = group_key(dig, n, digest_mask, chan);
        const uint64_t h = online_probe(T, key);
        uint32_t idx = *reinterpret_cast<volatile uint32_t*>(&T.head[h]);
        uint64_t gl = L.gid[r];
        bool found = false;
        const uint8_t* px = L.arena + L.off[r];
        const uint64_t nblk = (n + 31) >> 5;
        while (idx != kNoRep) {
            const OnlineRep e = T.pool[idx];
            if (e.size == n && e.chan == chan && ((e.dig ^ dig) & refine_mask) == 0) {
                const uint8_t* py = L.arena + e.off;
                bool diff = false;
                for (uint64_t b0 = 0; b0 < nblk && !diff; b0 += 8) {
                    const uint64_t b = b0 + g;
                    bool d = false;
                    if (b < nblk) {
                        Blk a = ld_stream(px + 32 * b);
                        Blk y = ld_keep(py + 32 * b);
                        mask_tail(a, n, b);
                        mask_tail(y, n, b);
                        d = !blk_equal(a, y);
                    }
                    diff = __ballot_sync(omask, d) != 0;
                }
                if (!diff) {   // the (only) equal stored class
                    gl = e.gid;
                    found = true;
                    break;
                }
            }
            idx = e.next;
        }
        if (g == 0) {
            G[r] = gl;
            if (!found) online_store<true>(T, L, r, key, dig, atomicAdd(T.count, 1u));
        }
    }
}

// Residual fix-up of a step whose labels went out speculatively (before its H4): a
// residual r was labelled a duplicate of its round-0 candidate and counted in the
// cumulative per-site sums; take that back and apply its final label (its class was
// matched against the table by k_online_probe / k_online_cmp over the residual list).
__global__ void k_online_fix(DevLog L, const uint32_t* __restrict__ leader, const uint64_t* __restrict__ G,
                             const uint32_t* __restrict__ list, uint32_t n_list, int64_t* __restrict__ dup_out,
                             uint64_t* __restrict__ ben, uint64_t* __restrict__ cnt) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_list) return;
    const uint32_t r = list[i];
    const uint32_t s = L.site[r];
    const uint64_t dur = L.dur[r];
    const uint64_t g = G[leader[r]];
    const int64_t d = g == L.gid[r] ? -1 : (int64_t)g;
    dup_out[r] = d;
    if (d < 0) {   // (integer sums mod 2^64: subtracting is adding the complement)
        atomicAdd((unsigned long long*)&ben[s], (unsigned long long)(0 - dur));
        atomicAdd((unsigned long long*)&cnt[s], ~0ull);
    }
}

// Tiny windows (<= kTinyWindow small records; ffm_online_step): one warp labels the
// window's records one after another, in gid order, directly against the table -- the
// record's NH digest (lane l takes 16-byte words l, l + 32, ...), its
// key's chain byte-compared, a new class stored at once -- so a duplicate inside the window
// finds its class in the table like any earlier one.  No group-by, no record order, one
// launch: the per-call latency of the paper's per-transfer check.
__global__ void __launch_bounds__(32) k_online_tiny(DevLog L, OnlineTable T, NHKeys nk, uint64_t digest_mask,
                                                    uint64_t refine_mask, int64_t* __restrict__ dup_out,
                                                    uint64_t* __restrict__ ben, uint64_t* __restrict__ cnt) {
    __shared__ uint32_t ska[16][6];
    const int lane = threadIdx.x;
    for (int i = lane; i < 96; i += 32) ska[i / 6][i % 6] = nk.ka[i / 6][i % 6];
    __syncwarp();
    for (uint32_t r = 0; r < L.n; ++r) {
        const uint64_t n = L.size[r], chan = L.chan[r];
        const uint8_t* px = L.arena + L.off[r];
        const uint64_t nw = (n + 15) >> 4;
        uint64_t A = 0, B = 0;
        for (uint64_t q = lane; q < nw; q += 32) {
            uint4 v = *reinterpret_cast<const uint4*>(px + 16 * q);
            uint32_t w[4] = {v.x, v.y, v.z, v.w};
            const int32_t valid = (int32_t)(n - 16 * q);
            if (valid < 16) {
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int32_t vb = valid - 4 * i;
                    w[i] &= vb >= 4 ? 0xFFFFFFFFu : (vb <= 0 ? 0u : ((1u << (8 * vb)) - 1u));
                }
            }
            uint32_t k[6];
            const uint32_t s = (uint32_t)(q >> 4);
#pragma unroll
            for (int j = 0; j < 6; ++j) k[j] = ska[q & 15][j] + s * kDA(j);
            A += (uint64_t)(w[0] + k[0]) * (uint64_t)(w[1] + k[1]);
            A += (uint64_t)(w[2] + k[2]) * (uint64_t)(w[3] + k[3]);
            B += (uint64_t)(w[0] + k[2]) * (uint64_t)(w[1] + k[3]);
            B += (uint64_t)(w[2] + k[4]) * (uint64_t)(w[3] + k[5]);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
            B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
        }
        const uint64_t dig = finalize_digest(A, B, n);
        const uint64_t key = group_key(dig, n, digest_mask, chan);
        const uint64_t h = online_probe(T, key);
        uint32_t idx = 0xFFFFFFFFu;   // (kNoRep)
        if (T.key[h] == key) idx = *reinterpret_cast<volatile uint32_t*>(&T.head[h]);
        uint64_t gl = L.gid[r];
        bool found = false;
        const uint64_t nblk = (n + 31) >> 5;
        while (idx != kNoRep && !found) {
            const OnlineRep e = T.pool[idx];
            if (e.size == n && e.chan == chan && ((e.dig ^ dig) & refine_mask) == 0) {
                const uint8_t* py = L.arena + e.off;
                bool diff = false;
                for (uint64_t b0 = 0; b0 < nblk && !diff; b0 += 32) {
                    const uint64_t b = b0 + lane;
                    bool d = false;
                    if (b < nblk) {
                        Blk x = ld_stream(px + 32 * b);
                        Blk y = ld_keep(py + 32 * b);
                        mask_tail(x, n, b);
                        mask_tail(y, n, b);
                        d = !blk_equal(x, y);
                    }
                    diff = __any_sync(0xFFFFFFFFu, d);
                }
                if (!diff) {
                    gl = e.gid;
                    found = true;
                }
            }
            idx = e.next;
        }
        if (lane == 0) {
            if (!found) online_store<false>(T, L, r, key, dig, atomicAdd(T.count, 1u));
            const int64_t d = found ? (int64_t)gl : -1;
            dup_out[r] = d;
            if (d >= 0) {
                ben[L.site[r]] += L.dur[r];
                cnt[L.site[r]] += 1;
            }
        }
        __syncwarp();   // (the next record's probe may meet this one's new entry)
    }
}

// Capacity growth: re-link every stored representative into a fresh (larger) table.
__global__ void k_online_rehash(OnlineTable T, uint32_t np, uint64_t digest_mask) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= np) return;
    const OnlineRep e = T.pool[i];
    online_link(T, group_key(e.dig, e.size, digest_mask, e.chan), i);
}

// Labels of the window and the cumulative per-site sums (block histograms in shared
// memory when the sites fit, then one atomic per (block, site)).
template <bool kHist>
__global__ void __launch_bounds__(1024) k_online_label(DevLog L, const uint32_t* __restrict__ leader,
                                                       const uint64_t* __restrict__ G, uint32_t n_sites,
                                                       int64_t* __restrict__ dup_out, uint64_t* __restrict__ ben,
                                                       uint64_t* __restrict__ cnt) {
    extern __shared__ unsigned long long sben[];
    uint32_t* scnt = (uint32_t*)(sben + n_sites);
    if (kHist) {
        for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
            sben[s] = 0;
            scnt[s] = 0;
        }
        __syncthreads();
    }
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < L.n; r += gridDim.x * blockDim.x) {
        const uint64_t g = G[leader[r]];
        const int64_t d = g == L.gid[r] ? -1 : (int64_t)g;
        dup_out[r] = d;
        if (d >= 0) {
            const uint32_t s = L.site[r];
            if (kHist) {
                atomicAdd(&sben[s], (unsigned long long)L.dur[r]);
                atomicAdd(&scnt[s], 1u);
            } else {
                atomicAdd((unsigned long long*)&ben[s], (unsigned long long)L.dur[r]);
                atomicAdd((unsigned long long*)&cnt[s], 1ull);
            }
        }
    }
    if (kHist) {
        __syncthreads();
        for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
            if (sben[s]) atomicAdd((unsigned long long*)&ben[s], sben[s]);
            if (scnt[s]) atomicAdd((unsigned long long*)&cnt[s], (unsigned long long)scnt[s]);
        }
    }
}

#define ONLINE_CHECK()                                    \
    do {                                                  \
        if (cudaGetLastError() != cudaSuccess) return -1; \
    } while (0)

int launch_online_rehash(OnlineTable& T, uint32_t np, uint64_t digest_mask, cudaStream_t st) {
    if (cudaMemsetAsync(T.key, 0xFF, (T.mask + 1) * sizeof(uint64_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(T.head, 0xFF, (T.mask + 1) * sizeof(uint32_t), st) != cudaSuccess) return -1;
    if (!np) return 0;
    k_online_rehash<<<blocks_for(np), 256, 0, st>>>(T, np, digest_mask);
    ONLINE_CHECK();
    return 1;
}

int launch_online_window(const DevLog& L, const Work& W, const uint64_t* accA, const uint64_t* accB,
                         OnlineTable& T, const Params& P, uint32_t n_sites, uint64_t* G, int64_t* dup_out,
                         uint64_t* ben, uint64_t* cnt, cudaStream_t st) {
    if (L.n == 0) return 0;
    // the compare list reuses the residual buffer res[1] (free after the window's H4);
    // its length lives in counters[12]
    uint32_t* n_cmp = W.counters + 12;
    if (cudaMemsetAsync(n_cmp, 0, sizeof(uint32_t), st) != cudaSuccess) return -1;
    k_online_probe<<<blocks_for(L.n), 256, 0, st>>>(L, W.leader, accA, accB, T, P.digest_mask, G, W.res[1], n_cmp,
                                                    nullptr, L.n);
    ONLINE_CHECK();
    k_online_cmp<<<std::min<uint32_t>(blocks_for((uint64_t)L.n * 8), (uint32_t)P.num_sms * 8), 256, 0, st>>>(
        L, accA, accB, T, P.digest_mask, P.refine_mask, G, W.res[1], n_cmp);
    ONLINE_CHECK();
    const size_t smem = label_smem_bytes(n_sites);
    const uint32_t grid = std::min<uint32_t>(blocks_for(L.n, 1024), (uint32_t)P.num_sms);
    if (smem <= (size_t)P.max_smem) {
        if (!smem_configured((const void*)k_online_label<true>, P.max_smem)) return -1;
        k_online_label<true><<<grid, 1024, smem, st>>>(L, W.leader, G, n_sites, dup_out, ben, cnt);
    } else {
        k_online_label<false><<<grid, 1024, 0, st>>>(L, W.leader, G, n_sites, dup_out, ben, cnt);
    }
    ONLINE_CHECK();
    return 3;
}

int launch_online_tiny(const DevLog& L, OnlineTable& T, const Params& P, int64_t* dup_out, uint64_t* ben,
                       uint64_t* cnt, cudaStream_t st) {
    if (L.n == 0) return 0;
    k_online_tiny<<<1, 32, 0, st>>>(L, T, make_nh_keys(), P.digest_mask, P.refine_mask, dup_out, ben, cnt);
    ONLINE_CHECK();
    return 1;
}

// After H4 of a step launched with speculative labels: the residual records (list) get
// their classes matched against the table and their labels / sums corrected.
int launch_online_fix(const DevLog& L, const Work& W, const uint64_t* accA, const uint64_t* accB, OnlineTable& T,
                      const Params& P, const uint32_t* list, uint32_t n_list, uint64_t* G, int64_t* dup_out,
                      uint64_t* ben, uint64_t* cnt, cudaStream_t st) {
    if (n_list == 0) return 0;
    uint32_t* n_cmp = W.counters + 12;
    if (cudaMemsetAsync(n_cmp, 0, sizeof(uint32_t), st) != cudaSuccess) return -1;
    k_online_probe<<<blocks_for(n_list), 256, 0, st>>>(L, W.leader, accA, accB, T, P.digest_mask, G, W.res[1], n_cmp,
                                                       list, n_list);
    ONLINE_CHECK();
    k_online_cmp<<<std::min<uint32_t>(blocks_for((uint64_t)n_list * 8), (uint32_t)P.num_sms * 8), 256, 0, st>>>(
        L, accA, accB, T, P.digest_mask, P.refine_mask, G, W.res[1], n_cmp);
    ONLINE_CHECK();
    k_online_fix<<<blocks_for(n_list), 256, 0, st>>>(L, W.leader, G, list, n_list, dup_out, ben, cnt);
    ONLINE_CHECK();
    return 3;
}

}  // namespace ffm
