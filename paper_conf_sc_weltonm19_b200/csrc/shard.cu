// shard.cu -- multi-GPU (sharded log) kernels, SURVEY.md 8(e) / DESIGN.md §9.
//
// Exact byte equality is transitive, so after H1-H4 on its own records each rank
// holds exact local classes.  One representative per local class (its min local
// gid) is exported as a tuple; ranks all-gather the tuples (comm.cu: NCCL over
// NVLink), then every rank resolves ITS OWN representatives:
//   global leader G(x) = min gid over representatives with bytes equal to x's.
// The global group-by gives the min-gid representative with x's key; a remote
// candidate is confirmed by a byte compare that loads the candidate's bytes straight
// from the owning GPU's arena (CUDA-IPC-mapped peer memory over NVLink) -- the
// transfer is fused into the verify kernel, there is no staging copy.  A
// representative whose candidate is local (same key, different exact local class)
// or fails the compare takes the slow path: the tuples of its key are gathered into
// a segment (only for keys that have such a representative) and scanned; the minimum
// gid among the remote ones with equal bytes wins.  Every step is stream-ordered and
// decided on the device (no host round trip when nothing is slow).
#include <cub/cub.cuh>

#include "digest.cuh"
#include "ffm_internal.h"

namespace ffm {

enum : uint32_t { kDone = 0, kVerify = 1, kSlow = 2 };

__device__ __forceinline__ int owner_of(uint32_t t, const uint32_t* __restrict__ rank_lo, int world) {
    int o = 0;
    for (int r = 1; r < world; ++r) o += (t >= rank_lo[r]);
    return o;
}

// ---- export --------------------------------------------------------------------
__global__ void k_rep_flag(DevLog L, const uint32_t* __restrict__ leader, uint32_t* __restrict__ flag) {
    uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r > L.n) return;
    flag[r] = (r < L.n && leader[r] == r) ? 1u : 0u;
}

__global__ void k_rep_export(DevLog L, Work W, const uint32_t* __restrict__ rep_idx, uint64_t digest_mask,
                             RepTuple* __restrict__ out) {
    uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= L.n || W.leader[r] != r) return;
    uint64_t n = L.size[r];
    RepTuple t;
    t.key = group_key(W.digest[r], n, digest_mask, L.chan[r]);
    t.size = n;
    t.gid = L.gid[r];
    t.off = L.off[r];
    t.chan = L.chan[r];
    t.dig = W.digest[r];
    out[rep_idx[r]] = t;
}

// ---- global group-by over all representatives ----------------------------------
__global__ void k_merge_insert(const RepTuple* __restrict__ T, uint32_t M, uint64_t cap_mask, uint64_t* tkey,
                               uint64_t* tgid, uint32_t* __restrict__ tslot) {
    uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= M) return;
    const uint64_t key = T[t].key;
    uint64_t h = key & cap_mask;
    while (true) {
        unsigned long long prev =
            atomicCAS((unsigned long long*)&tkey[h], (unsigned long long)kEmptyKey, (unsigned long long)key);
        if (prev == kEmptyKey || prev == key) break;
        h = (h + 1) & cap_mask;
    }
    atomicMin((unsigned long long*)&tgid[h], (unsigned long long)T[t].gid);
    tslot[t] = (uint32_t)h;
}

__global__ void k_merge_index(const RepTuple* __restrict__ T, uint32_t M, const uint64_t* __restrict__ tgid,
                              const uint32_t* __restrict__ tslot, uint32_t* __restrict__ tidx) {
    uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= M) return;
    uint32_t h = tslot[t];
    if (T[t].gid == tgid[h]) tidx[h] = t;
}

// Classify this rank's representatives; count verify work units for remote candidates.
__global__ void k_merge_classify(const RepTuple* __restrict__ T, uint32_t lo, uint32_t nloc,
                                 const uint32_t* __restrict__ tslot, const uint32_t* __restrict__ tidx,
                                 const uint32_t* __restrict__ rank_lo, int world, int rank, uint32_t chunk_bytes,
                                 ShardWork S) {
    uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j > nloc) return;
    if (j == nloc) {
        S.vcount[j] = 0;
        return;
    }
    const uint32_t t = lo + j;
    const uint32_t c = tidx[tslot[t]];
    uint32_t st, cnt = 0;
    if (c == t) {
        st = kDone;
        S.G[j] = T[t].gid;
    } else if (owner_of(c, rank_lo, world) == rank || T[c].size != T[t].size || T[c].chan != T[t].chan) {
        st = kSlow;     // same key, different exact local class (or size / channel): not equal
    } else {
        st = kVerify;
        S.cand[j] = c;
        uint64_t n = T[t].size;
        cnt = n == 0 ? 1u : (uint32_t)((n + chunk_bytes - 1) / chunk_bytes);
        if (n) atomicAdd(&S.sctr[2], (unsigned long long)n);   // B_x: bytes read from the peer
    }
    S.state[j] = st;
    S.vcount[j] = cnt;
}

__global__ void k_merge_fill(uint32_t nloc, ShardWork S) {
    const uint32_t* nolist = nullptr;
    FFM_WARP_COMPACT(nloc, nolist, (S.vcount[r_] != 0), {
        const uint32_t s0 = S.vstart[rec], c_n = S.vcount[rec];
        for (uint32_t c = lane; c < c_n; c += 32) S.vitems[s0 + c] = make_uint2(rec, c);
    })
}

// Byte-compare a local representative with its remote candidate, chunk by chunk.
// The candidate's bytes are loaded from the peer GPU's arena over NVLink.
__global__ void __launch_bounds__(256) k_merge_verify(const RepTuple* __restrict__ T, uint32_t lo,
                                                      const uint32_t* __restrict__ rank_lo, int world, int rank,
                                                      const uint8_t* const* __restrict__ bases, uint32_t chunk_bytes,
                                                      const uint32_t* __restrict__ n_items_ptr, ShardWork S) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t n_items = *n_items_ptr;
    const uint32_t cblk = chunk_bytes >> 5;
    for (uint32_t it = warp; it < n_items; it += nwarps) {
        const uint2 w = S.vitems[it];
        const uint32_t j = w.x;
        const uint32_t x = lo + j, y = S.cand[j];
        const uint64_t n = T[x].size;
        const uint8_t* px = bases[rank] + T[x].off;
        const uint8_t* py = bases[owner_of(y, rank_lo, world)] + T[y].off;
        const uint32_t nblk = (uint32_t)((n + 31) >> 5);
        const uint32_t bb = w.y * cblk, be = min(bb + cblk, nblk);
        bool diff = false;
        for (uint32_t b = bb + lane; b < be; b += 32) {
            Blk a = ld_stream(px + 32ull * b);
            Blk r = ld_remote(py + 32ull * b);
            mask_tail(a, n, b);
            mask_tail(r, n, b);
            diff |= !blk_equal(a, r);
        }
        if (__any_sync(0xFFFFFFFFu, diff) && lane == 0) atomicExch(&S.state[j], (uint32_t)kSlow);
    }
}

__global__ void k_merge_finish(const RepTuple* __restrict__ T, uint32_t lo, uint32_t nloc,
                               const uint32_t* __restrict__ tslot, ShardWork S) {
    uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nloc) {
        uint32_t st = S.state[j];
        if (st == kVerify) S.G[j] = T[S.cand[j]].gid;
        if (st == kSlow) {
            S.slow_list[atomicAdd(&S.sctr[0], 1ull)] = j;
            S.need[tslot[lo + j]] = 1u;   // this key's tuples are gathered into a segment
        }
    }
}

// Slow path (digest collisions, or a candidate from this rank's own other class):
// segments of the keys that have a slow representative -- count, allocate, fill.  Each
// kernel returns at once when no representative is slow (decided on the device).
__global__ void k_seg_count(uint32_t M, const uint32_t* __restrict__ tslot, ShardWork S) {
    if (S.sctr[0] == 0) return;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < M; t += gridDim.x * blockDim.x) {
        const uint32_t h = tslot[t];
        if (S.need[h]) atomicAdd(&S.scnt[h], 1u);
    }
}

__global__ void k_seg_alloc(uint32_t M, const uint32_t* __restrict__ tslot, const uint32_t* __restrict__ tidx,
                            ShardWork S) {
    if (S.sctr[0] == 0) return;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < M; t += gridDim.x * blockDim.x) {
        const uint32_t h = tslot[t];
        if (S.need[h] && tidx[h] == t) {   // one owner per key: its min-gid tuple
            S.sbase[h] = (uint32_t)atomicAdd(&S.sctr[1], (unsigned long long)S.scnt[h]);
            S.sfill[h] = 0;
        }
    }
}

__global__ void k_seg_fill(uint32_t M, const uint32_t* __restrict__ tslot, ShardWork S) {
    if (S.sctr[0] == 0) return;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < M; t += gridDim.x * blockDim.x) {
        const uint32_t h = tslot[t];
        if (S.need[h]) S.seg[S.sbase[h] + atomicAdd(&S.sfill[h], 1u)] = t;
    }
}

// One warp per slow representative x: scan its key's segment, 32 tuples per step; a
// candidate y is an earlier representative (gid below the best so far) on another rank
// with x's size and channel (and, unless refine_bits weakens it, x's full digest -- a
// function of the bytes, so a different digest cannot be equal bytes).  Candidates are
// byte-compared against x (peer bytes over NVLink), stopping at the first differing
// 1 KiB step; the least gid among equal ones is x's global leader.
__global__ void __launch_bounds__(256) k_merge_slow(const RepTuple* __restrict__ T, uint32_t lo,
                                                    const uint32_t* __restrict__ tslot,
                                                    const uint32_t* __restrict__ rank_lo, int world, int rank,
                                                    const uint8_t* const* __restrict__ bases, uint64_t refine_mask,
                                                    ShardWork S) {
    const uint32_t n_slow = (uint32_t)S.sctr[0];
    if (n_slow == 0) return;
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    unsigned long long bx = 0;
    for (uint32_t q = warp; q < n_slow; q += nwarps) {
        const uint32_t j = S.slow_list[q];
        const uint32_t x = lo + j;
        const RepTuple tx = T[x];
        const uint64_t nblk = (tx.size + 31) >> 5;
        const uint8_t* px = bases[rank] + tx.off;
        const uint32_t h = tslot[x];
        const uint32_t s0 = S.sbase[h], sn = S.scnt[h];
        uint64_t best = tx.gid;
        for (uint32_t i0 = 0; i0 < sn; i0 += 32) {
            const uint32_t y = i0 + lane < sn ? S.seg[s0 + i0 + lane] : x;
            const RepTuple ty = T[y];
            const bool cand = ty.gid < best && ty.key == tx.key && ty.size == tx.size && ty.chan == tx.chan &&
                              ((ty.dig ^ tx.dig) & refine_mask) == 0 && owner_of(y, rank_lo, world) != rank;
            unsigned cm = __ballot_sync(0xFFFFFFFFu, cand);
            while (cm) {
                const int src = __ffs(cm) - 1;
                cm &= cm - 1;
                const uint64_t gy = __shfl_sync(0xFFFFFFFFu, ty.gid, src);
                const uint64_t oy = __shfl_sync(0xFFFFFFFFu, ty.off, src);
                const uint32_t yy = __shfl_sync(0xFFFFFFFFu, y, src);
                if (gy >= best) continue;   // an equal earlier one is already known
                const uint8_t* py = bases[owner_of(yy, rank_lo, world)] + oy;
                bool diff = false;
                for (uint64_t b0 = 0; b0 < nblk && !diff; b0 += 32) {
                    const uint64_t b = b0 + lane;
                    bool d = false;
                    if (b < nblk) {
                        Blk a = ld_stream(px + 32 * b);
                        Blk r = ld_remote(py + 32 * b);
                        mask_tail(a, tx.size, b);
                        mask_tail(r, tx.size, b);
                        d = !blk_equal(a, r);
                        bx += 32;
                    }
                    diff = __any_sync(0xFFFFFFFFu, d);
                }
                if (!diff) best = gy;
            }
        }
        if (lane == 0) S.G[j] = best;
    }
    if (bx) atomicAdd(&S.sctr[2], bx);
}

// Segments are cleared where they were used (the arrays stay zero between runs).
__global__ void k_seg_clear(uint32_t lo, const uint32_t* __restrict__ tslot, ShardWork S) {
    const uint32_t n_slow = (uint32_t)S.sctr[0];
    for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < n_slow; q += gridDim.x * blockDim.x) {
        const uint32_t h = tslot[lo + S.slow_list[q]];
        S.need[h] = 0;
        S.scnt[h] = 0;
    }
}

// H5 + H6 for a shard: record r's class representative is its local leader; the
// class's global leader G comes from the merge.  Benefit / count partials per rank.
__global__ void __launch_bounds__(1024) k_merge_label(DevLog L, const uint32_t* __restrict__ leader,
                                                     const uint32_t* __restrict__ rep_idx,
                                                     const uint64_t* __restrict__ G, uint32_t n_sites,
                                                     int64_t* __restrict__ dup_out, uint64_t* __restrict__ part,
                                                     uint32_t* __restrict__ cpart, uint64_t* __restrict__ ben_global,
                                                     uint64_t* __restrict__ cnt_global) {
    extern __shared__ unsigned long long sben[];
    uint32_t* scnt = (uint32_t*)(sben + n_sites);
    const bool hist = part != nullptr;
    if (hist) {
        for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
            sben[s] = 0;
            scnt[s] = 0;
        }
        __syncthreads();
    }
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < L.n; r += gridDim.x * blockDim.x) {
        uint64_t g = G[rep_idx[leader[r]]];
        int64_t d = g == L.gid[r] ? -1 : (int64_t)g;
        dup_out[r] = d;
        if (d >= 0) {
            const uint32_t s = L.site[r];
            if (hist) {
                atomicAdd(&sben[s], (unsigned long long)L.dur[r]);
                atomicAdd(&scnt[s], 1u);
            } else {
                atomicAdd((unsigned long long*)&ben_global[s], (unsigned long long)L.dur[r]);
                atomicAdd((unsigned long long*)&cnt_global[s], 1ull);
            }
        }
    }
    if (hist) {
        __syncthreads();
        uint64_t* row = part + (uint64_t)blockIdx.x * n_sites;
        uint32_t* crow = cpart + (uint64_t)blockIdx.x * n_sites;
        for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
            row[s] = sben[s];
            crow[s] = scnt[s];
        }
    }
}

// ---- launchers -------------------------------------------------------------------
#define SHARD_CHECK()                                     \
    do {                                                  \
        if (cudaGetLastError() != cudaSuccess) return -1; \
    } while (0)

int launch_rep_export(const DevLog& L, Work& W, ShardWork& S, const Params& P, RepTuple* out, cudaStream_t st) {
    k_rep_flag<<<blocks_for((uint64_t)L.n + 1), 256, 0, st>>>(L, W.leader, S.flag);
    SHARD_CHECK();
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, S.flag, S.rep_idx, (int)(L.n + 1), st) != cudaSuccess)
        return -1;
    if (L.n) {
        k_rep_export<<<blocks_for(L.n), 256, 0, st>>>(L, W, S.rep_idx, P.digest_mask, out);
        SHARD_CHECK();
    }
    return 3;
}

int launch_merge(const DevLog& L, Work& W, ShardWork& S, const Params& P, const RepTuple* T, uint32_t M,
                 uint32_t lo, uint32_t nloc, int world, int rank, uint64_t cap, cudaStream_t st) {
    int k = 0;
    if (cudaMemsetAsync(S.tkey, 0xFF, cap * sizeof(uint64_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(S.tgid, 0xFF, cap * sizeof(uint64_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(S.sctr, 0, 4 * sizeof(unsigned long long), st) != cudaSuccess) return -1;
    if (M) {
        k_merge_insert<<<blocks_for(M), 256, 0, st>>>(T, M, cap - 1, S.tkey, S.tgid, S.tslot);
        SHARD_CHECK();
        k_merge_index<<<blocks_for(M), 256, 0, st>>>(T, M, S.tgid, S.tslot, S.tidx);
        SHARD_CHECK();
        k += 2;
    }
    k_merge_classify<<<blocks_for((uint64_t)nloc + 1), 256, 0, st>>>(T, lo, nloc, S.tslot, S.tidx, S.rank_lo, world,
                                                                      rank, P.chunk_bytes, S);
    SHARD_CHECK();
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, S.vcount, S.vstart, (int)(nloc + 1), st) != cudaSuccess)
        return -1;
    k += 2;
    if (nloc) {
        k_merge_fill<<<blocks_for(nloc), 256, 0, st>>>(nloc, S);
        SHARD_CHECK();
        uint32_t grid = resident_grid((const void*)k_merge_verify, P.num_sms);
        k_merge_verify<<<grid, 256, 0, st>>>(T, lo, S.rank_lo, world, rank, S.bases, P.chunk_bytes, S.vstart + nloc,
                                             S);
        SHARD_CHECK();
        k_merge_finish<<<blocks_for(nloc), 256, 0, st>>>(T, lo, nloc, S.tslot, S);
        SHARD_CHECK();
        k += 3;
        // slow path, decided on the device (each kernel exits when nothing is slow)
        const uint32_t gm = std::min<uint32_t>(blocks_for(M), (uint32_t)P.num_sms * 4);
        k_seg_count<<<gm, 256, 0, st>>>(M, S.tslot, S);
        SHARD_CHECK();
        k_seg_alloc<<<gm, 256, 0, st>>>(M, S.tslot, S.tidx, S);
        SHARD_CHECK();
        k_seg_fill<<<gm, 256, 0, st>>>(M, S.tslot, S);
        SHARD_CHECK();
        k_merge_slow<<<resident_grid((const void*)k_merge_slow, P.num_sms), 256, 0, st>>>(
            T, lo, S.tslot, S.rank_lo, world, rank, S.bases, P.refine_mask, S);
        SHARD_CHECK();
        k_seg_clear<<<std::min<uint32_t>(blocks_for(nloc), (uint32_t)P.num_sms), 256, 0, st>>>(lo, S.tslot, S);
        SHARD_CHECK();
        k += 5;
    }
    return k;
}

int launch_merge_label(const DevLog& L, Work& W, ShardWork& S, const Params& P, uint32_t n_sites, int64_t* dup_out,
                       cudaStream_t st) {
    if (L.n == 0) {
        if (cudaMemsetAsync(W.ben, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
        return cudaMemsetAsync(W.cnt, 0, (uint64_t)n_sites * 8, st) == cudaSuccess ? 0 : -1;
    }
    const size_t smem = label_smem_bytes(n_sites);
    if (W.label_part && smem <= (size_t)P.max_smem) {
        if (!smem_configured((const void*)k_merge_label, P.max_smem)) return -1;
        const uint32_t rows = label_hist_rows(P.num_sms);
        k_merge_label<<<rows, 1024, smem, st>>>(L, W.leader, S.rep_idx, S.G, n_sites, dup_out, W.label_part,
                                               W.label_cpart, nullptr, nullptr);
        SHARD_CHECK();
        return 1 + launch_site_reduce(W.label_part, W.label_cpart, rows, n_sites, W.ben, W.cnt, st);
    }
    if (cudaMemsetAsync(W.ben, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(W.cnt, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
    k_merge_label<<<(uint32_t)P.num_sms * 4, 512, 0, st>>>(L, W.leader, S.rep_idx, S.G, n_sites, dup_out, nullptr,
                                                           nullptr, W.ben, W.cnt);
    SHARD_CHECK();
    return 1;
}

// The per-rank header exchanged after the local pass: representatives exported, residual
// members (a rank with residuals re-exports after resolving them), arena generation (peers
// re-map a reallocated arena), record count.
__global__ void k_shard_header(const uint32_t* __restrict__ rep_count, const uint32_t* __restrict__ counters,
                               uint64_t gen, uint64_t n, uint64_t* __restrict__ hdr) {
    if (threadIdx.x == 0) {
        hdr[0] = *rep_count;
        hdr[1] = counters[0];
        hdr[2] = gen;
        hdr[3] = n;
    }
}

int launch_shard_header(const uint32_t* rep_count, const uint32_t* counters, uint64_t gen, uint64_t n,
                        uint64_t* hdr, cudaStream_t st) {
    k_shard_header<<<1, 32, 0, st>>>(rep_count, counters, gen, n, hdr);
    SHARD_CHECK();
    return 1;
}

}  // namespace ffm
