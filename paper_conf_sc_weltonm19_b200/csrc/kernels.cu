// kernels.cu -- sm_100a kernels of the duplicate-transfer hot path.
//
// Steps:
//   H1 hash    k_hash_small / k_hash_large   ("the data being transferred is hashed")
//   H2 group   k_group_insert / k_leader     ("compared to the stored hashes from prior transfers")
//   H3 verify  k_verify_small / k_verify_large (reading R2: every hash match is byte-verified)
//   H4 resolve k_refine + H2/H3 over the residuals (exact classes under digest collisions)
//   H5/H6      k_label  ("marks the transfer as being a duplicate ... the location of the
//              first transfer"; Fig. 5 P:956-960 benefit = duration; P:1021-1026 per call site)
//
// All of it is integer, HBM-bound streaming: 256-bit non-coalescing-free loads
// (LDG.256, sm_100), per-lane NH multiply-accumulate, warp / 8-lane shuffles.
// No tensor cores: there is no dense contraction on this path.
#include <cub/cub.cuh>

#include <mutex>
#include <unordered_map>

#include "ffm_internal.h"
#include "digest.cuh"

// Tuning knobs of the fused pass; defaults are the measured best on B200 (config 5 / 4,
// profiles/r01_fused_variants.md): leader-first layout, members' compare loads
// L2::evict_last, everyone's own loads L2::evict_first (evict_last or normal priority on
// the leaders' own loads measured 12-13% slower), 2 loads in flight per lane when
// comparing, 3 CTAs/SM.
#ifndef FFM_FUSED_CMP_U
#define FFM_FUSED_CMP_U 2
#endif
#ifndef FFM_FUSED_LEADER_FIRST
#define FFM_FUSED_LEADER_FIRST 1
#endif
#ifndef FFM_FUSED_KEEP_OWN
#define FFM_FUSED_KEEP_OWN 0
#endif
#ifndef FFM_FUSED_SKEW
#define FFM_FUSED_SKEW 0x7FFFFFFF   /* measured: leader-first (no skew) is best */
#endif
#ifndef FFM_FUSED_Y_POLICY
#define FFM_FUSED_Y_POLICY 1
#endif

namespace ffm {

// ----------------------------------------------------------------------------
// Digest.  16-byte words W[q], q < ceil(n/16), zero-padded;
// four little-endian u32 lanes w0..w3.  Position g = q mod 16, stripe s = q div 16.
// k_j = KA[g][j] + s * DA[j]  (mod 2^32), j = 0..5
// A = sum (w0+k0)(w1+k1) + (w2+k2)(w3+k3)   B = sum (w0+k2)(w1+k3) + (w2+k4)(w3+k5)   (mod 2^64)
// digest = fmix64(A ^ fmix64(B ^ n * 0x9E3779B97F4A7C15))
// The per-stripe key steps DA are compile-time constants (immediate operands), so a
// lane keeps only its 12 current keys in registers.
// ----------------------------------------------------------------------------
struct NHKeys {
    uint32_t ka[16][6];
};

constexpr uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

constexpr NHKeys make_nh_keys() {
    NHKeys k{};
    uint64_t s = 0xD10E5E5FF1ull;
    for (int g = 0; g < 16; ++g)
        for (int j = 0; j < 6; ++j) k.ka[g][j] = (uint32_t)(sm64(s++) >> 16);
    return k;
}

// per-stripe key increments (odd => full period mod 2^32)
__host__ __device__ constexpr uint32_t kDA(int j) {
    return j == 0 ? 0x9E3779B9u : j == 1 ? 0x7F4A7C15u : j == 2 ? 0xF39CC061u
         : j == 3 ? 0x5CEDC835u : j == 4 ? 0x1B873593u : 0xCC9E2D51u;
}

__constant__ NHKeys c_nh = make_nh_keys();

struct LaneKeys {
    uint32_t k[2][6];
};

// Keys of positions p0, p0+1 at stripe s.
__device__ __forceinline__ void load_keys(LaneKeys& K, int p0, uint32_t s) {
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int j = 0; j < 6; ++j) K.k[h][j] = c_nh.ka[p0 + h][j] + s * kDA(j);
}

// Advance MULT stripes (immediate-operand adds).
template <uint32_t MULT>
__device__ __forceinline__ void advance(LaneKeys& K) {
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int j = 0; j < 6; ++j) K.k[h][j] += kDA(j) * MULT;
}

__device__ __forceinline__ void nh_word(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, const uint32_t* k,
                                        uint64_t& A, uint64_t& B) {
    A += (uint64_t)(w0 + k[0]) * (uint64_t)(w1 + k[1]);
    A += (uint64_t)(w2 + k[2]) * (uint64_t)(w3 + k[3]);
    B += (uint64_t)(w0 + k[2]) * (uint64_t)(w1 + k[3]);
    B += (uint64_t)(w2 + k[4]) * (uint64_t)(w3 + k[5]);
}

// NH of block b (words 2b, 2b+1) of a record of n bytes; the second word only if it
// exists (16*(2b+1) < n).
__device__ __forceinline__ void nh_blk(const Blk& x, const LaneKeys& K, uint64_t n, uint64_t b, uint64_t& A,
                                       uint64_t& B) {
    nh_word(x.v[0], x.v[1], x.v[2], x.v[3], K.k[0], A, B);
    if (32 * b + 16 < n) nh_word(x.v[4], x.v[5], x.v[6], x.v[7], K.k[1], A, B);
}

// H3 helpers (byte comparison, mismatch reporting)
__device__ __forceinline__ int blk_diff(const Blk& x, const Blk& y) {
    // -1: equal; 0: first word differs; 1: only second word differs
    uint32_t d0 = (x.v[0] ^ y.v[0]) | (x.v[1] ^ y.v[1]) | (x.v[2] ^ y.v[2]) | (x.v[3] ^ y.v[3]);
    uint32_t d1 = (x.v[4] ^ y.v[4]) | (x.v[5] ^ y.v[5]) | (x.v[6] ^ y.v[6]) | (x.v[7] ^ y.v[7]);
    return d0 ? 0 : (d1 ? 1 : -1);
}

__device__ __forceinline__ void report_mismatch(Work& W, uint32_t m, uint64_t word, uint32_t* res_out, bool atomic) {
    if (atomic) {
        atomicMin((unsigned long long*)&W.mis[m], (unsigned long long)word);
        if (atomicExch(&W.eq[m], 0u) == 1u) res_out[atomicAdd(&W.counters[0], 1u)] = m;
    } else {
        W.mis[m] = word;
        W.eq[m] = 0;
        res_out[atomicAdd(&W.counters[0], 1u)] = m;
    }
}

constexpr int kVerifyU = 2;

// ----------------------------------------------------------------------------
// H1a: payloads <= small_bytes, one 8-lane group ("octet") per record.  Lane g
// reads 32-B block g of each 256-B stripe: positions 2g, 2g+1.
// ----------------------------------------------------------------------------
constexpr int kSmallU = 2;

__global__ void __launch_bounds__(256, 4) k_hash_small(DevLog L, uint32_t small_bytes, uint64_t* __restrict__ accA,
                                                    uint64_t* __restrict__ accB) {
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3;
    const uint32_t noct = (gridDim.x * blockDim.x) >> 3;
    const unsigned omask = 0xFFu << (threadIdx.x & 24);
    LaneKeys K0;
    load_keys(K0, 2 * g, 0);
    for (uint32_t i = oct; i < L.n_small; i += noct) {
        const uint32_t r = L.small_order[i];
        const uint64_t n = L.size[r];
        const uint8_t* base = L.arena + L.off[r];
        const uint32_t nblk = (uint32_t)((n + 31) >> 5);
        LaneKeys K = K0;
        uint64_t A = 0, B = 0;
        for (uint32_t b0 = 0; b0 < nblk; b0 += 8 * kSmallU) {
            Blk x[kSmallU];
#pragma unroll
            for (int u = 0; u < kSmallU; ++u) {
                uint32_t b = b0 + 8 * u + g;
                x[u] = b < nblk ? ld_stream(base + 32ull * b) : zero_blk();
            }
#pragma unroll
            for (int u = 0; u < kSmallU; ++u) {
                uint32_t b = b0 + 8 * u + g;
                if (b < nblk) {
                    mask_tail(x[u], n, b);
                    nh_blk(x[u], K, n, b, A, B);
                }
                advance<1>(K);
            }
        }
#pragma unroll
        for (int o = 4; o; o >>= 1) {
            A += __shfl_xor_sync(omask, A, o);
            B += __shfl_xor_sync(omask, B, o);
        }
        if (g == 0) {
            accA[r] = A;
            accB[r] = B;
        }
    }
}

// ----------------------------------------------------------------------------
// H1b: payloads > small_bytes, one warp per (record, chunk) work unit.  Lane l
// reads block b0 + l + 32t: positions 2(l mod 8), stripe (b0 + l)/8 + 4t.
// Each unit writes its partial (A, B); k_hash_combine sums them per record.
// ----------------------------------------------------------------------------
constexpr int kLargeU = 4;

// phase 0: every unit; phase 1: first chunks only (the prefix pass of round 0).
__global__ void __launch_bounds__(256, 3) k_hash_large(DevLog L, const uint2* __restrict__ items,
                                                    const uint32_t* __restrict__ n_items_ptr, uint32_t chunk_bytes,
                                                    uint64_t* __restrict__ part, int phase) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t n_items = *n_items_ptr;
    const uint32_t cblk = chunk_bytes >> 5;
    for (uint32_t it = warp; it < n_items; it += nwarps) {
        const uint2 w = items[it];
        const uint32_t r = w.x;
        if (phase == 1 && w.y != 0) continue;
        const uint64_t n = L.size[r];
        const uint8_t* base = L.arena + L.off[r];
        const uint32_t nblk = (uint32_t)((n + 31) >> 5);
        const uint32_t bb = w.y * cblk;
        const uint32_t be = min(bb + cblk, nblk);
        LaneKeys K;
        load_keys(K, 2 * (lane & 7), (uint32_t)((bb + lane) >> 3));
        uint64_t A = 0, B = 0;
        for (uint32_t b0 = bb; b0 < be; b0 += 32 * kLargeU) {
            Blk x[kLargeU];
#pragma unroll
            for (int u = 0; u < kLargeU; ++u) {
                uint32_t b = b0 + 32 * u + lane;
                x[u] = b < be ? ld_stream(base + 32ull * b) : zero_blk();
            }
#pragma unroll
            for (int u = 0; u < kLargeU; ++u) {
                uint32_t b = b0 + 32 * u + lane;
                if (b < be) {
                    mask_tail(x[u], n, b);
                    nh_blk(x[u], K, n, b, A, B);
                }
                advance<4>(K);
            }
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
            B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
        }
        if (lane == 0) {
            part[2ull * it] = A;
            part[2ull * it + 1] = B;
        }
    }
}

// Work-unit planning for H1b / H3b: counts -> exclusive scan -> scatter.
__global__ void k_hash_count(DevLog L, uint32_t small_bytes, uint32_t chunk_bytes, uint32_t* __restrict__ cnt) {
    uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r > L.n) return;
    uint32_t c = 0;
    if (r < L.n) {
        uint64_t n = L.size[r];
        if (n > small_bytes) c = (uint32_t)((n + chunk_bytes - 1) / chunk_bytes);
    }
    cnt[r] = c;
}

__global__ void k_hash_fill(DevLog L, uint32_t small_bytes, uint32_t chunk_bytes, const uint32_t* __restrict__ start,
                            uint2* __restrict__ items) {
    const uint32_t* nolist = nullptr;
    FFM_WARP_COMPACT(L.n, nolist, (L.size[r_] > small_bytes), {
        const uint32_t c_n = start[rec + 1] - start[rec];
        const uint32_t s0 = start[rec];
        for (uint32_t c = lane; c < c_n; c += 32) items[s0 + c] = make_uint2(rec, c);
    })
}

// ----------------------------------------------------------------------------
// H2: group-by (size, digest) in an open-addressing table; value = min local index
// ("the first transfer").  Round 0 keys all records from their digest;
// resolve rounds re-key residual lists (k_refine) and reuse this kernel.
// ----------------------------------------------------------------------------
__global__ void k_group_insert(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list,
                               uint64_t cap_mask, uint64_t digest_mask, int round, uint32_t small_bytes) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_list) return;
    uint32_t r = list ? list[i] : i;
    uint64_t key;
    if (round <= 0) {                 // 0: fused round 0 (prefix keys); -1: two-pass round 0
        uint64_t n = L.size[r];
        if (n <= small_bytes || round < 0) {
            // small payload: its full digest
            uint64_t d = finalize_digest(W.accA[r], W.accB[r], n);
            W.digest[r] = d;
            key = group_key(d, n, digest_mask, L.chan[r]);
        } else {
            // large payload: the digest of its FIRST chunk (computed by the prefix pass);
            // equal payloads have equal first chunks, so every candidate still shares a group
            const uint32_t it = W.hstart[r];
            uint64_t pd = finalize_digest(W.hpart[2ull * it], W.hpart[2ull * it + 1], n);
            key = group_key(pd, n, digest_mask, L.chan[r]);
        }
        W.key[r] = key;
    } else {
        key = W.key[r];
    }
    uint64_t h = key & cap_mask;
    while (true) {
        unsigned long long prev =
            atomicCAS((unsigned long long*)&W.tkey[h], (unsigned long long)kEmptyKey, (unsigned long long)key);
        if (prev == kEmptyKey || prev == key) break;
        h = (h + 1) & cap_mask;
    }
    atomicMin(&W.tval[h], r);
    W.slot[r] = (uint32_t)h;
}

// Leader lookup.  Members (leader != self) are reset for verification; a large
// member of its leader's size gets a position in its leader's group so that the
// verify work of a class is laid out chunk-major: (chunk c, member p) at
// lstart[leader] + c * gcount[leader] + p -- all members read leader chunk c back
// to back, so the leader streams from HBM once and is re-read from L2.
__global__ void k_leader(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list, uint32_t small_bytes,
                         uint32_t chunk_bytes, uint32_t* __restrict__ res_out) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    bool member = false;
    if (i < n_list) {
        uint32_t r = list ? list[i] : i;
        uint32_t ld = W.tval[W.slot[r]];
        W.leader[r] = ld;
        if (ld != r) {
            member = true;
            uint64_t n = L.size[r];
            if (L.size[ld] != n || L.chan[ld] != L.chan[r]) {
                // a key collision across sizes / channels: not equal by definition
                W.eq[r] = 0;
                W.mis[r] = 0;
                res_out[atomicAdd(&W.counters[0], 1u)] = r;
            } else {
                W.eq[r] = 1;
                W.mis[r] = ~0ull;
            }
            if (n > small_bytes && L.size[ld] == n && L.chan[ld] == L.chan[r]) {
                atomicAdd(&W.lcount[ld], (uint32_t)((n + chunk_bytes - 1) / chunk_bytes));
                W.pos[r] = atomicAdd(&W.gcount[ld], 1u);
            }
        }
    }
    unsigned b = __ballot_sync(0xFFFFFFFFu, member);
    if ((threadIdx.x & 31) == 0 && b) atomicAdd(&W.counters[1], (uint32_t)__popc(b));
}

// Round 0 leader lookup.  Small payloads as in k_leader.  A large payload joins the
// fused pass's group of its leader (same size and channel): the group's work is laid
// out chunk-major, (chunk c, position p) at lstart[head] + c * (gcount[head] + 1) + p,
// with the leader itself at p = 0 -- the leader's chunk c is read from HBM once, by
// its own hashing unit, and re-read from L2 by every member comparing against it.
__global__ void k_leader0(DevLog L, Work W, uint32_t n, uint32_t small_bytes, uint32_t chunk_bytes,
                          uint32_t* __restrict__ res_out) {
    uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    bool member = false;
    if (r < n) {
        const uint32_t ld = W.tval[W.slot[r]];
        W.leader[r] = ld;
        const uint64_t sz = L.size[r];
        const bool same = L.size[ld] == sz && L.chan[ld] == L.chan[r];
        if (ld != r) {
            member = true;
            if (!same) {
                W.eq[r] = 0;            // key collision across sizes / channels: not equal
                W.mis[r] = 0;
                res_out[atomicAdd(&W.counters[0], 1u)] = r;
            } else {
                W.eq[r] = 1;
                W.mis[r] = ~0ull;
            }
        }
        if (sz > small_bytes) {
            uint32_t head = r, p = 0;
            if (ld != r && same) {
                head = ld;
                p = 1u + atomicAdd(&W.gcount[ld], 1u);
            }
            W.fhead[r] = head;
            W.pos[r] = p;
            atomicAdd(&W.lcount[head], (uint32_t)((sz + chunk_bytes - 1) / chunk_bytes));
        }
    }
    unsigned b = __ballot_sync(0xFFFFFFFFu, member);
    if ((threadIdx.x & 31) == 0 && b) atomicAdd(&W.counters[1], (uint32_t)__popc(b));
}

__global__ void k_fused_fill(DevLog L, Work W, uint32_t small_bytes, uint32_t chunk_bytes) {
    const uint32_t* nolist = nullptr;
    FFM_WARP_COMPACT(L.n, nolist, (L.size[r_] > small_bytes), {
        const uint32_t h = W.fhead[rec];
        const uint32_t k = W.gcount[h] + 1, p = W.pos[rec], base = W.lstart[h];
        const uint32_t c_n = (uint32_t)((L.size[rec] + chunk_bytes - 1) / chunk_bytes);
#if FFM_FUSED_LEADER_FIRST
        // skewed chunk-major layout: the leader runs D chunks ahead of its members, so a
        // member compares against a leader chunk fetched a little earlier -- an L2 hit,
        // not a wait on the same in-flight miss, and not yet evicted.  Step t holds the
        // leader's chunk t and the members' chunk t - D; no holes:
        //   [0, D) leader only | [D, nch) leader + members | [nch, nch + D) members only
        const uint32_t D = min((uint32_t)FFM_FUSED_SKEW, c_n);
        for (uint32_t c = lane; c < c_n; c += 32) {
            uint32_t at;
            if (p == 0) {
                at = c < D ? c : D + (c - D) * k;
            } else {
                const uint32_t t = c + D;
                at = t < c_n ? D + c * k + p : D + (c_n - D) * k + (t - c_n) * (k - 1) + (p - 1);
            }
            W.vitems[base + at] = make_uint2(rec, c);
        }
#else
        for (uint32_t c = lane; c < c_n; c += 32) W.vitems[base + c * k + p] = make_uint2(rec, c);
#endif
    })
}

// With FFM_FLAG_PREFILTER a leader whose fused group has no member has a unique
// (size, first chunk, channel): it cannot equal any other payload, so its remaining
// chunks are not read.
__device__ __forceinline__ bool prefix_unique(const Work& W, uint32_t r) {
    return W.fhead[r] == r && W.gcount[r] == 0 && W.leader[r] == r;
}

// H1 + H3 fused for large payloads (round 0): one pass over every chunk c >= 1 hashes
// it (chunk 0 was hashed by the prefix pass) and, for a member, byte-compares it with
// the leader's chunk c (L2-resident: the group's units run back to back); members
// also compare chunk 0.  A member's first mismatching word is the exact minimum (a
// chunk's compare is skipped only when a lower mismatch is known); failures go to the
// residual list and are resolved exactly (H4) with their full digests.
template <int U, bool kCmp>
__device__ __forceinline__ void fused_chunk(const uint8_t* pr, const uint8_t* ph, uint64_t n, uint32_t bb,
                                            uint32_t be, int lane, bool hashc, bool keep_own, LaneKeys& K,
                                            uint64_t& A, uint64_t& B, uint64_t& found) {
    for (uint32_t b0 = bb; b0 < be; b0 += 32 * U) {
        Blk x[U], y[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t b = b0 + 32 * u + lane;
            // a group leader's own chunk is re-read by its members: keep it in L2
            x[u] = b < be ? (keep_own ? ld_keep(pr + 32ull * b) : ld_stream(pr + 32ull * b)) : zero_blk();
#if FFM_FUSED_Y_POLICY == 0
            if (kCmp) y[u] = b < be ? ld_remote(ph + 32ull * b) : zero_blk();   // default L2 policy
#elif FFM_FUSED_Y_POLICY == 2
            if (kCmp) y[u] = b < be ? ld_stream(ph + 32ull * b) : zero_blk();
#else
            if (kCmp) y[u] = b < be ? ld_keep(ph + 32ull * b) : zero_blk();
#endif
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t b = b0 + 32 * u + lane;
            if (b < be) {
                mask_tail(x[u], n, b);
                if (hashc) nh_blk(x[u], K, n, b, A, B);
                if (kCmp) {
                    mask_tail(y[u], n, b);
                    int d = blk_diff(x[u], y[u]);
                    if (d >= 0 && found == ~0ull) found = 2ull * b + d;
                }
            }
            advance<4>(K);
        }
    }
}

#ifndef FFM_FUSED_MINB
#define FFM_FUSED_MINB 3
#endif
__global__ void __launch_bounds__(256, FFM_FUSED_MINB) k_fused(DevLog L, Work W, const uint32_t* __restrict__ n_items_ptr,
                                                  uint32_t chunk_bytes, int prefilter, uint32_t* res_out) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t n_items = *n_items_ptr;
    const uint32_t cblk = chunk_bytes >> 5;
    for (uint32_t it = warp; it < n_items; it += nwarps) {
        const uint2 w = W.vitems[it];
        const uint32_t r = w.x, c = w.y;
        const uint32_t h = W.fhead[r];
        const bool hashc = c > 0 && !(prefilter && prefix_unique(W, r));
        bool cmp = h != r;
        if (cmp) {
            uint64_t known = lane == 0 ? *((volatile uint64_t*)&W.mis[r]) : 0;
            known = __shfl_sync(0xFFFFFFFFu, known, 0);
            cmp = 2ull * c * cblk < known;         // no lower mismatch known yet
        }
        if (!hashc && !cmp) continue;
        const uint64_t n = L.size[r];
        const uint32_t nblk = (uint32_t)((n + 31) >> 5);
        const uint32_t bb = c * cblk, be = min(bb + cblk, nblk);
        const uint8_t* pr = L.arena + L.off[r];
        const uint8_t* ph = L.arena + L.off[h];
        const bool keep_own = FFM_FUSED_KEEP_OWN && h == r && W.gcount[r] > 0;
        LaneKeys K;
        load_keys(K, 2 * (lane & 7), (bb + lane) >> 3);
        uint64_t A = 0, B = 0, found = ~0ull;
        if (cmp)
            fused_chunk<FFM_FUSED_CMP_U, true>(pr, ph, n, bb, be, lane, hashc, keep_own, K, A, B, found);
        else
            fused_chunk<4, false>(pr, ph, n, bb, be, lane, hashc, keep_own, K, A, B, found);
        if (hashc) {
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
                B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
            }
            if (lane == 0) {
                const uint64_t slot = W.hstart[r] + c;
                W.hpart[2 * slot] = A;
                W.hpart[2 * slot + 1] = B;
            }
        }
        if (cmp && __any_sync(0xFFFFFFFFu, found != ~0ull)) {
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                uint64_t other = __shfl_xor_sync(0xFFFFFFFFu, found, o);
                found = other < found ? other : found;
            }
            if (lane == 0) report_mismatch(W, r, found, res_out, true);
        }
    }
}

// Combine the chunk partial sums of large records (NH is a plain sum, so the record's
// accumulators are the sums of its chunks' -- no atomics, deterministic) and finish
// their digests.  Also totals the bytes hashed beyond first chunks (roofline stats).
__global__ void __launch_bounds__(256) k_hash_combine(DevLog L, Work W, uint32_t small_bytes, uint32_t chunk_bytes,
                                                      int prefilter) {
    __shared__ unsigned long long s_rest[8];
    const int lane = threadIdx.x & 31;
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    const bool act = i < L.n && L.size[i] > small_bytes;
    unsigned bal = __ballot_sync(0xFFFFFFFFu, act);
    unsigned long long rest = 0;
    while (bal) {
        const int src = __ffs(bal) - 1;
        bal &= bal - 1;
        const uint32_t rec = __shfl_sync(0xFFFFFFFFu, i, src);
        const uint32_t s0 = W.hstart[rec];
        const bool skip = prefilter && prefix_unique(W, rec);
        const uint32_t e0 = skip ? s0 + 1 : W.hstart[rec + 1];
        uint64_t A = 0, B = 0;
        for (uint32_t it = s0 + lane; it < e0; it += 32) {
            A += W.hpart[2ull * it];
            B += W.hpart[2ull * it + 1];
        }
        for (int o = 16; o; o >>= 1) {
            A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
            B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
        }
        const uint64_t n = L.size[rec];
        if (lane == 0) {
            W.accA[rec] = A;
            W.accB[rec] = B;
            W.digest[rec] = finalize_digest(A, B, n);
            if (!skip && n > chunk_bytes) rest += n - chunk_bytes;
        }
    }
    if (lane == 0) s_rest[threadIdx.x >> 5] = rest;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += s_rest[w];
        if (t) atomicAdd((unsigned long long*)(W.counters + 4), t);
    }
}

__global__ void k_verify_fill(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list,
                              uint32_t small_bytes, uint32_t chunk_bytes) {
    FFM_WARP_COMPACT(n_list, list,
                     (W.leader[r_] != r_ && L.size[r_] > small_bytes && L.size[W.leader[r_]] == L.size[r_] &&
                      L.chan[W.leader[r_]] == L.chan[r_]), {
        const uint32_t ld = W.leader[rec];
        const uint64_t n = L.size[rec];
        const uint32_t c_n = (uint32_t)((n + chunk_bytes - 1) / chunk_bytes);
        const uint32_t base = W.lstart[ld], k = W.gcount[ld], p = W.pos[rec];
        for (uint32_t c = lane; c < c_n; c += 32) W.vitems[base + c * k + p] = make_uint2(rec, c);
    })
}

// ----------------------------------------------------------------------------
// H3: byte verification of every member against its candidate leader.  Records the
// first mismatching 16-B word (exact minimum: a chunk is skipped only when a
// mismatch at a lower word is already known), and appends failures to a residual list.
// ----------------------------------------------------------------------------

__global__ void __launch_bounds__(256, 4) k_verify_small(DevLog L, Work W, const uint32_t* __restrict__ list,
                                                      uint32_t n_list, uint32_t small_bytes, uint32_t* res_out) {
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3;
    const uint32_t noct = (gridDim.x * blockDim.x) >> 3;
    const unsigned omask = 0xFFu << (threadIdx.x & 24);
    for (uint32_t i = oct; i < n_list; i += noct) {
        const uint32_t m = list ? list[i] : i;
        const uint32_t ld = W.leader[m];
        if (ld == m) continue;
        const uint64_t n = L.size[m];
        if (n > small_bytes || L.size[ld] != n || L.chan[ld] != L.chan[m]) continue;   // large / k_leader
        uint64_t word = ~0ull;
        {
            const uint8_t* pm = L.arena + L.off[m];
            const uint8_t* pl = L.arena + L.off[ld];
            const uint32_t nblk = (uint32_t)((n + 31) >> 5);
            for (uint32_t b0 = 0; b0 < nblk; b0 += 8 * kVerifyU) {
                Blk x[kVerifyU], y[kVerifyU];
#pragma unroll
                for (int u = 0; u < kVerifyU; ++u) {
                    uint32_t b = b0 + 8 * u + g;
                    x[u] = b < nblk ? ld_stream(pm + 32ull * b) : zero_blk();
                    y[u] = b < nblk ? ld_keep(pl + 32ull * b) : zero_blk();
                }
                uint64_t found = ~0ull;
#pragma unroll
                for (int u = 0; u < kVerifyU; ++u) {
                    uint32_t b = b0 + 8 * u + g;
                    if (b < nblk) {
                        mask_tail(x[u], n, b);
                        mask_tail(y[u], n, b);
                        int d = blk_diff(x[u], y[u]);
                        if (d >= 0 && found == ~0ull) found = 2ull * b + d;
                    }
                }
                // octet min over lanes
#pragma unroll
                for (int o = 4; o; o >>= 1) {
                    uint64_t other = __shfl_xor_sync(omask, found, o);
                    found = other < found ? other : found;
                }
                if (found != ~0ull) {
                    word = found;
                    break;
                }
            }
        }
        if (word != ~0ull && g == 0) report_mismatch(W, m, word, res_out, false);
    }
}

__global__ void __launch_bounds__(256, 3) k_verify_large(DevLog L, Work W, const uint2* __restrict__ items,
                                                      const uint32_t* __restrict__ n_items_ptr, uint32_t chunk_bytes,
                                                      uint32_t* res_out) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t n_items = *n_items_ptr;
    const uint32_t cblk = chunk_bytes >> 5;
    for (uint32_t it = warp; it < n_items; it += nwarps) {
        const uint2 w = items[it];
        const uint32_t m = w.x;
        const uint32_t ld = W.leader[m];
        const uint64_t n = L.size[m];
        if (L.size[ld] != n) {
            if (lane == 0) report_mismatch(W, m, 0, res_out, true);
            continue;
        }
        const uint32_t nblk = (uint32_t)((n + 31) >> 5);
        const uint32_t bb = w.y * cblk;
        const uint32_t be = min(bb + cblk, nblk);
        uint64_t known = lane == 0 ? *((volatile uint64_t*)&W.mis[m]) : 0;
        known = __shfl_sync(0xFFFFFFFFu, known, 0);
        if (2 * bb >= known) continue;   // a mismatch at a lower word is already known
        const uint8_t* pm = L.arena + L.off[m];
        const uint8_t* pl = L.arena + L.off[ld];
        uint64_t word = ~0ull;
        for (uint32_t b0 = bb; b0 < be; b0 += 32 * kVerifyU) {
            Blk x[kVerifyU], y[kVerifyU];
#pragma unroll
            for (int u = 0; u < kVerifyU; ++u) {
                uint32_t b = b0 + 32 * u + lane;
                x[u] = b < be ? ld_stream(pm + 32ull * b) : zero_blk();
                y[u] = b < be ? ld_keep(pl + 32ull * b) : zero_blk();
            }
            uint64_t found = ~0ull;
#pragma unroll
            for (int u = 0; u < kVerifyU; ++u) {
                uint32_t b = b0 + 32 * u + lane;
                if (b < be) {
                    mask_tail(x[u], n, b);
                    mask_tail(y[u], n, b);
                    int d = blk_diff(x[u], y[u]);
                    if (d >= 0 && found == ~0ull) found = 2ull * b + d;
                }
            }
            if (__any_sync(0xFFFFFFFFu, found != ~0ull)) {
#pragma unroll
                for (int o = 16; o; o >>= 1) {
                    uint64_t other = __shfl_xor_sync(0xFFFFFFFFu, found, o);
                    found = other < found ? other : found;
                }
                word = found;
                break;
            }
        }
        if (word != ~0ull && lane == 0) report_mismatch(W, m, word, res_out, true);
    }
}

// ----------------------------------------------------------------------------
// H4: re-key residual members.  Round 1 refines by the full, untruncated NH sums;
// later rounds by (first mismatching word index vs the previous leader, that word).
// Byte-equal records always receive equal keys, so exactness never depends on the key.
// ----------------------------------------------------------------------------
__global__ void k_refine(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list, int round,
                         uint64_t refine_mask) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_list) return;
    uint32_t m = list[i];
    uint64_t ref;
    if (round == 1) {
        ref = (fmix64(W.accA[m]) ^ W.accB[m]) & refine_mask;
    } else {
        uint64_t q = W.mis[m];
        uint64_t n = L.size[m];
        uint32_t w[4] = {0, 0, 0, 0};
        if (16 * q < n) {
            const uint8_t* p = L.arena + L.off[m] + 16 * q;
            for (int j = 0; j < 16 && 16 * q + j < n; ++j) w[j >> 2] |= (uint32_t)p[j] << (8 * (j & 3));
        }
        ref = fmix64(q * 0x9E3779B97F4A7C15ull ^ ((uint64_t)w[1] << 32 | w[0])) ^ fmix64((uint64_t)w[3] << 32 | w[2]);
    }
    W.key[m] = not_empty(fmix64(W.key[m] ^ fmix64(ref + (uint64_t)round)));
}

// ----------------------------------------------------------------------------
// H5 + H6: labels and per-site benefit.  Integer sums are exact and order
// independent.  With n_sites fitting in shared memory each block keeps a private
// histogram (no global atomic contention on hot call sites -- Zipf-skewed logs put
// 10% of all records on one site) and a second kernel sums the block partials.
// ----------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_label_hist(DevLog L, const uint32_t* __restrict__ leader, uint32_t n_sites,
                                                    int64_t* __restrict__ dup_out, uint64_t* __restrict__ part,
                                                    uint32_t* __restrict__ cpart) {
    extern __shared__ unsigned long long sben[];
    uint32_t* scnt = (uint32_t*)(sben + n_sites);
    for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
        sben[s] = 0;
        scnt[s] = 0;
    }
    __syncthreads();
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < L.n; r += gridDim.x * blockDim.x) {
        uint32_t ld = leader[r];
        int64_t d = ld == r ? -1 : (int64_t)L.gid[ld];
        dup_out[r] = d;
        if (d >= 0) {
            const uint32_t s = L.site[r];
            atomicAdd(&sben[s], (unsigned long long)L.dur[r]);
            atomicAdd(&scnt[s], 1u);
        }
    }
    __syncthreads();
    uint64_t* row = part + (uint64_t)blockIdx.x * n_sites;
    uint32_t* crow = cpart + (uint64_t)blockIdx.x * n_sites;
    for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
        row[s] = sben[s];
        crow[s] = scnt[s];
    }
}

__global__ void k_site_reduce(const uint64_t* __restrict__ part, const uint32_t* __restrict__ cpart, uint32_t rows,
                              uint32_t n_sites, uint64_t* __restrict__ ben, uint64_t* __restrict__ cnt) {
    uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n_sites) return;
    uint64_t acc = 0, c = 0;
    for (uint32_t b = 0; b < rows; ++b) {
        acc += part[(uint64_t)b * n_sites + s];
        c += cpart[(uint64_t)b * n_sites + s];
    }
    ben[s] = acc;
    cnt[s] = c;
}

__global__ void __launch_bounds__(256) k_label_global(DevLog L, const uint32_t* __restrict__ leader,
                                                      int64_t* __restrict__ dup_out, uint64_t* __restrict__ ben,
                                                      uint64_t* __restrict__ cnt) {
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < L.n; r += gridDim.x * blockDim.x) {
        uint32_t ld = leader[r];
        int64_t d = ld == r ? -1 : (int64_t)L.gid[ld];
        dup_out[r] = d;
        if (d >= 0) {
            atomicAdd((unsigned long long*)&ben[L.site[r]], (unsigned long long)L.dur[r]);
            atomicAdd((unsigned long long*)&cnt[L.site[r]], 1ull);
        }
    }
}

// Folded grouping (S8(f) #1): per-group sums of per-site values.
__global__ void k_fold(const uint64_t* __restrict__ site_vals, const uint32_t* __restrict__ site_to_group,
                       uint32_t n_sites, uint64_t* __restrict__ group_vals) {
    uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n_sites) return;
    uint64_t v = site_vals[s];
    if (v) atomicAdd((unsigned long long*)&group_vals[site_to_group[s]], (unsigned long long)v);
}

// ----------------------------------------------------------------------------
// H0 helper: snapshot device-resident payloads into the arena (one warp per record).
// desc[3i] = src address, desc[3i+1] = arena offset, desc[3i+2] = size.
// ----------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_gather(const uint64_t* __restrict__ desc, uint32_t n,
                                                uint8_t* __restrict__ arena) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    constexpr int U = 4;   // 4 x 16 B in flight per lane: PCIe (pinned host) reads are latency-bound
    for (uint32_t i = warp; i < n; i += nwarps) {
        const uint8_t* src = (const uint8_t*)desc[3 * i];
        uint8_t* dst = arena + desc[3 * i + 1];
        const uint64_t sz = desc[3 * i + 2];
        if (((uintptr_t)src & 15) == 0) {
            const uint64_t nv = sz >> 4;
            for (uint64_t k0 = 0; k0 < nv; k0 += 32 * U) {
                uint4 v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    uint64_t k = k0 + 32 * u + lane;
                    if (k < nv) v[u] = ((const uint4*)src)[k];
                }
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    uint64_t k = k0 + 32 * u + lane;
                    if (k < nv) ((uint4*)dst)[k] = v[u];
                }
            }
            for (uint64_t k = (nv << 4) + lane; k < sz; k += 32) dst[k] = src[k];
        } else {
            for (uint64_t k = lane; k < sz; k += 32) dst[k] = src[k];
        }
    }
}

// ----------------------------------------------------------------------------
// Launchers
// ----------------------------------------------------------------------------
uint32_t blocks_for(uint64_t threads, uint32_t bs) {
    return (uint32_t)((threads + bs - 1) / bs);
}

// Opt-in dynamic shared memory for a kernel, once per (device, kernel).
bool smem_configured(const void* kernel, int bytes) {
    static std::mutex mu;
    static std::unordered_map<uint64_t, int> done;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return false;
    const uint64_t key = (uint64_t)(uintptr_t)kernel * 131 + (uint64_t)dev;
    std::lock_guard<std::mutex> g(mu);
    auto it = done.find(key);
    if (it != done.end() && it->second >= bytes) return true;
    if (cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess) return false;
    done[key] = bytes;
    return true;
}

// Persistent launch: exactly the resident blocks (num_sms x occupancy), one wave.
uint32_t resident_grid(const void* kernel, int num_sms, int block) {
    static std::mutex mu;
    static std::unordered_map<const void*, int> cache;
    std::lock_guard<std::mutex> g(mu);
    auto it = cache.find(kernel);
    int occ;
    if (it == cache.end()) {
        occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, block, 0) != cudaSuccess || occ < 1) {
            cudaGetLastError();
            occ = 1;
        }
        cache[kernel] = occ;
    } else {
        occ = it->second;
    }
    return (uint32_t)(occ * num_sms);
}

#define FFM_LAUNCH_CHECK() \
    do {                                      \
        if (cudaGetLastError() != cudaSuccess) return -1; \
    } while (0)

size_t cub_scan_bytes(uint64_t n) {
    size_t bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, bytes, (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)n);
    return bytes;
}

int launch_hash_small(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    if (L.n == 0) return 0;
    if (L.n_small == 0) return 0;
    uint32_t grid = resident_grid((const void*)k_hash_small, P.num_sms);
    uint32_t need = blocks_for((uint64_t)L.n_small * 8);
    k_hash_small<<<need < grid ? need : grid, 256, 0, st>>>(L, P.small_bytes, W.accA, W.accB);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_hash_plan(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    k_hash_count<<<blocks_for((uint64_t)L.n + 1), 256, 0, st>>>(L, P.small_bytes, P.chunk_bytes, W.hcount);
    FFM_LAUNCH_CHECK();
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.hcount, W.hstart, (int)(L.n + 1), st) != cudaSuccess)
        return -1;
    if (L.n) {
        k_hash_fill<<<blocks_for((uint64_t)L.n), 256, 0, st>>>(L, P.small_bytes, P.chunk_bytes, W.hstart,
                                                                    W.hitems);
        FFM_LAUNCH_CHECK();
    }
    return 3;
}

int launch_hash_large(const DevLog& L, Work& W, const Params& P, uint64_t n_items, cudaStream_t st, int phase) {
    if (n_items == 0) return 0;
    uint32_t grid = resident_grid((const void*)k_hash_large, P.num_sms);
    uint32_t need = blocks_for(n_items * 32);
    k_hash_large<<<need < grid ? need : grid, 256, 0, st>>>(L, W.hitems, W.hstart + L.n, P.chunk_bytes, W.hpart,
                                                            phase);
    FFM_LAUNCH_CHECK();
    return 1;
}

// Round 0, large payloads: fused groups (scan of lcount), work units, the fused
// hash + compare pass, then the per-record combine of chunk partial sums.
int launch_combine(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    if (L.n == 0) return 0;
    k_hash_combine<<<blocks_for((uint64_t)L.n), 256, 0, st>>>(L, W, P.small_bytes, P.chunk_bytes, 0);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_fused(const DevLog& L, Work& W, const Params& P, uint64_t n_units, bool prefilter, uint32_t* res_out,
                 cudaStream_t st, cudaEvent_t ev_a, cudaEvent_t ev_b) {
    if (L.n == 0 || n_units == 0) return 0;
    int k = 0;
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.lcount, W.lstart, (int)(L.n + 1), st) != cudaSuccess)
        return -1;
    ++k;
    k_fused_fill<<<blocks_for((uint64_t)L.n), 256, 0, st>>>(L, W, P.small_bytes, P.chunk_bytes);
    FFM_LAUNCH_CHECK();
    ++k;
    if (ev_a && cudaEventRecord(ev_a, st) != cudaSuccess) return -1;
    uint32_t grid = resident_grid((const void*)k_fused, P.num_sms);
    uint32_t need = blocks_for(n_units * 32);
    k_fused<<<need < grid ? need : grid, 256, 0, st>>>(L, W, W.lstart + L.n, P.chunk_bytes, prefilter ? 1 : 0,
                                                       res_out);
    FFM_LAUNCH_CHECK();
    ++k;
    if (ev_b && cudaEventRecord(ev_b, st) != cudaSuccess) return -1;
    k_hash_combine<<<blocks_for((uint64_t)L.n), 256, 0, st>>>(L, W, P.small_bytes, P.chunk_bytes,
                                                              prefilter ? 1 : 0);
    FFM_LAUNCH_CHECK();
    return k + 1;
}

int launch_group(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list, uint64_t cap,
                 int round, uint32_t* res_out, cudaStream_t st) {
    if (n_list == 0) return 0;
    int k = 0;
    if (round > 0) {
        k_refine<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, round, P.refine_mask);
        FFM_LAUNCH_CHECK();
        ++k;
    }
    if (cudaMemsetAsync(W.tkey, 0xFF, cap * sizeof(uint64_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(W.tval, 0xFF, cap * sizeof(uint32_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(W.lcount, 0, ((uint64_t)L.n + 1) * sizeof(uint32_t), st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(W.gcount, 0, ((uint64_t)L.n + 1) * sizeof(uint32_t), st) != cudaSuccess) return -1;
    k_group_insert<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, cap - 1, P.digest_mask, round,
                                                        P.small_bytes);
    FFM_LAUNCH_CHECK();
    if (round == 0)
        k_leader0<<<blocks_for(n_list), 256, 0, st>>>(L, W, n_list, P.small_bytes, P.chunk_bytes, res_out);
    else if (round < 0)
        k_leader<<<blocks_for(n_list), 256, 0, st>>>(L, W, nullptr, n_list, P.small_bytes, P.chunk_bytes, res_out);
    else
        k_leader<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, P.small_bytes, P.chunk_bytes, res_out);
    FFM_LAUNCH_CHECK();
    return k + 2;
}

int launch_verify(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                  uint32_t* res_out, uint64_t vitem_cap, cudaStream_t st, cudaStream_t side, cudaEvent_t ev_fork,
                  cudaEvent_t ev_join) {
    if (n_list == 0) return 0;
    int k = 0;
    // small members (and any size-mismatched member) on the side stream, concurrently
    // with the bandwidth-bound large path: the latency-bound small kernel fills gaps.
    cudaStream_t ss = side ? side : st;
    if (side) {
        if (cudaEventRecord(ev_fork, st) != cudaSuccess || cudaStreamWaitEvent(side, ev_fork, 0) != cudaSuccess)
            return -1;
    }
    // main pass: the size-ordered small records; resolve rounds: the residual list
    const uint32_t* slist = list ? list : L.small_order;
    const uint32_t sn = list ? n_list : L.n_small;
    uint32_t need = 0;
    if (sn) {
        uint32_t grid_s = resident_grid((const void*)k_verify_small, P.num_sms);
        need = blocks_for((uint64_t)sn * 8);
        k_verify_small<<<need < grid_s ? need : grid_s, 256, 0, ss>>>(L, W, slist, sn, P.small_bytes, res_out);
        FFM_LAUNCH_CHECK();
        ++k;
    }
    if (vitem_cap) {
        // large members: chunk-major groups per leader (scan of lcount) then scatter work units
        size_t bytes = W.cub_tmp_bytes;
        if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.lcount, W.lstart, (int)(L.n + 1), st) != cudaSuccess)
            return -1;
        ++k;
        uint32_t* n_vitems = W.lstart + L.n;   // total large verify work units
        k_verify_fill<<<blocks_for((uint64_t)n_list), 256, 0, st>>>(L, W, list, n_list, P.small_bytes,
                                                                    P.chunk_bytes);
        FFM_LAUNCH_CHECK();
        ++k;
        uint32_t grid = resident_grid((const void*)k_verify_large, P.num_sms);
        need = blocks_for(vitem_cap * 32);
        k_verify_large<<<need < grid ? need : grid, 256, 0, st>>>(L, W, W.vitems, n_vitems, P.chunk_bytes, res_out);
        FFM_LAUNCH_CHECK();
        ++k;
    }
    if (side) {
        if (cudaEventRecord(ev_join, side) != cudaSuccess || cudaStreamWaitEvent(st, ev_join, 0) != cudaSuccess)
            return -1;
    }
    return k;
}

uint32_t label_hist_rows(int num_sms) { return (uint32_t)num_sms; }

int launch_site_reduce(const uint64_t* part, const uint32_t* cpart, uint32_t rows, uint32_t n_sites, uint64_t* ben,
                       uint64_t* cnt, cudaStream_t st) {
    k_site_reduce<<<blocks_for(n_sites), 256, 0, st>>>(part, cpart, rows, n_sites, ben, cnt);
    FFM_LAUNCH_CHECK();
    return 1;
}

size_t label_smem_bytes(uint32_t n_sites) { return (size_t)n_sites * (sizeof(uint64_t) + sizeof(uint32_t)); }

int launch_label(const DevLog& L, Work& W, const Params& P, uint32_t n_sites, int64_t* dup_out, cudaStream_t st) {
    if (L.n == 0) {
        if (cudaMemsetAsync(W.ben, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
        return cudaMemsetAsync(W.cnt, 0, (uint64_t)n_sites * 8, st) == cudaSuccess ? 0 : -1;
    }
    const size_t smem = label_smem_bytes(n_sites);
    if (W.label_part && smem <= (size_t)P.max_smem) {
        if (!smem_configured((const void*)k_label_hist, P.max_smem)) return -1;
        const uint32_t rows = label_hist_rows(P.num_sms);
        k_label_hist<<<rows, 1024, smem, st>>>(L, W.leader, n_sites, dup_out, W.label_part, W.label_cpart);
        FFM_LAUNCH_CHECK();
        if (launch_site_reduce(W.label_part, W.label_cpart, rows, n_sites, W.ben, W.cnt, st) < 0) return -1;
        return 2;
    }
    if (cudaMemsetAsync(W.ben, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
    if (cudaMemsetAsync(W.cnt, 0, (uint64_t)n_sites * 8, st) != cudaSuccess) return -1;
    uint32_t grid = blocks_for(L.n);
    if (grid > (uint32_t)P.num_sms * 8) grid = (uint32_t)P.num_sms * 8;
    k_label_global<<<grid, 256, 0, st>>>(L, W.leader, dup_out, W.ben, W.cnt);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_fold(const uint64_t* site_vals, const uint32_t* site_to_group, uint32_t n_sites, uint64_t* group_vals,
                uint32_t n_groups, cudaStream_t st) {
    if (cudaMemsetAsync(group_vals, 0, (uint64_t)n_groups * 8, st) != cudaSuccess) return -1;
    if (n_sites == 0) return 0;
    k_fold<<<blocks_for(n_sites), 256, 0, st>>>(site_vals, site_to_group, n_sites, group_vals);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_gather(const uint64_t* d_desc, uint32_t n, uint8_t* arena, cudaStream_t st) {
    if (n == 0) return 0;
    uint32_t grid = blocks_for((uint64_t)n * 32);
    if (grid > 148u * 16) grid = 148u * 16;
    k_gather<<<grid, 256, 0, st>>>(d_desc, n, arena);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_zero_counters(Work& W, cudaStream_t st) {
    return cudaMemsetAsync(W.counters, 0, 16 * sizeof(uint32_t), st) == cudaSuccess ? 0 : -1;
}

}  // namespace ffm
