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
#ifndef FFM_SMALL_U
#define FFM_SMALL_U 2
#endif
constexpr int kSmallU = FFM_SMALL_U;

__global__ void __launch_bounds__(256, 4) k_hash_small(DevLog L, uint32_t small_bytes, uint64_t* __restrict__ accA,
                                                    uint64_t* __restrict__ accB, uint64_t* __restrict__ digest) {
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3;
    const uint32_t noct = (gridDim.x * blockDim.x) >> 3;
    const unsigned omask = 0xFFu << (threadIdx.x & 24);
    LaneKeys K0;
    load_keys(K0, 2 * g, 0);
    for (uint32_t i = oct; i < L.n_small; i += noct) {
        const uint32_t r = L.small_order[i];
        const uint64_t n = L.size[r];
        if (n > small_bytes) continue;   // (a residual list may hold large records too)
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
            digest[r] = finalize_digest(A, B, n);
        }
    }
}

// ----------------------------------------------------------------------------
// H1b: payloads > small_bytes, one warp per (record, chunk) work unit.  Lane l
// reads block b0 + l + 32t: positions 2(l mod 8), stripe (b0 + l)/8 + 4t.
// Each unit writes its partial (A, B); k_hash_combine sums them per record.
// ----------------------------------------------------------------------------
constexpr int kLargeU = 4;

// (two-pass round 0: every chunk of every large payload)
__global__ void __launch_bounds__(256, 3) k_hash_large(DevLog L, const uint2* __restrict__ items,
                                                    const uint32_t* __restrict__ n_items_ptr, uint32_t chunk_bytes,
                                                    uint64_t* __restrict__ part) {
    const int lane = threadIdx.x & 31;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t n_items = *n_items_ptr;
    const uint32_t cblk = chunk_bytes >> 5;
    for (uint32_t it = warp; it < n_items; it += nwarps) {
        const uint2 w = items[it];
        const uint32_t r = w.x;
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

// Fused round 0, prefix pass: one warp per large payload hashes its first
// prefix_bytes into accA / accB (the group key of H2; k_hash_combine adds the rest).
#ifndef FFM_PREFIX_MINB
#define FFM_PREFIX_MINB 4   // 4 CTAs per SM: 2x the records in flight (prefix pass 0.117 -> 0.086 ms on config 5)
#endif
__global__ void __launch_bounds__(256, FFM_PREFIX_MINB) k_prefix_hash(DevLog L, Work W, uint32_t prefix_bytes) {
    FFM_WARP_EACH(L.n_large, L.large_order[w_], true, {
        const uint64_t n = L.size[rec];
        const uint8_t* base = L.arena + L.off[rec];
        const uint32_t be = (uint32_t)((min(n, (uint64_t)prefix_bytes) + 31) >> 5);
        LaneKeys K;
        load_keys(K, 2 * (lane & 7), (uint32_t)lane >> 3);
        uint64_t A = 0, B = 0;
        for (uint32_t b0 = 0; b0 < be; b0 += 32 * kLargeU) {
            Blk x[kLargeU];
_Pragma("unroll")
            for (int u = 0; u < kLargeU; ++u) {
                const uint32_t b = b0 + 32 * u + lane;
                x[u] = b < be ? ld_stream(base + 32ull * b) : zero_blk();
            }
_Pragma("unroll")
            for (int u = 0; u < kLargeU; ++u) {
                const uint32_t b = b0 + 32 * u + lane;
                if (b < be) {
                    mask_tail(x[u], n, b);
                    nh_blk(x[u], K, n, b, A, B);
                }
                advance<4>(K);
            }
        }
_Pragma("unroll")
        for (int o = 16; o; o >>= 1) {
            A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
            B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
        }
        if (lane == 0) {
            W.accA[rec] = A;
            W.accB[rec] = B;
        }
    })
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
    FFM_WARP_EACH(L.n_large, L.large_order[w_], true, {
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
        if (round < 0) {
            // two-pass round 0: every payload by its full digest
            uint64_t d = finalize_digest(W.accA[r], W.accB[r], n);
            if (n <= small_bytes) W.digest[r] = d;
            key = group_key(d, n, digest_mask, L.chan[r]);
        } else if (n <= small_bytes) {
            // fused round 0, small payload: its first 32 bytes (equal payloads have equal
            // prefixes; k_fused_small hashes and byte-compares the rest)
            Blk x = zero_blk();
            if (n) {
                x = ld_stream(L.arena + L.off[r]);
                mask_tail(x, n, 0);
            }
            uint64_t pd = 0x5851F42D4C957F2Dull;
#pragma unroll
            for (int i = 0; i < 8; i += 2) pd = fmix64(pd ^ ((uint64_t)x.v[i + 1] << 32 | x.v[i]));
            key = group_key(pd, n, digest_mask, L.chan[r]);
        } else {
            // large payload: the NH of its first prefix_bytes (the prefix pass); equal
            // payloads have equal prefixes, so every candidate still shares a group
            uint64_t pd = finalize_digest(W.accA[r], W.accB[r], n);
            key = group_key(pd, n, digest_mask, L.chan[r]);
        }
        W.key[r] = key;
    } else {
        key = W.key[r];
    }
    uint64_t h = key & cap_mask;
    // one 64-bit slot per group: (32-bit key fingerprint << 32 | min local index) -- one
    // random access per insert and per lookup.  Two keys with the same slot chain and
    // fingerprint merge their groups; every member is byte-verified, so that only costs
    // a residual, never a wrong result.
    const unsigned long long packed = ((unsigned long long)(uint32_t)(key >> 32) << 32) | r;
    while (true) {
        const unsigned long long prev =
            atomicCAS((unsigned long long*)&W.tkey[h], (unsigned long long)kEmptyKey, packed);
        if (prev == kEmptyKey) break;
        if ((prev >> 32) == (packed >> 32)) {
            if (packed < prev) atomicMin((unsigned long long*)&W.tkey[h], packed);
            break;
        }
        h = (h + 1) & cap_mask;
    }
    W.slot[r] = (uint32_t)h;
}

// min local index of the group at table slot h
__device__ __forceinline__ uint32_t table_leader(const Work& W, uint32_t h) { return (uint32_t)W.tkey[h]; }

// Leader lookup.  Members (leader != self) are reset for verification; a large
// member of its leader's size gets a position in its leader's group so that the
// verify work of a class is laid out chunk-major: (chunk c, member p) at
// lstart[leader] + c * gcount[leader] + p -- all members read leader chunk c back
// to back, so the leader streams from HBM once and is re-read from L2.
// Exact comparison of two large members of one fused round-0 group through their
// difference lists against the group head h (k_fused_fx compared every word of both with
// h): a == b iff D(a) == D(b) as sets of (word, value) -- at a word where one differs from
// h the other must hold the same value, elsewhere both equal h.  Returns the first word
// where they differ, ~0 if equal.
__device__ __forceinline__ uint64_t diff_compare(const Work& W, uint32_t a, uint32_t b, uint32_t ca, uint32_t cb) {
    uint64_t first = ~0ull;
    for (uint32_t i = 0; i < ca; ++i) {
        const uint32_t q = W.dq[(uint64_t)a * kDiffK + i];
        const uint4 v = W.dv[(uint64_t)a * kDiffK + i];
        bool same = false;
        for (uint32_t j = 0; j < cb; ++j) {
            if (W.dq[(uint64_t)b * kDiffK + j] != q) continue;
            const uint4 u = W.dv[(uint64_t)b * kDiffK + j];
            same = ((u.x ^ v.x) | (u.y ^ v.y) | (u.z ^ v.z) | (u.w ^ v.w)) == 0;
        }
        if (!same && q < first) first = q;
    }
    for (uint32_t j = 0; j < cb; ++j) {
        const uint32_t q = W.dq[(uint64_t)b * kDiffK + j];
        bool present = false;
        for (uint32_t i = 0; i < ca; ++i) present |= W.dq[(uint64_t)a * kDiffK + i] == q;
        if (!present && q < first) first = q;
    }
    return first;
}

// use_diff: resolve rounds after a fused round 0 -- a large member whose new leader
// comes from the same round-0 group, both with complete difference lists, is settled
// here (equal, or a residual with its exact first mismatching word) and not re-read.
__global__ void k_leader(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list, uint32_t small_bytes,
                         uint32_t chunk_bytes, uint32_t* __restrict__ res_out, int use_diff) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    bool member = false;
    if (i < n_list) {
        uint32_t r = list ? list[i] : i;
        uint32_t ld = table_leader(W, W.slot[r]);
        W.leader[r] = ld;
        // residuals whose difference list overflowed: heavy mismatch against their head
        // (the adaptive round-0 choice, run_local)
        if (use_diff && L.size[r] > small_bytes && W.dcnt[r] > kDiffK) atomicAdd(&W.counters[11], 1u);
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
                bool settled = false;
                if (use_diff && W.fhead[r] == W.fhead[ld]) {
                    const uint32_t ca = W.dcnt[r], cb = W.dcnt[ld];
                    if (ca <= kDiffK && cb <= kDiffK) {
                        settled = true;
                        W.pos[r] = 0xFFFFFFFFu;   // no verify work (k_fx_vfill skips it)
                        const uint64_t first = diff_compare(W, r, ld, ca, cb);
                        if (first != ~0ull) {
                            W.eq[r] = 0;
                            W.mis[r] = first;
                            res_out[atomicAdd(&W.counters[0], 1u)] = r;
                        }
                    }
                }
                if (!settled) {   // compare the bytes again (k_fx_vfill + k_fused_fx verify mode)
                    atomicAdd(&W.lcount[ld], (uint32_t)((n + chunk_bytes - 1) / chunk_bytes));
                    W.pos[r] = atomicAdd(&W.gcount[ld], 1u);
                    atomicAdd(&W.counters[10], 1u);
                }
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
// record r's part of the round-0 leader lookup; returns its table leader (the min local
// index of its group: the candidate of a member, r itself for a leader)
__device__ __forceinline__ uint32_t leader0_record(const DevLog& L, Work& W, uint32_t r, uint32_t small_bytes,
                                                   uint32_t* __restrict__ res_out) {
    const uint32_t i = L.order_pos[r];
    const uint32_t ld = table_leader(W, W.slot[r]);
    W.leader[r] = ld;
    const uint64_t sz = L.size[r];
    const bool same = L.size[ld] == sz && L.chan[ld] == L.chan[r];
    if (ld != r) {
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
    } else {
        const uint64_t off = L.off[r], loff = (ld != r && same) ? L.off[ld] : ~0ull;
        W.sdesc[2ull * i] = make_uint4((uint32_t)off, (uint32_t)(off >> 32), (uint32_t)loff, (uint32_t)(loff >> 32));
        W.sdesc[2ull * i + 1] = make_uint4((uint32_t)sz, r, 0, 0);
    }
    return ld;
}

__global__ void k_leader0(DevLog L, Work W, uint32_t n, uint32_t small_bytes, uint32_t* __restrict__ res_out) {
    // thread r: record r (gid order: its metadata loads and per-record writes coalesce);
    // a small record's compare descriptor lands at its position i in k_fused_small's
    // size-class order
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    bool member = false;
    if (r < n) member = leader0_record(L, W, r, small_bytes, res_out) != r;
    unsigned b = __ballot_sync(0xFFFFFFFFu, member);
    if ((threadIdx.x & 31) == 0 && b) atomicAdd(&W.counters[1], (uint32_t)__popc(b));
}

// Round-0 leader lookup with H5 + H6 folded in: each member's table leader is its label
// unless H3 finds a difference (a residual: the labels and sums are then recomputed after
// resolution), so the labels (dup_out, if given) and the per-block site histograms of
// k_label_hist are produced here, from registers the lookup already holds -- no separate
// pass over the records after H3.  Persistent 1024-thread blocks (one per SM) over the
// records in gid order; k_site_reduce sums the rows.
__global__ void __launch_bounds__(1024) k_leader0_label(DevLog L, Work W, uint32_t n, uint32_t small_bytes,
                                                        uint32_t* __restrict__ res_out, uint32_t n_sites,
                                                        int64_t* __restrict__ dup_out, uint64_t* __restrict__ part,
                                                        uint32_t* __restrict__ cpart) {
    extern __shared__ unsigned long long sben[];
    uint32_t* scnt = (uint32_t*)(sben + n_sites);
    for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
        sben[s] = 0;
        scnt[s] = 0;
    }
    __syncthreads();
    // kL0U records per thread per step, each stage's loads of all of them in flight
    // together (slot -> table leader -> the leader's metadata are three dependent
    // latencies per record)
    constexpr int kL0U = 2;
    const uint32_t stride = gridDim.x * blockDim.x;
    uint32_t members = 0;
    for (uint32_t r0 = blockIdx.x * blockDim.x; r0 < n; r0 += kL0U * stride) {   // block-uniform trip count
        uint32_t r[kL0U], ld[kL0U];
#pragma unroll
        for (int u = 0; u < kL0U; ++u) {
            r[u] = r0 + threadIdx.x + u * stride;
            ld[u] = r[u] < n ? W.slot[r[u]] : 0;
        }
#pragma unroll
        for (int u = 0; u < kL0U; ++u) ld[u] = r[u] < n ? table_leader(W, ld[u]) : r[u];
        uint64_t sz[kL0U], szl[kL0U], ch[kL0U], chl[kL0U];
#pragma unroll
        for (int u = 0; u < kL0U; ++u) {
            const bool ok = r[u] < n;
            sz[u] = ok ? L.size[r[u]] : 0;
            ch[u] = ok ? L.chan[r[u]] : 0;
            szl[u] = ok ? L.size[ld[u]] : 0;
            chl[u] = ok ? L.chan[ld[u]] : 0;
        }
#pragma unroll
        for (int u = 0; u < kL0U; ++u) {
            if (r[u] >= n) continue;
            const uint32_t rr = r[u], l = ld[u];
            W.leader[rr] = l;
            const bool member = l != rr;
            const bool same = szl[u] == sz[u] && chl[u] == ch[u];
            if (member) {
                if (!same) {
                    W.eq[rr] = 0;            // key collision across sizes / channels: not equal
                    W.mis[rr] = 0;
                    res_out[atomicAdd(&W.counters[0], 1u)] = rr;
                } else {
                    W.eq[rr] = 1;
                    W.mis[rr] = ~0ull;
                }
            }
            if (sz[u] > small_bytes) {
                uint32_t head = rr, p = 0;
                if (member && same) {
                    head = l;
                    p = 1u + atomicAdd(&W.gcount[l], 1u);
                }
                W.fhead[rr] = head;
                W.pos[rr] = p;
            } else {
                const uint32_t i = L.order_pos[rr];
                const uint64_t off = L.off[rr], loff = (member && same) ? L.off[l] : ~0ull;
                W.sdesc[2ull * i] = make_uint4((uint32_t)off, (uint32_t)(off >> 32), (uint32_t)loff, (uint32_t)(loff >> 32));
                W.sdesc[2ull * i + 1] = make_uint4((uint32_t)sz[u], rr, 0, 0);
            }
            if (dup_out) dup_out[rr] = member ? (int64_t)L.gid[l] : -1;
            if (member) {
                const uint32_t site = L.site[rr];
                atomicAdd(&sben[site], (unsigned long long)L.dur[rr]);
                atomicAdd(&scnt[site], 1u);
            }
        }
#pragma unroll
        for (int u = 0; u < kL0U; ++u) members += __popc(__ballot_sync(0xFFFFFFFFu, r[u] < n && ld[u] != r[u]));
    }
    if ((threadIdx.x & 31) == 0 && members) atomicAdd(&W.counters[1], members);
    __syncthreads();
    uint64_t* row = part + (uint64_t)blockIdx.x * n_sites;
    uint32_t* crow = cpart + (uint64_t)blockIdx.x * n_sites;
    for (uint32_t s = threadIdx.x; s < n_sites; s += blockDim.x) {
        row[s] = sben[s];
        crow[s] = scnt[s];
    }
}

// With FFM_FLAG_PREFILTER a leader whose fused group has no member has a unique
// (size, first chunk, channel): it cannot equal any other payload, so its remaining
// chunks are not read.
__device__ __forceinline__ bool prefix_unique(const Work& W, uint32_t r) {
    return W.fhead[r] == r && W.gcount[r] == 0 && W.leader[r] == r;
}

// ----------------------------------------------------------------------------
// H1 + H3 fused, pipelined (round 0, large payloads; the default).  Every byte of the
// pass is read from HBM exactly once (the prefix-chunk compares aside), with no
// reliance on L2 for the leaders' bytes:
//
//   * the pass works on pieces of <= kFxPiece bytes (a chunk, or an equal split of a
//     larger chunk); a task is (group head h, piece t) with all of the group's members:
//     stages [leader piece, member 1 piece, ..., member k-1 piece];
//   * k_fx_fill writes one self-contained 32-byte descriptor per (record, piece), laid
//     out task by task; one producer warp per CTA takes segments of kFxSeg descriptors
//     (dynamic scheduling), prefetches them a batch ahead and streams every stage into
//     a ring of kFxStages shared-memory buffers with cp.async.bulk (TMA engine, mbarrier
//     complete_tx, L2 evict_first);
//   * eight consumer warps own the piece word by word: the leader's words are hashed
//     (outside chunk 0, which the prefix pass hashed) and kept in registers for the
//     whole task, and every member's words are compared against them -- no member byte
//     is hashed.
//
// A member's NH sums follow from its leader's: NH is a plain positional sum, so over
// a chunk the member's partial equals the leader's plus, for each differing word,
// nh(member word) - nh(leader word) (mod 2^64).  Those deltas (zero for a duplicate)
// are added into the member's chunk slot; k_hash_combine forms
// acc[m] = acc_prefix[m] + sum_{c>=1} (part[h][c] + delta[m][c]).  The first
// mismatching word is the exact minimum (every word is compared).
// ----------------------------------------------------------------------------
#ifndef FFM_FX_PIECE
#define FFM_FX_PIECE 32768
#endif
#ifndef FFM_FX_STAGES
#define FFM_FX_STAGES 3
#endif
#ifndef FFM_FX_CTAS
#define FFM_FX_CTAS 2
#endif
#ifndef FFM_FX_MINB          // __launch_bounds__ min blocks (register budget)
#define FFM_FX_MINB FFM_FX_CTAS
#endif
constexpr int kFxConsumers = 8;                       // consumer warps
constexpr int kFxThreads = 32 * (kFxConsumers + 1);   // + one producer warp
constexpr uint32_t kFxPiece = FFM_FX_PIECE;           // bytes per stage (max)
constexpr int kFxWords = kFxPiece / 16 / (32 * kFxConsumers);   // 16-B words per consumer thread per stage
constexpr int kFxStages = FFM_FX_STAGES;
constexpr uint32_t kFxSeg = 64;                       // descriptors per scheduler grab

enum : uint32_t { kFxLeader = 1u, kFxHash = 2u, kFxDelta = 4u, kFxReduce = 8u, kFxSkip = 16u, kFxDone = 32u };

// one stage of the pipelined pass (descriptor in HBM, meta in shared memory)
struct FxDesc {
    uint64_t src;     // arena offset of the piece
    uint32_t rec;     // record
    uint32_t lenf;    // piece bytes (bits 0-23) | kFx* flags << 24
    uint32_t w0;      // first 16-B word of the piece (record-relative)
    uint32_t slot;    // the record's hpart slot of the piece's chunk
    uint32_t k;       // on a task's first descriptor: the task's length (entries); else 0
    uint32_t pad;
};

constexpr size_t kFxSmem = (size_t)kFxStages * kFxPiece + (size_t)kFxStages * sizeof(FxDesc) +
                           2 * kFxStages * sizeof(uint64_t) + 2 * kFxConsumers * 2 * sizeof(uint64_t);

// pieces of a record of n bytes: chunks of chunk_bytes, each split into ppc pieces of ps
struct FxSplit {
    uint32_t chunk, ppc, ps;
};
__host__ __device__ __forceinline__ FxSplit fx_split(uint32_t chunk_bytes) {
    FxSplit f;
    f.chunk = chunk_bytes;
    f.ppc = (chunk_bytes + kFxPiece - 1) / kFxPiece;
    f.ps = ((chunk_bytes + f.ppc - 1) / f.ppc + 1023u) & ~1023u;
    return f;
}
__host__ __device__ __forceinline__ uint32_t fx_pieces(const FxSplit& f, uint64_t n) {
    const uint64_t full = n / f.chunk, rem = n % f.chunk;
    return (uint32_t)(full * f.ppc + (rem + f.ps - 1) / f.ps);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "FFM_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra FFM_WAIT_%=;\n}" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            dst),
        "l"(src), "r"(bytes), "r"(bar), "l"(pol)
        : "memory");
}

// A consumer releases a stage with one arrive per LANE on the stage's empty barrier, after
// that lane's own last read of it: each read is ordered before the producer's next bulk
// write by the reading thread's own release (compute-sanitizer racecheck follows this
// chain; it does not follow __syncwarp + one arrive per warp, which it flagged as 4.9 M
// hazards in round 1 -- profiles/sanitizer/README.md).  Measured no slower (r02i).
constexpr uint32_t kFxEmptyArrivals = 32u * kFxConsumers;
__device__ __forceinline__ void fx_release(uint32_t bar) { mbar_arrive(bar); }

// keep the first `valid` bytes of a 16-B word, zero the rest
__device__ __forceinline__ void mask_word(uint4& w, int32_t valid) {
    if (valid >= 16) return;
    uint32_t* v = reinterpret_cast<uint32_t*>(&w);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int32_t vb = valid - 4 * i;
        v[i] &= vb >= 4 ? 0xFFFFFFFFu : (vb <= 0 ? 0u : ((1u << (8 * vb)) - 1u));
    }
}

// NH keys of word q: position q mod 16 (fixed per consumer thread), stripe q div 16.
__device__ __forceinline__ void word_keys(uint32_t* k, const uint32_t* ka, uint32_t s) {
#pragma unroll
    for (int j = 0; j < 6; ++j) k[j] = ka[j] + s * kDA(j);
}

// Task layout.  Head h's group (k = members + 1 records) becomes, per piece t, S =
// ceil((k - 1) / (kFxMaxK - 1)) sub-tasks (at least 1) of <= kFxMaxK entries: a copy of
// the head's descriptor, then up to kFxMaxK - 1 members.  Long groups thus spread over
// CTAs (a leader piece is re-staged once per kFxMaxK - 1 members, hashed only in
// sub-task 0).  Entries of a head: pieces x (k - 1 + S), contiguous from lstart[h].
constexpr uint32_t kFxMaxK = 64;

__device__ __forceinline__ uint32_t fx_subtasks(uint32_t k) {
    return k <= 1 ? 1u : (k - 1 + kFxMaxK - 2) / (kFxMaxK - 1);
}

// verify = 0: round-0 fused groups (every large head, singletons included);
// verify = 1: verify groups of k_leader (leaders with >= 1 large member).
__global__ void k_fx_count(DevLog L, Work W, uint32_t small_bytes, uint32_t chunk_bytes, int verify) {
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r > L.n) return;
    uint32_t c = 0;
    if (r < L.n && L.size[r] > small_bytes && (verify ? W.gcount[r] > 0 : W.fhead[r] == r)) {
        const uint32_t k = W.gcount[r] + 1;
        c = fx_pieces(fx_split(chunk_bytes), L.size[r]) * (k - 1 + fx_subtasks(k));
    }
    W.lcount[r] = c;
}

// Verify-only descriptors (two-pass round 0 and resolve rounds): each large member of
// `list` whose leader has its size and channel, at position pos + 1 of its leader's
// group; the member at pos 0 also writes the leader's copies.  No hashing: the
// digests are final.
__global__ void k_fx_vfill(DevLog L, Work W, const uint32_t* __restrict__ list, uint32_t n_list,
                           uint32_t small_bytes, uint32_t chunk_bytes, FxDesc* __restrict__ items) {
    if (blockIdx.x == 0 && threadIdx.x == 0) W.counters[8] = 0;   // segment scheduler
    const FxSplit f = fx_split(chunk_bytes);
    FFM_WARP_EACH(list ? n_list : L.n_large, list ? list[w_] : L.large_order[w_],
                  (W.leader[rec] != rec && L.size[rec] > small_bytes && L.size[W.leader[rec]] == L.size[rec] &&
                   L.chan[W.leader[rec]] == L.chan[rec] && W.pos[rec] != 0xFFFFFFFFu), {
        const uint32_t ld = W.leader[rec];
        const uint32_t k = W.gcount[ld] + 1, p = W.pos[rec] + 1, base = W.lstart[ld];
        const uint32_t S = fx_subtasks(k), K = k - 1 + S;
        const uint64_t n = L.size[rec];
        const uint32_t np = fx_pieces(f, n);
        for (uint32_t t = lane; t < np; t += 32) {
            const uint32_t c = t / f.ppc, j = t - c * f.ppc;
            const uint64_t st = (uint64_t)c * f.chunk + (uint64_t)j * f.ps;
            const uint64_t en = min(min(st + f.ps, (uint64_t)(c + 1) * f.chunk), n);
            const uint64_t pb = base + (uint64_t)t * K;
            FxDesc d;
            d.w0 = (uint32_t)(st >> 4);
            d.slot = 0;
            d.pad = 0;
            d.lenf = (uint32_t)(en - st);
            const uint32_t q = (p - 1) / (kFxMaxK - 1), i = (p - 1) - q * (kFxMaxK - 1) + 1;
            d.src = L.off[rec] + st;
            d.rec = rec;
            d.k = 0;
            items[pb + (uint64_t)q * kFxMaxK + i] = d;
            if (p == 1) {
                d.src = L.off[ld] + st;
                d.rec = ld;
                d.lenf |= kFxLeader << 24;
                for (uint32_t qq = 0; qq < S; ++qq) {
                    d.k = qq + 1 < S ? kFxMaxK : k - qq * (kFxMaxK - 1);
                    items[pb + (uint64_t)qq * kFxMaxK] = d;
                }
            }
        }
    })
}

// One descriptor per (record, piece, sub-task copy); also zeroes the chunk slots the
// pass accumulates into.  The first prefix_bytes of every record were hashed by the
// prefix pass: a group's pieces still cover them (the members' compares), a
// singleton's first piece starts after them.
__global__ void k_fx_fill(DevLog L, Work W, uint32_t chunk_bytes, uint32_t prefix_bytes, int prefilter,
                          FxDesc* __restrict__ items) {
    if (blockIdx.x == 0 && threadIdx.x == 0) W.counters[8] = 0;   // segment scheduler
    const FxSplit f = fx_split(chunk_bytes);
    FFM_WARP_EACH(L.n_large, L.large_order[w_], true, {
        const uint32_t h = W.fhead[rec];
        const uint32_t k = W.gcount[h] + 1, p = W.pos[rec], base = W.lstart[h];
        const uint32_t S = fx_subtasks(k), K = k - 1 + S;   // sub-tasks, entries per piece
        const uint64_t n = L.size[rec], off = L.off[rec];
        const uint32_t np = fx_pieces(f, n), hs = W.hstart[rec];
        const bool skip_all = prefilter && prefix_unique(W, rec);
        const uint32_t last0 = min(k - 1, kFxMaxK - 1);      // position ending sub-task 0
        if (lane == 0) W.dcnt[rec] = 0;                       // difference list vs the head (k_fused_fx)
        for (uint32_t t = lane; t < np; t += 32) {
            const uint32_t c = t / f.ppc, j = t - c * f.ppc;
            uint64_t st = (uint64_t)c * f.chunk + (uint64_t)j * f.ps;
            const uint64_t en = min(min(st + f.ps, (uint64_t)(c + 1) * f.chunk), n);
            const bool hashes = en > prefix_bytes;             // has words beyond the prefix
            bool skip = skip_all;
            if (k == 1 && st < prefix_bytes) {                 // singleton: skip the prefix
                if (!hashes) skip = true;
                else st = prefix_bytes;
            }
            FxDesc d;
            d.src = off + st;
            d.rec = rec;
            d.w0 = (uint32_t)(st >> 4);
            d.slot = hs + c;
            d.pad = 0;
            const uint64_t pb = base + (uint64_t)t * K;
            if (p == 0) {
                for (uint32_t q = 0; q < S; ++q) {
                    uint32_t fl = kFxLeader;
                    if (q == 0 && hashes) fl |= kFxHash;
                    if (skip) fl |= kFxSkip;
                    if (q == 0 && last0 == 0 && hashes) fl |= kFxReduce;
                    d.lenf = (uint32_t)(en - st) | (fl << 24);
                    d.k = q + 1 < S ? kFxMaxK : k - q * (kFxMaxK - 1);
                    items[pb + (uint64_t)q * kFxMaxK] = d;
                }
            } else {
                const uint32_t q = (p - 1) / (kFxMaxK - 1), i = (p - 1) - q * (kFxMaxK - 1) + 1;
                uint32_t fl = hashes ? kFxDelta : 0u;
                if (p == last0 && hashes) fl |= kFxReduce;
                d.lenf = (uint32_t)(en - st) | (fl << 24);
                d.k = 0;
                items[pb + (uint64_t)q * kFxMaxK + i] = d;
            }
            if (j == 0) {
                W.hpart[2ull * (hs + c)] = 0;
                W.hpart[2ull * (hs + c) + 1] = 0;
            }
        }
    })
}

template <bool kVerify>
__global__ void __launch_bounds__(kFxThreads, FFM_FX_MINB) k_fused_fx(DevLog L, Work W,
                                                                      const FxDesc* __restrict__ items,
                                                                      const uint32_t* __restrict__ n_items_ptr,
                                                                      uint32_t pw, uint32_t* res_out) {
    // pw: words below it were hashed by the prefix pass (not hashed, no deltas here)
    extern __shared__ __align__(128) uint8_t fx_smem[];
    uint8_t* bufs = fx_smem;
    FxDesc* meta = reinterpret_cast<FxDesc*>(fx_smem + (size_t)kFxStages * kFxPiece);
    uint64_t* full = reinterpret_cast<uint64_t*>(meta + kFxStages);
    uint64_t* empty = full + kFxStages;
    uint64_t* red = empty + kFxStages;   // [2][kFxConsumers][2]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kFxStages; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), kFxEmptyArrivals);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();

    if (warp == kFxConsumers) {
        // ------------------------------------------------------------ producer
        uint64_t pol;
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
        const uint32_t E = *n_items_ptr;
        int stage = 0;
        uint32_t phase = 0;
        const uint4* raw = reinterpret_cast<const uint4*>(items);
        // verify-only mode (resolve rounds, two-pass): a member's piece that starts after
        // its already-recorded first mismatch cannot lower it -- it is not streamed (the
        // member's mismatch word is read a batch ahead; a stale value only skips less)
        constexpr bool vmode = kVerify;
        const volatile unsigned long long* vmis = reinterpret_cast<const volatile unsigned long long*>(W.mis);
        // lane-parallel batch of 32 descriptors [bb, bb + 32), the next one prefetched
        auto load = [&](uint32_t bb, uint4& a, uint4& b, uint64_t& mi) {
            const uint32_t i = bb + lane;
            mi = ~0ull;
            if (i < E) {
                a = raw[2ull * i];
                b = raw[2ull * i + 1];
                if (vmode && !((a.w >> 24) & kFxLeader)) mi = vmis[a.z];
            } else {
                a = make_uint4(0, 0, 0, 0);
                b = make_uint4(0, 0, 0, 0);
            }
        };
        uint32_t seg = 0;
        if (lane == 0) seg = atomicAdd(&W.counters[8], 1u);
        seg = __shfl_sync(0xFFFFFFFFu, seg, 0);
        uint32_t lo = seg * kFxSeg;
        uint32_t bb = lo;
        uint4 ca, cb, na, nb;
        uint64_t cm, nm;
        load(bb, ca, cb, cm);
        load(bb + 32, na, nb, nm);
        uint32_t rem = 0;          // entries left in the current task
        bool started = false;      // a task starting in this segment has been seen
        while (lo < E) {
            const uint32_t hi = min(E, lo + kFxSeg);
            // walk descriptors from bb; stop after the last task that starts before hi
            bool seg_done = false;
            while (!seg_done) {
#pragma unroll 1
                for (int j = 0; j < 32; ++j) {
                    const uint32_t e = bb + j;
                    const uint32_t k = __shfl_sync(0xFFFFFFFFu, cb.z, j);
                    if (rem == 0) {
                        if (e >= hi || e >= E) {
                            seg_done = true;
                            break;
                        }
                        if (k == 0) {   // a member of a task that started in an earlier segment
                            if (started) {
                                seg_done = true;   // cannot happen: tasks are contiguous
                                break;
                            }
                            continue;
                        }
                        rem = k;
                        started = true;
                    }
                    --rem;
                    const uint32_t s_lo = __shfl_sync(0xFFFFFFFFu, ca.x, j);
                    const uint32_t s_hi = __shfl_sync(0xFFFFFFFFu, ca.y, j);
                    const uint32_t rec = __shfl_sync(0xFFFFFFFFu, ca.z, j);
                    const uint32_t lenf = __shfl_sync(0xFFFFFFFFu, ca.w, j);
                    const uint32_t w0 = __shfl_sync(0xFFFFFFFFu, cb.x, j);
                    const uint32_t slot = __shfl_sync(0xFFFFFFFFu, cb.y, j);
                    if ((lenf >> 24) & kFxSkip) continue;
                    if (vmode && __shfl_sync(0xFFFFFFFFu, cm, j) < (uint64_t)w0) continue;
                    if (lane == 0) {
                        mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                        FxDesc& m = meta[stage];
                        m.rec = rec;
                        m.lenf = lenf;
                        m.w0 = w0;
                        m.slot = slot;
                        const uint32_t len = lenf & 0xFFFFFFu;
                        const uint32_t bytes = (len + 15u) & ~15u;
                        const uint32_t fb = smem_u32(&full[stage]);
                        mbar_arrive_tx(fb, bytes);
                        bulk_g2s(smem_u32(bufs + (size_t)stage * kFxPiece),
                                 L.arena + (((uint64_t)s_hi << 32) | s_lo), bytes, fb, pol);
                    }
                    if (++stage == kFxStages) {
                        stage = 0;
                        phase ^= 1;
                    }
                }
                if (seg_done) break;
                bb += 32;
                ca = na;
                cb = nb;
                cm = nm;
                load(bb + 32, na, nb, nm);
            }
            // next segment
            if (lane == 0) seg = atomicAdd(&W.counters[8], 1u);
            seg = __shfl_sync(0xFFFFFFFFu, seg, 0);
            lo = seg * kFxSeg;
            rem = 0;
            started = false;
            if (lo >= E) break;
            bb = lo;
            load(bb, ca, cb, cm);
            load(bb + 32, na, nb, nm);
        }
        if (lane == 0) {
            mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
            meta[stage].lenf = kFxDone << 24;
            mbar_arrive(smem_u32(&full[stage]));
        }
        return;
    }

    // ---------------------------------------------------------------- consumers
    const int t = threadIdx.x;                 // 0 .. 32 * kFxConsumers - 1
    const int g = t & 15;                      // NH position of every word this thread owns
    uint32_t ka[6];
#pragma unroll
    for (int j = 0; j < 6; ++j) ka[j] = c_nh.ka[g][j];
    uint4 x[kFxWords];                         // the current piece of the leader
    uint64_t A = 0, B = 0;
    uint32_t lslot = 0;
    int stage = 0, rbuf = 0;
    uint32_t phase = 0;
    constexpr uint32_t kStride = 32 * kFxConsumers;   // words between a thread's words
    for (;;) {
        mbar_wait(smem_u32(&full[stage]), phase);
        const uint32_t lenf = meta[stage].lenf;
        const uint32_t flags = lenf >> 24;
        if (flags & kFxDone) break;
        const uint32_t w0 = meta[stage].w0, slot = meta[stage].slot, rec = meta[stage].rec;
        const int32_t len = (int32_t)(lenf & 0xFFFFFFu);
        const uint8_t* buf = bufs + (size_t)stage * kFxPiece;
        if (flags & kFxLeader) {
#pragma unroll
            for (int u = 0; u < kFxWords; ++u) {
                const int32_t vb = len - 16 * (int32_t)(t + kStride * u);
                x[u] = vb > 0 ? *reinterpret_cast<const uint4*>(buf + 16 * (t + kStride * u)) : make_uint4(0, 0, 0, 0);
            }
            fx_release(smem_u32(&empty[stage]));
#pragma unroll
            for (int u = 0; u < kFxWords; ++u) mask_word(x[u], len - 16 * (int32_t)(t + kStride * u));
            if (flags & kFxHash) {
                lslot = slot;
                uint32_t k[6];
                word_keys(k, ka, (w0 + t) >> 4);
#pragma unroll
                for (int u = 0; u < kFxWords; ++u) {
                    if (len > 16 * (int32_t)(t + kStride * u) && w0 + t + kStride * u >= pw)
                        nh_word(x[u].x, x[u].y, x[u].z, x[u].w, k, A, B);
#pragma unroll
                    for (int j = 0; j < 6; ++j) k[j] += kDA(j) * (kStride / 16);
                }
            }
        } else {
            uint4 y[kFxWords];
#pragma unroll
            for (int u = 0; u < kFxWords; ++u) {
                const int32_t vb = len - 16 * (int32_t)(t + kStride * u);
                y[u] = vb > 0 ? *reinterpret_cast<const uint4*>(buf + 16 * (t + kStride * u)) : make_uint4(0, 0, 0, 0);
            }
            fx_release(smem_u32(&empty[stage]));
            uint32_t dmask = 0;
#pragma unroll
            for (int u = 0; u < kFxWords; ++u) {
                mask_word(y[u], len - 16 * (int32_t)(t + kStride * u));
                if ((y[u].x ^ x[u].x) | (y[u].y ^ x[u].y) | (y[u].z ^ x[u].z) | (y[u].w ^ x[u].w)) dmask |= 1u << u;
            }
            if (__any_sync(0xFFFFFFFFu, dmask != 0)) {
                // rare: a near-duplicate or a collision -- first mismatching word and NH deltas
                uint64_t found = dmask ? (uint64_t)(w0 + t + kStride * (__ffs(dmask) - 1)) : ~0ull;
                if (!kVerify) {
                    // the member's difference list against its head (every word of a group
                    // member is compared in round 0): its count, and the (word, value) pairs
                    // while they fit -- one atomic per warp, none once the list overflowed
                    uint32_t cur = 0;
                    if (lane == 0) cur = *reinterpret_cast<const volatile uint32_t*>(&W.dcnt[rec]);
                    cur = __shfl_sync(0xFFFFFFFFu, cur, 0);
                    if (cur <= kDiffK) {
                        const uint32_t nd = __popc(dmask);
                        uint32_t incl = nd;
#pragma unroll
                        for (int o = 1; o < 32; o <<= 1) {
                            const uint32_t v = __shfl_up_sync(0xFFFFFFFFu, incl, o);
                            if (lane >= o) incl += v;
                        }
                        uint32_t base = 0;
                        if (lane == 31) base = atomicAdd(&W.dcnt[rec], incl);
                        base = __shfl_sync(0xFFFFFFFFu, base, 31);
                        uint32_t sl = base + incl - nd;
#pragma unroll
                        for (int u = 0; u < kFxWords; ++u) {
                            if (!(dmask & (1u << u))) continue;
                            if (sl < kDiffK) {
                                W.dq[(uint64_t)rec * kDiffK + sl] = w0 + t + kStride * u;
                                W.dv[(uint64_t)rec * kDiffK + sl] = y[u];
                            }
                            ++sl;
                        }
                    }
                }
                uint64_t dA = 0, dB = 0;
                if ((flags & kFxDelta) && dmask) {
                    uint64_t xA = 0, xB = 0;
#pragma unroll
                    for (int u = 0; u < kFxWords; ++u) {
                        if ((dmask & (1u << u)) && w0 + t + kStride * u >= pw) {
                            uint32_t k[6];
                            word_keys(k, ka, (w0 + t + kStride * u) >> 4);
                            nh_word(y[u].x, y[u].y, y[u].z, y[u].w, k, dA, dB);
                            nh_word(x[u].x, x[u].y, x[u].z, x[u].w, k, xA, xB);
                        }
                    }
                    dA -= xA;
                    dB -= xB;
                }
#pragma unroll
                for (int o = 16; o; o >>= 1) {
                    const uint64_t of = __shfl_xor_sync(0xFFFFFFFFu, found, o);
                    found = of < found ? of : found;
                    dA += __shfl_xor_sync(0xFFFFFFFFu, dA, o);
                    dB += __shfl_xor_sync(0xFFFFFFFFu, dB, o);
                }
                if (lane == 0) {
                    report_mismatch(W, rec, found, res_out, true);
                    if ((flags & kFxDelta) && (dA | dB)) {
                        atomicAdd((unsigned long long*)&W.hpart[2ull * slot], (unsigned long long)dA);
                        atomicAdd((unsigned long long*)&W.hpart[2ull * slot + 1], (unsigned long long)dB);
                    }
                }
            }
        }
        if (flags & kFxReduce) {
            // the leader's piece partial: CTA reduction over the consumer threads, added
            // into the chunk slot (a chunk may span several pieces)
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
                B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
            }
            if (lane == 0) {
                red[(rbuf * kFxConsumers + warp) * 2] = A;
                red[(rbuf * kFxConsumers + warp) * 2 + 1] = B;
            }
            asm volatile("bar.sync 1, %0;" ::"n"(32 * kFxConsumers) : "memory");
            if (t == 0) {
                uint64_t sA = 0, sB = 0;
#pragma unroll
                for (int w = 0; w < kFxConsumers; ++w) {
                    sA += red[(rbuf * kFxConsumers + w) * 2];
                    sB += red[(rbuf * kFxConsumers + w) * 2 + 1];
                }
                atomicAdd((unsigned long long*)&W.hpart[2ull * lslot], (unsigned long long)sA);
                atomicAdd((unsigned long long*)&W.hpart[2ull * lslot + 1], (unsigned long long)sB);
            }
            rbuf ^= 1;
            A = B = 0;
        }
        if (++stage == kFxStages) {
            stage = 0;
            phase ^= 1;
        }
    }
}

// Combine the chunk partial sums of large records (NH is a plain sum, so the record's
// accumulators are the sums of its parts' -- deterministic) and finish their digests.
// Two-pass: the chunk slots of k_hash_large.  After the pipelined fused pass (fx): the
// prefix partial + the record's chunk slots, and for a member also its head's chunk
// slots (its own slots hold NH deltas).  Also totals the bytes hashed beyond the
// prefixes (roofline stats).
__global__ void __launch_bounds__(256) k_hash_combine(DevLog L, Work W, uint32_t chunk_bytes, uint32_t prefix_bytes,
                                                      int prefilter, int fx) {
    unsigned long long rest = 0;
    // (an identity order -- online windows -- lists small records too: no chunk slots)
    FFM_WARP_EACH(L.n_large, L.large_order[w_], (W.hstart[rec + 1] != W.hstart[rec]), {
        const uint32_t s0 = W.hstart[rec];
        const bool skip = fx && prefilter && prefix_unique(W, rec);
        const uint32_t e0 = skip ? s0 : W.hstart[rec + 1];
        const uint32_t h = fx ? W.fhead[rec] : rec;
        const int64_t dh = (int64_t)W.hstart[h] - (int64_t)s0;   // head slot of the same chunk
        uint64_t A0 = 0, B0 = 0, A1 = 0, B1 = 0;
        uint32_t it = s0 + lane;
        for (; it + 32 < e0; it += 64) {
            A0 += W.hpart[2ull * it];
            B0 += W.hpart[2ull * it + 1];
            A1 += W.hpart[2ull * (it + 32)];
            B1 += W.hpart[2ull * (it + 32) + 1];
            if (h != rec) {   // a member: head's partials + own deltas
                A0 += W.hpart[2ull * (it + dh)];
                B0 += W.hpart[2ull * (it + dh) + 1];
                A1 += W.hpart[2ull * (it + 32 + dh)];
                B1 += W.hpart[2ull * (it + 32 + dh) + 1];
            }
        }
        if (it < e0) {
            A0 += W.hpart[2ull * it];
            B0 += W.hpart[2ull * it + 1];
            if (h != rec) {
                A0 += W.hpart[2ull * (it + dh)];
                B0 += W.hpart[2ull * (it + dh) + 1];
            }
        }
        uint64_t A = A0 + A1, B = B0 + B1;
        for (int o = 16; o; o >>= 1) {
            A += __shfl_xor_sync(0xFFFFFFFFu, A, o);
            B += __shfl_xor_sync(0xFFFFFFFFu, B, o);
        }
        const uint64_t n = L.size[rec];
        if (fx) {   // + the prefix pass's partial (accA/accB hold it until here)
            A += W.accA[rec];
            B += W.accB[rec];
        }
        __syncwarp();
        if (lane == 0) {
            W.accA[rec] = A;
            W.accB[rec] = B;
            W.digest[rec] = finalize_digest(A, B, n);
            if (fx && !skip && n > prefix_bytes) rest += n - prefix_bytes;
        }
    })
    if (rest) atomicAdd((unsigned long long*)(W.counters + 4), rest);
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

// H1 + H3 fused for small payloads (round 0): one 8-lane group per record, records in
// size-class order.  A record that leads its prefix group is hashed (its full digest:
// the cross-shard / online merges and any collision resolution key on it); a member is
// only byte-compared with its group's leader -- an equal member has its leader's bytes,
// hence its digest, so hashing it would be wasted issue slots (the pass is issue-bound);
// a member that differs becomes a residual and is hashed before the resolve rounds
// (k_hash_small over the residual list).  Re-uploads of one content share their leader,
// so its bytes are L2-hot; the member's own bytes are read from HBM once.
// Per-thread cp.async pipeline: every lane is its own producer.  A lane's work is the
// sequence of steps (record, 16*U 16-byte words of it) of its octet; it keeps S-1 steps
// of its own and its leader's words in flight in shared memory (cp.async, no registers
// held) while it hashes and compares the oldest, across record boundaries.  Default
// U=2, S=2, 128 threads: 37 KB per CTA, 6 CTAs (24 warps) per SM -- occupancy beat depth
// (S=3 / S=4 / U=1 / U=3 measured slower, profiles/r01e/README.md).
// Lane g takes words g, g+8 of each 256-byte stripe (one warp instruction = 128
// contiguous bytes per octet); NH is a positional sum, so the digest is unchanged.
// Each lane reads back only what it copied itself: cp.async.wait_group is the only ordering.
#ifndef FFM_SA_U
#define FFM_SA_U 2
#endif
#ifndef FFM_SA_S
#define FFM_SA_S 2
#endif
#ifndef FFM_SA_T
#define FFM_SA_T 128
#endif
constexpr int kSaU = FFM_SA_U, kSaS = FFM_SA_S, kSaT = FFM_SA_T, kSaJ = 2 * kSaU;   // words per lane per step
constexpr int kSaSmem = kSaS * kSaT * 16 * (2 * kSaJ);                               // 16-B data slots (own, leader)
static_assert(kSaS == 2, "k_fused_small carries the in-flight step's meta in registers (one step ahead)");
constexpr uint32_t kSaEnd = 1u << 31, kSaFirst = 1u << 30, kSaLast = 1u << 29, kSaCmp = 1u << 28;

__device__ __forceinline__ void cp16(uint32_t dst, const uint8_t* src, uint64_t pol) {
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "l"(pol)
                 : "memory");
}

__device__ __forceinline__ void lds16(uint32_t a, uint32_t* v) {
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(a)
                 : "memory");
}

// zero the bytes of 16-byte word w at or beyond n
__device__ __forceinline__ void mask_word(uint32_t* v, uint32_t n, uint32_t w) {
    const int32_t valid = (int32_t)n - (int32_t)(16 * w);
    if (valid >= 16) return;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int32_t vb = valid - 4 * i;
        v[i] &= vb >= 4 ? 0xFFFFFFFFu : (vb <= 0 ? 0u : ((1u << (8 * vb)) - 1u));
    }
}

__global__ void __launch_bounds__(kSaT) k_fused_small(DevLog L, Work W, uint32_t* res_out) {
    extern __shared__ __align__(16) uint8_t sa_smem[];
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3;
    const uint32_t noct = (gridDim.x * blockDim.x) >> 3;
    const uint32_t sbase = smem_u32(sa_smem) + threadIdx.x * 16;
    // slot of word j of stage s (part 0 own, 1 leader); lanes interleaved so a warp's
    // 16-B accesses to one slot are 512 contiguous bytes (conflict-free)
    auto slot = [&](int s, int j, int part) { return sbase + (uint32_t)(((s * kSaJ + j) * 2 + part) * kSaT * 16); };
    uint64_t pol_own, pol_keep;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_own));
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_keep));

    // ---- producer state: current record (position fi, next word fw0).  The descriptor
    // of the octet's next record is held spread over its 8 lanes (lane g: 32-bit word g
    // of the 32-byte descriptor, one coalesced load per octet), loaded a whole record
    // ahead and gathered by shuffles when the record changes -- the load's destination is
    // read only then, so no step waits on it.
    const uint32_t* sd32 = reinterpret_cast<const uint32_t*>(W.sdesc);
    // producer state of the octet's current record: next word fw0 of fnw, this lane's
    // next source addresses (own, and the leader's for a compared record), bytes, record
    uint32_t fi = oct, fw0 = 0, fnw = 0, fn = 0, fr = 0, nd = 0;
    bool fcmp = false;
    const uint8_t* fsrc = nullptr;
    const uint8_t* flsrc = nullptr;
    auto start_record = [&](uint64_t off, uint64_t loff, uint32_t n, uint32_t rec) {
        fw0 = 0;
        fn = n;
        fr = rec;
        fnw = (n + 15) >> 4;
        fcmp = loff != ~0ull;
        fsrc = L.arena + off + 16 * g;
        flsrc = L.arena + (fcmp ? loff : off) + 16 * g;
    };
    if (fi < L.n_small) {
        const uint4 a = W.sdesc[2ull * fi], b = W.sdesc[2ull * fi + 1];
        start_record((uint64_t)a.y << 32 | a.x, (uint64_t)a.w << 32 | a.z, b.x, b.y);
        if (fi + noct < L.n_small) nd = sd32[8ull * (fi + noct) + g];
    }
    const int obase = threadIdx.x & 24;
    // meta of the step a fetch issued: (bytes, record, word | flags), consumed one iteration later
    uint32_t mn = 0, mr = 0, meta_z = kSaEnd;
    auto fetch = [&](int s) {
        meta_z = kSaEnd;
        mn = 0;
        mr = 0;
        if (fi < L.n_small) {
            // word j of the step is 128 * j bytes further (immediate offsets); shared-memory
            // slot j of part p is (2 j + p) * kSaT * 16 further
            const uint32_t s0 = slot(s, 0, 0);
            if (fw0 + 8 * kSaJ <= fnw) {   // every lane's words exist
#pragma unroll
                for (int j = 0; j < kSaJ; ++j) cp16(s0 + (uint32_t)(2 * j * kSaT * 16), fsrc + 128 * j, pol_own);
                if (fcmp) {
#pragma unroll
                    for (int j = 0; j < kSaJ; ++j)
                        cp16(s0 + (uint32_t)((2 * j + 1) * kSaT * 16), flsrc + 128 * j, pol_keep);
                }
            } else {
#pragma unroll
                for (int j = 0; j < kSaJ; ++j) {
                    if (fw0 + 8 * j + g < fnw) {
                        cp16(s0 + (uint32_t)(2 * j * kSaT * 16), fsrc + 128 * j, pol_own);
                        if (fcmp) cp16(s0 + (uint32_t)((2 * j + 1) * kSaT * 16), flsrc + 128 * j, pol_keep);
                    }
                }
            }
            meta_z = fw0 | (fw0 == 0 ? kSaFirst : 0u) | (fcmp ? kSaCmp : 0u);
            mn = fn;
            mr = fr;
            fw0 += 8 * kSaJ;
            fsrc += 128 * kSaJ;
            flsrc += 128 * kSaJ;
            if (fw0 >= fnw) meta_z |= kSaLast;
        }
        // last step of the octet's record: move to the next one (shuffles executed by the
        // whole warp; an octet that is not changing ignores them)
        const bool change = (meta_z & (kSaLast | kSaEnd)) == kSaLast;
        if (__any_sync(0xFFFFFFFFu, change)) {
            const uint32_t d0 = __shfl_sync(0xFFFFFFFFu, nd, obase + 0), d1 = __shfl_sync(0xFFFFFFFFu, nd, obase + 1);
            const uint32_t d2 = __shfl_sync(0xFFFFFFFFu, nd, obase + 2), d3 = __shfl_sync(0xFFFFFFFFu, nd, obase + 3);
            const uint32_t d4 = __shfl_sync(0xFFFFFFFFu, nd, obase + 4), d5 = __shfl_sync(0xFFFFFFFFu, nd, obase + 5);
            if (change) {
                fi += noct;
                start_record((uint64_t)d1 << 32 | d0, (uint64_t)d3 << 32 | d2, d4, d5);
                if (fi + noct < L.n_small) nd = sd32[8ull * (fi + noct) + g];
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
#pragma unroll 1
    for (int s = 0; s < kSaS - 1; ++s) fetch(s);

    // ---- consumer state
    LaneKeys K;   // k[0]: stripe position g, k[1]: position g + 8
    // stripe-0 keys of the 16 positions in shared memory (6 keys padded to 8 per position):
    // a record start reloads a lane's 12 keys with 4 conflict-free 16-byte loads (from the
    // constant bank the 8 positions of a warp were 8 serialised accesses per key)
    __shared__ uint4 s_ka[16][2];
    if (threadIdx.x < 32) {
        const int q = threadIdx.x >> 1, h = threadIdx.x & 1;
        s_ka[q][h] = h ? make_uint4(c_nh.ka[q][4], c_nh.ka[q][5], 0u, 0u)
                       : make_uint4(c_nh.ka[q][0], c_nh.ka[q][1], c_nh.ka[q][2], c_nh.ka[q][3]);
    }
    __syncthreads();
    uint64_t A = 0, B = 0, A2 = 0, B2 = 0;
    uint32_t found = ~0u;   // first differing 16-byte word of a compared record (lane's own)
    // The warp stays converged across the loop (an octet whose records are done idles
    // until all four are), so the octet reductions at record ends use full-mask shuffles
    // (xor 4 / 2 / 1 stay inside an octet) executed warp-uniformly -- no per-octet masks.
    // one iteration consuming stage sc and refilling stage sf; unrolled over the two
    // stages so every shared-memory slot address is a compile-time offset
    auto iteration = [&](const int sc, const int sf) -> bool {
        // refill the stage consumed last iteration (its values were used, so read), then
        // wait for the oldest: S-1 steps stay in flight while this one is hashed
        const uint32_t n = mn, r = mr, z = meta_z;   // the step fetched last iteration
        fetch(sf);
        asm volatile("cp.async.wait_group %0;" ::"n"(kSaS - 1) : "memory");
        const bool done = (z & kSaEnd) != 0;
        if (__all_sync(0xFFFFFFFFu, done)) return false;
        if (!done) {
            if (z & kSaFirst) {
                A = B = A2 = B2 = 0;
                found = ~0u;
                const uint4 a0 = s_ka[g][0], a1 = s_ka[g][1], b0 = s_ka[g + 8][0], b1 = s_ka[g + 8][1];
                K.k[0][0] = a0.x, K.k[0][1] = a0.y, K.k[0][2] = a0.z, K.k[0][3] = a0.w, K.k[0][4] = a1.x, K.k[0][5] = a1.y;
                K.k[1][0] = b0.x, K.k[1][1] = b0.y, K.k[1][2] = b0.z, K.k[1][3] = b0.w, K.k[1][4] = b1.x, K.k[1][5] = b1.y;
            }
            const uint32_t w0 = z & 0x0FFFFFFFu, nw = (n + 15) >> 4;
            const bool full = 16 * (w0 + 8 * kSaJ) <= n;   // every word of the step whole
            if (z & kSaCmp) {
                // member: compare only, until its first differing word
                if (found == ~0u) {
                    uint32_t d = 0;
                    if (full) {
#pragma unroll
                        for (int j = 0; j < kSaJ; ++j) {
                            uint32_t x[4], y[4];
                            lds16(slot(sc, j, 0), x);
                            lds16(slot(sc, j, 1), y);
                            d |= (x[0] ^ y[0]) | (x[1] ^ y[1]) | (x[2] ^ y[2]) | (x[3] ^ y[3]);
                        }
                    } else {
#pragma unroll
                        for (int j = 0; j < kSaJ; ++j) {
                            const uint32_t w = w0 + 8 * j + g;
                            if (w < nw) {
                                uint32_t x[4], y[4];
                                lds16(slot(sc, j, 0), x);
                                lds16(slot(sc, j, 1), y);
#pragma unroll
                                for (int e = 0; e < 4; ++e) x[e] ^= y[e];
                                if (w + 1 == nw) mask_word(x, n, w);   // only the last word is partial
                                d |= x[0] | x[1] | x[2] | x[3];
                            }
                        }
                    }
                    if (d) {   // rare: the lowest differing word of this step
#pragma unroll 1
                        for (int j = 0; j < kSaJ; ++j) {
                            const uint32_t w = w0 + 8 * j + g;
                            if (w >= nw) break;
                            uint32_t x[4], y[4];
                            lds16(slot(sc, j, 0), x);
                            lds16(slot(sc, j, 1), y);
                            mask_word(x, n, w);
                            mask_word(y, n, w);
                            if ((x[0] ^ y[0]) | (x[1] ^ y[1]) | (x[2] ^ y[2]) | (x[3] ^ y[3])) {
                                found = w;
                                break;
                            }
                        }
                    }
                }
            } else {
                // leader / singleton: hash (two accumulator chains: even / odd words)
                if (full) {
#pragma unroll
                    for (int j = 0; j < kSaJ; ++j) {
                        uint32_t x[4];
                        lds16(slot(sc, j, 0), x);
                        if (j & 1) nh_word(x[0], x[1], x[2], x[3], K.k[1], A2, B2);
                        else nh_word(x[0], x[1], x[2], x[3], K.k[0], A, B);
                        if (j & 1) advance<1>(K);
                    }
                } else {
#pragma unroll
                    for (int j = 0; j < kSaJ; ++j) {
                        const uint32_t w = w0 + 8 * j + g;
                        if (w < nw) {
                            uint32_t x[4];
                            lds16(slot(sc, j, 0), x);
                            if (w + 1 == nw) mask_word(x, n, w);   // only the last word is partial
                            if (j & 1) nh_word(x[0], x[1], x[2], x[3], K.k[1], A2, B2);
                            else nh_word(x[0], x[1], x[2], x[3], K.k[0], A, B);
                        }
                        if (j & 1) advance<1>(K);
                    }
                }
            }
        }
        // record ends (warp-uniform: any octet finishing one reduces with all four); the
        // NH sums only when a hashed record ends, the first-mismatch minimum only when an
        // ending compared record has a mismatch (rare)
        const bool last = !done && (z & kSaLast) != 0;
        if (__any_sync(0xFFFFFFFFu, last)) {
            const bool cmp_end = last && (z & kSaCmp) != 0;
            if (__any_sync(0xFFFFFFFFu, last && !cmp_end)) {
                uint64_t a = A + A2, b = B + B2;
#pragma unroll
                for (int o = 4; o; o >>= 1) {
                    a += __shfl_xor_sync(0xFFFFFFFFu, a, o);
                    b += __shfl_xor_sync(0xFFFFFFFFu, b, o);
                }
                if (last && !cmp_end && g == 0) {
                    W.accA[r] = a;
                    W.accB[r] = b;
                    W.digest[r] = finalize_digest(a, b, n);
                }
            }
            if (__any_sync(0xFFFFFFFFu, cmp_end && found != ~0u)) {
                uint32_t f = found;
#pragma unroll
                for (int o = 4; o; o >>= 1) f = min(f, __shfl_xor_sync(0xFFFFFFFFu, f, o));
                if (cmp_end && g == 0 && f != ~0u) report_mismatch(W, r, f, res_out, false);
            }
        }
        return true;
    };
#pragma unroll 1
    while (iteration(0, 1) && iteration(1, 0)) {
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
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
    // kLabelU records per thread per step: their leader -> gid loads are independent
    constexpr int kLabelU = 4;
    const uint32_t stride = gridDim.x * blockDim.x;
    for (uint32_t r0 = blockIdx.x * blockDim.x + threadIdx.x; r0 < L.n; r0 += kLabelU * stride) {
        uint32_t ld[kLabelU];
#pragma unroll
        for (int u = 0; u < kLabelU; ++u) {
            const uint32_t r = r0 + u * stride;
            ld[u] = r < L.n ? leader[r] : r;
        }
        int64_t d[kLabelU];
#pragma unroll
        for (int u = 0; u < kLabelU; ++u) {
            const uint32_t r = r0 + u * stride;
            // (no labels to write -- they went out speculatively: membership suffices)
            d[u] = (r >= L.n || ld[u] == r) ? -1 : (dup_out ? (int64_t)L.gid[ld[u]] : 0);
        }
#pragma unroll
        for (int u = 0; u < kLabelU; ++u) {
            const uint32_t r = r0 + u * stride;
            if (r >= L.n) break;
            if (dup_out) dup_out[r] = d[u];   // (null: written speculatively before H3)
            if (d[u] >= 0) {
                const uint32_t s = L.site[r];
                atomicAdd(&sben[s], (unsigned long long)L.dur[r]);
                atomicAdd(&scnt[s], 1u);
            }
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
    // 8 lanes per site, each summing every 8th row (independent loads in flight), then
    // an 8-lane shuffle sum: ~rows / 8 dependent steps instead of rows
    const uint32_t s = (blockIdx.x * blockDim.x + threadIdx.x) >> 3;
    const uint32_t q = threadIdx.x & 7;
    uint64_t acc = 0, c = 0;
    if (s < n_sites) {
        for (uint32_t b = q; b < rows; b += 8) {
            acc += part[(uint64_t)b * n_sites + s];
            c += cpart[(uint64_t)b * n_sites + s];
        }
    }
#pragma unroll
    for (int o = 4; o; o >>= 1) {
        acc += __shfl_xor_sync(0xFFFFFFFFu, acc, o);
        c += __shfl_xor_sync(0xFFFFFFFFu, c, o);
    }
    if (s < n_sites && q == 0) {
        ben[s] = acc;
        cnt[s] = c;
    }
}

__global__ void __launch_bounds__(256) k_label_global(DevLog L, const uint32_t* __restrict__ leader,
                                                      int64_t* __restrict__ dup_out, uint64_t* __restrict__ ben,
                                                      uint64_t* __restrict__ cnt) {
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < L.n; r += gridDim.x * blockDim.x) {
        uint32_t ld = leader[r];
        int64_t d = ld == r ? -1 : (int64_t)L.gid[ld];
        if (dup_out) dup_out[r] = d;
        if (d >= 0) {
            atomicAdd((unsigned long long*)&ben[L.site[r]], (unsigned long long)L.dur[r]);
            atomicAdd((unsigned long long*)&cnt[L.site[r]], 1ull);
        }
    }
}

// Speculative labels right after the round-0 group-by: a member's candidate is its
// label unless H3 finds it differs (a residual -- rare; its final label is written after
// resolution).  Lets the D2H of duplicate_of overlap H3 (PCIe under the HBM stream).
__global__ void k_spec_label(DevLog L, const uint32_t* __restrict__ leader, int64_t* __restrict__ dup_out) {
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= L.n) return;
    const uint32_t ld = leader[r];
    dup_out[r] = ld == r ? -1 : (int64_t)L.gid[ld];
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

// grid for one warp per item (FFM_WARP_EACH): at most one resident wave of 256-thread blocks
static uint32_t warp_grid(uint64_t items, int num_sms) {
    const uint64_t b = (items * 32 + 255) / 256, cap = (uint64_t)num_sms * 8;
    return (uint32_t)(b == 0 ? 1 : (b < cap ? b : cap));
}

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
    k_hash_small<<<need < grid ? need : grid, 256, 0, st>>>(L, P.small_bytes, W.accA, W.accB, W.digest);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_fused_small(const DevLog& L, Work& W, const Params& P, uint32_t* res_out, cudaStream_t st) {
    if (L.n == 0 || L.n_small == 0) return 0;

    // (measured: capping its grid so that it co-resides with the persistent large pass
    // slowed that pass more than it hid -- profiles/r01b/README.md)
    if (!smem_configured((const void*)k_fused_small, kSaSmem)) return -1;
    static int occ = 0;   // per process: one device type
    if (occ == 0 && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_fused_small, kSaT, kSaSmem) != cudaSuccess ||
                     occ < 1))
        occ = 1;
    uint32_t grid = (uint32_t)(occ * P.num_sms);
    uint32_t need = blocks_for((uint64_t)L.n_small * 8, kSaT);
    k_fused_small<<<need < grid ? need : grid, kSaT, kSaSmem, st>>>(L, W, res_out);
    FFM_LAUNCH_CHECK();
    return 1;
}

// Chunk slots of large payloads (count -> scan); two-pass also scatters the
// (record, chunk) work units of k_hash_large.
int launch_hash_plan(const DevLog& L, Work& W, const Params& P, bool units, cudaStream_t st) {
    k_hash_count<<<blocks_for((uint64_t)L.n + 1), 256, 0, st>>>(L, P.small_bytes, P.chunk_bytes, W.hcount);
    FFM_LAUNCH_CHECK();
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.hcount, W.hstart, (int)(L.n + 1), st) != cudaSuccess)
        return -1;
    if (units && L.n_large) {
        k_hash_fill<<<warp_grid(L.n_large, P.num_sms), 256, 0, st>>>(L, P.small_bytes, P.chunk_bytes, W.hstart,
                                                                     W.hitems);
        FFM_LAUNCH_CHECK();
        return 3;
    }
    return 2;
}

int launch_hash_large(const DevLog& L, Work& W, const Params& P, uint64_t n_items, cudaStream_t st) {
    if (n_items == 0) return 0;
    uint32_t grid = resident_grid((const void*)k_hash_large, P.num_sms);
    uint32_t need = blocks_for(n_items * 32);
    k_hash_large<<<need < grid ? need : grid, 256, 0, st>>>(L, W.hitems, W.hstart + L.n, P.chunk_bytes, W.hpart);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_prefix(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    if (L.n_large == 0) return 0;
    k_prefix_hash<<<warp_grid(L.n_large, P.num_sms), 256, 0, st>>>(L, W, P.prefix_bytes);
    FFM_LAUNCH_CHECK();
    return 1;
}

// Round 0, large payloads: fused groups (scan of lcount), work units, the fused
// hash + compare pass, then the per-record combine of chunk partial sums.
int launch_combine(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    if (L.n == 0) return 0;
    k_hash_combine<<<warp_grid(L.n_large, P.num_sms), 256, 0, st>>>(L, W, P.chunk_bytes, P.prefix_bytes, 0, 0);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_fused(const DevLog& L, Work& W, const Params& P, uint64_t n_units, bool prefilter, uint32_t* res_out,
                 cudaStream_t st, cudaEvent_t ev_a, cudaEvent_t ev_b) {
    if (L.n == 0 || n_units == 0 || L.n_large == 0) return 0;
    if (!smem_configured((const void*)k_fused_fx<false>, (int)kFxSmem)) return -1;
    int k = 0;
    // entries per head (pieces x (members + sub-task leader copies)), their scan, the
    // stage descriptors, the pipelined pass, the per-record combine
    k_fx_count<<<blocks_for((uint64_t)L.n + 1), 256, 0, st>>>(L, W, P.small_bytes, P.chunk_bytes, 0);
    FFM_LAUNCH_CHECK();
    size_t bytes = W.cub_tmp_bytes;
    if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.lcount, W.lstart, (int)(L.n + 1), st) != cudaSuccess)
        return -1;
    k_fx_fill<<<warp_grid(L.n_large, P.num_sms), 256, 0, st>>>(L, W, P.chunk_bytes, P.prefix_bytes,
                                                               prefilter ? 1 : 0, reinterpret_cast<FxDesc*>(W.fitems));
    FFM_LAUNCH_CHECK();
    k += 3;
    if (ev_a && cudaEventRecord(ev_a, st) != cudaSuccess) return -1;
    k_fused_fx<false><<<P.num_sms * FFM_FX_CTAS, kFxThreads, kFxSmem, st>>>(
        L, W, reinterpret_cast<const FxDesc*>(W.fitems), W.lstart + L.n, P.prefix_bytes >> 4, res_out);
    FFM_LAUNCH_CHECK();
    ++k;
    if (ev_b && cudaEventRecord(ev_b, st) != cudaSuccess) return -1;
    k_hash_combine<<<warp_grid(L.n_large, P.num_sms), 256, 0, st>>>(L, W, P.chunk_bytes, P.prefix_bytes,
                                                                   prefilter ? 1 : 0, 1);
    FFM_LAUNCH_CHECK();
    return k + 1;
}

// Capacity (entries) the pipelined fused pass may need beyond the chunk count: pieces
// smaller than chunks and one leader copy per extra sub-task (host-side bound).
uint64_t fx_entry_cap(uint64_t n_large_chunks, uint32_t chunk_bytes) {
    const FxSplit f = fx_split(chunk_bytes);
    return n_large_chunks * (uint64_t)f.ppc + (n_large_chunks * (uint64_t)f.ppc) / (kFxMaxK - 1) + 64;
}

int launch_group(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list, uint64_t cap,
                 int round, uint32_t* res_out, cudaStream_t st, bool use_diff, uint32_t label_sites, int64_t* label_dup) {
    if (n_list == 0) return 0;
    int k = 0;
    if (round > 0) {
        k_refine<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, round, P.refine_mask);
        FFM_LAUNCH_CHECK();
        ++k;
    }
    if (cudaMemsetAsync(W.tkey, 0xFF, cap * sizeof(uint64_t), st) != cudaSuccess) return -1;
    // per-leader large-member counts: only large records use them
    if (L.n_large) {
        if (cudaMemsetAsync(W.lcount, 0, ((uint64_t)L.n + 1) * sizeof(uint32_t), st) != cudaSuccess) return -1;
        if (cudaMemsetAsync(W.gcount, 0, ((uint64_t)L.n + 1) * sizeof(uint32_t), st) != cudaSuccess) return -1;
    }
    k_group_insert<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, cap - 1, P.digest_mask, round,
                                                        P.small_bytes);
    FFM_LAUNCH_CHECK();
    if (round == 0 && label_sites) {
        // H5 + H6 folded into the lookup (speculative; label_fused_ok decided it fits)
        if (!smem_configured((const void*)k_leader0_label, P.max_smem)) return -1;
        const uint32_t rows = label_hist_rows(P.num_sms);
        k_leader0_label<<<rows, 1024, label_smem_bytes(label_sites), st>>>(
            L, W, n_list, P.small_bytes, res_out, label_sites, label_dup, W.label_part, W.label_cpart);
        FFM_LAUNCH_CHECK();
        return k + 2;   // (the caller launches k_site_reduce over the rows: launch_site_reduce)
    } else if (round == 0)
        k_leader0<<<blocks_for(n_list), 256, 0, st>>>(L, W, n_list, P.small_bytes, res_out);
    else if (round < 0)
        k_leader<<<blocks_for(n_list), 256, 0, st>>>(L, W, nullptr, n_list, P.small_bytes, P.chunk_bytes, res_out, 0);
    else
        k_leader<<<blocks_for(n_list), 256, 0, st>>>(L, W, list, n_list, P.small_bytes, P.chunk_bytes, res_out,
                                                     use_diff ? 1 : 0);
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
    if (vitem_cap && L.n_large) {
        // large members: groups per leader (scan of per-leader entry counts), then the
        // pipelined pass in verify mode (leader piece in registers, members compared)
        if (!smem_configured((const void*)k_fused_fx<true>, (int)kFxSmem)) return -1;
        k_fx_count<<<blocks_for((uint64_t)L.n + 1), 256, 0, st>>>(L, W, P.small_bytes, P.chunk_bytes, 1);
        FFM_LAUNCH_CHECK();
        size_t bytes = W.cub_tmp_bytes;
        if (cub::DeviceScan::ExclusiveSum(W.cub_tmp, bytes, W.lcount, W.lstart, (int)(L.n + 1), st) != cudaSuccess)
            return -1;
        k_fx_vfill<<<warp_grid(list ? n_list : L.n_large, P.num_sms), 256, 0, st>>>(
            L, W, list, n_list, P.small_bytes, P.chunk_bytes, reinterpret_cast<FxDesc*>(W.fitems));
        FFM_LAUNCH_CHECK();
        k_fused_fx<true><<<P.num_sms * FFM_FX_CTAS, kFxThreads, kFxSmem, st>>>(
            L, W, reinterpret_cast<const FxDesc*>(W.fitems), W.lstart + L.n, 0xFFFFFFFFu, res_out);
        FFM_LAUNCH_CHECK();
        k += 4;
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
    k_site_reduce<<<blocks_for((uint64_t)n_sites * 8), 256, 0, st>>>(part, cpart, rows, n_sites, ben, cnt);
    FFM_LAUNCH_CHECK();
    return 1;
}

size_t label_smem_bytes(uint32_t n_sites) { return (size_t)n_sites * (sizeof(uint64_t) + sizeof(uint32_t)); }

bool label_fused_ok(const Work& W, const Params& P, uint32_t n_sites) {
    return W.label_part != nullptr && label_smem_bytes(n_sites) <= (size_t)P.max_smem;
}

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

// Debug digests after a fused round 0: an equal small member was never hashed -- its
// digest is its final leader's (equal bytes).
__global__ void k_digest_fill(DevLog L, Work W, uint32_t small_bytes) {
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= L.n || L.size[r] > small_bytes) return;
    const uint32_t ld = W.leader[r];
    if (ld == r) W.digest[r] = finalize_digest(W.accA[r], W.accB[r], L.size[r]);   // hashed (maybe as a residual)
}

// (second pass: members copy their leader's digest, final after the pass above)
__global__ void k_digest_copy(DevLog L, Work W, uint32_t small_bytes) {
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= L.n || L.size[r] > small_bytes) return;
    const uint32_t ld = W.leader[r];
    if (ld != r) W.digest[r] = W.digest[ld];
}

int launch_spec_label(const DevLog& L, Work& W, int64_t* dup_out, cudaStream_t st) {
    if (L.n == 0) return 0;
    k_spec_label<<<blocks_for(L.n), 256, 0, st>>>(L, W.leader, dup_out);
    FFM_LAUNCH_CHECK();
    return 1;
}

int launch_digest_fill(const DevLog& L, Work& W, const Params& P, cudaStream_t st) {
    if (L.n == 0) return 0;
    k_digest_fill<<<blocks_for(L.n), 256, 0, st>>>(L, W, P.small_bytes);
    FFM_LAUNCH_CHECK();
    k_digest_copy<<<blocks_for(L.n), 256, 0, st>>>(L, W, P.small_bytes);
    FFM_LAUNCH_CHECK();
    return 2;
}

// NH sums of the small records of a list (the residual members of a fused round 0).
int launch_hash_small_list(const DevLog& L, Work& W, const Params& P, const uint32_t* list, uint32_t n_list,
                           cudaStream_t st) {
    if (n_list == 0) return 0;
    DevLog D = L;
    D.small_order = list;
    D.n_small = n_list;
    return launch_hash_small(D, W, P, st);
}

__global__ void k_iota(uint32_t* __restrict__ a, uint32_t n) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) a[i] = i;
}

int launch_iota(uint32_t* a, uint32_t n, cudaStream_t st) {
    if (n == 0) return 0;
    k_iota<<<blocks_for(n), 256, 0, st>>>(a, n);
    FFM_LAUNCH_CHECK();
    return 1;
}

__global__ void k_invert(const uint32_t* __restrict__ order, uint32_t n, uint32_t* __restrict__ inv) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) inv[order[i]] = i;
}

int launch_invert(const uint32_t* order, uint32_t n, uint32_t* inv, cudaStream_t st) {
    if (n == 0) return 0;
    k_invert<<<blocks_for(n), 256, 0, st>>>(order, n, inv);
    FFM_LAUNCH_CHECK();
    return 1;
}

// Online window order (counting sort by size class, 2 kernels): class c of a record =
// maxb - (its 32-byte block count) for a small one (largest first), maxb + 1 for a large
// one.  bins = [count | cursor | done], zero between windows.
__device__ __forceinline__ uint32_t window_class(uint64_t sz, uint32_t small_bytes) {
    const uint32_t maxb = (small_bytes + 31) / 32;
    return sz <= small_bytes ? maxb - (uint32_t)((sz + 31) / 32) : maxb + 1;
}

__host__ __device__ uint32_t window_bins(uint32_t small_bytes) { return (small_bytes + 31) / 32 + 2; }

// gathers the window's metadata into the fixed buffers, counts its classes; the last block
// turns the counts into the classes' start positions (and zeroes the counts for the next)
__global__ void __launch_bounds__(1024) k_wclass_count(DevLog L, const uint64_t* __restrict__ d_a, uint32_t n,
                                                      WinMeta wm, uint32_t small_bytes, uint32_t* __restrict__ bins) {
    extern __shared__ uint32_t hist[];
    __shared__ bool last;
    const uint32_t nb = window_bins(small_bytes);
    uint32_t* cnt = bins;
    uint32_t* cur = bins + nb;
    uint32_t* done = bins + 2 * nb;
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) hist[b] = 0;
    __syncthreads();
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) {
        const uint64_t j = *d_a + i;
        const uint64_t sz = L.size[j];
        wm.off[i] = L.off[j];
        wm.size[i] = sz;
        wm.dur[i] = L.dur[j];
        wm.gid[i] = L.gid[j];
        wm.chan[i] = L.chan[j];
        wm.site[i] = L.site[j];
        atomicAdd(&hist[window_class(sz, small_bytes)], 1u);
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x)
        if (hist[b]) atomicAdd(&cnt[b], hist[b]);
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!last) return;
    // the last block: exclusive scan of the counts (read and zeroed atomically)
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) hist[b] = atomicExch(&cnt[b], 0u);
    __syncthreads();
    if (threadIdx.x < 32) {
        uint32_t base = 0;
        for (uint32_t b0 = 0; b0 < nb; b0 += 32) {
            const uint32_t b = b0 + threadIdx.x;
            const uint32_t v = b < nb ? hist[b] : 0u;
            uint32_t x = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
                if ((int)threadIdx.x >= o) x += y;
            }
            if (b < nb) cur[b] = base + x - v;
            base += __shfl_sync(0xFFFFFFFFu, x, 31);
        }
        if (threadIdx.x == 0) *done = 0;
    }
}

// each record takes the next position of its class: ranks within the block from shared
// memory atomics, then one global atomic per (block, class present) reserves the range
__global__ void __launch_bounds__(1024) k_wclass_scatter(const WinMeta wm, uint32_t n, uint32_t small_bytes,
                                                         uint32_t* __restrict__ bins, uint32_t* __restrict__ order,
                                                         uint32_t* __restrict__ inv) {
    extern __shared__ uint32_t hist[];   // [nb] counts, then [nb] bases
    const uint32_t nb = window_bins(small_bytes);
    uint32_t* base = hist + nb;
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) hist[b] = 0;
    __syncthreads();
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t c = 0, rank = 0;
    if (i < n) {
        c = window_class(wm.size[i], small_bytes);
        rank = atomicAdd(&hist[c], 1u);
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x)
        if (hist[b]) base[b] = atomicAdd(&bins[nb + b], hist[b]);
    __syncthreads();
    if (i < n) {
        const uint32_t pos = base[c] + rank;
        order[pos] = i;
        inv[i] = pos;
    }
}

int launch_window_order(const DevLog& L, const uint64_t* d_a, uint32_t n, const WinMeta& wm, uint32_t small_bytes,
                        uint32_t* bins, uint32_t* order, uint32_t* inv, cudaStream_t st) {
    if (n == 0) return 0;
    const uint32_t nb = window_bins(small_bytes);
    k_wclass_count<<<blocks_for(n, 1024), 1024, nb * sizeof(uint32_t), st>>>(L, d_a, n, wm, small_bytes, bins);
    FFM_LAUNCH_CHECK();
    k_wclass_scatter<<<blocks_for(n, 1024), 1024, 2 * nb * sizeof(uint32_t), st>>>(wm, n, small_bytes, bins, order,
                                                                                  inv);
    FFM_LAUNCH_CHECK();
    return 2;
}

int launch_zero_counters(Work& W, cudaStream_t st) {
    return cudaMemsetAsync(W.counters, 0, 16 * sizeof(uint32_t), st) == cudaSuccess ? 0 : -1;
}

}  // namespace ffm
