// digest.cuh -- device helpers shared by the hot-path kernels (kernels.cu, shard.cu):
// 64-bit mixing, the group key, 32-byte block loads with cache-policy hints.
#pragma once

#include <stdint.h>

#include "ffm_internal.h"

namespace ffm {

// NH keys of the digest: KA[position][j] from splitmix64, per-stripe
// steps DA[j] (see kernels.cu for the formula).
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

__host__ __device__ __forceinline__ uint64_t fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}

__device__ __forceinline__ uint64_t finalize_digest(uint64_t A, uint64_t B, uint64_t n) {
    return fmix64(A ^ fmix64(B ^ (n * 0x9E3779B97F4A7C15ull)));
}

__device__ __forceinline__ uint64_t not_empty(uint64_t k) { return k == kEmptyKey ? k - 1 : k; }

// Group key of (digest, size, channel).  Equal bytes, size and channel => equal key;
// digest_bits truncation (mask) forces collisions without changing results.
__device__ __forceinline__ uint64_t group_key(uint64_t digest, uint64_t n, uint64_t mask, uint64_t chan) {
    return not_empty(fmix64((digest & mask) ^ fmix64(n + 0x632BE59BD9B4E019ull) ^
                            fmix64(chan ^ 0x2545F4914F6CDD1Dull)));
}

// 32-byte block = two 16-byte words.
struct Blk {
    uint32_t v[8];
};

// Streamed payload bytes: read once, do not pollute L1, evict first from L2.
__device__ __forceinline__ Blk ld_stream(const uint8_t* p) {
    Blk r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
                   "=r"(r.v[6]), "=r"(r.v[7])
                 : "l"(p));
    return r;
}

// Leader bytes during verify: re-read by every member of the class -> keep in L2.
__device__ __forceinline__ Blk ld_keep(const uint8_t* p) {
    Blk r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_last.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
                   "=r"(r.v[6]), "=r"(r.v[7])
                 : "l"(p));
    return r;
}

__device__ __forceinline__ Blk zero_blk() {
    Blk r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.v[i] = 0;
    return r;
}

// Zero the bytes of block b at or beyond n (only the record's last block is partial).
__device__ __forceinline__ void mask_tail(Blk& x, uint64_t n, uint64_t b) {
    int64_t valid = (int64_t)n - (int64_t)(32 * b);
    if (valid >= 32) return;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        int64_t vb = valid - 4 * i;
        uint32_t m = vb >= 4 ? 0xFFFFFFFFu : (vb <= 0 ? 0u : ((1u << (8 * vb)) - 1u));
        x.v[i] &= m;
    }
}


// Remote (peer-GPU, NVLink) payload bytes: plain non-coherent 256-bit load.
__device__ __forceinline__ Blk ld_remote(const uint8_t* p) {
    Blk r;
    asm volatile("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
                   "=r"(r.v[6]), "=r"(r.v[7])
                 : "l"(p));
    return r;
}

__device__ __forceinline__ bool blk_equal(const Blk& x, const Blk& y) {
    uint32_t d = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) d |= x.v[i] ^ y.v[i];
    return d == 0;
}

// Each warp scans 32 consecutive list entries, ballots the ones that need work and
// then serves them one at a time with all 32 lanes (cheap skipping of small records).
#define FFM_WARP_COMPACT(n_list, list, PRED, ...)                                         \
    {                                                                                      \
        const int lane_ = threadIdx.x & 31;                                                \
        const uint32_t i_ = blockIdx.x * blockDim.x + threadIdx.x;                         \
        uint32_t r_ = 0;                                                                   \
        bool act_ = false;                                                                 \
        if (i_ < (n_list)) {                                                               \
            r_ = (list) ? (list)[i_] : i_;                                                 \
            act_ = (PRED);                                                                 \
        }                                                                                  \
        unsigned bal_ = __ballot_sync(0xFFFFFFFFu, act_);                                  \
        while (bal_) {                                                                     \
            const int src_ = __ffs(bal_) - 1;                                              \
            bal_ &= bal_ - 1;                                                              \
            const uint32_t rec = __shfl_sync(0xFFFFFFFFu, r_, src_);                       \
            const int lane = lane_;                                                        \
            __VA_ARGS__                                                                    \
        }                                                                                  \
    }

// One warp per item (grid-stride over warps): item w is record REC_EXPR (may use w_);
// the body runs with all 32 lanes when PRED(rec) holds.  For per-record planning work
// whose size varies by orders of magnitude (a few records of ~1000 chunks each, or
// millions of single-chunk ones).
#define FFM_WARP_EACH(COUNT, REC_EXPR, PRED, ...)                                         \
    {                                                                                      \
        const int lane = threadIdx.x & 31;                                                 \
        const uint32_t nw_ = (gridDim.x * blockDim.x) >> 5;                                \
        for (uint32_t w_ = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w_ < (COUNT); w_ += nw_) { \
            const uint32_t rec = (REC_EXPR);                                               \
            if (!(PRED)) continue;                                                         \
            __VA_ARGS__                                                                    \
        }                                                                                  \
    }

}  // namespace ffm
