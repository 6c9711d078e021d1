// probe_small_read.cu -- how fast can the small-payload records of a config-2-shaped arena
// be READ (no hashing / comparing), per access pattern?  Separates the memory system's limit
// from the small pass's instruction overhead.  Not part of the product.
//
// Arena: N records, sizes log-uniform [256, 4096] B, 32-B aligned slots back to back (as the
// library lays them out).  Orders: gid (arena order) and size-class (stable, block count
// descending: k_fused_small's order).  Kernels:
//   octet_ldg   8 lanes per record, 256-bit loads, every lane all its blocks in flight (<= 2)
//   octet_cp    8 lanes per record, cp.async 16 B into private smem slots, S=2 steps of 4 words
//   warp_rec    32 lanes per record, 256-bit loads (one instruction = 1 KiB of the record)
//   flat        the arena as one contiguous stream, 256-bit loads, 4 in flight per lane
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>

struct B8 {
    uint32_t v[8];
};
__device__ __forceinline__ B8 ld(const void* p) {
    B8 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]), "=r"(r.v[6]),
                   "=r"(r.v[7])
                 : "l"(p));
    return r;
}

__global__ void __launch_bounds__(256) k_octet_ldg(const uint8_t* arena, const uint64_t* off, const uint32_t* nb,
                                                   const uint32_t* order, uint32_t n, uint32_t* sink) {
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3, noct = (gridDim.x * blockDim.x) >> 3;
    uint32_t acc = 0;
    for (uint32_t i = oct; i < n; i += noct) {
        const uint32_t r = order[i];
        const uint8_t* p = arena + off[r];
        const uint32_t k = nb[r];
        for (uint32_t b = g; b < k; b += 32) {
            B8 x[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) x[u] = b + 8 * u < k ? ld(p + 32ull * (b + 8 * u)) : B8{};
#pragma unroll
            for (int u = 0; u < 4; ++u)
                for (int j = 0; j < 8; ++j) acc ^= x[u].v[j];
        }
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

__global__ void __launch_bounds__(256) k_warp_rec(const uint8_t* arena, const uint64_t* off, const uint32_t* nb,
                                                  const uint32_t* order, uint32_t n, uint32_t* sink) {
    const int lane = threadIdx.x & 31;
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nwp = (gridDim.x * blockDim.x) >> 5;
    uint32_t acc = 0;
    for (uint32_t i = w; i < n; i += 2 * nwp) {
        // two records per iteration: their loads in flight together
        const uint32_t r0 = order[i], r1 = i + nwp < n ? order[i + nwp] : order[i];
        const uint8_t* p0 = arena + off[r0];
        const uint8_t* p1 = arena + off[r1];
        const uint32_t k0 = nb[r0], k1 = i + nwp < n ? nb[r1] : 0;
        B8 x[8];
#pragma unroll
        for (int u = 0; u < 4; ++u) x[u] = lane + 32u * u < k0 ? ld(p0 + 32ull * (lane + 32 * u)) : B8{};
#pragma unroll
        for (int u = 0; u < 4; ++u) x[4 + u] = lane + 32u * u < k1 ? ld(p1 + 32ull * (lane + 32 * u)) : B8{};
#pragma unroll
        for (int u = 0; u < 8; ++u)
            for (int j = 0; j < 8; ++j) acc ^= x[u].v[j];
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

__device__ __forceinline__ void cp16(uint32_t dst, const uint8_t* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}

// octet per record, each lane 4 x 16 B per step, 2 stages (the small pass's memory pattern)
__global__ void __launch_bounds__(128) k_octet_cp(const uint8_t* arena, const uint64_t* off, const uint32_t* nb,
                                                  const uint32_t* order, uint32_t n, uint32_t* sink) {
    extern __shared__ __align__(16) uint8_t sm[];
    const int g = threadIdx.x & 7;
    const uint32_t oct = (blockIdx.x * blockDim.x + threadIdx.x) >> 3, noct = (gridDim.x * blockDim.x) >> 3;
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm) + threadIdx.x * 16;
    uint32_t fi = oct, fw = 0, nw = 0;
    const uint8_t* p = nullptr;
    if (fi < n) {
        p = arena + off[order[fi]];
        nw = 2 * nb[order[fi]];
    }
    auto fetch = [&](int s) {
        if (fi < n) {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (fw + 8 * j + g < nw) cp16(base + (uint32_t)((s * 4 + j) * 128 * 16), p + 16ull * (fw + 8 * j + g));
            fw += 32;
            if (fw >= nw) {
                fi += noct;
                fw = 0;
                if (fi < n) {
                    p = arena + off[order[fi]];
                    nw = 2 * nb[order[fi]];
                }
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    uint32_t acc = 0;
    fetch(0);
    int sc = 0;
    for (int it = 0;; ++it) {
        const bool more = fi < n;
        fetch(sc ^ 1);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            uint32_t v[4];
            asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
                         : "r"(base + (uint32_t)((sc * 4 + j) * 128 * 16)));
            acc ^= v[0] ^ v[1] ^ v[2] ^ v[3];
        }
        sc ^= 1;
        if (!__any_sync(0xFFFFFFFFu, more)) break;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

__global__ void __launch_bounds__(256) k_flat(const uint8_t* p, uint64_t nblk, uint32_t* sink) {
    uint32_t acc = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b < nblk; b += 4 * stride) {
        B8 x[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) x[u] = b + u * stride < nblk ? ld(p + 32 * (b + u * stride)) : B8{};
#pragma unroll
        for (int u = 0; u < 4; ++u)
            for (int j = 0; j < 8; ++j) acc ^= x[u].v[j];
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

int main(int argc, char** argv) {
    const uint32_t n = argc > 1 ? (uint32_t)atoi(argv[1]) : 1000000u;
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    std::mt19937_64 rng(0x5C19);
    std::vector<uint64_t> off(n);
    std::vector<uint32_t> nb(n);
    uint64_t cur = 0, payload = 0;
    for (uint32_t i = 0; i < n; ++i) {
        const double u = std::uniform_real_distribution<double>(0, 1)(rng);
        const uint32_t sz = (uint32_t)std::exp(std::log(256.0) + u * (std::log(4096.0) - std::log(256.0)));
        off[i] = cur;
        nb[i] = (sz + 31) / 32;
        cur += ((uint64_t)sz + 31) / 32 * 32;
        payload += sz;
    }
    std::vector<uint32_t> gid(n), cls(n);
    for (uint32_t i = 0; i < n; ++i) gid[i] = cls[i] = i;
    std::stable_sort(cls.begin(), cls.end(), [&](uint32_t a, uint32_t b) { return nb[a] > nb[b]; });
    uint8_t* arena;
    uint64_t* doff;
    uint32_t *dnb, *dgid, *dcls, *sink;
    cudaMalloc(&arena, cur + 4096);
    cudaMemset(arena, 7, cur + 4096);
    cudaMalloc(&doff, 8ull * n);
    cudaMalloc(&dnb, 4ull * n);
    cudaMalloc(&dgid, 4ull * n);
    cudaMalloc(&dcls, 4ull * n);
    cudaMalloc(&sink, 4);
    cudaMemcpy(doff, off.data(), 8ull * n, cudaMemcpyHostToDevice);
    cudaMemcpy(dnb, nb.data(), 4ull * n, cudaMemcpyHostToDevice);
    cudaMemcpy(dgid, gid.data(), 4ull * n, cudaMemcpyHostToDevice);
    cudaMemcpy(dcls, cls.data(), 4ull * n, cudaMemcpyHostToDevice);
    // a buffer larger than L2 to flush between timed runs
    uint8_t* flush;
    cudaMalloc(&flush, 512ull << 20);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaFuncSetAttribute(k_octet_cp, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 4 * 128 * 16);
    auto timeit = [&](const char* name, const char* ord, auto launch) {
        float best = 1e9f;
        for (int it = 0; it < 8; ++it) {
            cudaMemsetAsync(flush, it, 512ull << 20);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = std::min(best, ms);
        }
        cudaError_t e = cudaGetLastError();
        printf("{\"kernel\": \"%s\", \"order\": \"%s\", \"ms\": %.4f, \"payload_gbs\": %.1f, \"slot_gbs\": %.1f, \"err\": \"%s\"}\n",
               name, ord, best, payload / (best * 1e-3) / 1e9, cur / (best * 1e-3) / 1e9, cudaGetErrorString(e));
    };
    for (int o = 0; o < 2; ++o) {
        const uint32_t* ord = o ? dcls : dgid;
        const char* on = o ? "size_class" : "gid";
        for (int bps : {4, 8})
            timeit(bps == 4 ? "octet_ldg_4cta" : "octet_ldg_8cta", on,
                   [&] { k_octet_ldg<<<sms * bps, 256>>>(arena, doff, dnb, ord, n, sink); });
        timeit("octet_cp_6cta", on, [&] { k_octet_cp<<<sms * 6, 128, 2 * 4 * 128 * 16>>>(arena, doff, dnb, ord, n, sink); });
        timeit("octet_cp_12cta", on, [&] { k_octet_cp<<<sms * 12, 128, 2 * 4 * 128 * 16>>>(arena, doff, dnb, ord, n, sink); });
        for (int bps : {4, 8})
            timeit(bps == 4 ? "warp_rec_4cta" : "warp_rec_8cta", on,
                   [&] { k_warp_rec<<<sms * bps, 256>>>(arena, doff, dnb, ord, n, sink); });
    }
    timeit("flat", "arena", [&] { k_flat<<<sms * 8, 256>>>(arena, cur / 32, sink); });
    return 0;
}
