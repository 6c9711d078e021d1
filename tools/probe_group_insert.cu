// probe_group_insert.cu -- where does the round-0 group insert's time go on a config-2-shaped
// log?  The same work as k_group_insert (metadata loads, the 32-byte payload prefix, a key,
// one CAS into a 2^21-slot table) and variants without parts of it.  Not part of the product.
//
// Log: 1,000,000 records, 256 "sites" with a fixed size each (log-uniform 256 B - 4 KiB,
// Zipf(1.0) site choice), 60% of records re-upload their site's current content (so equal
// prefixes -> shared groups), 32-B aligned arena slots in gid order.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>

__device__ __forceinline__ uint64_t fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}

struct B8 {
    uint32_t v[8];
};
__device__ __forceinline__ B8 ld_stream(const void* p) {
    B8 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]), "=r"(r.v[6]),
                   "=r"(r.v[7])
                 : "l"(p));
    return r;
}

// MODE 0: full; 1: no CAS (slot = home); 2: no prefix read (key from size); 3: prefix read only
template <int MODE>
__global__ void __launch_bounds__(256) k_insert(const uint8_t* arena, const uint64_t* off, const uint64_t* size,
                                                const uint64_t* chan, uint32_t n, uint64_t* tkey, uint64_t* key_out,
                                                uint32_t* slot_out, uint64_t cap_mask) {
    const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= n) return;
    const uint64_t sz = size[r];
    uint64_t pd = 0x5851F42D4C957F2Dull;
    if (MODE != 2) {
        B8 x = ld_stream(arena + off[r]);
#pragma unroll
        for (int i = 0; i < 8; i += 2) pd = fmix64(pd ^ ((uint64_t)x.v[i + 1] << 32 | x.v[i]));
    }
    const uint64_t key = fmix64(pd ^ fmix64(sz + 0x632BE59BD9B4E019ull) ^ fmix64(chan[r] ^ 0x2545F4914F6CDD1Dull));
    key_out[r] = key;
    if (MODE == 3) return;
    uint64_t h = key & cap_mask;
    if (MODE == 0) {
        const unsigned long long packed = ((unsigned long long)(uint32_t)(key >> 32) << 32) | r;
        while (true) {
            const unsigned long long prev = atomicCAS((unsigned long long*)&tkey[h], ~0ull, packed);
            if (prev == ~0ull) break;
            if ((prev >> 32) == (packed >> 32)) {
                if (packed < prev) atomicMin((unsigned long long*)&tkey[h], packed);
                break;
            }
            h = (h + 1) & cap_mask;
        }
    }
    slot_out[r] = (uint32_t)h;
}

int main() {
    const uint32_t n = 1000000, nsites = 256;
    std::mt19937_64 rng(0x5C19);
    std::vector<uint32_t> site_size(nsites);
    for (auto& s : site_size) {
        const double u = std::uniform_real_distribution<double>(0, 1)(rng);
        s = (uint32_t)std::exp(std::log(256.0) + u * (std::log(4096.0) - std::log(256.0)));
    }
    std::vector<double> w(nsites);
    for (uint32_t i = 0; i < nsites; ++i) w[i] = 1.0 / (i + 1);
    std::discrete_distribution<uint32_t> zipf(w.begin(), w.end());
    std::vector<uint64_t> off(n), size(n), chan(n, 0);
    std::vector<uint32_t> cur_content(nsites, 0);
    std::vector<uint64_t> content_of(n);
    uint64_t next_content = 1, cursor = 0;
    for (uint32_t i = 0; i < n; ++i) {
        const uint32_t s = zipf(rng);
        const bool reup = cur_content[s] && std::uniform_real_distribution<double>(0, 1)(rng) < 0.6;
        if (!reup) cur_content[s] = (uint32_t)next_content++;
        content_of[i] = cur_content[s];
        size[i] = site_size[s];
        off[i] = cursor;
        cursor += (size[i] + 31) / 32 * 32;
    }
    std::vector<uint8_t> arena(cursor + 64, 0);
    for (uint32_t i = 0; i < n; ++i) {   // the first 32 bytes identify the content
        const uint64_t c = content_of[i] * 0x9E3779B97F4A7C15ull;
        for (int b = 0; b < 32; ++b) arena[off[i] + b] = (uint8_t)(c >> (8 * (b & 7))) ^ (uint8_t)b;
    }
    uint8_t* d_arena;
    uint64_t *d_off, *d_size, *d_chan, *d_tkey, *d_key;
    uint32_t* d_slot;
    const uint64_t cap = 1ull << 21;
    cudaMalloc(&d_arena, arena.size());
    cudaMalloc(&d_off, 8ull * n);
    cudaMalloc(&d_size, 8ull * n);
    cudaMalloc(&d_chan, 8ull * n);
    cudaMalloc(&d_key, 8ull * n);
    cudaMalloc(&d_slot, 4ull * n);
    cudaMalloc(&d_tkey, 8 * cap);
    cudaMemcpy(d_arena, arena.data(), arena.size(), cudaMemcpyHostToDevice);
    cudaMemcpy(d_off, off.data(), 8ull * n, cudaMemcpyHostToDevice);
    cudaMemcpy(d_size, size.data(), 8ull * n, cudaMemcpyHostToDevice);
    cudaMemcpy(d_chan, chan.data(), 8ull * n, cudaMemcpyHostToDevice);
    uint8_t* flush;
    cudaMalloc(&flush, 512ull << 20);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto run = [&](const char* name, auto launch) {
        float best = 1e9f;
        for (int it = 0; it < 10; ++it) {
            cudaMemsetAsync(flush, it, 512ull << 20);   // arena out of L2, as after a small pass
            cudaMemsetAsync(d_tkey, 0xFF, 8 * cap);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = std::min(best, ms);
        }
        printf("{\"variant\": \"%s\", \"us\": %.1f, \"err\": \"%s\"}\n", name, best * 1e3,
               cudaGetErrorString(cudaGetLastError()));
    };
    const uint32_t grid = (n + 255) / 256;
    run("full", [&] { k_insert<0><<<grid, 256>>>(d_arena, d_off, d_size, d_chan, n, d_tkey, d_key, d_slot, cap - 1); });
    run("no_cas", [&] { k_insert<1><<<grid, 256>>>(d_arena, d_off, d_size, d_chan, n, d_tkey, d_key, d_slot, cap - 1); });
    run("no_prefix", [&] { k_insert<2><<<grid, 256>>>(d_arena, d_off, d_size, d_chan, n, d_tkey, d_key, d_slot, cap - 1); });
    run("prefix_only", [&] { k_insert<3><<<grid, 256>>>(d_arena, d_off, d_size, d_chan, n, d_tkey, d_key, d_slot, cap - 1); });
    return 0;
}
