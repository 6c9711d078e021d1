/*
 * loggen/fill.c -- seeded synthetic payload materialiser (input generator).
 *
 * Shared input infrastructure: both the CPU oracle (oracle/) and the CUDA
 * path are fed from the bytes this file produces.  It contains NONE of the
 * deduplication method's arithmetic (no hashing of payloads, no grouping,
 * no comparison): it only turns a content descriptor
 *     (kind, seed, size, base content, byte flips)
 * into bytes with a counter-based generator, so that every payload is a pure
 * function of its descriptor.
 *
 * Content kinds:
 *   0 RANDOM : 64-bit word i = mix64(seed ^ (i * 0xD1B54A32D192ED03)), little endian
 *   1 ZERO   : all bytes 0
 *   2 SMOOTH : word 0 as RANDOM (a unique 8-byte header); then float32 element
 *              k >= 2 is  (float)((int32)(A + k*B) >> 16) * 2^-10   -- a slowly
 *              varying, low-entropy field (memset/solver-array like data)
 *   any kind with base >= 0: start from the bytes of content `base` (same size),
 *              then xor byte flip_pos[j] with flip_xor[j] for the content's flips.
 */
#include <stdint.h>
#include <string.h>
#include <stdlib.h>
#include <omp.h>

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

static void fill_random(uint8_t* dst, uint64_t size, uint64_t seed, uint64_t w0, uint64_t w1) {
    /* words [w0, w1) */
    for (uint64_t i = w0; i < w1; ++i) {
        uint64_t w = mix64(seed ^ (i * 0xD1B54A32D192ED03ull));
        uint64_t at = i * 8;
        if (at + 8 <= size) memcpy(dst + at, &w, 8);
        else memcpy(dst + at, &w, size - at);
    }
}

static void fill_smooth(uint8_t* dst, uint64_t size, uint64_t seed, uint64_t e0, uint64_t e1) {
    /* float elements [e0, e1); elements 0,1 are the random header word */
    uint64_t h = mix64(seed ^ 0x5EEDull);
    uint32_t A = (uint32_t)h, B = 1u + (uint32_t)((h >> 32) % 4096u);
    for (uint64_t k = e0; k < e1; ++k) {
        uint64_t at = k * 4;
        uint32_t bits;
        if (k < 2) {
            uint64_t w = mix64(seed ^ 0ull);
            bits = (uint32_t)(w >> (32 * k));
        } else {
            int32_t v = (int32_t)(A + (uint32_t)k * B) >> 16;
            float f = (float)v * (1.0f / 1024.0f);
            memcpy(&bits, &f, 4);
        }
        if (at + 4 <= size) memcpy(dst + at, &bits, 4);
        else memcpy(dst + at, &bits, size - at);
    }
}

/* Fill one base (non-derived) content, parallel over 1 MiB pieces. */
static void fill_base(uint8_t* dst, uint64_t size, int32_t kind, uint64_t seed) {
    const uint64_t piece = 1ull << 20;
    uint64_t np = (size + piece - 1) / piece;
    #pragma omp parallel for schedule(dynamic, 1) if (np > 1)
    for (uint64_t p = 0; p < np; ++p) {
        uint64_t b0 = p * piece, b1 = b0 + piece < size ? b0 + piece : size;
        if (kind == 1) memset(dst + b0, 0, b1 - b0);
        else if (kind == 2) fill_smooth(dst, size, seed, b0 / 4, (b1 + 3) / 4);
        else fill_random(dst, size, seed, b0 / 8, (b1 + 7) / 8);
    }
}

/*
 * Materialise contents [0, m) into out (content c at out + off[c]).
 * Derived contents must have base < c.  Returns 0 or -1 on bad input.
 */
int loggen_materialize(int64_t m, const int32_t* kind, const uint64_t* seed,
                       const uint64_t* size, const int64_t* base,
                       const int64_t* flip_start, const uint64_t* flip_pos,
                       const uint8_t* flip_xor, const uint64_t* off,
                       uint8_t* out, int nthreads) {
    if (nthreads > 0) omp_set_num_threads(nthreads);
    /* pass 1: base contents.  Small ones in parallel across contents, large ones
       parallel inside. */
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t c = 0; c < m; ++c) {
        if (base[c] >= 0 || size[c] > (1ull << 20)) continue;
        uint8_t* d = out + off[c];
        if (kind[c] == 1) memset(d, 0, size[c]);
        else if (kind[c] == 2) fill_smooth(d, size[c], seed[c], 0, (size[c] + 3) / 4);
        else fill_random(d, size[c], seed[c], 0, (size[c] + 7) / 8);
    }
    for (int64_t c = 0; c < m; ++c)
        if (base[c] < 0 && size[c] > (1ull << 20)) fill_base(out + off[c], size[c], kind[c], seed[c]);
    /* pass 2: derived contents in id order (base < c), copy + flips */
    for (int64_t c = 0; c < m; ++c) {
        int64_t b = base[c];
        if (b < 0 || size[c] == 0) continue;     /* size 0: not materialised (subset) */
        if (b >= c || size[b] != size[c]) return -1;
        uint8_t* d = out + off[c];
        const uint8_t* s = out + off[b];
        uint64_t n = size[c];
        const uint64_t piece = 1ull << 22;
        uint64_t np = (n + piece - 1) / piece;
        #pragma omp parallel for schedule(static) if (np > 1)
        for (uint64_t p = 0; p < np; ++p) {
            uint64_t b0 = p * piece, len = b0 + piece < n ? piece : n - b0;
            memcpy(d + b0, s + b0, len);
        }
        for (int64_t j = flip_start[c]; j < flip_start[c + 1]; ++j) {
            if (flip_pos[j] >= n) return -1;
            d[flip_pos[j]] ^= flip_xor[j];
        }
    }
    return 0;
}
