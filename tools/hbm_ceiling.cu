// hbm_ceiling.cu -- practical HBM read-stream and copy ceilings on this B200
// (SURVEY.md 7 step 1).  Read: 256-bit LDG over a buffer >> L2, xor-reduced.
// Copy: 256-bit LDG + STG.  Best of 10, CUDA events.  Not part of the product.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

struct B { uint32_t v[8]; };
__device__ __forceinline__ B ld(const void* p) {
  B r; asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
    : "=r"(r.v[0]),"=r"(r.v[1]),"=r"(r.v[2]),"=r"(r.v[3]),"=r"(r.v[4]),"=r"(r.v[5]),"=r"(r.v[6]),"=r"(r.v[7]) : "l"(p));
  return r; }
template <int U>
__global__ void __launch_bounds__(256) rd(const uint8_t* p, uint64_t nblk, uint32_t* out) {
  uint32_t acc = 0;
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b < nblk; b += stride * U) {
    B x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { uint64_t bb = b + u * stride; x[u] = bb < nblk ? ld(p + 32 * bb) : B{}; }
#pragma unroll
    for (int u = 0; u < U; ++u) for (int i = 0; i < 8; ++i) acc ^= x[u].v[i];
  }
  if (acc == 0x12345678u) out[0] = acc;
}
__global__ void cp(const uint4* a, uint4* b, uint64_t n) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) b[i] = a[i];
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint64_t bytes = 32ull << 30;
  uint8_t* p; uint32_t* o;
  if (cudaMalloc(&p, bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMalloc(&o, 4); cudaMemset(p, 1, bytes);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int occ : {4, 8}) {
    float best = 1e9;
    for (int it = 0; it < 10; ++it) {
      cudaEventRecord(e0); rd<4><<<sms * occ, 256>>>(p, bytes / 32, o); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; }
    printf("{\"test\": \"read_stream_256b\", \"blocks_per_sm\": %d, \"gbs\": %.1f, \"bytes\": %llu}\n", occ, bytes / (best * 1e-3) / 1e9, (unsigned long long)bytes);
  }
  uint64_t half = bytes / 2;
  float best = 1e9;
  for (int it = 0; it < 10; ++it) {
    cudaEventRecord(e0); cp<<<sms * 8, 256>>>((const uint4*)p, (uint4*)(p + half), half / 16); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; }
  printf("{\"test\": \"copy_128b\", \"gbs_read_plus_write\": %.1f, \"bytes_each_way\": %llu}\n", 2.0 * half / (best * 1e-3) / 1e9, (unsigned long long)half);
  return 0;
}
