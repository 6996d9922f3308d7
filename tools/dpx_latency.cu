// Dependent-chain latency of the DPX / integer ops used by the SW cell update (1 warp, 1 SM).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/dpx_latency tools/dpx_latency.cu
#include <cstdio>
#include <cstdint>
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b) {
  uint32_t d;
  asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "n"(SEL));
  return d;
}
template <int OP>
__global__ void k(uint32_t* out, uint32_t s, long long* cyc) {
  uint32_t v = s + threadIdx.x, b = s ^ 0x30003u, c = s * 7u;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < 4096; ++i) {
    if constexpr (OP == 0) v = __viaddmax_s16x2(v, b, c);
    if constexpr (OP == 1) v = __viaddmax_s16x2_relu(v, b, c);
    if constexpr (OP == 2) v = __vimax3_s16x2(v, b, c ^ i);
    if constexpr (OP == 3) v = __vadd2(v, b);
    if constexpr (OP == 4) v = prmt<0xC480u>(v, b);
    if constexpr (OP == 5) { v = __viaddmax_s16x2(v, b, c); v = __viaddmax_s16x2(v, c, b); }  // the fs -> h chain
  }
  long long t1 = clock64();
  if (v == 0x12345678u) out[threadIdx.x] = v;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
template <int OP>
void run(const char* name, uint32_t* d, long long* c) {
  k<OP><<<1, 32>>>(d, 1, c);
  k<OP><<<1, 32>>>(d, 2, c);
  long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
  printf("%s: %.2f cycles per dependent op\n", name, (double)h / (OP == 5 ? 8192.0 : 4096.0));
}
int main() {
  uint32_t* d; long long* c;
  cudaMalloc(&d, 128); cudaMalloc(&c, 8);
  run<0>("VIADDMNMX.S16x2", d, c);
  run<1>("VIADDMNMX.S16x2.RELU", d, c);
  run<2>("VIMNMX3.S16x2", d, c);
  run<3>("VIADD.16x2", d, c);
  run<4>("PRMT", d, c);
  run<5>("VIADDMNMX chain (fs->h)", d, c);
  return 0;
}
