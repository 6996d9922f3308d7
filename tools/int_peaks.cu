// Integer / DPX pipe throughput microbenchmark for sm_100a (B200).
// Defines the roofline denominator for the Smith-Waterman cell update
// (SURVEY.md §8(d)): measured warp-instructions / clock / SM for each
// instruction class the SW inner loop issues, plus the actual 6.5-op
// s16x2 cell mix used by the kernels.  Output: one JSON line.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peaks tools/int_peaks.cu -lnvidia-ml
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CHAINS 8
#define ITERS 4096

template <int OP>
__device__ __forceinline__ uint32_t op(uint32_t a, uint32_t b, uint32_t c) {
  if constexpr (OP == 0) return __viaddmax_s16x2(a, b, c);          // VIADDMNMX.S16x2
  if constexpr (OP == 1) return __vimax3_s16x2_relu(a, b, c);       // VIMNMX3.S16x2.RELU
  if constexpr (OP == 2) return __vmaxs2(a, c);                     // VIMNMX.S16x2
  if constexpr (OP == 3) return __vadd2(a, b);                      // VIADD.16x2
  if constexpr (OP == 4) return __byte_perm(a, c, 0xC480);          // PRMT
  if constexpr (OP == 5) return a + b + c;                          // IADD3
  if constexpr (OP == 6) return (uint32_t)max((int)a, (int)c);      // IMNMX
  if constexpr (OP == 7) return __viaddmax_s16x2_relu(a, b, c);     // VIADDMNMX.S16x2.RELU
  if constexpr (OP == 8) return (uint32_t)__viaddmax_s32((int)a, (int)b, (int)c);  // VIADDMNMX (s32)
  return a;
}

template <int OP>
__global__ void __launch_bounds__(512) k_peak(uint32_t* out, uint32_t seed, long long* cyc) {
  uint32_t v[CHAINS];
#pragma unroll
  for (int k = 0; k < CHAINS; ++k) v[k] = seed * (threadIdx.x + 1) + k;
  uint32_t b = seed ^ 0x00030003u, c = seed ^ 0x00070007u;
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int k = 0; k < CHAINS; ++k) v[k] = op<OP>(v[k], b, c ^ k);
  }
  long long t1 = clock64();
  uint32_t acc = 0;
#pragma unroll
  for (int k = 0; k < CHAINS; ++k) acc ^= v[k];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// The s16x2 Smith-Waterman cell mix exactly as the kernels issue it
// (per row: PRMT + VIADDMNMX x2 + VIMNMX + VIADDMNMX.RELU + VIADD + 0.5 VIMNMX3).
__global__ void __launch_bounds__(512) k_cellmix(uint32_t* out, uint32_t seed, long long* cyc) {
  constexpr int R = 16;
  uint32_t hr[R], e[R];
#pragma unroll
  for (int r = 0; r < R; ++r) { hr[r] = seed + r; e[r] = seed * 3 + r; }
  uint32_t best = 0, hrup0 = seed, f0 = seed * 7;
  const uint32_t nsig = 0xFFFEFFFEu, nrho = 0xFFF6FFF6u;
  uint32_t p0 = seed * 0x01010101u, p1 = seed * 0x02020202u;
  long long t0 = clock64();
  for (int it = 0; it < ITERS / 8; ++it) {
    uint32_t hrup = hrup0 ^ it, f = f0, hrdiag = hrup0;
    uint32_t hprev = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t w = __byte_perm(p0 + it, p1, 0xC480 + (r & 3) * 0x1111);
      e[r] = __viaddmax_s16x2(e[r], nsig, hr[r]);
      f = __viaddmax_s16x2(f, nsig, hrup);
      uint32_t ef = __vmaxs2(e[r], f);
      uint32_t h = __viaddmax_s16x2_relu(hrdiag, w, ef);
      hrdiag = hr[r];
      hr[r] = __vadd2(h, nrho);
      hrup = hr[r];
      if (r & 1) best = __vimax3_s16x2_relu(best, h, hprev); else hprev = h;
    }
    hrup0 = hrup; f0 = f;
  }
  long long t1 = clock64();
  uint32_t acc = best;
#pragma unroll
  for (int r = 0; r < R; ++r) acc ^= hr[r] ^ e[r];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <typename K>
static void run(const char* name, K kern, double instr_per_thread, int blocks, int threads, uint32_t* d_out,
                long long* d_cyc, int first) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  kern<<<blocks, threads>>>(d_out, 1u, d_cyc);
  cudaEventRecord(a);
  const int reps = 5;
  for (int i = 0; i < reps; ++i) kern<<<blocks, threads>>>(d_out, 1u + i, d_cyc);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0; cudaEventElapsedTime(&ms, a, b);
  long long h_cyc[4096];
  cudaMemcpy(h_cyc, d_cyc, sizeof(long long) * blocks, cudaMemcpyDeviceToHost);
  double mean_cyc = 0; for (int i = 0; i < blocks; ++i) mean_cyc += (double)h_cyc[i]; mean_cyc /= blocks;
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  double warps_per_sm = (double)blocks * threads / 32.0 / nsm;
  double warp_instr_per_clk_sm = warps_per_sm * instr_per_thread / mean_cyc;
  double thread_instr_per_s = (double)blocks * threads * instr_per_thread * reps / (ms * 1e-3);
  double clk_ghz = mean_cyc / ((ms * 1e-3) / reps) / 1e9;
  printf("%s\"%s\": {\"warp_instr_per_clk_per_sm\": %.3f, \"thread_instr_per_s\": %.4e, \"sm_clock_ghz_est\": %.3f}",
         first ? "" : ", ", name, warp_instr_per_clk_sm, thread_instr_per_s, clk_ghz);
}

int main() {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int threads = 512, blocks = nsm * 2;
  uint32_t* d_out; long long* d_cyc;
  cudaMalloc(&d_out, sizeof(uint32_t) * blocks * threads);
  cudaMalloc(&d_cyc, sizeof(long long) * blocks);
  const double ipt = (double)CHAINS * ITERS;
  printf("{\"sms\": %d, ", nsm);
  run("VIADDMNMX.S16x2", k_peak<0>, ipt, blocks, threads, d_out, d_cyc, 1);
  run("VIMNMX3.S16x2.RELU", k_peak<1>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("VIMNMX.S16x2", k_peak<2>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("VIADD.16x2", k_peak<3>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("PRMT", k_peak<4>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("IADD3", k_peak<5>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("IMNMX", k_peak<6>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("VIADDMNMX.S16x2.RELU", k_peak<7>, ipt, blocks, threads, d_out, d_cyc, 0);
  run("VIADDMNMX.S32", k_peak<8>, ipt, blocks, threads, d_out, d_cyc, 0);
  // cell mix: per iteration R=16 rows x 6.5 ops = 104 ALU ops / thread
  run("cellmix_s16x2_per_row6.5", k_cellmix, (ITERS / 8) * 16 * 6.5, blocks, threads, d_out, d_cyc, 0);
  printf("}\n");
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { fprintf(stderr, "CUDA error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
