// Integer / DPX pipe throughput microbenchmark for sm_100a (B200).
// Defines the roofline denominator for the Smith-Waterman cell update
// (SURVEY.md §8(d)): measured warp-instructions / clock / SM for each
// instruction class the SW inner loop issues, plus the actual 6.5-op
// s16x2 cell mix used by the kernels.  Output: one JSON line.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peaks tools/int_peaks.cu -lnvidia-ml
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <cuda_runtime.h>

#define CHAINS 8
#define ITERS 4096

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

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
  unsigned long long g0 = gtimer();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int k = 0; k < CHAINS; ++k) v[k] = op<OP>(v[k], b, c ^ k);
  }
  long long t1 = clock64();
  unsigned long long g1 = gtimer();
  uint32_t acc = 0;
#pragma unroll
  for (int k = 0; k < CHAINS; ++k) acc ^= v[k];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) { cyc[2 * blockIdx.x] = t1 - t0; cyc[2 * blockIdx.x + 1] = (long long)(g1 - g0); }
}

// The s16x2 Smith-Waterman cell update exactly as sw_engine.cuh issues it (per row: PRMT +
// VIADDMNMX x2 + VIMNMX + VIADDMNMX.RELU + VIADD + 0.5 VIMNMX3), profile words varying per
// column, no memory traffic: the ALU speed of light of the engine's arithmetic.
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt_imm(uint32_t a, uint32_t b) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "n"(SEL));
  return d;
}
constexpr int CM_R = 16;
__global__ void __launch_bounds__(512) k_cellmix(uint32_t* out, uint32_t seed, long long* cyc) {
  constexpr int R = CM_R;
  uint32_t hr[R], e[R];
#pragma unroll
  for (int r = 0; r < R; ++r) { hr[r] = 0xFFF6FFF6u; e[r] = 0xFFF6FFF6u; }
  uint32_t best = 0, hrup0 = 0xFFF6FFF6u, f0 = 0xFFF6FFF6u, hrdiag0 = 0xFFF6FFF6u;
  const uint32_t nsig = 0xFFFEFFFEu, nrho = 0xFFF6FFF6u;
  // profile rows in shared memory, read with LDS.128 exactly like the engine (25 letters)
  __shared__ __align__(16) uint32_t sprof[25 * R];
  for (int i = threadIdx.x; i < 25 * R; i += blockDim.x) sprof[i] = (seed + i) * 0x01010101u;
  __syncthreads();
  uint32_t res = threadIdx.x * 7u + seed;
  long long t0 = clock64();
  unsigned long long g0 = gtimer();
  for (int it = 0; it < ITERS / 8; ++it) {
    uint32_t wlo[R / 4], whi[R / 4];
    const uint4* plo = reinterpret_cast<const uint4*>(sprof + (res & 15) * R);
    const uint4* phi = reinterpret_cast<const uint4*>(sprof + ((res >> 4) & 15) * R);
#pragma unroll
    for (int k = 0; k < R / 16; ++k) {
      const uint4 a = plo[k], b = phi[k];
      wlo[4 * k] = a.x; wlo[4 * k + 1] = a.y; wlo[4 * k + 2] = a.z; wlo[4 * k + 3] = a.w;
      whi[4 * k] = b.x; whi[4 * k + 1] = b.y; whi[4 * k + 2] = b.z; whi[4 * k + 3] = b.w;
    }
    res = res * 0x9E37u + 0x79B9u;
    uint32_t hrup = hrup0, f = f0, hrdiag = hrdiag0, hprev = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t w;
      switch (r & 3) {
        case 0: w = prmt_imm<0xC480u>(wlo[r >> 2], whi[r >> 2]); break;
        case 1: w = prmt_imm<0xD591u>(wlo[r >> 2], whi[r >> 2]); break;
        case 2: w = prmt_imm<0xE6A2u>(wlo[r >> 2], whi[r >> 2]); break;
        default: w = prmt_imm<0xF7B3u>(wlo[r >> 2], whi[r >> 2]); break;
      }
      e[r] = __viaddmax_s16x2(e[r], nsig, hr[r]);
      f = __viaddmax_s16x2(f, nsig, hrup);
      const uint32_t ef = __vmaxs2(e[r], f);
      const uint32_t h = __viaddmax_s16x2_relu(hrdiag, w, ef);
      hrdiag = hr[r];
      hr[r] = __vadd2(h, nrho);
      hrup = hr[r];
      if (r & 1) best = __vimax3_s16x2(best, hprev, h); else hprev = h;
    }
    hrdiag0 = hrup0; hrup0 = hrup ^ (uint32_t)it; f0 = f;
  }
  long long t1 = clock64();
  unsigned long long g1 = gtimer();
  uint32_t acc = best;
#pragma unroll
  for (int r = 0; r < R; ++r) acc ^= hr[r] ^ e[r];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) { cyc[2 * blockIdx.x] = t1 - t0; cyc[2 * blockIdx.x + 1] = (long long)(g1 - g0); }
}

static double g_last_rate = 0, g_last_clk = 0;
// Rate in warp-instructions per SM clock: all blocks resident (one wave), per-block SM cycles
// from clock64 and wall time from %globaltimer give the clock the kernel actually ran at; the
// GPU is warmed up for ~1.5 s first so the clock has ramped (an earlier version of this tool
// measured a cold GPU and under-estimated the clock).
template <typename K>
static void run(const char* name, K kern, double instr_per_thread, int blocks, int threads, uint32_t* d_out,
                long long* d_cyc, int first) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  int warm = 0;
  for (;;) {
    kern<<<blocks, threads>>>(d_out, 1u + warm, d_cyc);
    ++warm;
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0; cudaEventElapsedTime(&ms, a, b);
    if (ms > 1500.f || warm > 20000) break;
  }
  const int reps = 20;
  double sum_rate = 0, sum_clk = 0;
  for (int i = 0; i < reps; ++i) {
    kern<<<blocks, threads>>>(d_out, 7u + i, d_cyc);
    static long long h_cyc[2 * 8192];
    cudaMemcpy(h_cyc, d_cyc, sizeof(long long) * 2 * blocks, cudaMemcpyDeviceToHost);
    double cyc = 0, ns = 0;
    for (int k = 0; k < blocks; ++k) { cyc += (double)h_cyc[2 * k]; ns += (double)h_cyc[2 * k + 1]; }
    const double clk_ghz = cyc / ns;                 // SM cycles per ns inside the timed loop
    int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const double warps_per_sm = (double)blocks * threads / 32.0 / nsm;
    sum_rate += warps_per_sm * instr_per_thread / (cyc / blocks);
    sum_clk += clk_ghz;
  }
  const double rate = sum_rate / reps, clk = sum_clk / reps;
  g_last_rate = rate; g_last_clk = clk;
  printf("%s\"%s\": {\"warp_instr_per_clk_per_sm\": %.3f, \"sm_clock_ghz\": %.3f}", first ? "" : ", ", name, rate, clk);
}

int main() {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int threads = 512;
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_cellmix, threads, 0);
  const int blocks = nsm * std::max(1, std::min(occ, 2));   // one resident wave
  uint32_t* d_out; long long* d_cyc;
  cudaMalloc(&d_out, sizeof(uint32_t) * blocks * threads);
  cudaMalloc(&d_cyc, sizeof(long long) * 2 * blocks);
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
  // cell mix, counted in CELLS: per iteration R rows x 2 cells (two sequences per s16x2 lane)
  run("cellmix_cells", k_cellmix, (ITERS / 8) * CM_R * 2.0, blocks, threads, d_out, d_cyc, 0);
  // g_last_rate is "warp-cells" per clk per SM -> x32 lanes x SMs = cells per clk per GPU
  printf(", \"cells_per_clk_per_gpu\": %.2f, \"sm_mhz_during\": %.0f, \"what\": \"cells_per_clk_per_gpu = measured rate "
         "of the engine's per-cell instruction mix (PRMT + 5 DPX + 0.5 VIMNMX3 per 2 cells, profile from smem), no "
         "boundary traffic; the DPX ops issue at the rate measured for VIADDMNMX.S16x2 above\"}\n",
         g_last_rate * 32.0 * nsm, g_last_clk * 1e3);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { fprintf(stderr, "CUDA error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
