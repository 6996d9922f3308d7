// Integer / DPX pipe throughput microbenchmark for sm_100a (B200).
// Defines the roofline denominator for the Smith-Waterman cell update (SURVEY.md §8(d),
// DESIGN.md §5): measured warp-instructions / clock / SM for each instruction class the SW
// inner loop issues, pairs of classes (which ones share a pipe), and the engine's exact s16x2
// cell mix.  Output: one JSON line (MEASURED_INT_PEAKS.json).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/int_peaks tools/int_peaks.cu
//
// Timing: every block records (smid, clock64 at start, clock64 at end) around its loop, with a
// __syncthreads on both sides so the window covers all of its warps.  The rate of an SM is
// (warp-instructions executed by all blocks on that SM) / (max end - min start over those
// blocks): the SM-cycle window in which its warps actually ran, whatever the co-residency.
// (The first version of this tool divided each block's own window into an assumed
// co-resident warp count, which over-stated every rate by ~1.33x when the two blocks of an SM
// did not overlap completely: ncu measured 92 % ALU-pipe activity for the cell mix at a rate
// 0.75x of what that version reported.)  Each op's operands come from other chains, and the
// ops are asm volatile, so nothing folds.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#define CHAINS 8
#define ITERS 2048

struct Rec { long long t0, t1; unsigned long long g0, g1; unsigned smid; unsigned pad; };

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned smid() {
  unsigned s;
  asm volatile("mov.u32 %0, %smid;" : "=r"(s));
  return s;
}

// one instruction of class OP (asm volatile: never folded, never hoisted)
template <int OP>
__device__ __forceinline__ uint32_t op(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  if constexpr (OP == 2) asm volatile("prmt.b32 %0, %1, %2, 0xC480;" : "=r"(d) : "r"(a), "r"(c));
  if constexpr (OP == 3) asm volatile("add.s32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(c));
  if constexpr (OP == 4) asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  if constexpr (OP == 5) asm volatile("max.s32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(c));
  if constexpr (OP == 6) asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  if constexpr (OP == 7) asm volatile("max.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(c));
  if constexpr (OP == 8) asm volatile("max.bf16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(c));
  return d;
}
// DPX classes through the intrinsics (ptxas emits one SASS op each); volatile via a barrier
// on the result so the compiler keeps every one.
template <int OP>
__device__ __forceinline__ uint32_t dpx(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  if constexpr (OP == 10) d = __viaddmax_s16x2(a, b, c);          // VIADDMNMX.S16x2
  if constexpr (OP == 11) d = __viaddmax_s16x2_relu(a, b, c);     // VIADDMNMX.S16x2.RELU
  if constexpr (OP == 12) d = __vimax3_s16x2(a, b, c);            // VIMNMX3.S16x2
  if constexpr (OP == 13) d = __vmaxs2(a, c);                     // VIMNMX.S16x2
  if constexpr (OP == 14) d = __vadd2(a, b);                      // VIADD.16x2 (HADD2-class?)
  if constexpr (OP == 15) d = (uint32_t)__viaddmax_s32((int)a, (int)b, (int)c);
  if constexpr (OP < 10) d = op<OP>(a, b, c);
  asm volatile("" : "+r"(d));
  return d;
}

// OPA on every chain; if OPB >= 0, chains alternate OPA / OPB (pipe-sharing test)
template <int OPA, int OPB>
__global__ void __launch_bounds__(512) k_peak(uint32_t* out, uint32_t seed, Rec* rec) {
  uint32_t v[CHAINS];
#pragma unroll
  for (int k = 0; k < CHAINS; ++k) v[k] = seed * (threadIdx.x + 1) + k * 0x00010003u;
  const uint32_t b = seed ^ 0xFFFEFFFEu;
  __syncthreads();
  long long t0 = clock64();
  unsigned long long g0 = gtimer();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int k = 0; k < CHAINS; ++k) {
      const uint32_t c = v[(k + 1) % CHAINS];
      if (OPB < 0 || (k & 1) == 0) v[k] = dpx<OPA>(v[k], b, c);
      else v[k] = dpx<(OPB < 0 ? OPA : OPB)>(v[k], b, c);
    }
  }
  __syncthreads();
  long long t1 = clock64();
  unsigned long long g1 = gtimer();
  uint32_t acc = 0;
#pragma unroll
  for (int k = 0; k < CHAINS; ++k) acc ^= v[k];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) rec[blockIdx.x] = Rec{t0, t1, g0, g1, smid(), 0};
}

// The s16x2 Smith-Waterman cell update exactly as sw_engine.cuh's cell_rows issues it, per row:
//   f    = VIADDMNMX(f, -sigma, hr_up)
//   h    = VIMNMX3.RELU(t, e, f)
//   hr   = VIADD.16x2(h, -rho)                 (FMA pipe)
//   e    = VIADDMNMX(e, -sigma, hr)
//   t    = VIADD.16x2(hr_up, w + rho)          (FMA pipe)
//   w    = PRMT(profile_lo, profile_hi)        (sign-extend two int8 scores)
//   best = VIMNMX3(best, h, h') every two rows
// = 4.5 ALU-pipe + 2 FMA-pipe instructions per two cells; the profile words come from shared
// memory (LDS.128, R/16 x 2 per column as in the engine) at a letter that changes every column.
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt_imm(uint32_t a, uint32_t b) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "n"(SEL));
  return d;
}
constexpr int CM_R = 32;
constexpr int CM_COLS = 256;
// SH = 1: the engine's step boundary as well (lane chain: (H, F + rho) and the residue pair
// arrive by __shfl_up_sync, lane 0 takes them from the stream, the profile address depends
// on the shuffled residues)
template <int R, int NT, int SH = 0>
__global__ void __launch_bounds__(NT) k_cellmix(uint32_t* out, uint32_t seed, Rec* rec) {
  uint32_t t[R], e[R];
  const uint32_t nsig = 0xFFFEFFFEu, nrho = 0xFFF6FFF6u, prho = 0x000A000Au;
#pragma unroll
  for (int r = 0; r < R; ++r) { t[r] = 0u; e[r] = nrho; }
  uint32_t best = 0, hup0 = 0, fs0 = 0;
  // profile: 16 letters x R rows of int8, per-lane copy so the LDS.128 are conflict-free
  __shared__ __align__(16) uint8_t sprof[16 * R * 32];
  for (int i = threadIdx.x; i < 16 * R * 32; i += blockDim.x) sprof[i] = (uint8_t)((seed + i * 37u) % 23u);
  // the residue stream (two letters per column), in shared memory like a staged DB tile
  __shared__ uint8_t sres[CM_COLS];
  for (int i = threadIdx.x; i < CM_COLS; i += blockDim.x) sres[i] = (uint8_t)((i * 0x9Du + seed) & 0xffu);
  __syncthreads();
  const int lane = threadIdx.x & 31;
  long long t0 = clock64();
  unsigned long long g0 = gtimer();
  uint32_t y_res = 0;
  for (int col = 0; col < ITERS / 4; ++col) {
    uint32_t res = sres[col & (CM_COLS - 1)];
    if constexpr (SH) {
      uint32_t x_hr = __shfl_up_sync(0xffffffffu, hup0, 1), x_f = __shfl_up_sync(0xffffffffu, fs0, 1);
      uint32_t x_res = __shfl_up_sync(0xffffffffu, y_res, 1);
      if (lane == 0) { x_hr = 0u; x_f = 0u; x_res = res; }
      hup0 = x_hr; fs0 = x_f; y_res = x_res; res = x_res;
    }
    const uint4* plo = reinterpret_cast<const uint4*>(sprof + ((res & 15) * R * 32)) + lane;
    const uint4* phi = reinterpret_cast<const uint4*>(sprof + ((res >> 4) * R * 32)) + lane;
    uint32_t wlo[R / 4], whi[R / 4];
#pragma unroll
    for (int k = 0; k < R / 16; ++k) {
      const uint4 a = plo[k * 32], bb = phi[k * 32];
      wlo[4 * k] = a.x; wlo[4 * k + 1] = a.y; wlo[4 * k + 2] = a.z; wlo[4 * k + 3] = a.w;
      whi[4 * k] = bb.x; whi[4 * k + 1] = bb.y; whi[4 * k + 2] = bb.z; whi[4 * k + 3] = bb.w;
    }
    // the engine's cell update (sw_engine.cuh cell_rows): F, H = max3.relu(T, E, F), H - rho,
    // E, T of the next column, best every two rows
    uint32_t hrup = __vadd2(hup0, nrho), f = __vadd2(fs0, nrho), hprev = 0, h = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t w;
      switch (r & 3) {
        case 0: w = prmt_imm<0xC480u>(wlo[r >> 2], whi[r >> 2]); break;
        case 1: w = prmt_imm<0xD591u>(wlo[r >> 2], whi[r >> 2]); break;
        case 2: w = prmt_imm<0xE6A2u>(wlo[r >> 2], whi[r >> 2]); break;
        default: w = prmt_imm<0xF7B3u>(wlo[r >> 2], whi[r >> 2]); break;
      }
      f = __viaddmax_s16x2(f, nsig, hrup);
      h = __vimax3_s16x2_relu(t[r], e[r], f);
      const uint32_t hr = __vadd2(h, nrho);
      e[r] = __viaddmax_s16x2(e[r], nsig, hr);
      t[r] = __vadd2(hrup, w);
      hrup = hr;
      if (r & 1) best = __vimax3_s16x2(best, hprev, h); else hprev = h;
    }
    // the next column's top input: this lane's bottom row (a chain of one lane)
    hup0 = h; fs0 = __vadd2(f, prho);
  }
  __syncthreads();
  long long t1 = clock64();
  unsigned long long g1 = gtimer();
  uint32_t acc = best;
#pragma unroll
  for (int r = 0; r < R; ++r) acc ^= t[r] ^ e[r];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) rec[blockIdx.x] = Rec{t0, t1, g0, g1, smid(), 0};
}

static double g_rate = 0, g_clk = 0;
// work_per_thread: instructions (or cells) per thread of the timed loop
template <typename K>
static void run(const char* name, K kern, double work_per_thread, int threads, uint32_t* d_out, Rec* d_rec,
                bool first) {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, threads, 0);
  occ = std::max(1, std::min(occ, 4));
  const int blocks = nsm * occ;                       // one resident wave
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  for (int warm = 0;; ++warm) {                       // ~1 s warm-up so the clock has ramped
    kern<<<blocks, threads>>>(d_out, 1u + warm, d_rec);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0; cudaEventElapsedTime(&ms, a, b);
    if (ms > 1000.f || warm > 20000) break;
  }
  const int reps = 10;
  std::vector<Rec> h(blocks);
  double sum_rate = 0, sum_clk = 0;
  for (int i = 0; i < reps; ++i) {
    kern<<<blocks, threads>>>(d_out, 7u + i, d_rec);
    cudaMemcpy(h.data(), d_rec, sizeof(Rec) * blocks, cudaMemcpyDeviceToHost);
    std::vector<long long> lo(nsm, INT64_MAX), hi(nsm, INT64_MIN);
    std::vector<unsigned long long> glo(nsm, UINT64_MAX), ghi(nsm, 0);
    std::vector<int> nb(nsm, 0);
    for (auto& r : h) {
      if (r.smid >= (unsigned)nsm) continue;
      lo[r.smid] = std::min(lo[r.smid], r.t0); hi[r.smid] = std::max(hi[r.smid], r.t1);
      glo[r.smid] = std::min(glo[r.smid], r.g0); ghi[r.smid] = std::max(ghi[r.smid], r.g1);
      nb[r.smid]++;
    }
    double rate = 0, clk = 0; int used = 0;
    for (int s = 0; s < nsm; ++s) {
      if (!nb[s]) continue;
      const double cyc = (double)(hi[s] - lo[s]);
      rate += nb[s] * (threads / 32.0) * work_per_thread / cyc;
      clk += cyc / (double)(ghi[s] - glo[s]);
      ++used;
    }
    sum_rate += rate / used; sum_clk += clk / used;
  }
  g_rate = sum_rate / reps; g_clk = sum_clk / reps;
  printf("%s\"%s\": {\"warp_instr_per_clk_per_sm\": %.3f, \"sm_clock_ghz\": %.3f, \"blocks_per_sm\": %d}",
         first ? "" : ", ", name, g_rate, g_clk, occ);
  fflush(stdout);
}

int main() {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int threads = 512;
  uint32_t* d_out; Rec* d_rec;
  cudaMalloc(&d_out, sizeof(uint32_t) * nsm * 4 * threads);
  cudaMalloc(&d_rec, sizeof(Rec) * nsm * 4);
  const double ipt = (double)CHAINS * ITERS;
  printf("{\"sms\": %d, ", nsm);
  run("VIADDMNMX.S16x2", k_peak<10, -1>, ipt, threads, d_out, d_rec, true);
  run("VIADDMNMX.S16x2.RELU", k_peak<11, -1>, ipt, threads, d_out, d_rec, false);
  run("VIMNMX3.S16x2", k_peak<12, -1>, ipt, threads, d_out, d_rec, false);
  run("VIMNMX.S16x2", k_peak<13, -1>, ipt, threads, d_out, d_rec, false);
  run("VIADD.16x2", k_peak<14, -1>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX.S32", k_peak<15, -1>, ipt, threads, d_out, d_rec, false);
  run("PRMT", k_peak<2, -1>, ipt, threads, d_out, d_rec, false);
  run("IADD3", k_peak<3, -1>, ipt, threads, d_out, d_rec, false);
  run("LOP3", k_peak<4, -1>, ipt, threads, d_out, d_rec, false);
  run("IMNMX", k_peak<5, -1>, ipt, threads, d_out, d_rec, false);
  run("IMAD", k_peak<6, -1>, ipt, threads, d_out, d_rec, false);
  // pipe sharing: the pair's combined rate is ~1 pipe's rate if both go to the same pipe
  run("VIADDMNMX+PRMT", k_peak<10, 2>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX+VIADD.16x2", k_peak<10, 14>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX+IMAD", k_peak<10, 6>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX+IADD3", k_peak<10, 3>, ipt, threads, d_out, d_rec, false);
  run("HMNMX2", k_peak<7, -1>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX+HMNMX2", k_peak<10, 7>, ipt, threads, d_out, d_rec, false);
  run("VIADDMNMX+HMNMX2.BF16", k_peak<10, 8>, ipt, threads, d_out, d_rec, false);
  // the cell mix, counted in CELLS: per column R rows x 2 cells (two sequences per s16x2 lane)
  run("cellmix_cells", k_cellmix<CM_R, 512>, (ITERS / 4) * CM_R * 2.0, threads, d_out, d_rec, false);
  const double mix_rate = g_rate;
  // the same mix at 3 warps per scheduler (the engine's 384-thread configurations), R = 32 / 48
  run("cellmix_cells_R32_384", k_cellmix<32, 384>, (ITERS / 4) * 32 * 2.0, 384, d_out, d_rec, false);
  run("cellmix_cells_R48_384", k_cellmix<48, 384>, (ITERS / 4) * 48 * 2.0, 384, d_out, d_rec, false);
  run("cellmix_shfl_R48_384", k_cellmix<48, 384, 1>, (ITERS / 4) * 48 * 2.0, 384, d_out, d_rec, false);
  run("cellmix_shfl_R32_512", k_cellmix<32, 512, 1>, (ITERS / 4) * 32 * 2.0, 512, d_out, d_rec, false);
  g_rate = mix_rate;
  printf(", \"cells_per_clk_per_gpu\": %.2f, \"sm_mhz_during\": %.0f, \"what\": \"rates = warp-instructions (cellmix: "
         "warp-cells) per SM clock over the per-SM window in which the blocks ran; cells_per_clk_per_gpu = 32 lanes x "
         "SMs x the cell-mix rate (per 2 cells: PRMT + 2 VIADDMNMX + VIMNMX3.RELU + 0.5 VIMNMX3 on the ALU pipe, 2 VIADD.16x2 on the FMA pipe; profile from smem via LDS.128)\"}\n",
         g_rate * 32.0 * nsm, g_clk * 1e3);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { fprintf(stderr, "CUDA error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
