// Cell-mix probe: one column per step (the engine's cell_rows) vs two columns per step with a
// one-row skew (two independent vertical chains per warp), both with the engine's step boundary
// (lane chain by __shfl_up_sync, lane-0 select, profile words by LDS.128 at shuffled letters).
// Reports cells/clk/GPU (per-SM clock64 windows) against the derived ALU-pipe bound 4209.8.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/chain_probe tools/chain_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <climits>

struct Rec { long long t0, t1; unsigned smid; };
__device__ __forceinline__ unsigned smid() { unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s)); return s; }
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "n"(SEL));
  return d;
}
template <int R>
__device__ __forceinline__ uint32_t wrow(const uint32_t (&lo)[R / 4], const uint32_t (&hi)[R / 4], int r) {
  switch (r & 3) {
    case 0: return prmt<0xC480u>(lo[r >> 2], hi[r >> 2]);
    case 1: return prmt<0xD591u>(lo[r >> 2], hi[r >> 2]);
    case 2: return prmt<0xE6A2u>(lo[r >> 2], hi[r >> 2]);
    default: return prmt<0xF7B3u>(lo[r >> 2], hi[r >> 2]);
  }
}
constexpr int COLS = 4096;
constexpr int RES = 256;

template <int R>
__device__ __forceinline__ void loadw(uint32_t (&lo)[R / 4], uint32_t (&hi)[R / 4], const uint8_t* sprof, uint32_t res,
                                      int lane) {
  const uint4* plo = reinterpret_cast<const uint4*>(sprof + ((res & 15) * R * 32)) + lane;
  const uint4* phi = reinterpret_cast<const uint4*>(sprof + (((res >> 8) & 15) * R * 32)) + lane;
#pragma unroll
  for (int k = 0; k < R / 16; ++k) {
    const uint4 a = plo[k * 32], b = phi[k * 32];
    lo[4 * k] = a.x; lo[4 * k + 1] = a.y; lo[4 * k + 2] = a.z; lo[4 * k + 3] = a.w;
    hi[4 * k] = b.x; hi[4 * k + 1] = b.y; hi[4 * k + 2] = b.z; hi[4 * k + 3] = b.w;
  }
}

// TWO = 0: one column per step (R rows); TWO = 1: columns A, B per step with a one-row skew
template <int R, int NT, int TWO>
__global__ void __launch_bounds__(NT, 1) k_probe(uint32_t* out, uint32_t seed, Rec* rec) {
  __shared__ __align__(16) uint8_t sprof[16 * R * 32];
  __shared__ uint16_t sres[RES];
  for (int i = threadIdx.x; i < 16 * R * 32; i += blockDim.x) sprof[i] = (uint8_t)((seed + i * 37u) % 23u);
  for (int i = threadIdx.x; i < RES; i += blockDim.x) sres[i] = (uint16_t)((i * 0x9Du + seed) & 0x0f0fu);
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const uint32_t nsig = 0xFFFEFFFEu, nrho = 0xFFF6FFF6u, prho = 0x000A000Au;
  uint32_t t[R], e[R];
#pragma unroll
  for (int r = 0; r < R; ++r) { t[r] = 0u; e[r] = nrho; }
  uint32_t best = 0;
  uint32_t yA_h = 0, yA_f = 0, yA_r = 0, yB_h = 0, yB_f = 0, yB_r = 0;
  long long t0 = clock64();
  for (int col = 0; col < COLS; col += 1 + TWO) {
    if constexpr (!TWO) {
      uint32_t xh = __shfl_up_sync(~0u, yA_h, 1), xf = __shfl_up_sync(~0u, yA_f, 1), xr = __shfl_up_sync(~0u, yA_r, 1);
      if (lane == 0) { xh = 0; xf = 0; xr = sres[col & (RES - 1)]; }
      uint32_t lo[R / 4], hi[R / 4];
      loadw<R>(lo, hi, sprof, xr, lane);
      uint32_t hrup = __vadd2(xh, nrho), f = __vadd2(xf, nrho), hprev = 0, h = 0;
#pragma unroll
      for (int r = 0; r < R; ++r) {
        f = __viaddmax_s16x2(f, nsig, hrup);
        h = __vimax3_s16x2_relu(t[r], e[r], f);
        const uint32_t hr = __vadd2(h, nrho);
        e[r] = __viaddmax_s16x2(e[r], nsig, hr);
        t[r] = __vadd2(hrup, wrow<R>(lo, hi, r));
        hrup = hr;
        if (r & 1) best = __vimax3_s16x2(best, hprev, h); else hprev = h;
      }
      yA_h = h; yA_f = __vadd2(f, prho); yA_r = xr;
      asm volatile("" : "+r"(yA_r) : "r"(yA_f));
    } else {
      uint32_t xAh = __shfl_up_sync(~0u, yA_h, 1), xAf = __shfl_up_sync(~0u, yA_f, 1), xAr = __shfl_up_sync(~0u, yA_r, 1);
      uint32_t xBh = __shfl_up_sync(~0u, yB_h, 1), xBf = __shfl_up_sync(~0u, yB_f, 1), xBr = __shfl_up_sync(~0u, yB_r, 1);
      if (lane == 0) {
        xAh = 0; xAf = 0; xAr = sres[col & (RES - 1)];
        xBh = 0; xBf = 0; xBr = sres[(col + 1) & (RES - 1)];
      }
      uint32_t loA[R / 4], hiA[R / 4], loB[R / 4], hiB[R / 4];
      loadw<R>(loA, hiA, sprof, xAr, lane);
      loadw<R>(loB, hiB, sprof, xBr, lane);
      uint32_t hrA = __vadd2(xAh, nrho), fA = __vadd2(xAf, nrho), hA = 0;
      uint32_t hrB = __vadd2(xBh, nrho), fB = __vadd2(xBf, nrho), hB = 0;
#pragma unroll
      for (int r = 0; r <= R; ++r) {
        const uint32_t hAp = hA;
        if (r < R) {
          fA = __viaddmax_s16x2(fA, nsig, hrA);
          hA = __vimax3_s16x2_relu(t[r], e[r], fA);
          const uint32_t hr = __vadd2(hA, nrho);
          e[r] = __viaddmax_s16x2(e[r], nsig, hr);
          t[r] = __vadd2(hrA, wrow<R>(loA, hiA, r));
          hrA = hr;
        }
        if (r >= 1) {
          const int q = r - 1;
          fB = __viaddmax_s16x2(fB, nsig, hrB);
          hB = __vimax3_s16x2_relu(t[q], e[q], fB);
          const uint32_t hr = __vadd2(hB, nrho);
          e[q] = __viaddmax_s16x2(e[q], nsig, hr);
          t[q] = __vadd2(hrB, wrow<R>(loB, hiB, q));
          hrB = hr;
          best = __vimax3_s16x2(best, hAp, hB);
        }
      }
      yA_h = hA; yA_f = __vadd2(fA, prho); yA_r = xAr;
      yB_h = hB; yB_f = __vadd2(fB, prho); yB_r = xBr;
      asm volatile("" : "+r"(yA_r), "+r"(yB_r) : "r"(yA_f), "r"(yB_f));
    }
  }
  __syncthreads();
  long long t1 = clock64();
  uint32_t acc = best;
#pragma unroll
  for (int r = 0; r < R; ++r) acc ^= t[r] ^ e[r];
  if (acc == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) rec[blockIdx.x] = Rec{t0, t1, smid()};
}

template <typename K>
static void run(const char* name, K kern, int R, int threads, uint32_t* d_out, Rec* d_rec) {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int blocks = nsm;
  for (int w = 0; w < 200; ++w) kern<<<blocks, threads>>>(d_out, 1u + w, d_rec);
  cudaDeviceSynchronize();
  std::vector<Rec> h(blocks);
  double sum = 0;
  const int reps = 10;
  for (int i = 0; i < reps; ++i) {
    kern<<<blocks, threads>>>(d_out, 7u + i, d_rec);
    cudaMemcpy(h.data(), d_rec, sizeof(Rec) * blocks, cudaMemcpyDeviceToHost);
    double rate = 0;
    for (auto& r : h) rate += (threads / 32.0) * 32.0 * (double)COLS * R * 2.0 / (double)(r.t1 - r.t0);
    sum += rate;
  }
  const double cpc = sum / reps;
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, kern);
  printf("%-22s cells/clk/GPU %8.1f  frac_of_4209.8 %.3f  regs %d  local %zu\n", name, cpc, cpc / 4209.8, fa.numRegs,
         (size_t)fa.localSizeBytes);
}

int main() {
  uint32_t* d_out; Rec* d_rec;
  cudaMalloc(&d_out, sizeof(uint32_t) * 148 * 1024);
  cudaMalloc(&d_rec, sizeof(Rec) * 148);
  run("one_R48_384", k_probe<48, 384, 0>, 48, 384, d_out, d_rec);
  run("one_R32_384", k_probe<32, 384, 0>, 32, 384, d_out, d_rec);
  run("one_R64_256", k_probe<64, 256, 0>, 64, 256, d_out, d_rec);
  run("two_R32_384", k_probe<32, 384, 1>, 32, 384, d_out, d_rec);
  run("two_R16_384", k_probe<16, 384, 1>, 16, 384, d_out, d_rec);
  run("two_R48_256", k_probe<48, 256, 1>, 48, 256, d_out, d_rec);
  run("two_R32_256", k_probe<32, 256, 1>, 32, 256, d_out, d_rec);
  run("two_R16_512", k_probe<16, 512, 1>, 16, 512, d_out, d_rec);
  run("one_R32_512", k_probe<32, 512, 0>, 32, 512, d_out, d_rec);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { fprintf(stderr, "CUDA error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
