// sw_profile.cu — query profile build (§II-A: "a query profile creates a
// vectorized lookup table for the similarity scores that is unique for a given query";
// L20 §III-B: four query rows per 32-bit word) and the kernel menu.
//
// Layout: prof[a * pstride + i] = int8(w(q_i, a) + rho) for a < A, i < m;
//         -128 for the pad letter a == A and for pad query rows m <= i < pstride.
// Storing w + rho (not w) lets the engine form H = max(hr_diag + (w + rho), E, F, 0) with a
// single VIADDMNMX.RELU on registers that hold hr = H - rho (sw_engine.cuh).
#include "sw_engine.cuh"
#include "sw_internal.h"

namespace swb {

__global__ void k_profile(uint8_t* __restrict__ prof, const uint8_t* __restrict__ q, int m,
                          const int8_t* __restrict__ W, int A, int rho, int pstride) {
  const int64_t n = (int64_t)(A + 1) * pstride;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const int a = (int)(t / pstride);
    const int i = (int)(t % pstride);
    int v = kPadValue;
    if (a < A && i < m) v = (int)W[q[i] * A + a] + rho;
    prof[t] = (uint8_t)(int8_t)v;
  }
}

cudaError_t launch_profile(uint8_t* prof, const uint8_t* q, int m, const int8_t* W, int A, int rho, int pstride,
                           cudaStream_t st) {
  const int64_t n = (int64_t)(A + 1) * pstride;
  const int threads = 256;
  const int blocks = (int)std::min<int64_t>((n + threads - 1) / threads, 4096);
  k_profile<<<blocks, threads, 0, st>>>(prof, q, m, W, A, rho, pstride);
  return cudaGetLastError();
}

}  // namespace swb
