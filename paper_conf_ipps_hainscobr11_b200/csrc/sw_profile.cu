// sw_profile.cu — query profile build (§II-A: "a query profile creates a
// vectorized lookup table for the similarity scores that is unique for a given query";
// L20 §III-B: four query rows per 32-bit word) and the kernel menu.
//
// Layout: see ProfLayout in sw_internal.h (chunk-major, letter stride a multiple of 128 B,
// one bank-rotated replica per chain of a warp).  Values: int8(w(q_i, a) + rho) for a < A,
// i < m; -128 for the pad letter a == A and for pad query rows i >= m.
// Storing w + rho (not w) lets the engine form H = max(hr_diag + (w + rho), E, F, 0) on
// registers that hold hr = H - rho (sw_engine.cuh).
#include "sw_engine.cuh"
#include "sw_internal.h"

namespace swb {

__global__ void k_profile(uint8_t* __restrict__ blob, const ProfLayout L, const uint8_t* __restrict__ q, int m,
                          const int8_t* __restrict__ W, int A, int rho) {
  const int rows = L.strips * L.G * L.R;
  const int64_t n = (int64_t)L.nrep * (A + 1) * rows;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const int i = (int)(t % rows);
    const int a = (int)((t / rows) % (A + 1));
    const int rep = (int)(t / ((int64_t)rows * (A + 1)));
    const int P = i / (L.G * L.R), qq = i % (L.G * L.R), gl = qq / L.R, r = qq % L.R;
    const int64_t addr = (int64_t)L.off + (int64_t)rep * L.rs + (int64_t)a * L.ls +
                         ((int64_t)(P * L.nch + r / L.cb) * L.G + gl) * L.cb + r % L.cb;
    int v = kPadValue;
    if (a < A && i < m) v = (int)W[q[i] * A + a] + rho;
    blob[addr] = (uint8_t)(int8_t)v;
  }
}

cudaError_t launch_profile(uint8_t* blob, const ProfLayout& L, const uint8_t* q, int m, const int8_t* W, int A,
                           int rho, cudaStream_t st) {
  const int64_t n = (int64_t)L.nrep * (A + 1) * L.strips * L.G * L.R;
  const int threads = 256;
  const int blocks = (int)std::min<int64_t>((n + threads - 1) / threads, 4096);
  k_profile<<<blocks, threads, 0, st>>>(blob, L, q, m, W, A, rho);
  return cudaGetLastError();
}

}  // namespace swb
