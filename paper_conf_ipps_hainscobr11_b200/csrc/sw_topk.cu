// sw_topk.cu — the top hits of a score array on the device (include/sw.h sw_top_hits; SURVEY.md
// f4 "traceback for top hits": the hits to align are the best-scoring database sequences).
//
// Radix select over order-preserving 32-bit keys (score ^ 0x80000000): four passes of an 8-bit
// digit histogram (256 bins in shared memory per CTA, merged with global atomics) restricted to
// the keys whose higher digits equal the prefix found so far; the host walks each 256-bin
// histogram from the top to the digit holding the k-th largest key.  Then one pass collects the
// keys above the threshold (fewer than k, any order) and an ordered compaction (per-CTA counts,
// their prefix, warp ballots) keeps the threshold ties with the smallest indices.
#include <cstdint>
#include <cuda_runtime.h>

#include "sw_internal.h"

namespace swb {

namespace {
constexpr int kTkThreads = 256;
constexpr int kTkPerCta = 4096;   // keys per CTA in the ordered tie compaction

__device__ __forceinline__ uint32_t key_of(int32_t s) { return (uint32_t)s ^ 0x80000000u; }

__global__ void k_tk_hist(const int32_t* __restrict__ s, int64_t n, int shift, uint32_t prefix, uint32_t pmask,
                          uint32_t* __restrict__ hist) {
  __shared__ uint32_t h[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) h[i] = 0u;
  __syncthreads();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t k = key_of(s[i]);
    if ((k & pmask) == prefix) atomicAdd(&h[(k >> shift) & 0xffu], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 256; i += blockDim.x)
    if (h[i]) atomicAdd(&hist[i], h[i]);
}

// keys > thr, any order (out_count counts them); per-CTA counts of keys == thr
__global__ void k_tk_above(const int32_t* __restrict__ s, int64_t n, uint32_t thr, int64_t* __restrict__ out_idx,
                           int32_t* __restrict__ out_score, uint32_t* __restrict__ out_count,
                           uint32_t* __restrict__ tie_count) {
  __shared__ uint32_t ties;
  if (threadIdx.x == 0) ties = 0u;
  __syncthreads();
  const int64_t b0 = (int64_t)blockIdx.x * kTkPerCta;
  const int64_t b1 = b0 + kTkPerCta < n ? b0 + kTkPerCta : n;
  for (int64_t i = b0 + threadIdx.x; i < b1; i += blockDim.x) {
    const uint32_t k = key_of(s[i]);
    if (k > thr) {
      const uint32_t o = atomicAdd(out_count, 1u);
      out_idx[o] = i;
      out_score[o] = s[i];
    } else if (k == thr) {
      atomicAdd(&ties, 1u);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) tie_count[blockIdx.x] = ties;
}

// the ties of CTA b in index order at tie_off[b] ..., only the first `need` overall
__global__ void k_tk_ties(const int32_t* __restrict__ s, int64_t n, uint32_t thr, const uint32_t* __restrict__ tie_off,
                          uint32_t need, int64_t* __restrict__ out_idx, int32_t* __restrict__ out_score) {
  __shared__ uint32_t wcount[kTkThreads / 32];
  __shared__ uint32_t base;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) base = tie_off[blockIdx.x];
  __syncthreads();
  if (base >= need) return;
  const int64_t b0 = (int64_t)blockIdx.x * kTkPerCta;
  for (int64_t c = b0; c < b0 + kTkPerCta && c < n; c += kTkThreads) {   // chunks of 256 keys, in order
    const int64_t i = c + threadIdx.x;
    const bool tie = i < n && key_of(s[i]) == thr;
    const uint32_t bal = __ballot_sync(0xffffffffu, tie);
    if (lane == 0) wcount[warp] = __popc(bal);
    __syncthreads();
    uint32_t before = base;
    for (int w = 0; w < warp; ++w) before += wcount[w];
    const uint32_t pos = before + __popc(bal & ((1u << lane) - 1u));
    if (tie && pos < need) { out_idx[pos] = i; out_score[pos] = s[i]; }
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t t = 0;
      for (int w = 0; w < kTkThreads / 32; ++w) t += wcount[w];
      base += t;
    }
    __syncthreads();
    if (base >= need) return;
  }
}
}  // namespace

int topk_ctas(int64_t n) { return (int)((n + kTkPerCta - 1) / kTkPerCta); }

cudaError_t launch_tk_hist(const int32_t* s, int64_t n, int shift, uint32_t prefix, uint32_t pmask, uint32_t* hist,
                           int grid, cudaStream_t st) {
  k_tk_hist<<<grid, kTkThreads, 0, st>>>(s, n, shift, prefix, pmask, hist);
  return cudaGetLastError();
}
cudaError_t launch_tk_above(const int32_t* s, int64_t n, uint32_t thr, int64_t* out_idx, int32_t* out_score,
                            uint32_t* out_count, uint32_t* tie_count, cudaStream_t st) {
  k_tk_above<<<topk_ctas(n), kTkThreads, 0, st>>>(s, n, thr, out_idx, out_score, out_count, tie_count);
  return cudaGetLastError();
}
cudaError_t launch_tk_ties(const int32_t* s, int64_t n, uint32_t thr, const uint32_t* tie_off, uint32_t need,
                           int64_t* out_idx, int32_t* out_score, cudaStream_t st) {
  k_tk_ties<<<topk_ctas(n), kTkThreads, 0, st>>>(s, n, thr, tie_off, need, out_idx, out_score);
  return cudaGetLastError();
}

}  // namespace swb
