// sw_tmode.cu — instantiation of the transposed long-sequence kernel (k_search_t) and the
// query-stream builder it reads.
#include "sw_engine.cuh"
#include "sw_internal.h"

namespace swb {

// qpair[i] = c_i | c_i << 8 for i < m, with c_i the compact index of q_i among the letters
// present in the query (qmask), and the compact pad (popcount(qmask)) beyond (qcols + kPadCols
// entries)
__global__ void k_qpair(uint16_t* __restrict__ out, const uint8_t* __restrict__ q, int m, int n, uint32_t qmask) {
  const int pad = __popc(qmask);
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int a = i < m ? __popc(qmask & ((1u << q[i]) - 1u)) : pad;
    out[i] = (uint16_t)(a | (a << 8));
  }
}

cudaError_t launch_qpair(uint16_t* out, const uint8_t* q, int m, int n, uint32_t qmask, cudaStream_t st) {
  k_qpair<<<(n + 255) / 256, 256, 0, st>>>(out, q, m, n, qmask);
  return cudaGetLastError();
}

// s32 = true: the 32-bit recompute of the flagged sequences (p.item_list / p.item_count)
cudaError_t launch_tmode(const TParams& p, int grid, int smem_bytes, cudaStream_t st, bool s32) {
  if (s32) {
    if (p.delta > 0) return launch_search_tmode<kTmodeC, kTmodeThreads, true, LaneS32>(p, grid, smem_bytes, st);
    return launch_search_tmode<kTmodeC, kTmodeThreads, false, LaneS32>(p, grid, smem_bytes, st);
  }
  if (p.delta > 0) return launch_search_tmode<kTmodeC, kTmodeThreads, true, LaneS16x2>(p, grid, smem_bytes, st);
  return launch_search_tmode<kTmodeC, kTmodeThreads, false, LaneS16x2>(p, grid, smem_bytes, st);
}

cudaError_t configure_tmode_kernel(int smem_bytes, int* blocks_per_sm, bool wide, bool s32) {
  if (s32) {
    if (wide) return configure_tmode<kTmodeC, kTmodeThreads, true, LaneS32>(smem_bytes, blocks_per_sm);
    return configure_tmode<kTmodeC, kTmodeThreads, false, LaneS32>(smem_bytes, blocks_per_sm);
  }
  if (wide) return configure_tmode<kTmodeC, kTmodeThreads, true, LaneS16x2>(smem_bytes, blocks_per_sm);
  return configure_tmode<kTmodeC, kTmodeThreads, false, LaneS16x2>(smem_bytes, blocks_per_sm);
}

}  // namespace swb
