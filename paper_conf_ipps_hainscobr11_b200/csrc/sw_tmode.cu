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

// s32 = true: the 32-bit recompute of the flagged sequences (p.item_list / p.item_count);
// p.packed selects the team stream's layout, p.delta > 0 the WIDE instantiation
template <bool WIDE, class L>
static cudaError_t launch_t(const TParams& p, int grid, int smem_bytes, cudaStream_t st, bool pdl) {
  if (p.packed) return launch_search_tmode<kTmodeC, kTmodeThreads, WIDE, L, true>(p, grid, smem_bytes, st, pdl);
  return launch_search_tmode<kTmodeC, kTmodeThreads, WIDE, L, false>(p, grid, smem_bytes, st, pdl);
}
template <bool WIDE, class L>
static cudaError_t configure_t2(int smem_bytes, int* blocks_per_sm, bool packed) {
  if (packed) return configure_tmode<kTmodeC, kTmodeThreads, WIDE, L, true>(smem_bytes, blocks_per_sm);
  return configure_tmode<kTmodeC, kTmodeThreads, WIDE, L, false>(smem_bytes, blocks_per_sm);
}

cudaError_t launch_tmode(const TParams& p, int grid, int smem_bytes, cudaStream_t st, bool s32, bool pdl) {
  if (s32) return p.delta > 0 ? launch_t<true, LaneS32>(p, grid, smem_bytes, st, pdl)
                              : launch_t<false, LaneS32>(p, grid, smem_bytes, st, pdl);
  return p.delta > 0 ? launch_t<true, LaneS16x2>(p, grid, smem_bytes, st, pdl)
                     : launch_t<false, LaneS16x2>(p, grid, smem_bytes, st, pdl);
}

cudaError_t configure_tmode_kernel(int smem_bytes, int* blocks_per_sm, bool wide, bool s32, bool packed) {
  if (s32) return wide ? configure_t2<true, LaneS32>(smem_bytes, blocks_per_sm, packed)
                       : configure_t2<false, LaneS32>(smem_bytes, blocks_per_sm, packed);
  return wide ? configure_t2<true, LaneS16x2>(smem_bytes, blocks_per_sm, packed)
              : configure_t2<false, LaneS16x2>(smem_bytes, blocks_per_sm, packed);
}

}  // namespace swb
