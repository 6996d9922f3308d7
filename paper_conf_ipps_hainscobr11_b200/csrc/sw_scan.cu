// sw_scan.cu — the row-scan kernel for the longest long pairs of an isolated long-path launch
// (DESIGN.md "Row scan on a cluster").
//
// The strip kernels (k_search_t's team stream and gangs) put one lane's 16 database positions on
// the critical path of every step and hand a strip to the next after a 32-lane skew, so a single
// pair's time is bounded by ~n row-steps of one warp: C2's 35,213-residue pair takes ~0.7 ms
// for query 567 however many CTAs it is spread over (profiles/r02_gang_*.txt).  Here one query
// row of Eq.(1) (§II) is computed by a whole cluster at once: the vertical and
// diagonal terms need only the previous row (F and H per column, in registers), and the
// horizontal term is a max-plus prefix scan along the row.  With Ht = max(H[i-1][j-1] + w, F, 0),
//   E[j+1] = max(E[j] - sigma, H[j] - rho) = max(E[j] - sigma', Ht[j] - rho),  sigma' = min(sigma, rho)
// (H[j] = max(Ht[j], E[j]) and E[j] - rho <= E[j] - sigma' — exact, also for sigma > rho), so
// a run of c columns maps its entering E to max(E - c sigma', b) and these maps compose:
// (a1, b1) then (a2, b2) = (a1 + a2, max(b1 - a2, b2)).  A lane owns kScanC = 4 columns and a
// warp scans its 32 lanes' maps with shuffles; the warps of the whole cluster then form one
// pipeline along the row (below): a warp needs only the E entering its first column from its
// left neighbour, and rows i, i+1, ... are in flight along the pipeline at once.  Values are
// s16x2 (the pair's two sequences) with the overflow flag of the other kernels; E + rho >= 0
// always (E >= H - rho >= -rho), so the scan runs on E + rho with the offsets clamped to 32767
// and never wraps.  (Measured and replaced: a CTA-wide scan per row with one cluster barrier
// per time step, 2.5-3x slower; release / acquire hand-off flags, which compile to
// MEMBAR.ALL.GPU per row here, 3.5x slower — profiles/r02_row_scan.txt.)
#include <cooperative_groups.h>

#include "sw_engine.cuh"
#include "sw_internal.h"

namespace swb {
namespace cg = cooperative_groups;

namespace {
constexpr int kRing = 8;   // rows in flight between two neighbouring warps

__device__ __forceinline__ uint32_t clamp_off(int v) { return LaneS16x2::splat(-min(v, 32767)); }
__device__ __forceinline__ uint32_t mapa(uint32_t saddr, int rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
// shared::cluster accesses (a 32-bit address of this CTA's or, after mapa, another CTA's smem).
// Hand-off words are 64-bit (tag << 32 | value), written and polled relaxed (single-copy
// atomic): no fence — a release/acquire at cluster scope compiles to MEMBAR.ALL.GPU here.
__device__ __forceinline__ void st_cl64(uint32_t a, unsigned long long v) {
  asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
// polls of this CTA's own slots (written by this CTA's warps or by the left CTA)
__device__ __forceinline__ unsigned long long ld_own64(uint32_t a) {
  unsigned long long v;
  asm volatile("ld.relaxed.cluster.shared::cta.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void st_cl32(uint32_t a, uint32_t v) {
  asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_cl32(uint32_t a) {   // (the right CTA's consumed counter)
  uint32_t v;
  asm volatile("ld.relaxed.cluster.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
}  // namespace

// cols_cta: columns per CTA (a multiple of 32 x kScanC; warps beyond cols_cta / 128 idle).
// The active warps of the cluster form ONE pipeline along the row (warp w of CTA k owns columns
// [k cols_cta + 128 w, + 128)): per row a warp computes Ht and its lanes' maps, scans them
// (shuffles) and then needs only the E entering its first column from its left neighbour —
// E_out = max(E_in - 128 sigma', B_warp) is one op, so E travels along the row one hop per
// warp while the warps' row work overlaps (rows i, i+1, ... are in flight along the pipeline).
// The left neighbour's last H of the previous row (the diagonal of the warp's first column)
// travels the same way.  Hand-off slots live in the receiver's shared memory (the left CTA
// writes them with st.shared::cluster and a release.cluster progress counter); a sender stays
// fewer than kRing rows ahead of its receiver (the receiver's consumed counter).  The slots are
// tagged words (row + 1 in the high half): no progress flags and no fences.
// One launch runs all row-scan items: cluster c (CTAs [c K, c K + K)) takes long pair c, with
// cols_cta = ceil(ncols / K) rounded up to 128 columns (the dynamic shared memory is sized for
// pair 0, the longest).
__global__ void __launch_bounds__(kScanThreads, 1) k_scan_pair(const TParams p, int item0) {
  using L = LaneS16x2;
  extern __shared__ __align__(16) uint8_t tab[];   // [(a * 2 + s) * cols_cta + j]: w, int8; then the query
  __shared__ unsigned long long s_eo[32][kRing];   // (row + 1) << 32 | E + rho entering warp w's first column
  __shared__ unsigned long long s_hl[32][kRing];   // (row + 1) << 32 | H of the left neighbour's last column
  __shared__ uint32_t s_cons[32];                  // rows consumed, per receiver
  __shared__ uint32_t s_best[kScanMaxCtas];
  __shared__ uint32_t s_red[32];
  __shared__ uint8_t s_real[33];
  cg::cluster_group cl = cg::this_cluster();
  const int k = (int)cl.block_rank(), K = (int)cl.num_blocks();
  const int item = item0 + (int)blockIdx.x / K;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int ncols = p.pair_ncols[item];
  const int cols_cta = ((ncols + K - 1) / K + 32 * kScanC - 1) / (32 * kScanC) * (32 * kScanC);
  const int act_warps = cols_cta / (32 * kScanC);
  const uint16_t* cp = p.cols + p.pair_off[item];
  const int A1 = p.A_used + 1;
  const int j0 = k * cols_cta;
  const int nrows = p.qcols;
  uint8_t* s_q = tab + (size_t)A1 * 2 * cols_cta;   // compact query letters (row i -> table row)

  if (tid < A1) s_real[tid] = tid < p.A_used ? (uint8_t)(__fns(p.qmask, 0, tid + 1)) : (uint8_t)255;
  if (tid < 32) s_cons[tid] = 0u;
  for (int i = tid; i < 32 * kRing; i += kScanThreads) { (&s_eo[0][0])[i] = 0ull; (&s_hl[0][0])[i] = 0ull; }
  for (int i = tid; i < nrows; i += kScanThreads) s_q[i] = (uint8_t)(p.qpair[i] & 0xff);
  __syncthreads();
  for (int j = tid; j < cols_cta; j += kScanThreads) {
    const int col = j0 + j;
    const uint32_t d = col < ncols ? (uint32_t)cp[col] : (uint32_t)p.pad_letter * 0x101u;
    const int dlo = d & 0xff, dhi = d >> 8;
    for (int a = 0; a < A1; ++a) {
      const int r = s_real[a];
      const int vlo = (r < p.A && dlo < p.A) ? (int)p.matrix[r * p.A + dlo] : kPadValue;
      const int vhi = (r < p.A && dhi < p.A) ? (int)p.matrix[r * p.A + dhi] : kPadValue;
      tab[(a * 2) * cols_cta + j] = (uint8_t)(int8_t)vlo;
      tab[(a * 2 + 1) * cols_cta + j] = (uint8_t)(int8_t)vhi;
    }
  }
  cl.sync();   // tables and counters of every CTA initialised before any hand-off
  // the T-mode kernel behind this one on the stream (programmatic dependent launch) may start
  // now: these clusters are resident, its CTAs take the remaining SMs
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

  uint32_t best = 0u;
  if (warp < act_warps) {
    const int rho = p.rho, sigma = p.sigma;
    const int sigp = min(sigma, rho);
    const int a_thr = kScanC * sigp;                 // one thread's offset (its 4 columns)
    const uint32_t nrho = L::splat(-rho), prho = L::splat(rho), nsig = L::splat(-sigma);
    const uint32_t nsigp = L::splat(-sigp);
    const uint32_t off_lane = clamp_off(lane * a_thr);   // lanes 0 .. lane-1 of this warp
    const uint32_t off_all = clamp_off(32 * a_thr);      // the whole warp
    uint32_t offl[5];                                     // Kogge-Stone step offsets
#pragma unroll
    for (int q = 0; q < 5; ++q) offl[q] = clamp_off((1 << q) * a_thr);
    // receiver side (this warp): its slots; sender side: the right neighbour's slots (this CTA's
    // next warp, or warp 0 of CTA k + 1)
    const bool has_left = warp > 0 || k > 0;
    const bool has_right = warp + 1 < act_warps || k + 1 < K;
    const int rw = warp + 1 < act_warps ? warp + 1 : 0;
    const int rk = warp + 1 < act_warps ? k : k + 1;
    const uint32_t my_eo = smem_u32(&s_eo[warp][0]), my_hl = smem_u32(&s_hl[warp][0]);
    const uint32_t my_cons = smem_u32(&s_cons[warp]);
    const uint32_t r_eo = has_right ? mapa(smem_u32(&s_eo[rw][0]), rk) : 0u;
    const uint32_t r_hl = has_right ? mapa(smem_u32(&s_hl[rw][0]), rk) : 0u;
    const uint32_t r_cons = has_right ? mapa(smem_u32(&s_cons[rw]), rk) : 0u;
    const uint8_t* tcol = tab + kScanC * tid;
    uint32_t hup[kScanC], f[kScanC];
#pragma unroll
    for (int c = 0; c < kScanC; ++c) { hup[c] = 0u; f[c] = nrho; }
    uint32_t r_cons_seen = 0u;   // the receiver's consumed rows, last read
    for (int i = 0; i < nrows; ++i) {
      const int slot = i & (kRing - 1);
      const int qa = s_q[i];
      const uint32_t wlo = *reinterpret_cast<const uint32_t*>(tcol + (qa * 2) * cols_cta);
      const uint32_t whi = *reinterpret_cast<const uint32_t*>(tcol + (qa * 2 + 1) * cols_cta);
      // the diagonal of column 0: H[i-1][j-1] of the left lane, or of the left warp's last column
      uint32_t dg = __shfl_up_sync(SWB_FULL, hup[kScanC - 1], 1);
      uint32_t hl = 0u;
      if (has_left && i > 0) {
        const uint32_t a = my_hl + 8 * ((i - 1) & (kRing - 1));
        unsigned long long v;
        while (((v = ld_own64(a)) >> 32) != (unsigned long long)i) { }
        hl = (uint32_t)v;
      }
      if (lane == 0) dg = hl;
      uint32_t ht[kScanC];
#pragma unroll
      for (int c = 0; c < kScanC; ++c) {
        f[c] = L::gap(f[c], nsig, L::add(hup[c], nrho));      // F = max(F - sigma, H_up - rho)
        const uint32_t w = c == 0 ? L::subst<0>(wlo, whi) : c == 1 ? L::subst<1>(wlo, whi)
                         : c == 2 ? L::subst<2>(wlo, whi) : L::subst<3>(wlo, whi);   // s16x2 (w_lo, w_hi)
        ht[c] = L::hmax(L::add(dg, w), f[c], f[c]);            // Ht = max(H_diag + w, F, 0)
        dg = hup[c];
      }
      // this lane's map: b = E entering the next lane's column 0 for E_in = -inf, + rho
      uint32_t b = L::add(ht[0], nrho);
#pragma unroll
      for (int c = 1; c < kScanC; ++c) b = L::gap(b, nsigp, L::add(ht[c], nrho));
      b = L::add(b, prho);
#pragma unroll
      for (int q = 0; q < 5; ++q) {   // warp inclusive scan (offset of the 2^q lanes between)
        const uint32_t o = __shfl_up_sync(SWB_FULL, b, 1 << q);
        if (lane >= (1 << q)) b = L::gap(o, offl[q], b);
      }
      uint32_t lex = __shfl_up_sync(SWB_FULL, b, 1);       // lanes 0 .. lane-1
      if (lane == 0) lex = 0u;                             // (+rho space: 0 = no contribution)
      const uint32_t bw = __shfl_sync(SWB_FULL, b, 31);    // the whole warp's map
      // E + rho entering this warp's first column (the left neighbour's row i)
      uint32_t ein = 0u;
      if (has_left) {
        const uint32_t a = my_eo + 8 * slot;
        unsigned long long v;
        while (((v = ld_own64(a)) >> 32) != (unsigned long long)(i + 1)) { }
        ein = (uint32_t)v;
        __syncwarp();
        if (lane == 0) st_cl32(my_cons, (uint32_t)(i + 1));   // both slots of row i read
      }
      // the sender side: the right neighbour's slots of row i must be free — its E of row
      // i - kRing and its H of row i - kRing (read when it started row i - kRing + 1)
      if (has_right && i >= kRing - 1) {
        while (r_cons_seen < (uint32_t)(i - kRing + 2)) r_cons_seen = ld_cl32(r_cons);
      }
      if (has_right && lane == 0)   // E + rho entering the right neighbour's first column
        st_cl64(r_eo + 8 * slot, (unsigned long long)(i + 1) << 32 | L::gap(ein, off_all, bw));
      uint32_t e = L::add(L::gap(ein, off_lane, lex), nrho);   // E entering this lane's column 0
      uint32_t hprev = 0u;
#pragma unroll
      for (int c = 0; c < kScanC; ++c) {
        const uint32_t h = L::max2(ht[c], e);                 // H = max(Ht, E)
        e = L::gap(e, nsig, L::add(h, nrho));                 // E[j+1] = max(E - sigma, H - rho)
        hup[c] = h;
        if (c & 1) best = L::max3(best, hprev, h); else hprev = h;
      }
      if (has_right && lane == 31)   // this warp's last H of row i: the right neighbour's diagonal
        st_cl64(r_hl + 8 * slot, (unsigned long long)(i + 1) << 32 | hup[kScanC - 1]);
    }
  }
  // the pair's maxima: warp, CTA, then cluster (CTA 0 emits)
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) best = L::max2(best, __shfl_xor_sync(SWB_FULL, best, o));
  if (lane == 0) s_red[warp] = best;
  __syncthreads();
  if (tid == 0) {
    uint32_t bb = s_red[0];
    for (int w = 1; w < kScanThreads / 32; ++w) bb = L::max2(bb, s_red[w]);
    *cl.map_shared_rank(&s_best[k], 0) = bb;
  }
  cl.sync();
  if (k == 0 && tid == 0) {
    uint32_t bb = s_best[0];
    for (int r = 1; r < K; ++r) bb = L::max2(bb, s_best[r]);
    emit_t(p, bb, item);
  }
  cl.sync();   // no CTA exits while a neighbour may still access its shared memory
}

int scan_cols_cta(int ncols, int ctas) {
  return ((ncols + ctas - 1) / ctas + 32 * kScanC - 1) / (32 * kScanC) * (32 * kScanC);
}
int scan_smem_bytes(int a_used, int cols_cta, int qcols) { return (a_used + 1) * 2 * cols_cta + qcols; }

cudaError_t configure_scan_kernel(int smem_bytes, int ctas, int* max_clusters) {
  cudaError_t e = cudaFuncSetAttribute(k_scan_pair, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_scan_pair, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = ctas;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.gridDim = dim3(ctas);
  cfg.blockDim = dim3(kScanThreads);
  cfg.dynamicSmemBytes = smem_bytes;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaOccupancyMaxActiveClusters(max_clusters, k_scan_pair, &cfg);
}

// items [item0, item0 + items) on clusters of `ctas` CTAs; pdl: programmatic dependent launch
// behind the previous scan launch on the stream (its clusters trigger once resident)
cudaError_t launch_scan_pairs(const TParams& p, int item0, int items, int ctas, int smem_bytes, cudaStream_t st,
                              bool pdl) {
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = ctas;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.gridDim = dim3(ctas * items);
  cfg.blockDim = dim3(kScanThreads);
  cfg.dynamicSmemBytes = smem_bytes;
  cfg.stream = st;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaLaunchAttribute attr2[2] = {attr[0], {}};
  if (pdl) {
    attr2[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr2[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr2;
    cfg.numAttrs = 2;
  }
  return cudaLaunchKernelEx(&cfg, k_scan_pair, p, item0);
}

}  // namespace swb
