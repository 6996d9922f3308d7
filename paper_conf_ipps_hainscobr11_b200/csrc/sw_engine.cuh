// sw_engine.cuh — the sm_100a Smith-Waterman engine.
//
// What every lane computes is Eq.(1) of PAPER.md (L12 §II):
//   E[i][j] = max(E[i][j-1] - sigma, H[i][j-1] - rho)
//   F[i][j] = max(F[i-1][j] - sigma, H[i-1][j] - rho)
//   H[i][j] = max(0, E[i][j], F[i][j], H[i-1][j-1] + w(q_i, d_j))
// in the "hr" form used here: registers hold hr = H - rho, so that the single value hr
// feeds both E of the right neighbour and F of the lower neighbour, and the query profile
// stores w + rho so that H = max(hr_diag + (w + rho), E, F, 0) is one fused DPX op.
//
// Work decomposition (B200 design, not the paper's; §III is prior art):
//   * a CHAIN is GC consecutive lanes of a warp; lane l owns R consecutive query rows of
//     the current strip (strip = GC*R rows, "a set of n_th * t_height rows
//     as a strip") and sweeps the database columns; lane l processes column j one step
//     after lane l-1, receiving (H-rho, F) of the row above through __shfl_up_sync
//     (registers for horizontal, shuffles for vertical/diagonal dependencies — the
//     paper's registers + shared memory split);
//   * strips are chained with a full row buffer of (H-rho, F) per column in global/L2
//     ("the bottom row of a strip must be saved for the next pass", L18-L20) and the lane
//     that finishes a strip moves straight on to the next one: one pipeline fill/flush per
//     alignment (future work item iii of PAPER.md L30 §VI);
//   * GROUP mode (inter-task, short sequences): GC = G <= 32 lanes per database pair,
//     several pairs per warp, persistent warps pull pairs longest-first;
//   * TEAM mode (intra-task, long sequences, §II-B.2 and L18 §III): a team of
//     W warps per database pair; warp w of the team takes strips w, w+W, ...; strip
//     hand-off through the row buffers with shared-memory progress flags (acquire/release);
//   * two database sequences share one 32-bit register as signed 16-bit lanes (LaneS16x2,
//     DPX VIADDMNMX/VIMNMX3) with an exact overflow flag; flagged sequences are recomputed
//     with 32-bit lanes (LaneS32) by the same engine.
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

#include "sw_internal.h"

namespace swb {

#define SWB_FULL 0xffffffffu
// packed T-mode team stream's progress tags (strip << 33 | columns); the distinct shift also
// enables run_pass's per-lane keep mask (sw_engine.cuh t_team_stream)
constexpr int kPackedTagShift = 33;

// PRMT with a compile-time selector.  Inline PTX because __byte_perm keeps only 3 bits per
// selector nibble, while the 4th bit (sign replication of the selected byte) is what turns
// the int8 profile entries into sign-extended 16/32-bit lanes in one instruction.
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "n"(SEL));
  return d;
}

// ------------------------------------------------------------------------------------ lanes
struct LaneS16x2 {
  static constexpr int kSeqs = 2;
  static __device__ __forceinline__ uint32_t splat(int v) { return ((uint32_t)v & 0xffffu) * 0x10001u; }
  // max(a - sigma, b): E / F update (a = E or F, nsig = -sigma, b = hr of left / upper cell)
  static __device__ __forceinline__ uint32_t gap(uint32_t a, uint32_t nsig, uint32_t b) {
    return __viaddmax_s16x2(a, nsig, b);
  }
  static __device__ __forceinline__ uint32_t max2(uint32_t a, uint32_t b) { return __vmaxs2(a, b); }
  // H = max(hr_diag + (w + rho), max(E, F), 0)
  static __device__ __forceinline__ uint32_t hcell(uint32_t d, uint32_t w, uint32_t ef) {
    return __viaddmax_s16x2_relu(d, w, ef);
  }
  static __device__ __forceinline__ uint32_t add(uint32_t a, uint32_t b) { return __vadd2(a, b); }
  static __device__ __forceinline__ uint32_t max3(uint32_t a, uint32_t b, uint32_t c) {
    return __vimax3_s16x2(a, b, c);
  }
  // max(t, e, f, 0)
  static __device__ __forceinline__ uint32_t hmax(uint32_t t, uint32_t e, uint32_t f) {
    return __vimax3_s16x2_relu(t, e, f);
  }
  // substitution value of profile row k (of a 4-row int8 word) for both sequences,
  // sign-extended to two s16 halves with one PRMT
  template <int K>
  static __device__ __forceinline__ uint32_t subst(uint32_t wlo, uint32_t whi) {
    return prmt<0xC480u + K * 0x1111u>(wlo, whi);
  }
};

struct LaneS32 {
  static constexpr int kSeqs = 1;
  static __device__ __forceinline__ uint32_t splat(int v) { return (uint32_t)v; }
  static __device__ __forceinline__ uint32_t gap(uint32_t a, uint32_t nsig, uint32_t b) {
    return (uint32_t)__viaddmax_s32((int)a, (int)nsig, (int)b);
  }
  static __device__ __forceinline__ uint32_t max2(uint32_t a, uint32_t b) { return (uint32_t)max((int)a, (int)b); }
  static __device__ __forceinline__ uint32_t hcell(uint32_t d, uint32_t w, uint32_t ef) {
    return (uint32_t)__viaddmax_s32_relu((int)d, (int)w, (int)ef);
  }
  static __device__ __forceinline__ uint32_t add(uint32_t a, uint32_t b) { return a + b; }
  static __device__ __forceinline__ uint32_t max3(uint32_t a, uint32_t b, uint32_t c) {
    return (uint32_t)__vimax3_s32((int)a, (int)b, (int)c);
  }
  static __device__ __forceinline__ uint32_t hmax(uint32_t t, uint32_t e, uint32_t f) {
    return (uint32_t)__vimax3_s32_relu((int)t, (int)e, (int)f);
  }
  template <int K>
  static __device__ __forceinline__ uint32_t subst(uint32_t wlo, uint32_t) {
    return prmt<0x8880u + K * 0x1111u>(wlo, 0u);
  }
};

// ------------------------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
// TMA bulk copy global -> shared (cp.async.bulk, completes on the mbarrier)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_LOOP:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_LOOP;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_smem(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_smem(uint32_t* p, uint32_t v) {
  asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}
// 64-bit progress tags (T-mode team stream: running strip index << 32 | query columns done)
__device__ __forceinline__ unsigned long long ld_acquire_smem(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.cta.shared::cta.u64 %0, [%1];" : "=l"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_smem(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.cta.shared::cta.u64 [%0], %1;" ::"r"(smem_u32(p)), "l"(v) : "memory");
}
// gpu-scope flags in global memory (T-mode gangs: a strip pipeline across CTAs)
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// tagged hand-off words (T-mode gangs): one 64-bit word = (tag << 32) | value, written and read
// as single-copy-atomic relaxed gpu-scope accesses, so a reader that sees the tag of the strip
// it waits for sees that strip's value (no release fence, no separate flag)
__device__ __forceinline__ unsigned long long ld_relaxed_gpu_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_gpu_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void team_bar(int team, int W) {
  if (W > 1) {
    asm volatile("bar.sync %0, %1;" ::"r"(team + 1), "r"(W * 32) : "memory");
  } else {
    __syncwarp();
  }
}

// R rows of one letter for one lane -> R/4 words (4 query rows per word, §III-B
// "stores the similarity scores of four symbols in a single variable").  The lane's rows are
// chunks of CB bytes, STRIDE bytes apart (ProfLayout); with CB = 16 the last chunk may be
// partial (R % 16 rows), read with the narrowest load that covers it.
template <int R, int CB, int STRIDE>
__device__ __forceinline__ void load_prof(uint32_t (&w)[(R + 3) / 4], const uint8_t* p) {
  if constexpr (CB == 16) {
#pragma unroll
    for (int k = 0; k < R / 16; ++k) {
      const uint4 v = *reinterpret_cast<const uint4*>(p + k * STRIDE);
      w[4 * k + 0] = v.x; w[4 * k + 1] = v.y; w[4 * k + 2] = v.z; w[4 * k + 3] = v.w;
    }
    constexpr int k = R / 16, rem = (R % 16 + 3) / 4;   // words of the partial chunk
    if constexpr (rem >= 3) {
      const uint4 v = *reinterpret_cast<const uint4*>(p + k * STRIDE);
      w[4 * k + 0] = v.x; w[4 * k + 1] = v.y; w[4 * k + 2] = v.z;
      if constexpr (rem == 4) w[4 * k + 3] = v.w;
    } else if constexpr (rem == 2) {
      const uint2 v = *reinterpret_cast<const uint2*>(p + k * STRIDE);
      w[4 * k + 0] = v.x; w[4 * k + 1] = v.y;
    } else if constexpr (rem == 1) {
      w[4 * k] = *reinterpret_cast<const uint32_t*>(p + k * STRIDE);
    }
  } else if constexpr (CB == 8) {
    static_assert(R % 8 == 0, "R must be a multiple of the chunk size");
#pragma unroll
    for (int k = 0; k < R / 8; ++k) {
      const uint2 v = *reinterpret_cast<const uint2*>(p + k * STRIDE);
      w[2 * k + 0] = v.x; w[2 * k + 1] = v.y;
    }
  } else {
#pragma unroll
    for (int k = 0; k < R / 4; ++k) w[k] = *reinterpret_cast<const uint32_t*>(p + k * STRIDE);
  }
}

// Profile chunk size for R rows per lane: 16-byte chunks (LDS.128, the last one partial when
// R % 16 != 0) from 12 rows up, else 8 or 4.  Must match make_layout (sw_api.cu).
template <int R>
__host__ __device__ constexpr int chunk_bytes() { return (R >= 12) ? 16 : (R % 8 == 0) ? 8 : 4; }
template <int R>
__host__ __device__ constexpr int chunks_per_lane() { return (R + chunk_bytes<R>() - 1) / chunk_bytes<R>(); }

// substitution value (w + rho) of row r of the lane's window, packed per Lane
template <class L, int R>
__device__ __forceinline__ uint32_t subst_row(const uint32_t (&wlo)[(R + 3) / 4], const uint32_t (&whi)[(R + 3) / 4], int r) {
  const uint32_t a = wlo[r >> 2];
  const uint32_t b = (L::kSeqs == 2) ? whi[r >> 2] : 0u;
  switch (r & 3) {
    case 0: return L::template subst<0>(a, b);
    case 1: return L::template subst<1>(a, b);
    case 2: return L::template subst<2>(a, b);
    default: return L::template subst<3>(a, b);
  }
}

// WIDE: rho + max(w) does not fit the int8 profile entry w + rho.  The profile then holds
// w + c with c = rho - delta (sw_api.cu), and the diagonal term adds delta back on the FMA pipe:
// t = (hr_up + delta) + (w + c) = H[i-1][j] + w (one more VIADD.16x2 per cell pair).
template <bool WIDE>
struct ChainConstT {
  static constexpr bool kWide = WIDE;
  int rho, sigma;
  int delta;              // rho - (profile offset c); 0 unless WIDE
  uint32_t padpair;       // residue pair of two pad letters
  uint32_t hi_mul;        // 1 << 24 at run time (SearchParams::hi_mul)
};
using ChainConst = ChainConstT<false>;

// The cell update (one row r of one column j, both sequences of the pair).  Besides E, each row
// keeps t = H[r-1][j] + w(q_r, d_{j+1}) for the NEXT column (the diagonal term of Eq.(1)),
// formed as soon as its inputs exist (the row above's H at this column).  Every per-row
// register (e[r], t[r]) is read and rewritten by its own row only, so the unrolled step loop
// needs no register rotation (an earlier form kept H - rho of the left column per row, whose
// old value had to survive one row longer than its new one: ~R register moves per step).
//   f    = max(f - sigma, hr_up)          F[r][j]                  VIADDMNMX
//   h    = max(t[r], e[r], f, 0)          H[r][j]                  VIMNMX3.RELU
//   hr   = h - rho                                                 VIADD.16x2 (FMA pipe)
//   e[r] = max(e[r] - sigma, hr)          E[r][j+1]                VIADDMNMX
//   t[r] = hr_up + (w + rho)              for column j+1           VIADD.16x2 (FMA pipe)
//   best = max(best, h, h') every two rows                         VIMNMX3
// plus one PRMT per row for w + rho of column j+1 (profile words of the next column's letters):
// 4.5 ALU-pipe + 2 FMA-pipe instructions per cell pair.  (The earlier "u" form,
// u = max(T, E, 0) by VIADDMNMX.RELU and H = max(F + rho - rho, u) by VIADDMNMX, kept the
// vertical chain at two ALU ops but spent 5.5 ALU-pipe instructions per cell pair; here the
// 3-input max with the zero clamp takes T, E and F at once and the adds move to the FMA pipe.
// The chain f -> h -> hr -> f now runs through the FMA pipe (~13 cycles per row); forming
// F - sigma beside H to keep it at two ALU ops cost one more FMA-pipe instruction per cell
// pair and measured 4-5 % slower: issue slots, not the chain, are the tighter limit.)
// Vertical values enter and leave as (H, F + rho), the format of the lane hand-off and of the
// strip row buffers.
// CHAIN2 ("u form", for latency-bound warps: the T-mode gangs, one warp per scheduler): the
// vertical chain is two ALU ops per row instead of three (through the FMA pipe):
//   g    = max(g - sigma, h_up)     F + rho, directly in the hand-off format   VIADDMNMX
//   u    = max(t[r], e[r], 0)       off the chain                               VIMNMX3.RELU
//   h    = max(g - rho, u)          H                                           VIADDMNMX
// at one more ALU-pipe instruction per cell pair (5.5 instead of 4.5; the t form wins where
// the ALU pipe, not the chain, is the limit — every throughput-bound launch).
template <class L, int R, bool WIDE = false, bool CHAIN2 = false>
__device__ __forceinline__ void cell_rows(uint32_t (&e)[R], uint32_t (&t)[R], const uint32_t (&wlo)[(R + 3) / 4],
                                          const uint32_t (&whi)[(R + 3) / 4], uint32_t nrho, uint32_t prho,
                                          uint32_t nsig, uint32_t& hup, uint32_t& fs, uint32_t& best,
                                          uint32_t dlt = 0u) {
  if constexpr (CHAIN2) {
    uint32_t hrup = L::add(hup, nrho), g = fs, h = hup, hprev = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint32_t u = L::hmax(t[r], e[r], e[r]);                  // max(H[i-1][j-1] + w, E, 0)
      g = L::gap(g, nsig, h);                                         // F + rho = max(F[i-1] + rho - sigma, H[i-1])
      h = L::gap(g, nrho, u);                                         // H = max(F, u)
      const uint32_t hr = L::add(h, nrho);
      e[r] = L::gap(e[r], nsig, hr);
      t[r] = L::add(WIDE ? L::add(hrup, dlt) : hrup, subst_row<L, R>(wlo, whi, r));
      hrup = hr;
      if (r & 1) best = L::max3(best, hprev, h); else hprev = h;
    }
    if constexpr (R & 1) best = L::max2(best, hprev);
    hup = h;
    fs = g;
    return;
  }
  uint32_t hrup = L::add(hup, nrho), f = L::add(fs, nrho), hprev = 0, h = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    f = L::gap(f, nsig, hrup);                                        // F = max(F[i-1] - sigma, H[i-1] - rho)
    h = L::hmax(t[r], e[r], f);                                       // H = max(H[i-1][j-1] + w, E, F, 0)
    const uint32_t hr = L::add(h, nrho);                              // H - rho
    e[r] = L::gap(e[r], nsig, hr);                                    // E[j+1] = max(E - sigma, H - rho)
    // H[i-1][j] + w(q_i, d_{j+1}) (WIDE: + delta, the part of rho the int8 profile cannot hold)
    t[r] = L::add(WIDE ? L::add(hrup, dlt) : hrup, subst_row<L, R>(wlo, whi, r));
    hrup = hr;
    if (r & 1) best = L::max3(best, hprev, h); else hprev = h;
  }
  if constexpr (R & 1) best = L::max2(best, hprev);
  hup = h;
  fs = L::add(f, prho);                                               // F + rho for the lane below
}

// One strip pass of a chain of GC lanes over the columns of one database pair (see the file
// header).  Lane l owns rows [(P*GC + l)*R, +R) of the query and processes column j at step
// j + l + 1: every lane (lane 0 included) first processes one pad column j = -1 in the neutral
// state, whose look-ahead forms u for column 0.  All lanes start the pass in the neutral state
// (H = 0, E = -inf -> -rho by reading c4, u = 0); a lane still in its pipeline fill sees
// neutral inputs and pad letters, which keep it exactly neutral, so no per-lane reset is
// needed inside the step loop.  The residue stream each lane receives is one column ahead (the
// letters of column j + 1, for the profile of u).  rb_in[-1] must be a neutral entry (0, 0)
// (the row buffers carry one leading slot, zero-initialised and only ever rewritten with the
// neutral fill values).  Returns max(best, this lane's H maxima) (packed per Lane).
// ONE_PASS: the query is one strip (no row buffer in or out): the first lane's top input is
// the constant boundary (0, 0), so the boundary rings and their loads disappear (registers).
// GPU_FLAGS (T-mode gangs, strips on different SMs): the row buffers hold ONE tagged 64-bit word
// per column, H | (F + rho) << 32, whose four s16 halves carry a 4-bit tag in their bit 15:
// every half is in [0, 32767) for a sequence that is not flagged (H >= 0, F + rho >= 0, both
// below the overflow flag), and a flagged sequence's values are recomputed anyway.  The
// producing strip's last lane writes the words as it goes; the consuming strip's lane 0 polls
// the words it needs (a per-column "flag in the data": no release fence, no progress flag, no
// publication granularity).  tag = 1 + P mod 15 (never 0, the cleared buffer), and slot reuse
// every GW + 1 strips changes it (the planner keeps (GW + 1) mod 15 != 0); the buffer is
// cleared before every gang launch.  prog_in / prog_out are unused then.
// keep (the packed T-mode team stream): 0 for a lane whose rows start a new database pair —
// its vertical input (the lane above's bottom row) is replaced by the neutral boundary.
template <class L, int GC, int R, bool TEAM, int PUB = 16, bool GPU_FLAGS = false, int TAG_SHIFT = 20,
          bool ONE_PASS = false, bool CHAIN2 = false, class CC = ChainConst, class TagT = uint32_t>
__device__ __forceinline__ uint32_t run_pass(const CC& c, const uint8_t* prow, int ls, int hi_off,
                                             const uint16_t* __restrict__ cols, int ncols,
                                             int half, int steps, int P, int passes_total,
                                             const uint2* __restrict__ rb_in, uint2* __restrict__ rb_out,
                                             const TagT* prog_in, TagT* prog_out, uint32_t best,
                                             int tagP = -1, uint32_t epoch = 0, uint32_t keep = 1u) {
  // progress tags: (strip index << TAG_SHIFT) | columns done, monotonic per flag slot; the
  // strip index is the pass P, or the team stream's running strip index tagP (64-bit tags,
  // TAG_SHIFT = 32: the running index is unbounded and the query may have up to 2^20 columns)
  static_assert(TAG_SHIFT < 8 * (int)sizeof(TagT), "tag type too narrow");
  const TagT tag_base = (TagT)(tagP >= 0 ? tagP : P) << TAG_SHIFT;
  const TagT tag_prev = tag_base - ((TagT)1 << TAG_SHIFT);
  static_assert(R % 4 == 0 || R >= 12, "R < 12 must be a multiple of 4");
  const int lane = threadIdx.x & 31;
  const int gl = lane & (GC - 1);
  const uint32_t nrho = L::splat(-c.rho), prho = L::splat(c.rho);
  const uint32_t nsig = L::splat(-c.sigma);
  const uint32_t dlt = L::splat(c.delta);
  const int hshift = 8 * half;
  constexpr int CB = chunk_bytes<R>();
  const bool store_out = !ONE_PASS && (gl == GC - 1) && (P < passes_total - 1);
  const bool from_prev = !ONE_PASS && P > 0;

  uint32_t e[R], t[R];
#pragma unroll
  for (int r = 0; r < R; ++r) { e[r] = nrho; t[r] = 0u; }
  uint32_t y_hr = 0, y_f = 0, y_res = c.padpair;   // (H, F + rho) of this lane's bottom row
  int col = -gl - 1;

  // Lane 0 streams residues (one column ahead) and the previous strip's bottom row through a
  // 4-deep register ring: the loads for step s + 4 are issued while step s is computed, so L2
  // latency is hidden behind four steps of DP work.  Every pair is stored with kPadCols
  // trailing pad columns, so the stream runs branch-free past the last column (clamped to the
  // last pad column): the lanes then compute the DP of the sequence extended by pad letters,
  // whose optimum is the same (a pad column only adds -128 substitutions or gaps, so
  // truncating an alignment at the last real column never lowers its score).  The previous
  // strip's last lane wrote columns -1 .. steps - GC - 1; later columns reuse the last one
  // (bounded, legitimate DP values of the extended matrix).
  const int cmax = ncols + kPadCols - 1;
  const int rlast = steps - GC - 1;
  // two 4-deep rings (A: this group's steps, B: the next group's), top boundary H[0][j] = 0,
  // F[0][j] + rho <= 0 when there is no previous strip
  uint32_t rrA[4], rhA[4], rfA[4], rrB[4], rhB[4], rfB[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) { rhA[k] = rfA[k] = rhB[k] = rfB[k] = 0; rrA[k] = rrB[k] = c.padpair; }
  TagT known = 0;       // team mode: last progress value seen for strip P - 1
  // Every lane of the chain runs the fetch (same addresses as its lane 0: broadcast loads, no
  // extra traffic) so the warp never diverges; only lane 0 consumes the values.  One fetch per
  // group of 4 steps (lane-0 columns c0 .. c0 + 3), one team-mode wait per group: a
  // warp-uniform spin on a shared-memory flag (a divergent spin makes every later shuffle take
  // the slow diverged path).
  // GPU_FLAGS: the tagged words of a group are loaded two groups ahead (gload right after
  // the ring's previous group was checked and unpacked) and their tags are checked only when
  // the group is about to run (gensure): the load latency hides behind two groups of DP work,
  // and the wait is for the data the group needs (the producer's column c0 + 3)
  constexpr unsigned long long kTagBits = 0x8000800080008000ull;
  auto tag_bits = [](uint32_t tg) -> unsigned long long {   // 4-bit tag -> bit 15 of each half
    return ((unsigned long long)(tg & 1) << 15) | ((unsigned long long)((tg >> 1) & 1) << 31) |
           ((unsigned long long)((tg >> 2) & 1) << 47) | ((unsigned long long)((tg >> 3) & 1) << 63);
  };
  const unsigned long long want = tag_bits(1u + (uint32_t)(P + 14) % 15u);   // strip P - 1's tag
  const unsigned long long mine = tag_bits(1u + (uint32_t)P % 15u);
  const unsigned long long* gq = reinterpret_cast<const unsigned long long*>(rb_in);
  unsigned long long gA[4], gB[4];
  int c0A = -1, c0B = 3;
  auto gload = [&](unsigned long long (&g)[4], int c0) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int i = min(c0 + k, rlast);
      g[k] = i < 0 ? want : ld_relaxed_gpu_u64(gq + i);
    }
  };
  auto gensure = [&](unsigned long long (&g)[4], uint32_t (&rh)[4], uint32_t (&rf)[4], int& c0) {
    bool ready = true;
#pragma unroll
    for (int k = 0; k < 4; ++k) ready &= (g[k] & kTagBits) == want;
    while (!ready) {
      __nanosleep(32);
      gload(g, c0);
      ready = true;
#pragma unroll
      for (int k = 0; k < 4; ++k) ready &= (g[k] & kTagBits) == want;
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const unsigned long long v = g[k] & ~kTagBits;
      rh[k] = (uint32_t)v; rf[k] = (uint32_t)(v >> 32);
    }
    c0 += 8;
    gload(g, c0);   // the ring's next group (two groups ahead)
  };
  if constexpr (GPU_FLAGS) {
    if (from_prev) { gload(gA, c0A); gload(gB, c0B); }
  }
  auto fetch_group = [&](uint32_t (&rr)[4], uint32_t (&rh)[4], uint32_t (&rf)[4], int c0) {
#pragma unroll
    for (int k = 0; k < 4; ++k) rr[k] = cols[min(c0 + k + 1, cmax)];
    if constexpr (GPU_FLAGS) return;
    if (from_prev) {
      if constexpr (TEAM) {
        const TagT need = tag_prev | (TagT)(min(c0 + 3, rlast) + 1);
        while (known < need) {
          if constexpr (GPU_FLAGS) known = ld_acquire_gpu(prog_in);
          else known = ld_acquire_smem(prog_in);
          if (known < need) __nanosleep(32);
        }
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint2 v = rb_in[min(c0 + k, rlast)];
        rh[k] = v.x; rf[k] = v.y;
      }
    }
  };

  auto step = [&](auto kc, const uint32_t (&rr)[4], const uint32_t (&rh)[4], const uint32_t (&rf)[4]) {
    constexpr int K = decltype(kc)::value;
    uint32_t x_hr = __shfl_up_sync(SWB_FULL, y_hr, 1, GC);
    uint32_t x_f = __shfl_up_sync(SWB_FULL, y_f, 1, GC);
    uint32_t x_res = __shfl_up_sync(SWB_FULL, y_res, 1, GC);
    if constexpr (ONE_PASS) {
      const uint32_t not0 = gl == 0 ? 0u : 1u;
      x_hr *= not0; x_f *= not0;     // (IMAD: the boundary row is 0 for the first lane)
      if (gl == 0) x_res = rr[K];
    } else {
      if (gl == 0) { x_hr = rh[K]; x_f = rf[K]; x_res = rr[K]; }
      if constexpr (TAG_SHIFT == kPackedTagShift) { x_hr *= keep; x_f *= keep; }   // (IMAD) packed stream
    }
    // query-profile words for the two letters of the NEXT column (look-ahead u)
    uint32_t wlo[(R + 3) / 4], whi[(R + 3) / 4];
    if constexpr (L::kSeqs == 2) {
      // letter offsets with FMA-pipe ops only: a_hi = x >> 8 as IMAD.HI, a_lo = x - 256 a_hi
      const int ahi = (int)__umulhi(x_res, c.hi_mul);
      const int off_hi = ahi * ls;
      load_prof<R, CB, GC * CB>(wlo, prow + ((int)x_res * ls - off_hi * 256));
      load_prof<R, CB, GC * CB>(whi, prow + hi_off + off_hi);
    } else {
      const int alo = (x_res >> hshift) & 0xff;
      load_prof<R, CB, GC * CB>(wlo, prow + alo * ls);
    }
    uint32_t hup = x_hr, fs = x_f;
    cell_rows<L, R, CC::kWide, CHAIN2>(e, t, wlo, whi, nrho, prho, nsig, hup, fs, best, dlt);
    y_hr = hup; y_f = fs; y_res = x_res;
    // last lane: save the strip's bottom row for the next strip (not after the last strip);
    // fill steps write neutral values (index -1 keeps its neutral entry) that the real column
    // overwrites later.
    if constexpr (GPU_FLAGS) {
      if (store_out && col >= 0) {
        const unsigned long long v = ((unsigned long long)y_f << 32 | y_hr) & ~kTagBits;
        st_relaxed_gpu_u64(reinterpret_cast<unsigned long long*>(rb_out) + col, v | mine);
      }
    } else if (store_out) {
      rb_out[max(col, -1)] = make_uint2(y_hr, y_f);
    }
    ++col;
  };
  // team mode: publish this strip's progress when a group crossed a multiple of PUB columns (16
  // in team mode, 4 = every group in T-mode) or reached the last one (release: the row-buffer
  // stores are visible first).  Measured: every group is +5 % on C3 with query 144 in T-mode
  // (short sweeps of the query: the next warp's wait is a larger share of each strip,
  // profiles/r01_pub_granularity.txt); team mode keeps 16.
  auto publish = [&]() {
    if (TEAM && !GPU_FLAGS && store_out) {
      const int done = col;   // the last lane's columns < col are stored
      if (done > 0 && (PUB == 4 || (done & 15) < 4 || done > rlast))
      {
        if constexpr (GPU_FLAGS) st_release_gpu(prog_out, tag_base | (TagT)min(done, rlast + 1));
        else st_release_smem(prog_out, tag_base | (TagT)min(done, rlast + 1));
      }
    }
  };

  // steps is a multiple of 4 (>= ncols + GC, <= ncols + kPadCols); extra steps only see pad
  // columns.  Lane 0's column at step s is s - 1.
  fetch_group(rrA, rhA, rfA, -1);
  for (int s = 0; s < steps; s += 8) {
    fetch_group(rrB, rhB, rfB, s + 3);
    if constexpr (GPU_FLAGS) { if (from_prev) gensure(gA, rhA, rfA, c0A); }
    step(std::integral_constant<int, 0>{}, rrA, rhA, rfA);
    step(std::integral_constant<int, 1>{}, rrA, rhA, rfA);
    step(std::integral_constant<int, 2>{}, rrA, rhA, rfA);
    step(std::integral_constant<int, 3>{}, rrA, rhA, rfA);
    publish();
    if (s + 4 >= steps) break;
    fetch_group(rrA, rhA, rfA, s + 7);
    if constexpr (GPU_FLAGS) { if (from_prev) gensure(gB, rhB, rfB, c0B); }
    step(std::integral_constant<int, 0>{}, rrB, rhB, rfB);
    step(std::integral_constant<int, 1>{}, rrB, rhB, rfB);
    step(std::integral_constant<int, 2>{}, rrB, rhB, rfB);
    step(std::integral_constant<int, 3>{}, rrB, rhB, rfB);
    publish();
  }
  return best;
}

// emit the score(s) of one chain result; s16x2: both sequences of the pair
template <class L>
__device__ __forceinline__ void emit(const SearchParams& p, uint32_t b, int pair, int half) {
  if constexpr (L::kSeqs == 2) {
    const int limit = p.flag_limit;
    const int s0 = 2 * pair, s1 = 2 * pair + 1;
    const int lo = (int)(int16_t)(b & 0xffffu), hi = (int)(int16_t)(b >> 16);
    if (lo >= limit) p.ovf_list[atomicAdd(p.ovf_count, 1)] = s0; else p.scores[p.perm[s0]] = lo;
    if (s1 < p.n_seqs) {
      if (hi >= limit) p.ovf_list[atomicAdd(p.ovf_count, 1)] = s1; else p.scores[p.perm[s1]] = hi;
    }
  } else {
    const int s = 2 * pair + half;
    p.scores[p.perm[s]] = (int)b;
  }
}

// Continuous group stream for whole-warp chains (G = 32, one pair per chain).  run_pass
// gives every (pair, strip) its own sweep: the chain fills for 31 steps and drains for 31 more,
// ~8 % of the lane-steps at Swiss-Prot lengths.  Here the strips and pairs a warp takes form
// ONE column stream (§VI: process the strips "in a single pass ... the pipeline
// only has to be filled and flushed once"): lane l processes stream position t - l at step t,
// so lane 0 starts the next segment (strip or pair) while the other lanes still finish the
// previous one.  Every segment starts with a gap of 4 pad positions (segment lengths are
// multiples of 4, so the gap is exactly the fetch set of one 4-step group); a lane moves into
// the next segment (resets its rows to the neutral state, c4) at the 4-step group boundary that
// falls inside its gap window, so the 4-step body stays branch-free.  In the gap:
//  * a lane that already switched sees pad letters and neutral vertical input (below), stays
//    exactly neutral and reaches the real columns in the neutral state;
//  * a lane that has not switched yet ("stale") computes pad cells from its old state; their H
//    cannot exceed the old segment's maximum (a pad column only adds -128 or gap costs);
//  * resets happen only at group boundaries and a lane's gap window starts one step after the
//    lane above's, so a switched lane can receive a stale value only at the boundary where both
//    switch, from the upper lane's last step: that lane neutralises its outgoing (H, F + rho)
//    as it switches.
// Segments are >= kMinCols + 4 = 52 positions, so at most two are in flight, and the strip
// hand-off is ordered: lane 31 writes row-buffer column j at step T + 4 + 31 + j, lane 0
// fetches it for the next strip at step T + len + 4 + j >= T + 52 + j (__syncwarp every group
// in between).  A pair's score is reduced across the lanes once its last lane has moved on
// (each lane parks its maximum in bdone when it leaves the pair's last strip).
// Warp-uniform scheduler state of group_stream, kept in shared memory (one per warp): it is
// touched once per 4-step group, and keeping it out of registers leaves the register file to
// the R-row DP state (e[R], u[R], profile words): no spills at R = 43 with 3 warps per
// scheduler.  Every lane executes the same updates (same addresses and values).
struct GsState {
  int64_t f_off;    // column offset of the pair being fetched (u16 units)
  int64_t nx_off;   // prefetched next pair's column offset
  int f_pair, f_len, f_P, f_col, f_seg;
  int nx_pair, nx_len;
  int pending, e_pair, e_due;
  uint32_t desc[2];
};

// MULTI = false: the query fits one strip (p.short_passes == 1), so there is no strip row
// buffer: the first lane's top input is the constant boundary (H, F + rho) = (0, 0) and only
// the residues go through the fetch ring (8 registers and 2 selects per step fewer).
template <class L, int R, bool MULTI, class CC>
__device__ __forceinline__ void group_stream(const SearchParams& p, const CC& c, const uint8_t* pbase,
                                             uint2* __restrict__ rb, volatile GsState* gs) {
  static_assert(R % 4 == 0 || R >= 12, "R < 12 must be a multiple of 4");
  constexpr int kGap = 4;
  const int lane = threadIdx.x & 31;
  const uint32_t not0 = lane == 0 ? 0u : 1u;
  const uint32_t nrho = L::splat(-c.rho), prho = L::splat(c.rho);
  const uint32_t nsig = L::splat(-c.sigma);
  const uint32_t dlt = L::splat(c.delta);
  constexpr int CB = chunk_bytes<R>();
  constexpr int kStripBytes = chunks_per_lane<R>() * 32 * CB;   // chunks x 32 lanes x CB bytes
  constexpr int kEndLen = 0xffffff;            // the END segment (after the last pair) never ends
  const int passes = p.short_passes;
  const int ls = p.lg.ls, ls256 = ls * 256;
  const uint32_t hi_mul = p.hi_mul;

  // ---- warp-uniform fetch cursor: lane 0's stream, one group (4 positions) ahead of lane 0
  auto prefetch = [&]() {   // next pair of the queue (its header loads overlap the current pair)
    int item = 0;
    if (lane == 0) item = atomicAdd(&p.work[1], 1);
    item = __shfl_sync(SWB_FULL, item, 0);
    if (item < p.n_pairs - p.short_begin) {
      const int pr = p.short_begin + item;
      gs->nx_pair = pr;
      gs->nx_off = p.pair_off[pr];
      gs->nx_len = p.pair_ncols[pr] + kGap;
    } else {
      gs->nx_pair = -1; gs->nx_len = kEndLen;
    }
    __syncwarp();
  };
  prefetch();
  if (gs->nx_pair < 0) return;
  gs->f_pair = gs->nx_pair; gs->f_len = gs->nx_len; gs->f_P = 0; gs->f_col = 0;
  gs->f_off = gs->nx_off;
  // descriptors (len | (P + 1) << 24) of the two newest segments, by segment parity
  gs->desc[0] = (uint32_t)gs->f_len | (1u << 24); gs->desc[1] = 0;
  gs->f_seg = 0;
  gs->pending = 0;            // a finished pair waits for its cross-lane reduction
  gs->e_pair = 0; gs->e_due = 0;
  gs->nx_pair = -2;           // -2: the next pair is not fetched yet
  __syncwarp();
  if (passes == 1) prefetch();
  // this group's 4 fetches: residues g_cols[k] and top-boundary rows g_rb[k]
  const uint16_t* g_cols;
  const uint2* g_rb;
  // Plain groups: most groups only advance the fetch cursor by 4 positions inside a segment.
  // plan_group (the full, shared-memory scheduler step) runs for a group that starts a segment,
  // ends the stream, is due to emit a finished pair, or follows a gap group; it then counts the
  // plain groups that follow (quiet) and pre-commits the cursor they reach, and the loop
  // advances g_cols / g_rb in registers for those (ncu on query 5478: the per-group scheduler
  // was 8.9 % of the warp samples of the step loop).
  // (measured on C2, T = 3072, one kernel per stream variant (k_search GS): query 729 / 1500
  // 24.08 / 47.27 -> 23.37 / 45.86 ms; query 5478 over the autotune's candidates R = 44 / 35 /
  // 45 / 46: 180.4 / 181.1 / 183.9 / 192.3 -> 175.4 / 177.1 / 182.4 / 186.6 ms, R = 43 174.0 ->
  // 174.9 ms — the step code's register allocation moves by ~1-2 % with any change to the loop)
  constexpr bool kPlain = true;
  int quiet = 0;
  int rb_inc = 0;             // 4 when the plain groups read the previous strip's row buffer
  // fn: index of the next fetch (= the stream position at which lane 0 consumes it); S: the
  // stream position of lane 0 at the start of the group (pending emissions are checked then)
  auto plan_group = [&](int fn, int S) {   // warp-uniform
    int f_pair = gs->f_pair, f_len = gs->f_len, f_P = gs->f_P, f_col = gs->f_col;
    if (f_col == f_len) {     // the next segment starts: this group fetches its gap
      if (f_P + 1 < passes) {
        ++f_P;
      } else {
        gs->pending = 1; gs->e_pair = f_pair; gs->e_due = fn + 35;
        __syncwarp();
        if (gs->nx_pair == -2) prefetch();
        if (gs->nx_pair >= 0) {
          f_pair = gs->nx_pair; f_len = gs->nx_len; gs->f_off = gs->nx_off; f_P = 0;
          gs->nx_pair = -2;
          __syncwarp();
          if (passes == 1) prefetch();
        } else {
          f_pair = -1; f_len = kEndLen; f_P = -1;   // END: gap positions for ever
        }
      }
      if (f_pair >= 0 && f_P == passes - 1 && passes > 1) prefetch();
      f_col = 0;
      const int f_seg = gs->f_seg + 1;
      gs->f_seg = f_seg;
      gs->desc[f_seg & 1] = (uint32_t)f_len | ((uint32_t)(f_P + 1) << 24);
      gs->f_pair = f_pair; gs->f_len = f_len; gs->f_P = f_P;
    }
    // residues one position ahead (look-ahead u, cell_rows): position f_col + k reads the
    // letters of column f_col + k - kGap + 1; in the gap that is the pad column(s) stored just
    // before the pair (kLeadCols / the previous pair's trailing pads), then its first column.
    // END: pad letters (the last pair's trailing pad columns, still at f_off + f_len).
    const uint16_t* f_cols = p.cols + gs->f_off;
    if (f_pair < 0) {
      g_cols = f_cols + p.pair_ncols[gs->e_pair];
      g_rb = p.rb_zero;
    } else {
      g_cols = f_cols + (f_col - kGap + 1);
      g_rb = (f_col >= kGap && f_P > 0) ? rb + (f_col - kGap) : p.rb_zero;
      if constexpr (kPlain) {
        // the groups after this one fetch f_col + 4, f_col + 8, ... < f_len: plain unless this
        // is the gap group (the next one switches g_rb from rb_zero to the row buffer) or a
        // pending emission falls due (the first group with S' >= e_due must run the full step)
        rb_inc = f_P > 0 ? 4 : 0;
        quiet = 0;
        if (f_col >= kGap) {
          quiet = (f_len - f_col - 4) >> 2;
          if (gs->pending) quiet = min(quiet, max(0, (gs->e_due - S - 1) >> 2));
        }
      }
    }
    if (f_pair >= 0) gs->f_col = f_col + 4 + 4 * quiet;
    __syncwarp();
  };
  uint32_t ring_res[4], ring_h[4], ring_f[4];
  auto fetch = [&](int k) {
    ring_res[k] = g_cols[k];
    if constexpr (MULTI) {
      const uint2 v = g_rb[k];
      ring_h[k] = v.x; ring_f[k] = v.y;
    }
  };

  // ---- per-lane state (look-ahead form, cell_rows)
  uint32_t e[R], t[R];
#pragma unroll
  for (int r = 0; r < R; ++r) { e[r] = nrho; t[r] = 0u; }
  uint32_t y_hr = 0, y_f = 0, y_res = c.padpair;
  uint32_t best = 0, bdone = 0;
  int my_pos = -lane, my_len = 0, my_P = -1, my_seg = -1;   // lane l reaches segment 0 at step l
  const uint8_t* prow = pbase;
  bool store_rb = false;      // lane 31 in a strip whose bottom row feeds the next strip

  plan_group(0, -4);
#pragma unroll
  for (int k = 0; k < 4; ++k) fetch(k);

  auto step = [&](auto kc) {
    constexpr int K = decltype(kc)::value;
    uint32_t x_hr = __shfl_up_sync(SWB_FULL, y_hr, 1);
    uint32_t x_f = __shfl_up_sync(SWB_FULL, y_f, 1);
    uint32_t x_res = __shfl_up_sync(SWB_FULL, y_res, 1);
    if constexpr (MULTI) {
      if (lane == 0) { x_hr = ring_h[K]; x_f = ring_f[K]; x_res = ring_res[K]; }
    } else {
      x_hr *= not0; x_f *= not0;     // (IMAD: the boundary row is 0 for the first lane)
      if (lane == 0) x_res = ring_res[K];
    }
    uint32_t wlo[(R + 3) / 4], whi[(R + 3) / 4];   // profile words of the next position's letters
    {
      // letter offsets with FMA-pipe ops only: a_hi = x >> 8 as IMAD.HI, a_lo = x - 256 a_hi
      const int ahi = (int)__umulhi(x_res, hi_mul);
      const int off_hi = ahi * ls;
      const int off_lo = (int)x_res * ls - ahi * ls256;
      load_prof<R, CB, 32 * CB>(wlo, prow + off_lo);
      load_prof<R, CB, 32 * CB>(whi, prow + off_hi);
    }
    fetch(K);
    uint32_t hup = x_hr, fs = x_f;
    cell_rows<L, R, CC::kWide>(e, t, wlo, whi, nrho, prho, nsig, hup, fs, best, dlt);
    y_hr = hup; y_f = fs; y_res = x_res;
    // keep the next step's residue shuffle (and so its profile loads) after this step's rows:
    // hoisting them would keep a second set of profile words live
    asm volatile("" : "+r"(y_res) : "r"(fs));
    // unconditional for the storing lane: gap positions land in the slot's kGap leading
    // entries, stale positions past the segment beyond its columns; neither is ever read
    if (store_rb) rb[my_pos + K - kGap] = make_uint2(hup, fs);
  };

  for (int S = 0;; S += 4) {
    // switch segments: a lane whose position entered the next segment's gap
    if (my_pos >= my_len) {
      if (my_pos > my_len) { y_hr = 0u; y_f = 0u; }   // last step was a stale gap cell
      ++my_seg;
      const uint32_t d = gs->desc[my_seg & 1];
      if (my_P == passes - 1) { bdone = best; best = 0; }
      my_pos -= my_len;
      my_len = (int)(d & (uint32_t)kEndLen);
      my_P = (int)(d >> 24) - 1;
      store_rb = MULTI && lane == 31 && my_P >= 0 && my_P < passes - 1;
      prow = pbase + max(my_P, 0) * kStripBytes;
#pragma unroll
      for (int r = 0; r < R; ++r) { e[r] = nrho; t[r] = 0u; }
    }
    __syncwarp();   // (also orders lane 31's row-buffer stores before lane 0's later loads)
    if (kPlain && quiet > 0) {   // plain group (warp-uniform): advance the fetch cursor only
      --quiet;
      g_cols += 4;
      g_rb += rb_inc;
    } else {
      if (gs->pending && S >= gs->e_due) {   // every lane has parked the finished pair's maximum
        uint32_t b = bdone;
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
        if (lane == 0) emit<L>(p, b, gs->e_pair, 0);
        __syncwarp();
        gs->pending = 0;
      }
      if (gs->f_pair < 0 && !gs->pending) break;
      plan_group(S + 4, S);   // the 4 fetches issued during this group (consumed in the next one)
    }
    step(std::integral_constant<int, 0>{});
    step(std::integral_constant<int, 1>{});
    step(std::integral_constant<int, 2>{});
    step(std::integral_constant<int, 3>{});
    my_pos += 4;
  }
}

// GS: which group-stream variants the kernel contains (G = 32): 0 = both, chosen per launch by
// p.short_passes; 1 = the single-strip stream only; 2 = the multi-strip stream only.  The
// launcher compiles and picks 1 / 2 separately, so that each stream loop gets the kernel's
// registers and instruction cache to itself (the two loops in one kernel shared one register
// allocation: a change to one moved the other's timing by up to 2 %).
template <class L, int G, int Rs, int Rl, int NT, bool WIDE = false, int GS = 0>
__global__ void __launch_bounds__(NT, 1) k_search(const SearchParams p) {
  constexpr int kWarps = NT / 32;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t sprog[2 * kWarps];
  __shared__ uint32_t sred[kWarps];
  __shared__ int32_t sitem[kWarps];

  // the 32-bit recompute launch exits at once when no sequence was flagged
  if (p.item_list != nullptr && *p.item_count == 0) return;

  // ---- stage the query profile in shared memory with TMA bulk copies (§III-B:
  //      the profile lives in texture memory there; on sm_100a it is smem-resident)
  if (threadIdx.x == 0) {
    mbar_init(&mbar, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    mbar_expect_tx(&mbar, (uint32_t)p.prof_bytes);
    constexpr int kChunk = 32768;
    for (int off = 0; off < p.prof_bytes; off += kChunk) {
      const int sz = min(kChunk, p.prof_bytes - off);
      bulk_g2s(smem + off, p.prof + off, (uint32_t)sz, &mbar);
    }
  }
  mbar_wait(&mbar, 0);

  ChainConstT<WIDE> c;
  c.rho = p.rho;
  c.sigma = p.sigma;
  c.delta = p.delta;
  c.padpair = (uint32_t)p.pad_letter | ((uint32_t)p.pad_letter << 8);
  c.hi_mul = p.hi_mul;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  // ---- phase 1: TEAM (intra-task) items — long sequences, or the 32-bit recompute list
  {
    const int W = p.team_warps;
    const int nteams = kWarps / W;
    const int team = warp / W, wt = warp % W;
    if (team < nteams) {
      uint32_t* prog = sprog + team * (W + 1);
      const int n_items = p.item_list ? *p.item_count : p.n_long;
      for (;;) {
        team_bar(team, W);
        if (wt == 0 && lane == 0) {
          sitem[team] = atomicAdd(&p.work[0], 1);
          for (int i = 0; i <= W; ++i) prog[i] = 0u;
        }
        team_bar(team, W);
        const int item = sitem[team];
        if (item >= n_items) break;
        int pair = item, half = 0;
        if (p.item_list) {
          const int sq = p.item_list[item];
          pair = sq >> 1;
          half = sq & 1;
        }
        const int ncols = p.pair_ncols[pair];
        const uint16_t* cp = p.cols + p.pair_off[pair];
        uint2* rb = p.rb_team + ((int64_t)(blockIdx.x * nteams + team) * (W + 1)) * p.rb_team_cols;
        // One strip per chain sweep (fill + flush per strip).  A warp must not start strip
        // P + W before all its lanes finished strip P: its lane 0 may wait for strip P + W - 1,
        // which transitively needs the tail of strip P (deadlock for short rows otherwise).
        uint32_t b = 0;
        const int tsteps = (ncols + 32 + 3) & ~3;
        for (int P = wt; P < p.long_passes; P += W) {
          const int si = (P + W) % (W + 1), so = P % (W + 1);   // slot of strip P-1 / strip P
          constexpr int CBl = chunk_bytes<Rl>();
          const uint8_t* prow = smem + p.lt.off + (P * chunks_per_lane<Rl>() * 32 + lane) * CBl;
          b = run_pass<L, 32, Rl, true>(c, prow, p.lt.ls, 0, cp, ncols, half, tsteps, P, p.long_passes,
                                        rb + (int64_t)si * p.rb_team_cols + 1, rb + (int64_t)so * p.rb_team_cols + 1,
                                        prog + si, prog + so, b);
        }
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
        if (lane == 0) sred[warp] = b;
        team_bar(team, W);
        if (wt == 0 && lane == 0) {
          uint32_t bb = sred[team * W];
          for (int i = 1; i < W; ++i) bb = L::max2(bb, sred[team * W + i]);
          emit<L>(p, bb, pair, half);
        }
      }
    }
  }

  // ---- phase 2: GROUP (inter-task) items — short sequences, G lanes per pair
  if constexpr (G == 32) {
    if (p.item_list == nullptr && p.group_stream) {
      constexpr int CBs = chunk_bytes<Rs>();
      __shared__ GsState sgs[kWarps];
      uint2* rbw = p.rb_group + (int64_t)(blockIdx.x * kWarps + warp) * p.rb_group_cols + 4;
      if constexpr (GS == 2) {
        group_stream<L, Rs, true>(p, c, smem + p.lg.off + lane * CBs, rbw, &sgs[warp]);
      } else if constexpr (GS == 1) {
        group_stream<L, Rs, false>(p, c, smem + p.lg.off + lane * CBs, rbw, &sgs[warp]);
      } else {
        if (p.short_passes > 1) group_stream<L, Rs, true>(p, c, smem + p.lg.off + lane * CBs, rbw, &sgs[warp]);
        else group_stream<L, Rs, false>(p, c, smem + p.lg.off + lane * CBs, rbw, &sgs[warp]);
      }
      return;
    }
  }
  if (p.item_list == nullptr) {
    constexpr int GPW = 32 / G;
    const int gi = lane / G, gl = lane & (G - 1);
    const int nshort = p.n_pairs - p.short_begin;
    for (;;) {
      int base = 0;
      if (lane == 0) base = atomicAdd(&p.work[1], GPW);
      base = __shfl_sync(SWB_FULL, base, 0);
      if (base >= nshort) break;
      const bool valid = base + gi < nshort;
      const int pair = p.short_begin + base + gi;
      const int ncols = valid ? p.pair_ncols[pair] : 0;
      const uint16_t* cp = p.cols + (valid ? p.pair_off[pair] : 0);
      const int steps = ((int)__reduce_max_sync(SWB_FULL, (unsigned)ncols) + G + 3) & ~3;
      uint2* rb = p.rb_group + ((int64_t)(blockIdx.x * kWarps + warp) * GPW + gi) * p.rb_group_cols;
      uint32_t b = 0;
      if (p.short_passes == 1) {
        constexpr int CBs = chunk_bytes<Rs>();
        const uint8_t* prow = smem + p.lg.off + gi * p.lg.rs + gl * CBs;
        b = run_pass<L, G, Rs, false, 16, false, 20, true>(c, prow, p.lg.ls, 0, cp, ncols, 0, steps, 0, 1, rb + 1,
                                                            rb + 1, (uint32_t*)nullptr, (uint32_t*)nullptr, b);
      } else {
        for (int P = 0; P < p.short_passes; ++P) {
          constexpr int CBs = chunk_bytes<Rs>();
          const uint8_t* prow = smem + p.lg.off + gi * p.lg.rs + (P * chunks_per_lane<Rs>() * G + gl) * CBs;
          b = run_pass<L, G, Rs, false>(c, prow, p.lg.ls, 0, cp, ncols, 0, steps, P, p.short_passes, rb + 1, rb + 1,
                                        (uint32_t*)nullptr, (uint32_t*)nullptr, b);
          __syncwarp();   // strip P's bottom row (written by lane G-1) is read by lane 0 in strip P+1
        }
      }
#pragma unroll
      for (int o = G / 2; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
      if (gl == 0 && valid) emit<L>(p, b, pair, 0);
    }
  }
}

// ------------------------------------------------------------------------------------ T-mode
// Long database sequences, transposed.  The paper's
// intra-task kernel gives one thread block to one long sequence and walks strips of QUERY rows
// (§III, Fig.4).  Here a CTA team walks strips of the DATABASE sequence instead:
// lane l of warp w owns C consecutive database positions of strip s = w, w + W, ..., and the
// chain sweeps the query, so a 35k-residue sequence yields ~70 strips of parallel work for any
// query length.  Eq.(1) is symmetric under transposition (E <-> F, w(q, d) read as w^T(d, q)),
// so the same engine (run_pass) computes it; the "profile" of a strip is built by its warp
// from the substitution matrix (tables P_lo[a][pos] = w(a, d_lo[pos]) + rho and P_hi for the
// pair's second sequence, chunk-major and conflict-free like the query profile) and the
// residue stream is the query.  Strip boundaries (the last database position of a strip over
// all query positions) go through the team row buffers with progress flags, as in team mode.
// One T-mode team (W warps) processing long pairs until the queue is exhausted.  first_item:
// an item already taken for this team (or -1).  max_strips: a team of W warps only keeps items
// with at most this many strips (> max_strips: the item is parked in *parked and the loop
// returns, so that the CTA can regroup into smaller teams for the remaining, shorter items).
// Build warp's strip tables for strip P of a long pair: position pos = P*LS + lane*C + r;
// P_lo[a][pos] = w(a, d_lo[pos]) + rho (a = compact query letter), P_hi likewise, chunk-major
// and lane-private like the query profile (every lane writes and later reads only its chunks).
// SEQS = 1 (32-bit recompute of one flagged sequence): only P_lo, for the pair's half-th sequence.
// pos0: the lane's first database position (P * 32C + lane * C for the strips of one pair; in
// the packed team stream every lane has its own pair, cp and position); ncols <= 0: pad lane.
template <int C, int SEQS = 2>
__device__ __forceinline__ void build_strip_tables(const TParams& p, uint8_t* tab, const int8_t* wp,
                                                   const uint16_t* cp, int ncols, int pos0, int half = 0) {
  constexpr int CB = chunk_bytes<C>();
  constexpr int LS = 32 * C;
  const int lane = threadIdx.x & 31;
  const int A1 = p.A_used + 1;
  const uint32_t db_pad = (uint32_t)p.pad_letter * 0x101u;
  __syncwarp();
  uint32_t dp[C];
#pragma unroll
  for (int r = 0; r < C; ++r) {
    const int pos = pos0 + r;
    dp[r] = pos < ncols ? (uint32_t)cp[pos] : db_pad;
  }
  for (int a = 0; a < A1; ++a) {
    const int8_t* wrow = wp + a * kWpStride;
#pragma unroll
    for (int k = 0; k < C / 4; ++k) {
      uint32_t lo = 0, hi = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t d = dp[4 * k + j];
        if constexpr (SEQS == 2) {
          lo |= (uint32_t)(uint8_t)wrow[d & 0xff] << (8 * j);
          hi |= (uint32_t)(uint8_t)wrow[d >> 8] << (8 * j);
        } else {
          lo |= (uint32_t)(uint8_t)wrow[(d >> (8 * half)) & 0xff] << (8 * j);
        }
      }
      const int r0 = 4 * k;
      const int off = a * LS + ((r0 / CB) * 32 + lane) * CB + (r0 % CB);
      *reinterpret_cast<uint32_t*>(tab + off) = lo;
      if constexpr (SEQS == 2) *reinterpret_cast<uint32_t*>(tab + A1 * LS + off) = hi;
    }
  }
  __syncwarp();
}

// scores of long pair `item` from its reduced s16x2 maximum (or its overflow flags)
__device__ __forceinline__ void emit_t(const TParams& p, uint32_t bb, int item) {
  const int limit = p.flag_limit;
  const int s0 = 2 * item, s1 = 2 * item + 1;
  const int lo = (int)(int16_t)(bb & 0xffffu), hi = (int)(int16_t)(bb >> 16);
  if (lo >= limit) p.ovf_list[atomicAdd(p.ovf_count, 1)] = s0; else p.scores[p.perm[s0]] = lo;
  if (s1 < p.n_seqs) {
    if (hi >= limit) p.ovf_list[atomicAdd(p.ovf_count, 1)] = s1; else p.scores[p.perm[s1]] = hi;
  }
}

// exact 32-bit score of sequence position sq (T-mode recompute of a flagged sequence)
__device__ __forceinline__ void emit_t32(const TParams& p, int score, int sq) { p.scores[p.perm[sq]] = score; }

// One T-mode team (W warps) processing long pairs until the queue is exhausted.  first_item:
// an item already taken for this team (or -1).  min_strips: a team of W warps only keeps items
// with at least this many strips (fewer: the item is parked in *parked and the loop returns,
// so that the CTA can regroup into smaller teams for the remaining, shorter items).  Items
// [0, gang_items) belong to the gangs (t_gang_item), [0, q0) to the gangs or the row-scan
// launches (sw_scan.cu); the queue starts at q0.
template <int C, class CC>
__device__ __forceinline__ void t_team_loop(const TParams& p, const CC& c, uint8_t* tab,
                                            const int8_t* wp, int W, int team, int wt, int first_item,
                                            int min_strips, int* parked, uint32_t* prog, uint2* rb,
                                            int32_t* sitem, uint32_t* sred) {
  using L = LaneS16x2;
  constexpr int CB = chunk_bytes<C>();
  constexpr int LS = 32 * C;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int A1 = p.A_used + 1;                 // compact query letters + the pad row
  const int qsteps = (p.qcols + 32 + 3) & ~3;
  int pending = first_item;
  for (;;) {
    team_bar(team, W);
    if (wt == 0 && lane == 0) {
      const int it = pending >= 0 ? pending : p.q0 + atomicAdd(p.work, 1);
      sitem[team] = it;
      for (int i = 0; i <= W; ++i) prog[i] = 0u;
    }
    pending = -1;
    team_bar(team, W);
    const int item = sitem[team];
    if (item >= p.n_items) return;
    const int ncols = p.pair_ncols[item];
    const int S = (ncols + LS - 1) / LS;       // strips of the database pair
    if (S < min_strips) {                      // too short for this team size: hand it back
      if (wt == 0 && lane == 0) *parked = item;
      return;
    }
    const uint16_t* cp = p.cols + p.pair_off[item];
    uint32_t b = 0;
    for (int P = wt; P < S; P += W) {
      build_strip_tables<C>(p, tab, wp, cp, ncols, P * LS + lane * C);
      const int si = (P + W) % (W + 1), so = P % (W + 1);
      b = run_pass<L, 32, C, true, 4>(c, tab + lane * CB, LS, A1 * LS, p.qpair, p.qcols, 0, qsteps, P, S,
                                     rb + (int64_t)si * p.rb_cols + 1, rb + (int64_t)so * p.rb_cols + 1, prog + si,
                                     prog + so, b);
    }
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
    if (lane == 0) sred[warp] = b;
    team_bar(team, W);
    if (wt == 0 && lane == 0) {
      uint32_t bb = sred[team * W];
      for (int i = 1; i < W; ++i) bb = L::max2(bb, sred[team * W + i]);
      emit_t(p, bb, item);
    }
  }
}

// T-mode team STREAM (phase 2): the strips of the pairs a team takes form one running strip
// sequence g = 0, 1, 2, ... (pair after pair, longest first from the global queue); warp wt of
// the W-warp team processes g = wt, wt + W, ...  A warp that has finished its strips of one
// pair goes straight on to the next pair's, so the team's pipeline is filled and drained once
// per launch instead of once per pair (the per-pair barrier and the (W - 1) x lag fill were
// ~10-20 % of T-mode time for short queries).  Hand-off and flags are the team pipeline's
// (slot g mod (W + 1), tag = g): strip g + 1 consumes strip g's bottom row only inside a pair.
// Each pair's maximum is combined with atomicMax in the team's shared ring of pairs; the
// warp finishing its last strip emits the scores.
// Per-pair team stream (used when the long pairs are a strip or more on average): every pair
// starts a new strip, strips of one pair are chained, a new pair's first strip depends on no
// other strip.  (The packed stream below is used for long sets of mostly short pairs.)
constexpr int kTQ = 16;      // pairs in a team's ring (a team spans at most ~W + 1 of them)
struct TStreamP {
  int lock, count, next, end;
  int item[kTQ], base[kTQ], S[kTQ], rem[kTQ], mlo[kTQ], mhi[kTQ];
};

// L = LaneS32: the 32-bit recompute of the flagged sequences (items = positions of
// p.item_list, one sequence each; long-query mode, where the k_search recompute's query profile
// does not fit shared memory).  Progress tags are 64-bit (running strip index << 32 | columns).
template <int C, class L, class CC>
__device__ __forceinline__ void t_team_stream_pairs(const TParams& p, const CC& c, uint8_t* tab,
                                                    const int8_t* wp, int W, int team, int wt, int first_item,
                                                    unsigned long long* prog, uint2* rb, TStreamP* ts) {
  constexpr bool S32 = L::kSeqs == 1;
  constexpr int CB = chunk_bytes<C>();
  constexpr int LS = 32 * C;
  const int lane = threadIdx.x & 31;
  const int A1 = p.A_used + 1;
  const int qsteps = (p.qcols + 32 + 3) & ~3;
  const int n_items = S32 ? *p.item_count : p.n_items;
  volatile TStreamP* vs = ts;
  // item -> (pair, half): s16x2 items are pairs, s32 items index the flagged-sequence list
  auto pair_of = [&](int item, int* half) {
    if constexpr (S32) {
      const int sq = p.item_list[item];
      *half = sq & 1;
      return sq >> 1;
    } else {
      *half = 0;
      return item;
    }
  };
  auto emit_item = [&](int item, int lo, int hi) {
    if constexpr (S32) emit_t32(p, lo, p.item_list[item]);
    else emit_t(p, ((uint32_t)lo & 0xffffu) | ((uint32_t)hi << 16), item);
  };
  // append one pair to the ring (lane 0 of the warp holding the lock); empty pairs score 0
  auto append = [&](int item) {
    int hf;
    const int S = (p.pair_ncols[pair_of(item, &hf)] + LS - 1) / LS;
    if (S == 0) { emit_item(item, 0, 0); return; }
    const int k = vs->count % kTQ;
    if (vs->count >= kTQ)   // the entry kTQ pairs back must be finished before it is reused
      while (vs->rem[k] != 0) __nanosleep(64);
    vs->item[k] = item; vs->base[k] = vs->next; vs->S[k] = S; vs->rem[k] = S; vs->mlo[k] = 0; vs->mhi[k] = 0;
    __threadfence_block();
    vs->count = vs->count + 1;
    vs->next = vs->next + S;
  };
  team_bar(team, W);
  if (wt == 0 && lane == 0) {
    for (int i = 0; i <= W; ++i) prog[i] = 0u;
    ts->lock = 0; ts->count = 0; ts->next = 0; ts->end = 0;
    if (first_item >= 0) append(first_item);
    __threadfence_block();
  }
  team_bar(team, W);
  for (int g = wt;; g += W) {
    // the ring entry of strip g (lane 0 decides, the warp follows)
    int k = -1;
    if (lane == 0) {
      for (;;) {
        const int next = vs->next, count = vs->count;
        if (g < next) {
          for (int j = count - 1; j >= 0 && j >= count - kTQ; --j) {
            const int kk = j % kTQ;
            if (vs->base[kk] <= g) { k = kk; break; }
          }
          break;
        }
        if (vs->end) break;
        if (atomicCAS(&ts->lock, 0, 1) == 0) {
          while (vs->next <= g && !vs->end) {
            const int item = p.q0 + atomicAdd(p.work, 1);
            if (item >= n_items) { vs->end = 1; break; }
            append(item);
          }
          __threadfence_block();
          atomicExch(&ts->lock, 0);
        } else {
          __nanosleep(64);
        }
      }
    }
    k = __shfl_sync(SWB_FULL, k, 0);
    if (k < 0) break;
    const int item = vs->item[k], P = g - vs->base[k], S = vs->S[k];
    int half;
    const int pair = pair_of(item, &half);
    const int ncols = p.pair_ncols[pair];
    const uint16_t* cp = p.cols + p.pair_off[pair];
    build_strip_tables<C, L::kSeqs>(p, tab, wp, cp, ncols, P * LS + lane * C, half);
    const int si = (g + W) % (W + 1), so = g % (W + 1);
    uint32_t b = run_pass<L, 32, C, true, 4, false, 32>(c, tab + lane * CB, LS, A1 * LS, p.qpair, p.qcols, 0, qsteps,
                                                       P, S, rb + (int64_t)si * p.rb_cols + 1,
                                                       rb + (int64_t)so * p.rb_cols + 1, prog + si, prog + so, 0u, g);
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
    if (lane == 0) {
      if constexpr (S32) {
        atomicMax(&ts->mlo[k], (int)b);
      } else {
        atomicMax(&ts->mlo[k], (int)(int16_t)(b & 0xffffu));
        atomicMax(&ts->mhi[k], (int)(int16_t)(b >> 16));
      }
      __threadfence_block();
      if (atomicSub(&ts->rem[k], 1) == 1) {   // this pair's last strip
        const int lo = atomicAdd(&ts->mlo[k], 0), hi = atomicAdd(&ts->mhi[k], 0);
        emit_item(item, lo, hi);
      }
    }
    __syncwarp();
  }
}

// PACKED: the team's pairs are laid out back to back in LANES of C database positions (a pair
// of n' columns takes ceil(n' / C) lanes) and strip g is the team's lanes [32g, 32g + 32): a
// strip holds the tail of one pair and the heads of the next ones, so short pairs no longer
// leave most of a 32-lane strip idle (a 350-column pair used 22 of 32 lanes).  A lane whose rows
// start a pair takes the neutral boundary instead of the lane above's bottom row (run_pass
// keep), strip g + 1 takes strip g's bottom row only when its first lane continues a pair, and
// every lane folds its maximum into its pair's entry (atomicMax in shared memory); the lane
// that completes a pair's last lane emits its scores.
// Ring capacity: a warp asking for strip g + W has finished strip g, and every strip before g + 1
// is finished (its warp moved on), so the unfinished pairs lie in strips g + 1 .. g + W: at most
// W x 32 / 3 + 1 pairs (>= 3 lanes per pair, n' >= 48).  A ring that small would let the
// appending warp wait for a pair whose lanes sit in a strip that itself waits for the append
// (deadlock), so each team gets cap = kTPool / teams >= 32 W / 3 + 2 entries of a per-CTA pool.
constexpr int kTPool = 112;
struct TStream {
  int lock, count, next, end;   // next: lanes appended so far
  int pend, pend_end;           // queue items taken (kTGrab at a time) but not appended yet
};
constexpr int kTGrab = 8;       // queue items per global atomic
struct TPool {
  int item[kTPool], base[kTPool], nl[kTPool], rem[kTPool], mlo[kTPool], mhi[kTPool];
};

// L = LaneS32: the 32-bit recompute of the flagged sequences (items = positions of
// p.item_list, one sequence each; long-query mode, where the k_search recompute's query profile
// does not fit shared memory).  Progress tags are 64-bit (running strip index << 32 | columns).
template <int C, class L, class CC>
__device__ __forceinline__ void t_team_stream(const TParams& p, const CC& c, uint8_t* tab,
                                              const int8_t* wp, int W, int team, int wt, int first_item,
                                              unsigned long long* prog, uint2* rb, TStream* ts, TPool* pool,
                                              int nteams) {
  constexpr bool S32 = L::kSeqs == 1;
  constexpr int CB = chunk_bytes<C>();
  constexpr int LS = 32 * C;
  const int lane = threadIdx.x & 31;
  const int A1 = p.A_used + 1;
  const int qsteps = (p.qcols + 32 + 3) & ~3;
  const int n_items = S32 ? *p.item_count : p.n_items;
  volatile TStream* vs = ts;
  volatile TPool* vp = pool;
  const int cap = kTPool / nteams, off = team * cap;
  // item -> (pair, half): s16x2 items are pairs, s32 items index the flagged-sequence list
  auto pair_of = [&](int item, int* half) {
    if constexpr (S32) {
      const int sq = p.item_list[item];
      *half = sq & 1;
      return sq >> 1;
    } else {
      *half = 0;
      return item;
    }
  };
  auto emit_item = [&](int item, int lo, int hi) {
    if constexpr (S32) emit_t32(p, lo, p.item_list[item]);
    else emit_t(p, ((uint32_t)lo & 0xffffu) | ((uint32_t)hi << 16), item);
  };
  // append one pair to the ring (lane 0 of the warp holding the lock)
  auto append = [&](int item) {
    int hf;
    const int nl = (p.pair_ncols[pair_of(item, &hf)] + C - 1) / C;   // >= 3 lanes (n' >= 48)
    const int k = off + vs->count % cap;
    if (vs->count >= cap)   // the entry cap pairs back must be finished before it is reused
      while (vp->rem[k] != 0) __nanosleep(64);
    // rem = lanes + 1: the lane that completes the pair emits first and then releases the entry
    // (the appender recycles an entry only at rem == 0, after its maxima were read)
    vp->item[k] = item; vp->base[k] = vs->next; vp->nl[k] = nl; vp->rem[k] = nl + 1; vp->mlo[k] = 0; vp->mhi[k] = 0;
    // publication order: the entry, then count, then next — a reader that sees next cover its
    // strip (and fences) sees the count that includes every entry of the strip
    __threadfence_block();
    vs->count = vs->count + 1;
    __threadfence_block();
    vs->next = vs->next + nl;
  };
  // the next queue item (-1 at the end).  Pairs shorter than a strip are taken kTGrab per
  // global atomic (one atomic round trip per pair was on every strip's critical path); longer
  // ones one at a time, so that the teams stay balanced at the end of the queue (items come
  // longest first, so the length of the item at the counter tells which case applies)
  auto take = [&]() -> int {
    if (vs->pend == vs->pend_end) {
      const int cur = *reinterpret_cast<volatile int*>(p.work) + p.q0;
      int hf = 0;
      const bool short_pairs = cur < n_items && p.pair_ncols[pair_of(cur, &hf)] < 32 * C;
      const int grab = short_pairs ? kTGrab : 1;
      const int b0 = atomicAdd(p.work, grab);
      vs->pend = b0; vs->pend_end = b0 + grab;
    }
    const int item = p.q0 + vs->pend;
    vs->pend = vs->pend + 1;
    return item < n_items ? item : -1;
  };
  team_bar(team, W);
  if (wt == 0 && lane == 0) {
    for (int i = 0; i <= W; ++i) prog[i] = 0u;
    ts->lock = 0; ts->count = 0; ts->next = 0; ts->end = 0; ts->pend = 0; ts->pend_end = 0;
    if (first_item >= 0) append(first_item);
    __threadfence_block();
  }
  team_bar(team, W);
  for (int g = wt;; g += W) {
    // strip g needs every pair that covers its lanes (lane 0 appends, the warp follows)
    int have = 0, count = 0;
    if (lane == 0) {
      for (;;) {
        const int nx = vs->next;
        if (nx >= 32 * g + 32 || vs->end) {
          __threadfence_block();
          have = vs->next > 32 * g;
          count = vs->count;   // read after next (fenced): includes every entry of the strip
          break;
        }
        if (atomicCAS(&ts->lock, 0, 1) == 0) {
          while (vs->next < 32 * g + 32 && !vs->end) {   // this strip's pairs (may wait for the ring)
            const int item = take();
            if (item < 0) { __threadfence_block(); vs->end = 1; break; }   // end after the last next
            append(item);
          }
          __threadfence_block();
          atomicExch(&ts->lock, 0);
        } else {
          __nanosleep(64);
        }
      }
    }
    have = __shfl_sync(SWB_FULL, have, 0);
    count = __shfl_sync(SWB_FULL, count, 0);
    if (!have) break;
    __threadfence_block();
    // this lane's pair: the newest ring entry starting at or before lane 32g + lane
    const int gl = 32 * g + lane;
    int k = -1;
    {
      for (int j = count - 1; j >= 0 && j >= count - cap; --j) {
        const int kk = off + j % cap;
        if (vp->base[kk] <= gl) { if (gl < vp->base[kk] + vp->nl[kk]) k = kk; break; }
      }
    }
    int item = -1, half = 0, pair = 0, ncols = 0, lip = 0;
    if (k >= 0) {
      item = vp->item[k];
      pair = pair_of(item, &half);
      ncols = p.pair_ncols[pair];
      lip = gl - vp->base[k];             // lane index within the pair
    }
    const uint16_t* cp = p.cols + (k >= 0 ? p.pair_off[pair] : 0);
    build_strip_tables<C, L::kSeqs>(p, tab, wp, cp, k >= 0 ? ncols : 0, lip * C, half);
    // strip g continues strip g - 1's pair in its first lane: take its bottom row
    const int cont = __shfl_sync(SWB_FULL, k >= 0 && lip > 0 ? 1 : 0, 0);
    const uint32_t keep = (lane > 0 && k >= 0 && lip == 0) ? 0u : 1u;
    const int si = (g + W) % (W + 1), so = g % (W + 1);
    uint32_t b = run_pass<L, 32, C, true, 4, false, kPackedTagShift>(c, tab + lane * CB, LS, A1 * LS, p.qpair, p.qcols,
                                                                    0, qsteps, cont, 3, rb + (int64_t)si * p.rb_cols + 1,
                                                       rb + (int64_t)so * p.rb_cols + 1, prog + si, prog + so, 0u, g,
                                                       0u, keep);
    if (k >= 0) {
      if constexpr (S32) {
        atomicMax(&pool->mlo[k], (int)b);
      } else {
        atomicMax(&pool->mlo[k], (int)(int16_t)(b & 0xffffu));
        atomicMax(&pool->mhi[k], (int)(int16_t)(b >> 16));
      }
      __threadfence_block();
      if (atomicSub(&pool->rem[k], 1) == 2) {   // this pair's last lane
        const int lo = atomicAdd(&pool->mlo[k], 0), hi = atomicAdd(&pool->mhi[k], 0);
        emit_item(item, lo, hi);
        __threadfence_block();
        atomicSub(&pool->rem[k], 1);             // release the entry
      }
    }
    __syncwarp();
  }
}

// A GANG: the longest pairs' strips spread over gang_ctas CTAs x gang_warps warps (one warp per
// scheduler of each SM), so that one 35k-residue sequence is not bound to one SM.  Global warp
// gw = rank * gang_warps + warp takes strips gw, gw + GW, ...; the strip hand-off is the team
// pipeline with its row buffers and progress flags in global memory at gpu scope
// (release / acquire).  The pair's maximum is combined with atomicMax over the GW warps and
// emitted by the last one.  Progress needs every rank of a gang to become resident
// eventually: slots are taken in CTA start order, so the gang slots go to the first
// gang_items * gang_ctas CTAs that start; a rank that started may spin on a later rank (from
// the second round of strips on) until that rank's CTA starts.  That CTA waits only for SMs
// held by kernels that finish on their own: every other CTA of this launch and every group /
// recompute launch makes progress without waiting on other CTAs, and enqueue_query
// (sw_api.cu) serialises the T-mode launches that have gangs across the handle's streams, so
// two gang launches never hold SMs while waiting for each other.
template <int C, class CC>
__device__ __forceinline__ void t_gang_item(const TParams& p, const CC& c, uint8_t* tab, const int8_t* wp,
                                            int gi, int rank, int K, int warp) {
  using L = LaneS16x2;
  constexpr int CB = chunk_bytes<C>();
  constexpr int LS = 32 * C;
  const int lane = threadIdx.x & 31;
  const int A1 = p.A_used + 1;
  const int qsteps = (p.qcols + 32 + 3) & ~3;
  const int GW = K * p.gang_warps;                 // this gang's warps
  const int GWmax = p.gang_ctas * p.gang_warps;    // buffer stride: the largest gang's slots
  const int gw = rank * p.gang_warps + warp;
  const int item = p.gang0 + gi;                   // the pair (gi indexes the gang buffers)
  const int ncols = p.pair_ncols[item];
  const int S = (ncols + LS - 1) / LS;
  const uint16_t* cp = p.cols + p.pair_off[item];
  // tagged hand-off slots: one 64-bit word per column (run_pass GPU_FLAGS)
  uint2* rb = p.grb + (int64_t)gi * (GWmax + 1) * p.rb_cols;
  uint32_t b = 0;
  for (int P = gw; P < S; P += GW) {
    build_strip_tables<C>(p, tab, wp, cp, ncols, P * LS + lane * C);
    if (p.dbg_times && gi == 0 && lane == 0 && P < 4096) {   // probe: strip start (ns)
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      p.dbg_times[2 * P] = t;
    }
    const int si = (P + GW) % (GW + 1), so = P % (GW + 1);
    uint2* in = rb + (int64_t)si * p.rb_cols + 1;
    uint2* out = rb + (int64_t)so * p.rb_cols + 1;
    if (p.gang_chain2)
      b = run_pass<L, 32, C, true, 16, true, 20, false, true>(c, tab + lane * CB, LS, A1 * LS, p.qpair, p.qcols, 0,
                                                              qsteps, P, S, in, out, (uint32_t*)nullptr,
                                                              (uint32_t*)nullptr, b, -1, p.gang_epoch);
    else
      b = run_pass<L, 32, C, true, 16, true>(c, tab + lane * CB, LS, A1 * LS, p.qpair, p.qcols, 0, qsteps, P, S, in,
                                            out, (uint32_t*)nullptr, (uint32_t*)nullptr, b, -1, p.gang_epoch);
    if (p.dbg_times && gi == 0 && lane == 0 && P < 4096) {   // probe: strip end (ns)
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      p.dbg_times[2 * P + 1] = t;
    }
  }
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) b = L::max2(b, __shfl_xor_sync(SWB_FULL, b, o));
  if (lane == 0) {
    atomicMax(&p.gbest[2 * gi], (int)(int16_t)(b & 0xffffu));
    atomicMax(&p.gbest[2 * gi + 1], (int)(int16_t)(b >> 16));
    __threadfence();
    if (atomicAdd(&p.gdone[gi], 1) == GW - 1) {   // the last warp of the gang
      __threadfence();
      const int lo = atomicAdd(&p.gbest[2 * gi], 0), hi = atomicAdd(&p.gbest[2 * gi + 1], 0);
      emit_t(p, ((uint32_t)lo & 0xffffu) | ((uint32_t)hi << 16), item);
    }
  }
}

// PACKED: the team stream's layout (compile-time, one stream per kernel: both in one kernel
// measured 15-30 % slower for either, code size)
template <int C, int NT, bool WIDE = false, class L = LaneS16x2, bool PACKED = false>
__global__ void __launch_bounds__(NT, 1) k_search_t(const TParams p) {
  constexpr int kWarps = NT / 32;
  constexpr int LS = 32 * C;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t sprog[2 * kWarps];
  __shared__ unsigned long long sprog64[2 * kWarps];
  __shared__ uint32_t sred[kWarps];
  __shared__ int32_t sitem[kWarps];
  __shared__ int32_t sparked;
  // rows = the query's letters in compact order (row k = the k-th set bit of qmask) + the pad
  // row; columns = database letters (the database pad letter A maps to the pad value)
  const int A1 = p.A_used + 1;
  const int table_bytes = L::kSeqs * A1 * LS;  // lo (+ hi) tables of one warp
  // (A_used+1) rows of kWpStride bytes: w + rho for database letters d < A, -128 for the
  // database pad letter d == A (which is 32 for a 32-letter alphabet: the stride must exceed A)
  int8_t* wp = reinterpret_cast<int8_t*>(smem);
  uint8_t* tables = smem + ((A1 * kWpStride + 127) & ~127);
  const int warp = threadIdx.x >> 5;
  for (int t = threadIdx.x; t < A1 * kWpStride; t += blockDim.x) {
    const int a = t / kWpStride, d = t % kWpStride;
    int v = kPadValue;
    if (a < p.A_used && d < p.A) v = (int)p.matrix[(int)__fns(p.qmask, 0, a + 1) * p.A + d] + p.rho - p.delta;
    wp[t] = (int8_t)v;
  }
  if (threadIdx.x == 0) sparked = -1;
  __syncthreads();
  if (warp >= p.warps) return;
  ChainConstT<WIDE> c;
  c.rho = p.rho;
  c.sigma = p.sigma;
  c.delta = p.delta;
  c.padpair = (uint32_t)p.A_used * 0x101u;     // the query stream's (compact) pad letter
  c.hi_mul = p.hi_mul;
  uint8_t* tab = tables + warp * table_bytes;
  uint2* rb_cta = p.rb + (int64_t)blockIdx.x * (2 * p.warps) * p.rb_cols;
  // Phase 1: one team of all warps for the longest pairs (items come longest-first), so the
  // very long ones get the most parallelism; stops at the first pair with few strips.
  // Phase 2: teams of team_warps for the rest — small teams waste less time in the pipeline
  // fill and in the end-of-item barrier (T-mode ncu: 17 % barrier stalls with 8-warp teams).
  // Phase 0 (gangs): every CTA takes one gang slot; slot s = (pair s / gang_ctas, rank
  // s % gang_ctas).  The CTA's first gang_warps warps (one per scheduler) work on that pair
  // while its other warps wait, so that the gang's dependency chain has its schedulers to
  // itself; then all warps go on to phase 2.
  // warps [wbase, p.warps) run the team stream; in a gang CTA with gang_share the gang's
  // warps leave when their strips are done and the CTA's other warps stream meanwhile
  int wbase = 0, W = p.team_warps;
  if constexpr (L::kSeqs == 1) {
    // 32-bit recompute (long-query mode): the team stream only (no gangs, no whole-CTA phase)
  } else if (p.gang_items > 0) {
    __shared__ int32_t sgslot;
    if (threadIdx.x == 0) sgslot = atomicAdd(p.gang_ctr, 1);
    __syncthreads();
    // slot -> (gang, rank): gangs have their own sizes (gang_base prefix of CTAs)
    int gi = 0;
    while (gi < p.gang_items && p.gang_base[gi + 1] <= sgslot) ++gi;
    const int rank = gi < p.gang_items ? sgslot - p.gang_base[gi] : 0;
    const int K = gi < p.gang_items ? p.gang_base[gi + 1] - p.gang_base[gi] : 0;
    if (gi < p.gang_items) {
      if (p.gang_share) {
        if (warp < p.gang_warps) {
          t_gang_item<C>(p, c, tab, wp, gi, rank, K, warp);
          return;
        }
        wbase = p.gang_warps;
        W = min(W, p.warps - wbase);
        while ((p.warps - wbase) % W) --W;
      } else {
        if (warp < p.gang_warps) t_gang_item<C>(p, c, tab, wp, gi, rank, K, warp);
        __syncthreads();
      }
    }
  } else if (p.warps > p.team_warps) {
    t_team_loop<C>(p, c, tab, wp, p.warps, 0, warp, -1, p.big_strips, &sparked, sprog, rb_cta, sitem, sred);
    __syncthreads();
  }
  const int nteams = (p.warps - wbase) / W;
  const int team = (warp - wbase) / W, wt = (warp - wbase) % W;
  if (team >= nteams) return;
  const int first = (team == 0) ? sparked : -1;
  if constexpr (PACKED) {
    __shared__ TStream sts[kTmodeThreads / 32];
    __shared__ TPool spool;
    t_team_stream<C, L>(p, c, tab, wp, W, team, wt, first, sprog64 + team * (W + 1),
                        rb_cta + (int64_t)team * (W + 1) * p.rb_cols, &sts[team], &spool, nteams);
  } else {
    __shared__ TStreamP stsp[kTmodeThreads / 32];
    t_team_stream_pairs<C, L>(p, c, tab, wp, W, team, wt, first, sprog64 + team * (W + 1),
                              rb_cta + (int64_t)team * (W + 1) * p.rb_cols, &stsp[team]);
  }
}

// pdl: programmatic dependent launch after the row-scan kernel on the same stream (its
// clusters are resident and have triggered before these CTAs fill the remaining SMs)
template <int C, int NT, bool WIDE, class L, bool PACKED>
cudaError_t launch_search_tmode(const TParams& p, int grid, int smem_bytes, cudaStream_t st, bool pdl = false) {
  if (!pdl) {
    k_search_t<C, NT, WIDE, L, PACKED><<<grid, NT, smem_bytes, st>>>(p);
    return cudaGetLastError();
  }
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(NT);
  cfg.dynamicSmemBytes = smem_bytes;
  cfg.stream = st;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_search_t<C, NT, WIDE, L, PACKED>, p);
}

template <int C, int NT, bool WIDE, class L, bool PACKED>
cudaError_t configure_tmode(int smem_bytes, int* blocks_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(k_search_t<C, NT, WIDE, L, PACKED>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_search_t<C, NT, WIDE, L, PACKED>, NT,
                                                       smem_bytes);
}

// G = 32 entries compile two kernels (GS = 1: single-strip group stream, GS = 2: multi-strip);
// the 32-bit recompute (item_list) never reaches the group phase, so either serves it.
template <class L, int G, int Rs, int Rl, int NT, bool WIDE>
cudaError_t launch_search_t(const SearchParams& p, int grid, int smem_bytes, cudaStream_t st) {
  if constexpr (G == 32) {
    if (p.short_passes > 1) k_search<L, G, Rs, Rl, NT, WIDE, 2><<<grid, NT, smem_bytes, st>>>(p);
    else k_search<L, G, Rs, Rl, NT, WIDE, 1><<<grid, NT, smem_bytes, st>>>(p);
  } else {
    k_search<L, G, Rs, Rl, NT, WIDE><<<grid, NT, smem_bytes, st>>>(p);
  }
  return cudaGetLastError();
}

template <class L, int G, int Rs, int Rl, int NT, bool WIDE, int GS>
cudaError_t configure_one(int smem_bytes, int* blocks_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(k_search<L, G, Rs, Rl, NT, WIDE, GS>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_search<L, G, Rs, Rl, NT, WIDE, GS>, NT,
                                                       smem_bytes);
}

template <class L, int G, int Rs, int Rl, int NT, bool WIDE>
cudaError_t configure_t(int smem_bytes, int* blocks_per_sm) {
  if constexpr (G == 32) {
    int b1 = 0, b2 = 0;
    cudaError_t e = configure_one<L, G, Rs, Rl, NT, WIDE, 1>(smem_bytes, &b1);
    if (e != cudaSuccess) return e;
    e = configure_one<L, G, Rs, Rl, NT, WIDE, 2>(smem_bytes, &b2);
    *blocks_per_sm = b1 < b2 ? b1 : b2;
    return e;
  } else {
    return configure_one<L, G, Rs, Rl, NT, WIDE, 0>(smem_bytes, blocks_per_sm);
  }
}

}  // namespace swb
