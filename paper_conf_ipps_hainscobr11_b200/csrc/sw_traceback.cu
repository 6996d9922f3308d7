// sw_traceback.cu — optimal local alignment of one (query, database sequence) pair
// ("The optimal alignment can be found by backtracking
// through H").  The search path only needs scores; this is the step after it, for the top hits.
//
// k_tb_fill: one CTA sweeps the anti-diagonals of Eq.(1) (cells of one diagonal are
// independent given the two previous diagonals), in int32, keeps H/E/F of the last two
// diagonals in global scratch and writes one direction byte per cell:
//   bits 0-1  H source: 0 = the 0 clamp (alignment start), 1 = diagonal, 2 = E, 3 = F
//   bit 2     E extended E[i][j-1] (1) or opened from H[i][j-1] (0)
//   bit 3     F extended F[i-1][j] (1) or opened from H[i-1][j] (0)
// Ties prefer diagonal > E > F > 0 and extension > opening; the end cell is the maximum H,
// first in (diagonal, row) order.
// k_tb_walk: one thread follows the bytes back from the end cell and writes run-length ops.
//
// Bounded memory (round 2): the direction bytes are only written for the alignment's bounding
// box.  (1) k_tb_fill without directions: the optimal score and its end cell (ie, je), O(m)
// scratch.  (2) k_tb_start: Eq.(1) on the reversed prefixes q[ie..0] x d[je..0] ANCHORED at
// (ie, je) (no 0 clamp, boundary -inf, the first cell a substitution): its value at (i, j) is the
// best score of an alignment from (ie - i, je - j) to (ie, je) that starts with a substitution,
// so a cell where it equals the optimum is the start (ib, jb) of an optimal local alignment (an
// optimal one never starts or ends with a gap).  (3) k_tb_fill with directions on the box
// q[ib..ie] x d[jb..je] only (its local optimum is the same score), and the walk.  Memory
// (ie - ib + 1)(je - jb + 1) bytes instead of m n.
#include <cstdint>
#include <cuda_runtime.h>

#include "sw_internal.h"

namespace swb {

namespace {
constexpr int kTbThreads = 1024;
constexpr int kNegInf = -(1 << 29);
}

__global__ void __launch_bounds__(kTbThreads, 1)
    k_tb_fill(const uint8_t* __restrict__ q, int m, const uint16_t* __restrict__ dcols, int half, int n,
              const int8_t* __restrict__ W, int A, int rho, int sigma, uint8_t* __restrict__ dir,
              int* __restrict__ diag_scratch, int* __restrict__ result) {
  // scratch: H for diagonals d-2, d-1, d (3m), E and F for d-1, d (2m each)
  int* Hb[3] = {diag_scratch, diag_scratch + m, diag_scratch + 2 * m};
  int* Eb[2] = {diag_scratch + 3 * m, diag_scratch + 4 * m};
  int* Fb[2] = {diag_scratch + 5 * m, diag_scratch + 6 * m};
  __shared__ int s_best[kTbThreads / 32], s_bd[kTbThreads / 32], s_bi[kTbThreads / 32];
  int best = 0, bd = 0x7fffffff, bi = 0x7fffffff;
  const int shift = 8 * half;
  for (int d = 0; d < m + n - 1; ++d) {
    int* H2 = Hb[(d + 1) % 3];   // diagonal d-2
    int* H1 = Hb[(d + 2) % 3];   // diagonal d-1
    int* Hn = Hb[d % 3];         // diagonal d
    const int* E1 = Eb[(d + 1) & 1];
    const int* F1 = Fb[(d + 1) & 1];
    int* En = Eb[d & 1];
    int* Fn = Fb[d & 1];
    const int i0 = max(0, d - (n - 1)), i1 = min(m - 1, d);
    for (int i = i0 + (int)threadIdx.x; i <= i1; i += blockDim.x) {
      const int j = d - i;
      // left neighbour (i, j-1) is on diagonal d-1 at row i; upper (i-1, j) at row i-1;
      // diagonal (i-1, j-1) on diagonal d-2 at row i-1 (boundaries: H = 0, E = F = -inf)
      const int hl = (j > 0) ? H1[i] : 0;
      const int el = (j > 0) ? E1[i] : kNegInf;
      const int hu = (i > 0) ? H1[i - 1] : 0;
      const int fu = (i > 0) ? F1[i - 1] : kNegInf;
      const int hd = (i > 0 && j > 0) ? H2[i - 1] : 0;
      const int e_ext = el - sigma, e_open = hl - rho;
      const int e = max(e_ext, e_open);
      const int f_ext = fu - sigma, f_open = hu - rho;
      const int f = max(f_ext, f_open);
      const int a = (dcols[j] >> shift) & 0xff;
      const int t = hd + (int)W[q[i] * A + a];
      int h = 0, src = 0;
      if (f > h) { h = f; src = 3; }
      if (e >= h && e > 0) { h = e; src = 2; }
      if (t >= h && t > 0) { h = t; src = 1; }
      Hn[i] = h;
      En[i] = e;
      Fn[i] = f;
      if (dir) dir[(int64_t)i * n + j] = (uint8_t)(src | ((e_ext >= e_open) ? 4 : 0) | ((f_ext >= f_open) ? 8 : 0));
      if (h > best || (h == best && (d < bd || (d == bd && i < bi)))) { best = h; bd = d; bi = i; }
    }
    __syncthreads();
  }
  // block argmax: (value desc, diagonal asc, row asc)
  for (int o = 16; o >= 1; o >>= 1) {
    const int ob = __shfl_xor_sync(0xffffffffu, best, o), od = __shfl_xor_sync(0xffffffffu, bd, o),
              oi = __shfl_xor_sync(0xffffffffu, bi, o);
    if (ob > best || (ob == best && (od < bd || (od == bd && oi < bi)))) { best = ob; bd = od; bi = oi; }
  }
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) { s_best[w] = best; s_bd[w] = bd; s_bi[w] = bi; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < (int)(blockDim.x >> 5); ++k) {
      if (s_best[k] > best || (s_best[k] == best && (s_bd[k] < bd || (s_bd[k] == bd && s_bi[k] < bi)))) {
        best = s_best[k]; bd = s_bd[k]; bi = s_bi[k];
      }
    }
    result[0] = best;
    result[1] = best > 0 ? bi : -1;
    result[2] = best > 0 ? bd - bi : -1;
  }
}

// (2) start cell: the anchored reverse sweep, anti-diagonals of the reversed prefixes; result
// [3] = ib, [4] = jb of the first cell (diagonal, row order) whose value equals result[0]
__global__ void __launch_bounds__(kTbThreads, 1)
    k_tb_start(const uint8_t* __restrict__ q, const uint16_t* __restrict__ dcols, int half, const int8_t* __restrict__ W,
               int A, int rho, int sigma, int* __restrict__ diag_scratch, int* __restrict__ result) {
  const int best = result[0], ie = result[1], je = result[2];
  if (best <= 0) {
    if (threadIdx.x == 0) { result[3] = -1; result[4] = -1; }
    return;
  }
  const int m = ie + 1, n = je + 1;   // reversed prefix: row i = q[ie - i], column j = d[je - j]
  int* Hb[3] = {diag_scratch, diag_scratch + m, diag_scratch + 2 * m};
  int* Eb[2] = {diag_scratch + 3 * m, diag_scratch + 4 * m};
  int* Fb[2] = {diag_scratch + 5 * m, diag_scratch + 6 * m};
  __shared__ int s_bd[kTbThreads / 32], s_bi[kTbThreads / 32];
  __shared__ int s_found;
  if (threadIdx.x == 0) s_found = 0;
  __syncthreads();
  int bd = 0x7fffffff, bi = 0x7fffffff;
  const int shift = 8 * half;
  for (int d = 0; d < m + n - 1; ++d) {
    int* H2 = Hb[(d + 1) % 3];
    int* H1 = Hb[(d + 2) % 3];
    int* Hn = Hb[d % 3];
    const int* E1 = Eb[(d + 1) & 1];
    const int* F1 = Fb[(d + 1) & 1];
    int* En = Eb[d & 1];
    int* Fn = Fb[d & 1];
    const int i0 = max(0, d - (n - 1)), i1 = min(m - 1, d);
    for (int i = i0 + (int)threadIdx.x; i <= i1; i += blockDim.x) {
      const int j = d - i;
      // anchored boundary: H(-1, -1) = 0, every other H / E / F outside the prefix = -inf
      const int hl = (j > 0) ? H1[i] : kNegInf;
      const int el = (j > 0) ? E1[i] : kNegInf;
      const int hu = (i > 0) ? H1[i - 1] : kNegInf;
      const int fu = (i > 0) ? F1[i - 1] : kNegInf;
      const int hd = (i > 0 && j > 0) ? H2[i - 1] : ((i == 0 && j == 0) ? 0 : kNegInf);
      const int e = max(el - sigma, hl - rho);
      const int f = max(fu - sigma, hu - rho);
      const int a = (dcols[je - j] >> shift) & 0xff;
      const int t = hd + (int)W[q[ie - i] * A + a];
      const int h = max(max(t, e), max(f, kNegInf));
      Hn[i] = h;
      En[i] = max(e, kNegInf);
      Fn[i] = max(f, kNegInf);
      if (h == best && (d < bd || (d == bd && i < bi))) { bd = d; bi = i; }
    }
    __syncthreads();
    // stop at the first diagonal that holds the start (all threads agree after the barrier)
    if (bd != 0x7fffffff) s_found = 1;
    __syncthreads();
    if (s_found) break;
  }
  for (int o = 16; o >= 1; o >>= 1) {
    const int od = __shfl_xor_sync(0xffffffffu, bd, o), oi = __shfl_xor_sync(0xffffffffu, bi, o);
    if (od < bd || (od == bd && oi < bi)) { bd = od; bi = oi; }
  }
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) { s_bd[w] = bd; s_bi[w] = bi; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < (int)(blockDim.x >> 5); ++k)
      if (s_bd[k] < bd || (s_bd[k] == bd && s_bi[k] < bi)) { bd = s_bd[k]; bi = s_bi[k]; }
    result[3] = ie - bi;          // ib
    result[4] = je - (bd - bi);   // jb
  }
}

// ops: run-length (len << 2 | op), op 0 = M (q_i with d_j), 1 = I (d_j against a gap: E),
// 2 = D (q_i against a gap: F); a gap reopened directly after a gap of the same kind starts a
// new run.  result: [0] score [1] end i [2] end j (inclusive) -> [3] begin i [4] begin j [5] ops
__global__ void k_tb_walk(const uint8_t* __restrict__ dir, int m, int n, int* __restrict__ result,
                          uint32_t* __restrict__ ops, int ops_cap) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  int i = result[1], j = result[2];
  int nops = 0, cur_op = -1, cur_len = 0;
  int bi = i, bj = j;
  auto push = [&](int op, bool new_run) {
    if (op == cur_op && !new_run) { ++cur_len; return; }
    if (cur_op >= 0) { if (nops < ops_cap) ops[nops] = ((uint32_t)cur_len << 2) | (uint32_t)cur_op; ++nops; }
    cur_op = op;
    cur_len = 1;
  };
  int state = 0;   // 0 = H, 1 = E, 2 = F
  bool opened = true;
  if (result[0] > 0) {
    while (i >= 0 && j >= 0) {
      const uint8_t b = dir[(int64_t)i * n + j];
      if (state == 0) {
        const int src = b & 3;
        if (src == 0) break;                     // H = 0: the alignment starts after this cell
        if (src == 1) { push(0, false); bi = i; bj = j; --i; --j; continue; }
        state = (src == 2) ? 1 : 2;
        opened = true;
        continue;
      }
      if (state == 1) {                          // E: d_j against a gap, came from (i, j-1)
        push(1, opened);
        bi = i; bj = j;
        const bool ext = (b & 4) != 0;
        --j;
        state = ext ? 1 : 0;
        opened = !ext;   // the next E column starts a new run only if this one was opened
        if (ext) opened = false;
        continue;
      }
      push(2, opened);                           // F: q_i against a gap, came from (i-1, j)
      bi = i; bj = j;
      const bool ext = (b & 8) != 0;
      --i;
      state = ext ? 2 : 0;
      opened = false;
    }
    if (cur_op >= 0) { if (nops < ops_cap) ops[nops] = ((uint32_t)cur_len << 2) | (uint32_t)cur_op; ++nops; }
  }
  // the runs were collected end -> begin: reverse them in place
  const int k = nops < ops_cap ? nops : ops_cap;
  for (int a = 0, z = k - 1; a < z; ++a, --z) { const uint32_t t = ops[a]; ops[a] = ops[z]; ops[z] = t; }
  result[3] = result[0] > 0 ? bi : -1;
  result[4] = result[0] > 0 ? bj : -1;
  result[5] = nops;
}

cudaError_t launch_tb_score_start(const uint8_t* q, int m, const uint16_t* dcols, int half, int n, const int8_t* W,
                                  int A, int rho, int sigma, int* scratch, int* result, cudaStream_t st) {
  k_tb_fill<<<1, kTbThreads, 0, st>>>(q, m, dcols, half, n, W, A, rho, sigma, nullptr, scratch, result);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  k_tb_start<<<1, kTbThreads, 0, st>>>(q, dcols, half, W, A, rho, sigma, scratch, result);
  return cudaGetLastError();
}

cudaError_t launch_traceback(const uint8_t* q, int m, const uint16_t* dcols, int half, int n, const int8_t* W, int A,
                             int rho, int sigma, uint8_t* dir, int* scratch, int* result, uint32_t* ops, int ops_cap,
                             cudaStream_t st) {
  k_tb_fill<<<1, kTbThreads, 0, st>>>(q, m, dcols, half, n, W, A, rho, sigma, dir, scratch, result);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  k_tb_walk<<<1, 32, 0, st>>>(dir, m, n, result, ops, ops_cap);
  return cudaGetLastError();
}

}  // namespace swb
