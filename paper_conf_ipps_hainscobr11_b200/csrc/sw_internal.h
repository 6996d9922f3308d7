// sw_internal.h — shared between the host side (sw_api.cu) and the kernel instantiations.
// Not part of the public ABI (include/sw.h is).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace swb {

constexpr int kMaxWarps = 16;            // at most 512 threads per CTA
constexpr int kMinCols = 48;             // every pair is padded to >= 48 columns (>= G + 16)
constexpr int kColAlign = 8;             // pair column counts are multiples of 8 (16 bytes)
constexpr int kPadCols = 32;             // trailing pad columns stored after every pair
constexpr int kLeadCols = 8;             // pad columns stored before the first pair, so that every
                                         // pair is preceded by >= 3 pad columns (the look-ahead
                                         // residue stream of group_stream reads them)
constexpr int kPadValue = -128;          // profile value of pad letters / pad query rows

// Bank-conflict-free shared-memory image of the query profile for chains of G lanes with R
// rows per lane.  Query row i lives in strip P = i / (G*R),
// lane gl = (i % (G*R)) / R, row r = i % R, chunk k = r / cb (cb = 4 or 8 rows = bytes):
//   byte(rep, a, i) = off + rep*rs + a*ls + ((P*nch + k)*G + gl)*cb + r % cb
// (nch = ceil(R / cb) chunks per lane and strip; cb = 16 from 12 rows up, the last chunk
// partial when R % 16 != 0: LDS.128 reads 4 query rows x 4 per instruction)
// so at a fixed (strip, chunk) the G lanes of a chain read consecutive cb-byte words of
// their own letter row: the letter term a*ls is a multiple of 128 B (32 banks) and drops
// out of the bank index, and the 32/G replicas (one per chain of a warp) are shifted by
// cb*G bytes, so any mix of letters across the warp is conflict-free.
struct ProfLayout {
  int off;     // byte offset of the image in the staged blob
  int G;       // lanes per chain (32 for team mode)
  int R;       // rows per lane
  int cb;      // chunk bytes
  int nch;     // chunks per lane and strip, ceil(R / cb)
  int strips;  // strips covered (strips * G * R >= m)
  int ls;      // letter stride, multiple of 128
  int rs;      // replica stride, == cb * G (mod 128)
  int nrep;    // replicas (32 / G for group mode, 1 for team mode)
  int bytes;   // nrep * rs
};

// One persistent search launch for one query.
struct SearchParams {
  // query profile (w(q_i, a) + rho - delta as int8, -128 for pad letters / rows), staged as one blob
  const uint8_t* prof;       // global blob: group image then (if different) team image
  int prof_bytes;            // blob size (multiple of 16)
  ProfLayout lg;             // group-mode image
  ProfLayout lt;             // team-mode image (may alias lg)
  int pad_letter;            // == A
  int rho, sigma, max_w;     // rho, sigma: the kernel's (clamped) penalties, DESIGN.md "Integer widths"
  int delta;                 // rho - profile offset (> 0 only for WIDE kernels)
  int flag_limit;            // s16x2: a best >= flag_limit is recomputed in 32 bits
  // database, sorted by length descending and paired (2p, 2p+1)
  const uint16_t* cols;      // interleaved columns: cols[pair_off[p] + j] = d_lo[j] | d_hi[j] << 8
  const int64_t* pair_off;   // in u16 units
  const int32_t* pair_ncols; // padded column count n' (multiple of 8, >= kMinCols); the pair
                             // occupies n' + kPadCols columns (the tail is pad letters)
  int n_pairs;
  int n_seqs;
  const int32_t* perm;       // sorted position -> caller index
  int32_t* scores;           // caller order, int32
  // work partition: items [0, n_long) run in team (intra-task) mode, [n_long, n_pairs) in
  // group (inter-task) mode.  For the 32-bit recompute kernel items come from item_list.
  int n_long;                // team-mode items (pairs [0, n_long)); 0 when T-mode takes them
  int short_begin;           // first pair of the group-mode (short) range
  const int32_t* item_list;  // s32 recompute: sorted sequence positions (nullptr otherwise)
  const int32_t* item_count; // s32 recompute: device count
  int32_t* work;             // [0] team-item counter, [1] group-item counter
  int32_t* ovf_list;         // sequences whose 16-bit best may have wrapped
  int32_t* ovf_count;
  // passes over the query: group mode G*R_s rows per pass, team mode 32*R_l rows per pass
  int short_passes;
  int long_passes;
  int team_warps;            // warps per team (1..warps per CTA), teams = warps / team_warps
  // row buffers (strip bottom rows, §III "the bottom row of a strip must
  // be saved for the next pass"), uint2 = (H - rho, F) per column
  uint2* rb_group; int64_t rb_group_cols;   // per group slot (>= max n' + kPadCols)
  int group_stream;          // G = 32: continuous stream over strips and pairs (group_stream)
  const uint2* rb_zero;      // 4 neutral row-buffer entries (H = 0, F + rho = 0)
  uint32_t hi_mul;           // 1 << 24, as a runtime value: umulhi(pair, hi_mul) = pair >> 8 on
                             // the FMA pipe (IMAD.HI), keeping letter extraction off the ALU pipe
  uint2* rb_team;  int64_t rb_team_cols;    // per (team slot, pass mod (team_warps+1))
};

// Kernel configuration menu entry: G lanes x R_s rows in group mode, 32 lanes x R_l rows
// in team mode.  Lane = 0 (s16x2, two sequences per register) or 1 (s32, one sequence).
struct KernelConfig {
  int lane;
  int G;
  int Rs;
  int Rl;
  int threads;   // CTA size (fewer threads for the register-heavy entries)
  int wide;      // 1: rho + max(w) > 127 variant (ChainConstT<true>, sw_engine.cuh)
};

// Launch one search; returns the CUDA error of the launch.
cudaError_t launch_search(const KernelConfig& cfg, const SearchParams& p, int grid, int smem_bytes,
                          cudaStream_t st);
// Max dynamic smem / occupancy helpers for a config.
cudaError_t configure_kernel(const KernelConfig& cfg, int smem_bytes, int* blocks_per_sm);
// The menu of compiled configurations.
int menu_size();
KernelConfig menu_entry(int i);
KernelConfig recompute_config(bool wide);

// T-mode (transposed long-sequence kernel, sw_engine.cuh k_search_t): C database positions
// per lane, one CTA team of up to kTmodeThreads / 32 warps per long pair.
constexpr int kTmodeC = 16;
constexpr int kTmodeThreads = 256;
constexpr int kTmodeMaxQuery = 3072;     // longer queries take team mode for long pairs
constexpr int kWpStride = 64;            // T-mode substitution table row: database letters 0..A <= 32
struct TParams {
  const int8_t* matrix;      // A x A, [query][db]
  int A, rho, sigma, max_w, pad_letter;
  int delta, flag_limit;     // as SearchParams (the strip tables hold w + rho - delta)
  const uint16_t* qpair;     // query as (q | q << 8), qcols + kPadCols entries, pad beyond m
  int qcols;                 // query length rounded up to 8
  const uint16_t* cols;
  const int64_t* pair_off;
  const int32_t* pair_ncols;
  int n_items;               // long pairs [0, n_items)
  int n_seqs;
  const int32_t* perm;
  int32_t* scores;
  int32_t* ovf_list;
  int32_t* ovf_count;
  const int32_t* item_list;  // 32-bit recompute (LaneS32 instantiation): flagged sequence positions
  const int32_t* item_count; //   and their device count; the items of the team stream
  int32_t* work;
  int warps;                 // warps used per CTA (<= NT / 32, bounded by shared memory)
  int team_warps;            // warps per team in phase 2 (divides warps)
  int big_strips;            // phase 1 (one team of all warps) keeps pairs with >= big_strips strips
  uint2* rb; int64_t rb_cols;   // per CTA: 2 * warps slots (teams x (team_warps + 1) <= 2 * warps)
  uint32_t hi_mul;           // 1 << 24 (see SearchParams::hi_mul)
  uint32_t qmask;            // letters present in the query (bit a = letter code a)
  int A_used;                // popcount(qmask): compact letter k = the k-th set bit; pad = A_used
  // gangs (k_search_t phase 0): pairs [0, gang_items) are spread over gang_ctas CTAs x
  // gang_warps warps each; all buffers below are per gang pair and zeroed before the launch
  int gang_items, gang_ctas, gang_warps;   // gang_ctas: the largest gang's CTAs (buffer stride)
  int gang0;                 // first gang pair: gang gi works on pair gang0 + gi (after the
                             // row-scan pairs [0, gang0), sw_scan.cu)
  int q0;                    // first item of the team queue: gang0 + gang_items
  const int32_t* gang_base;  // gang_items + 1 CTA-slot offsets: gang i has CTAs base[i] .. base[i+1]
  int gang_share;            // 1: the gang CTAs' other warps run the team stream meanwhile
  int gang_chain2;           // 1: the gang warps use the two-op vertical chain (cell_rows CHAIN2)
  int packed;                // team stream layout: 1 packed lanes (mostly short pairs), 0 one pair per strip
  uint32_t gang_epoch;       // tag epoch of this launch's hand-off words (20 bits, != the last launch's)
  unsigned long long* dbg_times;   // probe (SW_DEBUG_GANG_TIMES): gang item 0's strip start / end (ns)
  int32_t* gang_ctr;         // slot counter
  uint32_t* gprog;           // (unused: the hand-off words carry their own tags)
  uint2* grb;                // gang_items x (GW + 1) x rb_cols x 2 tagged hand-off words (uint2 each)
  int32_t* gbest;            // gang_items x 2: maxima of the pair's two sequences
  int32_t* gdone;            // gang_items: warps finished
};

cudaError_t launch_tmode(const TParams& p, int grid, int smem_bytes, cudaStream_t st, bool s32 = false,
                         bool pdl = false);
cudaError_t configure_tmode_kernel(int smem_bytes, int* blocks_per_sm, bool wide, bool s32 = false,
                                   bool packed = false);
cudaError_t launch_qpair(uint16_t* out, const uint8_t* q, int m, int n, uint32_t qmask, cudaStream_t st);

// Row scan (sw_scan.cu): long pairs on clusters of ceil(ncols / kScanCols) CTAs (<= 16), the
// pairs of one cluster size in one launch; ceil(ncols / K) columns per CTA rounded up to 128
// (<= kScanCols); the scores are emitted like k_search_t's (emit_t).
constexpr int kScanThreads = 1024;
constexpr int kScanC = 4;
constexpr int kScanCols = kScanThreads * kScanC;
constexpr int kScanMaxCtas = 16;         // cluster size limit (non-portable above 8)
constexpr int kScanMaxLetters = 26;      // (A_used + 1) x 2 x cols_cta bytes of tables + the query
constexpr int kScanMinCols = 16384;
constexpr int kMaxScanItems = 32;
constexpr double kScanRowSteps = 10.0;   // a scan row's time in strip steps, calibrated on C2 long sets (queries 144-729, r02_row_scan.txt)
int scan_cols_cta(int ncols, int ctas);
int scan_smem_bytes(int a_used, int cols_cta, int qcols);
cudaError_t configure_scan_kernel(int smem_bytes, int ctas, int* max_clusters);
cudaError_t launch_scan_pairs(const TParams& p, int item0, int items, int ctas, int smem_bytes, cudaStream_t st,
                              bool pdl);

// Top hits (sw_topk.cu): radix-select histogram passes, the keys above the threshold, the
// threshold ties with the smallest indices (tie_off: exclusive prefix of the per-CTA tie counts).
int topk_ctas(int64_t n);
cudaError_t launch_tk_hist(const int32_t* s, int64_t n, int shift, uint32_t prefix, uint32_t pmask, uint32_t* hist,
                           int grid, cudaStream_t st);
cudaError_t launch_tk_above(const int32_t* s, int64_t n, uint32_t thr, int64_t* out_idx, int32_t* out_score,
                            uint32_t* out_count, uint32_t* tie_count, cudaStream_t st);
cudaError_t launch_tk_ties(const int32_t* s, int64_t n, uint32_t thr, const uint32_t* tie_off, uint32_t need,
                           int64_t* out_idx, int32_t* out_score, cudaStream_t st);
// Traceback, bounded memory: score + end cell (no directions), then the anchored reverse sweep
// for the start cell; result[0..2] = score, end i, end j; [3..4] = start i, start j (-1: none).
cudaError_t launch_tb_score_start(const uint8_t* q, int m, const uint16_t* dcols, int half, int n, const int8_t* W,
                                  int A, int rho, int sigma, int* scratch, int* result, cudaStream_t st);
// Traceback of one pair (sw_traceback.cu): dir = m*n bytes, scratch = 7*m ints, result = 6 ints.
cudaError_t launch_traceback(const uint8_t* q, int m, const uint16_t* dcols, int half, int n, const int8_t* W, int A,
                             int rho, int sigma, uint8_t* dir, int* scratch, int* result, uint32_t* ops, int ops_cap,
                             cudaStream_t st);

// Profile image build: byte(rep, a, i) = (i < m && a < A) ? W[q_i][a] + rho : -128 (rho here is the
// profile offset c = rho - delta).
cudaError_t launch_profile(uint8_t* blob, const ProfLayout& L, const uint8_t* q, int m, const int8_t* W, int A,
                           int rho, cudaStream_t st);

}  // namespace swb
