// sw_api.cu — the C ABI (include/sw.h): validation, host preprocessing of the database
// (§II-C: "The database is sorted by length"), per-query planning and
// stream-ordered launches of the sm_100a kernels.  No CPU fallback: every score is computed
// by k_search (sw_engine.cuh) on the device.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <numeric>
#include <string>
#include <thread>
#include <vector>
#include <unistd.h>

#include "../../include/sw.h"
#include "sw_internal.h"

using namespace swb;

namespace {

struct QuerySlot {
  int cap_m = 0;
  uint8_t* d_query = nullptr;
  uint8_t* d_prof = nullptr;
  size_t prof_cap = 0;
  int32_t* d_work = nullptr;      // 4 counters
  int32_t* d_ovf_count = nullptr;
  int32_t* d_ovf_list = nullptr;
  int64_t ovf_cap = 0;
  uint2* d_rb_group = nullptr;
  size_t rb_group_cap = 0;        // bytes
  uint2* d_rb_team = nullptr;
  size_t rb_team_cap = 0;
  uint2* d_rb_t = nullptr;        // T-mode strip boundaries
  size_t rb_t_cap = 0;
  uint16_t* d_qpair = nullptr;    // T-mode query stream
  size_t qpair_cap = 0;
  int32_t* d_gang = nullptr;      // T-mode gangs: counter, maxima, done counts, progress flags
  size_t gang_cap = 0;
  uint2* d_grb = nullptr;         // T-mode gangs: row buffers
  size_t grb_cap = 0;
  cudaStream_t stream = nullptr;
  cudaStream_t aux = nullptr;      // T-mode launch, concurrent with the group launch
  cudaStream_t scan = nullptr;     // row-scan cluster launches (sw_scan.cu), beside the T-mode launch
  cudaEvent_t scan_fork = nullptr, scan_done = nullptr;
  int scan_smem = -1;              // the row-scan kernel's configured dynamic shared memory
  uint32_t scan_ctas_ok = 0;       // cluster sizes checked for that configuration (bit K)
  cudaEvent_t done = nullptr;
  cudaEvent_t fork = nullptr, join = nullptr;
};

// One device-resident database in the search layout.
struct DbState {
  bool loaded = false;
  int64_t n_seqs = 0;
  int n_pairs = 0;
  std::vector<int64_t> sorted_len;        // lengths in sorted (descending) order
  std::vector<int32_t> h_pair_ncols;
  std::vector<int64_t> pair_cols_prefix;  // prefix sums of h_pair_ncols
  std::vector<int64_t> h_pair_off;        // u16 offset of every pair in d_cols
  std::vector<int32_t> inv_perm;          // caller index -> sorted position
  uint16_t* d_cols = nullptr; size_t cols_cap = 0;
  int64_t* d_pair_off = nullptr; size_t pair_off_cap = 0;
  int32_t* d_pair_ncols = nullptr; size_t pair_ncols_cap = 0;
  int32_t* d_perm = nullptr; size_t perm_cap = 0;
  void* h_stage = nullptr; size_t stage_cap = 0;   // pinned staging for asynchronous uploads
  void release() {
    cudaFree(d_cols); cudaFree(d_pair_off); cudaFree(d_pair_ncols); cudaFree(d_perm);
    if (h_stage) cudaFreeHost(h_stage);
    d_cols = nullptr; d_pair_off = nullptr; d_pair_ncols = nullptr; d_perm = nullptr; h_stage = nullptr;
    cols_cap = pair_off_cap = pair_ncols_cap = perm_cap = stage_cap = 0;
    loaded = false;
  }
};

// One of the two alternating chunk slots of sw_search_stream (kept on the handle so repeated
// streamed searches reuse the pinned staging and device buffers).
struct StreamSlot {
  DbState db;
  cudaStream_t up = nullptr;                 // upload stream
  cudaEvent_t uploaded = nullptr, searched = nullptr;
  int32_t* d_sc = nullptr; size_t d_sc_cap = 0;
  int32_t* h_sc = nullptr; size_t h_sc_cap = 0;   // pinned
  int32_t* h_ovf = nullptr; int ovf_cap = 0;      // pinned, per query of the chunk
  int64_t s0 = 0, n = 0;
  bool pending = false;
  void release() {
    if (up) { cudaStreamSynchronize(up); cudaStreamDestroy(up); }
    if (uploaded) cudaEventDestroy(uploaded);
    if (searched) { cudaEventSynchronize(searched); cudaEventDestroy(searched); }
    cudaFree(d_sc);
    if (h_sc) cudaFreeHost(h_sc);
    if (h_ovf) cudaFreeHost(h_ovf);
    db.release();
    *this = StreamSlot{};
  }
};

}  // namespace

struct sw_handle_s {
  int device = 0;
  int num_sms = 0;
  // scoring scheme
  int A = 0, rho = 0, sigma = 0, max_w = 0, min_w = 0;
  // Kernel-side penalties: any rho, sigma >= 0 is accepted.
  //  * profile offset c = min(rho, 127 - max_w): the int8 profile holds w + c; delta = rho - c > 0
  //    selects the WIDE kernels, which add delta back per cell (sw_engine.cuh ChainConstT);
  //  * s16x2 lanes: rho16 = min(rho, 16384), sigma16 = min(sigma, 16384) and, if either was
  //    clamped, flag_limit = 16384: for a sequence whose every H is <= flag_limit - 1 a penalty
  //    above that bound can never make a positive E / F term (E, F <= H - penalty < 0) in either
  //    system, so its H values are identical; any sequence reaching flag_limit is recomputed;
  //    rho16 + sigma16 <= 32768 keeps E - sigma, F - sigma >= -32768 (no wrap);
  //  * s32 lanes (recompute, traceback): the same clamp at 2^29 (every H <= m * 127 < 2^27).
  int c_prof = 0, rho16 = 0, sigma16 = 0, flag_limit = 0, rho32 = 0, sigma32 = 0;
  bool wide = false;
  int8_t* d_matrix = nullptr;
  std::vector<uint8_t> query;
  // database (the loaded one; sw_search_stream points db at its chunk slots)
  DbState main_db;
  DbState* db = &main_db;
  StreamSlot stream_slot[2];
  int64_t stat_recomputed = -1;   // >= 0: set by sw_search_stream (sum over its chunks)
  // traceback scratch
  uint8_t* d_tb_dir = nullptr; size_t tb_dir_cap = 0;
  int* d_tb_scratch = nullptr; size_t tb_scratch_cap = 0;
  int* d_tb_result = nullptr; size_t tb_result_cap = 0;
  uint32_t* d_tb_ops = nullptr; size_t tb_ops_cap = 0;
  uint8_t* d_tk = nullptr; size_t tk_cap = 0;         // sw_top_hits scratch
  uint8_t* d_tb_query = nullptr; size_t tb_query_cap = 0;
  KernelConfig last_cfg{};
  int32_t last_threshold = 0;
  // measured plan choice per (query length, threshold) on the loaded database (run_batch
  // autotune; -1 = keep the model's choice); cleared by sw_load_db
  std::map<std::pair<int, int32_t>, int> tuned;
  // measured automatic threshold per query length on the loaded database (run_batch autotune of
  // SW_AUTO_THRESHOLD: the model's best candidates and the all-short endpoint, timed); cleared by
  // sw_load_db
  std::map<int, int64_t> tuned_T;
  int tune_force = -1;            // menu entry forced while tuning / from the tuned table
  std::vector<uint32_t> qmask;    // letters present in each query of the current batch
  // scratch
  std::vector<QuerySlot> slots;
  int32_t* d_scores_tmp = nullptr;
  int64_t scores_tmp_cap = 0;
  uint8_t* d_batch_q = nullptr;
  int64_t batch_q_cap = 0;
  cudaEvent_t fork = nullptr;
  // completion of the last T-mode launch with gangs: the next one waits for it (gang CTAs spin
  // on each other, so two gang launches must never hold SMs at the same time; sw_engine.cuh
  // t_gang_item)
  cudaEvent_t gang_ev = nullptr;
  cudaStream_t copy_st = nullptr;   // blocking API: per-query score copies as queries finish
  uint32_t gang_epoch = 0;        // tag epoch of the last gang launch (sw_engine.cuh run_pass GPU_FLAGS)
  // stats
  int64_t stat_long = 0, stat_short = 0, stat_launches = 0;
  int stat_nq = 0;
  int32_t* h_ovf = nullptr;       // pinned, one overflow count per query of the last batch
  int h_ovf_cap = 0;
  // kEvPerQuery per query: [0] before the search launches, [1] after them (long path joined),
  // [2] after the recompute, [3] / [4] around the separate long-path (T-mode) launch
  std::vector<cudaEvent_t> ev;
  std::vector<char> long_fused;   // per query of the last batch: long pairs ran inside k_search
  std::string err;
};

namespace {

constexpr int kEvPerQuery = 5;

int fail(sw_handle h, int code, const std::string& msg) {
  if (h) h->err = msg;
  return code;
}

int cuda_fail(sw_handle h, cudaError_t e, const char* what) {
  std::string m = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
  if (h) h->err = m;
  return e == cudaErrorMemoryAllocation ? SW_E_NOMEM : SW_E_CUDA;
}

#define SW_CUDA(h, call)                                   \
  do {                                                     \
    cudaError_t _e = (call);                               \
    if (_e != cudaSuccess) return cuda_fail((h), _e, #call); \
  } while (0)

template <class T>
int grow(sw_handle h, T** p, size_t* cap, size_t bytes, const char* what, cudaStream_t busy = nullptr,
         bool zero = false) {
  if (*cap >= bytes && *p) return SW_OK;
  if (busy) cudaStreamSynchronize(busy);  // the old buffer may still be in use on this stream
  if (*p) cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  if (bytes == 0) return SW_OK;
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), bytes);
  if (e != cudaSuccess) return cuda_fail(h, e, what);
  // zero: the row buffers' leading slot of every strip buffer must read as the neutral entry
  // (H, F + rho) = (0, 0) (run_pass); it is only ever rewritten with neutral values.  Ordered
  // on the stream that will use the buffer.
  if (zero) {
    e = cudaMemsetAsync(*p, 0, bytes, busy);
    if (e != cudaSuccess) return cuda_fail(h, e, what);
  }
  *cap = bytes;
  return SW_OK;
}

int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// G = 32 group items run as one continuous stream per warp (sw_engine.cuh group_stream);
// SW_GROUP_STREAM=0 selects the per-strip sweeps instead (A/B measurements, tests)
bool group_stream_enabled() {
  const char* f = getenv("SW_GROUP_STREAM");
  return !(f && f[0] == '0');
}

// ------------------------------------------------------------------------------------ planning
ProfLayout make_layout(int off, int G, int R, int m, int A1, int nrep) {
  ProfLayout L;
  L.off = off;
  L.G = G;
  L.R = R;
  L.cb = (R >= 12) ? 16 : (R % 8 == 0) ? 8 : 4;   // == chunk_bytes<R>() (sw_engine.cuh)
  L.nch = (R + L.cb - 1) / L.cb;
  L.strips = (m + G * R - 1) / (G * R);
  L.ls = (int)round_up((int64_t)L.strips * L.nch * G * L.cb, 128);
  L.nrep = nrep;
  L.rs = (int)round_up((int64_t)A1 * L.ls, 128) + (nrep > 1 ? (L.cb * G) % 128 : 0);
  L.bytes = (int)round_up((int64_t)(nrep - 1) * L.rs + (int64_t)A1 * L.ls, 128);
  return L;
}

struct Plan {
  KernelConfig cfg;
  int short_passes, long_passes, team_warps;
  ProfLayout lg, lt;   // main kernel blob
  int prof_bytes;
  // s32 recompute
  KernelConfig rcfg;
  int r_passes, r_team_warps;
  ProfLayout rl;       // recompute blob (team image only)
  int r_prof_bytes;
  int grid, rgrid;
  double cost;         // estimated cycles of the main launch
  double thr, tail_s;  // its throughput term and the critical path of the longest short item
  double thr_full;     // the throughput term at full occupancy (no few-items penalty)
};

int team_warps_for(int passes, int warps) {
  if (passes <= 1) return 1;
  const int rounds = (passes + warps - 1) / warps;
  return (passes + rounds - 1) / rounds;
}

void main_layouts(const KernelConfig& c, int m, int A1, ProfLayout* lg, ProfLayout* lt, int* bytes) {
  *lg = make_layout(0, c.G, c.Rs, m, A1, 32 / c.G);
  if (c.G == 32 && c.Rs == c.Rl) {
    *lt = *lg;
    *bytes = lg->bytes;
  } else {
    *lt = make_layout(lg->bytes, 32, c.Rl, m, A1, 1);
    *bytes = lg->bytes + lt->bytes;
  }
}

constexpr int kMaxProfileSmem = SW_MAX_PROFILE_BYTES;   // include/sw.h

// Workload summary of one regime split (from the sorted, paired layout).
struct Split {
  int n_long = 0, n_short = 0;          // pairs
  int64_t long_cols = 0, short_cols = 0;
  int64_t long_max_cols = 0, short_max_cols = 0;
};

// Pick the menu entry with the smallest estimated time: the larger of
//  * throughput: warp-steps x ALU instructions per step / the SM array's measured issue rate
//    (group steps = sum over short pairs of (n' + G - 1) x strips / pairs per warp; team
//    steps = sum over long pairs of (n' + 31) x strips), and
//  * the critical path of the longest item (long: its strips split over the team's warps;
//    short: one group), at the issue rate one warp gets while sharing its scheduler.
int make_plan(sw_handle h, int m, const Split& sp, Plan* pl, int force = -1,
              std::vector<std::pair<double, int>>* ranked = nullptr) {
  const int A1 = h->A + 1;
  const double kGpuIssue = 2.7 * h->num_sms;  // ALU warp-instructions per clock, whole GPU
  const double kWarpIssue = 0.2;              // one warp's share of its scheduler
  double best = 1e300;
  int best_i = -1;
  for (int i = 0; i < menu_size(); ++i) {
    const KernelConfig c = menu_entry(i);
    if (c.lane != 0 || (c.wide != 0) != h->wide) continue;
    ProfLayout lg, lt;
    int bytes = 0;
    main_layouts(c, m, A1, &lg, &lt, &bytes);
    if (bytes > kMaxProfileSmem) continue;
    // several strips with G < 32 (run_pass per strip): each strip pays its own pipeline fill
    // (counted below) and the row-buffer store / ring fetch per step (~8 instructions);
    // measured best for m = 464-1000 (profiles/r01_plan_check.jsonl)
    const double strip_extra = (lg.strips > 1 && c.G < 32) ? 8.0 : 0.0;
    // ALU instructions per step; 2 warps per scheduler hide the F -> H -> H - rho chain (~13
    // cycles per row, through the FMA pipe) worse than 3: measured +11 % time (R = 43, 256 vs
    // 384 threads, profiles/r01_plan_check.jsonl); 4 warps per scheduler measured no better than 3
    const double wps = c.threads / 128.0;
    const double lat = wps < 2.5 ? 1.10 : 1.0;
    const double is = (6.5 * c.Rs + 24.0 + strip_extra) * lat, il = (6.5 * c.Rl + 40.0) * lat;
    const int W = team_warps_for(lt.strips, c.threads / 32);
    // (G = 32 streams: a 4-column gap per segment plus ~3 steps' worth of per-lane resets)
    const double fill = (c.G == 32 && group_stream_enabled()) ? 7.0 : c.G - 1.0;
    const double gsteps = ((double)sp.short_cols + (double)sp.n_short * fill) * lg.strips / (32 / c.G);
    const double tsteps = ((double)sp.long_cols + 31.0 * sp.n_long) * lt.strips;
    // team mode: a CTA holds floor(warps / W) teams; warps beyond the last whole team idle
    // (W = 7 of 12 warps measured 32 % slower than W = 6 on C3 with query 5478)
    const int cta_warps = c.threads / 32;
    const double team_util = (double)((cta_warps / W) * W) / cta_warps;
    double thr = (gsteps * is + tsteps * il / team_util) / kGpuIssue;
    // few items: the issue rate needs ~2 busy warps per scheduler (4 per SM)
    const double active_warps = (double)sp.n_short / (32 / c.G) + (double)sp.n_long * W;
    const double thr_full = thr;
    thr /= std::min(1.0, std::max(0.05, active_warps / (8.0 * h->num_sms)));
    const double tail_l = sp.n_long ? (sp.long_max_cols + 31.0) * ((lt.strips + W - 1) / W) * il / kWarpIssue : 0.0;
    const double tail_s = sp.n_short ? (sp.short_max_cols + c.G - 1.0) * lg.strips * is / kWarpIssue : 0.0;
    const double cost = std::max(thr, std::max(tail_l, tail_s));
    if (ranked) ranked->emplace_back(cost, i);
    if (cost < best) { best = cost; best_i = i; pl->thr = thr; pl->tail_s = tail_s; pl->thr_full = thr_full; }
  }
  // a forced entry must be able to hold the profile values: WIDE entries compute any rho
  // (delta = 0 included), the others only rho + max_w <= 127
  auto usable = [&](int i) {
    return i >= 0 && i < menu_size() && menu_entry(i).lane == 0 && (menu_entry(i).wide || !h->wide);
  };
  if (usable(force)) best_i = force;
  pl->cost = best;
  // test hooks: force a menu entry / team size (used by the parity tests to cover every
  // compiled configuration; never needed for correctness)
  if (const char* f = getenv("SW_FORCE_MENU")) {
    const int i = atoi(f);
    if (usable(i)) best_i = i;
  }
  if (best_i < 0) return fail(h, SW_E_UNSUPPORTED, "query profile does not fit in shared memory (query_len * (alphabet_size + 1) too large)");
  const KernelConfig c = menu_entry(best_i);
  if (getenv("SW_DEBUG_PLAN"))
    fprintf(stderr, "plan m=%d menu=%d G=%d Rs=%d Rl=%d threads=%d cost=%.4g\n", m, best_i, c.G, c.Rs, c.Rl, c.threads,
            best);
  pl->cfg = c;
  main_layouts(c, m, A1, &pl->lg, &pl->lt, &pl->prof_bytes);
  if (pl->prof_bytes > kMaxProfileSmem) return fail(h, SW_E_UNSUPPORTED, "query profile does not fit in shared memory");
  pl->short_passes = pl->lg.strips;
  pl->long_passes = pl->lt.strips;
  pl->team_warps = team_warps_for(pl->long_passes, c.threads / 32);
  if (const char* f = getenv("SW_FORCE_TEAM_WARPS")) {
    const int w = atoi(f);
    if (w >= 1 && w <= c.threads / 32) pl->team_warps = std::min(w, std::max(1, pl->long_passes));
  }
  pl->rcfg = recompute_config(h->wide);
  pl->rl = make_layout(0, 32, pl->rcfg.Rl, m, A1, 1);
  pl->r_prof_bytes = pl->rl.bytes;
  if (pl->r_prof_bytes > kMaxProfileSmem) return fail(h, SW_E_UNSUPPORTED, "query profile does not fit in shared memory");
  pl->r_passes = pl->rl.strips;
  pl->r_team_warps = team_warps_for(pl->r_passes, pl->rcfg.threads / 32);
  int bps = 0;
  cudaError_t e = configure_kernel(c, pl->prof_bytes, &bps);
  if (e != cudaSuccess) return cuda_fail(h, e, "configure search kernel");
  if (bps < 1) return fail(h, SW_E_UNSUPPORTED, "search kernel cannot be resident");
  pl->grid = bps * h->num_sms;
  e = configure_kernel(pl->rcfg, pl->r_prof_bytes, &bps);
  if (e != cudaSuccess) return cuda_fail(h, e, "configure recompute kernel");
  if (bps < 1) return fail(h, SW_E_UNSUPPORTED, "recompute kernel cannot be resident");
  pl->rgrid = bps * h->num_sms;
  return SW_OK;
}

int ensure_slots(sw_handle h, int n) {
  while ((int)h->slots.size() < n) {
    QuerySlot s;
    SW_CUDA(h, cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking));
    SW_CUDA(h, cudaStreamCreateWithFlags(&s.aux, cudaStreamNonBlocking));
    {   // the row-scan clusters must be placed before the T-mode kernel's persistent CTAs fill the
        // GPU (launched first on their own stream, but only priority makes the order hold)
      int lo = 0, hi = 0;
      SW_CUDA(h, cudaDeviceGetStreamPriorityRange(&lo, &hi));
      SW_CUDA(h, cudaStreamCreateWithPriority(&s.scan, cudaStreamNonBlocking, hi));
    }
    SW_CUDA(h, cudaEventCreateWithFlags(&s.scan_fork, cudaEventDisableTiming));
    SW_CUDA(h, cudaEventCreateWithFlags(&s.scan_done, cudaEventDisableTiming));
    SW_CUDA(h, cudaEventCreateWithFlags(&s.fork, cudaEventDisableTiming));
    SW_CUDA(h, cudaEventCreateWithFlags(&s.join, cudaEventDisableTiming));
    SW_CUDA(h, cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming));
    // 4 work counters, then 4 neutral row-buffer entries (uint2 zeros) read by group_stream
    SW_CUDA(h, cudaMalloc(&s.d_work, 12 * sizeof(int32_t)));
    SW_CUDA(h, cudaMemset(s.d_work, 0, 12 * sizeof(int32_t)));
    SW_CUDA(h, cudaMalloc(&s.d_ovf_count, sizeof(int32_t)));
    h->slots.push_back(s);
  }
  return SW_OK;
}

// Make stream st wait for all work the previous call enqueued on the internal slot streams
// (each slot records `done` after its last query, with its T-mode stream joined back).
int wait_slots(sw_handle h, cudaStream_t st) {
  for (QuerySlot& s : h->slots)
    if (s.stream != st) SW_CUDA(h, cudaStreamWaitEvent(st, s.done, 0));
  return SW_OK;
}

int validate_query(sw_handle h, const uint8_t* q, int32_t m) {
  if (!q) return fail(h, SW_E_INVALID, "query is NULL");
  if (m <= 0 || m > SW_MAX_QUERY_LEN) return fail(h, SW_E_INVALID, "query_len out of range [1, 65536]");
  for (int32_t i = 0; i < m; ++i)
    if (q[i] >= h->A) return fail(h, SW_E_INVALID, "query code >= alphabet_size at position " + std::to_string(i));
  return SW_OK;
}

// regime split: sorted_len is descending; long = n >= T (§II-B)
Split make_split(sw_handle h, int64_t T, int64_t* n_long_seqs_out) {
  const int64_t n_long_seqs =
      std::lower_bound(h->db->sorted_len.begin(), h->db->sorted_len.end(), T, std::greater_equal<int64_t>()) -
      h->db->sorted_len.begin();
  const int n_long = (int)((n_long_seqs + 1) / 2);
  Split sp;
  sp.n_long = n_long;
  sp.n_short = h->db->n_pairs - n_long;
  sp.long_cols = h->db->pair_cols_prefix[n_long];
  sp.short_cols = h->db->pair_cols_prefix[h->db->n_pairs] - sp.long_cols;
  sp.long_max_cols = n_long ? h->db->h_pair_ncols[0] : 0;
  sp.short_max_cols = sp.n_short ? h->db->h_pair_ncols[n_long] : 0;
  if (n_long_seqs_out) *n_long_seqs_out = n_long_seqs;
  return sp;
}

// Automatic inter/intra-task threshold (§VI: "characterize
// the relative performance of the inter-task and intra-task kernels based on the mean and
// maximum lengths ... during the database preprocessing step, we can find the transition
// point").  For each candidate T the planner's time model gives the group (inter-task)
// launch's throughput time and the critical path of its longest item; the long (intra-task)
// pairs run concurrently in T-mode at ~1.8x the group cost per cell (measured,
// profiles/r01_sweep_*.jsonl).  Estimated time = max(throughput of both launches,
// group tail / 0.8); the cheapest candidate wins (ties: the larger T).
std::vector<std::pair<double, int64_t>> rank_thresholds(sw_handle h, int m);

int64_t choose_threshold(sw_handle h, int m) {
  if (h->db == &h->main_db) {
    const auto it = h->tuned_T.find(m);
    if (it != h->tuned_T.end()) return it->second;
  }
  const auto ranked = rank_thresholds(h, m);
  return ranked.empty() ? 3072 : ranked.front().second;
}

// The candidates of choose_threshold with the model's estimated time, cheapest first (ties
// within 0.5 %: the larger T, i.e. the candidate order).
std::vector<std::pair<double, int64_t>> rank_thresholds(sw_handle h, int m) {
  std::vector<std::pair<double, int64_t>> out;
  const int64_t maxlen = h->db->sorted_len.empty() ? 0 : h->db->sorted_len[0];
  const int64_t cands[] = {maxlen + 1, 16384, 12288, 8192, 6144, 4096, 3072, 2048, 1536, 1024, 768, 512};
  const std::string saved = h->err;
  // group cost per database column, from the plan with every pair in the group launch
  double per_col = 0.0;
  {
    Split sp = make_split(h, maxlen + 1, nullptr);
    Plan pl;
    if (!make_plan(h, m, sp, &pl) && sp.short_cols > 0) per_col = pl.thr_full * (2.7 / 2.0) / (double)sp.short_cols;
  }
  // long path cost per column relative to the group path at full occupancy, measured (C3 all
  // long vs C2 short-only, profiles/r01_sweep_*.jsonl, with the T-mode team stream): 2.02 at
  // m = 144, 1.55 at 567, 1.44 at 1500, 1.16 at 5478 (linear in between)
  const double lm[] = {144, 567, 1500, 5478}, lf[] = {2.02, 1.55, 1.44, 1.16};
  double long_factor = lf[3];
  if (m <= lm[0]) long_factor = lf[0];
  for (int k = 0; k < 3; ++k)
    if (m > lm[k] && m <= lm[k + 1]) long_factor = lf[k] + (lf[k + 1] - lf[k]) * (m - lm[k]) / (lm[k + 1] - lm[k]);
  for (int64_t T : cands) {
    if (T > maxlen + 1) continue;
    Split sp = make_split(h, T, nullptr);
    const double long_cols = (double)sp.long_cols;
    sp.n_long = 0; sp.long_cols = 0; sp.long_max_cols = 0;   // the group launch alone
    Plan pl;
    if (sp.n_short > 0 && make_plan(h, m, sp, &pl)) continue;
    if (sp.n_short == 0) { pl.thr = 0.0; pl.tail_s = 0.0; }
    // measured rates: the whole GPU sustains ~0.5 ALU warp-instructions / clock / scheduler
    // (not the model's 2.7 / SM), and a tail warp ~0.15 (profiles/r01_ncu_*, query sweeps)
    const double thr = pl.thr * (2.7 / 2.0), tail = pl.tail_s * (0.2 / 0.15);
    const double thr_long = per_col * long_cols * long_factor;
    const double cost = std::max(thr + thr_long, tail / 0.8);
    if (getenv("SW_DEBUG_AUTO"))
      fprintf(stderr, "auto m=%d T=%lld G=%d Rs=%d thr=%.3f long=%.3f tail=%.3f cost=%.3f ms\n", m, (long long)T,
              pl.cfg.G, pl.cfg.Rs, thr / 1.965e6, thr_long / 1.965e6, tail / 1.965e6, cost / 1.965e6);
    out.emplace_back(cost, T);
  }
  h->err = saved;
  // stable: equal (within 0.5 %) costs keep the candidate order, larger T first
  std::stable_sort(out.begin(), out.end(), [](const std::pair<double, int64_t>& a, const std::pair<double, int64_t>& b) {
    return a.first < b.first * 0.995;
  });
  return out;
}

// Long-query mode: the smallest query-profile image (the s32 recompute's team image, 32 lanes x
// 16 rows per strip, one replica; every group / team image is at least as large) exceeds the
// shared memory of one CTA.  SW_LONG_QUERY=1 forces the mode (tests, probes).
bool long_query_mode(sw_handle h, int m) {
  if (const char* f = getenv("SW_LONG_QUERY"))
    if (f[0] == '1') return true;
  const KernelConfig rc = recompute_config(h->wide);
  return make_layout(0, 32, rc.Rl, m, h->A + 1, 1).bytes > kMaxProfileSmem;
}

// Enqueue one query (device query pointer) on slot s; scores to d_out (device, caller order).
int enqueue_query(sw_handle h, QuerySlot& s, const uint8_t* d_q, int m, uint32_t qmask, int32_t* d_out, int32_t T,
                  int32_t* h_ovf, cudaEvent_t* ev) {
  // Long-query mode: when even the smallest query-profile image
  // does not fit one CTA's shared memory, every pair takes T-mode, which streams the query
  // from global memory and builds its substitution tables per database strip (no query
  // profile), and the flagged sequences are recomputed by T-mode's 32-bit instantiation.
  // The threshold then only names the path: every sequence is a "long" one.
  const bool longq = long_query_mode(h, m);
  if (longq) T = 0;
  else if (T == SW_AUTO_THRESHOLD) T = (int32_t)std::min<int64_t>(choose_threshold(h, m), INT32_MAX);
  h->last_threshold = T;
  int64_t n_long_seqs = 0;
  const Split sp = make_split(h, T, &n_long_seqs);
  const int n_long = sp.n_long;
  // menu entry: forced while tuning, else the measured one for (m, T) if run_batch tuned it
  int force = h->tune_force;
  if (force < 0 && h->db == &h->main_db) {
    const auto it = h->tuned.find({m, T});
    if (it != h->tuned.end()) force = it->second;
  }
  Plan pl{};
  int rc = longq ? SW_OK : make_plan(h, m, sp, &pl, force);
  if (rc) return rc;
  // Long pairs: T-mode (strips along the database sequence) when the query is short enough
  // that team mode would have few query strips to spread over warps; team mode otherwise.
  // Measured on C3 (all long, profiles/r01_longmode_grid.txt): T-mode ahead up to m = 2504
  // (567: 3347 vs 1190 GCUPS, 1500: 3676 vs 2655, 2504: 3765 vs 3507), team mode from
  // m = 3564 (3916 vs 3795, 5478: 4335 vs 3838).  SW_LONG_MODE=team|t overrides (tests).
  bool use_t = n_long > 0 && m < kTmodeMaxQuery;
  if (const char* f = getenv("SW_LONG_MODE")) {
    if (!strcmp(f, "team")) use_t = false;
    if (!strcmp(f, "t")) use_t = n_long > 0;
  }
  if (longq) use_t = n_long > 0;
  if (use_t && !longq) {
    // the main launch then only sees the short pairs: plan it for them
    Split ss = sp;
    ss.n_long = 0; ss.long_cols = 0; ss.long_max_cols = 0;
    rc = make_plan(h, m, ss, &pl, force);
    if (rc) return rc;
  }
  h->last_cfg = pl.cfg;

  // scratch: profile, overflow list, row buffers
  const int r_off = (int)round_up(pl.prof_bytes, 256);
  rc = grow(h, &s.d_prof, &s.prof_cap, (size_t)(r_off + pl.r_prof_bytes), "alloc profile", s.stream);
  if (rc) return rc;
  size_t ovf_bytes = (size_t)std::max<int64_t>(h->db->n_seqs, 1) * sizeof(int32_t);
  size_t ovf_cap = (size_t)s.ovf_cap * sizeof(int32_t);
  rc = grow(h, &s.d_ovf_list, &ovf_cap, ovf_bytes, "alloc overflow list", s.stream);
  if (rc) return rc;
  s.ovf_cap = (int64_t)(ovf_cap / sizeof(int32_t));
  // row-buffer slots: the pair's columns (+ pad tail) plus one leading neutral entry
  const int64_t max_cols_all = h->db->n_pairs ? h->db->h_pair_ncols[0] + kPadCols + 1 : 0;
  const int64_t max_cols_short = (n_long < h->db->n_pairs) ? h->db->h_pair_ncols[n_long] + kPadCols + 1 : 0;
  const int G = pl.cfg.G;
  size_t rbg = 0;
  if (pl.short_passes > 1 && max_cols_short > 0)
    rbg = (size_t)pl.grid * (pl.cfg.threads / 32) * (32 / G) * (max_cols_short + 4) * sizeof(uint2);
  size_t rbt = 0;
  if (pl.long_passes > 1 && n_long > 0 && !use_t) {
    const int nteams = (pl.cfg.threads / 32) / pl.team_warps;
    rbt = (size_t)pl.grid * nteams * (pl.team_warps + 1) * max_cols_all * sizeof(uint2);
  }
  if (pl.r_passes > 1) {
    // the recompute list is rare and unknown until the search ran: bound its row buffers by
    // shrinking the (persistent) recompute grid instead of sizing for every CTA (a database
    // with a 1M-residue sequence would otherwise need ~15 GB per slot)
    const int nteams = (pl.rcfg.threads / 32) / pl.r_team_warps;
    const size_t per_cta = (size_t)nteams * (pl.r_team_warps + 1) * max_cols_all * sizeof(uint2);
    constexpr size_t kRecomputeRbBudget = (size_t)256 << 20;
    pl.rgrid = (int)std::max<size_t>(1, std::min<size_t>(pl.rgrid, kRecomputeRbBudget / std::max<size_t>(per_cta, 1)));
    rbt = std::max(rbt, (size_t)pl.rgrid * per_cta);
  }
  rc = grow(h, &s.d_rb_group, &s.rb_group_cap, rbg, "alloc group row buffers", s.stream, true);
  if (rc) return rc;
  rc = grow(h, &s.d_rb_team, &s.rb_team_cap, rbt, "alloc team row buffers", s.stream, true);
  if (rc) return rc;

  const int qcols = (int)round_up(m, 8);
  // T-mode strip tables hold one row per letter PRESENT in the query plus the pad row (the
  // query stream carries compact letter indices): 21 rows for a 20-letter query instead of 25,
  // so more warps fit in shared memory
  const int a_used = __builtin_popcount(qmask);
  const int wp_bytes = (int)round_up((int64_t)(a_used + 1) * kWpStride, 128);
  const int per_warp = 2 * (a_used + 1) * 32 * kTmodeC;
  // (k_search_t also holds ~3 KB of static shared memory: progress flags, the team streams' pair
  // pool; 220 KB + 3 KB stays below the 227 KB per CTA)
  int t_warps = std::min(kTmodeThreads / 32, (kMaxProfileSmem - wp_bytes) / per_warp);
  if (t_warps < 1) use_t = false;
  int t_grid = 0;
  const int t_smem = wp_bytes + t_warps * per_warp;
  // team-stream layout (a compile-time variant of k_search_t): packed lanes when the long pairs
  // average one to three strips (their one-pair-per-strip padding is large and they hand off
  // between strips anyway: C2 at T = 512, 3558 vs 2962 GCUPS); one pair per strip otherwise —
  // longer pairs (T = 1172: 3553 vs 3413; T = 3072: 0.96 vs 1.23 ms) and sub-strip pairs, whose
  // strips then need no hand-off at all (T = 0: 2147 vs 1966) (profiles/r02_tmode_packed.txt)
  const double t_mean_cols = n_long > 0 ? (double)sp.long_cols / n_long : 0.0;
  bool t_packed = t_mean_cols >= 32 * kTmodeC && t_mean_cols < 3.0 * 32 * kTmodeC;
  if (const char* f = getenv("SW_T_PACKED")) t_packed = atoi(f) != 0;
  if (use_t) {
    int bps = 0;
    cudaError_t e = configure_tmode_kernel(t_smem, &bps, h->wide, false, t_packed);
    if (e != cudaSuccess) return cuda_fail(h, e, "configure long-sequence kernel");
    t_grid = std::max(1, bps) * h->num_sms;
    rc = grow(h, &s.d_qpair, &s.qpair_cap, (size_t)(qcols + kPadCols) * sizeof(uint16_t), "alloc query stream",
              s.stream);
    if (rc) return rc;
    rc = grow(h, &s.d_rb_t, &s.rb_t_cap, (size_t)t_grid * 2 * t_warps * (qcols + kPadCols + 1) * sizeof(uint2),
              "alloc long-sequence row buffers", s.stream, true);
    if (rc) return rc;
  }

  cudaStream_t st = s.stream;
  SW_CUDA(h, cudaMemsetAsync(s.d_work, 0, 4 * sizeof(int32_t), st));
  SW_CUDA(h, cudaMemsetAsync(s.d_ovf_count, 0, sizeof(int32_t), st));
  if (!longq) {
    SW_CUDA(h, launch_profile(s.d_prof, pl.lg, d_q, m, h->d_matrix, h->A, h->c_prof, st));
    if (pl.lt.off != pl.lg.off) SW_CUDA(h, launch_profile(s.d_prof, pl.lt, d_q, m, h->d_matrix, h->A, h->c_prof, st));
    SW_CUDA(h, launch_profile(s.d_prof + r_off, pl.rl, d_q, m, h->d_matrix, h->A, h->c_prof, st));
  }

  SearchParams p{};
  p.prof = s.d_prof;
  p.prof_bytes = pl.prof_bytes;
  p.lg = pl.lg;
  p.lt = pl.lt;
  p.pad_letter = h->A;
  p.rho = h->rho16;
  p.sigma = h->sigma16;
  p.delta = h->rho16 - h->c_prof;
  p.flag_limit = h->flag_limit;
  p.max_w = h->max_w;
  p.cols = h->db->d_cols;
  p.pair_off = h->db->d_pair_off;
  p.pair_ncols = h->db->d_pair_ncols;
  p.n_pairs = h->db->n_pairs;
  p.n_seqs = (int)h->db->n_seqs;
  p.perm = h->db->d_perm;
  p.scores = d_out;
  p.n_long = use_t ? 0 : n_long;
  p.short_begin = n_long;
  p.item_list = nullptr;
  p.item_count = nullptr;
  p.work = s.d_work;
  p.rb_zero = reinterpret_cast<const uint2*>(s.d_work + 4);
  p.hi_mul = 1u << 24;
  p.ovf_list = s.d_ovf_list;
  p.ovf_count = s.d_ovf_count;
  p.short_passes = pl.short_passes;
  p.long_passes = pl.long_passes;
  p.team_warps = pl.team_warps;
  p.rb_group = s.d_rb_group;
  p.rb_group_cols = max_cols_short + 4;   // + 4 leading entries (group_stream gap-position stores)
  // (the stream addresses columns with 32-bit indices)
  p.group_stream = group_stream_enabled() && h->db->h_pair_off[h->db->n_pairs] < (int64_t)INT32_MAX;
  p.rb_team = s.d_rb_team;
  p.rb_team_cols = max_cols_all;
  SW_CUDA(h, cudaEventRecord(ev[0], st));
  {   // team mode: the long pairs run inside k_search (no separate long-path interval)
    const size_t k = (size_t)(ev - h->ev.data()) / kEvPerQuery;
    if (k < h->long_fused.size()) h->long_fused[k] = (char)(n_long > 0 && !use_t);
  }
  if (!use_t) {   // no separate long-path launch: an empty interval
    SW_CUDA(h, cudaEventRecord(ev[3], st));
    SW_CUDA(h, cudaEventRecord(ev[4], st));
  }
  if (use_t) {
    // T-mode runs on the slot's second stream, concurrently with the group launch: its CTAs
    // take every SM first (launched first), and as they run out of long pairs the group
    // launch's CTAs take their SMs, so the longest long pair overlaps the short-pair work.
    // (long-query mode: T-mode is the only search launch and runs on the slot's stream)
    SW_CUDA(h, launch_qpair(s.d_qpair, d_q, m, qcols + kPadCols, qmask, st));
    cudaStream_t tst = longq ? st : s.aux;
    if (!longq) {
      SW_CUDA(h, cudaEventRecord(s.fork, st));
      SW_CUDA(h, cudaStreamWaitEvent(s.aux, s.fork, 0));
    }
    TParams t{};
    std::vector<int32_t> h_gang_base;   // per-gang CTA slot offsets (uploaded with the gang scratch)
    std::vector<int> scan_ctas, scan_cols;   // row-scan items [0, size): cluster size, columns per CTA
    t.matrix = h->d_matrix;
    t.A = h->A;
    t.rho = h->rho16;
    t.sigma = h->sigma16;
    t.delta = h->rho16 - h->c_prof;
    t.flag_limit = h->flag_limit;
    t.max_w = h->max_w;
    t.pad_letter = h->A;
    t.qmask = qmask;
    t.A_used = a_used;
    t.qpair = s.d_qpair;
    t.qcols = qcols;
    t.cols = h->db->d_cols;
    t.pair_off = h->db->d_pair_off;
    t.pair_ncols = h->db->d_pair_ncols;
    t.n_items = n_long;
    t.n_seqs = (int)h->db->n_seqs;
    t.perm = h->db->d_perm;
    t.scores = d_out;
    t.ovf_list = s.d_ovf_list;
    t.ovf_count = s.d_ovf_count;
    t.work = s.d_work + 3;
    t.warps = t_warps;
    // Team sizes from a time model.  A team of W warps walks
    // the S strips of a pair; strip s + 1 trails strip s by ~lag steps (32-lane fill + the
    // 16-column progress granularity), each strip is qsteps = m + 32 steps, so a team is
    // pipeline-bound unless W * lag <= qsteps.  Phase 1 (pairs with >= big_strips strips, one
    // team of all t_warps warps) only pays when the longest pair's time dominates.
    //   est = max(sum over phases of warp-steps / (all warps x utilisation), longest pair)
    {
      const double lag = 44.0, qsteps = (double)round_up(qcols + 32, 4);
      const double nw = (double)t_grid * t_warps;
      const int spos = 32 * kTmodeC;
      // busy fraction of a W-warp team: the team stream (t_team_stream) runs its pairs' strips
      // back to back, so only the pipeline bound remains (strip s + 1 trails strip s by lag
      // steps inside a pair); the whole-CTA phase 1 still pays the per-pair rounding
      auto util = [&](int W, double S, bool whole_cta) {
        return std::min(1.0, qsteps / (W * lag)) * (whole_cta ? S / (W * std::ceil(S / W)) : 1.0);
      };
      auto item_time = [&](int W, double S) {
        return std::max(std::ceil(S / W) * qsteps, (S - 1.0) * lag + qsteps);
      };
      const int kBig = 16;
      double best_est = 1e300;
      int bestW = 1, best_big = 1 << 30;
      // (single-warp teams measured slower than the model says: not considered)
      for (int W = std::min(2, t_warps); W <= t_warps; ++W) {
        if (t_warps % W) continue;
        for (int phase1 = 0; phase1 < 2; ++phase1) {
          if (phase1 && W == t_warps) continue;
          double t_steps = 0.0, tail = 0.0;
          for (int pp = 0; pp < n_long; ++pp) {
            const double S = std::ceil((double)h->db->h_pair_ncols[pp] / spos);
            const bool whole = phase1 && S >= kBig;
            const int Wi = whole ? t_warps : W;
            t_steps += S * qsteps / util(Wi, S, whole);
            tail = std::max(tail, item_time(Wi, S));
          }
          const double est = std::max(t_steps / nw, tail) * (phase1 ? 1.05 : 1.0);
          // ties (within 2 %) go to the larger team: its pairs finish sooner (measured on C3:
          // W = 8 vs 4 +3.6 % for query 567, +3.8 % for 2504)
          if (est < 0.98 * best_est || (est <= 1.02 * best_est && W > bestW)) {
            best_est = std::min(est, best_est); bestW = W; best_big = phase1 ? kBig : (1 << 30);
          }
        }
      }
      int W = bestW;
      if (const char* f = getenv("SW_T_TEAM")) W = std::max(1, std::min(t_warps, atoi(f)));
      while (t_warps % W) --W;
      t.team_warps = W;
      t.big_strips = best_big;
      if (const char* f = getenv("SW_T_BIG")) t.big_strips = std::max(1, atoi(f));
      // Gangs (k_search_t phase 0): when the long pairs are not
      // hidden under a larger short-pair launch, a pair whose time alone exceeds the launch's
      // throughput estimate is spread over K CTAs x W warps (one warp per scheduler, the
      // CTA's other warps wait) until it reaches its wavefront bound ((S - 1) lag + qsteps).
      const int WG = std::min(4, t_warps);   // gang warps per CTA: one per scheduler
      t.gang_items = 0; t.gang_ctas = 1; t.gang_warps = WG;
      {
        constexpr int kMaxGangItems = 64, kMaxGangCtas = 8;
        double t_thr = 0.0;
        for (int pp = 0; pp < n_long; ++pp) {
          const double S = std::ceil((double)h->db->h_pair_ncols[pp] / spos);
          t_thr += S * qsteps / util(W, S, false);
        }
        t_thr /= nw;
        const bool hidden = (double)sp.short_cols > 0.5 * (double)sp.long_cols;
        int K = 0, items = 0;
        // Row scan (sw_scan.cu): in a launch that is not
        // hidden, a prefix of the longest pairs runs one query row per step on clusters of
        // K = ceil(ncols / kScanCols) CTAs.  The prefix length j minimises the launch estimate
        //   max(the scans: (qcols + K) x kScanRowSteps steps, all concurrent,
        //       the longest remaining wavefront (S - 1) lag + qsteps,
        //       the remaining pairs' throughput time on the SMs the clusters leave),
        // j = 0 being today's plan; at most 3/4 of the SMs in clusters.  SW_SCAN=0 disables it,
        // SW_SCAN=N forces it for the (up to 4) longest pairs of >= N columns.
        {
          int scan_min = kScanMinCols;
          bool forced = false;
          if (const char* f = getenv("SW_SCAN"); f && *f) { scan_min = atoi(f); forced = scan_min > 0; }
          double row_steps = kScanRowSteps;
          if (const char* f = getenv("SW_SCAN_ROW_STEPS")) row_steps = atof(f);   // probes
          int sms = 0;
          if (scan_min > 0 && (forced || !hidden) && !h->wide && a_used + 1 <= kScanMaxLetters) {
            std::vector<double> thr_tail(n_long + 1, 0.0);   // throughput steps of pairs [pp, n_long)
            for (int pp = n_long - 1; pp >= 0; --pp) {
              const double S = std::ceil((double)h->db->h_pair_ncols[pp] / spos);
              thr_tail[pp] = thr_tail[pp + 1] + S * qsteps / util(W, S, false) / nw;
            }
            auto wavefront = [&](int pp) {
              return pp < n_long ? (std::ceil((double)h->db->h_pair_ncols[pp] / spos) - 1.0) * lag + qsteps : 0.0;
            };
            double best = std::max(wavefront(0), thr_tail[0]), scan_t = 0.0;
            int best_j = 0;
            std::vector<int> ks, cs;
            for (int pp = 0; pp < n_long && pp < (forced ? 4 : kMaxScanItems); ++pp) {
              const int nc = h->db->h_pair_ncols[pp];
              if (nc < scan_min || nc > kScanMaxCtas * kScanCols) break;
              const int Kc = (nc + kScanCols - 1) / kScanCols;
              if (!forced && sms + Kc > 3 * h->num_sms / 4) break;
              sms += Kc;
              ks.push_back(Kc);
              cs.push_back(scan_cols_cta(nc, Kc));
              scan_t = std::max(scan_t, (qcols + Kc) * row_steps);
              const double left = 1.0 - (double)sms / h->num_sms;
              const double est = std::max({scan_t, wavefront(pp + 1), thr_tail[pp + 1] / left});
              if (forced || est < 0.97 * best) { best = std::min(best, est); best_j = pp + 1; }
            }
            scan_ctas.assign(ks.begin(), ks.begin() + best_j);
            scan_cols.assign(cs.begin(), cs.begin() + best_j);
            sms = 0;
            for (int k2 : scan_ctas) sms += k2;
          }
          if (getenv("SW_DEBUG_PLAN") && !scan_cols.empty())
            fprintf(stderr, "tmode scan items=%zu (%d SMs; first %d CTAs x %d columns)\n", scan_cols.size(), sms,
                    scan_ctas[0], scan_cols[0]);
        }
        // gangs for the long pairs after the scanned ones (gang gi = pair scan items + gi)
        const int s0 = (int)scan_cols.size();
        std::vector<int> Ks;   // CTAs of each gang (the longest pairs need more than the others)
        if (!hidden) {
          // a gang of GW warps: each warp runs ceil(S / GW) strips back to back after a ramp of
          // (GW - 1) lags, unless the wavefront (S - 1) lag + qsteps is longer (measured per
          // strip with SW_DEBUG_GANG_TIMES: the C2 35,213-residue pair, query 567: 3 CTAs
          // 0.81 ms, 4-8 CTAs 0.72 ms, profiles/r02_gang_*.txt)
          auto gang_time = [&](int GW, double S) {
            return std::max(std::ceil(S / GW) * qsteps + (std::min<double>(GW, S) - 1.0) * lag,
                            (S - 1.0) * lag + qsteps);
          };
          for (int pp = s0; pp < n_long && pp - s0 < kMaxGangItems; ++pp) {
            const double S = std::ceil((double)h->db->h_pair_ncols[pp] / spos);
            const double alone = item_time(S >= t.big_strips ? t_warps : W, S);
            if (alone <= 1.15 * t_thr || S < 2.0 * W) break;
            double best_g = 1e300;
            for (int k = 2; k <= kMaxGangCtas; ++k) best_g = std::min(best_g, gang_time(k * WG, S));
            const double goal = std::max(1.15 * t_thr, 1.03 * best_g);
            int k = 2;
            while (k < kMaxGangCtas && gang_time(k * WG, S) > goal) ++k;
            // the 4-bit hand-off tags (run_pass GPU_FLAGS) repeat every 15 strips: a slot is
            // reused every GW + 1 strips, which must not be a multiple of 15
            while (k > 2 && (k * WG + 1) % 15 == 0) --k;
            if ((k * WG + 1) % 15 == 0) break;
            Ks.push_back(k);
            K = std::max(K, k);
            ++items;
          }
          int total = 0;
          for (int i = 0; i < items; ++i) total += Ks[i];
          while (items > 0 && total > t_grid / 2) total -= Ks[--items];
          Ks.resize(items);
        }
        if (const char* f = getenv("SW_T_GANG")) {   // tests: "K" or "K:items" (one size for all)
          K = atoi(f);
          while (K >= 2 && (K * WG + 1) % 15 == 0) --K;
          const char* comma = strchr(f, ':');
          items = comma ? atoi(comma + 1) : n_long;
          items = std::min(items, std::min(n_long - s0, t_grid / std::max(1, K)));
          Ks.assign(std::max(items, 0), K);
        }
        if (getenv("SW_DEBUG_PLAN")) {
          fprintf(stderr, "tmode m=%d long_pairs=%d W=%d t_warps=%d big=%d thr=%.0f steps gangs=%d (CTAs", m,
                  n_long, W, t_warps, t.big_strips, t_thr, items);
          for (int i = 0; i < items; ++i) fprintf(stderr, " %d", Ks[i]);
          fprintf(stderr, ")\n");
        }
        if (items > 0 && K >= 2) {
          t.gang_items = items;
          t.gang_ctas = K;           // the largest gang (buffer stride); per-gang sizes in gang_base
          h_gang_base.assign(1, 0);
          for (int i = 0; i < items; ++i) h_gang_base.push_back(h_gang_base.back() + Ks[i]);
          t.big_strips = 1 << 30;
          // the gang CTAs' other warps wait (measured: letting them stream meanwhile slows the
          // gang's latency-bound strip pipeline more than it gains: C2 query 567 long-only at
          // T = 3072 1.156 -> 1.359 ms, profiles/r02_gang_share.txt); SW_T_GANG_SHARE=1 for A/B
          t.gang_share = 0;
          if (const char* f = getenv("SW_T_GANG_SHARE")) t.gang_share = atoi(f) != 0;
        }
      }
    }
    t.gang0 = (int)scan_cols.size();
    t.q0 = t.gang0 + t.gang_items;
    if (t.gang_items > 0) {
      const int GW = t.gang_ctas * t.gang_warps;
      const size_t ints = 1 + 3 * (size_t)t.gang_items + (size_t)t.gang_items * (GW + 1);
      rc = grow(h, &s.d_gang, &s.gang_cap, (ints + t.gang_items + 1) * sizeof(int32_t), "alloc gang scratch", tst);
      if (rc) return rc;
      const size_t grb_bytes = (size_t)t.gang_items * (GW + 1) * (qcols + kPadCols + 1) * sizeof(uint2);
      rc = grow(h, &s.d_grb, &s.grb_cap, grb_bytes, "alloc gang row buffers", tst, true);
      if (rc) return rc;
      // the hand-off words carry a 4-bit strip tag (never 0): clear what an earlier launch left
      SW_CUDA(h, cudaMemsetAsync(s.d_grb, 0, grb_bytes, tst));
      t.gang_epoch = 0;
      t.gang_chain2 = 1;
      if (const char* f = getenv("SW_T_GANG_CHAIN2")) t.gang_chain2 = atoi(f) != 0;
      if (getenv("SW_DEBUG_GANG_TIMES")) {   // probe: per-strip times of gang item 0, printed below
        static unsigned long long* d_dbg = nullptr;
        if (!d_dbg) cudaMalloc(&d_dbg, 2 * 4096 * sizeof(unsigned long long));
        cudaMemsetAsync(d_dbg, 0, 2 * 4096 * sizeof(unsigned long long), tst);
        t.dbg_times = d_dbg;
      }
      SW_CUDA(h, cudaMemsetAsync(s.d_gang, 0, ints * sizeof(int32_t), tst));
      t.gang_ctr = s.d_gang;
      t.gbest = s.d_gang + 1;
      t.gdone = s.d_gang + 1 + 2 * t.gang_items;
      t.gprog = reinterpret_cast<uint32_t*>(s.d_gang + 1 + 3 * t.gang_items);
      int32_t* d_base = s.d_gang + ints;   // gang_items + 1 slot offsets (CTAs of gang i: base[i] .. base[i+1])
      SW_CUDA(h, cudaMemcpyAsync(d_base, h_gang_base.data(), h_gang_base.size() * sizeof(int32_t),
                                 cudaMemcpyHostToDevice, tst));
      t.gang_base = d_base;
      t.grb = s.d_grb;
    }
    t.rb = s.d_rb_t;
    t.rb_cols = qcols + kPadCols + 1;
    t.hi_mul = 1u << 24;
    t.packed = t_packed;
    if (t.gang_items > 0) SW_CUDA(h, cudaStreamWaitEvent(tst, h->gang_ev, 0));
    SW_CUDA(h, cudaEventRecord(ev[3], tst));
    if (!scan_cols.empty()) {
      // the row-scan clusters go first on the T-mode stream and the T-mode kernel follows as a
      // programmatic dependent launch (the scan kernel triggers once its clusters are resident):
      // launched on another stream, the T-mode kernel's persistent CTAs could take every SM
      // first and leave no GPC free for a 16-CTA cluster until they finish (measured: the two
      // kernels serialised).  The T-mode queue starts after the scanned pairs (t.q0).
      // one launch per cluster size (sizes are non-increasing along the longest-first items),
      // each behind the previous one as a programmatic dependent launch
      int smax = 0;
      for (size_t i = 0; i < scan_cols.size(); ++i) smax = std::max(smax, scan_smem_bytes(a_used, scan_cols[i], qcols));
      bool pdl = false;
      for (size_t i0 = 0; i0 < scan_cols.size();) {
        size_t i1 = i0;
        while (i1 < scan_cols.size() && scan_ctas[i1] == scan_ctas[i0]) ++i1;
        const int K = scan_ctas[i0];
        if (s.scan_smem != smax || (s.scan_ctas_ok & (1u << K)) == 0) {
          int maxc = 0;
          cudaError_t e = configure_scan_kernel(smax, K, &maxc);
          if (e != cudaSuccess) return cuda_fail(h, e, "configure row-scan kernel");
          if (maxc < 1) return fail(h, SW_E_UNSUPPORTED, "row-scan cluster cannot be placed");
          if (s.scan_smem != smax) s.scan_ctas_ok = 0;
          s.scan_smem = smax;
          s.scan_ctas_ok |= 1u << K;
        }
        SW_CUDA(h, launch_scan_pairs(t, (int)i0, (int)(i1 - i0), K, smax, tst, pdl));
        pdl = true;
        i0 = i1;
      }
    }
    SW_CUDA(h, launch_tmode(t, t_grid, t_smem, tst, false, !scan_cols.empty()));
    SW_CUDA(h, cudaEventRecord(ev[4], tst));
    if (t.gang_items > 0) SW_CUDA(h, cudaEventRecord(h->gang_ev, tst));
    if (t.dbg_times) {   // probe output: strip P start / end relative to strip 0's start (us)
      std::vector<unsigned long long> tv(2 * 4096);
      cudaStreamSynchronize(tst);
      cudaMemcpy(tv.data(), t.dbg_times, tv.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
      const int S = (h->db->h_pair_ncols[0] + 32 * kTmodeC - 1) / (32 * kTmodeC);
      fprintf(stderr, "gang item 0: %d strips, GW=%d, qsteps=%d\n", S, t.gang_ctas * t.gang_warps,
              (int)round_up(qcols + 32, 4));
      for (int P = 0; P < std::min(S, 4096); ++P)
        fprintf(stderr, "strip %d start %.2f end %.2f us\n", P, (tv[2 * P] - tv[0]) / 1e3, (tv[2 * P + 1] - tv[0]) / 1e3);
    }
    if (longq) {
      SW_CUDA(h, cudaEventRecord(ev[1], st));
      // exact 32-bit recompute of the flagged sequences: T-mode's LaneS32 instantiation (one
      // sequence per strip table; items from the overflow list, exits at once when it is empty)
      TParams r = t;
      r.rho = h->rho32;
      r.sigma = h->sigma32;
      r.delta = h->rho32 - h->c_prof;
      r.item_list = s.d_ovf_list;
      r.item_count = s.d_ovf_count;
      r.work = s.d_work + 2;
      r.gang_items = 0;
      r.q0 = 0;
      r.big_strips = 1 << 30;
      r.team_warps = std::min(2, t.warps);
      while (t.warps % r.team_warps) --r.team_warps;
      const int smem32 = wp_bytes + t.warps * per_warp / 2;
      int bps = 0;
      cudaError_t e = configure_tmode_kernel(smem32, &bps, h->wide, true, r.packed);
      if (e != cudaSuccess) return cuda_fail(h, e, "configure long-sequence recompute kernel");
      SW_CUDA(h, launch_tmode(r, std::min(t_grid, std::max(1, bps) * h->num_sms), smem32, st, true));
      SW_CUDA(h, cudaEventRecord(ev[2], st));
      SW_CUDA(h, cudaMemcpyAsync(h_ovf, s.d_ovf_count, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
      h->stat_long += n_long_seqs;
      h->stat_short += h->db->n_seqs - n_long_seqs;
      h->stat_launches += 6;
      return SW_OK;
    }
    SW_CUDA(h, cudaEventRecord(s.join, s.aux));
  } else if (longq) {   // no sequences: nothing to search
    SW_CUDA(h, cudaEventRecord(ev[1], st));
    SW_CUDA(h, cudaEventRecord(ev[2], st));
    SW_CUDA(h, cudaMemcpyAsync(h_ovf, s.d_ovf_count, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    return SW_OK;
  }
  SW_CUDA(h, launch_search(pl.cfg, p, pl.grid, pl.prof_bytes, st));
  if (use_t) SW_CUDA(h, cudaStreamWaitEvent(st, s.join, 0));
  SW_CUDA(h, cudaEventRecord(ev[1], st));

  // exact 32-bit recompute of sequences whose 16-bit best reached 32767 - max_w
  SearchParams r = p;
  r.prof = s.d_prof + r_off;
  r.prof_bytes = pl.r_prof_bytes;
  r.lg = pl.rl;
  r.lt = pl.rl;
  r.rho = h->rho32;
  r.sigma = h->sigma32;
  r.delta = h->rho32 - h->c_prof;
  r.item_list = s.d_ovf_list;
  r.item_count = s.d_ovf_count;
  r.work = s.d_work + 2;
  r.long_passes = pl.r_passes;
  r.team_warps = pl.r_team_warps;
  SW_CUDA(h, launch_search(pl.rcfg, r, pl.rgrid, pl.r_prof_bytes, st));
  SW_CUDA(h, cudaEventRecord(ev[2], st));
  SW_CUDA(h, cudaMemcpyAsync(h_ovf, s.d_ovf_count, sizeof(int32_t), cudaMemcpyDeviceToHost, st));

  h->stat_long += n_long_seqs;
  h->stat_short += h->db->n_seqs - n_long_seqs;
  h->stat_launches += 4 + (pl.lt.off != pl.lg.off ? 1 : 0) + (use_t ? 2 : 0);
  return SW_OK;
}

int validate_db(sw_handle h, const uint8_t* residues, int64_t total_residues, const int64_t* offsets,
                int64_t num_seqs) {
  if (num_seqs < 0 || total_residues < 0) return fail(h, SW_E_INVALID, "negative size");
  if (num_seqs > (int64_t)0x7ffffffe) return fail(h, SW_E_INVALID, "num_seqs too large");
  if (!offsets) return fail(h, SW_E_INVALID, "offsets is NULL");
  if (total_residues > 0 && !residues) return fail(h, SW_E_INVALID, "residues is NULL");
  if (offsets[0] != 0 || offsets[num_seqs] != total_residues)
    return fail(h, SW_E_INVALID, "offsets[0] must be 0 and offsets[num_seqs] == total_residues");
  for (int64_t k = 0; k < num_seqs; ++k) {
    const int64_t len = offsets[k + 1] - offsets[k];
    if (len < 0) return fail(h, SW_E_INVALID, "offsets not non-decreasing at " + std::to_string(k));
    if (len > SW_MAX_SEQ_LEN) return fail(h, SW_E_INVALID, "sequence longer than SW_MAX_SEQ_LEN at " + std::to_string(k));
  }
  uint8_t mx = 0;
  for (int64_t t = 0; t < total_residues; ++t) mx = std::max(mx, residues[t]);
  if (mx >= h->A)
    for (int64_t t = 0; t < total_residues; ++t)
      if (residues[t] >= h->A) return fail(h, SW_E_INVALID, "residue code >= alphabet_size at " + std::to_string(t));
  return SW_OK;
}

// Host preprocessing of a (validated) CSR database into db (§II-C "The database is
// sorted by length"): stable sort by length descending, pairing, interleaved u16 columns with
// kPadCols pad columns per pair, upload.  st == nullptr: blocking upload; otherwise the columns
// are packed into db's pinned staging buffer and copied asynchronously on st (the device
// buffers are reused when large enough — the caller guarantees they are no longer read).
int build_db(sw_handle h, DbState& db, const uint8_t* residues, const int64_t* offsets, int64_t num_seqs,
             cudaStream_t st) {
  db.loaded = false;
  std::vector<int64_t> len((size_t)num_seqs);
  for (int64_t k = 0; k < num_seqs; ++k) len[k] = offsets[k + 1] - offsets[k];
  // stable sort by length descending as a counting sort (lengths <= SW_MAX_SEQ_LEN): linear,
  // and it sits on the unhidden first chunk of sw_search_stream
  std::vector<int32_t> perm((size_t)num_seqs);
  {
    int64_t lmax = 0;
    for (int64_t k = 0; k < num_seqs; ++k) lmax = std::max(lmax, len[k]);
    std::vector<int64_t> start((size_t)lmax + 2, 0);   // start[l] = #sequences longer than l
    for (int64_t k = 0; k < num_seqs; ++k) ++start[(size_t)len[k]];
    int64_t acc = 0;
    for (int64_t l = lmax; l >= 0; --l) {
      const int64_t c = start[(size_t)l];
      start[(size_t)l] = acc;
      acc += c;
    }
    for (int64_t k = 0; k < num_seqs; ++k) perm[(size_t)start[(size_t)len[k]]++] = (int32_t)k;
  }
  db.sorted_len.resize((size_t)num_seqs);
  for (int64_t k = 0; k < num_seqs; ++k) db.sorted_len[k] = len[perm[k]];
  const int n_pairs = (int)((num_seqs + 1) / 2);
  db.h_pair_off.assign((size_t)n_pairs + 1, kLeadCols);
  db.h_pair_ncols.assign((size_t)n_pairs, 0);
  for (int p = 0; p < n_pairs; ++p) {
    const int64_t lo = db.sorted_len[2 * p];
    const int64_t hi = (2 * p + 1 < num_seqs) ? db.sorted_len[2 * p + 1] : 0;
    const int64_t nc = round_up(std::max<int64_t>({lo, hi, (int64_t)kMinCols}), kColAlign);
    db.h_pair_ncols[p] = (int32_t)nc;
    db.h_pair_off[p + 1] = db.h_pair_off[p] + nc + kPadCols;
  }
  const int64_t total_cols = db.h_pair_off[n_pairs];
  db.inv_perm.assign((size_t)num_seqs, 0);
  for (int64_t k = 0; k < num_seqs; ++k) db.inv_perm[perm[k]] = (int32_t)k;
  db.pair_cols_prefix.assign((size_t)n_pairs + 1, 0);
  for (int p = 0; p < n_pairs; ++p) db.pair_cols_prefix[p + 1] = db.pair_cols_prefix[p] + db.h_pair_ncols[p];
  db.n_seqs = num_seqs;
  db.n_pairs = n_pairs;
  const size_t cols_bytes = (size_t)std::max<int64_t>(total_cols, 1) * sizeof(uint16_t);
  std::vector<uint16_t> cols_vec;
  uint16_t* cols = nullptr;
  if (st) {
    if (db.stage_cap < cols_bytes) {
      if (db.h_stage) cudaFreeHost(db.h_stage);
      db.h_stage = nullptr;
      db.stage_cap = 0;
      cudaError_t e = cudaMallocHost(&db.h_stage, cols_bytes);
      if (e != cudaSuccess) return cuda_fail(h, e, "alloc pinned staging");
      db.stage_cap = cols_bytes;
    }
    cols = static_cast<uint16_t*>(db.h_stage);
  } else {
    cols_vec.resize(cols_bytes / sizeof(uint16_t));
    cols = cols_vec.data();
  }
  const uint16_t pad = (uint16_t)h->A;
  for (int j = 0; j < kLeadCols; ++j) cols[j] = (uint16_t)(pad | (pad << 8));
  auto pack = [&](int p0, int p1) {
    for (int p = p0; p < p1; ++p) {
      uint16_t* dst = cols + db.h_pair_off[p];
      const int64_t nc = db.h_pair_ncols[p];
      const int64_t s0 = perm[2 * p];
      const int64_t l0 = len[s0];
      const uint8_t* r0 = residues ? residues + offsets[s0] : nullptr;
      const bool has1 = 2 * p + 1 < num_seqs;
      const int64_t s1 = has1 ? perm[2 * p + 1] : 0;
      const int64_t l1 = has1 ? len[s1] : 0;
      const uint8_t* r1 = (has1 && residues) ? residues + offsets[s1] : nullptr;
      for (int64_t j = 0; j < nc + kPadCols; ++j) {
        const uint16_t a = j < l0 ? r0[j] : pad;
        const uint16_t b = j < l1 ? r1[j] : pad;
        dst[j] = (uint16_t)(a | (b << 8));
      }
    }
  };
  // packing is host memory bound: split the pairs over a few threads for large databases
  const int nthreads = n_pairs < (1 << 15) ? 1 : (int)std::min<unsigned>(16u, std::max(1u, std::thread::hardware_concurrency()));
  if (nthreads == 1) {
    pack(0, n_pairs);
  } else {
    std::vector<std::thread> pool;
    for (int t = 0; t < nthreads; ++t)
      pool.emplace_back(pack, (int)((int64_t)n_pairs * t / nthreads), (int)((int64_t)n_pairs * (t + 1) / nthreads));
    for (auto& t : pool) t.join();
  }
  if (num_seqs == 0) { db.loaded = true; return SW_OK; }
  int rc = grow(h, &db.d_cols, &db.cols_cap, cols_bytes, "alloc database");
  if (!rc) rc = grow(h, &db.d_pair_off, &db.pair_off_cap, (size_t)n_pairs * sizeof(int64_t), "alloc pair offsets");
  if (!rc) rc = grow(h, &db.d_pair_ncols, &db.pair_ncols_cap, (size_t)n_pairs * sizeof(int32_t), "alloc pair columns");
  if (!rc) rc = grow(h, &db.d_perm, &db.perm_cap, (size_t)num_seqs * sizeof(int32_t), "alloc permutation");
  if (rc) return rc;
  if (st) {
    SW_CUDA(h, cudaMemcpyAsync(db.d_cols, cols, cols_bytes, cudaMemcpyHostToDevice, st));
    // the small index arrays are pageable: their copies complete before returning
    SW_CUDA(h, cudaMemcpyAsync(db.d_pair_off, db.h_pair_off.data(), (size_t)n_pairs * sizeof(int64_t),
                               cudaMemcpyHostToDevice, st));
    SW_CUDA(h, cudaMemcpyAsync(db.d_pair_ncols, db.h_pair_ncols.data(), (size_t)n_pairs * sizeof(int32_t),
                               cudaMemcpyHostToDevice, st));
    SW_CUDA(h, cudaMemcpyAsync(db.d_perm, perm.data(), (size_t)num_seqs * sizeof(int32_t), cudaMemcpyHostToDevice, st));
    SW_CUDA(h, cudaStreamSynchronize(st));   // perm (a local) must outlive its copy
  } else {
    SW_CUDA(h, cudaMemcpy(db.d_cols, cols, cols_bytes, cudaMemcpyHostToDevice));
    SW_CUDA(h, cudaMemcpy(db.d_pair_off, db.h_pair_off.data(), (size_t)n_pairs * sizeof(int64_t), cudaMemcpyHostToDevice));
    SW_CUDA(h, cudaMemcpy(db.d_pair_ncols, db.h_pair_ncols.data(), (size_t)n_pairs * sizeof(int32_t), cudaMemcpyHostToDevice));
    SW_CUDA(h, cudaMemcpy(db.d_perm, perm.data(), (size_t)num_seqs * sizeof(int32_t), cudaMemcpyHostToDevice));
  }
  db.loaded = true;
  return SW_OK;
}

// Autotune (run_batch): the planner's time model ranks the compiled configurations, but its
// error is up to ~10 % in team mode (profiles/r01_menu_c3.txt) and a few % in group mode
// (profiles/r01_plan_check*.jsonl).  The first batch that searches a (query length, threshold)
// on the loaded database with >= kTuneMinCells cells therefore times the model's kTuneTop best
// candidates, one search each (every configuration computes the same exact scores, so the
// candidates write the real output), and keeps the fastest for later searches.  SW_AUTOTUNE=0
// disables it (model choice only); the tuned table is cleared by sw_load_db.
constexpr double kTuneMinCells = 1e10;
constexpr double kTuneTMinCells = 1e9;   // threshold tuning (3 searches of ~0.2 ms and up)
constexpr int kTuneTop = 5;

int autotune(sw_handle h, const uint8_t* d_queries, const int64_t* qoff, int nq, int32_t* d_out, int32_t T,
             cudaStream_t user) {
  if (h->db != &h->main_db || getenv("SW_FORCE_MENU")) return SW_OK;
  if (const char* f = getenv("SW_AUTOTUNE"))
    if (!strcmp(f, "0")) return SW_OK;
  bool forked = false;
  const double residues = std::accumulate(h->db->sorted_len.begin(), h->db->sorted_len.end(), 0.0);
  auto fork = [&]() -> int {
    if (!forked) {   // the queries were uploaded on the caller's stream
      SW_CUDA(h, cudaEventRecord(h->fork, user));
      SW_CUDA(h, cudaStreamWaitEvent(h->slots[0].stream, h->fork, 0));
      forked = true;
    }
    return SW_OK;
  };
  // one timed search of query k at threshold Tk with the plan enqueue_query makes (device ms
  // of the search launches, profile build to join, on the first slot)
  auto time_search = [&](int k, int32_t Tk, float* ms) -> int {
    const int m = (int)(qoff[k + 1] - qoff[k]);
    cudaEvent_t* ev = h->ev.data() + kEvPerQuery * k;
    int rc = enqueue_query(h, h->slots[0], d_queries + qoff[k], m, h->qmask[k], d_out + (int64_t)k * h->db->n_seqs,
                           Tk, h->h_ovf + k, ev);
    if (rc) return rc;
    SW_CUDA(h, cudaEventSynchronize(ev[1]));
    SW_CUDA(h, cudaEventElapsedTime(ms, ev[0], ev[1]));
    return SW_OK;
  };
  for (int k = 0; k < nq; ++k) {
    const int m = (int)(qoff[k + 1] - qoff[k]);
    if (long_query_mode(h, m)) continue;
    // Automatic threshold: the model's estimate misses the occupancy of group
    // launches with few items and the long path's tail, by up to 4x on long-sequence databases
    // (C3 query 144).  The first search of a query length with
    // SW_AUTO_THRESHOLD on a loaded database of >= kTuneTMinCells cells times the model's four
    // best thresholds and the endpoints (all short: T > max length; all long: T = min length,
    // for long-sequence databases) and keeps the fastest.
    if (T == SW_AUTO_THRESHOLD && (double)m * residues >= kTuneTMinCells && !h->tuned_T.count(m)) {
      const auto ranked = rank_thresholds(h, m);
      std::vector<int64_t> cand;
      for (const auto& c : ranked) {   // (the model's ranking is off by up to ~10 % between
        if ((int)cand.size() >= 4) break;   // neighbouring candidates: profiles/r02_variance_sweep)
        cand.push_back(c.second);
      }
      const int64_t all_short = h->db->sorted_len.empty() ? 0 : h->db->sorted_len[0] + 1;
      if (std::find(cand.begin(), cand.end(), all_short) == cand.end()) cand.push_back(all_short);
      // the all-long endpoint only for databases of long sequences (C3-like: every sequence
      // >= 512), where it is a real contender; on Swiss-Prot-like ones it is hopeless
      const int64_t min_len = h->db->sorted_len.empty() ? 0 : h->db->sorted_len.back();
      if (min_len >= 512 && std::find(cand.begin(), cand.end(), min_len) == cand.end()) cand.push_back(min_len);
      int rc = fork();
      if (rc) return rc;
      float best_ms = 1e30f;
      int64_t best_T = cand.front();
      for (int64_t Tc : cand) {
        float ms = 0.f;
        rc = time_search(k, (int32_t)std::min<int64_t>(Tc, INT32_MAX), &ms);
        if (rc) return rc;
        if (getenv("SW_DEBUG_PLAN")) fprintf(stderr, "tune-T m=%d T=%lld %.3f ms\n", m, (long long)Tc, ms);
        if (ms < best_ms) { best_ms = ms; best_T = Tc; }
      }
      h->tuned_T[m] = best_T;
    }
    if ((double)m * residues < kTuneMinCells) continue;
    int32_t Tk = T;
    if (Tk == SW_AUTO_THRESHOLD) Tk = (int32_t)std::min<int64_t>(choose_threshold(h, m), INT32_MAX);
    const std::pair<int, int32_t> key{m, Tk};
    if (h->tuned.count(key)) continue;
    // the candidates of the launch enqueue_query plans (short pairs only when T-mode takes
    // the long ones)
    Split sp = make_split(h, Tk, nullptr);
    if (sp.n_long > 0 && m < kTmodeMaxQuery) { sp.n_long = 0; sp.long_cols = 0; sp.long_max_cols = 0; }
    if (sp.n_long == 0 && sp.n_short == 0) { h->tuned[key] = -1; continue; }
    std::vector<std::pair<double, int>> ranked;
    Plan pl;
    int rc = make_plan(h, m, sp, &pl, -1, &ranked);
    if (rc) return rc;
    std::sort(ranked.begin(), ranked.end());
    if (ranked.size() > (size_t)kTuneTop) ranked.resize(kTuneTop);
    rc = fork();
    if (rc) return rc;
    // one timed search per candidate, then the two fastest again (min of two): a single
    // disturbed timing once kept a 4 % slower entry for a whole session (query 2504 on C2)
    std::vector<std::pair<float, int>> timed;
    for (const auto& c : ranked) {
      h->tune_force = c.second;
      float ms = 0.f;
      rc = time_search(k, Tk, &ms);
      h->tune_force = -1;
      if (rc) return rc;
      if (getenv("SW_DEBUG_PLAN")) fprintf(stderr, "tune m=%d T=%d menu=%d %.3f ms\n", m, (int)Tk, c.second, ms);
      timed.push_back({ms, c.second});
    }
    std::sort(timed.begin(), timed.end());
    for (size_t j = 0; j < std::min<size_t>(2, timed.size()); ++j) {
      h->tune_force = timed[j].second;
      float ms = 0.f;
      rc = time_search(k, Tk, &ms);
      h->tune_force = -1;
      if (rc) return rc;
      if (getenv("SW_DEBUG_PLAN")) fprintf(stderr, "tune m=%d T=%d menu=%d %.3f ms (again)\n", m, (int)Tk, timed[j].second, ms);
      timed[j].first = std::min(timed[j].first, ms);
    }
    std::sort(timed.begin(), timed.end());
    h->tuned[key] = timed.empty() ? -1 : timed[0].second;
  }
  if (forked) SW_CUDA(h, cudaStreamSynchronize(h->slots[0].stream));
  h->stat_long = h->stat_short = h->stat_launches = 0;
  return SW_OK;
}

int run_batch(sw_handle h, const uint8_t* h_queries, const uint8_t* d_queries, const int64_t* qoff, int nq,
              int32_t* d_out, int32_t T, cudaStream_t user) {
  h->stat_long = h->stat_short = h->stat_launches = 0;
  h->stat_recomputed = -1;
  h->stat_nq = nq;
  if (h->db->n_seqs == 0 || nq == 0) return SW_OK;
  // queries run concurrently on up to SW_STREAMS internal streams (default 4) so that the
  // tail of one query's persistent launch overlaps the next query
  int max_streams = 4;
  if (const char* f = getenv("SW_STREAMS")) max_streams = std::max(1, std::min(16, atoi(f)));
  int rc = ensure_slots(h, std::min(nq, max_streams));
  if (rc) return rc;
  if (h->h_ovf_cap < nq) {
    if (h->h_ovf) { cudaDeviceSynchronize(); cudaFreeHost(h->h_ovf); }
    h->h_ovf = nullptr;
    h->h_ovf_cap = 0;
    SW_CUDA(h, cudaMallocHost(&h->h_ovf, (size_t)nq * sizeof(int32_t)));
    h->h_ovf_cap = nq;
  }
  memset(h->h_ovf, 0, (size_t)nq * sizeof(int32_t));
  h->long_fused.assign((size_t)nq, 0);
  while ((int)h->ev.size() < kEvPerQuery * nq) {
    cudaEvent_t e;
    SW_CUDA(h, cudaEventCreate(&e));
    h->ev.push_back(e);
  }
  // letters present in each query (T-mode builds its strip tables for these only)
  h->qmask.assign(nq, 0u);
  for (int k = 0; k < nq; ++k)
    for (int64_t i = qoff[k]; i < qoff[k + 1]; ++i) h->qmask[k] |= 1u << h_queries[i];
  rc = autotune(h, d_queries, qoff, nq, d_out, T, user);
  if (rc) return rc;
  const int ns = std::min(nq, max_streams);
  SW_CUDA(h, cudaEventRecord(h->fork, user));
  for (int k = 0; k < ns; ++k) SW_CUDA(h, cudaStreamWaitEvent(h->slots[k].stream, h->fork, 0));
  for (int k = 0; k < nq; ++k) {
    QuerySlot& s = h->slots[k % ns];
    rc = enqueue_query(h, s, d_queries + qoff[k], (int)(qoff[k + 1] - qoff[k]), h->qmask[k],
                       d_out + (int64_t)k * h->db->n_seqs, T,
                       h->h_ovf + k, h->ev.data() + kEvPerQuery * k);
    if (rc) return rc;
  }
  for (int k = 0; k < ns; ++k) {
    SW_CUDA(h, cudaEventRecord(h->slots[k].done, h->slots[k].stream));
    SW_CUDA(h, cudaStreamWaitEvent(user, h->slots[k].done, 0));
  }
  return SW_OK;
}

}  // namespace

// ============================================================================ C ABI
extern "C" {

const char* sw_strerror(int status) {
  switch (status) {
    case SW_OK: return "ok";
    case SW_E_INVALID: return "invalid argument";
    case SW_E_STATE: return "call out of order";
    case SW_E_NOMEM: return "out of memory";
    case SW_E_CUDA: return "CUDA error";
    case SW_E_UNSUPPORTED: return "unsupported device or parameters";
    default: return "unknown status";
  }
}

const char* sw_last_error(sw_handle h) { return h ? h->err.c_str() : ""; }

const char* sw_version(void) { return "sw_b200 1.0 sm_100a"; }

int sw_create(sw_handle* out, const uint8_t* query, int32_t query_len, const int8_t* matrix, int32_t alphabet_size,
              int32_t gap_open, int32_t gap_extend) {
  if (!out) return SW_E_INVALID;
  *out = nullptr;
  if (!matrix || alphabet_size < 1 || alphabet_size > SW_MAX_ALPHABET) return SW_E_INVALID;
  if (gap_open < 0 || gap_extend < 0) return SW_E_INVALID;
  sw_handle h = new (std::nothrow) sw_handle_s();
  if (!h) return SW_E_NOMEM;
  h->A = alphabet_size;
  h->rho = gap_open;
  h->sigma = gap_extend;
  h->max_w = -128;
  h->min_w = 127;
  for (int i = 0; i < alphabet_size * alphabet_size; ++i) {
    h->max_w = std::max<int>(h->max_w, matrix[i]);
    h->min_w = std::min<int>(h->min_w, matrix[i]);
  }
  int rc = validate_query(h, query, query_len);
  if (rc) { delete h; return rc; }
  h->c_prof = std::min(gap_open, 127 - h->max_w);
  h->wide = gap_open > h->c_prof;
  const bool clamp16 = gap_open > 16384 || gap_extend > 16384;
  h->rho16 = std::min(gap_open, 16384);
  h->sigma16 = std::min(gap_extend, 16384);
  h->flag_limit = clamp16 ? std::min(32767 - h->max_w, 16384) : 32767 - h->max_w;
  h->rho32 = std::min(gap_open, 1 << 29);
  h->sigma32 = std::min(gap_extend, 1 << 29);
  cudaError_t e = cudaGetDevice(&h->device);
  cudaDeviceProp prop;
  if (e == cudaSuccess) e = cudaGetDeviceProperties(&prop, h->device);
  if (e != cudaSuccess) { delete h; return SW_E_UNSUPPORTED; }
  if (!(prop.major == 10 && prop.minor == 0)) { delete h; return SW_E_UNSUPPORTED; }
  h->num_sms = prop.multiProcessorCount;
  if (cudaMalloc(&h->d_matrix, (size_t)alphabet_size * alphabet_size) != cudaSuccess ||
      cudaMemcpy(h->d_matrix, matrix, (size_t)alphabet_size * alphabet_size, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaEventCreateWithFlags(&h->fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&h->gang_ev, cudaEventDisableTiming) != cudaSuccess ||
      cudaStreamCreateWithFlags(&h->copy_st, cudaStreamNonBlocking) != cudaSuccess) {
    sw_destroy(h);
    return SW_E_CUDA;
  }
  h->query.assign(query, query + query_len);
  *out = h;
  return SW_OK;
}

int sw_set_query(sw_handle h, const uint8_t* query, int32_t query_len) {
  if (!h) return SW_E_INVALID;
  int rc = validate_query(h, query, query_len);
  if (rc) return rc;
  h->query.assign(query, query + query_len);
  return SW_OK;
}

int sw_load_db(sw_handle h, const uint8_t* residues, int64_t total_residues, const int64_t* offsets,
               int64_t num_seqs) {
  if (!h) return SW_E_INVALID;
  int rc = validate_db(h, residues, total_residues, offsets, num_seqs);
  if (rc) return rc;
  h->db = &h->main_db;
  h->main_db.release();
  h->tuned.clear();
  h->tuned_T.clear();
  return build_db(h, h->main_db, residues, offsets, num_seqs, nullptr);
}

int sw_search_stream(sw_handle h, const uint8_t* queries, const int64_t* q_offsets, int32_t num_queries,
                     const uint8_t* residues, int64_t total_residues, const int64_t* offsets, int64_t num_seqs,
                     int32_t* scores_out, int32_t length_threshold, int64_t chunk_residues) {
  if (!h) return SW_E_INVALID;
  int64_t own_qo[2] = {0, (int64_t)h->query.size()};
  if (!queries) {                       // the handle's own query
    queries = h->query.data();
    q_offsets = own_qo;
    num_queries = 1;
  }
  if (num_queries < 0 || !q_offsets) return fail(h, SW_E_INVALID, "bad query batch");
  if (q_offsets[0] != 0) return fail(h, SW_E_INVALID, "q_offsets[0] != 0");
  for (int k = 0; k < num_queries; ++k) {
    const int64_t m = q_offsets[k + 1] - q_offsets[k];
    if (m <= 0 || m > SW_MAX_QUERY_LEN) return fail(h, SW_E_INVALID, "query length out of range in batch");
    int rc = validate_query(h, queries + q_offsets[k], (int32_t)m);
    if (rc) return rc;
  }
  if (num_seqs > 0 && num_queries > 0 && !scores_out) return fail(h, SW_E_INVALID, "scores_out is NULL");
  if (chunk_residues <= 0) return fail(h, SW_E_INVALID, "chunk_residues <= 0");
  if (length_threshold < 0 && length_threshold != SW_AUTO_THRESHOLD)
    return fail(h, SW_E_INVALID, "length_threshold < 0 (use SW_AUTO_THRESHOLD for automatic)");
  int rc = validate_db(h, residues, total_residues, offsets, num_seqs);
  if (rc) return rc;
  h->stat_long = h->stat_short = h->stat_launches = 0;
  h->stat_recomputed = 0;
  if (num_seqs == 0 || num_queries == 0) return SW_OK;
  rc = ensure_slots(h, 1);
  if (rc) return rc;
  cudaStream_t st = h->slots[0].stream;
  rc = wait_slots(h, st);   // earlier calls' slot streams may still read d_batch_q
  if (rc) return rc;
  const int nq = num_queries;
  const int64_t qtot = q_offsets[nq];
  size_t qcap = (size_t)h->batch_q_cap;
  rc = grow(h, &h->d_batch_q, &qcap, (size_t)qtot, "alloc stream queries", st);
  if (rc) return rc;
  h->batch_q_cap = (int64_t)qcap;
  std::vector<int64_t> qo(q_offsets, q_offsets + nq + 1);
  SW_CUDA(h, cudaMemcpyAsync(h->d_batch_q, queries, (size_t)qtot, cudaMemcpyHostToDevice, st));
  SW_CUDA(h, cudaStreamSynchronize(st));     // the caller's query buffer is pageable
  // chunk boundaries: whole sequences, about chunk_residues residues each; the first three
  // chunks ramp up (1/8, 1/4, 1/2) because nothing hides the host packing of the first one
  // (packing runs ~3x faster than the search of the same residues, so doubling stays hidden;
  // every chunk adds a launch tail, so a longer ramp measured slower:
  // profiles/r01_stream_chunk_sweep*.jsonl)
  int kRamp = 3;
  if (const char* f = getenv("SW_STREAM_RAMP")) kRamp = std::max(0, std::min(10, atoi(f)));   // probes
  std::vector<int64_t> cut{0};
  while (cut.back() < num_seqs) {
    const int64_t s0 = cut.back();
    const int ramp = std::max(0, kRamp - (int)(cut.size() - 1));
    const int64_t target = std::max<int64_t>(chunk_residues >> ramp, 1);
    int64_t e = std::upper_bound(offsets + s0, offsets + num_seqs + 1, offsets[s0] + target) - offsets - 1;
    cut.push_back(std::min(std::max(e, s0 + 1), num_seqs));
  }
  const int nchunks = (int)cut.size() - 1;
  for (auto& ss : h->stream_slot) {
    if (!ss.up && cudaStreamCreateWithFlags(&ss.up, cudaStreamNonBlocking) != cudaSuccess)
      return fail(h, SW_E_CUDA, "stream setup");
    if (!ss.uploaded && cudaEventCreateWithFlags(&ss.uploaded, cudaEventDisableTiming) != cudaSuccess)
      return fail(h, SW_E_CUDA, "stream setup");
    if (!ss.searched && cudaEventCreateWithFlags(&ss.searched, cudaEventDisableTiming) != cudaSuccess)
      return fail(h, SW_E_CUDA, "stream setup");
    ss.pending = false;
  }
  int64_t stat_long = 0, stat_short = 0, stat_launches = 0, stat_rec = 0;
  // wait for slot k's search; hand its scores over
  auto finish = [&](StreamSlot& ss) -> int {
    if (!ss.pending) return SW_OK;
    ss.pending = false;
    cudaError_t e = cudaEventSynchronize(ss.searched);
    if (e != cudaSuccess) return cuda_fail(h, e, "streamed chunk search");
    for (int q = 0; q < nq; ++q) {
      memcpy(scores_out + (int64_t)q * num_seqs + ss.s0, ss.h_sc + (int64_t)q * ss.n, (size_t)ss.n * sizeof(int32_t));
      stat_rec += ss.h_ovf[q];
    }
    return SW_OK;
  };
  // run_batch keeps its overflow counts in h->h_ovf: point it at the chunk slot's array
  int32_t* const saved_ovf = h->h_ovf;
  const int saved_ovf_cap = h->h_ovf_cap;
  for (int c = 0; c < nchunks && rc == SW_OK; ++c) {
    StreamSlot& ss = h->stream_slot[c & 1];
    rc = finish(ss);                     // slot's previous chunk must be done before reuse
    if (rc) break;
    const int64_t s0 = cut[c], s1 = cut[c + 1], n = s1 - s0;
    std::vector<int64_t> off((size_t)n + 1);
    for (int64_t i = 0; i <= n; ++i) off[i] = offsets[s0 + i] - offsets[s0];
    // host packing + upload of chunk c overlap the device search of chunk c - 1
    // ("copy a slice of the database to the GPU, start aligning, and copy the rest of the
    // database in the background", §VI)
    const auto tb0 = std::chrono::steady_clock::now();
    rc = build_db(h, ss.db, residues + offsets[s0], off.data(), n, ss.up);
    if (getenv("SW_DEBUG_STREAM"))
      fprintf(stderr, "stream chunk %d: %lld seqs, %lld residues, host build+upload %.2f ms\n", c, (long long)n,
              (long long)(offsets[s1] - offsets[s0]),
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tb0).count());
    if (rc) break;
    const size_t need = (size_t)nq * (size_t)n * sizeof(int32_t);
    if (ss.d_sc_cap < need) {
      cudaFree(ss.d_sc);
      ss.d_sc = nullptr; ss.d_sc_cap = 0;
      if (cudaMalloc(&ss.d_sc, need) != cudaSuccess) { rc = fail(h, SW_E_NOMEM, "stream score buffer"); break; }
      ss.d_sc_cap = need;
    }
    if (ss.h_sc_cap < need) {
      if (ss.h_sc) cudaFreeHost(ss.h_sc);
      ss.h_sc = nullptr; ss.h_sc_cap = 0;
      if (cudaMallocHost(&ss.h_sc, need) != cudaSuccess) { rc = fail(h, SW_E_NOMEM, "stream score buffer"); break; }
      ss.h_sc_cap = need;
    }
    if (ss.ovf_cap < nq) {
      if (ss.h_ovf) cudaFreeHost(ss.h_ovf);
      ss.h_ovf = nullptr; ss.ovf_cap = 0;
      if (cudaMallocHost(&ss.h_ovf, (size_t)nq * sizeof(int32_t)) != cudaSuccess) {
        rc = fail(h, SW_E_NOMEM, "stream overflow counts");
        break;
      }
      ss.ovf_cap = nq;
    }
    if (cudaEventRecord(ss.uploaded, ss.up) != cudaSuccess || cudaStreamWaitEvent(st, ss.uploaded, 0) != cudaSuccess) {
      rc = fail(h, SW_E_CUDA, "stream event");
      break;
    }
    h->db = &ss.db;
    h->h_ovf = ss.h_ovf;
    h->h_ovf_cap = ss.ovf_cap;
    rc = run_batch(h, queries, h->d_batch_q, qo.data(), nq, ss.d_sc, length_threshold, st);
    h->db = &h->main_db;
    if (rc) break;
    stat_long += h->stat_long; stat_short += h->stat_short; stat_launches += h->stat_launches;
    if (cudaMemcpyAsync(ss.h_sc, ss.d_sc, need, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaEventRecord(ss.searched, st) != cudaSuccess) {
      rc = fail(h, SW_E_CUDA, "stream score copy");
      break;
    }
    ss.s0 = s0; ss.n = n; ss.pending = true;
  }
  for (auto& ss : h->stream_slot) {
    const int r2 = finish(ss);
    if (rc == SW_OK) rc = r2;
  }
  h->db = &h->main_db;
  h->h_ovf = saved_ovf;
  h->h_ovf_cap = saved_ovf_cap;
  h->stat_long = stat_long; h->stat_short = stat_short; h->stat_launches = stat_launches;
  h->stat_recomputed = stat_rec;
  return rc;
}

int sw_search_batch_async(sw_handle h, const uint8_t* queries, const int64_t* q_offsets, int32_t num_queries,
                          int32_t* d_scores_out, int32_t length_threshold, void* cuda_stream) {
  if (!h) return SW_E_INVALID;
  if (!h->db->loaded) return fail(h, SW_E_STATE, "sw_load_db has not been called");
  if (num_queries < 0 || !q_offsets || (num_queries > 0 && !queries)) return fail(h, SW_E_INVALID, "bad query batch");
  if (length_threshold < 0 && length_threshold != SW_AUTO_THRESHOLD)
    return fail(h, SW_E_INVALID, "length_threshold < 0 (use SW_AUTO_THRESHOLD for automatic)");
  if (h->db->n_seqs > 0 && num_queries > 0 && !d_scores_out) return fail(h, SW_E_INVALID, "d_scores_out is NULL");
  if (q_offsets[0] != 0) return fail(h, SW_E_INVALID, "q_offsets[0] != 0");
  for (int k = 0; k < num_queries; ++k) {
    const int64_t m = q_offsets[k + 1] - q_offsets[k];
    if (m <= 0 || m > SW_MAX_QUERY_LEN) return fail(h, SW_E_INVALID, "query length out of range in batch");
    int rc = validate_query(h, queries + q_offsets[k], (int32_t)m);
    if (rc) return rc;
  }
  cudaStream_t st = reinterpret_cast<cudaStream_t>(cuda_stream);
  const int64_t tot = q_offsets[num_queries];
  // the previous call's slot streams may still read d_batch_q (its profile builds and query
  // streams): order the upload after them, whatever stream that call was issued on
  int rc = wait_slots(h, st);
  if (rc) return rc;
  size_t cap = (size_t)h->batch_q_cap;
  rc = grow(h, &h->d_batch_q, &cap, (size_t)std::max<int64_t>(tot, 1), "alloc batch queries", st);
  if (rc) return rc;
  h->batch_q_cap = (int64_t)cap;
  if (tot > 0) SW_CUDA(h, cudaMemcpyAsync(h->d_batch_q, queries, (size_t)tot, cudaMemcpyHostToDevice, st));
  return run_batch(h, queries, h->d_batch_q, q_offsets, num_queries, d_scores_out, length_threshold, st);
}

int sw_search_async(sw_handle h, int32_t* d_scores_out, int32_t length_threshold, void* cuda_stream) {
  if (!h) return SW_E_INVALID;
  const int64_t qo[2] = {0, (int64_t)h->query.size()};
  return sw_search_batch_async(h, h->query.data(), qo, 1, d_scores_out, length_threshold, cuda_stream);
}

int sw_search_batch(sw_handle h, const uint8_t* queries, const int64_t* q_offsets, int32_t num_queries,
                    int32_t* scores_out, int32_t length_threshold) {
  if (!h) return SW_E_INVALID;
  if (!h->db->loaded) return fail(h, SW_E_STATE, "sw_load_db has not been called");
  if (num_queries < 0) return fail(h, SW_E_INVALID, "num_queries < 0");
  const int64_t need = (int64_t)num_queries * h->db->n_seqs;
  if (need > 0 && !scores_out) return fail(h, SW_E_INVALID, "scores_out is NULL");
  size_t cap = (size_t)h->scores_tmp_cap * sizeof(int32_t);
  int rc = grow(h, &h->d_scores_tmp, &cap, (size_t)std::max<int64_t>(need, 1) * sizeof(int32_t), "alloc scores");
  if (rc) return rc;
  h->scores_tmp_cap = (int64_t)(cap / sizeof(int32_t));
  rc = sw_search_batch_async(h, queries, q_offsets, num_queries, h->d_scores_tmp, length_threshold, nullptr);
  if (rc) return rc;
  // each query's scores are final at its ev[2] (after its 32-bit recompute): copy them as the
  // queries finish, on a stream of their own, so the copies overlap the queries still running
  // (the caller's stream waits for every query; a copy there would wait for the last one)
  const int64_t ns = h->db->n_seqs;
  if (need > 0 && (int)h->ev.size() >= kEvPerQuery * num_queries) {
    std::vector<char> copied((size_t)num_queries, 0);
    for (int left = num_queries; left > 0;) {
      int progressed = 0;
      for (int k = 0; k < num_queries; ++k) {
        if (copied[(size_t)k]) continue;
        const cudaError_t q = cudaEventQuery(h->ev[(size_t)kEvPerQuery * k + 2]);
        if (q == cudaErrorNotReady) continue;
        if (q != cudaSuccess) return cuda_fail(h, q, "query completion");
        SW_CUDA(h, cudaMemcpyAsync(scores_out + (int64_t)k * ns, h->d_scores_tmp + (int64_t)k * ns,
                                   (size_t)ns * sizeof(int32_t), cudaMemcpyDeviceToHost, h->copy_st));
        copied[(size_t)k] = 1;
        --left;
        ++progressed;
      }
      if (!progressed) std::this_thread::yield();
    }
    SW_CUDA(h, cudaStreamSynchronize(h->copy_st));
  } else if (need > 0) {
    SW_CUDA(h, cudaMemcpy(scores_out, h->d_scores_tmp, (size_t)need * sizeof(int32_t), cudaMemcpyDeviceToHost));
  }
  SW_CUDA(h, cudaDeviceSynchronize());
  return SW_OK;
}

int sw_search(sw_handle h, int32_t* scores_out, int32_t length_threshold) {
  if (!h) return SW_E_INVALID;
  const int64_t qo[2] = {0, (int64_t)h->query.size()};
  return sw_search_batch(h, h->query.data(), qo, 1, scores_out, length_threshold);
}

int sw_last_stats(sw_handle h, int64_t out[4]) {
  if (!h || !out) return SW_E_INVALID;
  int64_t ovf = 0;
  // valid once the last search's stream work has completed
  for (int k = 0; k < std::min(h->stat_nq, h->h_ovf_cap); ++k) ovf += h->h_ovf[k];
  out[0] = h->stat_recomputed >= 0 ? h->stat_recomputed : ovf;
  out[1] = h->stat_long;
  out[2] = h->stat_short;
  out[3] = h->stat_launches;
  return SW_OK;
}

int32_t sw_last_threshold(sw_handle h) { return h ? h->last_threshold : -1; }

int sw_align(sw_handle h, int64_t seq_index, sw_alignment* out, uint32_t* ops, int32_t ops_cap) {
  if (!h) return SW_E_INVALID;
  if (!h->db->loaded) return fail(h, SW_E_STATE, "sw_load_db has not been called");
  if (!out || ops_cap < 0 || (ops_cap > 0 && !ops)) return fail(h, SW_E_INVALID, "bad output buffers");
  if (seq_index < 0 || seq_index >= h->db->n_seqs) return fail(h, SW_E_INVALID, "seq_index out of range");
  memset(out, 0, sizeof(*out));
  const int64_t pos = h->db->inv_perm[(size_t)seq_index];
  const int64_t n = h->db->sorted_len[(size_t)pos];
  const int m = (int)h->query.size();
  if (n == 0) { out->q_begin = out->q_end = out->d_begin = out->d_end = 0; return SW_OK; }
  int rc = grow(h, &h->d_tb_scratch, &h->tb_scratch_cap, (size_t)7 * m * sizeof(int), "alloc traceback scratch");
  if (rc) return rc;
  rc = grow(h, &h->d_tb_result, &h->tb_result_cap, 16 * sizeof(int), "alloc traceback result");
  if (rc) return rc;
  rc = grow(h, &h->d_tb_query, &h->tb_query_cap, (size_t)m, "alloc traceback query");
  if (rc) return rc;
  SW_CUDA(h, cudaMemcpy(h->d_tb_query, h->query.data(), (size_t)m, cudaMemcpyHostToDevice));
  const int64_t pair = pos >> 1;
  const int half = (int)(pos & 1);
  const uint16_t* dcols = h->db->d_cols + h->db->h_pair_off[(size_t)pair];
  // (1) score and end cell, (2) start cell — O(m) scratch (sw_traceback.cu)
  SW_CUDA(h, launch_tb_score_start(h->d_tb_query, m, dcols, half, (int)n, h->d_matrix, h->A, h->rho32, h->sigma32,
                                   h->d_tb_scratch, h->d_tb_result, nullptr));
  int se[5];
  SW_CUDA(h, cudaMemcpy(se, h->d_tb_result, sizeof(se), cudaMemcpyDeviceToHost));
  out->score = se[0];
  if (se[0] <= 0) { out->n_ops = 0; return SW_OK; }
  const int ib = se[3], jb = se[4], ie = se[1], je = se[2];
  if (ib < 0 || jb < 0 || ib > ie || jb > je) return fail(h, SW_E_CUDA, "traceback: no start cell found");
  // (3) directions for the alignment's bounding box only, then the walk
  const int mb = ie - ib + 1, nb = je - jb + 1;
  rc = grow(h, &h->d_tb_dir, &h->tb_dir_cap, (size_t)mb * (size_t)nb, "alloc traceback directions");
  if (rc) return rc;
  const int cap_dev = std::max(1, mb + nb);
  rc = grow(h, &h->d_tb_ops, &h->tb_ops_cap, (size_t)cap_dev * sizeof(uint32_t), "alloc traceback ops");
  if (rc) return rc;
  SW_CUDA(h, launch_traceback(h->d_tb_query + ib, mb, dcols + jb, half, nb, h->d_matrix, h->A, h->rho32, h->sigma32,
                              h->d_tb_dir, h->d_tb_scratch, h->d_tb_result + 8, h->d_tb_ops, cap_dev, nullptr));
  int res[6];
  SW_CUDA(h, cudaMemcpy(res, h->d_tb_result + 8, sizeof(res), cudaMemcpyDeviceToHost));
  if (res[0] != se[0]) return fail(h, SW_E_CUDA, "traceback: box score differs from the full score");
  out->q_begin = ib + res[3]; out->d_begin = jb + res[4];
  out->q_end = ib + res[1] + 1; out->d_end = jb + res[2] + 1;
  out->n_ops = res[5];
  if (res[5] > ops_cap) return fail(h, SW_E_INVALID, "ops buffer too small (need " + std::to_string(res[5]) + ")");
  if (res[5] > 0) SW_CUDA(h, cudaMemcpy(ops, h->d_tb_ops, (size_t)res[5] * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  return SW_OK;
}

int sw_top_hits(sw_handle h, const int32_t* scores, int64_t n, int32_t k, int64_t* idx_out, int32_t* score_out) {
  if (!h) return SW_E_INVALID;
  if (k <= 0 || n <= 0) return SW_OK;
  if (!scores || !idx_out || !score_out) return fail(h, SW_E_INVALID, "NULL buffer");
  const int64_t kk = std::min<int64_t>(k, n);
  const int ctas = topk_ctas(n);
  auto al = [](size_t b) { return (b + 255) & ~(size_t)255; };
  const size_t o_s = 0, o_hist = o_s + al((size_t)n * 4), o_cnt = o_hist + al(256 * 4),
               o_tie = o_cnt + al(4), o_off = o_tie + al((size_t)ctas * 4), o_idx = o_off + al((size_t)ctas * 4),
               o_sc = o_idx + al((size_t)kk * 8), total = o_sc + al((size_t)kk * 4);
  int rc = grow(h, &h->d_tk, &h->tk_cap, total, "alloc top-hits scratch");
  if (rc) return rc;
  int32_t* d_s = reinterpret_cast<int32_t*>(h->d_tk + o_s);
  uint32_t* d_hist = reinterpret_cast<uint32_t*>(h->d_tk + o_hist);
  uint32_t* d_cnt = reinterpret_cast<uint32_t*>(h->d_tk + o_cnt);
  uint32_t* d_tie = reinterpret_cast<uint32_t*>(h->d_tk + o_tie);
  uint32_t* d_off = reinterpret_cast<uint32_t*>(h->d_tk + o_off);
  int64_t* d_idx = reinterpret_cast<int64_t*>(h->d_tk + o_idx);
  int32_t* d_sc = reinterpret_cast<int32_t*>(h->d_tk + o_sc);
  SW_CUDA(h, cudaMemcpy(d_s, scores, (size_t)n * 4, cudaMemcpyHostToDevice));
  // radix select: the k-th largest key, 8 bits per pass from the top
  uint32_t prefix = 0, pmask = 0;
  int64_t remaining = kk;   // how many keys equal to the prefix-so-far are still wanted
  std::vector<uint32_t> hist(256);
  const int hgrid = std::max(1, std::min(ctas, 4 * h->num_sms));
  for (int shift = 24; shift >= 0; shift -= 8) {
    SW_CUDA(h, cudaMemset(d_hist, 0, 256 * 4));
    SW_CUDA(h, launch_tk_hist(d_s, n, shift, prefix, pmask, d_hist, hgrid, nullptr));
    SW_CUDA(h, cudaMemcpy(hist.data(), d_hist, 256 * 4, cudaMemcpyDeviceToHost));
    int64_t cum = 0;
    int digit = 0;
    for (int d = 255; d >= 0; --d) {
      if (cum + hist[d] >= (uint64_t)remaining) { digit = d; break; }
      cum += hist[d];
    }
    remaining -= cum;
    prefix |= (uint32_t)digit << shift;
    pmask |= 0xffu << shift;
  }
  const uint32_t thr = prefix;   // the k-th largest key; kk - remaining keys are above it
  SW_CUDA(h, cudaMemset(d_cnt, 0, 4));
  SW_CUDA(h, launch_tk_above(d_s, n, thr, d_idx, d_sc, d_cnt, d_tie, nullptr));
  uint32_t above = 0;
  SW_CUDA(h, cudaMemcpy(&above, d_cnt, 4, cudaMemcpyDeviceToHost));
  if ((int64_t)above != kk - remaining) return fail(h, SW_E_CUDA, "top hits: selection count mismatch");
  std::vector<uint32_t> ties((size_t)ctas), off((size_t)ctas);
  SW_CUDA(h, cudaMemcpy(ties.data(), d_tie, (size_t)ctas * 4, cudaMemcpyDeviceToHost));
  uint64_t acc = 0;
  for (int b = 0; b < ctas; ++b) { off[(size_t)b] = (uint32_t)std::min<uint64_t>(acc, 0xffffffffu); acc += ties[(size_t)b]; }
  SW_CUDA(h, cudaMemcpy(d_off, off.data(), (size_t)ctas * 4, cudaMemcpyHostToDevice));
  SW_CUDA(h, launch_tk_ties(d_s, n, thr, d_off, (uint32_t)remaining, d_idx + above, d_sc + above, nullptr));
  std::vector<int64_t> idx((size_t)kk);
  std::vector<int32_t> sc((size_t)kk);
  SW_CUDA(h, cudaMemcpy(idx.data(), d_idx, (size_t)kk * 8, cudaMemcpyDeviceToHost));
  SW_CUDA(h, cudaMemcpy(sc.data(), d_sc, (size_t)kk * 4, cudaMemcpyDeviceToHost));
  // the k selected hits, best first (score descending, index ascending)
  std::vector<int64_t> ord((size_t)kk);
  for (int64_t i = 0; i < kk; ++i) ord[(size_t)i] = i;
  std::sort(ord.begin(), ord.end(), [&](int64_t a, int64_t b) {
    return sc[(size_t)a] != sc[(size_t)b] ? sc[(size_t)a] > sc[(size_t)b] : idx[(size_t)a] < idx[(size_t)b];
  });
  for (int64_t i = 0; i < kk; ++i) { idx_out[i] = idx[(size_t)ord[(size_t)i]]; score_out[i] = sc[(size_t)ord[(size_t)i]]; }
  return SW_OK;
}

int sw_last_kernel_ms(sw_handle h, double out[2]) {
  if (!h || !out) return SW_E_INVALID;
  out[0] = out[1] = 0.0;
  for (int k = 0; k < h->stat_nq && kEvPerQuery * k + 2 < (int)h->ev.size(); ++k) {
    float a = 0.f, b = 0.f;
    const cudaEvent_t* ev = h->ev.data() + kEvPerQuery * k;
    cudaError_t e = cudaEventElapsedTime(&a, ev[0], ev[1]);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&b, ev[1], ev[2]);
    if (e != cudaSuccess) return cuda_fail(h, e, "cudaEventElapsedTime");
    out[0] += a;
    out[1] += b;
  }
  return SW_OK;
}

int sw_last_regime_ms(sw_handle h, double out[3]) {
  if (!h || !out) return SW_E_INVALID;
  out[0] = out[1] = out[2] = 0.0;
  for (int k = 0; k < h->stat_nq && kEvPerQuery * k + 4 < (int)h->ev.size(); ++k) {
    float a = 0.f, b = 0.f;
    const cudaEvent_t* ev = h->ev.data() + kEvPerQuery * k;
    cudaError_t e = cudaEventElapsedTime(&a, ev[3], ev[4]);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&b, ev[0], ev[1]);
    if (e != cudaSuccess) return cuda_fail(h, e, "cudaEventElapsedTime");
    out[0] += a;
    out[1] += b;
    if (k < (int)h->long_fused.size() && h->long_fused[k]) out[2] += 1.0;
  }
  return SW_OK;
}

void sw_destroy(sw_handle h) {
  if (!h) return;
  for (cudaEvent_t e : h->ev) cudaEventDestroy(e);
  for (QuerySlot& s : h->slots) {
    if (s.stream) cudaStreamSynchronize(s.stream);
    cudaFree(s.d_prof); cudaFree(s.d_work); cudaFree(s.d_ovf_count); cudaFree(s.d_ovf_list);
    cudaFree(s.d_rb_group); cudaFree(s.d_rb_team); cudaFree(s.d_query); cudaFree(s.d_rb_t); cudaFree(s.d_qpair);
    cudaFree(s.d_gang); cudaFree(s.d_grb);
    if (s.stream) cudaStreamDestroy(s.stream);
    if (s.aux) { cudaStreamSynchronize(s.aux); cudaStreamDestroy(s.aux); }
    if (s.scan) { cudaStreamSynchronize(s.scan); cudaStreamDestroy(s.scan); }
    if (s.scan_fork) cudaEventDestroy(s.scan_fork);
    if (s.scan_done) cudaEventDestroy(s.scan_done);
    if (s.fork) cudaEventDestroy(s.fork);
    if (s.join) cudaEventDestroy(s.join);
    if (s.done) cudaEventDestroy(s.done);
  }
  cudaFree(h->d_matrix);
  h->main_db.release();
  for (auto& ss : h->stream_slot) ss.release();
  cudaFree(h->d_scores_tmp); cudaFree(h->d_batch_q);
  cudaFree(h->d_tb_dir); cudaFree(h->d_tb_scratch); cudaFree(h->d_tb_result); cudaFree(h->d_tb_ops);
  cudaFree(h->d_tk);
  cudaFree(h->d_tb_query);
  if (h->fork) cudaEventDestroy(h->fork);
  if (h->gang_ev) cudaEventDestroy(h->gang_ev);
  if (h->copy_st) cudaStreamDestroy(h->copy_st);
  if (h->h_ovf) cudaFreeHost(h->h_ovf);
  delete h;
}

}  // extern "C"
