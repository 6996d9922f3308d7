/*
 * sw.h — C ABI of the B200-native Smith-Waterman database-search hot path
 * (Hains, Cashero, Ottenberg, Bohm, Rajopadhye, "Improving CUDASW++", IPDPS 2011).
 *
 * The operation (PAPER.md L10 abstract; L12 §II Eq.(1); L14 §II-B): "computes the
 * similarity scores of a query sequence paired with each sequence in a database".  For a
 * query q (length m), database sequence d (length n), scoring function w, gap open rho and
 * gap extension sigma, the score is max_{i,j} H[i][j] of
 *
 *     E[i][j] = max(E[i][j-1] - sigma, H[i][j-1] - rho)
 *     F[i][j] = max(F[i-1][j] - sigma, H[i-1][j] - rho)
 *     H[i][j] = max(0, E[i][j], F[i][j], H[i-1][j-1] + w(q_i, d_j))
 *
 * with H = 0 on row/column 0 and E/F = -inf there (readings c1-c4).  A gap of
 * length k therefore costs rho + (k-1)*sigma (reading c2).  The result is exact (int32),
 * identical for every length_threshold and every sharding (reading c8, c20).
 *
 * Conventions
 *   - Every call returns an int status (SW_OK = 0); nothing aborts or exits.
 *   - Residue / query codes are integers in [0, alphabet_size); the library never sees
 *     letters.  matrix is row-major int8 [alphabet_size][alphabet_size], indexed
 *     [query symbol][database symbol] (reading c5; it need not be symmetric).
 *   - Ownership: the caller owns every input buffer; the library COPIES query, matrix and
 *     database (device copies belong to the handle until sw_destroy).  Output buffers are
 *     caller-allocated.
 *   - A handle is bound to the CUDA device current at sw_create and is not thread-safe;
 *     distinct handles may be used concurrently.  There is no CPU fallback: on a device
 *     that is not compute capability 10.0 (sm_100a) sw_create returns SW_E_UNSUPPORTED.
 */
#ifndef SW_B200_H
#define SW_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sw_handle_s* sw_handle;

enum {
  SW_OK = 0,
  SW_E_INVALID = 1,      /* bad argument (NULL, length, code >= alphabet, bad offsets, ...) */
  SW_E_STATE = 2,        /* call out of order (e.g. search before sw_load_db) */
  SW_E_NOMEM = 3,        /* host or device allocation failed */
  SW_E_CUDA = 4,         /* CUDA runtime error; detail in sw_last_error */
  SW_E_UNSUPPORTED = 5   /* device is not sm_100 / parameters outside the supported range */
};

/* Limits (validated; SW_E_INVALID / SW_E_UNSUPPORTED otherwise). */
#define SW_MAX_ALPHABET 32          /* alphabet_size in [1, 32] */
#define SW_MAX_QUERY_LEN (1 << 16)  /* 1 <= query_len <= 65536 (SW_E_INVALID beyond) */
/* The int8 query profile (alphabet_size + 1 rows of query_len bytes, padded to the kernel's
 * strip layout) is staged whole in one CTA's shared memory when it fits SW_MAX_PROFILE_BYTES
 * (query_len up to ~8,900 for the 24-letter protein alphabet; the paper's queries reach 5478).
 * Longer queries run in long-query mode: every database sequence takes the transposed
 * long-sequence kernel, which streams the query from device memory and builds substitution
 * tables per database strip (no query profile); the flagged sequences are recomputed by its
 * 32-bit instantiation.  Same exact scores, every query length up to SW_MAX_QUERY_LEN. */
#define SW_MAX_PROFILE_BYTES (220 * 1024)
#define SW_MAX_SEQ_LEN ((1 << 20) - 64)  /* every database sequence length <= 1,048,512 */

/* length_threshold value asking the library to choose the inter/intra-task threshold itself
 * (§VI "automatic detection of the optimal threshold value"). */
#define SW_AUTO_THRESHOLD (-1)

/* Create a handle for one query and one scoring scheme (§II: q, w, rho, sigma).
 *   query[query_len]      codes < alphabet_size, 1 <= query_len <= SW_MAX_QUERY_LEN
 *   matrix[A*A]           int8, row = query symbol, column = database symbol
 *   gap_open  (rho)       >= 0;  gap_extend (sigma) >= 0  (any int32 values; Eq.(1) bounds
 *                         neither: rho + max(matrix) > 127 selects the WIDE kernels, whose
 *                         int8 profile holds w + c with c < rho and adds rho - c per cell;
 *                         penalties above 16384 are clamped for the 16-bit lanes with the
 *                         overflow flag lowered to 16384, which is exact: DESIGN.md "Integer
 *                         widths")
 * Uploads the query and builds the query profile on the device (§II-A). */
int sw_create(sw_handle* out, const uint8_t* query, int32_t query_len,
              const int8_t* matrix, int32_t alphabet_size, int32_t gap_open, int32_t gap_extend);

/* Replace the query (same matrix and penalties); keeps the loaded database. */
int sw_set_query(sw_handle h, const uint8_t* query, int32_t query_len);

/* Load a CSR database (copied): sequence k is residues[offsets[k] .. offsets[k+1]).
 *   offsets[0] == 0, non-decreasing, offsets[num_seqs] == total_residues; each length
 *   <= SW_MAX_SEQ_LEN; codes < alphabet_size; num_seqs >= 0 (length-0 sequences score 0).
 * Host preprocessing (§II-C "sorted by length"): stable sort by length
 * descending, pairing of neighbours, packing into the device layout.
 * Replaces any previously loaded database. */
int sw_load_db(sw_handle h, const uint8_t* residues, int64_t total_residues,
               const int64_t* offsets, int64_t num_seqs);

/* Score the handle's query against every database sequence (blocking).
 *   scores_out: HOST int32[num_seqs], caller's database order.
 *   length_threshold T >= 0: sequences with n >= T take the long-sequence (intra-task)
 *   path, n < T the short-sequence (inter-task) path (§II-B: "If the
 *   database sequence length is below 3072, the inter-task kernel is used. Otherwise,
 *   the intra-task kernel is used.").  Scores do not depend on T. */
int sw_search(sw_handle h, int32_t* scores_out, int32_t length_threshold);
/* (length_threshold == SW_AUTO_THRESHOLD: chosen per query by the library's time model;
 * sw_last_threshold reports the value used by the last query.) */
int32_t sw_last_threshold(sw_handle h);

/* Same, stream-ordered: d_scores_out is a DEVICE int32[num_seqs] (e.g. a torch tensor);
 * cuda_stream is a cudaStream_t (NULL = legacy default stream).  Returns after enqueueing. */
int sw_search_async(sw_handle h, int32_t* d_scores_out, int32_t length_threshold, void* cuda_stream);

/* Batch of queries against the loaded database (extension): query k is
 * queries[q_offsets[k] .. q_offsets[k+1]); scores for query k go to
 * d_scores_out[k*num_seqs .. (k+1)*num_seqs) (DEVICE pointer, stream-ordered).  The
 * handle's own query is not changed.  Queries run concurrently on internal streams that
 * are joined back into cuda_stream. */
int sw_search_batch_async(sw_handle h, const uint8_t* queries, const int64_t* q_offsets,
                          int32_t num_queries, int32_t* d_scores_out, int32_t length_threshold,
                          void* cuda_stream);

/* Autotune (all search calls on a database loaded with sw_load_db): the first search of a
 * (query length, threshold) whose cells (query length x database residues) reach 1e10 times
 * the planner's 5 best kernel configurations, one search each, on the handle's first internal
 * stream, and keeps the fastest for later searches of that (query length, threshold).  With
 * length_threshold == SW_AUTO_THRESHOLD the first search of a query length with >= 1e9 cells
 * also times the threshold model's four best candidates and the all-short endpoint (plus the
 * all-long one on databases whose sequences are all >= 512) and keeps the fastest threshold
 * for that query length.  That first call therefore synchronises with the device (the async
 * variants block for it) and costs a few searches; its scores are the exact ones (every
 * configuration and threshold computes the same scores).  The tables are cleared by
 * sw_load_db.  Environment SW_AUTOTUNE=0 disables both (the planner's model choices only). */

/* Host-pointer variant of sw_search_batch_async (blocking; host int32[num_queries*num_seqs]). */
int sw_search_batch(sw_handle h, const uint8_t* queries, const int64_t* q_offsets,
                    int32_t num_queries, int32_t* scores_out, int32_t length_threshold);

/* Streamed database search (extension; §VI: "copy a slice of
 * the database to the GPU, start aligning, and copy the rest of the database in the
 * background").  A batch of queries (same form as sw_search_batch; queries == NULL: the
 * handle's own query, num_queries/q_offsets ignored) against a HOST-resident database (same
 * CSR form as sw_load_db, only read during the call).  The database is cut into chunks of
 * whole sequences of about chunk_residues residues (the first three ramp up: about 1/8, 1/4
 * and 1/2 of it, so that the packing of the first chunk, which no search hides, is short);
 * each chunk is sorted and packed on the
 * host (pinned staging) and copied on an upload stream while the previous chunk is searched,
 * two device slots alternating (kept on the handle for the next call).  The handle's loaded
 * database (if any) is neither used nor changed.
 *   scores_out: HOST int32[num_queries * num_seqs], query-major, caller order.
 * Blocking.  Errors: as sw_load_db and sw_search_batch; chunk_residues <= 0 -> SW_E_INVALID.
 * sw_last_stats afterwards sums over the chunks. */
int sw_search_stream(sw_handle h, const uint8_t* queries, const int64_t* q_offsets, int32_t num_queries,
                     const uint8_t* residues, int64_t total_residues, const int64_t* offsets,
                     int64_t num_seqs, int32_t* scores_out, int32_t length_threshold,
                     int64_t chunk_residues);

/* Statistics of the last search on h (for measurement / tests):
 *   out[0] = number of sequences recomputed in 32-bit after the 16-bit overflow flag,
 *   out[1] = long-path (intra-task) sequences, out[2] = short-path sequences,
 *   out[3] = kernel launches enqueued by the last search call. */
int sw_last_stats(sw_handle h, int64_t out[4]);

/* Device time of the last search call's kernels, from CUDA events recorded on the launching
 * streams (valid after the work completed): out[0] = sum over queries of the search kernel
 * (both regimes, one fused launch per query), out[1] = sum of the 32-bit recompute launches.
 * Milliseconds. */
int sw_last_kernel_ms(sw_handle h, double out[2]);

/* Per-regime device time of the last search call (valid after its work completed), for the
 * threshold sweeps (Fig.5 analog: share of the time in the intra-task kernel):
 *   out[0] = sum over queries of the separate long-sequence launch (T-mode, on the query's
 *            second stream, concurrent with the short-sequence launch; 0 when none ran),
 *   out[1] = sum over queries of the whole search interval (== sw_last_kernel_ms out[0]),
 *   out[2] = number of queries whose long sequences ran inside the fused search launch (team
 *            mode, queries >= 3072 residues): their long-path time is part of out[1] only.
 * Milliseconds (out[2]: a count). */
int sw_last_regime_ms(sw_handle h, double out[3]);

/* Optimal local alignment of the handle's query with database sequence seq_index (caller
 * order) — the traceback step after the search ("The optimal
 * alignment can be found by backtracking through H").  Computed on the device in bounded
 * memory: an anti-diagonal sweep of Eq.(1) for the score and the end cell (O(m) scratch), a
 * sweep of the reversed prefixes anchored at the end cell for the start cell, then a sweep of
 * the alignment's bounding box only, writing one direction byte per cell ((q_end - q_begin) x
 * (d_end - d_begin) bytes of device scratch instead of m*n), and a walk back from the first
 * maximal cell of the box.  Query rows [q_begin, q_end) are aligned to
 * database columns [d_begin, d_end) (0-based, end exclusive; all 0 when score == 0).
 * ops[0 .. n_ops): runs (length << 2) | op, op 0 = M (q_i against d_j), 1 = I (d_j against a
 * gap), 2 = D (q_i against a gap); a gap closed and reopened (possible when sigma > rho) is two
 * runs.  The score of the runs (sum of w over M columns, rho + (len-1)*sigma per gap run)
 * equals out->score.  If ops_cap < n_ops nothing is copied and SW_E_INVALID is returned with
 * out->n_ops set.  Blocking. */
typedef struct {
  int32_t score;
  int32_t q_begin, q_end;
  int32_t d_begin, d_end;
  int32_t n_ops;
} sw_alignment;
int sw_align(sw_handle h, int64_t seq_index, sw_alignment* out, uint32_t* ops, int32_t ops_cap);

/* The top hits of a score array ("traceback for top hits"): the k largest of
 * scores[0 .. n) (host array, e.g. sw_search's output), ties broken by the smaller index,
 * selected on the device (radix-select histograms over the 32-bit keys, then the < k + ties
 * candidates ordered).  idx_out / score_out (host, min(k, n) entries) receive them best first.
 * k <= 0 or n == 0: nothing.  Returns SW_E_INVALID for NULL buffers with k > 0 and n > 0.
 * Blocking.  The handle's stream resources are used; no database is needed. */
int sw_top_hits(sw_handle h, const int32_t* scores, int64_t n, int32_t k, int64_t* idx_out, int32_t* score_out);

/* Free everything (NULL-safe). */
void sw_destroy(sw_handle h);

/* Static text for a status code. */
const char* sw_strerror(int status);

/* Detail of the last failing call on h (never NULL; "" when none). */
const char* sw_last_error(sw_handle h);

/* Library / build identification, e.g. "sw_b200 sm_100a". */
const char* sw_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SW_B200_H */
