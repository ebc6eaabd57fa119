/*
 * eim.h -- C ABI of the B200-native eIM hot path: IMM influence maximisation
 * (Tang, Shi, Xiao, SIGMOD'15 = [22]) with GPU RRR-set sampling and greedy
 * max-coverage seed selection, after Doney, Huang, Lee, "eIM", SC-W'25.
 *
 * Citations: "P:NNN" = line NNN of PAPER.md; "Rn" = reading n in DESIGN.md §3.
 *
 * Conventions (all entry points)
 *   - Plain C types only.  Host input arrays are BORROWED for the duration of
 *     the call (copied to the device); outputs are CALLER-ALLOCATED host
 *     buffers.  The library owns every device allocation; eim_graph_free /
 *     eim_destroy release them.
 *   - Every call returns an eim_status; no exception or longjmp crosses the
 *     ABI.  On failure eim_last_error(ctx) describes the cause; output
 *     buffers are then unspecified unless stated otherwise.
 *   - A context is single-threaded: do not call into one ctx concurrently.
 *   - Results are pure functions of (graph, model, k, eps, ell, seed): they do
 *     not depend on the device count, launch configuration or scheduling
 *     (randomness is counter-based Philox keyed per sample and edge, R1).
 *   - Graph: reverse CSR (CSC of the adjacency).  Row v lists the
 *     in-neighbours u of v (edges u -> v) in ASCENDING order; position e in
 *     in_neighbors is the edge id.  Self-loops and multi-edges are accepted
 *     and count toward the in-degree d^-(v).
 *   - Models use weighted-cascade weights p_uv = 1 / d^-(v)
 *     (LT weights R3).
 */
#ifndef EIM_H
#define EIM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  EIM_OK = 0,
  EIM_E_INVAL = -1,     /* bad argument (see each call) */
  EIM_E_NOMEM = -2,     /* device or host allocation failed */
  EIM_E_CUDA = -3,      /* CUDA runtime error (message in eim_last_error) */
  EIM_E_NCCL = -4,      /* NCCL error (multi-GPU contexts only) */
  EIM_E_CAPACITY = -5,  /* caller buffer too small; required size is still reported */
  EIM_E_STATE = -6      /* object used after free / wrong context */
} eim_status;

typedef enum { EIM_IC = 0, EIM_LT = 1 } eim_model;

typedef struct eim_ctx eim_ctx;      /* one device, one stream, optional NCCL communicator */
typedef struct eim_graph eim_graph;  /* device-resident reverse CSR + IC thresholds */

/* Per-run statistics (nullable output of eim_imm_run). */
typedef struct {
  uint32_t rounds;              /* martingale rounds executed ([22] Alg. 2 loop) */
  uint64_t theta_i[64];         /* |R| after round i */
  uint64_t cov_i[64];           /* coverage of S_i on R after round i */
  double lambda_p, lambda_s;    /* lambda' and lambda* ([22] Eq. 9 and 6) */
  double lb;                    /* lower bound LB on OPT (1 if the loop never broke) */
  uint64_t theta;               /* final |R| */
  uint64_t cov;                 /* coverage of the final seed set */
  uint64_t edges_examined;      /* IC: sum of d^-(u) over expanded u; LT: walk steps (local rank) */
  uint64_t arena_elems;         /* members stored in R (all ranks) */
  uint64_t spilled_samples;     /* IC samples finished in the shared frontier queue (local rank) */
  uint64_t kernel_launches;     /* eim kernels launched by this call (local rank) */
  uint32_t sample_launches;     /* sampler kernel launches */
  double ms_total;              /* wall time of the call (host clock) */
  double ms_sample;             /* wall time in sampling (incl. retries, exchange) */
  double ms_select;             /* wall time in greedy NodeSelection (incl. index build) */
  double ms_comm;               /* wall time in NCCL exchanges */
  double ms_sample_kernel;      /* device time of the sampler kernels (CUDA events on the ctx stream) */
  uint64_t ids_sampled;         /* sample ids drawn by the run, all ranks (> theta with EIM_F_SOURCE_ELIM) */
  uint64_t arena_bytes;         /* device bytes of the stored sets R (log-encoded with an EIM_G_LOG_ENCODE graph) */
  double ms_select_kernel;      /* device time of the greedy pick kernels (CUDA events on their streams; two
                                   concurrent selections both count) */
  uint32_t select_launches;     /* greedy NodeSelections run */
  uint64_t select_picks;        /* greedy picks over all NodeSelections (k per selection) */
} eim_stats;

/* Run flags of eim_imm_run_ex / eim_sample_rrr_ex. */
enum {
  /* Source-vertex elimination (R22): the root of every
   * RRR set is left out of the stored set.  In eim_imm_run_ex a set left
   * empty is discarded and does not count toward |R|: R holds the first
   * theta non-empty sets in sample-id order.  spread_out keeps the method's
   * n*cov/|R| (biased under elimination, see R22). */
  EIM_F_SOURCE_ELIM = 1u,
  /* Fresh final phase ([22]; R23): the final NodeSelection
   * runs on theta = ceil(lambda* / LB) sets drawn afresh from sample ids
   * EIM_FRESH_BASE, EIM_FRESH_BASE+1, ... (eim_imm_run_ex only). */
  EIM_F_FRESH_FINAL = 2u
};
#define EIM_FRESH_BASE (1ULL << 61)

/* IMM parameters of [22] (host-only, no device needed). */
typedef struct {
  double ell_p;     /* l' = l (1 + ln 2 / ln n) */
  double eps_p;     /* eps' = sqrt(2) eps */
  double lnC;       /* ln binom(n, k), summed as sum_{i=1..k} ln(n-k+i) - ln i */
  double lambda_p;  /* lambda' = (2 + 2/3 eps')(lnC + l' ln n + ln log2 n) n / eps'^2 */
  double lambda_s;  /* lambda* = 2 n ((1-1/e) alpha + beta)^2 / eps^2 */
  double log2n;     /* log2(n): the round loop runs while i < log2n */
} eim_imm_params_t;

#define EIM_NCCL_ID_BYTES 128

/* ---------------------------------------------------------------- context
 * eim_create: bind a context to CUDA `device`.  For world > 1 the caller
 * runs one process per GPU, obtains an id from eim_nccl_get_id on rank 0,
 * broadcasts its EIM_NCCL_ID_BYTES bytes (e.g. with torch.distributed) and
 * passes it on every rank; the context then owns an NCCL communicator.
 * `stream` is a cudaStream_t cast to uint64 (0 = the library creates its own
 * non-blocking stream).  All device work of the context is issued on it.
 * Errors: EIM_E_INVAL (device < 0, world < 1, rank not in [0, world),
 * world > 1 without nccl_id), EIM_E_CUDA, EIM_E_NCCL, EIM_E_NOMEM.
 */
eim_status eim_create(int device, int rank, int world, const void* nccl_id, uint64_t stream,
                      eim_ctx** out);
eim_status eim_nccl_get_id(void* out /* EIM_NCCL_ID_BYTES */);
/* eim_create_group: `world` contexts in ONE process, out[r] = rank r on CUDA
 * device devices[r] (caller-allocated array of `world` pointers).  Devices
 * may repeat: several ranks may share one GPU ("virtual ranks").  The ranks
 * share an in-process communicator (host rendezvous + stream-ordered device
 * copies) in place of NCCL and run exactly the multi-rank code of a
 * one-process-per-GPU context: each rank samples a contiguous share of every
 * round's sample ids, the shares are exchanged in rank (= sample-id) order,
 * and every rank's result equals the 1-GPU run.  Collective calls
 * (eim_imm_run, eim_imm_run_ex) must be made on all ranks concurrently, one
 * host thread per rank; the other calls are local to their context.  If one
 * rank's collective call fails, the others fail with EIM_E_NCCL instead of
 * waiting, and the group is unusable afterwards (every later collective
 * call fails).  Each context is released with eim_destroy.
 * Errors: EIM_E_INVAL (NULL arguments, world < 1, a device < 0 or out of
 * range), EIM_E_CUDA, EIM_E_NOMEM; on failure no context is left. */
eim_status eim_create_group(const int* devices, int world, eim_ctx** out);
void eim_destroy(eim_ctx* ctx);
/* Message for the last failed call on ctx (or for the last failed
 * eim_create / host-only call when ctx is NULL).  Valid until the next call. */
const char* eim_last_error(const eim_ctx* ctx);
const char* eim_version(void);

/* ---------------------------------------------------------------- graph
 * eim_load_graph_csr: copy the reverse CSR to the device
 * (replicated on every rank), validate it on the device and derive the IC
 * thresholds T_v = floor((2^32-1) / d^-(v)) (R2: an edge into v is live iff
 * its 32-bit draw <= T_v, i.e. P = 1/d^-(v)).
 *   n: vertices, 2 <= n < 2^32 - 1.  m: edges, m < 2^40.
 *   in_offsets[n+1]: in_offsets[0] = 0, non-decreasing, in_offsets[n] = m.
 *   in_neighbors[m]: values < n.
 * Pinned host buffers make the copies asynchronous and fast.
 * Errors: EIM_E_INVAL for any violation above (nothing is kept), EIM_E_NOMEM,
 * EIM_E_CUDA.
 */
eim_status eim_load_graph_csr(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                              const uint32_t* in_neighbors, eim_graph** out);
eim_status eim_graph_free(eim_graph* g);

/* eim_load_graph_csr_ex: eim_load_graph_csr with graph flags.
 * EIM_G_LOG_ENCODE (Fig. 1; NEXT-2; R19, R24): after
 * validation the device store is log-encoded -- in_offsets packed with
 * bit_width(m) bits per value and in_neighbors with bit_width(max
 * neighbour) bits, value j at bits [j n_b, (j+1) n_b) of a little-endian
 * bit stream of 32-bit containers -- and the plain arrays and per-vertex
 * thresholds are freed; the kernels decode on the fly (T_v recomputed from
 * the decoded degree).  eim_imm_run / eim_sample_rrr on such a graph also
 * store the RRR sets R log-encoded, bit_width(n-1) bits per member (P:99:
 * "applied to both the network data and the RRR sets").  Every result is
 * identical to the plain store's.
 * Errors: those of eim_load_graph_csr, EIM_E_INVAL for an unknown flag. */
enum { EIM_G_LOG_ENCODE = 1u };
eim_status eim_load_graph_csr_ex(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                                 const uint32_t* in_neighbors, uint32_t gflags, eim_graph** out);
/* eim_load_graph_csr_weighted: general edge probabilities (NEXT-3; P:57
 * "each edge (u,v) is assigned a random weight p_uv", P:61 LT "sum <= 1",
 * P:377; R25).  edge_x[m] (host, borrowed; NULL = weighted
 * cascade, i.e. eim_load_graph_csr_ex) gives in-edge e (the position in
 * in_neighbors) the probability p_e = (edge_x[e] + 1) / 2^32; an edge with
 * p = 0 must be left out of the graph.  IC: e is live iff its 32-bit draw
 * <= edge_x[e].  LT: with w_j = edge_x[j] + 1 over a row, the first j with
 * w_0 + ... + w_j > tau is chosen; none (the walk stops) if the row's sum
 * <= tau.  LT needs every row's sum <= 2^32 (sum p <= 1): otherwise the
 * graph loads but LT calls on it return EIM_E_INVAL.  The thresholds are
 * streamed from HBM (4 B per examined in-edge, one 16-B load per Philox
 * quad); LT keeps a per-edge cumulative array (+4 B per edge).
 * With EIM_G_LOG_ENCODE the offsets and in-neighbours are log-encoded as
 * for eim_load_graph_csr_ex while edge_x (and the LT cumulative
 * weights) stay 32-bit; the results are those of the plain weighted store.
 * Errors: those of eim_load_graph_csr_ex. */
eim_status eim_load_graph_csr_weighted(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                                       const uint32_t* in_neighbors, const uint32_t* edge_x, uint32_t gflags,
                                       eim_graph** out);
/* Device bytes held by the graph store (plain: 8(n+1) + 4 max(m,4) + 4n;
 * log-encoded: the two container arrays incl. 2 padding words each; with
 * edge probabilities + 4 (m rounded up to 4, + 4) + 4 max(m,1) for x and
 * the LT cumulative weights).  The LT walk store (a cache built on the
 * first LT run of a plain graph) is not included.
 * Errors: EIM_E_STATE (freed graph), EIM_E_INVAL (bytes NULL). */
eim_status eim_graph_bytes(const eim_graph* g, uint64_t* bytes);

/* ---------------------------------------------------------------- IMM
 * eim_imm_run (Alg. 1, with [22] Alg. 2-3): theta estimation by the
 * martingale loop, RRR sampling of sample ids 0..theta-1 (sets are reused
 * across rounds and topped up, R14), and greedy NodeSelection.
 *   k in [1, n]; eps in (0, 1); ell > 0 (IMM failure exponent, default 1).
 *   seeds_out[k]: seed vertices in pick order.  theta_out: final |R|.
 *   spread_out: n * cov / |R| (RIS estimate).  stats_out nullable.
 * Multi-rank contexts (NCCL or eim_create_group): every rank calls with
 * identical arguments; each rank samples a contiguous share of every
 * round's new ids, the shares are exchanged (all-gather of counts, one
 * broadcast per share) and the greedy runs replicated, so every rank
 * returns the same result, identical to a single-GPU run (also with
 * EIM_F_SOURCE_ELIM: the first theta non-empty sets in sample-id order,
 * wherever the cut falls).  stats_out->edges_examined, spilled_samples,
 * sample_launches and the ms_* fields are this rank's.
 * Errors: EIM_E_INVAL (also when theta = ceil(lambda* / LB) would exceed
 * 2^32 - 1 sets), EIM_E_STATE (graph from another ctx / freed),
 * EIM_E_NOMEM, EIM_E_CUDA, EIM_E_NCCL.
 * Large theta is sampled in several launches, each sized to keep its
 * membership table within 8 GiB (the results do not depend on the split).
 */
eim_status eim_imm_run(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell,
                       eim_model model, uint64_t seed, uint32_t* seeds_out, uint64_t* theta_out,
                       double* spread_out, eim_stats* stats_out);

/* eim_imm_run_ex: eim_imm_run with run flags (EIM_F_SOURCE_ELIM |
 * EIM_F_FRESH_FINAL; 0 = eim_imm_run).  stats_out->ids_sampled counts the
 * sample ids drawn.  Errors: those of eim_imm_run, and EIM_E_INVAL for an
 * unknown flag, or EIM_F_SOURCE_ELIM on a graph with no edge u -> v,
 * u != v (every set would be empty).
 */
eim_status eim_imm_run_ex(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell,
                          eim_model model, uint64_t seed, uint32_t flags, uint32_t* seeds_out,
                          uint64_t* theta_out, double* spread_out, eim_stats* stats_out);

/* eim_sample_rrr (Alg. 2; LT P:134-140): RRR sets of sample ids
 * [first_id, first_id + count), first_id + count <= 2^62, on this context's
 * device (no communication).  Output in sample-id order, each set ascending
 * (P:130): offsets_out[count+1] (offsets_out[0] = 0), members_out[<= cap].
 * *members_total is always set to the number of members.  If members_cap is
 * too small the call returns EIM_E_CAPACITY (offsets_out still valid,
 * members_out unspecified).  Concatenating [a,b) and [b,c) gives [a,c).
 */
eim_status eim_sample_rrr(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                          uint64_t first_id, uint64_t count, uint64_t* offsets_out,
                          uint32_t* members_out, uint64_t members_cap, uint64_t* members_total);
/* eim_sample_rrr_ex: flags = 0 or EIM_F_SOURCE_ELIM.  With EIM_F_SOURCE_ELIM
 * every set is written without its root, possibly empty; the
 * output still has one set per sample id.  Errors: those of eim_sample_rrr,
 * EIM_E_INVAL for any other flag. */
eim_status eim_sample_rrr_ex(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed,
                             uint64_t first_id, uint64_t count, uint32_t flags, uint64_t* offsets_out,
                             uint32_t* members_out, uint64_t members_cap, uint64_t* members_total);

/* eim_select_seeds (Alg. 3): greedy max coverage of an arbitrary
 * arena of num_sets sets over vertices [0, n): offsets[num_sets+1]
 * (offsets[0] = 0, non-decreasing), members[offsets[num_sets]] (< n, no
 * duplicates within a set; order within a set is free).  k in [1, n].
 * seeds_out[k] in pick order; ties go to the lowest vertex id; when every
 * set is covered the remaining picks are the lowest unselected ids (R10).
 * gains_out[k] (nullable) = marginal coverage of each pick.
 * Errors: EIM_E_INVAL for num_sets >= 2^32, decreasing offsets, a member
 * >= n or a member repeated within a set, k outside [1, n].
 */
eim_status eim_select_seeds(eim_ctx* ctx, uint32_t n, uint64_t num_sets, const uint64_t* offsets,
                            const uint32_t* members, uint32_t k, uint32_t* seeds_out,
                            uint64_t* gains_out);

/* eim_get_coverage: the coverage counts C[v] = number of RRR sets of R that
 * contain v ("counts the occurrences of each vertex across all RRR
 * sets"; Alg. 2 l.25), for the R of the most recent eim_imm_run /
 * eim_imm_run_ex (the final R, theta sets; the fresh sets with
 * EIM_F_FRESH_FINAL) or eim_select_seeds (the given arena) on ctx.  These are
 * the counts the first greedy pick of the final NodeSelection maximises.
 * C_out[n] is a caller-allocated host buffer; n must equal the vertex count
 * of that call.  Errors: EIM_E_STATE (no such call on ctx yet, or the last
 * hot-path call was eim_sample_rrr, which builds no counts), EIM_E_INVAL
 * (C_out NULL or n different), EIM_E_CUDA. */
eim_status eim_get_coverage(eim_ctx* ctx, uint32_t n, uint32_t* C_out);

/* Statistics of the most recent eim_imm_run / eim_sample_rrr call on ctx
 * (for eim_sample_rrr: theta = count, edges_examined, sample_launches,
 * spilled_samples, ms_sample_kernel, ms_sample, ms_total, arena_elems,
 * kernel_launches).  Errors: EIM_E_STATE, EIM_E_INVAL (out NULL). */
eim_status eim_get_stats(const eim_ctx* ctx, eim_stats* out);

/* ---------------------------------------------------------------- host-only
 * These need no device and may be called with no context. */
/* IMM parameters (formulas above; R17 fixes the evaluation order).
 * Errors: EIM_E_INVAL if n < 2, k == 0, k > n, eps not in (0,1), ell <= 0. */
eim_status eim_imm_params(uint32_t n, uint32_t k, double eps, double ell, eim_imm_params_t* out);
/* Contiguous share of rank r among `world` ranks of the id range
 * [first, first+count): [first + floor(r count / world), first + floor((r+1) count / world)). */
eim_status eim_shard_range(uint64_t first, uint64_t count, int rank, int world, uint64_t* lo,
                           uint64_t* hi);

#ifdef __cplusplus
}
#endif
#endif /* EIM_H */
