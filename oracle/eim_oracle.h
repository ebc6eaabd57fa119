/*
 * eim_oracle.h -- plain, slow, single-threaded CPU oracle for the eIM hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path may include, link or
 * call this file: only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs use it.  It shares no code, header,
 * table or constant with paper_conf_sc_doneyhl25_b200/csrc (the CUDA path).
 *
 * Citations: "P:NNN" is line NNN of PAPER.md (Doney, Huang, Lee, eIM, SC-W'25);
 * "[22]" is Tang, Shi, Xiao, IMM, SIGMOD'15 (cited at P:409), from which the
 * paper takes every IMM formula.  "R#" is a numbered reading in DESIGN.md §3.
 *
 * Parity status per function (see DESIGN.md §4 for the pins):
 *   orc_philox4x32_10 .. pinned (Random123 known-answer vectors)
 *   orc_root ........... pinned (closed form for n = 2^a, chi-square)
 *   orc_ic_live ........ pinned (exact rational comparison, exhaustive)
 *   orc_lt_choice ...... pinned (closed form floor(tau*d), exhaustive bounds)
 *   orc_rrr_set ........ pinned (materialised live-edge world + library BFS;
 *                        exact enumeration of worlds, RIS unbiasedness)
 *   orc_coverage ....... pinned (closed forms: path/cycle/empty graph,
 *                        sum = arena size, brute-force membership count)
 *   orc_greedy ......... pinned (brute force OPT, (1-1/e) bound, marginal
 *                        gains, tie order)
 *   orc_imm_params ..... pinned (mpmath 40-digit evaluation of [22] Eq. 6/9)
 *   orc_imm ............ pinned through its parts + LB/theta recomputation
 *   source elimination . pinned (set = plain set minus root; closed forms on
 *                        path/star; enumeration of the retained-set law)
 *   fresh final phase .. pinned (estimation identical to the plain run;
 *                        final = greedy over ids from ORC_FRESH_BASE)
 *   *_w (NEXT-3) ....... pinned (WC-derived weights reproduce the WC path;
 *                        exact enumeration with general weights incl. the
 *                        LT "no neighbour" outcome; boundary draws)
 *   orc_log_* .......... pinned (Fig. 1 example, hand-built containers,
 *                        numpy unpackbits layout, round trip)
 */
#ifndef EIM_ORACLE_H
#define EIM_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_IC = 0, ORC_LT = 1 };
enum { ORC_TAG_EDGE = 0, ORC_TAG_ROOT = 1, ORC_TAG_LT = 2 };
/* run flags (NEXT rows of SURVEY §8(f); R22, R23) */
enum { ORC_SOURCE_ELIM = 1, ORC_FRESH_FINAL = 2 };
#define ORC_FRESH_BASE (1ULL << 61) /* first sample id of a fresh final phase */

/* ---- randomness (reading R1) ---------------------------------------- */
void     orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* word `word` (0..3) of Philox(counter(q, s, tag), key(seed)) */
uint32_t orc_draw(uint64_t seed, uint64_t s, uint32_t tag, uint64_t q, uint32_t word);
uint32_t orc_edge_draw(uint64_t seed, uint64_t s, uint64_t e);
uint32_t orc_lt_draw(uint64_t seed, uint64_t s, uint32_t u);
uint32_t orc_root(uint64_t seed, uint64_t s, uint32_t n);

/* ---- diffusion-model decisions -------------------------------------- */
int      orc_ic_live(uint32_t draw, uint64_t d);      /* r <= p_vu with p = 1/d (R2) */
uint32_t orc_lt_choice(uint32_t tau, uint64_t d);     /* prefix-scan choice (R3-R5) */

/* general edge probabilities (NEXT-3, R25): p_e = (x_e + 1) / 2^32 */
int      orc_ic_live_w(uint32_t draw, uint32_t x);
/* first j with sum_{i<=j} (x_row[i] + 1) > tau, UINT32_MAX if none */
uint32_t orc_lt_choice_w(uint32_t tau, const uint32_t* x_row, uint64_t d);
/* every row's sum of (x_e + 1) <= 2^32 (LT: sum p <= 1) */
int      orc_lt_weights_ok(uint32_t n, const uint64_t* off, const uint32_t* x);

/* ---- one RRR set ------------------------------------------------------
 * Writes the members of RRR set `s` (ascending) to out[] (capacity n) and
 * returns the set size.  stamp[] is caller scratch of n uint64 that must be
 * all-zero before the first call (it is reused across calls). */
uint32_t orc_rrr_set(uint32_t n, const uint64_t* off, const uint32_t* nbr, int model,
                     uint64_t seed, uint64_t s, uint32_t* out, uint64_t* stamp);

/* ---- a range of RRR sets (the arena) ---------------------------- */
typedef struct {
  uint64_t  num_sets;
  uint64_t  total;      /* number of members */
  uint64_t* offsets;    /* num_sets + 1 */
  uint32_t* members;    /* total */
  uint64_t  edges_examined;  /* IC: sum of in-degrees of expanded vertices; LT: walk steps */
  uint64_t* set_edges;  /* num_sets: the examined edges (walk steps) of each set */
} orc_arena;

/* nthreads > 1 splits the id range over threads; the result is identical. */
orc_arena* orc_sample(uint32_t n, const uint64_t* off, const uint32_t* nbr, int model,
                      uint64_t seed, uint64_t first, uint64_t count, int nthreads);
/* flags & ORC_SOURCE_ELIM: each set without its source (root) vertex,
 * possibly empty. */
orc_arena* orc_sample_ex(uint32_t n, const uint64_t* off, const uint32_t* nbr, int model,
                         uint64_t seed, uint64_t first, uint64_t count, uint32_t flags, int nthreads);
/* x: per-edge probabilities (R25), NULL = weighted cascade */
orc_arena* orc_sample_w(uint32_t n, const uint64_t* off, const uint32_t* nbr, const uint32_t* x, int model,
                        uint64_t seed, uint64_t first, uint64_t count, uint32_t flags, int nthreads);
void       orc_arena_free(orc_arena* a);

/* ---- greedy NodeSelection (Alg. 3) ------------------------- */
/* returns cov = sum of gains */
uint64_t orc_greedy(uint32_t n, uint64_t num_sets, const uint64_t* offsets, const uint32_t* members,
                    uint32_t k, uint32_t* seeds_out, uint64_t* gains_out);

/* coverage counts C[v] = #sets containing v (Alg. 2 l.25) */
void orc_coverage(uint32_t n, uint64_t num_sets, const uint64_t* offsets, const uint32_t* members, uint32_t* C);

/* ---- IMM (Alg. 1; [22] Alg. 1-3, Eq. 6 and 9) --------------- */
typedef struct {
  double ell_p, eps_p, lnC, lambda_p, lambda_s, log2n;
} orc_params;
int orc_imm_params(uint32_t n, uint32_t k, double eps, double ell, orc_params* out);

typedef struct {
  uint32_t rounds;
  uint64_t theta_i[64];
  uint64_t cov_i[64];
  double   lambda_p, lambda_s, lb;
  uint64_t theta;            /* final |R| */
  uint64_t cov;              /* coverage of the final seed set */
  uint64_t edges_examined;
  uint64_t arena_elems;
  uint64_t ids_sampled;      /* sample ids drawn (> theta with source elimination) */
} orc_imm_stats;

int orc_imm(uint32_t n, const uint64_t* off, const uint32_t* nbr, uint32_t k, double eps,
            double ell, int model, uint64_t seed, int nthreads,
            uint32_t* seeds_out, uint64_t* theta_out, double* spread_out, orc_imm_stats* st);
/* flags: ORC_SOURCE_ELIM | ORC_FRESH_FINAL.  Returns -1 for invalid
 * parameters, including ORC_SOURCE_ELIM on a graph without an edge u->v,
 * u != v (every eliminated set would be empty). */
int orc_imm_ex(uint32_t n, const uint64_t* off, const uint32_t* nbr, uint32_t k, double eps,
               double ell, int model, uint64_t seed, uint32_t flags, int nthreads,
               uint32_t* seeds_out, uint64_t* theta_out, double* spread_out, orc_imm_stats* st);

/* ---- log encoding (Fig. 1; R19, R24) ------------------------- */
uint32_t orc_log_bits(uint64_t x_max);                 /* bit_width(x_max) */
uint64_t orc_log_words(uint64_t count, uint32_t b);    /* 32-bit containers */
void     orc_log_encode(const uint64_t* x, uint64_t count, uint32_t b, uint32_t* words);
uint64_t orc_log_decode(const uint32_t* words, uint64_t j, uint32_t b);

int orc_imm_w(uint32_t n, const uint64_t* off, const uint32_t* nbr, const uint32_t* x, uint32_t k, double eps,
              double ell, int model, uint64_t seed, uint32_t flags, int nthreads,
              uint32_t* seeds_out, uint64_t* theta_out, double* spread_out, orc_imm_stats* st);

#ifdef __cplusplus
}
#endif
#endif
