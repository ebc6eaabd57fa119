// imm.cpp -- IMM driver (Alg. 1) with the martingale theta estimation
// of [22] Alg. 2.  Scalars are host doubles (compiled with -ffp-contract=off,
// evaluation order of reading R17); all data work is on the device.
//
// Multi-GPU (world > 1): each round's new sample ids [|R|, theta_i) are split
// into contiguous shares (eim_shard_range), every rank samples its share,
// the shares are all-gathered over NCCL in rank (= sample-id) order and the
// greedy runs replicated on identical data, so results equal the 1-GPU run.
#include <chrono>
#include <cstdlib>
#include <cmath>
#include <cstring>

#include "eim_internal.h"

namespace eim {

uint64_t compact_range(eim_ctx* ctx, uint64_t lo, uint64_t count, uint64_t** d_offsets, uint32_t** d_members);

void imm_params(uint32_t n, uint32_t k, double eps, double ell, eim_imm_params_t* p) {
  const double dn = (double)n;
  const double ln_n = std::log(dn);
  p->ell_p = ell * (1.0 + std::log(2.0) / ln_n);                 // [22] Alg. 1 l.1
  p->eps_p = std::sqrt(2.0) * eps;                                // [22] Alg. 2
  double lnC = 0.0;                                               // ln binom(n,k), in order
  for (uint32_t i = 1; i <= k; ++i) lnC += std::log((double)(n - k + i)) - std::log((double)i);
  p->lnC = lnC;
  p->log2n = std::log2(dn);
  p->lambda_p = (2.0 + (2.0 / 3.0) * p->eps_p) * (lnC + p->ell_p * ln_n + std::log(p->log2n)) * dn /
                (p->eps_p * p->eps_p);                            // Eq. 9
  const double e1 = 1.0 - 1.0 / std::exp(1.0);
  const double alpha = std::sqrt(p->ell_p * ln_n + std::log(2.0));
  const double beta = std::sqrt(e1 * (lnC + p->ell_p * ln_n + std::log(2.0)));
  const double t = e1 * alpha + beta;
  p->lambda_s = 2.0 * dn * (t * t) / (eps * eps);                 // Eq. 6
}

namespace {

using clk = std::chrono::steady_clock;
double ms_since(clk::time_point t0) {
  return std::chrono::duration<double, std::milli>(clk::now() - t0).count();
}

clk::time_point trace_t0;
bool trace_on = false;

struct Exchange {
  DevBuf counts, offs_recv, mem_recv;
};

// After this every rank holds the sets [a, b): rank q contributes its part
// parts[q] (set indices; the parts are contiguous, in rank order = sample-id
// order, and cover [a, b)), which it has already appended to its own arena.
// Each rank compacts its part, the member counts are all-gathered and every
// part is broadcast from its owner and appended by the others; then every
// rank adds the histogram of the whole range to C (the rounds of a
// multi-rank context are launched without it).
void exchange_sets(eim_ctx* ctx, uint64_t a, uint64_t b, const std::vector<std::pair<uint64_t, uint64_t>>& parts,
                   Exchange& ex, eim_stats* st) {
  const auto t0 = clk::now();
  cudaStream_t s = ctx->stream;
  Comm* comm = ctx->comm;
  const int W = ctx->world, me = ctx->rank;
  for (int q = 0; q < W; ++q)
    if (parts[q].second < parts[q].first || parts[q].first != (q ? parts[q - 1].second : a) ||
        (q == W - 1 && parts[q].second != b))
      fail(EIM_E_STATE, "exchange_sets: parts are not a rank-ordered partition of the range");
  ensure_sets(ctx, b);
  uint64_t* d_off = nullptr;
  uint32_t* d_mem = nullptr;
  const uint64_t my_total = compact_range(ctx, parts[me].first, parts[me].second - parts[me].first, &d_off, &d_mem);
  ex.counts.reserve(2 * W * sizeof(uint64_t), false, s);
  uint64_t* d_counts = ex.counts.as<uint64_t>();
  EIM_CUDA(cudaMemcpyAsync(d_counts, &my_total, sizeof(uint64_t), cudaMemcpyHostToDevice, s));
  comm->allgather_u64(d_counts, d_counts + W, s);
  std::vector<uint64_t> totals(W);
  EIM_CUDA(cudaMemcpyAsync(totals.data(), d_counts + W, W * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  EIM_CUDA(cudaStreamSynchronize(s));
  uint64_t max_total = 1, max_sets = 1;
  for (int q = 0; q < W; ++q) {
    max_total = std::max(max_total, totals[q]);
    max_sets = std::max(max_sets, parts[q].second - parts[q].first + 1);
  }
  ex.offs_recv.reserve(max_sets * sizeof(uint64_t), false, s);
  ex.mem_recv.reserve(max_total * sizeof(uint32_t), false, s);
  for (int q = 0; q < W; ++q) {
    const uint64_t pa = parts[q].first, pb = parts[q].second;
    if (pb == pa) continue;
    uint64_t* offs = (q == me) ? d_off : ex.offs_recv.as<uint64_t>();
    uint32_t* mem = (q == me) ? d_mem : ex.mem_recv.as<uint32_t>();
    comm->group_start();
    comm->broadcast(offs, (pb - pa + 1) * sizeof(uint64_t), q, s);
    if (totals[q]) comm->broadcast(mem, totals[q] * sizeof(uint32_t), q, s);
    comm->group_end();
    if (q != me) append_sets(ctx, pa, pb - pa, offs, mem, totals[q]);
  }
  hist_sets(ctx, a, b);
  EIM_CUDA(cudaStreamSynchronize(s));
  // the same on every rank (the launch sizes of all ranks must agree)
  ctx->est_mean_size = std::max(1.0, (double)arena_cursor(ctx) / (double)std::max<uint64_t>(b, 1));
  st->ms_comm += ms_since(t0);
}

// all-gather of one host u64 per rank
std::vector<uint64_t> allgather_host(eim_ctx* ctx, Exchange& ex, uint64_t v) {
  const int W = ctx->world;
  std::vector<uint64_t> out(W, v);
  if (W == 1) return out;
  cudaStream_t s = ctx->stream;
  ex.counts.reserve(2 * W * sizeof(uint64_t), false, s);
  uint64_t* d = ex.counts.as<uint64_t>();
  EIM_CUDA(cudaMemcpyAsync(d, &v, sizeof(uint64_t), cudaMemcpyHostToDevice, s));
  ctx->comm->allgather_u64(d, d + W, s);
  EIM_CUDA(cudaMemcpyAsync(out.data(), d + W, W * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  EIM_CUDA(cudaStreamSynchronize(s));
  return out;
}

// Supplies the sets of sample ids [|R|, to) to the arena.
//
// Every rank of a W-rank context (W = 1 on one GPU) launches its contiguous
// share (eim_shard_range) of a launch range [first, end) and appends its
// part of each requested range [|R|, to); with W > 1 the parts are then
// exchanged (exchange_sets), so every rank holds all sets in sample-id order.
//
// Lookahead (default on; EIM_NO_LOOKAHEAD=1 turns it off): the IMM driver
// may ask one launch to sample the ids of later rounds too (extend_to); their
// sets are then appended from the same round table without a launch -- one
// round tail (the heavy samples' critical paths; for LT the longest walk)
// instead of several.  Sample ids are fixed labels, so the sets are the
// same; if the estimation loop stops first the extra sets are discarded.
//
// Speculation (opt-in EIM_SPECULATE=1, one GPU): the next round's ids are
// launched on a second stream right behind the current round's launch and
// paused while the greedy runs (measured on C2: the speculative round slows
// the current round's critical chains as much as it fills their idle SMs).
//
// Source elimination (R22, elim = true): sets are the non-empty root-less
// sets in sample-id order; a round launches enough ids for the sets still
// needed (from the kept fraction so far); every rank counts the non-empty
// sets of its share, the counts are all-gathered, and the cut (the id of the
// |R|-th kept set) falls in one rank's share: the ranks before it keep all
// their sets and consume all their ids, the cut rank keeps a prefix, the
// ranks after it keep and consume nothing.
class RoundSampler {
 public:
  RoundSampler(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, eim_stats* st, bool elim)
      : ctx_(ctx), g_(g), model_(model), seed_(seed), st_(st), elim_(elim) {
    speculate_ = ctx->world == 1 && !elim && std::getenv("EIM_SPECULATE") != nullptr;
    lookahead_ = !elim && !speculate_ && std::getenv("EIM_NO_LOOKAHEAD") == nullptr;
  }

  // Continue with an empty arena from sample id `id_base` (fresh final phase, R23).
  void restart(uint64_t id_base) {
    cancel();
    drop_held();
    id_base_ = next_id_ = id_base;
  }
  ~RoundSampler() {
    ex_.counts.release();
    ex_.offs_recv.release();
    ex_.mem_recv.release();
  }

  // make sets [R, to) final; extend_to > to: the launch also samples the
  // later rounds' ids [to, extend_to) (lookahead), or the next round is
  // launched speculatively (EIM_SPECULATE)
  void grow(uint64_t& R, uint64_t to, uint64_t extend_to) {
    if (to <= R) return;
    const auto t0 = clk::now();
    if (elim_) {
      grow_elim(R, to);
    } else if (speculate_) {
      st_->ids_sampled += to - R;
      grow_speculate(R, to, extend_to);
    } else {
      st_->ids_sampled += to - R;
      grow_shared(R, to, extend_to);
    }
    st_->ms_sample += ms_since(t0);
  }

  // the held lookahead launch can supply sets [from, to) without a launch
  bool holds(uint64_t from, uint64_t to) const { return held_ && held_done_ == from && launch_end_ >= to; }

  // One GPU, plain runs: can [R, to) come from one launch (held or new)?
  bool can_multi(uint64_t R, uint64_t to) const {
    return W() == 1 && !elim_ && !speculate_ && lookahead_ &&
           (holds(R, to) || to - R <= max_launch_ids(ctx_));
  }

  // Sets [R, ends.back()) from one launch, appended in one pass; for every
  // earlier end t the append leaves snaps[t] = C over sets [0, ends[t]) and
  // totals[t] = the arena elements up to ends[t] (run-ahead selections).
  void grow_multi(uint64_t& R, const std::vector<uint64_t>& ends, uint32_t* const* snaps,
                  std::vector<uint64_t>& totals) {
    const auto t0 = clk::now();
    const uint64_t to = ends.back();
    st_->ids_sampled += to - R;
    if (!holds(R, to)) {
      drop_held();
      launch_range(R, to);
    }
    AppendCuts cuts;
    cuts.n = (uint32_t)ends.size() - 1;
    if (cuts.n > 2) fail(EIM_E_STATE, "grow_multi: at most three rounds per append");
    for (uint32_t j = 0; j < cuts.n; ++j) {
      cuts.cut[j] = ends[j] - launch_first_;
      cuts.snap[j] = snaps[j];
    }
    Round& rd = ctx_->rounds[0];
    account(round_finalize(ctx_, g_, rd, to - launch_first_, R - launch_first_, to < launch_end_, false, &cuts));
    totals.assign(cuts.total, cuts.total + cuts.n);
    totals.push_back(arena_cursor(ctx_));
    held_done_ = to;
    if (to >= launch_end_) drop_held();
    R = to;
    st_->ms_sample += ms_since(t0);
  }

  void cancel() {
    if (spec_) {
      round_cancel(ctx_, *spec_);
      spec_ = nullptr;
    }
    drop_held();
  }

 private:
  cudaStream_t stream_of(const Round& rd) const { return &rd == &ctx_->rounds[0] ? ctx_->rstream[0] : ctx_->rstream[1]; }
  void account(const SampleResult& r) {
    st_->spilled_samples += r.spilled;
    st_->sample_launches += r.launches;
    st_->ms_sample_kernel += r.kernel_ms;
  }
  int W() const { return ctx_->world; }

  // ---- plain runs, any number of ranks.  The held launch covers set
  // indices [launch_first_, launch_end_) (this rank: [my_lo_, my_hi_));
  // sets [launch_first_, held_done_) are appended on every rank.
  void grow_shared(uint64_t& R, uint64_t to, uint64_t extend_to) {
    if (held_) {
      if (held_done_ == R) {
        append_part(R, std::min(launch_end_, to));
        R = held_done_;
      } else {
        drop_held();
      }
    }
    if (to <= R) return;
    drop_held();
    // launches sized for the membership-table budget: a range above it is
    // sampled in several launches (sample ids are fixed labels, same sets)
    const uint64_t cap = max_launch_ids(ctx_) * (uint64_t)W();
    while (to - R > cap) {
      launch_range(R, R + cap);
      append_part(R, R + cap);
      R += cap;
    }
    uint64_t end = (lookahead_ && extend_to > to) ? extend_to : to;
    if (end - R > cap) end = to;
    launch_range(R, end);
    append_part(R, to);
    R = to;
  }

  // Launch this rank's share of the set indices [first, end) and hold it.
  void launch_range(uint64_t first, uint64_t end) {
    const uint64_t R = first;
    launch_first_ = R;
    launch_end_ = end;
    eim_shard_range(R, end - R, ctx_->rank, W(), &my_lo_, &my_hi_);
    trace_mark("launch", first, end);
    Round& rd = ctx_->rounds[0];
    if (my_hi_ > my_lo_)
      round_launch(ctx_, g_, model_, seed_, id_base_ + my_lo_, my_hi_ - my_lo_, id_base_, W() == 1, rd, stream_of(rd),
                   false);
    held_ = true;
    held_done_ = R;
  }

  // Append the sets [a, b) of the held launch (a = held_done_) on every rank.
  void append_part(uint64_t a, uint64_t b) {
    Round& rd = ctx_->rounds[0];
    auto clampr = [](uint64_t x, uint64_t lo, uint64_t hi) { return std::min(std::max(x, lo), hi); };
    const uint64_t pa = clampr(a, my_lo_, my_hi_), pb = clampr(b, my_lo_, my_hi_);
    if (my_hi_ > my_lo_ && rd.launched) account(round_finalize(ctx_, g_, rd, pb - my_lo_, pa - my_lo_, pb < my_hi_));
    if (W() > 1) {
      std::vector<std::pair<uint64_t, uint64_t>> parts(W());
      for (int q = 0; q < W(); ++q) {
        uint64_t lo, hi;
        eim_shard_range(launch_first_, launch_end_ - launch_first_, q, W(), &lo, &hi);
        parts[q] = {clampr(lo, a, b), clampr(hi, a, b)};  // [max(a, lo), min(b, hi)), empty parts at their place
      }
      exchange_sets(ctx_, a, b, parts, ex_, st_);
    }
    held_done_ = b;
    if (b >= launch_end_) drop_held();
  }

  // Discard the rest of a held launch (the loop stopped or moved on).
  void drop_held() {
    if (!held_) return;
    Round& rd = ctx_->rounds[0];
    rd.launched = false;
    rd.waited = false;
    held_ = false;
  }

  // ---- one GPU, EIM_SPECULATE=1
  void grow_speculate(uint64_t& R, uint64_t to, uint64_t next_to) {
    Round* cur = nullptr;
    if (spec_ && spec_->first == id_base_ + R) {
      cur = spec_;
      spec_ = nullptr;
      round_resume(ctx_, g_, *cur, stream_of(*cur));
    } else {
      cancel();
      cur = &ctx_->rounds[0];
      round_launch(ctx_, g_, model_, seed_, id_base_ + R, to - R, id_base_, true, *cur, stream_of(*cur), false);
    }
    const uint64_t cur_end = R + cur->count;
    if (next_to > cur_end) {
      Round& nx = (cur == &ctx_->rounds[0]) ? ctx_->rounds[1] : ctx_->rounds[0];
      round_launch(ctx_, g_, model_, seed_, id_base_ + cur_end, next_to - cur_end, id_base_, true, nx, stream_of(nx),
                   true);
      spec_ = &nx;
    }
    const uint64_t use = std::min<uint64_t>(cur->count, to - R);
    account(round_finalize(ctx_, g_, *cur, use));
    R += use;
    if (to > R) {  // the speculative range was shorter than needed: sample the rest now
      cancel();
      Round& rd = ctx_->rounds[0];
      round_launch(ctx_, g_, model_, seed_, id_base_ + R, to - R, id_base_, true, rd, stream_of(rd), false);
      account(round_finalize(ctx_, g_, rd, to - R));
      R = to;
    }
    if (spec_ && !std::getenv("EIM_SPEC_NOPAUSE")) round_pause(ctx_, *spec_);
  }

  // ---- source elimination, any number of ranks
  void grow_elim(uint64_t& R, uint64_t to) {
    while (R < to) {
      const uint64_t need = to - R;
      // kept fraction so far (first launch: 1/4), 5% + 64 ids of slack
      const double q = consumed_ ? std::max(1e-6, (double)std::max<uint64_t>(kept_, 1) / (double)consumed_) : 0.25;
      const double want = std::ceil((double)need / q * 1.05) + 64.0;
      const uint64_t count = (uint64_t)std::min(want, (double)max_launch_ids(ctx_) * W());
      if (next_id_ + count > (1ull << 62)) fail(EIM_E_INVAL, "sample ids exhausted (< 2^62)");
      uint64_t lo, hi;
      eim_shard_range(next_id_, count, ctx_->rank, W(), &lo, &hi);
      Round& rd = ctx_->rounds[0];
      if (hi > lo)
        round_launch(ctx_, g_, model_, seed_, lo, hi - lo, lo, W() == 1, rd, stream_of(rd), false,
                     RF_DROP_ROOT | RF_DROP_EMPTY);
      const uint64_t kept_mine = (hi > lo) ? round_elim_kept(ctx_, g_, rd) : 0;
      const std::vector<uint64_t> kept = allgather_host(ctx_, ex_, kept_mine);
      // the cut: rank c holds the need-th kept set (none if too few were kept)
      int c = -1;
      uint64_t prefix = 0, my_base = 0, my_take = 0;
      std::vector<std::pair<uint64_t, uint64_t>> parts(W());
      for (int r = 0; r < W(); ++r) {
        const uint64_t take = std::min(kept[r], need - std::min(need, prefix));
        if (c < 0 && prefix + kept[r] >= need) c = r;
        parts[r] = {R + std::min(prefix, need), R + std::min(prefix, need) + take};
        if (r == ctx_->rank) {
          my_base = R + std::min(prefix, need);
          my_take = take;
        }
        prefix += kept[r];
      }
      const uint64_t taken = std::min(prefix, need);
      const bool consume_all = c < 0 || ctx_->rank < c;
      SampleResult r{};
      if (hi > lo) {
        rd.set_base = lo - my_base;  // this rank's kept set j goes to set index my_base + j
        ensure_sets(ctx_, R + taken);
        r = round_finalize(ctx_, g_, rd, my_take, 0, false, consume_all);
        account(r);
      }
      // ids consumed by the whole round: everything up to the cut rank's cut
      uint64_t gconsumed = count;
      if (c >= 0) {
        const std::vector<uint64_t> cons = allgather_host(ctx_, ex_, ctx_->rank == c ? r.consumed : 0);
        uint64_t clo, chi;
        eim_shard_range(next_id_, count, c, W(), &clo, &chi);
        gconsumed = (clo - next_id_) + cons[c];
      }
      if (W() > 1) exchange_sets(ctx_, R, R + taken, parts, ex_, st_);
      R += taken;
      next_id_ += gconsumed;
      kept_ += taken;
      consumed_ += gconsumed;
      st_->ids_sampled += gconsumed;
    }
  }

  eim_ctx* ctx_;
  const eim_graph* g_;
  eim_model model_;
  uint64_t seed_;
  eim_stats* st_;
  bool elim_;
  uint64_t id_base_ = 0;              // sample id of set index 0 (plain runs)
  uint64_t next_id_ = 0;              // next sample id (source elimination)
  uint64_t kept_ = 0, consumed_ = 0;  // kept sets / ids used so far (source elimination, all ranks)
  Exchange ex_;
  bool speculate_ = false;
  Round* spec_ = nullptr;
  bool lookahead_ = false, held_ = false;
  uint64_t launch_first_ = 0, launch_end_ = 0, held_done_ = 0, my_lo_ = 0, my_hi_ = 0;
};

}  // namespace

void trace_reset() {
  trace_on = std::getenv("EIM_TRACE") != nullptr;
  trace_t0 = clk::now();
}

void trace_mark(const char* what, uint64_t a, uint64_t b) {
  if (!trace_on) return;
  std::fprintf(stderr, "trace %9.3f ms  %s %llu %llu\n", ms_since(trace_t0), what, (unsigned long long)a,
               (unsigned long long)b);
}

void imm_run(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell, eim_model model,
             uint64_t seed, uint32_t flags, uint32_t* seeds_out, uint64_t* theta_out, double* spread_out,
             eim_stats* st) {
  const auto t_start = clk::now();
  trace_reset();
  const uint32_t n = g->view.n;
  const bool elim = (flags & EIM_F_SOURCE_ELIM) != 0, fresh = (flags & EIM_F_FRESH_FINAL) != 0;
  if (elim && !graph_has_proper_edge(ctx, g))
    fail(EIM_E_INVAL, "EIM_F_SOURCE_ELIM: the graph has no edge u->v with u != v (every set would be empty)");
  eim_imm_params_t p;
  imm_params(n, k, eps, ell, &p);
  std::memset(st, 0, sizeof(*st));
  st->lambda_p = p.lambda_p;
  st->lambda_s = p.lambda_s;
  const uint64_t launches0 = ctx->kernel_launches;
  cudaStream_t s = ctx->stream;
  // fresh arena + coverage for this graph; R is log-encoded with the graph (NEXT-2)
  const uint32_t arena_b = g->packed ? bit_width((uint64_t)n - 1) : 32u;
  arena_reset(ctx, arena_b);
  edges_reset(ctx);
  uint64_t dropped_edges = 0;  // examined edges of sets dropped again (paired rounds)
  ctx->C_total.reserve((uint64_t)n * sizeof(uint32_t), false, s);
  EIM_CUDA(cudaMemsetAsync(ctx->C_total.p, 0, (uint64_t)n * sizeof(uint32_t), s));
  RoundSampler sampler(ctx, g, model, seed, st, elim);
  std::vector<uint32_t> S(k);
  uint64_t R = 0, cov = 0;
  uint64_t R_selected = UINT64_MAX;  // |R| the last NodeSelection ran on
  // Run-ahead selections: when one launch has sampled rounds i..J (J <= i+2),
  // the NodeSelections of all of them run concurrently (greedy slots 0..J-i,
  // each on its prefix R_t of the arena with a snapshot of C taken after
  // round t's append), and the later rounds' results wait here.  If round t
  // stops the loop, the sets the final phase does not need are dropped again
  // (drop_sets: counts, arena, examined edges), so every reported number is
  // the sequential loop's.  One GPU, plain 32-bit arena; EIM_NO_PAIR=1: off.
  struct Pre {
    uint64_t R, cov;
    std::vector<uint32_t> S;
  };
  std::vector<Pre> pre;
  const bool pairing = ctx->world == 1 && !elim && g->view.off && !g->packed && std::getenv("EIM_NO_PAIR") == nullptr;
  double LB = 1.0;
  auto theta_round = [&](uint32_t i) { return (uint64_t)std::ceil(std::ldexp(p.lambda_p, (int)i) / (double)n); };
  auto has_round = [&](uint32_t i) { return (double)i < p.log2n; };
  // Round t is predicted not to stop the loop when the last round's coverage
  // fraction f, times 2^t, stays below (1+eps') by a margin of three
  // standard errors of f (the fraction falls slowly as R grows: C2 0.098,
  // 0.094, 0.090, 0.087, 0.085).  A scheduling guess only: the results never
  // depend on it (a wrong guess samples ids the loop does not use).
  auto continues = [&](uint32_t t) {
    if (R_selected == UINT64_MAX || R_selected == 0) return false;
    const double f = (double)cov / (double)R_selected;
    if (f <= 0.0) return true;
    const double m = std::min(0.95, std::max(0.5, 1.0 - 3.0 * std::sqrt((1.0 - f) / (f * (double)R_selected))));
    return f * std::ldexp(1.0, (int)t) < m * (1.0 + p.eps_p);
  };
  try {
    for (uint32_t i = 1; has_round(i); ++i) {
      uint64_t R_sel = R;
      if (!pre.empty()) {  // this round's selection ran with an earlier one
        R_sel = pre.front().R;
        cov = pre.front().cov;
        S.swap(pre.front().S);
        pre.erase(pre.begin());
      } else {
        // the launch extent: round i+1 when it adds no more ids than round i
        // (cheap even if round i stops) or round i is predicted to continue;
        // round i+2 as well when rounds i and i+1 are both predicted to
        // continue (run-ahead selections only)
        uint32_t J = i;
        if (has_round(i + 1) && (theta_round(i + 1) - theta_round(i) <= theta_round(i) - R || continues(i))) {
          J = i + 1;
          if (pairing && has_round(i + 2) && continues(i) && continues(i + 1)) J = i + 2;
        }
        // run the selections of rounds i..i+nsel-1 at once: slot nsel-1-t
        // runs round i+t on Rs[t] sets (arena prefix totals[t]) with C
        // snapshot t (round J on the live counts, in slot 0); the later
        // rounds' results wait in `pre`
        auto run_ahead = [&](uint32_t nsel, const std::vector<uint64_t>& Rs, const std::vector<uint64_t>& totals,
                             uint32_t* const* snaps) {
          for (uint32_t t = 0; t < nsel; ++t)
            greedy_setup(ctx, nsel - 1 - t, n, Rs[t], totals[t],
                         t + 1 == nsel ? ctx->C_total.as<uint32_t>() : snaps[t]);
          uint32_t share[3];
          greedy_shares(ctx, nsel, Rs.data(), share);
          for (uint32_t t = 0; t < nsel; ++t) greedy_picks(ctx, nsel - 1 - t, n, Rs[t], k, share[t]);
          trace_mark("selections enqueued", nsel, Rs[nsel - 1]);
          for (uint32_t t = 0; t < nsel; ++t) {
            if (t == 0) {
              cov = greedy_collect(ctx, nsel - 1, k, S.data(), nullptr, &st->ms_select_kernel);
            } else {
              Pre q{Rs[t], 0, std::vector<uint32_t>(k)};
              q.cov = greedy_collect(ctx, nsel - 1 - t, k, q.S.data(), nullptr, &st->ms_select_kernel);
              pre.push_back(std::move(q));
            }
          }
          trace_mark("selections collected", nsel, Rs[nsel - 1]);
          st->select_launches += nsel;
          st->select_picks += (uint64_t)nsel * k;
        };
        DevBuf* snapb[2] = {&ctx->C_snap, &ctx->C_snap2};
        const uint32_t nsel = J - i + 1;
        if (pairing && J > i && sampler.can_multi(R, theta_round(J))) {
          // rounds i..J from one launch and ONE append (one scan, one host
          // read-back, one scatter that also fills the round snapshots of C)
          std::vector<uint64_t> Rs(nsel), totals;
          uint32_t* snaps[2] = {nullptr, nullptr};
          for (uint32_t t = 0; t < nsel; ++t) Rs[t] = theta_round(i + t);
          for (uint32_t t = 0; t + 1 < nsel; ++t) {
            snapb[t]->reserve((uint64_t)n * sizeof(uint32_t), false, s);
            snaps[t] = snapb[t]->as<uint32_t>();
          }
          sampler.grow_multi(R, Rs, snaps, totals);
          R_sel = Rs[0];
          const auto ts = clk::now();
          run_ahead(nsel, Rs, totals, snaps);
          st->ms_select += ms_since(ts);
        } else {
          sampler.grow(R, theta_round(i), theta_round(J));
          R_sel = R;
          const auto ts = clk::now();
          if (pairing && J > i && sampler.holds(R, theta_round(i + 1))) {
            // (a launch split for the table budget) one append per round
            std::vector<uint64_t> Rs(nsel), totals(nsel);
            uint32_t* snaps[2] = {nullptr, nullptr};
            for (uint32_t t = 0; t < nsel; ++t) {
              Rs[t] = R;
              totals[t] = arena_cursor(ctx);
              if (t + 1 == nsel) break;
              snapb[t]->reserve((uint64_t)n * sizeof(uint32_t), false, s);
              snaps[t] = snapb[t]->as<uint32_t>();
              EIM_CUDA(cudaMemcpyAsync(snaps[t], ctx->C_total.p, (uint64_t)n * sizeof(uint32_t),
                                       cudaMemcpyDeviceToDevice, s));
              const auto tg = clk::now();
              sampler.grow(R, theta_round(i + t + 1), theta_round(J));  // appends the held sets, no launch
              st->ms_select -= ms_since(tg);
            }
            run_ahead(nsel, Rs, totals, snaps);
          } else {
            trace_mark("selection", R);
            cov = greedy(ctx, n, R, k, S.data(), nullptr, &st->ms_select_kernel);
            trace_mark("selection collected", R);
            st->select_launches += 1;
            st->select_picks += k;
          }
          st->ms_select += ms_since(ts);
        }
      }
      R_selected = R_sel;
      if (st->rounds < 64) {
        st->theta_i[st->rounds] = R_sel;
        st->cov_i[st->rounds] = cov;
      }
      st->rounds++;
      if ((double)cov * std::ldexp(1.0, (int)i) >= (1.0 + p.eps_p) * (double)R_sel) {
        LB = ((double)n * (double)cov) / ((1.0 + p.eps_p) * (double)R_sel);
        break;
      }
    }
    st->lb = LB;
    const double theta_d = std::ceil(p.lambda_s / LB);
    // set ids of the greedy's inverted index are 32-bit
    if (!(theta_d < 4294967295.0)) fail(EIM_E_INVAL, "theta = ceil(lambda*/LB) exceeds 2^32 - 1 sets");
    const uint64_t theta = (uint64_t)theta_d;
    if (R > R_selected && R_selected != UINT64_MAX) {
      // the loop stopped at a round whose later rounds' sets are appended:
      // keep max(theta, |R_i|) of them (the sequential loop's final |R|; with
      // a fresh final phase the estimation phase sampled exactly |R_i|)
      const uint64_t keep = fresh ? R_selected : std::max<uint64_t>(theta, R_selected);
      if (keep < R) {
        drop_sets(ctx, g, model == EIM_IC, keep, R, &dropped_edges);
        st->ids_sampled -= R - keep;
        R = keep;
      }
      for (Pre& q : pre)  // a run-ahead selection on exactly the final R is the final one
        if (q.R == R) {
          R_selected = R;
          S.swap(q.S);
          cov = q.cov;
        }
    }
    pre.clear();
    if (fresh) {  // R23: the final sets are drawn afresh from ids 2^61..
      sampler.restart(EIM_FRESH_BASE);
      arena_reset(ctx, arena_b);
      EIM_CUDA(cudaMemsetAsync(ctx->C_total.p, 0, (uint64_t)n * sizeof(uint32_t), s));
      R = 0;
      R_selected = UINT64_MAX;
    }
    sampler.grow(R, theta, 0);
    sampler.cancel();
  } catch (...) {
    sampler.cancel();
    throw;
  }
  if (R != R_selected) {  // NodeSelection is deterministic: reuse the last run on the same R
    const auto ts = clk::now();
    trace_mark("final selection", R);
    cov = greedy(ctx, n, R, k, S.data(), nullptr, &st->ms_select_kernel);
    st->select_launches += 1;
    st->select_picks += k;
    st->ms_select += ms_since(ts);
  }
  std::memcpy(seeds_out, S.data(), (size_t)k * sizeof(uint32_t));
  st->edges_examined = edges_read(ctx) - dropped_edges;
  st->theta = R;
  st->cov = cov;
  st->arena_elems = arena_cursor(ctx);
  st->arena_bytes = ctx->arena_b == 32 ? 4 * st->arena_elems : 4 * arena_words(st->arena_elems, ctx->arena_b);
  if (theta_out) *theta_out = R;
  if (spread_out) *spread_out = (double)n * (double)cov / (double)R;
  st->kernel_launches = ctx->kernel_launches - launches0;
  st->ms_total = ms_since(t_start);
  trace_mark("imm done", R);
}

}  // namespace eim
