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

struct Exchange {
  DevBuf counts, offs_recv, mem_recv, len_send;
};

// Sets [R, R_new) (sample ids id_base + set index) across ranks; afterwards
// every rank holds all of them.
void sample_round(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, uint64_t id_base, uint64_t R,
                  uint64_t R_new, eim_stats* st, Exchange& ex) {
  const auto t0 = clk::now();
  cudaStream_t s = ctx->stream;
  uint64_t lo, hi;
  eim_shard_range(R, R_new - R, ctx->rank, ctx->world, &lo, &hi);
  SampleResult r = sample_range(ctx, g, model, seed, id_base + lo, hi - lo, id_base, false);
  st->edges_examined += r.edges;
  st->spilled_samples += r.spilled;
  st->sample_launches += r.launches;
  st->ms_sample_kernel += r.kernel_ms;
  const auto tc = clk::now();
  ensure_sets(ctx, R_new);
  // own share, compacted in sample-id order (offsets relative to the share)
  uint64_t* d_off = nullptr;
  uint32_t* d_mem = nullptr;
  const uint64_t my_total = compact_range(ctx, lo, hi - lo, &d_off, &d_mem);
  const int W = ctx->world;
  ex.counts.reserve(2 * W * sizeof(uint64_t), false, s);
  uint64_t* d_counts = ex.counts.as<uint64_t>();
  EIM_CUDA(cudaMemcpyAsync(d_counts, &my_total, sizeof(uint64_t), cudaMemcpyHostToDevice, s));
  comm_allgather_u64(ctx->comm, d_counts, d_counts + W, s);
  std::vector<uint64_t> totals(W);
  EIM_CUDA(cudaMemcpyAsync(totals.data(), d_counts + W, W * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  EIM_CUDA(cudaStreamSynchronize(s));
  uint64_t max_total = 1, max_sets = 1;
  for (int q = 0; q < W; ++q) {
    uint64_t a, b;
    eim_shard_range(R, R_new - R, q, W, &a, &b);
    max_total = std::max(max_total, totals[q]);
    max_sets = std::max(max_sets, b - a + 1);
  }
  ex.offs_recv.reserve(max_sets * sizeof(uint64_t), false, s);
  ex.mem_recv.reserve(max_total * sizeof(uint32_t), false, s);
  for (int q = 0; q < W; ++q) {
    uint64_t a, b;
    eim_shard_range(R, R_new - R, q, W, &a, &b);
    if (b == a) continue;
    uint64_t* offs = (q == ctx->rank) ? d_off : ex.offs_recv.as<uint64_t>();
    uint32_t* mem = (q == ctx->rank) ? d_mem : ex.mem_recv.as<uint32_t>();
    comm_group_start();
    comm_broadcast(ctx->comm, offs, (b - a + 1) * sizeof(uint64_t), q, s);
    if (totals[q]) comm_broadcast(ctx->comm, mem, totals[q] * sizeof(uint32_t), q, s);
    comm_group_end();
    if (q != ctx->rank) append_sets(ctx, a, b - a, offs, mem, totals[q]);
  }
  hist_sets(ctx, R, R_new);
  EIM_CUDA(cudaStreamSynchronize(s));
  st->ms_comm += ms_since(tc);
  st->ms_sample += ms_since(t0);
}

// Supplies the sets of sample ids [|R|, to) to the arena.  On one GPU the
// next round's ids [to, next_to) are launched SPECULATIVELY on a second
// stream right behind the current round's launch: its blocks take the SMs
// that the current round's tail (its last, longest reverse-BFS chains)
// leaves idle.  While the greedy of the current round runs, the speculative
// round is paused (it takes no new ids, so the greedy has the GPU); it is
// resumed when its ids are needed, or cancelled when they are not.  Sample
// ids are fixed labels, so a speculative set is exactly the set the next
// round needs and results are unchanged.
//
// Source elimination (R22, elim = true): sets are the non-empty root-less
// sets in sample-id order; a round launches enough ids for the sets still
// needed (from the kept fraction so far), keeps the first of them and
// continues from the id after the last kept one.
class RoundSampler {
 public:
  RoundSampler(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, eim_stats* st, bool elim)
      : ctx_(ctx), g_(g), model_(model), seed_(seed), st_(st), elim_(elim) {
    // opt-in (EIM_SPECULATE=1): measured on C2 the speculative round slows the
    // current round's critical chains as much as it fills their idle SMs
    speculate_ = ctx->world == 1 && !elim && std::getenv("EIM_SPECULATE") != nullptr;
    // Lookahead (default on, one GPU, plain runs): when the next round adds no
    // more ids than this one, one launch samples both and the next round's
    // sets are appended from the same round table without a launch -- one
    // round tail (the heavy samples' critical paths) instead of two.  Sample
    // ids are fixed labels, so the sets are the same; if the estimation loop
    // stops first, the extra sets are discarded.  EIM_NO_LOOKAHEAD=1: off.
    lookahead_ = ctx->world == 1 && !elim && !speculate_ && std::getenv("EIM_NO_LOOKAHEAD") == nullptr;
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

  // make sets [R, to) final; speculate [to, next_to)
  void grow(uint64_t& R, uint64_t to, uint64_t next_to) {
    if (to <= R) return;
    const auto t0 = clk::now();
    if (elim_) {
      grow_elim(R, to);
      st_->ms_sample += ms_since(t0);
      return;
    }
    st_->ids_sampled += to - R;
    if (ctx_->world > 1) {
      sample_round(ctx_, g_, model_, seed_, id_base_, R, to, st_, ex_);
      R = to;
      return;
    }
    if (lookahead_) {
      grow_lookahead(R, to, next_to);
      st_->ms_sample += ms_since(t0);
      return;
    }
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
    if (speculate_ && next_to > cur_end) {
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
    st_->edges_examined += r.edges;
    st_->spilled_samples += r.spilled;
    st_->sample_launches += r.launches;
    st_->ms_sample_kernel += r.kernel_ms;
  }
  // The held launch covers ids id_base_ + [held_first_, held_end_); sets
  // [held_first_, held_done_) are appended.
  void grow_lookahead(uint64_t& R, uint64_t to, uint64_t next_to) {
    Round& rd = ctx_->rounds[0];
    if (held_) {
      if (held_done_ == R) {
        const uint64_t upto = std::min(held_end_, to);
        const bool keep = upto < held_end_;
        account(round_finalize(ctx_, g_, rd, upto - held_first_, held_done_ - held_first_, keep));
        R = held_done_ = upto;
        if (!keep) held_ = false;
      } else {
        drop_held();
      }
    }
    if (to <= R) return;
    drop_held();
    const uint64_t end = (next_to > to && next_to - to <= to - R) ? next_to : to;
    round_launch(ctx_, g_, model_, seed_, id_base_ + R, end - R, id_base_, true, rd, stream_of(rd), false);
    const bool keep = end > to;
    account(round_finalize(ctx_, g_, rd, to - R, 0, keep));
    if (keep) {
      held_ = true;
      held_first_ = R;
      held_done_ = to;
      held_end_ = end;
    }
    R = to;
  }

  // Discard the rest of a held launch (the loop stopped or moved on).
  void drop_held() {
    if (!held_) return;
    Round& rd = ctx_->rounds[0];
    rd.launched = false;
    rd.waited = false;
    held_ = false;
  }

  void grow_elim(uint64_t& R, uint64_t to) {
    while (R < to) {
      const uint64_t need = to - R;
      // kept fraction so far (first launch: 1/4), 5% + 64 ids of slack
      const double q = consumed_ ? std::max(1e-6, (double)std::max<uint64_t>(kept_, 1) / (double)consumed_) : 0.25;
      const double want = std::ceil((double)need / q * 1.05) + 64.0;
      const uint64_t count = (uint64_t)std::min(want, (double)(1ull << 29));
      if (next_id_ + count > (1ull << 62)) fail(EIM_E_INVAL, "sample ids exhausted (< 2^62)");
      Round& rd = ctx_->rounds[0];
      round_launch(ctx_, g_, model_, seed_, next_id_, count, next_id_ - R, true, rd, stream_of(rd), false,
                   RF_DROP_ROOT | RF_DROP_EMPTY);
      const SampleResult r = round_finalize(ctx_, g_, rd, need);
      account(r);
      R += r.kept;
      next_id_ += r.consumed;
      kept_ += r.kept;
      consumed_ += r.consumed;
      st_->ids_sampled += r.consumed;
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
  uint64_t kept_ = 0, consumed_ = 0;  // kept sets / ids used so far (source elimination)
  Exchange ex_;
  bool speculate_ = false;
  Round* spec_ = nullptr;
  bool lookahead_ = false, held_ = false;
  uint64_t held_first_ = 0, held_done_ = 0, held_end_ = 0;
};

}  // namespace

void imm_run(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell, eim_model model,
             uint64_t seed, uint32_t flags, uint32_t* seeds_out, uint64_t* theta_out, double* spread_out,
             eim_stats* st) {
  const auto t_start = clk::now();
  const uint32_t n = g->view.n;
  const bool elim = (flags & EIM_F_SOURCE_ELIM) != 0, fresh = (flags & EIM_F_FRESH_FINAL) != 0;
  if (elim && ctx->world > 1) fail(EIM_E_INVAL, "EIM_F_SOURCE_ELIM needs a single-GPU context");
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
  ctx->C_total.reserve((uint64_t)n * sizeof(uint32_t), false, s);
  EIM_CUDA(cudaMemsetAsync(ctx->C_total.p, 0, (uint64_t)n * sizeof(uint32_t), s));
  RoundSampler sampler(ctx, g, model, seed, st, elim);
  std::vector<uint32_t> S(k);
  uint64_t R = 0, cov = 0;
  uint64_t R_selected = UINT64_MAX;  // |R| the last NodeSelection ran on
  double LB = 1.0;
  auto theta_round = [&](uint32_t i) { return (uint64_t)std::ceil(std::ldexp(p.lambda_p, (int)i) / (double)n); };
  try {
    for (uint32_t i = 1; (double)i < p.log2n; ++i) {
      const uint64_t next = (double)(i + 1) < p.log2n ? theta_round(i + 1) : 0;
      sampler.grow(R, theta_round(i), next);
      const auto ts = clk::now();
      cov = greedy(ctx, n, R, k, S.data(), nullptr);
      st->ms_select += ms_since(ts);
      R_selected = R;
      if (st->rounds < 64) {
        st->theta_i[st->rounds] = R;
        st->cov_i[st->rounds] = cov;
      }
      st->rounds++;
      if ((double)cov * std::ldexp(1.0, (int)i) >= (1.0 + p.eps_p) * (double)R) {
        LB = ((double)n * (double)cov) / ((1.0 + p.eps_p) * (double)R);
        break;
      }
    }
    st->lb = LB;
    const uint64_t theta = (uint64_t)std::ceil(p.lambda_s / LB);
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
    cov = greedy(ctx, n, R, k, S.data(), nullptr);
    st->ms_select += ms_since(ts);
  }
  std::memcpy(seeds_out, S.data(), (size_t)k * sizeof(uint32_t));
  st->theta = R;
  st->cov = cov;
  st->arena_elems = arena_cursor(ctx);
  st->arena_bytes = ctx->arena_b == 32 ? 4 * st->arena_elems : 4 * arena_words(st->arena_elems, ctx->arena_b);
  if (theta_out) *theta_out = R;
  if (spread_out) *spread_out = (double)n * (double)cov / (double)R;
  st->kernel_launches = ctx->kernel_launches - launches0;
  st->ms_total = ms_since(t_start);
}

}  // namespace eim
