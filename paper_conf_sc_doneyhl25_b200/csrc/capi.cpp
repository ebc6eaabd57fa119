// capi.cpp -- the extern "C" boundary declared in include/eim.h: argument
// validation, error capture (no exception crosses the ABI), object lifetime.
#include <chrono>
#include <cstring>
#include <mutex>
#include <vector>

#include "eim_internal.h"

namespace eim {

void fail(eim_status code, const std::string& msg) { throw Error{code, msg}; }

void cuda_check(cudaError_t e, const char* what, const char* file, int line) {
  if (e == cudaSuccess) return;
  const eim_status code = (e == cudaErrorMemoryAllocation) ? EIM_E_NOMEM : EIM_E_CUDA;
  cudaGetLastError();  // clear sticky-free errors
  fail(code, std::string(cudaGetErrorString(e)) + " in " + what + " (" + file + ":" + std::to_string(line) + ")");
}

// Stream-ordered allocation (cudaMallocAsync / cudaFreeAsync): growing a
// buffer never synchronises the device, so a speculative sampler running on
// another stream keeps running while the main stream reallocates.
void DevBuf::reserve(size_t need, bool keep, cudaStream_t st) {
  if (need <= bytes) return;
  size_t nb = std::max(need, bytes + bytes / 2);
  nb = (nb + 255) & ~size_t(255);
  void* q = nullptr;
  cudaError_t e = cudaMallocAsync(&q, nb, st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    nb = (need + 255) & ~size_t(255);
    e = cudaMallocAsync(&q, nb, st);
    if (e != cudaSuccess) {
      cudaGetLastError();
      fail(EIM_E_NOMEM, "cudaMallocAsync of " + std::to_string(nb) + " bytes failed");
    }
  }
  if (keep && p && bytes) EIM_CUDA(cudaMemcpyAsync(q, p, bytes, cudaMemcpyDeviceToDevice, st));
  if (p) EIM_CUDA(cudaFreeAsync(p, st));
  p = q;
  bytes = nb;
}

void DevBuf::release() {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = 0;
}

void GreedySlot::release() {
  DevBuf* b[] = {&C_work, &inv_off, &inv_fill, &inv, &best, &seeds, &gains, &cand, &cidx, &arena_c, &selected, &covered,
                 &scratch, &dirty};
  for (DevBuf* x : b) x->release();
  for (cudaEvent_t& e : ev) {
    if (e) cudaEventDestroy(e);
    e = nullptr;
  }
  if (own_stream && stream) {
    cudaStreamSynchronize(stream);
    cudaStreamDestroy(stream);
  }
  stream = nullptr;
  own_stream = false;
}

}  // namespace eim

using namespace eim;

namespace {

std::mutex g_err_mu;
std::string g_err;  // errors with no context

void set_global_error(const std::string& m) {
  std::lock_guard<std::mutex> lk(g_err_mu);
  g_err = m;
}

template <class F>
eim_status guarded(eim_ctx* ctx, F&& f) {
  try {
    if (ctx) {
      EIM_CUDA(cudaSetDevice(ctx->device));
      ctx->last_error.clear();
    }
    f();
    return EIM_OK;
  } catch (const Error& e) {
    if (ctx) ctx->last_error = e.msg;
    else set_global_error(e.msg);
    return e.code;
  } catch (const std::bad_alloc&) {
    if (ctx) ctx->last_error = "host allocation failed";
    else set_global_error("host allocation failed");
    return EIM_E_NOMEM;
  } catch (...) {
    if (ctx) ctx->last_error = "unknown error";
    else set_global_error("unknown error");
    return EIM_E_CUDA;
  }
}

bool ctx_ok(const eim_ctx* ctx) { return ctx && ctx->magic == CTX_MAGIC; }

void free_ctx_buffers(eim_ctx* c) {
  DevBuf* bufs[] = {&c->arena, &c->set_start, &c->set_len, &c->ctl, &c->C_total, &c->C_snap, &c->C_snap2, &c->edges_acc,
                    &c->scratch,
                    &c->stage_a, &c->stage_b, &c->stage_c};
  for (DevBuf* b : bufs) b->release();
  for (GreedySlot& g : c->gs) g.release();
  for (Round& r : c->rounds) round_release(r);
}

}  // namespace

extern "C" {

const char* eim_version(void) { return "eim-b200 0.1 (sm_100a)"; }

const char* eim_last_error(const eim_ctx* ctx) {
  if (ctx_ok(ctx)) return ctx->last_error.c_str();
  std::lock_guard<std::mutex> lk(g_err_mu);
  return g_err.c_str();
}

eim_status eim_nccl_get_id(void* out) {
  return guarded(nullptr, [&] {
    if (!out) fail(EIM_E_INVAL, "out is NULL");
    comm_get_id(out);
  });
}

}  // extern "C"

namespace {

// A context on `device`; the communicator is made by make_comm (world > 1).
template <class MakeComm>
eim_ctx* new_ctx(int device, int rank, int world, uint64_t stream, MakeComm&& make_comm) {
  int ndev = 0;
  EIM_CUDA(cudaGetDeviceCount(&ndev));
  if (device >= ndev) fail(EIM_E_INVAL, "device index out of range");
  EIM_CUDA(cudaSetDevice(device));
  eim_ctx* c = new eim_ctx();
  c->magic = CTX_MAGIC;
  c->device = device;
  c->rank = rank;
  c->world = world;
  c->comm = nullptr;
  c->kernel_launches = 0;
  c->own_stream = stream == 0;
  try {
    if (c->own_stream) EIM_CUDA(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
    else c->stream = reinterpret_cast<cudaStream_t>(stream);
    EIM_CUDA(cudaStreamCreateWithFlags(&c->rstream[0], cudaStreamNonBlocking));
    EIM_CUDA(cudaStreamCreateWithFlags(&c->rstream[1], cudaStreamNonBlocking));
    EIM_CUDA(cudaStreamCreateWithFlags(&c->aux_stream, cudaStreamNonBlocking));
    c->gs[0].stream = c->stream;
    for (int q = 1; q < 3; ++q) {
      EIM_CUDA(cudaStreamCreateWithFlags(&c->gs[q].stream, cudaStreamNonBlocking));
      c->gs[q].own_stream = true;
    }
    EIM_CUDA(cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, device));
    // keep freed stream-ordered memory in the device's pool: reloading a
    // graph or regrowing a buffer reuses it instead of cudaMalloc/cudaFree
    cudaMemPool_t pool;
    EIM_CUDA(cudaDeviceGetDefaultMemPool(&pool, device));
    uint64_t keep_all = UINT64_MAX;
    EIM_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep_all));
    EIM_CUDA(cudaMallocHost(&c->h_pinned, 4096));
    EIM_CUDA(cudaEventCreate(&c->ev0));
    EIM_CUDA(cudaEventCreate(&c->ev1));
    c->scratch.reserve(1 << 20, false, c->stream);
    if (world > 1) c->comm = make_comm();
  } catch (...) {
    free_ctx_buffers(c);
    if (c->h_pinned) cudaFreeHost(c->h_pinned);
    if (c->own_stream && c->stream) cudaStreamDestroy(c->stream);
    c->magic = 0;
    delete c;
    throw;
  }
  return c;
}

}  // namespace

extern "C" {

eim_status eim_create(int device, int rank, int world, const void* nccl_id, uint64_t stream, eim_ctx** out) {
  return guarded(nullptr, [&] {
    if (!out) fail(EIM_E_INVAL, "out is NULL");
    *out = nullptr;
    if (device < 0) fail(EIM_E_INVAL, "device < 0");
    if (world < 1 || rank < 0 || rank >= world) fail(EIM_E_INVAL, "rank/world out of range");
    if (world > 1 && !nccl_id) fail(EIM_E_INVAL, "world > 1 needs an NCCL unique id");
    *out = new_ctx(device, rank, world, stream, [&] { return comm_create(rank, world, nccl_id); });
  });
}

eim_status eim_create_group(const int* devices, int world, eim_ctx** out) {
  return guarded(nullptr, [&] {
    if (!out || !devices) fail(EIM_E_INVAL, "NULL argument");
    if (world < 1) fail(EIM_E_INVAL, "world < 1");
    for (int r = 0; r < world; ++r) {
      out[r] = nullptr;
      if (devices[r] < 0) fail(EIM_E_INVAL, "device < 0");
    }
    LocalGroup* grp = world > 1 ? local_group_new(world) : nullptr;
    int made = 0;
    try {
      for (int r = 0; r < world; ++r) {
        out[r] = new_ctx(devices[r], r, world, 0, [&] { return comm_create_local(grp, r); });
        made++;
      }
    } catch (...) {
      for (int r = 0; r < made; ++r) {
        eim_destroy(out[r]);
        out[r] = nullptr;
      }
      if (grp && made == 0) delete_local_group(grp);
      throw;
    }
  });
}

void eim_destroy(eim_ctx* ctx) {
  if (!ctx_ok(ctx)) return;
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->stream);
  comm_destroy(ctx->comm);
  free_ctx_buffers(ctx);
  cudaFreeHost(ctx->h_pinned);
  cudaMemPool_t pool;  // hand the pooled memory back
  if (cudaDeviceGetDefaultMemPool(&pool, ctx->device) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
  cudaEventDestroy(ctx->ev0);
  cudaEventDestroy(ctx->ev1);
  for (cudaStream_t rs : ctx->rstream) {
    cudaStreamSynchronize(rs);
    cudaStreamDestroy(rs);
  }
  cudaStreamDestroy(ctx->aux_stream);
  if (ctx->own_stream) cudaStreamDestroy(ctx->stream);
  ctx->magic = 0;
  delete ctx;
}

eim_status eim_load_graph_csr(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                              const uint32_t* in_neighbors, eim_graph** out) {
  return eim_load_graph_csr_ex(ctx, n, m, in_offsets, in_neighbors, 0u, out);
}

eim_status eim_load_graph_csr_ex(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                                 const uint32_t* in_neighbors, uint32_t gflags, eim_graph** out) {
  return eim_load_graph_csr_weighted(ctx, n, m, in_offsets, in_neighbors, nullptr, gflags, out);
}

eim_status eim_load_graph_csr_weighted(eim_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* in_offsets,
                                       const uint32_t* in_neighbors, const uint32_t* edge_x, uint32_t gflags,
                                       eim_graph** out) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  return guarded(ctx, [&] {
    if (!out) fail(EIM_E_INVAL, "out is NULL");
    if (gflags & ~(uint32_t)EIM_G_LOG_ENCODE) fail(EIM_E_INVAL, "unknown graph flag");
    *out = nullptr;
    if (n < 2 || n >= 0xFFFFFFFFu) fail(EIM_E_INVAL, "n must be in [2, 2^32-1)");
    if (m >= (1ull << 40)) fail(EIM_E_INVAL, "m must be < 2^40");
    if (!in_offsets || (m > 0 && !in_neighbors)) fail(EIM_E_INVAL, "NULL graph array");
    eim_graph* g = new eim_graph();
    g->magic = GRAPH_MAGIC;
    g->ctx = ctx;
    cudaStream_t st = ctx->stream;
    try {
      // stream-ordered from the context's pool (no device-wide sync)
      EIM_CUDA(cudaMallocAsync(&g->d_off, ((uint64_t)n + 1) * sizeof(uint64_t), st));
      EIM_CUDA(cudaMallocAsync(&g->d_nbr, std::max<uint64_t>(m, 4) * sizeof(uint32_t), st));
      EIM_CUDA(cudaMallocAsync(&g->d_thr, (uint64_t)n * sizeof(uint32_t), st));
      EIM_CUDA(cudaMemcpyAsync(g->d_off, in_offsets, ((uint64_t)n + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, st));
      if (m) EIM_CUDA(cudaMemcpyAsync(g->d_nbr, in_neighbors, m * sizeof(uint32_t), cudaMemcpyHostToDevice, st));
      g->view.n = n;
      g->view.m = m;
      g->view.off = static_cast<const uint64_t*>(g->d_off);
      g->view.nbr = static_cast<const uint32_t*>(g->d_nbr);
      g->view.thr = static_cast<const uint32_t*>(g->d_thr);
      graph_validate_and_thresholds(ctx, g);
      g->bytes = ((uint64_t)n + 1) * sizeof(uint64_t) + std::max<uint64_t>(m, 4) * sizeof(uint32_t) +
                 (uint64_t)n * sizeof(uint32_t);
      if (edge_x) graph_attach_weights(ctx, g, edge_x);  // (its LT scan reads the plain offsets)
      if (gflags & EIM_G_LOG_ENCODE) graph_log_encode(ctx, g);
    } catch (...) {
      if (g->d_off) cudaFreeAsync(g->d_off, st);
      if (g->d_nbr) cudaFreeAsync(g->d_nbr, st);
      if (g->d_thr) cudaFreeAsync(g->d_thr, st);
      if (g->d_offw) cudaFreeAsync(g->d_offw, st);
      if (g->d_x) cudaFreeAsync(g->d_x, st);
      if (g->d_cum) cudaFreeAsync(g->d_cum, st);
      if (g->d_nbrw) cudaFreeAsync(g->d_nbrw, st);
      cudaStreamSynchronize(st);
      g->magic = 0;
      delete g;
      throw;
    }
    *out = g;
  });
}

eim_status eim_graph_free(eim_graph* g) {
  if (!g || g->magic != GRAPH_MAGIC) return EIM_E_STATE;
  eim_ctx* ctx = g->ctx;
  if (ctx_ok(ctx)) {
    // every kernel that reads the graph has finished when a hot-path call
    // returns (the calls end synchronised), so the free is stream-ordered
    cudaSetDevice(ctx->device);
    for (void* p : {g->d_off, g->d_nbr, g->d_thr, g->d_offw, g->d_nbrw, g->d_x, g->d_cum, g->d_aug})
      if (p) cudaFreeAsync(p, ctx->stream);
    cudaStreamSynchronize(ctx->stream);
  } else {
    for (void* p : {g->d_off, g->d_nbr, g->d_thr, g->d_offw, g->d_nbrw, g->d_x, g->d_cum, g->d_aug})
      if (p) cudaFree(p);
  }
  g->magic = 0;
  delete g;
  return EIM_OK;
}

eim_status eim_graph_bytes(const eim_graph* g, uint64_t* bytes) {
  if (!g || g->magic != GRAPH_MAGIC) return EIM_E_STATE;
  if (!bytes) return EIM_E_INVAL;
  *bytes = g->bytes;
  return EIM_OK;
}

static void check_graph(eim_ctx* ctx, const eim_graph* g) {
  if (!g || g->magic != GRAPH_MAGIC) fail(EIM_E_STATE, "graph is freed or invalid");
  if (g->ctx != ctx) fail(EIM_E_STATE, "graph belongs to another context");
}

eim_status eim_imm_run(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell, eim_model model,
                       uint64_t seed, uint32_t* seeds_out, uint64_t* theta_out, double* spread_out,
                       eim_stats* stats_out) {
  return eim_imm_run_ex(ctx, g, k, eps, ell, model, seed, 0u, seeds_out, theta_out, spread_out, stats_out);
}

eim_status eim_imm_run_ex(eim_ctx* ctx, const eim_graph* g, uint32_t k, double eps, double ell, eim_model model,
                          uint64_t seed, uint32_t flags, uint32_t* seeds_out, uint64_t* theta_out,
                          double* spread_out, eim_stats* stats_out) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  return guarded(ctx, [&] {
    try {
      check_graph(ctx, g);
      if (flags & ~(uint32_t)(EIM_F_SOURCE_ELIM | EIM_F_FRESH_FINAL)) fail(EIM_E_INVAL, "unknown flag");
      if (!seeds_out) fail(EIM_E_INVAL, "seeds_out is NULL");
      if (k == 0 || k > g->view.n) fail(EIM_E_INVAL, "k must be in [1, n]");
      if (!(eps > 0.0 && eps < 1.0)) fail(EIM_E_INVAL, "eps must be in (0, 1)");
      if (!(ell > 0.0)) fail(EIM_E_INVAL, "ell must be > 0");
      if (model != EIM_IC && model != EIM_LT) fail(EIM_E_INVAL, "unknown model");
      if (model == EIM_LT && !g->lt_ok) fail(EIM_E_INVAL, "LT: a row's edge weights sum to more than 1");
      ctx->cov_n = 0;
      imm_run(ctx, g, k, eps, ell, model, seed, flags, seeds_out, theta_out, spread_out, &ctx->last_stats);
    } catch (...) {
      // a collective call: release the peers of a local group (they would
      // wait for this rank forever); the group cannot be used afterwards
      if (ctx->comm) ctx->comm->abort();
      throw;
    }
    ctx->cov_n = g->view.n;
    if (stats_out) *stats_out = ctx->last_stats;
  });
}

eim_status eim_sample_rrr(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, uint64_t first_id,
                          uint64_t count, uint64_t* offsets_out, uint32_t* members_out, uint64_t members_cap,
                          uint64_t* members_total) {
  return eim_sample_rrr_ex(ctx, g, model, seed, first_id, count, 0u, offsets_out, members_out, members_cap,
                           members_total);
}

eim_status eim_sample_rrr_ex(eim_ctx* ctx, const eim_graph* g, eim_model model, uint64_t seed, uint64_t first_id,
                             uint64_t count, uint32_t flags, uint64_t* offsets_out, uint32_t* members_out,
                             uint64_t members_cap, uint64_t* members_total) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  eim_status cap_status = EIM_OK;
  eim_status s = guarded(ctx, [&] {
    check_graph(ctx, g);
    if (flags & ~(uint32_t)EIM_F_SOURCE_ELIM) fail(EIM_E_INVAL, "unknown flag");
    if (!offsets_out || !members_total) fail(EIM_E_INVAL, "NULL output");
    if (model != EIM_IC && model != EIM_LT) fail(EIM_E_INVAL, "unknown model");
    if (model == EIM_LT && !g->lt_ok) fail(EIM_E_INVAL, "LT: a row's edge weights sum to more than 1");
    if (first_id + count < first_id || first_id + count > (1ull << 62)) fail(EIM_E_INVAL, "sample ids must be < 2^62");
    cudaStream_t st = ctx->stream;
    const auto t0 = std::chrono::steady_clock::now();
    const uint64_t launches0 = ctx->kernel_launches;
    ctx->cov_n = 0;
    arena_reset(ctx, g->packed ? bit_width((uint64_t)g->view.n - 1) : 32u);
    edges_reset(ctx);
    const SampleResult r = sample_range(ctx, g, model, seed, first_id, count, first_id, false,
                                        (flags & EIM_F_SOURCE_ELIM) ? RF_DROP_ROOT : 0u);
    std::memset(&ctx->last_stats, 0, sizeof(eim_stats));
    ctx->last_stats.edges_examined = edges_read(ctx);
    ctx->last_stats.spilled_samples = r.spilled;
    ctx->last_stats.sample_launches = r.launches;
    ctx->last_stats.ms_sample_kernel = r.kernel_ms;
    ctx->last_stats.theta = count;
    ctx->last_stats.ids_sampled = count;
    ctx->last_stats.ms_sample = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    uint64_t* d_off = nullptr;
    uint32_t* d_mem = nullptr;
    const uint64_t total = export_sets(ctx, count, &d_off, &d_mem, members_cap);
    *members_total = total;
    EIM_CUDA(cudaMemcpyAsync(offsets_out, d_off, (count + 1) * sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    if (total > members_cap) {
      EIM_CUDA(cudaStreamSynchronize(st));
      ctx->last_error = "members_cap too small";
      cap_status = EIM_E_CAPACITY;
      return;
    }
    if (total) {
      if (!members_out) fail(EIM_E_INVAL, "members_out is NULL");
      EIM_CUDA(cudaMemcpyAsync(members_out, d_mem, total * sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    }
    EIM_CUDA(cudaStreamSynchronize(st));
    ctx->last_stats.arena_elems = total;
    ctx->last_stats.kernel_launches = ctx->kernel_launches - launches0;
    ctx->last_stats.ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  });
  return s != EIM_OK ? s : cap_status;
}

eim_status eim_select_seeds(eim_ctx* ctx, uint32_t n, uint64_t num_sets, const uint64_t* offsets,
                            const uint32_t* members, uint32_t k, uint32_t* seeds_out, uint64_t* gains_out) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  return guarded(ctx, [&] {
    if (n < 1 || n >= 0xFFFFFFFFu) fail(EIM_E_INVAL, "n must be in [1, 2^32-1)");
    if (k == 0 || k > n) fail(EIM_E_INVAL, "k must be in [1, n]");
    if (!offsets || !seeds_out) fail(EIM_E_INVAL, "NULL argument");
    if (offsets[0] != 0) fail(EIM_E_INVAL, "offsets[0] != 0");
    for (uint64_t i = 0; i < num_sets; ++i)
      if (offsets[i + 1] < offsets[i]) fail(EIM_E_INVAL, "offsets not non-decreasing");
    if (num_sets >= (1ull << 32)) fail(EIM_E_INVAL, "at most 2^32 - 1 sets");
    const uint64_t total = offsets[num_sets];
    if (total && !members) fail(EIM_E_INVAL, "members is NULL");
    // members < n and distinct within each set (a duplicate would count a
    // set twice in C and corrupt the gains): stamp[v] = last set index + 1
    std::vector<uint32_t> stamp(n, 0u);
    for (uint64_t i = 0; i < num_sets; ++i)
      for (uint64_t j = offsets[i]; j < offsets[i + 1]; ++j) {
        const uint32_t v = members[j];
        if (v >= n) fail(EIM_E_INVAL, "member id >= n");
        if (stamp[v] == (uint32_t)(i + 1)) fail(EIM_E_INVAL, "duplicate member within a set");
        stamp[v] = (uint32_t)(i + 1);
      }
    cudaStream_t st = ctx->stream;
    ctx->cov_n = 0;
    arena_reset(ctx);
    ctx->stage_a.reserve((num_sets + 1) * sizeof(uint64_t), false, st);
    ctx->stage_b.reserve(std::max<uint64_t>(total, 1) * sizeof(uint32_t), false, st);
    EIM_CUDA(cudaMemcpyAsync(ctx->stage_a.p, offsets, (num_sets + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, st));
    if (total) EIM_CUDA(cudaMemcpyAsync(ctx->stage_b.p, members, total * sizeof(uint32_t), cudaMemcpyHostToDevice, st));
    ctx->C_total.reserve((uint64_t)n * sizeof(uint32_t), false, st);
    EIM_CUDA(cudaMemsetAsync(ctx->C_total.p, 0, (uint64_t)n * sizeof(uint32_t), st));
    append_sets(ctx, 0, num_sets, ctx->stage_a.as<uint64_t>(), ctx->stage_b.as<uint32_t>(), total);
    hist_sets(ctx, 0, num_sets);
    const auto t0 = std::chrono::steady_clock::now();
    double kms = 0;
    const uint64_t cov = greedy(ctx, n, num_sets, k, seeds_out, gains_out, &kms);
    std::memset(&ctx->last_stats, 0, sizeof(eim_stats));
    ctx->last_stats.ms_select_kernel = kms;
    ctx->last_stats.select_launches = 1;
    ctx->last_stats.select_picks = k;
    ctx->last_stats.cov = cov;
    ctx->last_stats.theta = num_sets;
    ctx->last_stats.arena_elems = total;
    ctx->last_stats.ms_select = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    ctx->cov_n = n;
  });
}

eim_status eim_get_coverage(eim_ctx* ctx, uint32_t n, uint32_t* C_out) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  return guarded(ctx, [&] {
    if (ctx->cov_n == 0) fail(EIM_E_STATE, "no coverage counts: run eim_imm_run or eim_select_seeds first");
    if (!C_out) fail(EIM_E_INVAL, "C_out is NULL");
    if (n != ctx->cov_n) fail(EIM_E_INVAL, "n differs from the vertex count of the last call");
    EIM_CUDA(cudaMemcpyAsync(C_out, ctx->C_total.p, (uint64_t)n * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                             ctx->stream));
    EIM_CUDA(cudaStreamSynchronize(ctx->stream));
  });
}

eim_status eim_get_stats(const eim_ctx* ctx, eim_stats* out) {
  if (!ctx_ok(ctx)) return EIM_E_STATE;
  if (!out) return EIM_E_INVAL;
  *out = ctx->last_stats;
  return EIM_OK;
}

eim_status eim_imm_params(uint32_t n, uint32_t k, double eps, double ell, eim_imm_params_t* out) {
  return guarded(nullptr, [&] {
    if (!out) fail(EIM_E_INVAL, "out is NULL");
    if (n < 2 || k == 0 || k > n || !(eps > 0.0 && eps < 1.0) || !(ell > 0.0))
      fail(EIM_E_INVAL, "invalid IMM parameters");
    imm_params(n, k, eps, ell, out);
  });
}

eim_status eim_shard_range(uint64_t first, uint64_t count, int rank, int world, uint64_t* lo, uint64_t* hi) {
  if (world < 1 || rank < 0 || rank >= world || !lo || !hi) return EIM_E_INVAL;
  const unsigned __int128 c = count;
  *lo = first + (uint64_t)(c * (unsigned)rank / (unsigned)world);
  *hi = first + (uint64_t)(c * (unsigned)(rank + 1) / (unsigned)world);
  return EIM_OK;
}

}  // extern "C"
