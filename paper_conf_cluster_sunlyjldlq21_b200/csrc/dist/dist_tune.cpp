// dist_tune.cpp — population-parallel evaluation of the csTuner GA (the
// paper's multi-process GA: "the operations of each sub-population are handled by a
// process").  Rank 0 runs cst_tune (tuner.cpp) with an internal evaluation callback; each
// batch of candidates it asks for — the dataset, the noise re-evaluations and every
// GA generation of 2 x 16 individuals — is broadcast to all ranks, rank k evaluates
// the candidates i with i % nranks == k on its own GPU, and the per-rank fitness / metric
// vectors are all-gathered and merged.  The other ranks serve batches until rank 0 sends
// the end marker, then everyone receives rank 0's result (always sent, success or not).
//
// Messages (all from rank 0, fixed layouts):
//   header   int64 n            n >= 0: a batch of n settings follows; -1: tuning ended
//   batch    n x cst_setting
//   gather   per rank n x double ms (NaN = not mine) + n x n_user_metrics doubles
//   result   Result (status, best setting, report, error text)
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstring>
#include <thread>

#include "dist_internal.h"

using namespace cst;

namespace {

struct Result {
  int32_t status;
  cst_setting best;
  cst_tune_report rep;
  char err[512];
};

#ifdef CST_HAVE_NCCL
cst_status nccl_ok(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return CST_OK;
  return fail(CST_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}
#endif

// Transport: host collectives (caller's) or NCCL with a device staging buffer.
struct Comm {
  cst_dist* D;
  void* dev = nullptr;
  size_t dev_bytes = 0;
  ~Comm() {
    if (dev) cudaFree(dev);
  }
  cst_status staging(size_t bytes) {
    if (bytes <= dev_bytes) return CST_OK;
    if (dev) cudaFree(dev);
    dev = nullptr;
    if (cudaMalloc(&dev, bytes) != cudaSuccess) {
      cudaGetLastError();
      dev_bytes = 0;
      return fail(CST_E_OOM, "cst_dist_tune: NCCL staging buffer");
    }
    dev_bytes = bytes;
    return CST_OK;
  }
  cst_status bcast(void* buf, int64_t bytes) {
    if (D->nranks == 1) return CST_OK;
    if (D->has_coll) {
      if (D->coll.bcast(D->coll.user, buf, bytes, 0) != 0)
        return fail(CST_E_INTERNAL, "cst_dist_tune: broadcast callback failed");
      return CST_OK;
    }
#ifdef CST_HAVE_NCCL
    cst_status st = staging((size_t)bytes);
    if (st != CST_OK) return st;
    CST_CUDA(cudaMemcpyAsync(dev, buf, bytes, cudaMemcpyHostToDevice, D->s_comm));
    st = nccl_ok(ncclBroadcast(dev, dev, (size_t)bytes, ncclChar, 0, D->comm, D->s_comm),
                 "ncclBroadcast");
    if (st != CST_OK) return st;
    CST_CUDA(cudaMemcpyAsync(buf, dev, bytes, cudaMemcpyDeviceToHost, D->s_comm));
    CST_CUDA(cudaStreamSynchronize(D->s_comm));
    return CST_OK;
#else
    return fail(CST_E_UNSUPPORTED, "cst_dist_tune: no collectives (libcst built without NCCL)");
#endif
  }
  cst_status allgather(const void* send, void* recv, int64_t bytes) {
    if (D->nranks == 1) {
      std::memcpy(recv, send, (size_t)bytes);
      return CST_OK;
    }
    if (D->has_coll) {
      if (D->coll.allgather(D->coll.user, send, recv, bytes) != 0)
        return fail(CST_E_INTERNAL, "cst_dist_tune: all-gather callback failed");
      return CST_OK;
    }
#ifdef CST_HAVE_NCCL
    const size_t total = (size_t)bytes * D->nranks;
    cst_status st = staging(total + (size_t)bytes);
    if (st != CST_OK) return st;
    char* sendd = (char*)dev + total;
    CST_CUDA(cudaMemcpyAsync(sendd, send, bytes, cudaMemcpyHostToDevice, D->s_comm));
    st = nccl_ok(ncclAllGather(sendd, dev, (size_t)bytes, ncclChar, D->comm, D->s_comm),
                 "ncclAllGather");
    if (st != CST_OK) return st;
    CST_CUDA(cudaMemcpyAsync(recv, dev, total, cudaMemcpyDeviceToHost, D->s_comm));
    CST_CUDA(cudaStreamSynchronize(D->s_comm));
    return CST_OK;
#else
    (void)send;
    (void)recv;
    return fail(CST_E_UNSUPPORTED, "cst_dist_tune: no collectives (libcst built without NCCL)");
#endif
  }
};

struct Server {
  cst_dist* D;
  Comm* comm;
  const cst_tune_opts* o;
  const double* const* in;
  double* const* out;
  cst_eval_fn local;
  void* local_user;
  cudaStream_t stream = nullptr;

  // evaluate this rank's share of a batch: ms[i] (NaN = not mine), metrics likewise
  void evaluate_share(const cst_setting* ss, int32_t n, std::vector<double>* ms,
                      std::vector<double>* met) {
    const int nm = std::max(0, o->n_user_metrics);
    ms->assign(n, NAN);
    met->assign((size_t)n * nm, NAN);
    std::vector<int32_t> mine;
    for (int32_t i = 0; i < n; ++i)
      if (i % D->nranks == D->rank) mine.push_back(i);
    if (mine.empty()) return;
    std::vector<cst_setting> sub;
    for (int32_t i : mine) sub.push_back(ss[i]);
    std::vector<double> sms(sub.size(), INFINITY), smet(sub.size() * nm, 0.0);
    if (local) {
      if (local(local_user, sub.data(), (int32_t)sub.size(), sms.data(),
                nm > 0 ? smet.data() : nullptr) != 0)
        std::fill(sms.begin(), sms.end(), INFINITY);  // reported as invalid, keep serving
    } else {
      // built-in: code generation of the share on host threads, then CUDA-event timing
      cst_stencil* h = D->h;
      const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
      std::vector<std::thread> pool;
      std::atomic<size_t> next{0};
      for (unsigned w = 0; w < nt; ++w)
        pool.emplace_back([&] {
          for (size_t i = next++; i < sub.size(); i = next++) {
            double cs = 0;
            cst_variant_compile(h, &sub[i], &cs);
          }
        });
      for (auto& th : pool) th.join();
      for (size_t i = 0; i < sub.size(); ++i) {
        if (check_rules(h->info, to_tuple(sub[i])) != nullptr) continue;
        double m = INFINITY;
        if (o->cool_ms > 0) std::this_thread::sleep_for(std::chrono::milliseconds(o->cool_ms));
        if (cst_time_setting(h, &sub[i], in, out, 1, o->warmup, std::max(1, o->reps), stream,
                             &m) == CST_OK)
          sms[i] = m;
      }
    }
    for (size_t k = 0; k < mine.size(); ++k) {
      const double m = sms[k];
      (*ms)[mine[k]] = (m > 0 && std::isfinite(m)) ? m : INFINITY;
      for (int q = 0; q < nm; ++q) (*met)[(size_t)mine[k] * nm + q] = smet[k * nm + q];
    }
  }

  // one batch, all ranks: broadcast (done by the caller on rank 0 for the header), serve,
  // gather and merge into ms / metrics (rank 0 only uses the merged result)
  cst_status round(std::vector<cst_setting>* ss, int64_t n, double* ms_out, double* met_out) {
    const int nm = std::max(0, o->n_user_metrics);
    ss->resize((size_t)n);
    cst_status st = comm->bcast(ss->data(), n * (int64_t)sizeof(cst_setting));
    if (st != CST_OK) return st;
    std::vector<double> ms, met;
    evaluate_share(ss->data(), (int32_t)n, &ms, &met);
    std::vector<double> send(ms);
    send.insert(send.end(), met.begin(), met.end());
    const int64_t per = (int64_t)send.size();
    std::vector<double> recv((size_t)per * D->nranks);
    st = comm->allgather(send.data(), recv.data(), per * (int64_t)sizeof(double));
    if (st != CST_OK) return st;
    if (ms_out)
      for (int64_t i = 0; i < n; ++i) {
        const int k = (int)(i % D->nranks);
        ms_out[i] = recv[(size_t)k * per + i];
        if (met_out)
          for (int q = 0; q < nm; ++q)
            met_out[i * nm + q] = recv[(size_t)k * per + n + i * nm + q];
      }
    return CST_OK;
  }
};

struct Rank0Ctx {
  Server* srv;
  cst_status err = CST_OK;
  std::string msg;
};

int rank0_eval(void* user, const cst_setting* settings, int32_t n, double* ms, double* metrics) {
  Rank0Ctx* c = (Rank0Ctx*)user;
  int64_t hdr = n;
  cst_status st = c->srv->comm->bcast(&hdr, sizeof hdr);
  std::vector<cst_setting> ss(settings, settings + n);
  if (st == CST_OK) st = c->srv->round(&ss, n, ms, metrics);
  if (st != CST_OK) {
    c->err = st;
    c->msg = cst_last_error();
    return 1;
  }
  return 0;
}

}  // namespace

extern "C" cst_status cst_dist_create_host(cst_stencil* h, int32_t nranks, int32_t rank,
                                           const cst_collectives* coll, cst_dist** out) {
  if (!h || !coll || !out || !coll->bcast || !coll->allgather)
    return fail(CST_E_INVALID, "null argument");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail(CST_E_INVALID, "bad nranks / rank");
  auto* D = new cst_dist();
  D->h = h;
  D->nranks = nranks;
  D->rank = rank;
  D->host_only = true;
  D->coll = *coll;
  D->has_coll = true;
  *out = D;
  return CST_OK;
}

extern "C" cst_status cst_dist_tune(cst_dist* D, const cst_tune_opts* o, const double* const* in,
                                    double* const* scratch_out, cst_eval_fn local_eval,
                                    void* local_user, cst_setting* best, cst_tune_report* rep) {
  if (!D || !o || !best || !rep) return fail(CST_E_INVALID, "null argument");
  if (!local_eval && (!in || !scratch_out))
    return fail(CST_E_INVALID, "cst_dist_tune: device buffers required without local_eval");
  if (!local_eval && o->nsteps > 1)
    return fail(CST_E_UNSUPPORTED, "cst_dist_tune: the built-in evaluator times single sweeps "
                                   "(nsteps = 1); pass local_eval for multi-step objectives");
  bool have_nccl = false;
#ifdef CST_HAVE_NCCL
  have_nccl = D->comm != nullptr;
#endif
  if (D->nranks > 1 && !D->has_coll && !have_nccl)
    return fail(CST_E_UNSUPPORTED, "cst_dist_tune needs the NCCL transport (a handle created "
                                   "with an nccl_unique_id) or cst_dist_create_host collectives");
  if (!D->has_coll || !local_eval) CST_CUDA(cudaSetDevice(D->h->device));  // NCCL staging / timing
  Comm comm{D};
  Server srv{D, &comm, o, in, scratch_out, local_eval, local_user};
  if (!local_eval) {
    CST_CUDA(cudaStreamCreateWithFlags(&srv.stream, cudaStreamNonBlocking));
  }
  struct StreamGuard {
    cudaStream_t s;
    ~StreamGuard() {
      if (s) cudaStreamDestroy(s);
    }
  } guard{srv.stream};
  Result res;
  std::memset(&res, 0, sizeof res);
  if (D->rank == 0) {
    Rank0Ctx ctx{&srv};
    cst_setting b{};
    cst_tune_report r{};
    cst_status st = cst_tune(D->h, o, in, scratch_out, rank0_eval, &ctx, &b, &r);
    if (st != CST_OK && ctx.err != CST_OK) st = ctx.err;  // the transport's error first
    const std::string msg = st == CST_OK ? "" : (ctx.err != CST_OK ? ctx.msg : cst_last_error());
    // the end marker and the result are always sent, so no rank blocks
    int64_t hdr = -1;
    cst_status cs = comm.bcast(&hdr, sizeof hdr);
    res.status = st;
    res.best = b;
    res.rep = r;
    std::strncpy(res.err, msg.c_str(), sizeof res.err - 1);
    if (cs == CST_OK) cs = comm.bcast(&res, sizeof res);
    if (st != CST_OK) return fail(st, msg);
    if (cs != CST_OK) return cs;
  } else {
    std::vector<cst_setting> ss;
    for (;;) {
      int64_t hdr = 0;
      cst_status st = comm.bcast(&hdr, sizeof hdr);
      if (st != CST_OK) return st;
      if (hdr < 0) break;
      st = srv.round(&ss, hdr, nullptr, nullptr);
      if (st != CST_OK) return st;
    }
    cst_status st = comm.bcast(&res, sizeof res);
    if (st != CST_OK) return st;
    if (res.status != CST_OK)
      return fail((cst_status)res.status, std::string("rank 0's tuner failed: ") + res.err);
  }
  *best = res.best;
  *rep = res.rep;
  return CST_OK;
}
