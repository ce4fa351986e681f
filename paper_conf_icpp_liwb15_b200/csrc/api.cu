// api.cu — the C-ABI of libinl.so (include/inl.h): argument checks, host-buffer
// staging, plan cache, error mapping, NCCL bootstrap.  No compute happens here:
// every step of the path runs in the kernels of plan.cu / spmv.cu / pagerank.cu /
// frontier.cu.  There is no CPU fallback.
#include <cstdarg>
#include <cstdio>
#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <new>

#include <nvtx3/nvToolsExt.h>

#include "comm.h"
#include "inl_internal.cuh"

#define INL_VERSION_STR "inl 0.1 (sm_100a)"

namespace inl {

void raise(inl_status code, const std::string &msg) { throw Error{code, msg}; }

NvtxRange::NvtxRange(const char *name) { nvtxRangePushA(name); }
NvtxRange::~NvtxRange() { nvtxRangePop(); }

void ctx_sync(inl_ctx ctx) {
  if (!ctx->comm) {
    INL_CUDA(cudaStreamSynchronize(ctx->stream));
    return;
  }
  static double limit_s = -1.0;
  if (limit_s < 0) {
    const char *e = getenv("INL_NCCL_TIMEOUT_S");
    limit_s = e ? atof(e) : 600.0;
  }
  const auto t0 = std::chrono::steady_clock::now();
  for (long spin = 0;; ++spin) {
    const cudaError_t q = cudaStreamQuery(ctx->stream);
    if (q == cudaSuccess) return;
    if (q != cudaErrorNotReady) INL_CUDA(q);
    ncclResult_t r = ncclSuccess;
    const ncclResult_t qr = ncclCommGetAsyncError(ctx->comm, &r);
    const bool failed = qr != ncclSuccess || (r != ncclSuccess && r != ncclInProgress);
    const double dt = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (failed || dt > limit_s) {
      ncclCommAbort(ctx->comm);
      ctx->comm = nullptr;
      raise(INL_ERR_NCCL, failed ? std::string("NCCL asynchronous error: ") + ncclGetErrorString(r)
                                 : "NCCL collective did not complete within INL_NCCL_TIMEOUT_S; communicator aborted");
    }
    if (spin > 2000) std::this_thread::sleep_for(std::chrono::microseconds(20));
  }
}

void *DevBuf::get(size_t need) {
  if (need == 0) need = 16;
  if (need > bytes) {
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
    const size_t want = need + need / 8;
    cudaError_t e = cudaMalloc(&p, want);
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
      raise(INL_ERR_OUT_OF_MEMORY, "cudaMalloc(" + std::to_string(want) + "): " + cudaGetErrorString(e));
    }
    bytes = want;
  }
  return p;
}

void DevBuf::release() {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = 0;
}

KTimer::Slot &KTimer::slot(const char *name) {
  for (auto &s : slots)
    if (s.name == name) return s;
  slots.emplace_back();
  slots.back().name = name;
  return slots.back();
}

cudaEvent_t KTimer::ev() {
  if (pool.empty()) {
    cudaEvent_t e;
    INL_CUDA(cudaEventCreate(&e));
    return e;
  }
  cudaEvent_t e = pool.back();
  pool.pop_back();
  return e;
}

void KTimer::resolve() {
  for (auto &s : slots) {
    for (auto &pr : s.pending) {
      float ms = 0.0f;
      INL_CUDA(cudaEventElapsedTime(&ms, pr.first, pr.second));
      s.ms += ms;
      s.launches += 1;
      pool.push_back(pr.first);
      pool.push_back(pr.second);
    }
    s.pending.clear();
  }
}

void KTimer::clear() {
  for (auto &s : slots)
    for (auto &pr : s.pending) {
      pool.push_back(pr.first);
      pool.push_back(pr.second);
    }
  slots.clear();
}

KTimer::~KTimer() {
  clear();
  for (cudaEvent_t e : pool) cudaEventDestroy(e);
}

Bins resolve_bins(const inl_bins *b) {
  Bins r{8, 1024, 16384, 8192, 256, 0};
  if (b) {
    if (b->t_thread > 0) r.t_thread = b->t_thread;
    if (b->t_thread < 0) r.t_thread = 0;
    if (b->t_warp > 0) r.t_warp = b->t_warp;
    if (b->t_block > 0) r.t_block = b->t_block;
    if (b->grid_chunk > 0) r.grid_chunk = b->grid_chunk;
    if (b->cta_threads > 0) r.cta = b->cta_threads;
    r.flags = b->flags;
  }
  INL_CHECK(r.cta >= 32 && r.cta <= 1024 && r.cta % 32 == 0, "bins.cta_threads must be a multiple of 32 in [32, 1024]");
  INL_CHECK(r.t_thread <= r.t_warp && r.t_warp <= r.t_block,
            "bins: need t_thread <= t_warp <= t_block");
  INL_CHECK(r.t_warp >= 16 && r.t_warp <= 4096, "bins.t_warp must be in [16, 4096]");
  INL_CHECK(r.grid_chunk >= 32 && r.grid_chunk <= (1 << 20), "bins.grid_chunk must be in [32, 2^20]");
  const int tpl = r.flags & kTemplateFlags;
  INL_CHECK((tpl & (tpl - 1)) == 0, "bins.flags: at most one paper template (INL_BINS_TPL_*)");
  INL_CHECK(!(tpl && (r.flags & (INL_BINS_THREAD_ONLY | INL_BINS_COLBLOCK | INL_BINS_SSSP_DEVLOOP))),
            "bins.flags: a paper template (INL_BINS_TPL_*) cannot be combined with other flags");
  INL_CHECK(!((r.flags & INL_BINS_THREAD_ONLY) && (r.flags & (INL_BINS_COLBLOCK | INL_BINS_SSSP_DEVLOOP))),
            "bins.flags: INL_BINS_THREAD_ONLY cannot be combined with other flags");
  if (r.flags & INL_BINS_THREAD_ONLY) {
    r.t_thread = r.t_warp = r.t_block = INT32_MAX / 2;
  }
  return r;
}

namespace {

thread_local std::string g_error;

struct DeviceGuard {
  int old = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&old) != cudaSuccess) {
      cudaGetLastError();
      old = -1;
    }
    if (old != dev) INL_CUDA(cudaSetDevice(dev));
  }
  ~DeviceGuard() {
    int cur = -1;
    if (old >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != old) cudaSetDevice(old);
  }
};

bool is_device(const void *p) {
  if (!p) return true;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

template <class T>
const T *stage_in(inl_ctx ctx, DevBuf &buf, const T *p, int64_t count) {
  if (!p || is_device(p)) return p;
  T *d = (T *)buf.get(sizeof(T) * (size_t)(count > 0 ? count : 1));
  if (count > 0)
    INL_CUDA(cudaMemcpyAsync(d, p, sizeof(T) * (size_t)count, cudaMemcpyHostToDevice, ctx->stream));
  return d;
}

template <class T>
struct StagedOut {
  T *user;
  T *dev;
  int64_t count;
  bool host;
};

template <class T>
StagedOut<T> stage_out(DevBuf &buf, T *p, int64_t count) {
  StagedOut<T> s{p, p, count, false};
  if (p && !is_device(p)) {
    s.host = true;
    s.dev = (T *)buf.get(sizeof(T) * (size_t)(count > 0 ? count : 1));
  }
  return s;
}

template <class T>
void finish_out(inl_ctx ctx, const StagedOut<T> &s) {
  if (s.host) {
    if (s.count > 0)
      INL_CUDA(cudaMemcpyAsync(s.user, s.dev, sizeof(T) * (size_t)s.count, cudaMemcpyDeviceToHost,
                               ctx->stream));
    INL_CUDA(cudaStreamSynchronize(ctx->stream));
  }
}

void check_csr(const inl_csr *A) {
  INL_CHECK(A != nullptr, "csr is NULL");
  INL_CHECK(A->n_rows >= 0 && A->n_global >= 0 && A->row_begin >= 0 && A->nnz >= 0,
            "csr: negative size");
  INL_CHECK(A->row_begin + A->n_rows <= A->n_global, "csr: row_begin + n_rows > n_global");
  INL_CHECK(A->n_global < INT32_MAX, "csr: n_global must be < 2^31 (int32 column ids)");
  INL_CHECK(A->row_ptr != nullptr, "csr.row_ptr is NULL");
  INL_CHECK(A->nnz == 0 || A->col_idx != nullptr, "csr.col_idx is NULL");
}

// Host CSR arrays are staged into ctx buffers; returns the device view.
inl_csr device_csr(inl_ctx ctx, const inl_csr *A) {
  inl_csr d = *A;
  d.row_ptr = stage_in(ctx, ctx->h_rp, A->row_ptr, A->n_rows + 1);
  d.col_idx = stage_in(ctx, ctx->h_ci, A->col_idx, A->nnz);
  return d;
}

bool same_csr(inl_plan p, const inl_csr &A) {
  return p->n_rows == A.n_rows && p->n_global == A.n_global && p->row_begin == A.row_begin &&
         p->nnz == A.nnz && p->row_ptr == A.row_ptr && p->col_idx == A.col_idx;
}

// plan (user or transient) for a device CSR
inl_plan get_plan(inl_ctx ctx, const inl_csr &A, inl_plan user) {
  if (user) {
    INL_CHECK(user->ctx == ctx, "plan belongs to another ctx");
    INL_CHECK(same_csr(user, A), "plan was created for a different CSR (pointers or sizes differ)");
    return user;
  }
  // the ctx keeps one transient plan whose buffers are reused across calls
  if (!ctx->tplan) ctx->tplan = new inl_plan_s();
  inl_plan p = ctx->tplan;
  p->ctx = ctx;
  p->transient = true;
  p->n_rows = A.n_rows;
  p->n_global = A.n_global;
  p->row_begin = A.row_begin;
  p->nnz = A.nnz;
  p->row_ptr = A.row_ptr;
  p->col_idx = A.col_idx;
  p->bins = resolve_bins(nullptr);
  build_plan(p);
  return p;
}

// SpMV on a device CSR: the T1 baseline, one of the paper's templates, or the default
// fused gather (transient plan when plan == NULL).
void spmv_dispatch(inl_ctx ctx, const inl_csr &d, const float *dval, const float *dx, float *ydev, inl_plan plan) {
  if (plan && (plan->bins.flags & INL_BINS_THREAD_ONLY)) {
    INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
    spmv_thread_only(ctx, d, dval, dx, ydev);
  } else if (plan && (plan->bins.flags & kTemplateFlags)) {
    INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
    spmv_template(ctx, d, plan->bins, dval, dx, ydev);
  } else {
    spmv_run(ctx, get_plan(ctx, d, plan), dval, dx, ydev);
  }
}

inl_status fail(inl_ctx ctx, inl_status code, const std::string &msg) {
  if (ctx) ctx->last_error = msg;
  g_error = msg;
  return code;
}

template <class F>
inl_status guarded(inl_ctx ctx, F &&f) {
  try {
    f();
    return INL_OK;
  } catch (const Error &e) {
    loop_abort(ctx);  // a failing loopback rank releases its peers (they fail, not hang)
    return fail(ctx, e.code, e.msg);
  } catch (const std::bad_alloc &) {
    loop_abort(ctx);
    return fail(ctx, INL_ERR_OUT_OF_MEMORY, "host allocation failed");
  } catch (...) {
    loop_abort(ctx);
    return fail(ctx, INL_ERR_INTERNAL, "unexpected C++ exception");
  }
}

__global__ void k_validate(const int64_t *rp, const int32_t *ci, int64_t n, int64_t nnz, int64_t ng,
                           unsigned long long *bad) {
  unsigned long long b = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s = rp[i], e = rp[i + 1];
    if (i == 0 && s != 0) ++b;
    if (i == n - 1 && e != nnz) ++b;
    if (e < s || s < 0 || e > nnz) {
      ++b;
      continue;
    }
    for (int64_t k = s; k < e; ++k)
      if (ci[k] < 0 || ci[k] >= ng) ++b;
  }
  if (b) atomicAdd(bad, b);
}

}  // namespace

void csr_validate(inl_ctx ctx, const inl_csr &A) {
  if (A.n_rows == 0) {
    INL_CHECK(A.nnz == 0, "csr: n_rows == 0 but nnz != 0");
    return;
  }
  unsigned long long *bad = (unsigned long long *)ctx->s_f.get(64);
  INL_CUDA(cudaMemsetAsync(bad, 0, 8, ctx->stream));
  k_validate<<<ctx->num_sms * 8, 256, 0, ctx->stream>>>(A.row_ptr, A.col_idx, A.n_rows, A.nnz,
                                                        A.n_global, bad);
  INL_CUDA(cudaGetLastError());
  unsigned long long h = 0;
  INL_CUDA(cudaMemcpyAsync(&h, bad, 8, cudaMemcpyDeviceToHost, ctx->stream));
  INL_CUDA(cudaStreamSynchronize(ctx->stream));
  INL_CHECK(h == 0, "csr_validate: " + std::to_string(h) + " malformed rows/entries");
}

void comm_allgather(inl_ctx ctx, const void *send, void *recv, int64_t count, ncclDataType_t dt,
                    const double *d_send, double *d_recv, cudaStream_t st) {
  if (!st) st = ctx->stream;
  if (ctx->loop) return loop_allgather(ctx, send, recv, count, dt, d_send, d_recv, st);
  INL_CHECK(ctx->comm != nullptr, "NCCL communicator not initialised (inl_comm_init)");
  INL_NCCL(ncclGroupStart());
  INL_NCCL(ncclAllGather(send, recv, (size_t)count, dt, ctx->comm, st));
  if (d_send) INL_NCCL(ncclAllGather(d_send, d_recv, 1, ncclFloat64, ctx->comm, st));
  INL_NCCL(ncclGroupEnd());
}

void comm_allreduce(inl_ctx ctx, void *buf, int64_t count, ncclDataType_t dt, ncclRedOp_t op, cudaStream_t st) {
  if (!st) st = ctx->stream;
  if (ctx->loop) return loop_allreduce(ctx, buf, count, dt, op, st);
  INL_CHECK(ctx->comm != nullptr, "NCCL communicator not initialised (inl_comm_init)");
  INL_NCCL(ncclAllReduce(buf, buf, (size_t)count, dt, op, ctx->comm, st));
}

void comm_barrier(inl_ctx ctx, cudaStream_t st) {
  if (!st) st = ctx->stream;
  if (ctx->loop) return loop_barrier(ctx, st);
  INL_CHECK(ctx->comm != nullptr, "NCCL communicator not initialised (inl_comm_init)");
  // a one-word allreduce: every rank's prior work on `st` precedes it, every rank's later work
  // follows its completion (NCCL's kernels order the peers' streams)
  int32_t *w = (int32_t *)ctx->s_bar.get(16);
  INL_NCCL(ncclAllReduce(w, w, 1, ncclInt32, ncclMax, ctx->comm, st));
}

static void close_peer_maps(inl_ctx ctx) {
  for (void *p : ctx->ipc_open)
    if (p) cudaIpcCloseMemHandle(p);
  ctx->ipc_open.clear();
  ctx->peer_bases.clear();
  ctx->peer_mine = nullptr;
  ctx->peer_bytes = 0;
}

const std::vector<void *> &comm_peer_bases(inl_ctx ctx, void *mine, size_t bytes) {
  if (ctx->peer_mine == mine && ctx->peer_bytes == bytes && !ctx->peer_bases.empty()) return ctx->peer_bases;
  close_peer_maps(ctx);
  if (ctx->loop) {
    loop_exchange_ptrs(ctx, mine, ctx->peer_bases);
  } else {
    INL_CHECK(ctx->comm != nullptr, "NCCL communicator not initialised (inl_comm_init)");
    const int P = ctx->nranks;
    cudaIpcMemHandle_t h;
    INL_CUDA(cudaIpcGetMemHandle(&h, mine));
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    char *dh = (char *)ctx->s_tmp.get(64 * (size_t)(P + 1));
    INL_CUDA(cudaMemcpyAsync(dh + 64 * (size_t)ctx->rank, &h, 64, cudaMemcpyHostToDevice, ctx->stream));
    INL_NCCL(ncclAllGather(dh + 64 * (size_t)ctx->rank, dh, 64, ncclUint8, ctx->comm, ctx->stream));
    std::vector<cudaIpcMemHandle_t> all(P);
    INL_CUDA(cudaMemcpyAsync(all.data(), dh, 64 * (size_t)P, cudaMemcpyDeviceToHost, ctx->stream));
    INL_CUDA(cudaStreamSynchronize(ctx->stream));
    ctx->peer_bases.assign(P, nullptr);
    for (int q = 0; q < P; ++q) {
      if (q == ctx->rank) {
        ctx->peer_bases[q] = mine;
        continue;
      }
      void *p = nullptr;
      INL_CUDA(cudaIpcOpenMemHandle(&p, all[q], cudaIpcMemLazyEnablePeerAccess));
      ctx->ipc_open.push_back(p);
      ctx->peer_bases[q] = p;
    }
  }
  ctx->peer_mine = mine;
  ctx->peer_bytes = bytes;
  return ctx->peer_bases;
}

cudaStream_t comm_stream(inl_ctx ctx) {
  if (!ctx->comm_stream) INL_CUDA(cudaStreamCreateWithFlags(&ctx->comm_stream, cudaStreamNonBlocking));
  return ctx->comm_stream;
}

cudaEvent_t ctx_event(inl_ctx ctx, int i) {
  INL_CHECK(i >= 0 && i < kCtxEvents, "ctx_event: index out of range");
  if (!ctx->events[i]) INL_CUDA(cudaEventCreateWithFlags(&ctx->events[i], cudaEventDisableTiming));
  return ctx->events[i];
}

}  // namespace inl

using namespace inl;

extern "C" {

const char *inl_version(void) { return INL_VERSION_STR; }

const char *inl_status_string(inl_status s) {
  switch (s) {
    case INL_OK: return "INL_OK";
    case INL_ERR_INVALID_ARGUMENT: return "INL_ERR_INVALID_ARGUMENT";
    case INL_ERR_OUT_OF_MEMORY: return "INL_ERR_OUT_OF_MEMORY";
    case INL_ERR_CUDA: return "INL_ERR_CUDA";
    case INL_ERR_NCCL: return "INL_ERR_NCCL";
    case INL_ERR_NOT_INITIALIZED: return "INL_ERR_NOT_INITIALIZED";
    case INL_ERR_UNSUPPORTED: return "INL_ERR_UNSUPPORTED";
    case INL_ERR_INTERNAL: return "INL_ERR_INTERNAL";
  }
  return "INL_ERR_UNKNOWN";
}

const char *inl_last_error(inl_ctx ctx) { return ctx ? ctx->last_error.c_str() : g_error.c_str(); }

inl_status inl_ctx_create(inl_ctx *out, int device, void *cuda_stream) {
  if (!out) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "out is NULL");
  inl_ctx c = new (std::nothrow) inl_ctx_s();
  if (!c) return fail(nullptr, INL_ERR_OUT_OF_MEMORY, "ctx allocation failed");
  inl_status s = guarded(nullptr, [&] {
    int ndev = 0;
    INL_CUDA(cudaGetDeviceCount(&ndev));
    INL_CHECK(device >= 0 && device < ndev, "device ordinal out of range");
    DeviceGuard g(device);
    c->device = device;
    c->stream = (cudaStream_t)cuda_stream;
    INL_CUDA(cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device));
    INL_CUDA(cudaMallocHost(&c->pinned, 64));
  });
  if (s != INL_OK) {
    delete c;
    return s;
  }
  *out = c;
  return INL_OK;
}

inl_status inl_ctx_set_stream(inl_ctx ctx, void *cuda_stream) {
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  ctx->stream = (cudaStream_t)cuda_stream;
  return INL_OK;
}

namespace inl {
static void free_ctx(inl_ctx ctx) {
  int old = -1;
  cudaGetDevice(&old);
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->stream);
  close_peer_maps(ctx);
  if (ctx->comm) ncclCommDestroy(ctx->comm);
  if (ctx->loop) loop_release(ctx->loop);
  if (ctx->comm_stream) {
    cudaStreamSynchronize(ctx->comm_stream);
    cudaStreamDestroy(ctx->comm_stream);
  }
  for (cudaEvent_t e : ctx->events)
    if (e) cudaEventDestroy(e);
  if (ctx->sssp_graph) sssp_graph_free(ctx->sssp_graph);
  if (ctx->pinned) cudaFreeHost(ctx->pinned);
  delete ctx->tplan;
  delete ctx;  // DevBuf destructors free device scratch
  if (old >= 0) cudaSetDevice(old);
}
}  // namespace inl

// Plans keep their ctx alive: the ctx is freed when it is destroyed AND its last plan is.
inl_status inl_ctx_destroy(inl_ctx ctx) {
  if (!ctx || ctx->closed) return INL_OK;
  ctx->closed = true;
  if (ctx->live_plans == 0) free_ctx(ctx);
  return INL_OK;
}

inl_status inl_ktimer_enable(inl_ctx ctx, int32_t enable) {
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    DeviceGuard g(ctx->device);
    INL_CUDA(cudaStreamSynchronize(ctx->stream));
    ctx->ktimer.clear();
    ctx->ktimer.on = enable != 0;
  });
}

inl_status inl_ktimer_read(inl_ctx ctx, const char *kernel, int64_t *launches, double *total_ms) {
  if (!ctx || !kernel || !launches || !total_ms)
    return fail(ctx, INL_ERR_INVALID_ARGUMENT, "ktimer_read: NULL argument");
  return guarded(ctx, [&] {
    DeviceGuard g(ctx->device);
    INL_CUDA(cudaStreamSynchronize(ctx->stream));
    ctx->ktimer.resolve();
    *launches = 0;
    *total_ms = 0.0;
    for (auto &s : ctx->ktimer.slots)
      if (s.name == kernel) {
        *launches = s.launches;
        *total_ms = s.ms;
      }
  });
}

inl_status inl_partition_rows(int64_t n, int32_t nranks, int64_t *bounds) {
  if (n < 0 || nranks < 1 || !bounds) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "partition: bad argument");
  const int64_t B = (n + nranks - 1) / nranks;
  for (int32_t p = 0; p <= nranks; ++p) {
    const int64_t b = (int64_t)p * B;
    bounds[p] = b < n ? b : n;
  }
  return INL_OK;
}

inl_status inl_nccl_unique_id(uint8_t out[128]) {
  return guarded(nullptr, [&] {
    INL_CHECK(out != nullptr, "out is NULL");
    ncclUniqueId id;
    INL_NCCL(ncclGetUniqueId(&id));
    static_assert(sizeof(id) == 128, "ncclUniqueId size");
    memcpy(out, &id, 128);
  });
}

inl_status inl_comm_init(inl_ctx ctx, const uint8_t uid[128], int32_t nranks, int32_t rank) {
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    INL_CHECK(uid != nullptr && nranks >= 1 && rank >= 0 && rank < nranks, "comm_init: bad argument");
    INL_CHECK(ctx->comm == nullptr && ctx->loop == nullptr, "comm already initialised on this ctx");
    DeviceGuard g(ctx->device);
    ncclUniqueId id;
    memcpy(&id, uid, 128);
    INL_NCCL(ncclCommInitRank(&ctx->comm, nranks, id, rank));
    ctx->nranks = nranks;
    ctx->rank = rank;
  });
}

inl_status inl_comm_init_loopback(inl_ctx ctx, inl_loop group, int32_t rank) {
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    INL_CHECK(group != nullptr, "loopback group is NULL");
    INL_CHECK(ctx->comm == nullptr && ctx->loop == nullptr, "comm already initialised on this ctx");
    DeviceGuard g(ctx->device);
    loop_join(ctx, reinterpret_cast<LoopGroup *>(group), rank);
  });
}

inl_status inl_plan_create(inl_ctx ctx, const inl_csr *A, const inl_bins *bins, inl_plan *out) {
  NvtxRange nvtx_("inl_plan_create");
  if (!ctx || ctx->closed) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL or destroyed");
  inl_plan p = nullptr;
  inl_status s = guarded(ctx, [&] {
    INL_CHECK(out != nullptr, "out is NULL");
    check_csr(A);
    DeviceGuard g(ctx->device);
    INL_CHECK(is_device(A->row_ptr) && is_device(A->col_idx),
              "plan_create needs a device CSR (host CSRs use plan = NULL)");
    p = new inl_plan_s();
    p->ctx = ctx;
    p->n_rows = A->n_rows;
    p->n_global = A->n_global;
    p->row_begin = A->row_begin;
    p->nnz = A->nnz;
    p->row_ptr = A->row_ptr;
    p->col_idx = A->col_idx;
    p->bins = resolve_bins(bins);
    if (!(p->bins.flags & (INL_BINS_THREAD_ONLY | kTemplateFlags)))
      build_plan(p);  // the T1 baseline and the paper's templates need no bins
  });
  if (s != INL_OK) {
    delete p;
    return s;
  }
  ctx->live_plans++;
  *out = p;
  return INL_OK;
}

inl_status inl_plan_get_info(inl_plan plan, inl_plan_info *info) {
  if (!plan || !info) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "plan/info is NULL");
  *info = plan->info;
  return INL_OK;
}

inl_status inl_plan_destroy(inl_plan plan) {
  if (!plan) return INL_OK;
  inl_ctx ctx = plan->ctx;
  int old = -1;
  cudaGetDevice(&old);
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->stream);
  delete plan;
  if (old >= 0) cudaSetDevice(old);
  if (--ctx->live_plans == 0 && ctx->closed) free_ctx(ctx);
  return INL_OK;
}

inl_status inl_csr_validate(inl_ctx ctx, const inl_csr *A) {
  NvtxRange nvtx_("inl_csr_validate");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(A);
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, A);
    csr_validate(ctx, d);
  });
}

inl_status inl_spmv(inl_ctx ctx, const inl_csr *A, const float *val, const float *x, float *y,
                    inl_plan plan) {
  NvtxRange nvtx_("inl_spmv");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(A);
    INL_CHECK(A->nnz == 0 || val != nullptr, "val is NULL");
    INL_CHECK(A->n_global == 0 || x != nullptr, "x is NULL");
    INL_CHECK(A->n_rows == 0 || y != nullptr, "y is NULL");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, A);
    const float *dval = stage_in(ctx, ctx->h_val, val, A->nnz);
    const float *dx = stage_in(ctx, ctx->h_x, x, A->n_global);
    StagedOut<float> yo = stage_out(ctx->h_y, y, A->n_rows);
    spmv_dispatch(ctx, d, dval, dx, yo.dev, plan);
    finish_out(ctx, yo);
  });
}

inl_status inl_spmv_allgather(inl_ctx ctx, const inl_csr *A, const float *val, const float *x, float *y_global,
                              inl_plan plan) {
  NvtxRange nvtx_("inl_spmv_allgather");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(A);
    INL_CHECK(A->nnz == 0 || val != nullptr, "val is NULL");
    INL_CHECK(A->n_global == 0 || (x != nullptr && y_global != nullptr), "x / y_global is NULL");
    const int64_t n = A->n_global;
    const int P = has_comm(ctx) ? ctx->nranks : 1;
    const int64_t B = (n + P - 1) / P;
    INL_CHECK(has_comm(ctx) || (A->row_begin == 0 && A->n_rows == n), "a partial CSR (row block) needs a communicator");
    INL_CHECK(A->row_begin == (int64_t)ctx->rank * B && A->n_rows == std::min(B, n - A->row_begin),
              "row block does not match inl_partition_rows for this rank");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, A);
    const float *dval = stage_in(ctx, ctx->h_val, val, A->nnz);
    const float *dx = stage_in(ctx, ctx->h_x, x, n);
    StagedOut<float> yo = stage_out(ctx->h_y, y_global, n);
    // NCCL's allgather moves equal counts: in place when P divides n, else through a padded copy
    float *full = B * P == n ? yo.dev : (float *)ctx->s_pad.get(sizeof(float) * (size_t)(B * P));
    spmv_dispatch(ctx, d, dval, dx, full + A->row_begin, plan);
    if (has_comm(ctx)) comm_allgather(ctx, full + A->row_begin, full, B, ncclFloat32, nullptr, nullptr);
    if (full != yo.dev && n > 0)
      INL_CUDA(cudaMemcpyAsync(yo.dev, full, sizeof(float) * (size_t)n, cudaMemcpyDeviceToDevice, ctx->stream));
    finish_out(ctx, yo);
  });
}

inl_status inl_pagerank(inl_ctx ctx, const inl_csr *A_in, const int32_t *out_degree, float damping,
                        int32_t iterations, float *rank, inl_plan plan) {
  NvtxRange nvtx_("inl_pagerank");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(A_in);
    INL_CHECK(damping >= 0.0f && damping < 1.0f, "damping must be in [0, 1)");
    INL_CHECK(iterations >= 0, "iterations must be >= 0");
    INL_CHECK(A_in->n_global == 0 || (out_degree && rank), "out_degree/rank is NULL");
    INL_CHECK(has_comm(ctx) || (A_in->row_begin == 0 && A_in->n_rows == A_in->n_global),
              "a partial CSR (row block) needs inl_comm_init");
    INL_CHECK(!has_comm(ctx) || ctx->nranks == 1 ||
                  A_in->row_begin == (int64_t)ctx->rank * ((A_in->n_global + ctx->nranks - 1) / ctx->nranks),
              "row block does not match inl_partition_rows for this rank");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, A_in);
    const int32_t *dod = stage_in(ctx, ctx->h_od, out_degree, A_in->n_global);
    StagedOut<float> ro = stage_out(ctx->h_y, rank, A_in->n_global);
    if (plan && (plan->bins.flags & (kTemplateFlags | INL_BINS_THREAD_ONLY))) {  // the template study (one GPU)
      INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
      pagerank_run(ctx, plan, dod, damping, iterations, ro.dev);
    } else {
      pagerank_run(ctx, get_plan(ctx, d, plan), dod, damping, iterations, ro.dev);
    }
    finish_out(ctx, ro);
  });
}

inl_status inl_sssp(inl_ctx ctx, const inl_csr *G, const uint32_t *w, int64_t source, uint32_t *dist,
                    inl_stats *stats, inl_plan plan) {
  NvtxRange nvtx_("inl_sssp");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(G);
    INL_CHECK(source >= 0 && source < G->n_global, "source out of range");
    INL_CHECK(G->nnz == 0 || w != nullptr, "w is NULL");
    INL_CHECK(dist != nullptr, "dist is NULL");
    INL_CHECK(has_comm(ctx) || (G->row_begin == 0 && G->n_rows == G->n_global),
              "a partial CSR (row block) needs inl_comm_init");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, G);
    const uint32_t *dw = stage_in(ctx, ctx->h_w, w, G->nnz);
    StagedOut<uint32_t> o = stage_out(ctx->h_y, dist, G->n_global);
    Bins b = plan ? plan->bins : resolve_bins(nullptr);
    if (plan) INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
    sssp_run(ctx, d, b, dw, source, o.dev, stats);
    finish_out(ctx, o);
    ctx_sync(ctx);
  });
}

inl_status inl_bfs(inl_ctx ctx, const inl_csr *G, int64_t source, int32_t *level, inl_stats *stats,
                   inl_plan plan) {
  NvtxRange nvtx_("inl_bfs");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(G);
    INL_CHECK(source >= 0 && source < G->n_global, "source out of range");
    INL_CHECK(level != nullptr, "level is NULL");
    INL_CHECK(has_comm(ctx) || (G->row_begin == 0 && G->n_rows == G->n_global),
              "a partial CSR (row block) needs inl_comm_init");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, G);
    StagedOut<int32_t> o = stage_out(ctx->h_y, level, G->n_global);
    Bins b = plan ? plan->bins : resolve_bins(nullptr);
    if (plan) INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
    BuStatic bus;
    if (plan && plan->symmetric && plan->bu_ns + plan->bu_nl > 0) {
      bus.s = (const int32_t *)plan->bu_lists.p;
      bus.l = bus.s + plan->n_global;
      bus.ns = plan->bu_ns;
      bus.nl = plan->bu_nl;
    }
    bfs_run(ctx, d, b, source, o.dev, stats, plan && plan->symmetric, bus);
    finish_out(ctx, o);
    ctx_sync(ctx);
  });
}

inl_status inl_bc(inl_ctx ctx, const inl_csr *G, const int64_t *sources, int64_t n_sources, double *bc,
                  inl_stats *stats, inl_plan plan) {
  NvtxRange nvtx_("inl_bc");
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(G);
    INL_CHECK(n_sources >= 0 && (n_sources == 0 || sources != nullptr), "sources is NULL");
    INL_CHECK(n_sources == 0 || !is_device(sources), "sources must be a host array");
    for (int64_t i = 0; i < n_sources; ++i)
      INL_CHECK(sources[i] >= 0 && sources[i] < G->n_global, "source out of range");
    INL_CHECK(G->n_global == 0 || bc != nullptr, "bc is NULL");
    INL_CHECK(G->row_begin == 0 && G->n_rows == G->n_global, "bc: one GPU, full CSR (no row blocks)");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, G);
    if (plan) INL_CHECK(plan->ctx == ctx && same_csr(plan, d), "plan was created for a different CSR");
    StagedOut<double> o = stage_out(ctx->h_y, bc, G->n_global);
    const Bins b = plan ? plan->bins : resolve_bins(nullptr);
    bc_run(ctx, d, b, sources, n_sources, o.dev, stats, plan && plan->symmetric);
    finish_out(ctx, o);
    ctx_sync(ctx);
  });
}

static inl_status tree_entry(inl_ctx ctx, const inl_csr *T, const int32_t *parent, int64_t root, int32_t method,
                             int64_t *out, inl_stats *stats, bool heights) {
  if (!ctx) return fail(nullptr, INL_ERR_INVALID_ARGUMENT, "ctx is NULL");
  return guarded(ctx, [&] {
    check_csr(T);
    INL_CHECK(T->row_begin == 0 && T->n_rows == T->n_global, "tree: one GPU, the whole children CSR");
    INL_CHECK(T->n_global == 0 || (root >= 0 && root < T->n_global), "tree: root out of range");
    INL_CHECK(T->n_global == 0 || out != nullptr, "tree: output is NULL");
    INL_CHECK(method == INL_TREE_FLAT || method == INL_TREE_LEVELS, "tree: unknown method");
    INL_CHECK(method != INL_TREE_FLAT || T->n_global == 0 || parent != nullptr, "tree: INL_TREE_FLAT needs parent[]");
    DeviceGuard g(ctx->device);
    inl_csr d = device_csr(ctx, T);
    const int32_t *dpar = stage_in(ctx, ctx->h_od, parent, T->n_global);
    StagedOut<int64_t> o = stage_out(ctx->h_y, out, T->n_global);
    tree_run(ctx, d, dpar, root, method, heights, o.dev, stats);
    finish_out(ctx, o);
    ctx_sync(ctx);
  });
}

inl_status inl_tree_descendants(inl_ctx ctx, const inl_csr *T, const int32_t *parent, int64_t root, int32_t method,
                                int64_t *desc, inl_stats *stats) {
  NvtxRange nvtx_("inl_tree_descendants");
  return tree_entry(ctx, T, parent, root, method, desc, stats, false);
}

inl_status inl_tree_heights(inl_ctx ctx, const inl_csr *T, const int32_t *parent, int64_t root, int32_t method,
                            int64_t *height, inl_stats *stats) {
  NvtxRange nvtx_("inl_tree_heights");
  return tree_entry(ctx, T, parent, root, method, height, stats, true);
}

}  // extern "C"
