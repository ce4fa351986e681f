// loopback.cu — a stand-in for NCCL behind the same exchange calls (comm.h), for P
// row-block contexts on ONE device (VERDICT r1 "put the multi-rank product
// path under oracle parity on one GPU").
//
// Each rank is an inl_ctx with its own stream, driven by its own host thread (the
// frontier ops block inside their iteration loop, exactly as the NCCL ranks of a
// torchrun job do).  A collective is stepped in lockstep:
//   1. every rank records "my input is ready" on its stream and arrives at a host barrier;
//   2. every rank makes its stream wait for all peers' ready events, then moves the data
//      with device work on its own stream (allgather: P-1 device-to-device copies from the
//      peers' buffers; allreduce: one kernel that reduces the P peers' buffers into this
//      rank's scratch);
//   3. every rank records "done reading my peers" and arrives at a second barrier, then
//      makes its stream wait for all peers' done events — so nothing a rank enqueues later
//      can overwrite a buffer a peer is still reading — and (allreduce) copies its scratch
//      back in place.
// Semantics are NCCL's: in-place allgather (send == recv + rank * count) or out-of-place;
// in-place allreduce with ncclMin / ncclMax / ncclSum over the dtypes the path uses.  A
// rank that fails marks the group aborted, so its peers fail at their next barrier instead
// of hanging; a barrier that waits more than kLoopTimeoutS raises INL_ERR_NCCL.
#include <chrono>
#include <condition_variable>
#include <mutex>
#include <vector>

#include "comm.h"
#include "inl_internal.cuh"

namespace inl {

constexpr int kLoopMax = 64;          // ranks per loopback group
constexpr double kLoopTimeoutS = 300;  // a peer that never arrives (a test bug, not a race)

struct LoopGroup {
  int nranks = 0;
  int refs = 1;
  std::mutex m;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  bool aborted = false;
  std::vector<int> joined;  // rank -> joined
  // per-rank slots of the collective in flight
  std::vector<const void *> src;
  std::vector<void *> dst;
  std::vector<const double *> dsrc;
  std::vector<cudaEvent_t> ready, done;

  explicit LoopGroup(int p) : nranks(p), joined(p, 0), src(p), dst(p), dsrc(p), ready(p), done(p) {}

  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    if (aborted) raise(INL_ERR_NCCL, "loopback group aborted by a failing rank");
    const uint64_t g = gen;
    if (++arrived == nranks) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return;
    }
    const bool ok = cv.wait_for(lk, std::chrono::duration<double>(kLoopTimeoutS),
                                [&] { return gen != g || aborted; });
    if (aborted) raise(INL_ERR_NCCL, "loopback group aborted by a failing rank");
    if (!ok) {
      aborted = true;
      cv.notify_all();
      raise(INL_ERR_NCCL, "loopback barrier timed out (a peer rank never reached the collective)");
    }
  }
  void abort() {
    std::lock_guard<std::mutex> lk(m);
    aborted = true;
    cv.notify_all();
  }
};

namespace {

template <class T>
struct PeerPtrs {
  const T *p[kLoopMax];
};

template <class T, int OP>  // OP: 0 min, 1 max, 2 sum
__device__ __forceinline__ T red_op(T a, T b) {
  if (OP == 0) return a < b ? a : b;
  if (OP == 1) return a > b ? a : b;
  return a + b;
}

// out[i] = op over ranks q = 0..P-1 (in rank order) of in_q[i]
template <class T, int OP>
__global__ void k_loop_reduce(PeerPtrs<T> in, int P, int64_t count, T *__restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x) {
    T v = in.p[0][i];
    for (int q = 1; q < P; ++q) v = red_op<T, OP>(v, in.p[q][i]);
    out[i] = v;
  }
}

size_t dt_size(ncclDataType_t dt) {
  switch (dt) {
    case ncclInt8: case ncclUint8: return 1;
    case ncclFloat16: case ncclBfloat16: return 2;
    case ncclInt32: case ncclUint32: case ncclFloat32: return 4;
    case ncclInt64: case ncclUint64: case ncclFloat64: return 8;
    default: break;
  }
  raise(INL_ERR_UNSUPPORTED, "loopback: unsupported NCCL datatype");
}

template <class T>
void launch_reduce(inl_ctx ctx, LoopGroup *g, ncclRedOp_t op, int64_t count, void *out, cudaStream_t st) {
  PeerPtrs<T> pp{};
  for (int q = 0; q < g->nranks; ++q) pp.p[q] = (const T *)g->src[q];
  int64_t grid = (count + 255) / 256;
  if (grid > (int64_t)ctx->num_sms * 8) grid = (int64_t)ctx->num_sms * 8;
  if (grid < 1) grid = 1;
  T *o = (T *)out;
  if (op == ncclMin) k_loop_reduce<T, 0><<<(int)grid, 256, 0, st>>>(pp, g->nranks, count, o);
  else if (op == ncclMax) k_loop_reduce<T, 1><<<(int)grid, 256, 0, st>>>(pp, g->nranks, count, o);
  else if (op == ncclSum) k_loop_reduce<T, 2><<<(int)grid, 256, 0, st>>>(pp, g->nranks, count, o);
  else raise(INL_ERR_UNSUPPORTED, "loopback: unsupported reduction op");
  INL_CUDA(cudaGetLastError());
}

// phase 1: publish + ready event + barrier + wait for the peers' inputs
void phase_in(inl_ctx ctx, LoopGroup *g, const void *src, void *dst, const double *dsrc, cudaStream_t st) {
  const int r = ctx->rank;
  g->src[r] = src;
  g->dst[r] = dst;
  g->dsrc[r] = dsrc;
  INL_CUDA(cudaEventRecord(g->ready[r], st));
  g->barrier();
  for (int q = 0; q < g->nranks; ++q)
    if (q != r) INL_CUDA(cudaStreamWaitEvent(st, g->ready[q], 0));
}

// phase 2: done event + barrier + wait until no peer still reads this rank's buffers
void phase_out(inl_ctx ctx, LoopGroup *g, cudaStream_t st) {
  const int r = ctx->rank;
  INL_CUDA(cudaEventRecord(g->done[r], st));
  g->barrier();
  for (int q = 0; q < g->nranks; ++q)
    if (q != r) INL_CUDA(cudaStreamWaitEvent(st, g->done[q], 0));
}

}  // namespace

void loop_allgather(inl_ctx ctx, const void *send, void *recv, int64_t count, ncclDataType_t dt,
                    const double *d_send, double *d_recv, cudaStream_t st) {
  LoopGroup *g = ctx->loop;
  const int r = ctx->rank, P = g->nranks;
  const size_t bytes = dt_size(dt) * (size_t)count;
  phase_in(ctx, g, send, recv, d_send, st);
  for (int q = 0; q < P; ++q) {
    char *to = (char *)recv + (size_t)q * bytes;
    if (bytes && to != g->src[q])  // in place for q == r: nothing to copy
      INL_CUDA(cudaMemcpyAsync(to, g->src[q], bytes, cudaMemcpyDeviceToDevice, st));
    if (d_send) INL_CUDA(cudaMemcpyAsync(d_recv + q, g->dsrc[q], sizeof(double), cudaMemcpyDeviceToDevice, st));
  }
  (void)r;
  phase_out(ctx, g, st);
}

void loop_allreduce(inl_ctx ctx, void *buf, int64_t count, ncclDataType_t dt, ncclRedOp_t op, cudaStream_t st) {
  LoopGroup *g = ctx->loop;
  const size_t es = dt_size(dt);
  void *tmp = ctx->s_loop.get(es * (size_t)(count > 0 ? count : 1));
  phase_in(ctx, g, buf, buf, nullptr, st);
  if (count > 0) {
    switch (dt) {
      case ncclUint8: launch_reduce<uint8_t>(ctx, g, op, count, tmp, st); break;
      case ncclInt8: launch_reduce<int8_t>(ctx, g, op, count, tmp, st); break;
      case ncclUint32: launch_reduce<uint32_t>(ctx, g, op, count, tmp, st); break;
      case ncclInt32: launch_reduce<int32_t>(ctx, g, op, count, tmp, st); break;
      case ncclUint64: launch_reduce<unsigned long long>(ctx, g, op, count, tmp, st); break;
      case ncclInt64: launch_reduce<long long>(ctx, g, op, count, tmp, st); break;
      case ncclFloat32: launch_reduce<float>(ctx, g, op, count, tmp, st); break;
      case ncclFloat64: launch_reduce<double>(ctx, g, op, count, tmp, st); break;
      default: raise(INL_ERR_UNSUPPORTED, "loopback: unsupported datatype for allreduce");
    }
  }
  phase_out(ctx, g, st);  // every peer has read this rank's buf: overwrite it in place
  if (count > 0) INL_CUDA(cudaMemcpyAsync(buf, tmp, es * (size_t)count, cudaMemcpyDeviceToDevice, st));
}

void loop_barrier(inl_ctx ctx, cudaStream_t st) {
  phase_in(ctx, ctx->loop, nullptr, nullptr, nullptr, st);
  phase_out(ctx, ctx->loop, st);
}

void loop_exchange_ptrs(inl_ctx ctx, void *mine, std::vector<void *> &out) {
  LoopGroup *g = ctx->loop;
  phase_in(ctx, g, mine, mine, nullptr, ctx->stream);
  out.assign(g->nranks, nullptr);
  for (int q = 0; q < g->nranks; ++q) out[q] = g->dst[q];
  phase_out(ctx, g, ctx->stream);
}

void loop_abort(inl_ctx ctx) {
  if (ctx && ctx->loop) ctx->loop->abort();
}

void loop_release(LoopGroup *g) {
  bool last = false;
  {
    std::lock_guard<std::mutex> lk(g->m);
    last = --g->refs == 0;
  }
  if (last) {
    for (auto e : g->ready)
      if (e) cudaEventDestroy(e);
    for (auto e : g->done)
      if (e) cudaEventDestroy(e);
    delete g;
  }
}

void loop_join(inl_ctx ctx, LoopGroup *g, int rank) {
  std::lock_guard<std::mutex> lk(g->m);
  INL_CHECK(rank >= 0 && rank < g->nranks, "loopback: rank out of range");
  INL_CHECK(!g->joined[rank], "loopback: rank already joined");
  INL_CUDA(cudaEventCreateWithFlags(&g->ready[rank], cudaEventDisableTiming));
  INL_CUDA(cudaEventCreateWithFlags(&g->done[rank], cudaEventDisableTiming));
  g->joined[rank] = 1;
  g->refs++;
  ctx->loop = g;
  ctx->nranks = g->nranks;
  ctx->rank = rank;
}

}  // namespace inl

using namespace inl;

extern "C" {

inl_status inl_loop_create(int32_t nranks, inl_loop *out) {
  if (!out || nranks < 1 || nranks > kLoopMax) return INL_ERR_INVALID_ARGUMENT;
  LoopGroup *g = new (std::nothrow) LoopGroup(nranks);
  if (!g) return INL_ERR_OUT_OF_MEMORY;
  *out = reinterpret_cast<inl_loop>(g);
  return INL_OK;
}

inl_status inl_loop_destroy(inl_loop group) {
  if (group) loop_release(reinterpret_cast<LoopGroup *>(group));
  return INL_OK;
}

}  // extern "C"
