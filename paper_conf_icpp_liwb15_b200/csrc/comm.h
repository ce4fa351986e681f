// comm.h — the per-iteration exchange of the multi-GPU row-block path (SURVEY §8a row
// a12): NCCL over NVLink between processes, or the loopback group (loopback.cu) between
// row-block contexts on one device.  Same calls, same semantics.
#pragma once
#include <vector>

#include "inl_internal.cuh"

namespace inl {
// true when the ctx is one rank of a row-block job (NCCL comm or loopback group; also P = 1)
inline bool has_comm(inl_ctx ctx) { return ctx->comm != nullptr || ctx->loop != nullptr; }
// In-place-capable allgather of `count` elements per rank (recv holds nranks*count),
// optionally grouped with an allgather of one double per rank (d_send -> d_recv).
// st: the stream the exchange is ordered on (nullptr = the ctx stream).
void comm_allgather(inl_ctx ctx, const void *send, void *recv, int64_t count, ncclDataType_t dt,
                    const double *d_send, double *d_recv, cudaStream_t st = nullptr);
// In-place allreduce.
void comm_allreduce(inl_ctx ctx, void *buf, int64_t count, ncclDataType_t dt, ncclRedOp_t op,
                    cudaStream_t st = nullptr);
// Stream-ordered barrier of all ranks: work a rank enqueued before it (including stores and
// atomics into peers' memory) is complete and visible before any rank's work after it runs.
void comm_barrier(inl_ctx ctx, cudaStream_t st = nullptr);
// The device base pointers of every rank's buffer `mine` (the same size on every rank; a
// collective): NCCL ranks map their peers' buffers with CUDA IPC (NVLink peer memory), loopback
// ranks share one device.  Cached until `mine` / `bytes` change.
const std::vector<void *> &comm_peer_bases(inl_ctx ctx, void *mine, size_t bytes);
// the ctx's second stream (created on first use): exchanges overlapped with the gather
cudaStream_t comm_stream(inl_ctx ctx);
cudaEvent_t ctx_event(inl_ctx ctx, int i);  // ctx-owned timing-free events, i < kCtxEvents
// loopback.cu
void loop_allgather(inl_ctx ctx, const void *send, void *recv, int64_t count, ncclDataType_t dt,
                    const double *d_send, double *d_recv, cudaStream_t st);
void loop_allreduce(inl_ctx ctx, void *buf, int64_t count, ncclDataType_t dt, ncclRedOp_t op, cudaStream_t st);
void loop_barrier(inl_ctx ctx, cudaStream_t st);
void loop_exchange_ptrs(inl_ctx ctx, void *mine, std::vector<void *> &out);
void loop_join(inl_ctx ctx, LoopGroup *g, int rank);
void loop_release(LoopGroup *g);
void loop_abort(inl_ctx ctx);
}  // namespace inl
