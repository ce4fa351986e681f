// comm.h — NCCL exchange used by the multi-GPU row-block path.
#pragma once
#include "inl_internal.cuh"

namespace inl {
// In-place-capable allgather of `count` elements per rank (recv holds nranks*count),
// optionally grouped with an allgather of one double per rank (d_send -> d_recv).
void comm_allgather(inl_ctx ctx, const void *send, void *recv, int64_t count, ncclDataType_t dt,
                    const double *d_send, double *d_recv);
void comm_allreduce(inl_ctx ctx, void *buf, int64_t count, ncclDataType_t dt, ncclRedOp_t op);
}  // namespace inl
