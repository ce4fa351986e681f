// spmv.cu — SpMV over CSR (PAPER.md P5@10072, P5@10497) on the binned gather.
#include "gather.cuh"

namespace inl {

namespace {
__global__ void k_build_xhot(const float *__restrict__ x, const int32_t *__restrict__ hot_cols, int n_hot,
                             float *__restrict__ x_hot) {
  for (int h = blockIdx.x * blockDim.x + threadIdx.x; h < n_hot; h += gridDim.x * blockDim.x)
    x_hot[h] = __ldg(x + hot_cols[h]);
}
}  // namespace

void build_xhot(inl_ctx ctx, inl_plan p, const float *x, const int32_t *hot_cols, int64_t n_hot) {
  const int n = (int)(n_hot >= 0 ? n_hot : p->n_hot);
  if (n == 0) return;
  k_build_xhot<<<(n + 255) / 256, 256, 0, ctx->stream>>>(
      x, hot_cols ? hot_cols : (const int32_t *)p->hot_cols.p, n, (float *)p->x_hot.p);
  INL_CUDA(cudaGetLastError());
}

void spmv_run(inl_ctx ctx, inl_plan p, const float *val, const float *x, float *y) {
  GatherArgs a{p->row_ptr, p->col_idx, val, x, p->nnz, p->n_rows,
               p->bins.t_thread, p->bins.t_warp, p->bins.t_block, p->bins.grid_chunk, false};
  launch_gather<true>(ctx, p, a, SpmvEpi{y}, nullptr, nullptr, nullptr, &p->cb);
}

void spmv_thread_only(inl_ctx ctx, const inl_csr &A, const float *val, const float *x, float *y) {
  if (A.n_rows == 0) return;
  GatherArgs a{A.row_ptr, A.col_idx, val, x, A.nnz, A.n_rows, 0, 0, 0, 0, false};
  int64_t g = (A.n_rows + 255) / 256;
  if (g > (int64_t)ctx->num_sms * 32) g = (int64_t)ctx->num_sms * 32;
  KScope ks(ctx, "k_gather_thread_only");
  k_gather_thread_only<<<(int)g, 256, 0, ctx->stream>>>(A.n_rows, a, SpmvEpi{y});
  INL_CUDA(cudaGetLastError());
}

}  // namespace inl
