// extern "C" entry points of include/spmv.h: argument checks, error
// translation (no exception crosses the ABI), thread-local last error.
#include <algorithm>
#include <cstring>
#include <string>

#include <nvtx3/nvToolsExt.h>

#include "plan.cuh"

// NVTX range over one ABI call (header-only NVTX v3: a no-op unless a tool
// such as nsys / ncu attaches), so plan / permute / exec / iterate show up as
// named ranges on a timeline
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

namespace spmv {
static thread_local std::string g_err;
void set_error(const std::string& m) { g_err = m; }
const char* get_error() { return g_err.c_str(); }
}  // namespace spmv

#define API_BEGIN try {
#define API_END                                             \
  }                                                         \
  catch (const spmv::Err& e) {                              \
    return e.st;                                            \
  }                                                         \
  catch (const std::bad_alloc&) {                           \
    spmv::set_error("out of host memory");                  \
    return SPMV_ENOMEM;                                     \
  }                                                         \
  catch (const std::exception& e) {                         \
    spmv::set_error(std::string("internal: ") + e.what());  \
    return SPMV_EINVAL;                                     \
  }                                                         \
  catch (...) {                                             \
    spmv::set_error("internal: unknown exception");         \
    return SPMV_EINVAL;                                     \
  }                                                         \
  return SPMV_OK;

static cudaStream_t S(void* s) { return (cudaStream_t)s; }

static void use_device(spmv_plan_s* p) { SPMV_CUDA(cudaSetDevice(p->device)); }

extern "C" {

void spmv_opts_default(spmv_opts_t* o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->l2_window = 1;
  o->evict_first = 1;
  o->rank = 0;
  o->world = 1;
  o->device = -1;
  o->l2_hit_ratio = 1.0;
  o->smem_window = 1;
}

const char* spmv_last_error(void) { return spmv::get_error(); }
const char* spmv_version(void) { return "spmv-b200 0.1 (sm_100a)"; }

spmv_status spmv_plan(const spmv_csr_t* A, const int32_t* perm, const spmv_opts_t* opts,
                      spmv_plan_t* out) {
  NvtxRange nvtx_("spmv_plan");
  spmv_plan_s* p = nullptr;
  API_BEGIN
  if (!A || !out) SPMV_FAIL(SPMV_EINVAL, "spmv_plan: NULL argument");
  *out = nullptr;
  if (A->n < 0 || A->nnz < 0) SPMV_FAIL(SPMV_EINVAL, "spmv_plan: negative n or nnz");
  if ((A->row_ptr32 == nullptr) == (A->row_ptr64 == nullptr))
    SPMV_FAIL(SPMV_EINVAL, "spmv_plan: exactly one of row_ptr32/row_ptr64 must be set");
  if (A->nnz && (!A->col_idx || !A->vals)) SPMV_FAIL(SPMV_EINVAL, "spmv_plan: NULL col/vals");
  if (A->n > (int64_t)INT32_MAX - 1) SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_plan: n must fit int32 column ids");
  if (A->row_ptr32 && A->nnz > (int64_t)INT32_MAX)
    SPMV_FAIL(SPMV_EINVAL, "spmv_plan: nnz >= 2^31 needs row_ptr64");
  p = new spmv_plan_s();
  spmv_opts_default(&p->opts);
  if (opts) p->opts = *opts;
  if (p->opts.world < 1 || p->opts.rank < 0 || p->opts.rank >= p->opts.world)
    SPMV_FAIL(SPMV_EINVAL, "spmv_plan: need 0 <= rank < world");
  if (p->opts.world > 1024) SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_plan: world > 1024");
  if (p->opts.hot_x > 0)
    SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_plan: the hot-column set (opts.hot_x) was removed");
  if (!(p->opts.l2_hit_ratio >= 0.0 && p->opts.l2_hit_ratio <= 1.0))
    SPMV_FAIL(SPMV_EINVAL, "spmv_plan: l2_hit_ratio must be in [0, 1]");
  int dev = p->opts.device;
  if (dev < 0) SPMV_CUDA(cudaGetDevice(&dev));
  p->device = dev;
  SPMV_CUDA(cudaSetDevice(dev));
  SPMV_CUDA(cudaStreamCreateWithFlags(&p->s, cudaStreamNonBlocking));
  p->world = p->opts.world;
  p->rank = p->opts.rank;
  p->n = A->n;
  p->nnz = A->nnz;
  p->off64 = A->nnz > (int64_t)INT32_MAX;
  p->A_rp32 = A->row_ptr32;
  p->A_rp64 = A->row_ptr64;
  p->A_col = A->col_idx;
  p->A_val = A->vals;
  spmv::plan_build(p, A, perm);
  *out = p;
  p = nullptr;
  }
  catch (const spmv::Err& e) {
    if (p) { spmv::plan_free(p); if (p->s) cudaStreamDestroy(p->s); delete p; }
    return e.st;
  }
  catch (...) {
    if (p) { spmv::plan_free(p); if (p->s) cudaStreamDestroy(p->s); delete p; }
    spmv::set_error("internal: exception in spmv_plan");
    return SPMV_EINVAL;
  }
  return SPMV_OK;
}

spmv_status spmv_permute(spmv_plan_t p, void* stream) {
  NvtxRange nvtx_("spmv_permute");
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_permute: NULL plan");
  use_device(p);
  spmv::plan_permute(p, S(stream));
  API_END
}

spmv_status spmv_permute_vec(spmv_plan_t p, const float* in, float* out, int inverse,
                             void* stream) {
  NvtxRange nvtx_("spmv_permute_vec");
  API_BEGIN
  if (!p || (p->n && (!in || !out))) SPMV_FAIL(SPMV_EINVAL, "spmv_permute_vec: NULL argument");
  if (p->n && in == out) SPMV_FAIL(SPMV_EINVAL, "spmv_permute_vec: in and out alias");
  use_device(p);
  spmv::permute_vec(p, in, out, inverse, S(stream));
  API_END
}

spmv_status spmv_pad_vec(spmv_plan_t p, const float* in, float* out, int to_padded,
                         void* stream) {
  API_BEGIN
  if (!p || (p->n && (!in || !out))) SPMV_FAIL(SPMV_EINVAL, "spmv_pad_vec: NULL argument");
  if (p->n && in == out) SPMV_FAIL(SPMV_EINVAL, "spmv_pad_vec: in and out alias");
  use_device(p);
  spmv::pad_vec(p, in, out, to_padded, S(stream));
  API_END
}

spmv_status spmv_exec(spmv_plan_t p, const float* x_B, float* y_B, void* stream) {
  NvtxRange nvtx_("spmv_exec");
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_exec: NULL plan");
  if (p->nrows && (!x_B || !y_B)) SPMV_FAIL(SPMV_EINVAL, "spmv_exec: NULL vector");
  use_device(p);
  spmv::exec(p, x_B, y_B, nullptr, nullptr, S(stream));
  API_END
}

spmv_status spmv_rabbitpp_gpu(const spmv_csr_t* A, const int32_t* perm_rabbit,
                              const int32_t* comm, int32_t* perm_out, void* stream) {
  NvtxRange nvtx_("spmv_rabbitpp_gpu");
  API_BEGIN
  if (!A || (A->n && (!perm_rabbit || !comm || !perm_out)))
    SPMV_FAIL(SPMV_EINVAL, "spmv_rabbitpp_gpu: NULL argument");
  if (A->n < 0 || A->nnz < 0 || (A->row_ptr32 == nullptr) == (A->row_ptr64 == nullptr) ||
      (A->nnz && !A->col_idx))
    SPMV_FAIL(SPMV_EINVAL, "spmv_rabbitpp_gpu: malformed CSR descriptor");
  if (A->n > (int64_t)INT32_MAX) SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_rabbitpp_gpu: n > INT32_MAX");
  spmv::rabbitpp_gpu(A, perm_rabbit, comm, perm_out, S(stream));
  API_END
}

spmv_status spmv_exec_spmm4(spmv_plan_t p, const float* X_B, float* Y_B, void* stream) {
  NvtxRange nvtx_("spmv_exec_spmm4");
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_spmm4: NULL plan");
  if (p->nrows && (!X_B || !Y_B)) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_spmm4: NULL matrix");
  use_device(p);
  spmv::exec_spmm4(p, X_B, Y_B, S(stream));
  API_END
}

spmv_status spmv_exec_coo(spmv_plan_t p, const float* x_B, float* y_B, void* stream) {
  NvtxRange nvtx_("spmv_exec_coo");
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_coo: NULL plan");
  if (p->nrows && (!x_B || !y_B)) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_coo: NULL vector");
  use_device(p);
  spmv::exec_coo(p, x_B, y_B, S(stream));
  API_END
}

spmv_status spmv_exec_scaled_bcast(spmv_plan_t p, const float* x_B, float* const* x_next,
                                   int n_next, const double* sumsq_in, double* sumsq_out,
                                   void* stream) {
  NvtxRange nvtx_("spmv_exec_scaled_bcast");
  API_BEGIN
  if (!p || !x_next) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_scaled_bcast: NULL argument");
  if (p->nrows && !x_B) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_scaled_bcast: NULL vector");
  if (n_next < 1 || n_next > 8 || n_next > p->world)
    SPMV_FAIL(SPMV_EINVAL, "spmv_exec_scaled_bcast: n_next must be in [1, min(world, 8)]");
  use_device(p);
  spmv::exec(p, x_B, nullptr, sumsq_in, sumsq_out, S(stream), x_next, n_next);
  API_END
}

spmv_status spmv_dev_alloc(int device, int64_t bytes, void** dev_ptr) {
  API_BEGIN
  if (!dev_ptr || bytes < 0) SPMV_FAIL(SPMV_EINVAL, "spmv_dev_alloc: bad argument");
  *dev_ptr = nullptr;
  SPMV_CUDA(cudaSetDevice(device));
  if (cudaMalloc(dev_ptr, (size_t)std::max<int64_t>(bytes, 256)) != cudaSuccess) {
    cudaGetLastError();
    SPMV_FAIL(SPMV_ENOMEM, "spmv_dev_alloc: cudaMalloc failed");
  }
  API_END
}

spmv_status spmv_dev_free(void* dev_ptr) {
  API_BEGIN
  if (dev_ptr) SPMV_CUDA(cudaFree(dev_ptr));
  API_END
}

spmv_status spmv_ipc_handle(const void* dev_ptr, void* handle) {
  API_BEGIN
  if (!dev_ptr || !handle) SPMV_FAIL(SPMV_EINVAL, "spmv_ipc_handle: NULL argument");
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "64-byte IPC handle");
  cudaIpcMemHandle_t h;
  SPMV_CUDA(cudaIpcGetMemHandle(&h, const_cast<void*>(dev_ptr)));
  std::memcpy(handle, &h, 64);
  API_END
}

spmv_status spmv_ipc_open(const void* handle, void** dev_ptr) {
  API_BEGIN
  if (!handle || !dev_ptr) SPMV_FAIL(SPMV_EINVAL, "spmv_ipc_open: NULL argument");
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, 64);
  SPMV_CUDA(cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess));
  API_END
}

spmv_status spmv_ipc_close(void* dev_ptr) {
  API_BEGIN
  if (!dev_ptr) SPMV_FAIL(SPMV_EINVAL, "spmv_ipc_close: NULL argument");
  SPMV_CUDA(cudaIpcCloseMemHandle(dev_ptr));
  API_END
}

spmv_status spmv_exec_scaled(spmv_plan_t p, const float* x_B, float* y_B,
                             const double* sumsq_in, double* sumsq_out, void* stream) {
  NvtxRange nvtx_("spmv_exec_scaled");
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_scaled: NULL plan");
  if (p->nrows && (!x_B || !y_B)) SPMV_FAIL(SPMV_EINVAL, "spmv_exec_scaled: NULL vector");
  use_device(p);
  spmv::exec(p, x_B, y_B, sumsq_in, sumsq_out, S(stream));
  API_END
}

spmv_status spmv_iterate(spmv_plan_t p, float* x_B, int iters, double* lambda_out,
                         void* stream) {
  NvtxRange nvtx_("spmv_iterate");
  API_BEGIN
  if (!p || (p->n && !x_B)) SPMV_FAIL(SPMV_EINVAL, "spmv_iterate: NULL argument");
  use_device(p);
  spmv::iterate(p, x_B, iters, lambda_out, S(stream));
  API_END
}

spmv_status spmv_scale_vec(const float* u, float* x, int64_t n, const double* sumsq_in,
                           void* stream) {
  API_BEGIN
  if (n < 0 || (n && (!u || !x))) SPMV_FAIL(SPMV_EINVAL, "spmv_scale_vec: bad argument");
  spmv::scale_vec(u, x, n, sumsq_in, S(stream));
  API_END
}

spmv_status spmv_iterate_finish(const float* u, float* x, int64_t n, const double* sumsq_dev,
                                double* lambda_out, void* stream) {
  API_BEGIN
  if (n < 0 || (n && (!u || !x)) || !sumsq_dev)
    SPMV_FAIL(SPMV_EINVAL, "spmv_iterate_finish: bad argument");
  spmv::iterate_finish(u, x, n, sumsq_dev, lambda_out, S(stream));
  API_END
}

spmv_status spmv_plan_info(spmv_plan_t p, spmv_plan_info_t* info) {
  API_BEGIN
  if (!p || !info) SPMV_FAIL(SPMV_EINVAL, "spmv_plan_info: NULL argument");
  std::memset(info, 0, sizeof(*info));
  info->n = p->n;
  info->nnz = p->nnz;
  info->row_begin = p->row_begin;
  info->row_end = p->row_end;
  info->nnz_local = p->nnz_local;
  info->x_len = p->x_len;
  info->x_stride = p->x_stride;
  info->y_offset = p->y_offset;
  info->n_tiles = p->K;
  info->n_warp_rows = p->n_warp;
  info->n_mid_rows = p->n_mid;
  info->n_cta_rows = p->n_cta;
  info->n_hub_rows = p->n_hub;
  info->n_hub_chunks = p->n_chunks;
  info->hot_prefix = p->H;
  info->offset_bytes = p->off64 ? 8 : 4;
  // P:96 with the real offset width: x (n reads... local rows), y, row_ptr, col, val
  info->ideal_bytes = 4 * p->n + 4 * p->nrows + (p->nrows + 1) * info->offset_bytes +
                      8 * p->nnz_local;
  if (p->world == 1) info->ideal_bytes = 8 * p->n + (p->n + 1) * info->offset_bytes + 8 * p->nnz;
  info->world = p->world;
  info->rank = p->rank;
  info->permuted = p->permuted ? 1 : 0;
  info->l2_window_bytes = (int32_t)p->l2_window_bytes;
  info->stream_evict_first = spmv::lane_ef_mode(p);
  info->exec_launches = spmv::exec_launches(p, false);
  info->spmm4_launches = spmv::spmm4_launches(p);
  info->hot_prefix_nnz = p->H_nnz;
  info->lane_nnz = p->lane_nnz;
  info->lane_waste_slots = p->lane_waste;
  info->lane_pred_gather = spmv::lane_pred_mode(p);
  API_END
}

spmv_status spmv_export_csr(spmv_plan_t p, int64_t* row_ptr, int32_t* col, float* val,
                            void* stream) {
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_export_csr: NULL plan");
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_export_csr before spmv_permute");
  use_device(p);
  cudaStream_t s = S(stream);
  if (row_ptr) {
    if (p->off64) {
      SPMV_CUDA(cudaMemcpyAsync(row_ptr, p->d_rp, 8 * (p->nrows + 1), cudaMemcpyDeviceToDevice, s));
    } else {
      // widen int32 -> int64 via host (introspection only)
      std::string buf(4 * (p->nrows + 1), '\0');
      SPMV_CUDA(cudaMemcpyAsync(&buf[0], p->d_rp, buf.size(), cudaMemcpyDeviceToHost, s));
      SPMV_CUDA(cudaStreamSynchronize(s));
      std::string w(8 * (p->nrows + 1), '\0');
      const int32_t* a = (const int32_t*)buf.data();
      int64_t* b = (int64_t*)&w[0];
      for (int64_t i = 0; i <= p->nrows; ++i) b[i] = a[i];
      SPMV_CUDA(cudaMemcpyAsync(row_ptr, w.data(), w.size(), cudaMemcpyHostToDevice, s));
      SPMV_CUDA(cudaStreamSynchronize(s));
    }
  }
  if (col && p->nnz_local)
    SPMV_CUDA(cudaMemcpyAsync(col, p->d_col, 4 * p->nnz_local, cudaMemcpyDeviceToDevice, s));
  if (val && p->nnz_local)
    SPMV_CUDA(cudaMemcpyAsync(val, p->d_val, 4 * p->nnz_local, cudaMemcpyDeviceToDevice, s));
  API_END
}

spmv_status spmv_export_bins(spmv_plan_t p, int32_t* tiles, int32_t* mid_rows, int32_t* warp_rows,
                             int32_t* cta_rows, int32_t* hub_rows, int32_t* chunk_row,
                             int32_t* chunk_idx, void* stream) {
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_export_bins: NULL plan");
  use_device(p);
  cudaStream_t s = S(stream);
  if (tiles) SPMV_CUDA(cudaMemcpyAsync(tiles, p->d_tiles, 4 * (p->K + 1), cudaMemcpyDeviceToDevice, s));
  if (mid_rows && p->n_mid)
    SPMV_CUDA(cudaMemcpyAsync(mid_rows, p->d_mid_rows, 4 * p->n_mid, cudaMemcpyDeviceToDevice, s));
  if (warp_rows && p->n_warp)
    SPMV_CUDA(cudaMemcpyAsync(warp_rows, p->d_warp_rows, 4 * p->n_warp, cudaMemcpyDeviceToDevice, s));
  if (cta_rows && p->n_cta)
    SPMV_CUDA(cudaMemcpyAsync(cta_rows, p->d_cta_rows, 4 * p->n_cta, cudaMemcpyDeviceToDevice, s));
  if (hub_rows && p->n_hub)
    SPMV_CUDA(cudaMemcpyAsync(hub_rows, p->d_hub_rows, 4 * p->n_hub, cudaMemcpyDeviceToDevice, s));
  if (chunk_row && p->n_chunks)
    SPMV_CUDA(cudaMemcpyAsync(chunk_row, p->d_chunk_row, 4 * p->n_chunks, cudaMemcpyDeviceToDevice, s));
  if (chunk_idx && p->n_chunks)
    SPMV_CUDA(cudaMemcpyAsync(chunk_idx, p->d_chunk_idx, 4 * p->n_chunks, cudaMemcpyDeviceToDevice, s));
  API_END
}

spmv_status spmv_export_partition(spmv_plan_t p, int64_t* bounds_host) {
  API_BEGIN
  if (!p || !bounds_host) SPMV_FAIL(SPMV_EINVAL, "spmv_export_partition: NULL argument");
  for (int k = 0; k <= p->world; ++k) bounds_host[k] = p->part[k];
  API_END
}

spmv_status spmv_export_inverse(spmv_plan_t p, int32_t* inv, void* stream) {
  API_BEGIN
  if (!p || (p->n && !inv)) SPMV_FAIL(SPMV_EINVAL, "spmv_export_inverse: NULL argument");
  use_device(p);
  if (p->n)
    SPMV_CUDA(cudaMemcpyAsync(inv, p->d_inv, 4 * p->n, cudaMemcpyDeviceToDevice, S(stream)));
  API_END
}

spmv_status spmv_export_coo_rows(spmv_plan_t p, int32_t* rows, void* stream) {
  API_BEGIN
  if (!p) SPMV_FAIL(SPMV_EINVAL, "spmv_export_coo_rows: NULL plan");
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_export_coo_rows before spmv_permute");
  use_device(p);
  spmv::export_coo_rows(p, rows, S(stream));
  API_END
}

spmv_status spmv_reset_persisting_l2(void* stream) {
  (void)stream;
  API_BEGIN
  SPMV_CUDA(cudaCtxResetPersistingL2Cache());
  API_END
}

void spmv_destroy(spmv_plan_t p) {
  if (!p) return;
  cudaSetDevice(p->device);
  cudaDeviceSynchronize();
  if (p->l2_limit_raised) {  // the window raised the device-wide persisting limit
    cudaCtxResetPersistingL2Cache();
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, p->l2_limit_before);
    cudaGetLastError();
  }
  spmv::plan_free(p);
  if (p->s) cudaStreamDestroy(p->s);
  delete p;
}

}  // extern "C"
