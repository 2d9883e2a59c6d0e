// spmv_iterate: power iteration, one GPU or row-block partitioned across ranks.
//
// Reading c22; north_star: "iterated SpMV (power iteration) is
// row-block partitioned on the reordered matrix, and each iteration exchanges
// x"; SURVEY §8(a9), §8(e).  Per step t (u_0 = x, s_0 = 1):
//   u_t = B u_{t-1} / s_{t-1}        spmv_exec_scaled (1/s folded into the SpMV)
//   s_t^2 = sum_rows u_t^2           fixed-order fp64 per rank, then all-reduce
//   exchange of the u_t row slices   all-gatherv (NCCL broadcasts / all-gather)
//                                    or peer stores from the SpMV itself
// and at the end x = fp32(u_T / s_T), lambda = s_T.  Everything above runs in
// this library: the caller passes a communicator (or a collective backend)
// and gets x and lambda back.
//
// NCCL is resolved at run time (dlsym): the communicator comes from the
// process's own libnccl (torch's, 2.28.9 here), so the library never links a
// second, possibly different, NCCL.
#include <dlfcn.h>

#include <chrono>
#include <cmath>
#include <cstdlib>
#include <mutex>
#include <thread>

#include "plan.cuh"

namespace spmv {
namespace {

__device__ __forceinline__ float alpha_of_ss(const double* ss) {
  if (!ss) return 1.f;
  const double v = *ss;
  return v > 0.0 ? (float)(1.0 / sqrt(v)) : 1.f;
}

__global__ void k_scale(const float* __restrict__ u, float* __restrict__ x, int64_t n,
                        const double* __restrict__ ss) {
  const float a = alpha_of_ss(ss);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    x[i] = __fmul_rn(u[i], a);
}

void launch_scale(const float* u, float* x, int64_t n, const double* ss, cudaStream_t s) {
  if (n <= 0) return;
  const int g = (int)std::min<int64_t>((n + 255) / 256, 148 * 16);
  k_scale<<<g, 256, 0, s>>>(u, x, n, ss);
  SPMV_LAUNCH_CHECK();
}

// ------------------------------------------------------------ NCCL (dlsym)
// Prototypes and enum values of nccl.h (NCCL 2.28.9: ncclFloat32 = 7,
// ncclFloat64 = 8, ncclSum = 0; ncclSuccess = 0).
struct Nccl {
  int (*all_reduce)(const void*, void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*broadcast)(const void*, void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*all_gather)(const void*, void*, size_t, int, void*, cudaStream_t) = nullptr;
  int (*group_start)() = nullptr;
  int (*group_end)() = nullptr;
  const char* (*error_string)(int) = nullptr;
  int (*async_error)(void*, int*) = nullptr;  // ncclCommGetAsyncError
  bool ok = false;
};
constexpr int kNcclInProgress = 7;  // ncclInProgress
constexpr int kNcclFloat32 = 7, kNcclFloat64 = 8, kNcclSum = 0;

const Nccl& nccl() {
  static Nccl N;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = RTLD_DEFAULT;
    if (!dlsym(h, "ncclAllReduce")) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    N.all_reduce = (decltype(N.all_reduce))dlsym(h, "ncclAllReduce");
    N.broadcast = (decltype(N.broadcast))dlsym(h, "ncclBroadcast");
    N.all_gather = (decltype(N.all_gather))dlsym(h, "ncclAllGather");
    N.group_start = (decltype(N.group_start))dlsym(h, "ncclGroupStart");
    N.group_end = (decltype(N.group_end))dlsym(h, "ncclGroupEnd");
    N.error_string = (decltype(N.error_string))dlsym(h, "ncclGetErrorString");
    N.async_error = (decltype(N.async_error))dlsym(h, "ncclCommGetAsyncError");
    N.ok = N.all_reduce && N.broadcast && N.all_gather && N.group_start && N.group_end;
  });
  return N;
}

struct NcclCtx {
  void* comm;
  int rank;
};

void nccl_fail(int r, const char* what) {
  const Nccl& N = nccl();
  set_error(std::string(what) + ": " + (N.error_string ? N.error_string(r) : "NCCL error"));
}

int nccl_allreduce(void* ctx, double* buf, int64_t count, void* stream) {
  const NcclCtx* c = (const NcclCtx*)ctx;
  const int r = nccl().all_reduce(buf, buf, (size_t)count, kNcclFloat64, kNcclSum, c->comm,
                                  (cudaStream_t)stream);
  if (r) nccl_fail(r, "ncclAllReduce");
  return r;
}

// all-gatherv in place: equal contiguous slices -> one ncclAllGather, else one
// ncclBroadcast per rank (root k sends x[b_k, b_k+1)) inside a group
int nccl_allgatherv(void* ctx, float* x, const int64_t* b, int world, void* stream) {
  const NcclCtx* c = (const NcclCtx*)ctx;
  const Nccl& N = nccl();
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t cnt0 = b[1] - b[0];
  bool equal = true;
  for (int k = 0; k < world; ++k) equal &= b[k + 1] - b[k] == cnt0;
  if (equal) {
    const int r = N.all_gather(x + b[c->rank], x + b[0], (size_t)cnt0, kNcclFloat32, c->comm, s);
    if (r) nccl_fail(r, "ncclAllGather");
    return r;
  }
  int r = N.group_start();
  for (int k = 0; k < world && !r; ++k)
    if (b[k + 1] > b[k])
      r = N.broadcast(x + b[k], x + b[k], (size_t)(b[k + 1] - b[k]), kNcclFloat32, k, c->comm, s);
  const int r2 = N.group_end();
  if (r || r2) nccl_fail(r ? r : r2, "grouped ncclBroadcast");
  return r ? r : r2;
}

// Wait for the step loop with NCCL's asynchronous error state polled: a
// failed or aborted peer turns into SPMV_ENCCL instead of a hang, and so does
// a loop that has not finished after SPMV_NCCL_TIMEOUT_S seconds (600).
void wait_nccl(void* comm, cudaStream_t s) {
  const Nccl& N = nccl();
  double limit = 600.0;
  if (const char* e = getenv("SPMV_NCCL_TIMEOUT_S")) limit = atof(e);
  const auto t0 = std::chrono::steady_clock::now();
  for (;;) {
    const cudaError_t q = cudaStreamQuery(s);
    if (q == cudaSuccess) return;
    if (q != cudaErrorNotReady) SPMV_CUDA(q);
    int st = 0;
    if (N.async_error && N.async_error(comm, &st) == 0 && st != 0 && st != kNcclInProgress) {
      nccl_fail(st, "NCCL asynchronous error");
      throw Err{SPMV_ENCCL};
    }
    if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > limit)
      SPMV_FAIL(SPMV_ENCCL, "spmv_iterate: collectives did not complete within SPMV_NCCL_TIMEOUT_S");
    std::this_thread::sleep_for(std::chrono::microseconds(200));
  }
}

}  // namespace

void scale_vec(const float* u, float* x, int64_t n, const double* ss, cudaStream_t s) {
  launch_scale(u, x, n, ss, s);
}

void iterate_finish(const float* u, float* x, int64_t n, const double* ss, double* lambda,
                    cudaStream_t s) {
  launch_scale(u, x, n, ss, s);
  double h = 0.0;
  if (ss) SPMV_CUDA(cudaMemcpyAsync(&h, ss, sizeof(double), cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  if (lambda) *lambda = ss ? std::sqrt(h) : 0.0;
}

void iterate(spmv_plan_s* p, float* x, int iters, double* lambda, cudaStream_t s) {
  if (iters < 1) SPMV_FAIL(SPMV_EINVAL, "iters must be >= 1");
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_iterate before spmv_permute");
  const int G = p->world;
  // SPMV_FORCE_COLL=1 (test knob): run the collectives even for world == 1
  // (an all-reduce / all-gatherv over one rank is the identity), so the NCCL
  // path is exercised on a one-GPU box
  bool force = false;
  if (const char* e = getenv("SPMV_FORCE_COLL")) force = atoi(e) != 0;
  const bool coll = G > 1 || force;
  const bool peer = G > 1 && p->opts.exchange == SPMV_EXCHANGE_PEER;
  NcclCtx nctx{p->opts.nccl_comm, p->rank};
  spmv_coll_t c{};
  if (coll) {
    if (p->has_coll) {
      c = p->coll;
    } else {
      if (!p->opts.nccl_comm)
        SPMV_FAIL(SPMV_EINVAL, "spmv_iterate: world > 1 needs opts.nccl_comm or spmv_set_coll");
      if (!nccl().ok) SPMV_FAIL(SPMV_ENCCL, "spmv_iterate: libnccl.so.2 not found in the process");
      c.ctx = &nctx;
      c.allreduce_sum_f64 = nccl_allreduce;
      c.allgatherv_f32 = nccl_allgatherv;
    }
    if (peer && (int)p->peers.size() != 2 * G)
      SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_iterate: SPMV_EXCHANGE_PEER needs spmv_set_peers");
  }
  // slice bounds of the exchange in the x layout
  std::vector<int64_t> xb(G + 1);
  for (int k = 0; k <= G; ++k)
    xb[k] = padded(p) ? (int64_t)k * p->x_stride : p->part[k];
  const int64_t xl = p->x_len;
  float* a = x;  // current u
  float* b = nullptr;
  if (!peer) {
    if (!p->d_u) {
      void* q = nullptr;
      if (cudaMalloc(&q, sizeof(float) * (size_t)std::max<int64_t>(xl, 1)) != cudaSuccess) {
        cudaGetLastError();
        SPMV_FAIL(SPMV_ENOMEM, "iterate buffer allocation failed");
      }
      p->d_u = (float*)q;
    }
    b = p->d_u;
  } else {
    a = p->peers[p->rank];
    if (xl) SPMV_CUDA(cudaMemcpyAsync(a, x, 4 * xl, cudaMemcpyDeviceToDevice, s));
  }
  const double* sin = nullptr;
  int cur = 0;
  struct Alt {  // window sizing for two alternating x buffers, for this call only
    spmv_plan_s* p;
    explicit Alt(spmv_plan_s* q) : p(q) { p->win_alternating = true; p->win_ptr = nullptr; }
    ~Alt() { p->win_alternating = false; p->win_ptr = nullptr; }
  } alt_(p);
  for (int t = 0; t < iters; ++t) {
    double* sout = p->d_ss + (t & 1);
    if (peer) {
      exec(p, a, nullptr, sin, sout, s, p->peers.data() + (1 - cur) * G, G);
    } else {
      exec(p, a, b + p->y_offset, sin, sout, s);
    }
    if (coll) {
      if (c.allreduce_sum_f64(c.ctx, sout, 1, s))
        SPMV_FAIL(SPMV_ENCCL, std::string("spmv_iterate: all-reduce failed: ") + get_error());
      if (!peer && c.allgatherv_f32(c.ctx, b, xb.data(), G, s))
        SPMV_FAIL(SPMV_ENCCL, std::string("spmv_iterate: all-gatherv failed: ") + get_error());
    }
    sin = sout;
    if (peer) {
      cur ^= 1;
      a = p->peers[cur * G + p->rank];
    } else {
      std::swap(a, b);
    }
  }
  if (coll && !p->has_coll) wait_nccl(p->opts.nccl_comm, s);
  iterate_finish(a, x, xl, sin, lambda, s);
}

}  // namespace spmv

extern "C" {

spmv_status spmv_set_coll(spmv_plan_t p, const spmv_coll_t* coll) {
  if (!p) {
    spmv::set_error("spmv_set_coll: NULL plan");
    return SPMV_EINVAL;
  }
  if (coll && (!coll->allreduce_sum_f64 || !coll->allgatherv_f32)) {
    spmv::set_error("spmv_set_coll: both collective functions are required");
    return SPMV_EINVAL;
  }
  p->has_coll = coll != nullptr;
  if (coll) p->coll = *coll;
  return SPMV_OK;
}

spmv_status spmv_set_peers(spmv_plan_t p, float* const* bufs, int world) {
  if (!p || (world && !bufs)) {
    spmv::set_error("spmv_set_peers: NULL argument");
    return SPMV_EINVAL;
  }
  if (world != p->world || world > 8) {
    spmv::set_error("spmv_set_peers: world must equal the plan's world and be <= 8");
    return SPMV_EINVAL;
  }
  for (int i = 0; i < 2 * world; ++i)
    if (!bufs[i]) {
      spmv::set_error("spmv_set_peers: NULL buffer");
      return SPMV_EINVAL;
    }
  p->peers.assign(bufs, bufs + 2 * world);
  return SPMV_OK;
}

}  // extern "C"
