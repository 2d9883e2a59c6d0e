// spmv_exec_spmm4: SpMM-CSR with four dense right-hand sides on the reordered
// matrix, Y_B = B X_B, X_B / Y_B row-major [rows][4] (the
// paper's Table IV "SpMM-CSR-4").
//
// Same plan, same row classes, same canonical per-row summation order as
// spmv_exec (include/spmv.h), applied to each of the four
// columns independently: column k of Y_B is bitwise equal to
// spmv_exec(B, X_B[:, k]).  What changes is the gather: one 16-byte row of X
// per non-zero instead of a 4-byte element, so community order
// matters 4x more per line and the ideal traffic becomes
// 8 NZ + (N+1) w_off + 16 N (X) + 16 N (Y)  ("compulsory traffic
// updated according to the kernel").
//
//   k_lane4       rows with L <= 32, one lane per row (sequential order),
//                 col/val streamed with 256-bit loads like k_lane;
//   k_warp_rows4  32 < L <= 2048, warp per row (32 strided partials + tree);
//   k_cta_rows4   2048 < L <= 16384, CTA per row (256 partials + tree);
//   k_hub_chunk4 / k_hub_fix4  L > 16384: 16384-entry chunks, fp64 combine.
#include <algorithm>
#include <cstdlib>

#include "plan.cuh"

namespace spmv {
void exec_streams(spmv_plan_s* p);  // exec.cu: lazily creates the plan's aux streams

namespace {

constexpr int L4_THREADS = 256;

__device__ __forceinline__ float4 ldx4(const float* X, int c) {
  return __ldg(reinterpret_cast<const float4*>(X) + c);
}

__device__ __forceinline__ void fma4(float4& s, float v, const float4& x) {
  s.x = __fadd_rn(s.x, __fmul_rn(v, x.x));
  s.y = __fadd_rn(s.y, __fmul_rn(v, x.y));
  s.z = __fadd_rn(s.z, __fmul_rn(v, x.z));
  s.w = __fadd_rn(s.w, __fmul_rn(v, x.w));
}

__device__ __forceinline__ float tree32(float s) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  return s;
}

template <int EF>
__device__ __forceinline__ void ld8_i(const int32_t* p, int (&r)[8]) {
  if constexpr (EF)
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.s32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7])
        : "l"(p));
  else
    asm("ld.global.nc.L1::no_allocate.v8.s32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7])
        : "l"(p));
}

template <int EF>
__device__ __forceinline__ void ld8_f(const float* p, float (&r)[8]) {
  if constexpr (EF)
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]),
          "=f"(r[7])
        : "l"(p));
  else
    asm("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]),
          "=f"(r[7])
        : "l"(p));
}

// lane per row, L <= SHORT_MAX, sequential: the association of k_lane.  As
// there, slots of a chunk outside the row read a valid X row (a neighbouring
// row's column or the zero tail padding) replaced by 0, so they contribute
// v * 0 = +-0 for a finite neighbouring value; when the plan holds a
// non-finite value (EF & 4) the value is masked too (0 * 0 = +0), so an Inf /
// NaN never reaches this row (Alg. 1).  The running sum is unchanged either
// way (it starts at +0 and is never -0): the loop is branch-free and both
// chunks of a 16-entry row are in flight at once.
template <typename OT, int EF, int MINB, int UNR>
__global__ void __launch_bounds__(L4_THREADS, MINB)
    k_lane4(const OT* __restrict__ rp, const int32_t* __restrict__ col,
            const float* __restrict__ val, const float* __restrict__ X, float* __restrict__ Y,
            int64_t nrows) {
  const int64_t stride = (int64_t)gridDim.x * L4_THREADS;
  for (int64_t r = (int64_t)blockIdx.x * L4_THREADS + threadIdx.x; r < nrows; r += stride) {
    const OT a = rp[r], e = rp[r + 1];
    const int L = (int)(e - a);
    if (L > SHORT_MAX) continue;  // MID / CTA / hub kernels
    float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
    const int32_t* cp = col + (a & ~(OT)7);
    const float* vp = val + (a & ~(OT)7);
    const int lo = (int)(a & 7), hi = lo + L;
#pragma unroll UNR
    for (int k = 0; k < hi; k += 8) {
      int cc[8];
      float vv[8];
      ld8_i<EF & 1>(cp + k, cc);
      ld8_f<EF & 1>(vp + k, vv);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const float4 xg = ldx4(X, cc[i]);
        const bool in = k + i >= lo && k + i < hi;
        const float4 xv = in ? xg : make_float4(0.f, 0.f, 0.f, 0.f);
        fma4(s, ((EF & 4) != 0 && !in) ? 0.f : vv[i], xv);
      }
    }
    reinterpret_cast<float4*>(Y)[r] = s;
  }
}

template <typename OT>
__global__ void __launch_bounds__(256)
    k_warp_rows4(const OT* __restrict__ rp, const int32_t* __restrict__ col,
                 const float* __restrict__ val, const float* __restrict__ X,
                 float* __restrict__ Y, const int32_t* __restrict__ rows, int64_t nrows) {
  const int lane = threadIdx.x & 31;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; q < nrows; q += W) {
    const int r = rows[q];
    const int64_t b = (int64_t)rp[r];
    const int L = (int)((int64_t)rp[r + 1] - b);
    float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
    const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int j = lane; j < L; j += 128) {  // four gathers in flight, ragged end guarded (+0)
      const bool p1 = j + 32 < L, p2 = j + 64 < L, p3 = j + 96 < L;
      const int c0 = __ldcs(col + b + j), c1 = p1 ? __ldcs(col + b + j + 32) : 0,
                c2 = p2 ? __ldcs(col + b + j + 64) : 0, c3 = p3 ? __ldcs(col + b + j + 96) : 0;
      const float v0 = __ldcs(val + b + j), v1 = p1 ? __ldcs(val + b + j + 32) : 0.f,
                  v2 = p2 ? __ldcs(val + b + j + 64) : 0.f, v3 = p3 ? __ldcs(val + b + j + 96) : 0.f;
      const float4 x0 = ldx4(X, c0), x1 = p1 ? ldx4(X, c1) : z4, x2 = p2 ? ldx4(X, c2) : z4,
                   x3 = p3 ? ldx4(X, c3) : z4;
      fma4(s, v0, x0);
      fma4(s, v1, x1);
      fma4(s, v2, x2);
      fma4(s, v3, x3);
    }
    s.x = tree32(s.x);
    s.y = tree32(s.y);
    s.z = tree32(s.z);
    s.w = tree32(s.w);
    if (lane == 0) reinterpret_cast<float4*>(Y)[r] = s;
  }
}

// canonical W = 256 sum of entries [b, b + L) (same tree as exec.cu cta_sum256)
__device__ __forceinline__ float4 cta_sum256x4(const int32_t* __restrict__ col,
                                               const float* __restrict__ val,
                                               const float* __restrict__ X, int64_t b,
                                               int64_t L, float4* red) {
  const int tid = threadIdx.x;
  float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t t = tid; t < L; t += 1024) {  // ragged end guarded (+0), as k_warp_rows4
    const bool p1 = t + 256 < L, p2 = t + 512 < L, p3 = t + 768 < L;
    const int c0 = __ldcs(col + b + t), c1 = p1 ? __ldcs(col + b + t + 256) : 0,
              c2 = p2 ? __ldcs(col + b + t + 512) : 0, c3 = p3 ? __ldcs(col + b + t + 768) : 0;
    const float v0 = __ldcs(val + b + t), v1 = p1 ? __ldcs(val + b + t + 256) : 0.f,
                v2 = p2 ? __ldcs(val + b + t + 512) : 0.f, v3 = p3 ? __ldcs(val + b + t + 768) : 0.f;
    const float4 x0 = ldx4(X, c0), x1 = p1 ? ldx4(X, c1) : z4, x2 = p2 ? ldx4(X, c2) : z4,
                 x3 = p3 ? ldx4(X, c3) : z4;
    fma4(s, v0, x0);
    fma4(s, v1, x1);
    fma4(s, v2, x2);
    fma4(s, v3, x3);
  }
  red[tid] = s;
  __syncthreads();
#pragma unroll
  for (int o = 128; o >= 32; o >>= 1) {
    if (tid < o) {
      float4 a = red[tid];
      const float4 c = red[tid + o];
      a.x = __fadd_rn(a.x, c.x);
      a.y = __fadd_rn(a.y, c.y);
      a.z = __fadd_rn(a.z, c.z);
      a.w = __fadd_rn(a.w, c.w);
      red[tid] = a;
    }
    __syncthreads();
  }
  float4 r = make_float4(0.f, 0.f, 0.f, 0.f);
  if (tid < 32) {
    r = red[tid];
    r.x = tree32(r.x);
    r.y = tree32(r.y);
    r.z = tree32(r.z);
    r.w = tree32(r.w);
  }
  return r;  // valid in thread 0
}

template <typename OT>
__global__ void __launch_bounds__(256)
    k_cta_rows4(const OT* __restrict__ rp, const int32_t* __restrict__ col,
                const float* __restrict__ val, const float* __restrict__ X, float* __restrict__ Y,
                const int32_t* __restrict__ rows) {
  __shared__ float4 red[256];
  const int r = rows[blockIdx.x];
  const int64_t b = (int64_t)rp[r], L = (int64_t)rp[r + 1] - b;
  const float4 s = cta_sum256x4(col, val, X, b, L, red);
  if (threadIdx.x == 0) reinterpret_cast<float4*>(Y)[r] = s;
}

template <typename OT>
__global__ void __launch_bounds__(256)
    k_hub_chunk4(const OT* __restrict__ rp, const int32_t* __restrict__ col,
                 const float* __restrict__ val, const float* __restrict__ X,
                 const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_idx,
                 double* __restrict__ part) {
  __shared__ float4 red[256];
  const int c = blockIdx.x;
  const int r = chunk_row[c];
  const int64_t rb = (int64_t)rp[r], L = (int64_t)rp[r + 1] - rb;
  const int64_t b = rb + (int64_t)chunk_idx[c] * HUB_CHUNK;
  const int64_t m = min((int64_t)HUB_CHUNK, rb + L - b);
  const float4 s = cta_sum256x4(col, val, X, b, m, red);
  if (threadIdx.x == 0) {
    part[4 * c + 0] = (double)s.x;
    part[4 * c + 1] = (double)s.y;
    part[4 * c + 2] = (double)s.z;
    part[4 * c + 3] = (double)s.w;
  }
}

__global__ void k_hub_fix4(const int32_t* __restrict__ hub_rows,
                           const int32_t* __restrict__ choff, int64_t nh,
                           const double* __restrict__ part, float* __restrict__ Y) {
  const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (h >= nh) return;
  double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
  for (int c = choff[h]; c < choff[h + 1]; ++c) {
    a0 += part[4 * c + 0];
    a1 += part[4 * c + 1];
    a2 += part[4 * c + 2];
    a3 += part[4 * c + 3];
  }
  reinterpret_cast<float4*>(Y)[hub_rows[h]] = make_float4((float)a0, (float)a1, (float)a2, (float)a3);
}

int sm_count(int dev) {
  static int n = 0;
  if (!n) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n > 0 ? n : 148;
}

template <typename OT>
void spmm4_typed(spmv_plan_s* p, const float* X, float* Y, cudaStream_t s) {
  const OT* rp = (const OT*)p->d_rp;
  const int sms = sm_count(p->device);
  if (p->nrows) {
    const int64_t blocks = (p->nrows + L4_THREADS - 1) / L4_THREADS;
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)sms * 32));
    // shape: 0 = 2 chunks in flight, 2 CTAs/SM; 1 = 2 chunks, 3 CTAs/SM (80
    // registers, default: SBM 0.178 vs 0.189 ms, RMAT-26 6.74 vs 7.23 ms, r41);
    // 2 = 1 chunk, 4 CTAs/SM (SPMV_L4_V dev knob)
    int v = 1;
    if (const char* e = getenv("SPMV_L4_V")) v = std::min(2, std::max(0, atoi(e)));
    // EF bit 0: evict_first stream; bit 2: the plan holds a non-finite value,
    // so foreign slots' values are masked too (exec.cu lane_row_sum)
    const int ef = (p->opts.evict_first && p->stream_ef ? 1 : 0) | (p->val_nonfinite ? 4 : 0);
    auto pick = [&](auto k0, auto k1, auto k4, auto k5) {
      return ef == 1 ? k1 : ef == 4 ? k4 : ef == 5 ? k5 : k0;
    };
    auto k = v == 2 ? pick(k_lane4<OT, 0, 4, 1>, k_lane4<OT, 1, 4, 1>, k_lane4<OT, 4, 4, 1>,
                           k_lane4<OT, 5, 4, 1>)
           : v == 1 ? pick(k_lane4<OT, 0, 3, 2>, k_lane4<OT, 1, 3, 2>, k_lane4<OT, 4, 3, 2>,
                           k_lane4<OT, 5, 3, 2>)
                    : pick(k_lane4<OT, 0, 2, 2>, k_lane4<OT, 1, 2, 2>, k_lane4<OT, 4, 2, 2>,
                           k_lane4<OT, 5, 2, 2>);
    k<<<g, L4_THREADS, 0, s>>>(rp, p->d_col, p->d_val, X, Y, p->nrows);
  }
  cudaStream_t s1 = s, s2 = s;
  const bool conc = p->conc && (p->n_mid > 0 || p->n_cta > 0 || p->n_chunks > 0);
  if (conc) {
    SPMV_CUDA(cudaEventRecord(p->ev_fork, s));
    s1 = p->aux[0];
    s2 = p->aux[1];
    SPMV_CUDA(cudaStreamWaitEvent(s1, p->ev_fork, 0));
    SPMV_CUDA(cudaStreamWaitEvent(s2, p->ev_fork, 0));
  }
  if (p->n_mid) {
    const unsigned g = (unsigned)std::min<int64_t>((p->n_mid + 7) / 8, (int64_t)sms * 16);
    k_warp_rows4<OT><<<g, 256, 0, s1>>>(rp, p->d_col, p->d_val, X, Y, p->d_mid_rows, p->n_mid);
  }
  if (p->n_cta)
    k_cta_rows4<OT><<<(unsigned)p->n_cta, 256, 0, s2>>>(rp, p->d_col, p->d_val, X, Y,
                                                        p->d_cta_rows);
  if (p->n_chunks) {
    k_hub_chunk4<OT><<<(unsigned)p->n_chunks, 256, 0, s2>>>(rp, p->d_col, p->d_val, X,
                                                            p->d_chunk_row, p->d_chunk_idx,
                                                            p->d_chunk_part4);
    k_hub_fix4<<<(unsigned)((p->n_hub + 127) / 128), 128, 0, s2>>>(
        p->d_hub_rows, p->d_hub_choff, p->n_hub, p->d_chunk_part4, Y);
  }
  if (conc) {
    SPMV_CUDA(cudaEventRecord(p->ev_join[0], s1));
    SPMV_CUDA(cudaEventRecord(p->ev_join[1], s2));
    SPMV_CUDA(cudaStreamWaitEvent(s, p->ev_join[0], 0));
    SPMV_CUDA(cudaStreamWaitEvent(s, p->ev_join[1], 0));
  }
  SPMV_LAUNCH_CHECK();
}

}  // namespace

void exec_spmm4(spmv_plan_s* p, const float* X, float* Y, cudaStream_t s) {
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_exec_spmm4 before spmv_permute");
  if (((uintptr_t)X & 15) || ((uintptr_t)Y & 15))
    SPMV_FAIL(SPMV_EINVAL, "spmv_exec_spmm4: X_B and Y_B must be 16-byte aligned");
  if (p->n_chunks && !p->d_chunk_part4) {
    void* q = nullptr;
    if (cudaMalloc(&q, sizeof(double) * 4 * (size_t)p->n_chunks) != cudaSuccess) {
      cudaGetLastError();
      SPMV_FAIL(SPMV_ENOMEM, "spmv_exec_spmm4: chunk partial allocation failed");
    }
    p->d_chunk_part4 = (double*)q;
  }
  exec_streams(p);
  if (p->off64) spmm4_typed<int64_t>(p, X, Y, s);
  else spmm4_typed<int32_t>(p, X, Y, s);
}

int spmm4_launches(const spmv_plan_s* p) {
  return (p->nrows ? 1 : 0) + (p->n_mid ? 1 : 0) + (p->n_cta ? 1 : 0) + (p->n_chunks ? 2 : 0);
}

}  // namespace spmv
