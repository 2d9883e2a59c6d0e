// spmv_exec / spmv_exec_scaled / spmv_iterate: the hot path.
//
// Alg. 1 of the paper:  Y[row] += values[i] * X[coords[i]].
// B200 design:
//   k_stream     one CTA per stream tile (TILE_D = 2048 rows+entries, row
//                aligned).  One elected thread moves the tile's col/val slice
//                global->shared with two cp.async.bulk copies (TMA bulk engine)
//                carrying an L2 evict_first policy and completing on an
//                mbarrier; all threads then gather x through L2 (__ldg),
//                form the fp32 products into a bank-padded product array, and
//                reduce rows in the canonical order of include/spmv.h: thread
//                per row (L <= 32, sequential) or warp per row (32 < L <=
//                2048, 32 strided partials + xor tree).  y is written once,
//                coalesced.
//   k_cta_rows   one CTA per row, 2048 < L <= 16384 (256 strided partials + tree).
//   k_hub_chunk  one CTA per 16384-entry chunk of a hub row (merge-path split);
//   k_hub_fix    fp64 combine of the chunk sums in chunk order.
//   k_ss_final   fixed-order fp64 sum of per-tile / per-row y^2 partials
//                (power iteration norm; deterministic).
// No tensor cores: SpMV is not a dense contraction (AI <= 0.25 flop/B).
#include <cmath>

#include "plan.cuh"

namespace spmv {
namespace {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ uint64_t l2_policy(int evict_first) {
  uint64_t pol;
  if (evict_first)
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  else
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes,
                                         uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint "
      "[%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

__device__ __forceinline__ float alpha_of(const double* ss_in) {
  if (!ss_in) return 1.f;
  double v = *ss_in;
  return v > 0.0 ? (float)(1.0 / sqrt(v)) : 1.f;
}

// bank-padded index of the product array (one pad word per 32)
__device__ __forceinline__ int pidx(int j) { return j + (j >> 5); }

constexpr int ST_THREADS = 256;
constexpr int PROD_LEN = TILE_BUF + TILE_BUF / 32 + 1;

template <bool SS>
__device__ __forceinline__ void block_sum_store(double acc, double* out) {
  __shared__ double wss[32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane == 0) wss[w] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += wss[i];
    *out = s;
  }
}

template <typename OT, bool SS>
__global__ void __launch_bounds__(ST_THREADS)
    k_stream(const OT* __restrict__ rp, const int32_t* __restrict__ col,
             const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
             const int32_t* __restrict__ tiles, const double* __restrict__ ss_in,
             double* __restrict__ tile_ss, int evict_first) {
  extern __shared__ __align__(16) unsigned char smraw[];
  int32_t* col_s = (int32_t*)smraw;                 // [TILE_BUF], reused as res_s
  float* val_s = (float*)(col_s + TILE_BUF);        // [TILE_BUF]
  float* prod_s = val_s + TILE_BUF;                 // [PROD_LEN]
  __shared__ __align__(8) uint64_t bar;
  __shared__ int mid_n;
  __shared__ int32_t mid_s[TILE_D / (SHORT_MAX + 1) + 2];
  float* res_s = (float*)col_s;

  const int k = blockIdx.x, tid = threadIdx.x;
  const int r0 = tiles[k], r1 = tiles[k + 1];
  if (r0 == r1) {
    if (SS && tid == 0) tile_ss[k] = 0.0;
    return;
  }
  const float alpha = alpha_of(ss_in);
  const int64_t e0 = (int64_t)rp[r0];
  const int64_t lastb = (int64_t)rp[r1 - 1], eend = (int64_t)rp[r1];
  const bool last_long = (eend - lastb) > STREAM_MAX;
  const int rend = last_long ? r1 - 1 : r1;
  const int64_t e1 = last_long ? lastb : eend;
  const int64_t a0 = e0 & ~3ll, a1 = (e1 + 3) & ~3ll;
  const int cnt = (int)(e1 - e0), sh = (int)(e0 - a0);
  if (tid == 0) {
    mid_n = 0;
    if (a1 > a0) {
      mbar_init(&bar, 1);
      const uint32_t bytes = (uint32_t)((a1 - a0) * 4);
      const uint64_t pol = l2_policy(evict_first);
      mbar_expect_tx(&bar, 2 * bytes);
      bulk_g2s(col_s, col + a0, bytes, &bar, pol);
      bulk_g2s(val_s, val + a0, bytes, &bar, pol);
    }
  }
  __syncthreads();
  if (a1 > a0) mbar_wait(&bar, 0);

  // products p_j = val_j * x[col_j] (fp32, rounded once)
  int i = tid;
  for (; i + 3 * ST_THREADS < cnt; i += 4 * ST_THREADS) {
    int c0 = col_s[sh + i], c1 = col_s[sh + i + ST_THREADS];
    int c2 = col_s[sh + i + 2 * ST_THREADS], c3 = col_s[sh + i + 3 * ST_THREADS];
    float x0 = __ldg(x + c0), x1 = __ldg(x + c1), x2 = __ldg(x + c2), x3 = __ldg(x + c3);
    prod_s[pidx(i)] = __fmul_rn(val_s[sh + i], x0);
    prod_s[pidx(i + ST_THREADS)] = __fmul_rn(val_s[sh + i + ST_THREADS], x1);
    prod_s[pidx(i + 2 * ST_THREADS)] = __fmul_rn(val_s[sh + i + 2 * ST_THREADS], x2);
    prod_s[pidx(i + 3 * ST_THREADS)] = __fmul_rn(val_s[sh + i + 3 * ST_THREADS], x3);
  }
  for (; i < cnt; i += ST_THREADS) prod_s[pidx(i)] = __fmul_rn(val_s[sh + i], __ldg(x + col_s[sh + i]));
  __syncthreads();

  // short rows: thread per row, sequential (canonical W = 1)
  for (int r = r0 + tid; r < rend; r += ST_THREADS) {
    const int b = (int)((int64_t)rp[r] - e0);
    const int L = (int)((int64_t)rp[r + 1] - (int64_t)rp[r]);
    if (L <= SHORT_MAX) {
      float s = 0.f;
      for (int t = 0; t < L; ++t) s = __fadd_rn(s, prod_s[pidx(b + t)]);
      res_s[r - r0] = s;
    } else {
      mid_s[atomicAdd(&mid_n, 1)] = r;
    }
  }
  __syncthreads();
  // medium rows: warp per row (canonical W = 32)
  const int warp = tid >> 5, lane = tid & 31;
  for (int q = warp; q < mid_n; q += ST_THREADS / 32) {
    const int r = mid_s[q];
    const int b = (int)((int64_t)rp[r] - e0);
    const int L = (int)((int64_t)rp[r + 1] - (int64_t)rp[r]);
    float s = 0.f;
    for (int t = lane; t < L; t += 32) s = __fadd_rn(s, prod_s[pidx(b + t)]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    if (lane == 0) res_s[r - r0] = s;
  }
  __syncthreads();
  double acc = 0.0;
  for (int r = r0 + tid; r < rend; r += ST_THREADS) {
    const float v = __fmul_rn(res_s[r - r0], alpha);
    y[r] = v;
    if (SS) acc += (double)v * (double)v;
  }
  if (SS) block_sum_store<SS>(acc, tile_ss + k);
}

// canonical W = 256 sum of entries [b, b + L) of a row (L >= 256 assumed by class)
__device__ __forceinline__ float cta_sum256(const int32_t* __restrict__ col,
                                            const float* __restrict__ val,
                                            const float* __restrict__ x, int64_t b, int64_t L,
                                            float* red) {
  const int tid = threadIdx.x;
  float s = 0.f;
#pragma unroll 8
  for (int64_t t = tid; t < L; t += 256) {
    const int c = __ldcs(col + b + t);
    const float v = __ldcs(val + b + t);
    s = __fadd_rn(s, __fmul_rn(v, __ldg(x + c)));
  }
  red[tid] = s;
  __syncthreads();
#pragma unroll
  for (int o = 128; o >= 32; o >>= 1) {
    if (tid < o) red[tid] = __fadd_rn(red[tid], red[tid + o]);
    __syncthreads();
  }
  float r = 0.f;
  if (tid < 32) {
    r = red[tid];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) r = __fadd_rn(r, __shfl_xor_sync(0xffffffffu, r, o));
  }
  return r;  // valid in thread 0
}

template <typename OT, bool SS>
__global__ void __launch_bounds__(256)
    k_cta_rows(const OT* __restrict__ rp, const int32_t* __restrict__ col,
               const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
               const int32_t* __restrict__ rows, const double* __restrict__ ss_in,
               double* __restrict__ row_ss) {
  __shared__ float red[256];
  const int r = rows[blockIdx.x];
  const int64_t b = (int64_t)rp[r], L = (int64_t)rp[r + 1] - b;
  const float s = cta_sum256(col, val, x, b, L, red);
  if (threadIdx.x == 0) {
    const float v = __fmul_rn(s, alpha_of(ss_in));
    y[r] = v;
    if (SS) row_ss[blockIdx.x] = (double)v * (double)v;
  }
}

template <typename OT>
__global__ void __launch_bounds__(256)
    k_hub_chunk(const OT* __restrict__ rp, const int32_t* __restrict__ col,
                const float* __restrict__ val, const float* __restrict__ x,
                const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_idx,
                double* __restrict__ part) {
  __shared__ float red[256];
  const int c = blockIdx.x;
  const int r = chunk_row[c];
  const int64_t rb = (int64_t)rp[r], L = (int64_t)rp[r + 1] - rb;
  const int64_t b = rb + (int64_t)chunk_idx[c] * HUB_CHUNK;
  const int64_t m = min((int64_t)HUB_CHUNK, rb + L - b);
  const float s = cta_sum256(col, val, x, b, m, red);
  if (threadIdx.x == 0) part[c] = (double)s;
}

template <bool SS>
__global__ void k_hub_fix(const int32_t* __restrict__ hub_rows, const int32_t* __restrict__ choff,
                          int64_t nh, const double* __restrict__ part,
                          const double* __restrict__ ss_in, float* __restrict__ y,
                          double* __restrict__ hub_ss) {
  const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (h >= nh) return;
  double acc = 0.0;
  for (int c = choff[h]; c < choff[h + 1]; ++c) acc += part[c];
  const float v = __fmul_rn((float)acc, alpha_of(ss_in));
  y[hub_rows[h]] = v;
  if (SS) hub_ss[h] = (double)v * (double)v;
}

__global__ void __launch_bounds__(1024)
    k_ss_final(const double* __restrict__ a, int64_t na, const double* __restrict__ b, int64_t nb,
               const double* __restrict__ c, int64_t nc, double* __restrict__ out) {
  double acc = 0.0;
  for (int64_t i = threadIdx.x; i < na; i += 1024) acc += a[i];
  for (int64_t i = threadIdx.x; i < nb; i += 1024) acc += b[i];
  for (int64_t i = threadIdx.x; i < nc; i += 1024) acc += c[i];
  block_sum_store<true>(acc, out);
}

__global__ void k_scale(const float* __restrict__ u, float* __restrict__ x, int64_t n,
                        const double* __restrict__ ss) {
  const float a = alpha_of(ss);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    x[i] = __fmul_rn(u[i], a);
}

constexpr size_t stream_smem_bytes() {
  return sizeof(int32_t) * TILE_BUF + sizeof(float) * TILE_BUF + sizeof(float) * PROD_LEN;
}

template <typename OT>
void exec_typed(spmv_plan_s* p, const float* x, float* y, const double* ss_in, double* ss_out,
                cudaStream_t s) {
  const OT* rp = (const OT*)p->d_rp;
  const bool SS = ss_out != nullptr;
  const int ef = p->opts.evict_first;
  if (p->K) {
    const size_t smem = stream_smem_bytes();
    if (SS) {
      static bool attr = false;
      if (!attr) {
        SPMV_CUDA(cudaFuncSetAttribute(k_stream<OT, true>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        attr = true;
      }
      k_stream<OT, true><<<(unsigned)p->K, ST_THREADS, smem, s>>>(
          rp, p->d_col, p->d_val, x, y, p->d_tiles, ss_in, p->d_tile_ss, ef);
    } else {
      static bool attr = false;
      if (!attr) {
        SPMV_CUDA(cudaFuncSetAttribute(k_stream<OT, false>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        attr = true;
      }
      k_stream<OT, false><<<(unsigned)p->K, ST_THREADS, smem, s>>>(
          rp, p->d_col, p->d_val, x, y, p->d_tiles, ss_in, p->d_tile_ss, ef);
    }
  }
  if (p->n_cta) {
    if (SS)
      k_cta_rows<OT, true><<<(unsigned)p->n_cta, 256, 0, s>>>(rp, p->d_col, p->d_val, x, y,
                                                             p->d_cta_rows, ss_in, p->d_cta_ss);
    else
      k_cta_rows<OT, false><<<(unsigned)p->n_cta, 256, 0, s>>>(rp, p->d_col, p->d_val, x, y,
                                                              p->d_cta_rows, ss_in, p->d_cta_ss);
  }
  if (p->n_chunks) {
    k_hub_chunk<OT><<<(unsigned)p->n_chunks, 256, 0, s>>>(rp, p->d_col, p->d_val, x,
                                                          p->d_chunk_row, p->d_chunk_idx,
                                                          p->d_chunk_part);
    const unsigned g = (unsigned)((p->n_hub + 127) / 128);
    if (SS)
      k_hub_fix<true><<<g, 128, 0, s>>>(p->d_hub_rows, p->d_hub_choff, p->n_hub, p->d_chunk_part,
                                        ss_in, y, p->d_hub_ss);
    else
      k_hub_fix<false><<<g, 128, 0, s>>>(p->d_hub_rows, p->d_hub_choff, p->n_hub,
                                         p->d_chunk_part, ss_in, y, p->d_hub_ss);
  }
  if (SS)
    k_ss_final<<<1, 1024, 0, s>>>(p->d_tile_ss, p->K, p->d_cta_ss, p->n_cta, p->d_hub_ss, p->n_hub,
                                  ss_out);
  SPMV_LAUNCH_CHECK();
}

void set_window(spmv_plan_s* p, const float* x, cudaStream_t s) {
  if (!p->opts.l2_window || p->H <= 0 || s == nullptr) return;
  if (p->win_ptr == (const void*)x && p->win_stream == s) return;
  int maxwin = 0, maxpers = 0;
  cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, p->device);
  cudaDeviceGetAttribute(&maxpers, cudaDevAttrMaxPersistingL2CacheSize, p->device);
  int64_t bytes = std::min<int64_t>(p->H * 4, (int64_t)maxwin);
  bytes = std::min<int64_t>(bytes, (int64_t)maxpers);
  if (bytes <= 0) return;
  size_t cur = 0;
  cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
  if ((int64_t)cur < bytes) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)bytes);
  cudaStreamAttrValue v{};
  v.accessPolicyWindow.base_ptr = (void*)x;
  v.accessPolicyWindow.num_bytes = (size_t)bytes;
  v.accessPolicyWindow.hitRatio = (float)p->opts.l2_hit_ratio;
  v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
  v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
  if (cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  p->win_ptr = x;
  p->win_stream = s;
  p->l2_window_bytes = bytes;
}

}  // namespace

void exec(spmv_plan_s* p, const float* x, float* y, const double* ss_in, double* ss_out,
          cudaStream_t s) {
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_exec before spmv_permute");
  if (ss_in && ss_in == ss_out) SPMV_FAIL(SPMV_EINVAL, "sumsq_in and sumsq_out alias");
  set_window(p, x, s);
  if (p->off64) exec_typed<int64_t>(p, x, y, ss_in, ss_out, s);
  else exec_typed<int32_t>(p, x, y, ss_in, ss_out, s);
}

void iterate(spmv_plan_s* p, float* x, int iters, double* lambda, cudaStream_t s) {
  if (iters < 1) SPMV_FAIL(SPMV_EINVAL, "iters must be >= 1");
  if (p->world != 1) SPMV_FAIL(SPMV_EUNSUPPORTED, "spmv_iterate drives world == 1; use spmv_exec_scaled + collectives for world > 1");
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_iterate before spmv_permute");
  if (!p->d_u) {
    void* q = nullptr;
    if (cudaMalloc(&q, sizeof(float) * (size_t)std::max<int64_t>(p->x_len, 1)) != cudaSuccess) {
      cudaGetLastError();
      SPMV_FAIL(SPMV_ENOMEM, "iterate buffer allocation failed");
    }
    p->d_u = (float*)q;
  }
  float* a = x;
  float* b = p->d_u;
  const double* sin = nullptr;
  for (int t = 0; t < iters; ++t) {
    double* sout = p->d_ss + (t & 1);
    exec(p, a, b, sin, sout, s);
    sin = sout;
    std::swap(a, b);
  }
  if (p->n) {
    int g = (int)std::min<int64_t>((p->n + 255) / 256, 148 * 16);
    k_scale<<<g, 256, 0, s>>>(a, x, p->n, sin);
    SPMV_LAUNCH_CHECK();
  }
  double ss = 0.0;
  SPMV_CUDA(cudaMemcpyAsync(&ss, sin, sizeof(double), cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  if (lambda) *lambda = std::sqrt(ss);
}

void scale_vec(const float* u, float* x, int64_t n, const double* ss, cudaStream_t s) {
  if (n <= 0) return;
  int g = (int)std::min<int64_t>((n + 255) / 256, 148 * 16);
  k_scale<<<g, 256, 0, s>>>(u, x, n, ss);
  SPMV_LAUNCH_CHECK();
}

}  // namespace spmv
