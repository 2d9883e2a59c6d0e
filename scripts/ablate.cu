// Dev-only ablation kernels (not part of the library): how fast can the
// matrix stream of the C2 workload go with (a) the k_lane access pattern
// (lane per row, 32-byte chunks) and no x gathers, (b) a fully coalesced
// contiguous read of the same bytes, (c) (a) plus x gathers through L2 only.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC -o /tmp/ablate.so scripts/ablate.cu
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void ldv8(const int32_t* p, int (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.s32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                 "=r"(r[6]), "=r"(r[7])
               : "l"(p));
}
__device__ __forceinline__ void ldv8f(const float* p, float (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]),
                 "=f"(r[6]), "=f"(r[7])
               : "l"(p));
}

// (a)/(c): lane per row, grid-stride over rows; mode 0 = no gathers, 1 = __ldg(x[c])
template <int MODE, typename OT>
__global__ void __launch_bounds__(256) k_rows(const OT* __restrict__ rp,
                                              const int32_t* __restrict__ col,
                                              const float* __restrict__ val,
                                              const float* __restrict__ x, float* __restrict__ y,
                                              int n) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const long a = rp[r], e = rp[r + 1];
    float s = 0.f;
    for (long k = a & ~7l; k < e; k += 8) {
      int c[8];
      float v[8];
      ldv8(col + k, c);
      ldv8f(val + k, v);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const float xv = MODE ? __ldg(x + c[i]) : __int_as_float(c[i]);
        s += (k + i >= a && k + i < e) ? v[i] * xv : 0.f;
      }
    }
    y[r] = s;
  }
}

__device__ __forceinline__ void ldv8h(const int32_t* p, uint64_t, int (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.s32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                 "=r"(r[6]), "=r"(r[7])
               : "l"(p));
}
__device__ __forceinline__ void ldv8fh(const float* p, uint64_t, float (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]),
                 "=f"(r[6]), "=f"(r[7])
               : "l"(p));
}

// canonical variants: F bit0 = canonical fmul_rn/fadd_rn, bit1 = bitmask masking,
// bit2 = evict_first hint on the stream, bit3 = contiguous 256-row panels per CTA
// (persistent) instead of grid-stride
template <int F, typename OT>
__global__ void __launch_bounds__(256) k_rows2(const OT* __restrict__ rp,
                                               const int32_t* __restrict__ col,
                                               const float* __restrict__ val,
                                               const float* __restrict__ x, float* __restrict__ y,
                                               int n) {
  uint64_t pol = 0;

  int r0, r1, step;
  if (F & 8) {
    const long NB = (n + 255) / 256;
    const long b0 = NB * blockIdx.x / gridDim.x, b1 = NB * (blockIdx.x + 1) / gridDim.x;
    r0 = (int)(b0 * 256) + threadIdx.x;
    r1 = (int)min((long)n, b1 * 256);
    step = 256;
  } else {
    r0 = blockIdx.x * blockDim.x + threadIdx.x;
    r1 = n;
    step = gridDim.x * blockDim.x;
  }
  for (int r = r0; r < r1; r += step) {
    const long a = rp[r], e = rp[r + 1];
    float s = 0.f;
    const int lo = a & 7, hi = lo + (int)(e - a);
    const uint64_t live = (((1ull << hi) - 1ull) >> lo) << lo;
    const int32_t* cp = col + (a & ~7l);
    const float* vp = val + (a & ~7l);
    for (int k = 0; k < hi; k += 8) {
      int c[8];
      float v[8];
      if (F & 4) { ldv8h(cp + k, pol, c); ldv8fh(vp + k, pol, v); }
      else { ldv8(cp + k, c); ldv8f(vp + k, v); }
      const uint32_t mk = (uint32_t)(live >> k);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float xv = (F & 16) ? __int_as_float(c[i]) : __ldg(x + c[i]);
        bool ok = (F & 2) ? ((mk >> i) & 1u) : (k + i >= lo && k + i < hi);
        if (F & 1) s = __fadd_rn(s, __fmul_rn(v[i], ok ? xv : 0.f));
        else s += ok ? v[i] * xv : 0.f;
      }
    }
    y[r] = s;
  }
}

// (b): contiguous, each thread 32 B of col and 32 B of val per step
__global__ void __launch_bounds__(256) k_flat(const int32_t* __restrict__ col,
                                              const float* __restrict__ val, float* __restrict__ y,
                                              long nnz) {
  float s = 0.f;
  for (long k = ((long)blockIdx.x * blockDim.x + threadIdx.x) * 8; k + 8 <= nnz;
       k += (long)gridDim.x * blockDim.x * 8) {
    int c[8];
    float v[8];
    ldv8(col + k, c);
    ldv8f(val + k, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) s += v[i] * __int_as_float(c[i]);
  }
  y[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <typename OT>
int ablate_t(int which, const OT* rp, const int32_t* col, const float* val, const float* x, float* y,
             int n, long nnz, int grid, cudaStream_t s) {
  if (which == 0) k_rows<0, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  else if (which == 1) k_rows<1, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  else if (which == 2) k_flat<<<grid, 256, 0, s>>>(col, val, y, nnz);
  else if (which == 10) k_rows2<1, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  else if (which == 12) k_rows2<5, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  else if (which == 13) k_rows2<13, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  else if (which == 20) k_rows2<16 + 5, OT><<<grid, 256, 0, s>>>(rp, col, val, x, y, n);
  return (int)cudaGetLastError();
}

extern "C" int ablate(int which, const void* rp, int rp64, const int32_t* col, const float* val,
                      const float* x, float* y, int n, long nnz, int grid, cudaStream_t s) {
  if (rp64) return ablate_t(which, (const long*)rp, col, val, x, y, n, nnz, grid, s);
  return ablate_t(which, (const int*)rp, col, val, x, y, n, nnz, grid, s);
}
