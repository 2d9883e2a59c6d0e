// Dev-only microbenchmark (not part of the library): the random-gather
// ceilings of one B200, the roofline of the x gathers of the gather-bound
// configs (C3, C5).  For uniformly random 4-byte gathers over a
// range of S bytes (L2-resident or not) it measures gathers per second for
//   ldg   -- LDG through L1 (the SpMV kernels' x path, __ldg)
//   na    -- ld.global.nc.L1::no_allocate
//   lds   -- shared-memory gathers from a 96 KB table (the hot-set option)
//   tma4  -- cp.async.bulk.tensor tile::gather4 (TMA, 4 x 16-byte rows per
//            instruction into shared memory), x viewed as [S/16][4] floats
// each with the index stream read coalesced, as col is in the SpMV.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gc scripts/gather_ceiling.cu -lcuda
//   /tmp/gc            (prints one JSON line per measurement)
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x)                                                                   \
  do {                                                                          \
    cudaError_t e_ = (x);                                                       \
    if (e_ != cudaSuccess) {                                                    \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      exit(1);                                                                  \
    }                                                                           \
  } while (0)

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void k_fill_idx(int32_t* idx, int64_t m, uint64_t range, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x)
    idx[i] = (int32_t)(mix64(seed + 0x9E3779B97F4A7C15ull * (uint64_t)(i + 1)) % range);
}

__global__ void k_fill_x(float* x, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    x[i] = (float)(i & 1023) * 0.001f;
}

template <int MODE>
__device__ __forceinline__ float gat(const float* x, int c) {
  if constexpr (MODE == 0) return __ldg(x + c);
  float r;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(x + c));
  return r;
}

// U gathers in flight per thread; idx read coalesced (ld.cs)
template <int MODE, int U>
__global__ void __launch_bounds__(256) k_gather(const int32_t* __restrict__ idx, int64_t m,
                                                const float* __restrict__ x, float* out) {
  const int64_t T = (int64_t)gridDim.x * blockDim.x;
  float s = 0.f;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += T * U) {
    int c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) c[u] = (i + T * u < m) ? __ldcs(idx + i + T * u) : 0;
#pragma unroll
    for (int u = 0; u < U; ++u) s += gat<MODE>(x, c[u]);
  }
  if (s == 12345.f) out[0] = s;
}

// shared-memory gathers from a TAB-float table (indices taken mod TAB)
constexpr int TAB = 24576;  // 96 KB
template <int U>
__global__ void __launch_bounds__(256) k_gather_smem(const int32_t* __restrict__ idx, int64_t m,
                                                     const float* __restrict__ x, float* out) {
  extern __shared__ float tab[];
  for (int i = threadIdx.x; i < TAB; i += blockDim.x) tab[i] = x[i];
  __syncthreads();
  const int64_t T = (int64_t)gridDim.x * blockDim.x;
  float s = 0.f;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += T * U) {
    int c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) c[u] = (i + T * u < m) ? __ldcs(idx + i + T * u) : 0;
#pragma unroll
    for (int u = 0; u < U; ++u) s += tab[c[u] % TAB];
  }
  if (s == 12345.f) out[0] = s;
}

// ---- TMA gather4
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// 128 threads per CTA; a stage = 32 gather4 (one per lane of warp 0) = 128
// rows of 16 B; each lane's 4 rows land in its own 128-byte-aligned slot
// (tensor copies need a 128-B aligned destination); NST stages in a ring.
// Every thread then reads the float its row needs (row r's element idx & 3).
constexpr int NST = 4;
__global__ void __launch_bounds__(128) k_gather_tma4(const __grid_constant__ CUtensorMap tm,
                                                     const int32_t* __restrict__ idx, int64_t m,
                                                     float* out, int* err) {
  __shared__ __align__(128) float4 buf[NST][32][8];  // [stage][lane][row 0..3 used]
  __shared__ alignas(8) uint64_t full[NST];
  __shared__ alignas(8) uint64_t empty[NST];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) {
    for (int s = 0; s < NST; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&full[s])), "r"(1));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(128));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int64_t per = 128;  // rows per stage
  const int64_t nst_total = m / per;
  float s = 0.f;
  int64_t k = 0;
  // producer issues stage j (j = k + NST - 1 ahead); everyone consumes stage k
  auto issue = [&](int64_t j) {
    const int st = (int)(j % NST);
    const int64_t base = (blockIdx.x + j * (int64_t)gridDim.x) * per;  // this CTA's j-th block
    if (w == 0) {
      if (lane == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[st])),
                     "r"(128 * 16)
                     : "memory");
      __syncwarp();
      const int32_t* ip = idx + base + lane * 4;
      const int r0 = __ldcs(ip) >> 2, r1 = __ldcs(ip + 1) >> 2, r2 = __ldcs(ip + 2) >> 2,
                r3 = __ldcs(ip + 3) >> 2;
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
          " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(&buf[st][lane][0])),
          "l"(&tm), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(&full[st]))
          : "memory");
    }
  };
  const int64_t mine = (nst_total - blockIdx.x + gridDim.x - 1) / gridDim.x;  // stages of this CTA
  for (int64_t j = 0; j < NST - 1 && j < mine; ++j) issue(j);
  for (k = 0; k < mine; ++k) {
    const int st = (int)(k % NST);
    const uint32_t ph = (uint32_t)((k / NST) & 1);
    // bounded wait: a wrong descriptor must not hang the GPU
    uint32_t ok = 0;
    for (int spin = 0; spin < (1 << 22) && !ok; ++spin)
      asm volatile(
          "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
          : "=r"(ok)
          : "r"(su32(&full[st])), "r"(ph)
          : "memory");
    if (!ok) {
      if (tid == 0) atomicExch(err, 1);
      return;
    }
    const int64_t base = (blockIdx.x + k * (int64_t)gridDim.x) * per;
    const int c = __ldcs(idx + base + tid);
    s += reinterpret_cast<const float*>(&buf[st][tid >> 2][tid & 3])[c & 3];
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[st])) : "memory");
    // the producer reuses stage (k + NST - 1) % NST = (k - 1) % NST: wait until it is drained
    const int64_t j = k + NST - 1;
    if (j < mine) {
      if (k >= 1) {
        const int pst = (int)((k - 1) % NST);
        const uint32_t pph = (uint32_t)(((k - 1) / NST) & 1);
        if (w == 0) {
          uint32_t ok2 = 0;
          for (int spin = 0; spin < (1 << 22) && !ok2; ++spin)
            asm volatile(
                "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                : "=r"(ok2)
                : "r"(su32(&empty[pst])), "r"(pph)
                : "memory");
          if (!ok2) {
            if (lane == 0) atomicExch(err, 2);
            return;
          }
        }
      }
      issue(j);
    }
  }
  if (s == 12345.f) out[0] = s;
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <typename F>
float time_ms(F f, int reps) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  f();
  CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(a));
  for (int i = 0; i < reps; ++i) f();
  CK(cudaEventRecord(b));
  CK(cudaEventSynchronize(b));
  float ms;
  CK(cudaEventElapsedTime(&ms, a, b));
  return ms / reps;
}

int main(int argc, char** argv) {
  const bool only_tma = argc > 1 && argv[1][0] == 't';
  int sms;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int64_t m = int64_t(1) << 28;           // 268 M gathers per launch
  const int64_t xn = int64_t(1) << 28;          // x up to 1 GiB
  int32_t* idx;
  float *x, *out;
  int* err;
  CK(cudaMalloc(&idx, m * 4));
  CK(cudaMalloc(&x, xn * 4));
  CK(cudaMalloc(&out, 4));
  CK(cudaMalloc(&err, 4));
  CK(cudaMemset(err, 0, 4));
  k_fill_x<<<sms * 8, 256>>>(x, xn);
  const int64_t ranges[] = {int64_t(1) << 22, int64_t(1) << 24, int64_t(1) << 26, xn};  // 16 MB .. 1 GB
  for (int64_t R : ranges) {
    if (only_tma) break;
    k_fill_idx<<<sms * 8, 256>>>(idx, m, (uint64_t)R, 12345);
    CK(cudaDeviceSynchronize());
    auto rep = [&](const char* mode, int U, int cps, float ms) {
      printf("{\"mode\": \"%s\", \"range_mb\": %.0f, \"U\": %d, \"ctas_per_sm\": %d, \"ms\": %.3f, "
             "\"ggather_per_s\": %.1f, \"per_sm_per_clk_at_1.9GHz\": %.3f}\n",
             mode, R * 4.0 / 1048576, U, cps, ms, m / ms / 1e6, m / ms / 1e6 * 1e9 / 1e9 / sms / 1.9);
      fflush(stdout);
    };
    for (int cps : {4, 8}) {
      const int g = sms * cps;
      rep("ldg", 4, cps, time_ms([&] { k_gather<0, 4><<<g, 256>>>(idx, m, x, out); }, 5));
      rep("ldg", 8, cps, time_ms([&] { k_gather<0, 8><<<g, 256>>>(idx, m, x, out); }, 5));
      rep("ldg", 16, cps, time_ms([&] { k_gather<0, 16><<<g, 256>>>(idx, m, x, out); }, 5));
      rep("na", 8, cps, time_ms([&] { k_gather<1, 8><<<g, 256>>>(idx, m, x, out); }, 5));
    }
  }
  // idx-stream-only control (gather the index's own position: coalesced)
  if (!only_tma) {
    int32_t* seq;
    CK(cudaMalloc(&seq, m * 4));
    k_fill_idx<<<sms * 8, 256>>>(seq, m, 1, 0);  // all zero -> every lane the same word
    CK(cudaDeviceSynchronize());
    const float ms = time_ms([&] { k_gather<0, 8><<<sms * 8, 256>>>(seq, m, x, out); }, 5);
    printf("{\"mode\": \"ldg_same_word\", \"U\": 8, \"ms\": %.3f, \"ggather_per_s\": %.1f}\n", ms, m / ms / 1e6);
    CK(cudaFree(seq));
  }
  // shared-memory table gathers (indices mod 24576)
  k_fill_idx<<<sms * 8, 256>>>(idx, m, (uint64_t)TAB, 777);
  CK(cudaFuncSetAttribute(k_gather_smem<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, TAB * 4));
  for (int cps : {1, 2}) {
    if (only_tma) break;
    const float ms = time_ms([&] { k_gather_smem<8><<<sms * cps, 256, TAB * 4>>>(idx, m, x, out); }, 5);
    printf("{\"mode\": \"lds\", \"U\": 8, \"ctas_per_sm\": %d, \"ms\": %.3f, \"ggather_per_s\": %.1f}\n", cps, ms,
           m / ms / 1e6);
  }
  // TMA gather4
  {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    EncodeFn enc = (EncodeFn)fn;
    for (int64_t R : ranges) {
      k_fill_idx<<<sms * 8, 256>>>(idx, m, (uint64_t)R, 999);
      CK(cudaDeviceSynchronize());
      CUtensorMap tm;
      const cuuint64_t dims[2] = {4, (cuuint64_t)(R / 4)};
      const cuuint64_t strides[1] = {16};
      const cuuint32_t box[2] = {4, 1};
      const cuuint32_t es[2] = {1, 1};
      CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, x, dims, strides, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                       CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) {
        printf("{\"mode\": \"tma4\", \"error\": \"encode %d\"}\n", (int)r);
        break;
      }
      for (int cps : {4, 8, 16}) {
        CK(cudaMemset(err, 0, 4));
        const float ms =
            time_ms([&] { k_gather_tma4<<<sms * cps, 128>>>(tm, idx, m, out, err); }, 3);
        int h;
        CK(cudaMemcpy(&h, err, 4, cudaMemcpyDeviceToHost));
        printf("{\"mode\": \"tma4\", \"range_mb\": %.0f, \"ctas_per_sm\": %d, \"ms\": %.3f, "
               "\"ggather_per_s\": %.1f, \"err\": %d}\n",
               R * 4.0 / 1048576, cps, ms, m / ms / 1e6, h);
        fflush(stdout);
        if (h) break;
      }
    }
  }
  CK(cudaDeviceSynchronize());
  return 0;
}
