// synth_gpu: the RMAT / Graph500 Kronecker generator of synth.cpp on the GPU.
//
// Input generation only (no SpMV, permutation or reordering arithmetic), and
// independent of libspmv: it shares no code with the product.  The matrix is
// the SAME function of (scale, edge factor, seeds) as synth_rmat in
// synth.cpp -- same counter-based draws, same scramble bijection, duplicates
// merged, columns sorted, values h2(seed_v, row, col) -- so both generators
// give bit-identical CSR (tests/test_synth_gpu.py), this one in seconds at
// scale 28 instead of minutes on the host.
//
// Pipeline (device memory only): edge e -> key (row << scale) | col; stable
// LSD radix sort of the 2 * scale key bits (8-bit digits: per-tile digit
// histograms, one exclusive scan over the digit-major counts, stable scatter
// ranked by warp match); duplicate keys dropped by a stream compaction; row
// pointer from the row boundaries of the sorted unique keys; values.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ uint64_t h1(uint64_t s, uint64_t a) {
  return mix64(s + kGolden * (a + 1));
}
__host__ __device__ __forceinline__ uint64_t h2(uint64_t s, uint64_t a, uint64_t b) {
  return h1(h1(s, a), b);
}
__device__ __forceinline__ float sym_f32(uint64_t h) {
  return (float)((double)(h >> 40) * (1.0 / 8388608.0) - 1.0);
}
__device__ __forceinline__ float pos_f32(uint64_t h) {
  return (float)((double)((h >> 40) + 1) * (1.0 / 16777216.0));
}

struct Bij {  // synth.cpp Bij: bijection on [0, 2^k)
  int k;
  uint64_t mask, mul[4], add[4];
  int shift;
  __host__ __device__ uint64_t operator()(uint64_t v) const {
    if (k == 0) return 0;
    for (int r = 0; r < 4; ++r) {
      v = (v * mul[r] + add[r]) & mask;
      v ^= v >> shift;
    }
    return v;
  }
};

Bij make_bij(int k, uint64_t seed) {
  Bij b;
  b.k = k;
  b.mask = (k >= 64) ? ~0ull : ((1ull << k) - 1);
  b.shift = (k + 1) / 2;
  if (b.shift < 1) b.shift = 1;
  for (int r = 0; r < 4; ++r) {
    b.mul[r] = (h1(seed, 2 * r) | 1ull) & b.mask;
    b.add[r] = h1(seed, 2 * r + 1) & b.mask;
  }
  return b;
}

__global__ void k_edges(int64_t E, int scale, uint64_t seed, uint64_t t1, uint64_t t2,
                        uint64_t t3, int scramble, Bij bij, uint64_t* keys) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < E;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t he = h1(seed, (uint64_t)e);
    uint64_t rr = 0, cc = 0;
    for (int l = 0; l < scale; ++l) {
      const uint64_t u = h1(he, (uint64_t)l) >> 11;
      const uint64_t rb = u >= t2;
      const uint64_t cb = (u >= t1 && u < t2) || (u >= t3);
      rr |= rb << (scale - 1 - l);
      cc |= cb << (scale - 1 - l);
    }
    if (scramble) {  // n = 2^scale: the cycle walk of synth.cpp never repeats
      rr = bij(rr);
      cc = bij(cc);
    }
    keys[e] = (rr << scale) | cc;
  }
}

// ------------------------------------------------------------ radix sort
constexpr int RS_T = 256;              // threads per tile
constexpr int RS_SUB = 32;             // sub-tiles of RS_T keys per tile
constexpr int64_t RS_TILE = RS_T * RS_SUB;

__global__ void __launch_bounds__(RS_T) k_hist(const uint64_t* __restrict__ keys, int64_t n,
                                                int shift, int64_t ntiles, uint32_t* cnt) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const int64_t t = blockIdx.x;
  const int64_t base = t * RS_TILE;
  for (int s = 0; s < RS_SUB; ++s) {
    const int64_t i = base + (int64_t)s * RS_T + threadIdx.x;
    if (i < n) atomicAdd(&h[(keys[i] >> shift) & 255], 1u);
  }
  __syncthreads();
  cnt[(int64_t)threadIdx.x * ntiles + t] = h[threadIdx.x];
}

// exclusive scan of m uint32 counts into int64 offsets (3 kernels)
constexpr int SC_T = 1024;
constexpr int64_t SC_B = SC_T * 8;

__global__ void __launch_bounds__(SC_T) k_scan_sums(const uint32_t* in, int64_t m, int64_t* bs) {
  __shared__ int64_t w[SC_T / 32];
  const int64_t b0 = (int64_t)blockIdx.x * SC_B;
  int64_t s = 0;
  for (int j = 0; j < 8; ++j) {
    const int64_t i = b0 + (int64_t)j * SC_T + threadIdx.x;
    if (i < m) s += in[i];
  }
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) w[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t a = 0;
    for (int k = 0; k < SC_T / 32; ++k) a += w[k];
    bs[blockIdx.x] = a;
  }
}

__global__ void k_scan_top(int64_t* bs, int64_t nb) {  // one thread: nb is small
  if (threadIdx.x | blockIdx.x) return;
  int64_t a = 0;
  for (int64_t i = 0; i < nb; ++i) {
    const int64_t v = bs[i];
    bs[i] = a;
    a += v;
  }
}

__global__ void __launch_bounds__(SC_T) k_scan_down(const uint32_t* in, int64_t m,
                                                    const int64_t* bs, int64_t* out) {
  __shared__ int64_t w[SC_T / 32];
  const int64_t b0 = (int64_t)blockIdx.x * SC_B;
  // each thread owns 8 consecutive counts
  const int64_t i0 = b0 + (int64_t)threadIdx.x * 8;
  uint32_t v[8];
  int64_t s = 0;
  for (int j = 0; j < 8; ++j) {
    v[j] = i0 + j < m ? in[i0 + j] : 0u;
    s += v[j];
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int64_t inc = s;
  for (int o = 1; o < 32; o <<= 1) {
    const int64_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) w[wid] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t a = 0;
    for (int k = 0; k < SC_T / 32; ++k) {
      const int64_t t = w[k];
      w[k] = a;
      a += t;
    }
  }
  __syncthreads();
  int64_t a = bs[blockIdx.x] + w[wid] + inc - s;
  for (int j = 0; j < 8; ++j) {
    if (i0 + j < m) out[i0 + j] = a;
    a += v[j];
  }
}

// stable scatter: keys of a tile in index order, ranked per digit by warp
// match + per-warp counts + running per-digit base
__global__ void __launch_bounds__(RS_T) k_scatter(const uint64_t* __restrict__ in, int64_t n,
                                                   int shift, int64_t ntiles,
                                                   const int64_t* __restrict__ off,
                                                   uint64_t* __restrict__ out) {
  __shared__ int64_t goff[256];
  __shared__ uint32_t wcnt[RS_T / 32][256];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t t = blockIdx.x, base = t * RS_TILE;
  goff[tid] = off[(int64_t)tid * ntiles + t];
  const unsigned lt = (1u << lane) - 1u;
  for (int s = 0; s < RS_SUB; ++s) {
    for (int w = 0; w < RS_T / 32; ++w) wcnt[w][tid] = 0;
    __syncthreads();
    const int64_t i = base + (int64_t)s * RS_T + tid;
    const bool ok = i < n;
    const uint64_t k = ok ? in[i] : 0ull;
    const unsigned d = ok ? (unsigned)((k >> shift) & 255) : 256u;
    const unsigned peers = __match_any_sync(0xffffffffu, d);
    const unsigned r = __popc(peers & lt);
    if (ok && r == 0) wcnt[wid][d] = __popc(peers);
    __syncthreads();
    {  // thread tid = digit tid: exclusive prefix over the warps, advance base
      int64_t run = goff[tid];
      for (int w = 0; w < RS_T / 32; ++w) {
        const uint32_t c = wcnt[w][tid];
        wcnt[w][tid] = (uint32_t)(run - goff[tid]);
        run += c;
      }
      __syncthreads();
      if (ok) out[goff[d] + wcnt[wid][d] + r] = k;
      __syncthreads();
      goff[tid] = run;
    }
  }
}

// ---------------------------------------------------- dedup + CSR
__global__ void k_uniq_count(const uint64_t* __restrict__ k, int64_t n, int64_t per,
                             uint32_t* cnt) {
  const int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t i0 = b * per;
  if (i0 >= n) return;
  const int64_t i1 = min(n, i0 + per);
  uint32_t c = 0;
  for (int64_t i = i0; i < i1; ++i) c += (i == 0 || k[i] != k[i - 1]);
  cnt[b] = c;
}

__global__ void k_uniq_write(const uint64_t* __restrict__ k, int64_t n, int64_t per,
                             const int64_t* __restrict__ pos, uint64_t* __restrict__ out) {
  const int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t i0 = b * per;
  if (i0 >= n) return;
  const int64_t i1 = min(n, i0 + per);
  int64_t o = pos[b];
  for (int64_t i = i0; i < i1; ++i)
    if (i == 0 || k[i] != k[i - 1]) out[o++] = k[i];
}

__global__ void k_csr(const uint64_t* __restrict__ k, int64_t m, int scale, int64_t nrows,
                      int valmode, uint64_t seed_v, int64_t* __restrict__ rp,
                      int32_t* __restrict__ col, float* __restrict__ val) {
  const uint64_t cmask = (1ull << scale) - 1;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t key = k[i];
    const int64_t r = (int64_t)(key >> scale), c = (int64_t)(key & cmask);
    col[i] = (int32_t)c;
    const uint64_t h = h2(seed_v, (uint64_t)r, (uint64_t)c);
    val[i] = valmode == 0 ? sym_f32(h) : valmode == 1 ? pos_f32(h) : 1.0f;
    const int64_t rprev = i == 0 ? -1 : (int64_t)(k[i - 1] >> scale);
    for (int64_t q = rprev + 1; q <= r; ++q) rp[q] = i;  // rows rprev+1 .. r start here
    if (i == m - 1)
      for (int64_t q = r + 1; q <= nrows; ++q) rp[q] = m;
  }
}

__global__ void k_fill64(int64_t* p, int64_t n, int64_t v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

int g_err = 0;
char g_msg[256];

bool ck(cudaError_t e, const char* what) {
  if (e != cudaSuccess) {
    snprintf(g_msg, sizeof(g_msg), "%s: %s", what, cudaGetErrorString(e));
    g_err = 1;
    return false;
  }
  return true;
}

void scan_u32(const uint32_t* in, int64_t m, int64_t* out, int64_t* bs, cudaStream_t s) {
  const int64_t nb = (m + SC_B - 1) / SC_B;
  k_scan_sums<<<(unsigned)nb, SC_T, 0, s>>>(in, m, bs);
  k_scan_top<<<1, 1, 0, s>>>(bs, nb);
  k_scan_down<<<(unsigned)nb, SC_T, 0, s>>>(in, m, bs, out);
}

}  // namespace

extern "C" {

typedef struct {
  int64_t n, nnz;
  int64_t* row_ptr;  // device
  int32_t* col;      // device
  float* val;        // device
} synth_gpu_csr;

const char* synth_gpu_error(void) { return g_msg; }

void synth_gpu_free(synth_gpu_csr* m) {
  if (!m) return;
  cudaFree(m->row_ptr);
  cudaFree(m->col);
  cudaFree(m->val);
  m->row_ptr = nullptr;
  m->col = nullptr;
  m->val = nullptr;
}

// synth_rmat on the device (see synth.cpp): 0 on success; the CSR arrays are
// cudaMalloc'ed on `device` and owned by the caller (synth_gpu_free).
int synth_rmat_gpu(int scale, int64_t edge_factor, uint64_t seed, double a, double b, double c,
                   int scramble, uint64_t seed_scr, int valmode, uint64_t seed_v, int device,
                   synth_gpu_csr* out) {
  g_err = 0;
  g_msg[0] = 0;
  if (scale < 1 || scale > 31 || edge_factor < 0 || !out) {
    snprintf(g_msg, sizeof(g_msg), "bad argument");
    return 1;
  }
  if (!ck(cudaSetDevice(device), "cudaSetDevice")) return 2;
  cudaStream_t s = nullptr;
  const int64_t n = 1ll << scale, E = edge_factor << scale;
  auto thr53 = [](double p) { return (uint64_t)(p * 9007199254740992.0); };
  const uint64_t t1 = thr53(a), t2 = thr53(a + b), t3 = thr53(a + b + c);
  const Bij bij = make_bij(scale, seed_scr);
  uint64_t *ka = nullptr, *kb = nullptr;
  uint32_t* cnt = nullptr;
  int64_t *off = nullptr, *bs = nullptr;
  out->n = n;
  out->nnz = 0;
  out->row_ptr = nullptr;
  out->col = nullptr;
  out->val = nullptr;
  const int64_t ntiles = (E + RS_TILE - 1) / RS_TILE;
  const int64_t m = 256 * ntiles;
  bool ok = ck(cudaMalloc(&ka, 8 * (size_t)(E > 0 ? E : 1)), "cudaMalloc keys") &&
            ck(cudaMalloc(&kb, 8 * (size_t)(E > 0 ? E : 1)), "cudaMalloc keys") &&
            ck(cudaMalloc(&cnt, 4 * (size_t)(m > 0 ? m : 1)), "cudaMalloc counts") &&
            ck(cudaMalloc(&off, 8 * (size_t)(m > 0 ? m : 1)), "cudaMalloc offsets") &&
            ck(cudaMalloc(&bs, 8 * (size_t)((m + SC_B - 1) / SC_B + 2)), "cudaMalloc scan");
  if (ok && E > 0) {
    k_edges<<<148 * 16, 256, 0, s>>>(E, scale, seed, t1, t2, t3, scramble, bij, ka);
    const int bits = 2 * scale;
    for (int shift = 0; shift < bits; shift += 8) {
      k_hist<<<(unsigned)ntiles, RS_T, 0, s>>>(ka, E, shift, ntiles, cnt);
      scan_u32(cnt, m, off, bs, s);
      k_scatter<<<(unsigned)ntiles, RS_T, 0, s>>>(ka, E, shift, ntiles, off, kb);
      uint64_t* t = ka;
      ka = kb;
      kb = t;
    }
    ok = ck(cudaGetLastError(), "radix sort");
  }
  // dedup: ka sorted -> kb unique
  int64_t nu = 0;
  const int64_t per = 4096;
  const int64_t nblk = E > 0 ? (E + per - 1) / per : 0;
  if (ok && E > 0) {
    uint32_t* ucnt = cnt;  // reuse (nblk <= m)
    int64_t* upos = off;
    k_uniq_count<<<(unsigned)((nblk + 255) / 256), 256, 0, s>>>(ka, E, per, ucnt);
    scan_u32(ucnt, nblk, upos, bs, s);
    k_uniq_write<<<(unsigned)((nblk + 255) / 256), 256, 0, s>>>(ka, E, per, upos, kb);
    int64_t last = 0;
    uint32_t lastc = 0;
    ok = ck(cudaMemcpy(&last, upos + nblk - 1, 8, cudaMemcpyDeviceToHost), "D2H") &&
         ck(cudaMemcpy(&lastc, ucnt + nblk - 1, 4, cudaMemcpyDeviceToHost), "D2H");
    nu = last + lastc;
  }
  cudaFree(ka);
  cudaFree(cnt);
  cudaFree(off);
  cudaFree(bs);
  ka = nullptr;
  if (ok) {
    ok = ck(cudaMalloc(&out->row_ptr, 8 * (size_t)(n + 1)), "cudaMalloc row_ptr") &&
         ck(cudaMalloc(&out->col, 4 * (size_t)(nu > 0 ? nu : 1)), "cudaMalloc col") &&
         ck(cudaMalloc(&out->val, 4 * (size_t)(nu > 0 ? nu : 1)), "cudaMalloc val");
  }
  if (ok) {
    if (nu == 0) k_fill64<<<148, 256, 0, s>>>(out->row_ptr, n + 1, 0);
    else
      k_csr<<<148 * 16, 256, 0, s>>>(kb, nu, scale, n, valmode, seed_v, out->row_ptr, out->col,
                                     out->val);
    ok = ck(cudaDeviceSynchronize(), "csr");
  }
  cudaFree(kb);
  if (!ok) {
    synth_gpu_free(out);
    return 3;
  }
  out->nnz = nu;
  return 0;
}

}  // extern "C"
