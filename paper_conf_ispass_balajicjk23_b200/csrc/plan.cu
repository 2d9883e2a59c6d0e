// spmv_plan / spmv_permute: validation, inverse permutation, B = P A P^T,
// stream tiles, row classes, hub chunks, hot prefix H, row-block partition.
//
// PAPER.md:86 (§IV-A): reordering "assigns community members consecutive
// IDs"; applied symmetrically B[perm[i], perm[j]] = A[i, j].
// The paper does this on the CPU and never describes it; here it is a chain
// of HBM-bound GPU kernels:
//   validate rows/cols -> inverse perm (bijection check) -> len_B[perm[i]] =
//   len_A[i] -> exclusive scan -> partition -> local row_ptr -> tiles/classes
//   (plan, synchronous) ; relabel+scatter -> per-row stable sort (permute,
//   stream-ordered).
#include <algorithm>
#include <cstring>

#include <cstdlib>

#include "plan.cuh"

namespace spmv {
namespace {

constexpr int TPB = 256;

inline int grid_for(int64_t n, int tpb = TPB, int cap = 148 * 32) {
  int64_t g = (n + tpb - 1) / tpb;
  if (g < 1) g = 1;
  if (g > cap) g = cap;
  return (int)g;
}

#define GRID_STRIDE(i, n)                                                      \
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (n); \
       i += (int64_t)gridDim.x * blockDim.x)

// ---------------------------------------------------------------- validation
template <typename T>
__global__ void k_validate_rp(const T* rp, int64_t n, int64_t nnz, int* flags) {
  GRID_STRIDE(i, n) {
    int64_t a = (int64_t)rp[i], b = (int64_t)rp[i + 1];
    if (b < a || a < 0 || b > nnz) flags[0] = 1;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if ((int64_t)rp[0] != 0 || (int64_t)rp[n] != nnz) flags[0] = 1;
  }
}

__global__ void k_validate_col(const int32_t* col, int64_t nnz, int64_t n, int* flags) {
  GRID_STRIDE(k, nnz) {
    int32_t c = col[k];
    if (c < 0 || (int64_t)c >= n) flags[1] = 1;
  }
}

__global__ void k_identity(int32_t* p, int64_t n) {
  GRID_STRIDE(i, n) p[i] = (int32_t)i;
}

__global__ void k_fill_i32(int32_t* p, int64_t n, int32_t v) {
  GRID_STRIDE(i, n) p[i] = v;
}

// inv[perm[i]] = i; a repeated or out-of-range target flags EPERM.
__global__ void k_inverse(const int32_t* perm, int64_t n, int32_t* inv, int* flags) {
  GRID_STRIDE(i, n) {
    int32_t v = perm[i];
    if (v < 0 || (int64_t)v >= n) {
      flags[2] = 1;
      continue;
    }
    int32_t old = atomicExch(&inv[v], (int32_t)i);
    if (old != -1) flags[2] = 1;
  }
}

// start of B's local row j in A: srcA[perm[i] - rb] = row_ptr_A[i] for the
// rows this rank holds (one coalesced read of row_ptr_A, no inv -> row_ptr_A
// dependent chain in the relabel kernels)
template <typename T>
__global__ void k_srcA(const T* rpA, const int32_t* perm, int64_t n, int64_t rb, int64_t re,
                       int64_t* srcA) {
  GRID_STRIDE(i, n) {
    const int64_t j = perm[i];
    if (j >= rb && j < re) srcA[j - rb] = (int64_t)rpA[i];
  }
}

template <typename T>
__global__ void k_lenB(const T* rpA, const int32_t* perm, int64_t n, int64_t* lenB) {
  GRID_STRIDE(i, n) lenB[perm[i]] = (int64_t)rpA[i + 1] - (int64_t)rpA[i];
}

// --------------------------------------------------------------------- scan
constexpr int SCAN_T = 512, SCAN_I = 8, SCAN_B = SCAN_T * SCAN_I;

__device__ __forceinline__ int64_t block_excl_scan(int64_t v, int64_t* sw, int64_t* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  int64_t inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int64_t t = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += t;
  }
  if (lane == 31) sw[w] = inc;
  __syncthreads();
  if (w == 0) {
    int64_t s = lane < nw ? sw[lane] : 0, si = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int64_t t = __shfl_up_sync(0xffffffffu, si, o);
      if (lane >= o) si += t;
    }
    if (lane < nw) sw[lane] = si - s;
    if (lane == 31) sw[32] = si;
  }
  __syncthreads();
  int64_t r = sw[w] + inc - v;
  if (total) *total = sw[32];
  __syncthreads();
  return r;
}

template <typename T>
__global__ void __launch_bounds__(SCAN_T) k_scan_reduce(const T* in, int64_t n, int64_t* bsum) {
  __shared__ int64_t sw[33];
  int64_t base = (int64_t)blockIdx.x * SCAN_B + (int64_t)threadIdx.x * SCAN_I, s = 0;
#pragma unroll
  for (int j = 0; j < SCAN_I; ++j)
    if (base + j < n) s += (int64_t)in[base + j];
  int64_t tot;
  block_excl_scan(s, sw, &tot);
  if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

// single CTA: exclusive scan of bsum[0..nb) in place, bsum[nb] = total
__global__ void __launch_bounds__(1024) k_scan_top(int64_t* bsum, int64_t nb) {
  __shared__ int64_t sw[33];
  __shared__ int64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < nb; base += 1024) {
    int64_t i = base + threadIdx.x;
    int64_t v = i < nb ? bsum[i] : 0, tot;
    int64_t e = block_excl_scan(v, sw, &tot);
    if (i < nb) bsum[i] = carry + e;
    __syncthreads();
    if (threadIdx.x == 0) carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) bsum[nb] = carry;
}

template <typename T>
__global__ void __launch_bounds__(SCAN_T)
    k_scan_down(const T* in, int64_t n, const int64_t* bsum, int64_t nb, int64_t* out) {
  __shared__ int64_t sw[33];
  int64_t base = (int64_t)blockIdx.x * SCAN_B + (int64_t)threadIdx.x * SCAN_I, s = 0;
  T v[SCAN_I];
#pragma unroll
  for (int j = 0; j < SCAN_I; ++j) {
    v[j] = base + j < n ? in[base + j] : (T)0;
    s += (int64_t)v[j];
  }
  int64_t e = block_excl_scan(s, sw, nullptr) + bsum[blockIdx.x];
#pragma unroll
  for (int j = 0; j < SCAN_I; ++j)
    if (base + j < n) {
      out[base + j] = e;
      e += (int64_t)v[j];
    }
  if (blockIdx.x == 0 && threadIdx.x == 0) out[n] = bsum[nb];
}

// out[0..n] = exclusive scan of in[0..n), out[n] = total.  Returns nothing;
// temp is a device buffer of >= nblocks+1 int64.
template <typename T>
void exclusive_scan(const T* in, int64_t n, int64_t* out, int64_t* temp, cudaStream_t s) {
  int64_t nb = (n + SCAN_B - 1) / SCAN_B;
  if (nb == 0) {
    SPMV_CUDA(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
    return;
  }
  k_scan_reduce<T><<<(unsigned)nb, SCAN_T, 0, s>>>(in, n, temp);
  k_scan_top<<<1, 1024, 0, s>>>(temp, nb);
  k_scan_down<T><<<(unsigned)nb, SCAN_T, 0, s>>>(in, n, temp, nb, out);
  SPMV_LAUNCH_CHECK();
}

int64_t scan_temp_len(int64_t n) { return (n + SCAN_B - 1) / SCAN_B + 2; }

// ---------------------------------------------------------------- partition
// Row blocks balanced on compulsory bytes (reading c29): row r
// starts at byte offset cost(r) = 8 row_ptr_B[r] + (w_off + 8) r of the P:96
// traffic (col + val per entry; row_ptr, x and y per row), and
// b_k = lower_bound(cost, ceil(k * cost(n) / G)).  cost is strictly increasing,
// so every block is a contiguous row range and b_0 = 0, b_G = n.  Grid-stride
// over k in [0, G] (G + 1 bounds).
__global__ void k_partition(const int64_t* rpB, int64_t n, int64_t nnz, int G, int64_t w_off,
                            int64_t* b) {
  const int64_t wr = w_off + 8, total = 8 * nnz + wr * n;
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k <= G; k += gridDim.x * blockDim.x) {
    if (k == 0) { b[0] = 0; continue; }
    if (k == G) { b[G] = n; continue; }
    const int64_t target = ((int64_t)k * total + G - 1) / G;
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (8 * rpB[mid] + wr * mid >= target) hi = mid; else lo = mid + 1;
    }
    b[k] = lo;
  }
}

template <typename OT>
__global__ void k_local_rp(const int64_t* rpB, int64_t rb, int64_t nrows, OT* rp) {
  int64_t base = rpB[rb];
  GRID_STRIDE(i, nrows + 1) rp[i] = (OT)(rpB[rb + i] - base);
}

template <typename OT>
__global__ void k_tiles(const OT* rp, int64_t nrows, int64_t K, int32_t* tiles) {
  GRID_STRIDE(k, K + 1) {
    int64_t target = k * (int64_t)TILE_D;
    int64_t lo = 0, hi = nrows;
    while (lo < hi) {
      int64_t mid = (lo + hi) >> 1;
      if ((int64_t)rp[mid] + mid >= target) hi = mid; else lo = mid + 1;
    }
    tiles[k] = (int32_t)lo;
  }
}

template <typename OT>
__global__ void k_tile_desc(const OT* rp, const int32_t* tiles, int64_t K, TileDesc* d) {
  GRID_STRIDE(t, K) {
    const int r0 = tiles[t], r1 = tiles[t + 1];
    const int64_t e0 = (int64_t)rp[r0];
    uint32_t cnt = 0, nr = 0, extra = 0;
    if (r1 > r0) {
      const int64_t lb = (int64_t)rp[r1 - 1], ee = (int64_t)rp[r1];
      const bool last_long = (ee - lb) > STREAM_MAX;
      cnt = (uint32_t)((last_long ? lb : ee) - e0);
      nr = (uint32_t)((last_long ? r1 - 1 : r1) - r0);
      extra = last_long ? 1u : 0u;
    }
    d[t].e0 = e0;
    d[t].r0 = r0;
    d[t].packed = cnt | (nr << 14) | (extra << 28);
  }
}

// short rows (1 <= L <= SHORT_MAX), those whose first or last 8-entry chunk
// is shared with a neighbouring row (start or end not a multiple of 8), their
// entries, and the chunk slots outside the row that k_lane reads in rows
// spanning >= 2 chunks (a lane gathers every slot of a chunk; slots of a
// neighbour read at another iteration are not merged with the owner's gather)
template <typename OT>
__global__ void k_chunk_share(const OT* rp, int64_t nrows, unsigned long long* cnt) {
  unsigned long long sh = 0, all = 0, ent = 0, waste = 0;
  GRID_STRIDE(r, nrows) {
    const int64_t a = (int64_t)rp[r], e = (int64_t)rp[r + 1];
    if (e - a >= 1 && e - a <= SHORT_MAX) {
      ++all;
      sh += ((a | e) & 7) != 0;
      ent += (unsigned long long)(e - a);
      const int64_t ch = ((e + 7) >> 3) - (a >> 3);
      if (ch >= 2) waste += (unsigned long long)(8 * ch - (e - a));
    }
  }
  for (int o = 16; o > 0; o >>= 1) {
    sh += __shfl_xor_sync(0xffffffffu, sh, o);
    all += __shfl_xor_sync(0xffffffffu, all, o);
    ent += __shfl_xor_sync(0xffffffffu, ent, o);
    waste += __shfl_xor_sync(0xffffffffu, waste, o);
  }
  if ((threadIdx.x & 31) == 0 && all) {
    atomicAdd(cnt, sh);
    atomicAdd(cnt + 1, all);
    atomicAdd(cnt + 2, ent);
    atomicAdd(cnt + 3, waste);
  }
}

// flags for a row-length predicate lo < L <= hi
template <typename OT>
__global__ void k_len_flag(const OT* rp, int64_t nrows, int64_t lo, int64_t hi, int last_only,
                           int32_t* f) {
  GRID_STRIDE(r, nrows) {
    int64_t L = (int64_t)rp[r + 1] - (int64_t)rp[r];
    bool ok = L > lo && L <= hi;
    if (ok && last_only && r + 1 < nrows) {  // only the last row of a stream tile leaves it
      const int64_t t0 = ((int64_t)rp[r] + r) / TILE_D;
      const int64_t t1 = ((int64_t)rp[r + 1] + r + 1) / TILE_D;
      ok = t1 != t0;
    }
    f[r] = ok ? 1 : 0;
  }
}

__global__ void k_compact(const int32_t* f, const int64_t* pos, int64_t n, int32_t* out) {
  GRID_STRIDE(i, n) if (f[i]) out[pos[i]] = (int32_t)i;
}

// MID-list positions q whose row is longer than MID_WIDE (k_small's wide rows)
template <typename OT>
__global__ void k_mid_wide_flag(const OT* rp, const int32_t* mid_rows, int64_t n_mid, int32_t* f) {
  GRID_STRIDE(q, n_mid) {
    const int r = mid_rows[q];
    f[q] = (int64_t)rp[r + 1] - (int64_t)rp[r] > MID_WIDE;
  }
}

template <typename OT>
__global__ void k_nchunks(const OT* rp, const int32_t* hub_rows, int64_t nh, int32_t* nch) {
  GRID_STRIDE(h, nh) {
    int r = hub_rows[h];
    int64_t L = (int64_t)rp[r + 1] - (int64_t)rp[r];
    nch[h] = (int32_t)((L + HUB_CHUNK - 1) / HUB_CHUNK);
  }
}

template <typename OT>
__global__ void k_row_len(const OT* rp, const int32_t* rows, int64_t nl, int64_t* len) {
  GRID_STRIDE(t, nl) len[t] = (int64_t)rp[rows[t] + 1] - (int64_t)rp[rows[t]];
}

__global__ void k_chunks(const int32_t* hub_rows, const int32_t* nch, const int64_t* off,
                         int64_t nh, int32_t* choff, int32_t* crow, int32_t* cidx) {
  GRID_STRIDE(h, nh) {
    int64_t o = off[h];
    choff[h] = (int32_t)o;
    for (int c = 0; c < nch[h]; ++c) {
      crow[o + c] = hub_rows[h];
      cidx[o + c] = c;
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) choff[nh] = (int32_t)off[nh];
}

// colcnt_B[perm[j]] = colcnt_A[j]: histogram of relabelled columns
__global__ void k_colcnt(const int32_t* colA, const int32_t* perm, int64_t nnz, uint32_t* cnt) {
  GRID_STRIDE(k, nnz) atomicAdd(&cnt[perm[colA[k]]], 1u);
}

// any non-finite value in B (permute time): selects the lane kernels that
// mask neighbouring values as well as x (exec.cu lane_row_sum)
__global__ void k_any_nonfinite(const float* v, int64_t n, int* flag) {
  int bad = 0;
  GRID_STRIDE(i, n) bad |= !isfinite(v[i]);
  if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(flag, 1);
}

__global__ void k_sum_u32(const uint32_t* a, int64_t n, unsigned long long* out) {
  unsigned long long acc = 0;
  GRID_STRIDE(i, n) acc += a[i];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(out, acc);
}

__global__ void k_first_cold(const uint32_t* cnt, int64_t n, int64_t nnz,
                             unsigned long long* H) {
  // smallest j with !(colcnt_B[j] * N > NZ): warp-level min first, one atomic per warp
  unsigned long long best = ~0ull;
  GRID_STRIDE(j, n) {
    if (!((int64_t)cnt[j] * n > nnz)) {
      best = (unsigned long long)j;
      break;  // grid-stride order is ascending per thread
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    unsigned long long other = __shfl_xor_sync(0xffffffffu, best, o);
    best = other < best ? other : best;
  }
  if ((threadIdx.x & 31) == 0 && best != ~0ull) atomicMin(H, best);
}

// ------------------------------------------------------------- P A P^T data
// Key (col_B << 32 | position in row) is unique inside a row, so any correct
// sort by key is the stable sort by col_B (duplicates keep A's order).
// rows up to this length are relabelled and sorted in registers (one pass)
constexpr int64_t REG_SORT_MAX = 256;

__device__ __forceinline__ uint64_t mkkey(int32_t c, int64_t rel) {
  return ((uint64_t)(uint32_t)c << 32) | (uint64_t)(uint32_t)rel;
}

// bitonic sort of one key (+ value) per lane over groups of W lanes (W = 16
// or 32; xor partners stay inside the group)
template <int W>
__device__ __forceinline__ void lane_bitonic(uint64_t& key, float& v, int gl) {
#pragma unroll
  for (int k = 2; k <= W; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      const uint64_t ok = __shfl_xor_sync(0xffffffffu, key, j);
      const float ov = __shfl_xor_sync(0xffffffffu, v, j);
      const bool take_min = ((gl & j) == 0) == ((gl & k) == 0);
      if (take_min == (ok < key)) {
        key = ok;
        v = ov;
      }
    }
  }
}

// Register bitonic networks.  Element g = base + k * 32 + lane lives in
// register k of lane `lane` of a warp; a warp holds 32 * E consecutive
// elements.  A compare-exchange stage (block size kk, distance j) orders the
// pair (g, g ^ j) ascending when (g & kk) == 0: partners j >= 32 are in the
// same lane (registers k, k ^ j/32), j < 32 in lane ^ j (shuffles).
template <int E>
__device__ __forceinline__ void warp_stage(uint64_t (&key)[E], float (&v)[E], int lane, int base,
                                           int kk, int j) {
  if (j >= 32) {
    const int jr = j >> 5;
#pragma unroll
    for (int k = 0; k < E; ++k) {
      const int pk = k ^ jr;
      if (pk > k) {
        const bool asc = ((base + (k << 5) + lane) & kk) == 0;
        if ((key[k] > key[pk]) == asc) {
          const uint64_t tk = key[k];
          key[k] = key[pk];
          key[pk] = tk;
          const float tv = v[k];
          v[k] = v[pk];
          v[pk] = tv;
        }
      }
    }
  } else {
#pragma unroll
    for (int k = 0; k < E; ++k) {
      const uint64_t ok = __shfl_xor_sync(0xffffffffu, key[k], j);
      const float ov = __shfl_xor_sync(0xffffffffu, v[k], j);
      const int g = base + (k << 5) + lane;
      const bool take_min = ((g & j) == 0) == ((g & kk) == 0);
      if (take_min == (ok < key[k])) {
        key[k] = ok;
        v[k] = ov;
      }
    }
  }
}

// full bitonic sort of a warp's 32 * E keys (blocks up to 32 * E; with a
// nonzero base, blocks alternate direction by (g & kk) as in a CTA-wide sort)
template <int E>
__device__ __forceinline__ void warp_bitonic(uint64_t (&key)[E], float (&v)[E], int lane,
                                             int base = 0) {
  constexpr int LOG = E == 4 ? 7 : 8;  // 32 * E = 2^LOG keys
  static_assert(E == 4 || E == 8, "warp_bitonic: 4 or 8 keys per lane");
#pragma unroll
  for (int lk = 1; lk <= LOG; ++lk) {  // counted loops: fully unrolled, registers stay registers
#pragma unroll
    for (int lj = lk - 1; lj >= 0; --lj) warp_stage<E>(key, v, lane, base, 1 << lk, 1 << lj);
  }
}

// CTA bitonic sort of NW * 256 keys (NW warps of 8 keys per lane): blocks up
// to 256 inside each warp, then for every larger block size kk the distances
// j >= 256 through shared memory (each thread keeps min or max of its element
// and the partner's, two barriers per stage) and j < 256 inside the warp.
// ~10 barriers for 4096 keys instead of the 78 of a shared-memory network.
template <int NW>
__device__ __forceinline__ void cta_bitonic_regs(uint64_t (&key)[8], float (&v)[8],
                                                 uint64_t* sk, float* sv) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, base = w * 256;
  warp_bitonic<8>(key, v, lane, base);
#pragma unroll 1
  for (int kk = 512; kk <= NW * 256; kk <<= 1) {
#pragma unroll 1
    for (int j = kk >> 1; j >= 256; j >>= 1) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        sk[base + (k << 5) + lane] = key[k];
        sv[base + (k << 5) + lane] = v[k];
      }
      __syncthreads();
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int g = base + (k << 5) + lane;
        const uint64_t ok = sk[g ^ j];
        const bool take_min = ((g & j) == 0) == ((g & kk) == 0);
        if (take_min == (ok < key[k])) {
          key[k] = ok;
          v[k] = sv[g ^ j];
        }
      }
      __syncthreads();
    }
#pragma unroll
    for (int lj = 7; lj >= 0; --lj) warp_stage<8>(key, v, lane, base, kk, 1 << lj);
  }
}

// one row with L <= 32 * E relabelled and sorted by the whole warp in registers
template <int E, typename OT>
__device__ __forceinline__ void warp_relabel_sort(const int32_t* __restrict__ colA,
                                                  const float* __restrict__ valA,
                                                  const int32_t* __restrict__ perm, int64_t a,
                                                  int64_t L, int64_t d, int lane,
                                                  int32_t* __restrict__ colB,
                                                  float* __restrict__ valB) {
  uint64_t key[E];
  float v[E];
#pragma unroll
  for (int k = 0; k < E; ++k) {
    const int i = (k << 5) | lane;
    key[k] = ~0ull;
    v[k] = 0.f;
    if (i < L) {
      key[k] = mkkey(perm[colA[a + i]], i);
      v[k] = valA[a + i];
    }
  }
  warp_bitonic<E>(key, v, lane);
#pragma unroll
  for (int k = 0; k < E; ++k) {
    const int i = (k << 5) | lane;
    if (i < L) {
      colB[d + i] = (int32_t)(key[k] >> 32);
      valB[d + i] = v[k];
    }
  }
}

// Rows with L <= 32 relabelled AND sorted in registers: one read of A's row,
// one gather of perm per entry, one write of B's row.  A warp
// takes rows 2q and 2q+1: a half-warp each when both have L <= 16 (width-16
// sort network), else the whole warp on each in turn (width 32).  Rows with
// 32 < L <= REG_SORT_MAX: k_relabel_sort_mid; longer rows: k_relabel_warp /
// k_relabel_cta and the shared-memory sorts.
template <typename AT, typename OT>
__global__ void __launch_bounds__(256)
    k_relabel_sort_short(const AT* __restrict__ rpA, const int32_t* __restrict__ colA,
                         const float* __restrict__ valA, const int32_t* __restrict__ perm,
                         const int64_t* __restrict__ srcA, int64_t nrows,
                         const OT* __restrict__ rpB, int32_t* __restrict__ colB,
                         float* __restrict__ valB) {
  const int lane = threadIdx.x & 31, half = lane >> 4, hl = lane & 15;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; 2 * q < nrows;
       q += nw) {
    const int64_t r = 2 * q + half;
    int64_t d = 0, L = 0;
    if (r < nrows) {
      d = (int64_t)rpB[r];
      L = (int64_t)rpB[r + 1] - d;
    }
    const int64_t Lo = __shfl_xor_sync(0xffffffffu, L, 16);
    if (L <= 16 && Lo <= 16) {
      uint64_t key = ~0ull;
      float v = 0.f;
      if (hl < L) {
        const int64_t a = srcA[r];
        key = mkkey(perm[colA[a + hl]], hl);
        v = valA[a + hl];
      }
      lane_bitonic<16>(key, v, hl);
      if (hl < L) {
        colB[d + hl] = (int32_t)(key >> 32);
        valB[d + hl] = v;
      }
    } else {
#pragma unroll 1
      for (int h = 0; h < 2; ++h) {
        const int64_t rr = 2 * q + h;
        const int64_t Lh = __shfl_sync(0xffffffffu, L, 16 * h);
        const int64_t dh = __shfl_sync(0xffffffffu, d, 16 * h);
        if (Lh > 32 || rr >= nrows) continue;  // (warp-uniform)
        uint64_t key = ~0ull;
        float v = 0.f;
        if (lane < Lh) {
          const int64_t a = srcA[rr];
          key = mkkey(perm[colA[a + lane]], lane);
          v = valA[a + lane];
        }
        lane_bitonic<32>(key, v, lane);
        if (lane < Lh) {
          colB[dh + lane] = (int32_t)(key >> 32);
          valB[dh + lane] = v;
        }
      }
    }
  }
}

// Rows with 32 < L <= REG_SORT_MAX (the plan's list s1): warp per row,
// relabelled and sorted in registers (4 or 8 keys per lane), one pass -- a
// kernel of its own so the L <= 32 kernel keeps its occupancy (64 registers)
template <typename AT, typename OT>
__global__ void __launch_bounds__(256)
    k_relabel_sort_mid(const int32_t* __restrict__ rows, int64_t nlist,
                       const int32_t* __restrict__ colA, const float* __restrict__ valA,
                       const int32_t* __restrict__ perm, const int64_t* __restrict__ srcA,
                       const OT* __restrict__ rpB, int32_t* __restrict__ colB,
                       float* __restrict__ valB) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; t < nlist; t += nw) {
    const int64_t r = rows[t];
    const int64_t d = (int64_t)rpB[r], L = (int64_t)rpB[r + 1] - d, a = srcA[r];
    if (L <= 128) warp_relabel_sort<4, OT>(colA, valA, perm, a, L, d, lane, colB, valB);
    else warp_relabel_sort<8, OT>(colA, valA, perm, a, L, d, lane, colB, valB);
  }
}

// warp per row for rows with REG_SORT_MAX < L <= WARP_MAX (relabel only; sorted after)
template <typename AT, typename OT>
__global__ void k_relabel_warp(const AT* rpA, const int32_t* colA, const float* valA,
                               const int32_t* perm, const int64_t* srcA,
                               int64_t nrows, const OT* rpB, int32_t* colB, float* valB) {
  const int lane = threadIdx.x & 31;
  int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = w; r < nrows; r += nw) {
    int64_t d = (int64_t)rpB[r], L = (int64_t)rpB[r + 1] - d;
    if (L <= REG_SORT_MAX || L > WARP_MAX) continue;  // k_relabel_sort_short / k_relabel_cta
    int64_t a = srcA[r];
    for (int64_t k = lane; k < L; k += 32) {
      colB[d + k] = perm[colA[a + k]];
      valB[d + k] = valA[a + k];
    }
  }
}

// CTA per long row (list)
template <typename AT, typename OT>
__global__ void k_relabel_cta(const AT* rpA, const int32_t* colA, const float* valA,
                              const int32_t* perm, const int64_t* srcA,
                              const int32_t* rows, int64_t nrows_list, const OT* rpB,
                              int32_t* colB, float* valB) {
  for (int64_t t = blockIdx.x; t < nrows_list; t += gridDim.x) {
    int64_t r = rows[t];
    int64_t d = (int64_t)rpB[r], L = (int64_t)rpB[r + 1] - d;
    int64_t a = srcA[r];
    for (int64_t k = threadIdx.x; k < L; k += blockDim.x) {
      colB[d + k] = perm[colA[a + k]];
      valB[d + k] = valA[a + k];
    }
  }
}

// ----------------------------------------------------------------- row sort
// one row of 256 < L <= P keys per CTA iteration, P / 256 warps of 8 keys
// per lane sorted in registers (cta_bitonic_regs), shared memory only for the
// cross-warp distances
template <int P, typename OT>
__global__ void __launch_bounds__(P / 8)
    k_sort_cta(const OT* rp, const int32_t* rows, int64_t nlist, int32_t* col, float* val) {
  extern __shared__ __align__(16) unsigned char sm[];
  uint64_t* sk = (uint64_t*)sm;
  float* sv = (float*)(sk + P);
  const int lane = threadIdx.x & 31, base = (threadIdx.x >> 5) * 256;
  for (int64_t t = blockIdx.x; t < nlist; t += gridDim.x) {
    const int64_t r = rows[t];
    const int64_t d = (int64_t)rp[r], L = (int64_t)rp[r + 1] - d;
    uint64_t key[8];
    float v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int i = base + (k << 5) + lane;
      key[k] = i < L ? mkkey(col[d + i], i) : ~0ull;
      v[k] = i < L ? val[d + i] : 0.f;
    }
    cta_bitonic_regs<P / 256>(key, v, sk, sv);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int i = base + (k << 5) + lane;
      if (i < L) {
        col[d + i] = (int32_t)(key[k] >> 32);
        val[d + i] = v[k];
      }
    }
    __syncthreads();  // (the next row reuses the exchange buffer)
  }
}

constexpr int BIG_CHUNK = 4096;

// big rows: load keys into a scratch buffer at big_off[b]
template <typename OT>
__global__ void k_big_load(const OT* rp, const int32_t* rows, const int64_t* boff, int64_t nb,
                           const int32_t* col, const float* val, uint64_t* K, float* V) {
  for (int64_t b = blockIdx.x; b < nb; b += gridDim.x) {
    int64_t r = rows[b], d = (int64_t)rp[r], L = (int64_t)rp[r + 1] - d, o = boff[b];
    for (int64_t i = threadIdx.x; i < L; i += blockDim.x) {
      K[o + i] = mkkey(col[d + i], i);
      V[o + i] = val[d + i];
    }
  }
}

// sort every BIG_CHUNK-run of every big row (one CTA of 16 warps per tile of
// the plan's tile list: no empty CTAs for the short big rows), in registers
__global__ void __launch_bounds__(BIG_CHUNK / 8) k_big_chunk_sort(const BigTile* tiles, uint64_t* K,
                                                                  float* V) {
  extern __shared__ __align__(16) unsigned char sm[];
  uint64_t* sk = (uint64_t*)sm;
  float* sv = (float*)(sk + BIG_CHUNK);
  const BigTile t = tiles[blockIdx.x];
  const int64_t e0 = t.o + t.q;
  const int64_t m = min((int64_t)BIG_CHUNK, t.L - t.q);
  const int lane = threadIdx.x & 31, base = (threadIdx.x >> 5) * 256;
  uint64_t key[8];
  float v[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const int i = base + (k << 5) + lane;
    key[k] = i < m ? K[e0 + i] : ~0ull;
    v[k] = i < m ? V[e0 + i] : 0.f;
  }
  cta_bitonic_regs<BIG_CHUNK / 256>(key, v, sk, sv);
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const int i = base + (k << 5) + lane;
    if (i < m) {
      K[e0 + i] = key[k];
      V[e0 + i] = v[k];
    }
  }
}

// One merge pass of width w over every big row, merge path per output tile.
// Runs [base, base + w) = A and [base + w, base + 2w) = B of a row (base a
// multiple of 2w) merge into the same positions of the output; keys are
// unique (column << 32 | position), so "A before B on ties" never arises.
// The tile at diagonal d (its first output, relative to base) takes
// split(d) = #A among the first d outputs = the smallest i with
// A[i] > B[d - i - 1]; k_big_split finds it for every tile (one thread each,
// binary search in global memory), k_big_merge_tile loads the tile's A and B
// pieces into shared memory and merges them (16 outputs per thread, their own
// merge-path search in shared memory), staging the outputs for a coalesced
// store.  Tiles never straddle a pair: 2w is a multiple of BIG_CHUNK.
__device__ __forceinline__ void big_pair(const BigTile& t, int64_t w, int64_t& base, int64_t& nA,
                                         int64_t& nB) {
  base = t.q / (2 * w) * (2 * w);
  nA = min(w, t.L - base);
  nB = max((int64_t)0, min(t.L, base + 2 * w) - (base + w));
}

__global__ void k_big_split(const BigTile* tiles, int64_t nt, int64_t w, const uint64_t* K,
                            int64_t* split) {
  GRID_STRIDE(i, nt) {
    const BigTile t = tiles[i];
    int64_t base, nA, nB;
    big_pair(t, w, base, nA, nB);
    const int64_t d = t.q - base;
    const uint64_t* A = K + t.o + base;
    const uint64_t* B = A + w;
    int64_t lo = max((int64_t)0, d - nB), hi = min(d, nA);
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (A[mid] < B[d - mid - 1]) lo = mid + 1;
      else hi = mid;
    }
    split[i] = lo;
  }
}

constexpr int MT_THREADS = 256, MT_PER = BIG_CHUNK / MT_THREADS;  // 16 outputs per thread
static_assert(MT_PER * MT_THREADS == BIG_CHUNK, "merge tile = BIG_CHUNK outputs");

__global__ void __launch_bounds__(MT_THREADS)
    k_big_merge_tile(const BigTile* tiles, int64_t nt, int64_t w, const int64_t* split,
                     const uint64_t* K, const float* V, uint64_t* K2, float* V2) {
  extern __shared__ __align__(16) unsigned char sm[];
  uint64_t* sk = (uint64_t*)sm;                // [BIG_CHUNK]: A piece then B piece, then outputs
  float* sv = (float*)(sk + BIG_CHUNK);
  const int64_t ti = blockIdx.x;
  const BigTile t = tiles[ti];
  int64_t base, nA, nB;
  big_pair(t, w, base, nA, nB);
  const int64_t d = t.q - base, d1 = min(d + (int64_t)BIG_CHUNK, nA + nB);
  const int64_t m = d1 - d;
  const int64_t out0 = t.o + base + d;
  if (nB == 0) {  // unpaired last run: already sorted, copy
#pragma unroll
    for (int u = 0; u < MT_PER; ++u) {  // (unrolled: every load of the tile in flight)
      const int k = threadIdx.x + u * MT_THREADS;
      if (k < m) {
        K2[out0 + k] = K[out0 + k];
        V2[out0 + k] = V[out0 + k];
      }
    }
    return;
  }
  const int64_t i0 = split[ti];
  const bool next_same = ti + 1 < nt && tiles[ti + 1].o == t.o && tiles[ti + 1].q < base + 2 * w;
  const int64_t i1 = next_same ? split[ti + 1] : nA;
  const int64_t j0 = d - i0, j1 = d1 - i1;
  const int na = (int)(i1 - i0), nb = (int)(j1 - j0);
  const uint64_t* A = K + t.o + base;
  const float* AV = V + t.o + base;
#pragma unroll
  for (int u = 0; u < MT_PER; ++u) {  // the A piece then the B piece, all loads in flight
    const int k = threadIdx.x + u * MT_THREADS;
    if (k < m) {
      const int64_t g = k < na ? i0 + k : w + j0 + (k - na);
      sk[k] = A[g];
      sv[k] = AV[g];
    }
  }
  __syncthreads();
  const uint64_t* sA = sk;
  const uint64_t* sB = sk + na;
  uint64_t ok[MT_PER];
  float ov[MT_PER];
  const int dk = threadIdx.x * MT_PER;
  if (dk < m) {
    int lo = max(0, dk - nb), hi = min(dk, na);
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (sA[mid] < sB[dk - mid - 1]) lo = mid + 1;
      else hi = mid;
    }
    int ia = lo, ib = dk - lo;
#pragma unroll
    for (int u = 0; u < MT_PER; ++u) {
      const bool takeA = ib >= nb || (ia < na && sA[ia] < sB[ib]);
      const int src = takeA ? ia : na + ib;
      ok[u] = sk[src];
      ov[u] = sv[src];
      ia += takeA;
      ib += !takeA;
    }
  }
  __syncthreads();
  if (dk < m) {
#pragma unroll
    for (int u = 0; u < MT_PER; ++u) {
      if (dk + u < m) {
        sk[dk + u] = ok[u];
        sv[dk + u] = ov[u];
      }
    }
  }
  __syncthreads();
#pragma unroll
  for (int u = 0; u < MT_PER; ++u) {
    const int k = threadIdx.x + u * MT_THREADS;
    if (k < m) {
      K2[out0 + k] = sk[k];
      V2[out0 + k] = sv[k];
    }
  }
}

template <typename OT>
__global__ void k_big_store(const OT* rp, const int32_t* rows, const int64_t* boff, int64_t nb,
                            const uint64_t* K, const float* V, int32_t* col, float* val) {
  for (int64_t b = blockIdx.x; b < nb; b += gridDim.x) {
    int64_t r = rows[b], d = (int64_t)rp[r], L = (int64_t)rp[r + 1] - d, o = boff[b];
    for (int64_t i = threadIdx.x; i < L; i += blockDim.x) {
      col[d + i] = (int32_t)(K[o + i] >> 32);
      val[d + i] = V[o + i];
    }
  }
}

// world > 1: global column -> padded x layout (monotone, keeps row order)
__global__ void k_pad_cols(int32_t* col, int64_t nnz, const int64_t* part, int G, int64_t M) {
  GRID_STRIDE(k, nnz) {
    int64_t c = col[k];
    int lo = 0, hi = G;  // owner: part[o] <= c < part[o+1]
    while (hi - lo > 1) {
      int mid = (lo + hi) >> 1;
      if (part[mid] <= c) lo = mid; else hi = mid;
    }
    col[k] = (int32_t)(lo * M + (c - part[lo]));
  }
}

__global__ void k_permute_vec(const int32_t* perm, int64_t n, const float* in, float* out,
                              int inverse) {
  GRID_STRIDE(i, n) {
    if (inverse) out[i] = in[perm[i]];
    else out[perm[i]] = in[i];
  }
}

__global__ void k_pad_vec(const int64_t* part, int G, int64_t M, int64_t n, const float* in,
                          float* out, int to_padded) {
  GRID_STRIDE(i, n) {
    int lo = 0, hi = G;
    while (hi - lo > 1) {
      int mid = (lo + hi) >> 1;
      if (part[mid] <= i) lo = mid; else hi = mid;
    }
    int64_t j = lo * M + (i - part[lo]);
    if (to_padded) out[j] = in[i];
    else out[i] = in[j];
  }
}

// ------------------------------------------------------------- host helpers
template <typename T>
T* dalloc(int64_t n) {
  void* p = nullptr;
  size_t bytes = sizeof(T) * (size_t)std::max<int64_t>(n, 1);
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    SPMV_FAIL(SPMV_ENOMEM, "cudaMalloc of " + std::to_string(bytes) + " bytes failed: " +
                               cudaGetErrorString(e));
  }
  return (T*)p;
}

template <typename T>
void dfree(T*& p) {
  if (p) cudaFree((void*)p);
  p = nullptr;
}

template <typename T>
T d2h_one(const T* d, cudaStream_t s) {
  T h;
  SPMV_CUDA(cudaMemcpyAsync(&h, d, sizeof(T), cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  return h;
}

// flags -> ascending list of rows; returns count
template <typename OT>
int64_t class_list(const OT* rp, int64_t nrows, int64_t lo, int64_t hi, int32_t** out,
                   int32_t* f, int64_t* pos, int64_t* tmp, cudaStream_t s, int last_only = 0) {
  k_len_flag<OT><<<grid_for(nrows), TPB, 0, s>>>(rp, nrows, lo, hi, last_only, f);
  exclusive_scan<int32_t>(f, nrows, pos, tmp, s);
  int64_t cnt = d2h_one(pos + nrows, s);
  *out = dalloc<int32_t>(cnt);
  if (cnt) k_compact<<<grid_for(nrows), TPB, 0, s>>>(f, pos, nrows, *out);
  SPMV_LAUNCH_CHECK();
  return cnt;
}

}  // namespace

template <typename AT, typename OT>
static void build_typed(spmv_plan_s* p, const AT* rpA) {
  cudaStream_t s = p->s;
  const int64_t n = p->n, nnz = p->nnz;
  int* d_flags = dalloc<int>(4);
  SPMV_CUDA(cudaMemsetAsync(d_flags, 0, 4 * sizeof(int), s));
  k_validate_rp<AT><<<grid_for(n), TPB, 0, s>>>(rpA, n, nnz, d_flags);
  k_validate_col<<<grid_for(nnz), TPB, 0, s>>>(p->A_col, nnz, n, d_flags);
  SPMV_LAUNCH_CHECK();
  int h_flags[4];
  SPMV_CUDA(cudaMemcpyAsync(h_flags, d_flags, sizeof(h_flags), cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  if (h_flags[0]) { dfree(d_flags); SPMV_FAIL(SPMV_EINVAL, "row_ptr is not a valid CSR row pointer (row_ptr[0]=0, non-decreasing, row_ptr[n]=nnz)"); }
  if (h_flags[1]) { dfree(d_flags); SPMV_FAIL(SPMV_EINVAL, "column index out of range [0, n)"); }

  // inverse permutation + bijection check
  k_fill_i32<<<grid_for(n), TPB, 0, s>>>(p->d_inv, n, -1);
  k_inverse<<<grid_for(n), TPB, 0, s>>>(p->d_perm, n, p->d_inv, d_flags);
  SPMV_LAUNCH_CHECK();
  int eperm = d2h_one(d_flags + 2, s);
  dfree(d_flags);
  if (eperm) SPMV_FAIL(SPMV_EPERM, "perm is not a bijection on [0, n)");

  // full row pointer of B
  int64_t* lenB = dalloc<int64_t>(n);
  int64_t* rpB = dalloc<int64_t>(n + 1);
  int64_t* tmp = dalloc<int64_t>(scan_temp_len(std::max<int64_t>(n, 1)));
  k_lenB<AT><<<grid_for(n), TPB, 0, s>>>(rpA, p->d_perm, n, lenB);
  exclusive_scan<int64_t>(lenB, n, rpB, tmp, s);
  dfree(lenB);

  // partition (reading c29): compulsory bytes balanced
  int64_t* d_part = dalloc<int64_t>(p->world + 1);
  k_partition<<<(unsigned)((p->world + 256) / 256), 256, 0, s>>>(rpB, n, nnz, p->world,
                                                                  p->off64 ? 8 : 4, d_part);
  p->part.assign(p->world + 1, 0);
  SPMV_CUDA(cudaMemcpyAsync(p->part.data(), d_part, sizeof(int64_t) * (p->world + 1),
                            cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  dfree(d_part);
  p->row_begin = p->part[p->rank];
  p->row_end = p->part[p->rank + 1];
  p->nrows = p->row_end - p->row_begin;
  int64_t lo_nz, hi_nz;
  SPMV_CUDA(cudaMemcpyAsync(&lo_nz, rpB + p->row_begin, 8, cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaMemcpyAsync(&hi_nz, rpB + p->row_end, 8, cudaMemcpyDeviceToHost, s));
  SPMV_CUDA(cudaStreamSynchronize(s));
  p->nnz_before = lo_nz;
  p->nnz_local = hi_nz - lo_nz;
  if (p->world > 1 && p->opts.x_layout == SPMV_XLAYOUT_PADDED) {
    int64_t M = 0;
    for (int k = 0; k < p->world; ++k) M = std::max<int64_t>(M, p->part[k + 1] - p->part[k]);
    M = (M + 31) / 32 * 32;
    if ((int64_t)p->world * M > (int64_t)INT32_MAX)
      SPMV_FAIL(SPMV_EUNSUPPORTED, "padded x layout exceeds int32 column range");
    p->x_stride = M;
    p->x_len = (int64_t)p->world * M;
    p->y_offset = (int64_t)p->rank * M;
  } else {  // global layout: x_B indexed by B's row id, this rank's y at row_begin
    p->x_stride = n;
    p->x_len = n;
    p->y_offset = p->row_begin;
  }

  // local row pointer
  const int64_t nr = p->nrows;
  OT* rp = dalloc<OT>(nr + 1);
  p->d_rp = rp;
  k_local_rp<OT><<<grid_for(nr + 1), TPB, 0, s>>>(rpB, p->row_begin, nr, rp);
  p->d_srcA = dalloc<int64_t>(nr);
  if (n) k_srcA<AT><<<grid_for(n), TPB, 0, s>>>(rpA, p->d_perm, n, p->row_begin, p->row_end, p->d_srcA);
  SPMV_LAUNCH_CHECK();

  // hot prefix H over the full B
  uint32_t* cnt = (uint32_t*)dalloc<uint32_t>(n);
  SPMV_CUDA(cudaMemsetAsync(cnt, 0, sizeof(uint32_t) * std::max<int64_t>(n, 1), s));
  unsigned long long* dH = dalloc<unsigned long long>(1);
  unsigned long long hinit = (unsigned long long)n;
  SPMV_CUDA(cudaMemcpyAsync(dH, &hinit, 8, cudaMemcpyHostToDevice, s));
  if (nnz) k_colcnt<<<grid_for(nnz), TPB, 0, s>>>(p->A_col, p->d_perm, nnz, cnt);
  if (n) k_first_cold<<<grid_for(n), TPB, 0, s>>>(cnt, n, nnz, dH);
  SPMV_LAUNCH_CHECK();
  p->H = (int64_t)d2h_one(dH, s);
  dfree(dH);
  // entries of B whose column lies in the hot prefix [0, H): the window of
  // exec is worth its L2 only if those columns are read much more often than
  // the average column
  p->H_nnz = 0;
  if (p->H > 0) {
    unsigned long long* dsum = dalloc<unsigned long long>(1);
    SPMV_CUDA(cudaMemsetAsync(dsum, 0, 8, s));
    k_sum_u32<<<grid_for(p->H), TPB, 0, s>>>(cnt, p->H, dsum);
    SPMV_LAUNCH_CHECK();
    p->H_nnz = (int64_t)d2h_one(dsum, s);
    dfree(dsum);
  }
  dfree(cnt);
  dfree(rpB);

  // tiles
  p->K = nr ? (p->nnz_local + nr + TILE_D - 1) / TILE_D : 0;
  p->d_tiles = dalloc<int32_t>(p->K + 1);
  k_tiles<OT><<<grid_for(p->K + 1), TPB, 0, s>>>(rp, nr, p->K, p->d_tiles);
  p->d_desc = dalloc<TileDesc>(p->K);
  if (p->K) k_tile_desc<OT><<<grid_for(p->K), TPB, 0, s>>>(rp, p->d_tiles, p->K, p->d_desc);
  SPMV_LAUNCH_CHECK();

  // stream cache policy of the short-row kernel: L2
  // evict_first only when no 8-entry chunk is read by two lanes (<= 1 % of the
  // short rows share one), else a shared chunk evicted early is refetched.
  // Gather policy: k_lane gathers x only for a row's own slots when the short
  // rows carry at least half of the entries and >= 20 % extra slot gathers
  // would be wasted in rows spanning several chunks (27-point stencil: 28 %;
  // r68: 5.68 vs 6.78 ms), else every slot (branch-free, cheaper when chunks
  // are row-aligned: SBM 0.088 vs 0.0996 ms).
  {
    unsigned long long* dc = dalloc<unsigned long long>(4);
    SPMV_CUDA(cudaMemsetAsync(dc, 0, 32, s));
    if (nr) k_chunk_share<OT><<<grid_for(nr), TPB, 0, s>>>(rp, nr, dc);
    SPMV_LAUNCH_CHECK();
    unsigned long long hc[4] = {0, 0, 0, 0};
    SPMV_CUDA(cudaMemcpyAsync(hc, dc, 32, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA(cudaStreamSynchronize(s));
    dfree(dc);
    p->stream_ef = hc[0] * 100 <= hc[1];
    p->lane_nnz = (int64_t)hc[2];
    p->lane_waste = (int64_t)hc[3];
    p->lane_pred = p->lane_nnz > 0 && 2 * p->lane_nnz >= p->nnz_local && 5 * p->lane_waste >= p->lane_nnz;
  }

  // row classes + sort buckets
  int32_t* f = dalloc<int32_t>(nr);
  int64_t* pos = dalloc<int64_t>(nr + 1);
  dfree(tmp);
  tmp = dalloc<int64_t>(scan_temp_len(std::max<int64_t>(nr, 1)));
  p->n_warp = class_list<OT>(rp, nr, STREAM_MAX, WARP_MAX, &p->d_warp_rows, f, pos, tmp, s, 1);
  p->n_mid = class_list<OT>(rp, nr, SHORT_MAX, WARP_MAX, &p->d_mid_rows, f, pos, tmp, s);
  p->n_cta = class_list<OT>(rp, nr, WARP_MAX, CTA_MAX, &p->d_cta_rows, f, pos, tmp, s);
  p->n_hub = class_list<OT>(rp, nr, CTA_MAX, INT64_MAX, &p->d_hub_rows, f, pos, tmp, s);
  if (p->n_hub == 0 && p->n_mid) {  // k_small's wide MID rows (any hub-free plan: SPMV_SMALL=1 forces k_small)
    k_mid_wide_flag<OT><<<grid_for(p->n_mid), TPB, 0, s>>>(rp, p->d_mid_rows, p->n_mid, f);
    exclusive_scan<int32_t>(f, p->n_mid, pos, tmp, s);
    p->n_mid_wide = d2h_one(pos + p->n_mid, s);
    p->d_mid_wide = dalloc<int32_t>(p->n_mid_wide);
    if (p->n_mid_wide) k_compact<<<grid_for(p->n_mid), TPB, 0, s>>>(f, pos, p->n_mid, p->d_mid_wide);
    SPMV_LAUNCH_CHECK();
  }
  spmv_plan_s* ps = p;
  ps->n1 = class_list<OT>(rp, nr, 32, REG_SORT_MAX, &ps->s1, f, pos, tmp, s);  // k_relabel_sort_mid
  ps->n2 = class_list<OT>(rp, nr, REG_SORT_MAX, 1024, &ps->s2, f, pos, tmp, s);
  ps->n3 = class_list<OT>(rp, nr, 1024, BIG_CHUNK, &ps->s3, f, pos, tmp, s);
  ps->nbig = class_list<OT>(rp, nr, BIG_CHUNK, INT64_MAX, &ps->big, f, pos, tmp, s);
  ps->nlong = class_list<OT>(rp, nr, WARP_MAX, INT64_MAX, &ps->longrows, f, pos, tmp, s);
  // big row offsets in the key scratch
  ps->boff = dalloc<int64_t>(ps->nbig + 1);
  if (ps->nbig) {
    int64_t* blen = dalloc<int64_t>(ps->nbig);
    int64_t* t3 = dalloc<int64_t>(scan_temp_len(ps->nbig));
    k_row_len<OT><<<grid_for(ps->nbig), TPB, 0, s>>>(rp, ps->big, ps->nbig, blen);
    exclusive_scan<int64_t>(blen, ps->nbig, ps->boff, t3, s);
    std::vector<int64_t> hl(ps->nbig);
    SPMV_CUDA(cudaMemcpyAsync(hl.data(), blen, 8 * ps->nbig, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA(cudaStreamSynchronize(s));
    std::vector<BigTile> tiles;
    for (int64_t L : hl) {
      for (int64_t q = 0; q < L; q += BIG_CHUNK) tiles.push_back({ps->big_total, L, q});
      ps->big_total += L;
      ps->big_max = std::max(ps->big_max, L);
    }
    ps->nbtile = (int64_t)tiles.size();
    ps->btile = dalloc<BigTile>(ps->nbtile);
    SPMV_CUDA(cudaMemcpyAsync(ps->btile, tiles.data(), sizeof(BigTile) * tiles.size(),
                              cudaMemcpyHostToDevice, s));
    SPMV_CUDA(cudaStreamSynchronize(s));  // host vector lifetime
    dfree(blen);
    dfree(t3);
  } else {
    SPMV_CUDA(cudaMemsetAsync(ps->boff, 0, 8, s));
  }
  // hub chunks
  p->d_hub_choff = dalloc<int32_t>(p->n_hub + 1);
  if (p->n_hub) {
    int32_t* nch = dalloc<int32_t>(p->n_hub);
    int64_t* off = dalloc<int64_t>(p->n_hub + 1);
    int64_t* t2 = dalloc<int64_t>(scan_temp_len(p->n_hub));
    k_nchunks<OT><<<grid_for(p->n_hub), TPB, 0, s>>>(rp, p->d_hub_rows, p->n_hub, nch);
    exclusive_scan<int32_t>(nch, p->n_hub, off, t2, s);
    p->n_chunks = d2h_one(off + p->n_hub, s);
    p->d_chunk_row = dalloc<int32_t>(p->n_chunks);
    p->d_chunk_idx = dalloc<int32_t>(p->n_chunks);
    k_chunks<<<grid_for(p->n_hub), TPB, 0, s>>>(p->d_hub_rows, nch, off, p->n_hub,
                                                  p->d_hub_choff, p->d_chunk_row, p->d_chunk_idx);
    SPMV_LAUNCH_CHECK();
    dfree(nch);
    dfree(off);
    dfree(t2);
  } else {
    SPMV_CUDA(cudaMemsetAsync(p->d_hub_choff, 0, 4, s));
  }
  dfree(f);
  dfree(pos);
  dfree(tmp);

  // local B storage (+8 elements of zero padding for 16-byte bulk copies)
  p->d_col = dalloc<int32_t>(p->nnz_local + 8);
  p->d_val = dalloc<float>(p->nnz_local + 8);
  SPMV_CUDA(cudaMemsetAsync(p->d_col + p->nnz_local, 0, 32, s));
  SPMV_CUDA(cudaMemsetAsync(p->d_val + p->nnz_local, 0, 32, s));
  // exec scratch
  p->d_chunk_part = dalloc<double>(p->n_chunks);
  p->d_ss = dalloc<double>(4);
  p->d_ss_part = dalloc<double>(nr / 16384 + 2);  // norm segment sums (exec.cu SS_ROWS rows each)
  SPMV_CUDA(cudaStreamSynchronize(s));
}

template <typename AT, typename OT>
static void permute_typed(spmv_plan_s* p, const AT* rpA, cudaStream_t s) {
  OT* rp = (OT*)p->d_rp;
  spmv_plan_s* ps = p;
  const int64_t nr = p->nrows;
  if (nr) {
    k_relabel_sort_short<AT, OT><<<grid_for((nr + 1) / 2 * 32), 256, 0, s>>>(
        rpA, p->A_col, p->A_val, p->d_perm, p->d_srcA, nr, rp, p->d_col, p->d_val);
    if (ps->n1)
      k_relabel_sort_mid<AT, OT><<<grid_for(ps->n1 * 32), 256, 0, s>>>(
          ps->s1, ps->n1, p->A_col, p->A_val, p->d_perm, p->d_srcA, rp, p->d_col, p->d_val);
    if (ps->n2 + ps->n3 + ps->nbig)  // rows with L > REG_SORT_MAX exist
      k_relabel_warp<AT, OT><<<grid_for(nr * 32), TPB, 0, s>>>(
          rpA, p->A_col, p->A_val, p->d_perm, p->d_srcA, nr, rp, p->d_col, p->d_val);
    if (ps->nlong)
      k_relabel_cta<AT, OT><<<(unsigned)std::min<int64_t>(ps->nlong, 148 * 8), 512, 0, s>>>(
          rpA, p->A_col, p->A_val, p->d_perm, p->d_srcA, ps->longrows, ps->nlong,
          rp, p->d_col, p->d_val);
    SPMV_LAUNCH_CHECK();
    if (ps->n2) {
      k_sort_cta<1024, OT><<<(unsigned)std::min<int64_t>(ps->n2, 148 * 16), 128, 1024 * 12, s>>>(
          rp, ps->s2, ps->n2, p->d_col, p->d_val);
    }
    if (ps->n3) {
      k_sort_cta<4096, OT><<<(unsigned)std::min<int64_t>(ps->n3, 148 * 4), 512, 4096 * 12, s>>>(
          rp, ps->s3, ps->n3, p->d_col, p->d_val);
    }
    SPMV_LAUNCH_CHECK();
    if (ps->nbig) {
      uint64_t* K1 = dalloc<uint64_t>(ps->big_total);
      uint64_t* K2 = dalloc<uint64_t>(ps->big_total);
      float* V1 = dalloc<float>(ps->big_total);
      float* V2 = dalloc<float>(ps->big_total);
      unsigned nb = (unsigned)std::min<int64_t>(ps->nbig, 148 * 8);
      k_big_load<OT><<<nb, 512, 0, s>>>(rp, ps->big, ps->boff, ps->nbig, p->d_col, p->d_val, K1, V1);
      k_big_chunk_sort<<<(unsigned)ps->nbtile, BIG_CHUNK / 8, BIG_CHUNK * 12, s>>>(ps->btile, K1, V1);
      SPMV_LAUNCH_CHECK();
      int64_t* split = dalloc<int64_t>(ps->nbtile);
      for (int64_t w = BIG_CHUNK; w < ps->big_max; w *= 2) {
        k_big_split<<<grid_for(ps->nbtile), TPB, 0, s>>>(ps->btile, ps->nbtile, w, K1, split);
        k_big_merge_tile<<<(unsigned)ps->nbtile, MT_THREADS, BIG_CHUNK * 12, s>>>(
            ps->btile, ps->nbtile, w, split, K1, V1, K2, V2);
        SPMV_LAUNCH_CHECK();
        std::swap(K1, K2);
        std::swap(V1, V2);
      }
      k_big_store<OT><<<nb, 512, 0, s>>>(rp, ps->big, ps->boff, ps->nbig, K1, V1, p->d_col, p->d_val);
      SPMV_LAUNCH_CHECK();
      SPMV_CUDA(cudaStreamSynchronize(s));  // scratch lifetime
      dfree(K1); dfree(K2); dfree(V1); dfree(V2); dfree(split);
    }
  }
  if (p->nnz_local) {
    int* fl = dalloc<int>(1);
    SPMV_CUDA(cudaMemsetAsync(fl, 0, sizeof(int), s));
    k_any_nonfinite<<<grid_for(p->nnz_local), TPB, 0, s>>>(p->d_val, p->nnz_local, fl);
    SPMV_LAUNCH_CHECK();
    p->val_nonfinite = d2h_one(fl, s) != 0;
    dfree(fl);
  }
  if (padded(p) && p->nnz_local) {
    int64_t* d_part = dalloc<int64_t>(p->world + 1);
    SPMV_CUDA(cudaMemcpyAsync(d_part, p->part.data(), 8 * (p->world + 1), cudaMemcpyHostToDevice, s));
    k_pad_cols<<<grid_for(p->nnz_local), TPB, 0, s>>>(p->d_col, p->nnz_local, d_part, p->world,
                                                      p->x_stride);
    SPMV_LAUNCH_CHECK();
    SPMV_CUDA(cudaStreamSynchronize(s));
    dfree(d_part);
  }
}

// ---------------------------------------------- RABBIT++ post-pass (GPU)
// SURVEY §8(f4).  Inputs by OLD vertex id: the RABBIT
// permutation and the top-level community of every vertex.
template <typename AT>
__global__ void k_pp_scan_entries(const AT* rp, const int32_t* col, int64_t n,
                                  const int32_t* comm, unsigned long long* colcnt,
                                  uint8_t* insular) {
  // warp per row: column counts (diagonal and duplicates included, reading
  // c13) and insularity (an off-diagonal entry (i, j) with comm[i] != comm[j]
  // makes both i and j non-insular: S = Bp + Bp^T, reading c5)
  const int lane = threadIdx.x & 31;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += W) {
    const int64_t a = (int64_t)rp[i], e = (int64_t)rp[i + 1];
    const int32_t ci = comm[i];
    for (int64_t k = a + lane; k < e; k += 32) {
      const int32_t j = col[k];
      atomicAdd(&colcnt[j], 1ull);
      if (j != i && comm[j] != ci) {
        insular[i] = 0;
        insular[j] = 0;
      }
    }
  }
}

// group of the vertex at RABBIT position q: 0 non-insular hub, 1 non-insular
// non-hub, 2 insular; flags[g * n + q] = (group == g)
__global__ void k_pp_groups(const int32_t* perm_rabbit, const unsigned long long* colcnt,
                            const uint8_t* insular, int64_t n, int64_t nnz, int32_t* flags) {
  GRID_STRIDE(v, n) {
    const int64_t q = perm_rabbit[v];
    const bool hub = (__int128)colcnt[v] * n > (__int128)nnz;  // P:181, reading c14
    const int g = insular[v] ? 2 : (hub ? 0 : 1);
    flags[q] = g == 0;
    flags[n + q] = g == 1;
    flags[2 * n + q] = g == 2;
  }
}

// new id = start of the vertex's group + its rank among the group in RABBIT order
__global__ void k_pp_assign(const int32_t* perm_rabbit, const int32_t* flags, const int64_t* pos,
                            int64_t n, int32_t* perm_out) {
  const int64_t c0 = pos[n], c1 = pos[2 * n + 1];
  GRID_STRIDE(v, n) {
    const int64_t q = perm_rabbit[v];
    int64_t id;
    if (flags[q]) id = pos[q];
    else if (flags[n + q]) id = c0 + pos[n + 1 + q];
    else id = c0 + c1 + pos[2 * n + 2 + q];
    perm_out[v] = (int32_t)id;
  }
}

void rabbitpp_gpu(const spmv_csr_t* A, const int32_t* perm_rabbit, const int32_t* comm,
                  int32_t* perm_out, cudaStream_t s) {
  const int64_t n = A->n, nnz = A->nnz;
  if (n == 0) return;
  {  // the header's EINVAL promise: CSR, column range, comm range, perm bijection
    int* fl = dalloc<int>(6);  // [0] row_ptr, [1] col, [2] perm, [4] comm
    int32_t* inv = dalloc<int32_t>(n);
    SPMV_CUDA(cudaMemsetAsync(fl, 0, 6 * sizeof(int), s));
    if (A->row_ptr64) k_validate_rp<int64_t><<<grid_for(n), TPB, 0, s>>>(A->row_ptr64, n, nnz, fl);
    else k_validate_rp<int32_t><<<grid_for(n), TPB, 0, s>>>(A->row_ptr32, n, nnz, fl);
    if (nnz) k_validate_col<<<grid_for(nnz), TPB, 0, s>>>(A->col_idx, nnz, n, fl);
    k_validate_col<<<grid_for(n), TPB, 0, s>>>(comm, n, n, fl + 3);  // comm[v] in [0, n) -> fl[4]
    k_fill_i32<<<grid_for(n), TPB, 0, s>>>(inv, n, -1);
    k_inverse<<<grid_for(n), TPB, 0, s>>>(perm_rabbit, n, inv, fl);
    SPMV_LAUNCH_CHECK();
    int h[6];
    SPMV_CUDA(cudaMemcpyAsync(h, fl, sizeof(h), cudaMemcpyDeviceToHost, s));
    SPMV_CUDA(cudaStreamSynchronize(s));
    dfree(fl);
    dfree(inv);
    if (h[0]) SPMV_FAIL(SPMV_EINVAL, "spmv_rabbitpp_gpu: row_ptr is not a valid CSR row pointer");
    if (h[1]) SPMV_FAIL(SPMV_EINVAL, "spmv_rabbitpp_gpu: column index out of range [0, n)");
    if (h[2]) SPMV_FAIL(SPMV_EPERM, "spmv_rabbitpp_gpu: perm_rabbit is not a bijection on [0, n)");
    if (h[4]) SPMV_FAIL(SPMV_EINVAL, "spmv_rabbitpp_gpu: community id out of range [0, n)");
  }
  unsigned long long* cnt = dalloc<unsigned long long>(n);
  uint8_t* ins = dalloc<uint8_t>(n);
  int32_t* flags = dalloc<int32_t>(3 * n);
  int64_t* pos = dalloc<int64_t>(3 * (n + 1));
  int64_t* tmp = dalloc<int64_t>(scan_temp_len(n));
  SPMV_CUDA(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * n, s));
  SPMV_CUDA(cudaMemsetAsync(ins, 1, (size_t)n, s));
  const unsigned gw = (unsigned)std::min<int64_t>((n + 7) / 8, 148 * 64);
  if (A->row_ptr64)
    k_pp_scan_entries<int64_t><<<gw, 256, 0, s>>>(A->row_ptr64, A->col_idx, n, comm, cnt, ins);
  else
    k_pp_scan_entries<int32_t><<<gw, 256, 0, s>>>(A->row_ptr32, A->col_idx, n, comm, cnt, ins);
  k_pp_groups<<<grid_for(n), TPB, 0, s>>>(perm_rabbit, cnt, ins, n, nnz, flags);
  for (int g = 0; g < 3; ++g) exclusive_scan<int32_t>(flags + g * n, n, pos + g * (n + 1), tmp, s);
  k_pp_assign<<<grid_for(n), TPB, 0, s>>>(perm_rabbit, flags, pos, n, perm_out);
  SPMV_LAUNCH_CHECK();
  SPMV_CUDA(cudaStreamSynchronize(s));  // scratch lifetime
  dfree(cnt);
  dfree(ins);
  dfree(flags);
  dfree(pos);
  dfree(tmp);
}

// ------------------------------------------------------------------ public
void plan_build(spmv_plan_s* p, const spmv_csr_t* A, const int32_t* perm) {
  const int64_t n = p->n;
  p->d_perm = dalloc<int32_t>(n);
  p->d_inv = dalloc<int32_t>(n);
  if (perm) {
    SPMV_CUDA(cudaMemcpyAsync(p->d_perm, perm, 4 * std::max<int64_t>(n, 0), cudaMemcpyDeviceToDevice, p->s));
  } else {
    k_identity<<<grid_for(n), TPB, 0, p->s>>>(p->d_perm, n);
    SPMV_LAUNCH_CHECK();
  }
  if (A->row_ptr64) {
    if (p->off64) build_typed<int64_t, int64_t>(p, A->row_ptr64);
    else build_typed<int64_t, int32_t>(p, A->row_ptr64);
  } else {
    if (p->off64) build_typed<int32_t, int64_t>(p, A->row_ptr32);
    else build_typed<int32_t, int32_t>(p, A->row_ptr32);
  }
}

void plan_permute(spmv_plan_s* p, cudaStream_t s) {
  if (p->A_rp64) {
    if (p->off64) permute_typed<int64_t, int64_t>(p, p->A_rp64, s);
    else permute_typed<int64_t, int32_t>(p, p->A_rp64, s);
  } else {
    if (p->off64) permute_typed<int32_t, int64_t>(p, p->A_rp32, s);
    else permute_typed<int32_t, int32_t>(p, p->A_rp32, s);
  }
  p->permuted = true;
}

void permute_vec(spmv_plan_s* p, const float* in, float* out, int inverse, cudaStream_t s) {
  if (p->n == 0) return;
  k_permute_vec<<<grid_for(p->n), TPB, 0, s>>>(p->d_perm, p->n, in, out, inverse);
  SPMV_LAUNCH_CHECK();
}

void pad_vec(spmv_plan_s* p, const float* in, float* out, int to_padded, cudaStream_t s) {
  if (p->n == 0) return;
  if (!padded(p)) {  // global layout: the padded form is the vector itself
    SPMV_CUDA(cudaMemcpyAsync(out, in, 4 * p->n, cudaMemcpyDeviceToDevice, s));
    return;
  }
  int64_t* d_part = dalloc<int64_t>(p->world + 1);
  SPMV_CUDA(cudaMemcpyAsync(d_part, p->part.data(), 8 * (p->world + 1), cudaMemcpyHostToDevice, s));
  k_pad_vec<<<grid_for(p->n), TPB, 0, s>>>(d_part, p->world, p->x_stride, p->n, in, out, to_padded);
  SPMV_LAUNCH_CHECK();
  SPMV_CUDA(cudaStreamSynchronize(s));
  dfree(d_part);
}

void plan_free(spmv_plan_s* p) {
  coo_free(p);
  dfree(p->s1); dfree(p->s2); dfree(p->s3); dfree(p->big); dfree(p->boff); dfree(p->btile);
  dfree(p->longrows);
  dfree(p->d_perm); dfree(p->d_inv); dfree(p->d_srcA);
  if (p->d_rp) { cudaFree(p->d_rp); p->d_rp = nullptr; }
  dfree(p->d_col); dfree(p->d_val); dfree(p->d_tiles); dfree(p->d_cta_rows); dfree(p->d_desc);
  dfree(p->d_warp_rows); dfree(p->d_mid_rows);
  dfree(p->d_mid_wide);
  dfree(p->d_chunk_part4);
  dfree(p->d_hub_rows); dfree(p->d_hub_choff); dfree(p->d_chunk_row); dfree(p->d_chunk_idx);
  dfree(p->d_chunk_part);
  dfree(p->d_ss); dfree(p->d_u); dfree(p->d_ss_part);
  for (int i = 0; i < 2; ++i) {
    if (p->aux[i]) { cudaStreamDestroy(p->aux[i]); p->aux[i] = nullptr; }
    if (p->ev_join[i]) { cudaEventDestroy(p->ev_join[i]); p->ev_join[i] = nullptr; }
  }
  if (p->ev_fork) { cudaEventDestroy(p->ev_fork); p->ev_fork = nullptr; }
}

}  // namespace spmv
