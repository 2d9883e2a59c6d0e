// spmv_exec_coo: SpMV with B in coordinate (COO) form on the reordered matrix
// (the paper's Table IV "SpMV-COO").
//
// B is read as (row, col, val) triplets sorted by row: the plan's col / val
// arrays plus a row-index array built once from row_ptr (k_coo_rows).  The
// kernel never reads row_ptr, so its compulsory traffic ("updated
// according to the kernel") is 12 NZ (row, col, val) + 4 N (x) + 4 N (y).
//
// k_coo: grid-stride over tiles of COO_TILE = 2048 entries, 8 per thread,
// streamed with 256-bit loads (L2 evict_first when the plan chose it for
// k_lane).  Each thread sums the runs of equal row in its 8 entries
// sequentially in fp32; runs complete inside a thread are written directly.
// A run that crosses a thread boundary is combined by the thread where it
// starts (its "owner"), which adds the following threads' pieces in thread
// order in fp64; a run that crosses a tile boundary leaves an fp64 piece per
// tile and k_coo_fix (one thread per tile) adds them in tile order.  The
// association is fixed by the tile layout, so y is bitwise repeatable; every
// y is rounded once from fp32 (<= 8 terms) or fp64 pieces, well inside the
// north-star tolerance.  Empty rows: each gap between consecutive rows (and
// before the first / after the last entry) is zeroed by the thread holding
// the entry after it, so y is written exactly once and needs no memset --
// unless the matrix has a run of more than 32 empty rows (e.g. RABBIT++ puts
// the isolated vertices last), then y is memset first (4 N bytes) and the
// variant-2 kernel skips the zeroing.
#include <algorithm>
#include <cstdlib>

#include "plan.cuh"

namespace spmv {
namespace {

constexpr int CO_THREADS = 256;
constexpr int CO_E = 8;
constexpr int COO_TILE = CO_THREADS * CO_E;

enum : uint8_t { T_SINGLE = 1, T_PREV = 2, T_NEXT = 4, T_OWN_LAST = 8 };

template <typename OT>
__global__ void k_coo_rows(const OT* __restrict__ rp, int64_t nrows, int32_t* __restrict__ row) {
  const int lane = threadIdx.x & 31;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < nrows; r += W) {
    const int64_t a = (int64_t)rp[r], e = (int64_t)rp[r + 1];
    for (int64_t k = a + lane; k < e; k += 32) row[k] = (int32_t)r;
  }
}

// a run of more than GAP_MAX empty rows somewhere (or before the first /
// after the last entry)?  Such gaps are zeroed by a memset instead of by the
// one thread that holds the entry after them.
constexpr int GAP_MAX = 32;
template <typename OT>
__global__ void k_coo_long_gap(const OT* __restrict__ rp, int64_t nrows, int* __restrict__ flag) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r + GAP_MAX < nrows;
       r += (int64_t)gridDim.x * blockDim.x)
    if (rp[r] == rp[r + GAP_MAX + 1]) {
      *flag = 1;
      return;
    }
}

template <int EF>
__device__ __forceinline__ void ld8(const int32_t* p, int (&r)[8]) {
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
__device__ __forceinline__ void ld8(const float* p, float (&r)[8]) {
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

__device__ __forceinline__ void zero_rows(float* __restrict__ y, int64_t a, int64_t b) {
  for (int64_t g = a; g < b; ++g) y[g] = 0.f;
}

template <int EF>
__global__ void __launch_bounds__(CO_THREADS)
    k_coo(const int32_t* __restrict__ row, const int32_t* __restrict__ col,
          const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
          int64_t nnz, int64_t nrows, int64_t ntiles, int32_t* __restrict__ t_frow,
          int32_t* __restrict__ t_lrow, double* __restrict__ t_fpart,
          double* __restrict__ t_lpart, uint8_t* __restrict__ t_flags) {
  __shared__ int s_hrow[CO_THREADS];
  __shared__ float s_hsum[CO_THREADS];
  __shared__ uint8_t s_single[CO_THREADS];
  const int tid = threadIdx.x;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t e0 = tile * COO_TILE;
    const int64_t eb = e0 + (int64_t)tid * CO_E;
    const int nh = (int)max((int64_t)0, min((int64_t)CO_E, nnz - eb));
    int rr[8], cc[8];
    float vv[8];
    if (nh == CO_E) {
      ld8<EF>(row + eb, rr);
      ld8<EF>(col + eb, cc);
      ld8<EF>(val + eb, vv);
    } else {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        rr[i] = i < nh ? row[eb + i] : -1;
        cc[i] = i < nh ? col[eb + i] : 0;
        vv[i] = i < nh ? val[eb + i] : 0.f;
      }
    }
    float xv[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) xv[i] = i < nh ? __ldg(x + cc[i]) : 0.f;
    // row of the entry before mine: the previous lane's last row (its chunk is
    // full whenever mine is not empty); lane 0 loads it
    int mylast = -1;
#pragma unroll
    for (int i = 0; i < 8; ++i) mylast = i < nh ? rr[i] : mylast;
    int prow = __shfl_up_sync(0xffffffffu, mylast, 1);
    if ((tid & 31) == 0) prow = eb > 0 && nh > 0 ? row[eb - 1] : -1;
    int hrow = -1, cur = -1;
    float hsum = 0.f, run = 0.f;
    bool single = true;
    int last = prow;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (i < nh) {
        const int r = rr[i];
        if (r != cur) {
          if (cur >= 0) {
            if (hrow < 0) {  // closing my head run
              hrow = cur;
              hsum = run;
              if (cur != prow) y[cur] = run;  // started here, ended here
            } else {
              y[cur] = run;  // interior run
            }
            single = false;
          }
          zero_rows(y, (int64_t)last + 1, r);  // empty rows before r
          cur = r;
          run = 0.f;
        }
        run = __fadd_rn(run, __fmul_rn(vv[i], xv[i]));
        last = r;
      }
    }
    if (nh > 0 && eb + nh == nnz) zero_rows(y, (int64_t)cur + 1, nrows);  // after the last entry
    // publish my head (or my only) run; my tail run is `cur` / `run`
    if (single) {
      hrow = cur;
      hsum = run;
    }
    s_hrow[tid] = nh > 0 ? hrow : -1;
    s_hsum[tid] = hsum;
    s_single[tid] = single ? 1 : 0;
    __syncthreads();
    const int64_t tile_end = min(nnz, e0 + COO_TILE);
    const int nthr = (int)((tile_end - e0 + CO_E - 1) / CO_E);
    // owner of my tail run: it starts in this thread unless I hold a single
    // run that continues the previous entry's row
    if (nh > 0 && !(single && cur == prow)) {
      double s = (double)run;
      int t = tid + 1;
      bool open = false;  // chain reached the end of the tile still in row `cur`
      for (;; ++t) {
        if (t >= nthr) {
          open = true;
          break;
        }
        if (s_hrow[t] != cur) break;
        s += (double)s_hsum[t];
        if (!s_single[t]) break;
      }
      const bool next_same = open && tile_end < nnz && row[tile_end] == cur;
      if (next_same) {
        t_lpart[tile] = s;  // k_coo_fix completes it
      } else {
        y[cur] = (float)s;  // == run when no other thread contributed
      }
    }
    if (tid == 0) {
      const int frow = s_hrow[0];
      const bool cprev = e0 > 0 && row[e0 - 1] == frow;
      uint8_t fl = 0;
      if (cprev) {
        double s = (double)s_hsum[0];
        bool whole = s_single[0] != 0;
        if (whole) {
          for (int t = 1; t < nthr; ++t) {
            if (s_hrow[t] != frow) {
              whole = false;
              break;
            }
            s += (double)s_hsum[t];
            if (!s_single[t]) {
              whole = false;
              break;
            }
          }
        }
        t_fpart[tile] = s;
        fl |= T_PREV;
        if (whole) fl |= T_SINGLE;
      }
      // last row of the tile and whether it continues into the next tile
      const int lrow = row[tile_end - 1];
      if (tile_end < nnz && row[tile_end] == lrow) {
        fl |= T_NEXT;
        if (!((fl & T_SINGLE) && cprev)) fl |= T_OWN_LAST;
      }
      t_frow[tile] = frow;
      t_lrow[tile] = lrow;
      t_flags[tile] = fl;
    }
    __syncthreads();
  }
}

// k_coo_w (variant 2): warp tiles of 32 E entries, E = 16 per lane (two
// 256-bit chunks of row / col / val, 16 gathers in flight), no shared memory
// and no CTA barrier.  Lane pieces of a row crossing lanes are combined with
// a segmented suffix scan over the warp in fp64 (shuffles; the association is
// fixed by the lane layout); pieces crossing warp tiles go through k_coo_fix
// exactly like the CTA tiles of k_coo.
constexpr int CW_TILE_MIN = 32 * 8;  // finest warp tile (8 entries per lane): sizes the tile arrays

template <int EF, int MINB, bool ZG, int E>
__global__ void __launch_bounds__(256, MINB)
    k_coo_w(const int32_t* __restrict__ row, const int32_t* __restrict__ col,
            const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
            int64_t nnz, int64_t nrows, int64_t ntiles, int32_t* __restrict__ t_frow,
            int32_t* __restrict__ t_lrow, double* __restrict__ t_fpart,
            double* __restrict__ t_lpart, uint8_t* __restrict__ t_flags) {
  const int lane = threadIdx.x & 31;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t tile = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile < ntiles;
       tile += W) {
    constexpr int TILE = 32 * E;
    const int64_t e0 = tile * TILE;
    const int64_t eb = e0 + (int64_t)lane * E;
    const int nh = (int)max((int64_t)0, min((int64_t)E, nnz - eb));
    int rr[E], cc[E];
    float vv[E];
    if (nh == E) {
      int r8[8], c8[8];
      float v8[8];
#pragma unroll
      for (int h = 0; h < E / 8; ++h) {
        ld8<EF>(row + eb + 8 * h, r8);
        ld8<EF>(col + eb + 8 * h, c8);
        ld8<EF>(val + eb + 8 * h, v8);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          rr[8 * h + i] = r8[i];
          cc[8 * h + i] = c8[i];
          vv[8 * h + i] = v8[i];
        }
      }
    } else {
#pragma unroll
      for (int i = 0; i < E; ++i) {
        rr[i] = i < nh ? row[eb + i] : -1;
        cc[i] = i < nh ? col[eb + i] : 0;
        vv[i] = i < nh ? val[eb + i] : 0.f;
      }
    }
    float xv[E];
#pragma unroll
    for (int i = 0; i < E; ++i) xv[i] = i < nh ? __ldg(x + cc[i]) : 0.f;
    int mylast = -1;
#pragma unroll
    for (int i = 0; i < E; ++i) mylast = i < nh ? rr[i] : mylast;
    int prow = __shfl_up_sync(0xffffffffu, mylast, 1);
    if (lane == 0) prow = e0 > 0 && nh > 0 ? row[e0 - 1] : -1;
    int hrow = -1, cur = -1, last = prow;
    float hsum = 0.f, run = 0.f;
    bool single = true;
#pragma unroll
    for (int i = 0; i < E; ++i) {
      if (i < nh) {
        const int r = rr[i];
        if (r != cur) {
          if (cur >= 0) {
            if (hrow < 0) {
              hrow = cur;
              hsum = run;
              if (cur != prow) y[cur] = run;  // started and ended in this lane
            } else {
              y[cur] = run;  // interior run
            }
            single = false;
          }
          if (ZG) zero_rows(y, (int64_t)last + 1, r);
          cur = r;
          run = 0.f;
        }
        run = __fadd_rn(run, __fmul_rn(vv[i], xv[i]));
        last = r;
      }
    }
    if (ZG && nh > 0 && eb + nh == nnz) zero_rows(y, (int64_t)cur + 1, nrows);
    if (single) {
      hrow = cur;
      hsum = run;
    }
    const int64_t tile_end = min(nnz, e0 + TILE);
    // first row of the next warp tile (decides whether lane 31's chain is open)
    int nxt = -1;
    if (lane == 31 && tile_end < nnz) nxt = row[tile_end];
    nxt = __shfl_sync(0xffffffffu, nxt, 31);
    // cont: my head run continues the previous lane's last row
    const bool cont = nh > 0 && hrow == prow;
    const unsigned contm = __ballot_sync(0xffffffffu, cont);
    // link: my (single) run is continued by the next lane (or next tile)
    const bool link = nh > 0 && single &&
                      (lane < 31 ? ((contm >> (lane + 1)) & 1u) != 0 : nxt == cur);
    const unsigned linkm = __ballot_sync(0xffffffffu, link);
    // segmented suffix sum S_l = v_l + (link_l ? S_{l+1} : 0), v_l = cont ? hsum : 0
    double v = cont ? (double)hsum : 0.0;
    bool f = link && lane < 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const double vo = __shfl_down_sync(0xffffffffu, v, d);
      const bool fo = __shfl_down_sync(0xffffffffu, f ? 1 : 0, d) != 0;
      if (f && lane + d < 32) {
        v += vo;
        f = fo;
      }
    }
    const double vnext = __shfl_down_sync(0xffffffffu, v, 1);  // S_{l+1}
    // chain from lane s runs through lane 31 into the next tile iff links s..31 are all set
    auto open_from = [&](int st) { return st <= 31 && (linkm >> st) == (0xffffffffu >> st); };
    // owner of my tail run (it starts in this lane)
    if (nh > 0 && !(single && cur == prow)) {
      const bool nc = lane < 31 && ((contm >> (lane + 1)) & 1u);
      const double tot = (double)run + (nc ? vnext : 0.0);
      const bool open = lane < 31 ? (nc && open_from(lane + 1)) : (nxt == cur);
      if (open && nxt == cur && tile_end < nnz) t_lpart[tile] = tot;
      else y[cur] = (float)tot;
    }
    if (lane == 0) {
      uint8_t fl = 0;
      if (cont) {
        t_fpart[tile] = v;  // S_0: the first row's piece of this tile
        fl |= T_PREV;
        if (open_from(0)) fl |= T_SINGLE;
      }
      const int lrow = row[tile_end - 1];
      if (tile_end < nnz && nxt == lrow) {
        fl |= T_NEXT;
        if (!((fl & T_SINGLE) && (fl & T_PREV))) fl |= T_OWN_LAST;
      }
      t_frow[tile] = hrow;
      t_lrow[tile] = lrow;
      t_flags[tile] = fl;
    }
  }
}

// rows spanning tiles: the tile where the row starts (T_OWN_LAST) adds the
// pieces of the following tiles in tile order (fp64), rounds once
__global__ void k_coo_fix(int64_t ntiles, const int32_t* __restrict__ t_frow,
                          const int32_t* __restrict__ t_lrow,
                          const double* __restrict__ t_fpart,
                          const double* __restrict__ t_lpart,
                          const uint8_t* __restrict__ t_flags, float* __restrict__ y) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= ntiles || !(t_flags[t] & T_OWN_LAST)) return;
  const int r = t_lrow[t];
  double s = t_lpart[t];
  for (int64_t u = t + 1; u < ntiles; ++u) {
    s += t_fpart[u];
    const uint8_t f = t_flags[u];
    if (!((f & T_SINGLE) && (f & T_NEXT))) break;
  }
  y[r] = (float)s;
}

int sms(int dev) {
  static int n = 0;
  if (!n) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n > 0 ? n : 148;
}

void* dmalloc(size_t bytes) {
  void* q = nullptr;
  if (cudaMalloc(&q, std::max<size_t>(bytes, 256)) != cudaSuccess) {
    cudaGetLastError();
    SPMV_FAIL(SPMV_ENOMEM, "spmv_exec_coo: allocation failed");
  }
  return q;
}

}  // namespace

void coo_build(spmv_plan_s* p, cudaStream_t s) {
  if (p->d_coo_row) return;
  const int64_t nz = p->nnz_local;
  p->coo_tiles = (nz + CW_TILE_MIN - 1) / CW_TILE_MIN;  // the finest tiling bounds every variant
  p->d_coo_row = (int32_t*)dmalloc(sizeof(int32_t) * (size_t)(nz + 8));
  const int64_t T = std::max<int64_t>(p->coo_tiles, 1);
  p->d_coo_trow = (int32_t*)dmalloc(sizeof(int32_t) * 2 * (size_t)T);
  p->d_coo_tpart = (double*)dmalloc(sizeof(double) * 2 * (size_t)T);
  p->d_coo_tflag = (uint8_t*)dmalloc((size_t)T);
  SPMV_CUDA(cudaMemsetAsync(p->d_coo_row, 0, sizeof(int32_t) * (size_t)(nz + 8), s));
  if (p->nrows) {
    const unsigned g = (unsigned)std::min<int64_t>((p->nrows + 7) / 8, (int64_t)sms(p->device) * 32);
    if (p->off64)
      k_coo_rows<int64_t><<<g, 256, 0, s>>>((const int64_t*)p->d_rp, p->nrows, p->d_coo_row);
    else
      k_coo_rows<int32_t><<<g, 256, 0, s>>>((const int32_t*)p->d_rp, p->nrows, p->d_coo_row);
    SPMV_LAUNCH_CHECK();
    int* dflag = (int*)dmalloc(sizeof(int));
    SPMV_CUDA(cudaMemsetAsync(dflag, 0, sizeof(int), s));
    const unsigned gg = (unsigned)std::min<int64_t>((p->nrows + 255) / 256, (int64_t)sms(p->device) * 8);
    if (p->off64) k_coo_long_gap<int64_t><<<gg, 256, 0, s>>>((const int64_t*)p->d_rp, p->nrows, dflag);
    else k_coo_long_gap<int32_t><<<gg, 256, 0, s>>>((const int32_t*)p->d_rp, p->nrows, dflag);
    SPMV_LAUNCH_CHECK();
    int hflag = 0;
    SPMV_CUDA(cudaMemcpyAsync(&hflag, dflag, sizeof(int), cudaMemcpyDeviceToHost, s));
    SPMV_CUDA(cudaStreamSynchronize(s));
    cudaFree(dflag);
    p->coo_memset = hflag != 0;
  }
}

void exec_coo(spmv_plan_s* p, const float* x, float* y, cudaStream_t s) {
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_exec_coo before spmv_permute");
  coo_build(p, s);
  if (!p->nrows) return;
  if (p->nnz_local == 0) {
    SPMV_CUDA(cudaMemsetAsync(y, 0, sizeof(float) * (size_t)p->nrows, s));
    return;
  }
  int v = 2;
  if (const char* e = getenv("SPMV_COO_V")) v = atoi(e) == 1 ? 1 : 2;  // dev knob
  int E = 16;  // entries per lane of k_coo_w
  if (const char* e = getenv("SPMV_COO_E")) E = atoi(e) == 8 ? 8 : 16;  // dev knob
  const int64_t tile = v == 1 ? COO_TILE : 32 * E;
  const int64_t T = (p->nnz_local + tile - 1) / tile;
  int32_t* frow = p->d_coo_trow;
  int32_t* lrow = p->d_coo_trow + T;
  double* fpart = p->d_coo_tpart;
  double* lpart = p->d_coo_tpart + T;
  // every chunk is read by exactly one thread, so evict_first never costs a refetch
  const int ef = p->opts.evict_first ? 1 : 0;
  if (v == 1) {
    const unsigned g = (unsigned)std::min<int64_t>(T, (int64_t)sms(p->device) * 8);
    if (ef)
      k_coo<1><<<g, CO_THREADS, 0, s>>>(p->d_coo_row, p->d_col, p->d_val, x, y, p->nnz_local,
                                        p->nrows, T, frow, lrow, fpart, lpart, p->d_coo_tflag);
    else
      k_coo<0><<<g, CO_THREADS, 0, s>>>(p->d_coo_row, p->d_col, p->d_val, x, y, p->nnz_local,
                                        p->nrows, T, frow, lrow, fpart, lpart, p->d_coo_tflag);
  } else {
    const unsigned g = (unsigned)std::min<int64_t>((T + 7) / 8, (int64_t)sms(p->device) * 16);
    const bool zg = !p->coo_memset;
    if (!zg) SPMV_CUDA(cudaMemsetAsync(y, 0, sizeof(float) * (size_t)p->nrows, s));
    // 16 entries per lane: <= 85 registers, 3 CTAs (24 warps) per SM;
    // 8 entries per lane: <= 51 registers, 5 CTAs (40 warps) per SM
    auto k = E == 8 ? (zg ? (ef ? k_coo_w<1, 5, true, 8> : k_coo_w<0, 5, true, 8>)
                          : (ef ? k_coo_w<1, 5, false, 8> : k_coo_w<0, 5, false, 8>))
                    : (zg ? (ef ? k_coo_w<1, 3, true, 16> : k_coo_w<0, 3, true, 16>)
                          : (ef ? k_coo_w<1, 3, false, 16> : k_coo_w<0, 3, false, 16>));
    k<<<g, 256, 0, s>>>(p->d_coo_row, p->d_col, p->d_val, x, y, p->nnz_local, p->nrows, T, frow,
                        lrow, fpart, lpart, p->d_coo_tflag);
  }
  k_coo_fix<<<(unsigned)((T + 255) / 256), 256, 0, s>>>(T, frow, lrow, fpart, lpart,
                                                        p->d_coo_tflag, y);
  SPMV_LAUNCH_CHECK();
}

void coo_free(spmv_plan_s* p) {
  cudaFree(p->d_coo_row);
  cudaFree(p->d_coo_trow);
  cudaFree(p->d_coo_tpart);
  cudaFree(p->d_coo_tflag);
  p->d_coo_row = p->d_coo_trow = nullptr;
  p->d_coo_tpart = nullptr;
  p->d_coo_tflag = nullptr;
}

void export_coo_rows(spmv_plan_s* p, int32_t* rows, cudaStream_t s) {
  coo_build(p, s);
  if (rows && p->nnz_local)
    SPMV_CUDA(cudaMemcpyAsync(rows, p->d_coo_row, sizeof(int32_t) * (size_t)p->nnz_local,
                              cudaMemcpyDeviceToDevice, s));
}

}  // namespace spmv
