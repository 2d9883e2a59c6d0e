// spmv_exec / spmv_exec_scaled / spmv_iterate: the hot path.
//
// Alg. 1 of the paper:  Y[row] += values[i] * X[coords[i]].
// B200 design:
//   k_panel      persistent CTAs over contiguous row panels of stream tiles
//                (TILE_D = 3072 rows+entries, row aligned); a 2-stage ring of
//                cp.async.bulk (TMA bulk engine) + mbarrier copies of tile
//                col/val (L2 evict_first); a sliding
//                shared-memory x window follows the diagonal, so
//                community-local gathers are shared-memory reads; rows reduced
//                in the canonical order of include/spmv.h (thread per row
//                L <= 32, warp per row 32 < L <= 1024); y written once.
//   k_warp_rows  one warp per row, 1024 < L <= 2048 (32 strided partials + tree),
//                col/val streamed with 4 independent 128-B warp loads in flight.
//   k_cta_rows   one CTA per row, 2048 < L <= 16384 (256 strided partials + tree).
//   k_hub_chunk  one CTA per 16384-entry chunk of a hub row (merge-path split);
//   k_hub_fix    fp64 combine of the chunk sums in chunk order.
//   k_ss_y / k_ss_final  power-iteration norm: fp64 sum of y^2 over fixed
//                16384-row segments of y, then the segment sums in order
//                (deterministic, independent of grid and row classes).
// No tensor cores: SpMV is not a dense contraction (AI <= 0.25 flop/B).
#include <atomic>
#include <cmath>
#include <cstdlib>

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
}

__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
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

// Fused exchange (spmv_exec_scaled_bcast): the scaled y of a
// row is stored straight into the next-x buffer of every rank (NVLink peer
// stores through CUDA IPC mappings) instead of a local y + NCCL all-gather.
// Only the exec_scaled (SS) instantiations look at it.
struct YDst {
  float* p[8];  // next-x buffers of ranks 0..n-1, each already offset by y_offset
  int n;        // 0: plain local y
};

template <bool SS>
__device__ __forceinline__ void store_y(float* __restrict__ y, const YDst& d, int64_t r, float v) {
  if constexpr (SS) {
    if (d.n) {
#pragma unroll
      for (int k = 0; k < 8; ++k)  // constant indices: the pointers stay in the param space
        if (k < d.n) d.p[k][r] = v;
      return;
    }
  }
  y[r] = v;
}

template <bool SS>
__device__ __forceinline__ void fence_bcast(const YDst& d) {
  if constexpr (SS) {
    if (d.n) __threadfence_system();  // peer stores visible before the caller's collective
  }
}

__device__ __forceinline__ float warp_tree(float s) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  return s;
}

__device__ __forceinline__ double warp_sum_d(double s) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  return s;
}

// x gather of the lane-mode kernels: L1-allocating read-only load (community
// order puts the columns of nearby rows on few lines)
__device__ __forceinline__ float gx(const float* __restrict__ x, int c) { return __ldg(x + c); }

// Streamed col / val entries of the MID / CTA / hub kernels.  SM 0: ld.cs
// (L1 and L2 evict-first); SM 1: no L1 allocation, so the L1 keeps gathered x
// lines only; SM 2: no L1 allocation and L2 evict_first.
// (SM 2 takes an L2::evict_first cache policy from createpolicy: the static
// qualifier exists only for 256-bit loads.)
template <int SM>
__device__ __forceinline__ int32_t lds(const int32_t* p, uint64_t pol) {
  if constexpr (SM == 0) {
    return __ldcs(p);
  } else {
    int32_t r;
    if constexpr (SM == 1)
      asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r) : "l"(p));
    else
      asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
  }
}
template <int SM>
__device__ __forceinline__ float lds(const float* p, uint64_t pol) {
  if constexpr (SM == 0) {
    return __ldcs(p);
  } else {
    float r;
    if constexpr (SM == 1)
      asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
    else
      asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(r) : "l"(p), "l"(pol));
    return r;
  }
}
template <int SM>
__device__ __forceinline__ uint64_t stream_policy() {
  uint64_t pol = 0;
  if constexpr (SM == 2) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

// ------------------------------------------------------------ stream tiles
// k_panel: persistent CTAs, each over a contiguous range of stream tiles (a
// panel of consecutive rows), two CTAs of 16 warps per SM.  Thread 0 keeps the
// next tile in flight while the current one is computed (2-stage ring) with
// cp.async.bulk copies (TMA bulk engine) of the tile's col / val (L2
// evict_first), completing on per-stage mbarriers; tile descriptors are
// precomputed by the plan and prefetched, so the producer has no dependent
// loads on its path.  Tiles are large (TILE_D = 3072 rows+entries, ~24 KB of
// matrix) so per-tile bookkeeping is amortised over ~6 entries per thread.
// x is read through a SLIDING WINDOW: a shared-memory ring of XWIN floats that
// holds x[c] at slot c % XWIN for c in [whi(t) - XWIN, whi(t)), whi(t) =
// (last row of tile t) + XLEAD.  Community-ordered matrices put most columns
// of a row near its diagonal (Fig. 1), so most gathers become
// shared-memory reads instead of one L1/L2 request per scattered line; other
// columns fall back to __ldg through L2.  The CTA advances the ring after the
// tile's last window read (prefetched into registers during the tile, ordered
// by __syncthreads), so no two writers ever race on a slot.  Rows are reduced
// in the canonical order of include/spmv.h, so where x came from never
// changes y.
constexpr int PT_THREADS = 512;
constexpr int PT_STAGES = 2;
constexpr int XWIN = 4096;   // x window ring (floats, power of two)
constexpr int XLEAD = 1536;  // window leads the tile's end row by this many columns
constexpr int PROD_LEN = TILE_BUF + TILE_BUF / 16 + 1;
constexpr int MID_CAP = (TILE_D + STREAM_MAX) / (SHORT_MAX + 1) + 2;

struct alignas(16) PanelSmem {
  int32_t col[PT_STAGES][TILE_BUF];
  float val[PT_STAGES][TILE_BUF];
  float win[XWIN];
  float prod[PROD_LEN];
  uint64_t bar[PT_STAGES];
  int32_t mid[MID_CAP];
  int mid_n;
};
static_assert((TILE_BUF * 4) % 16 == 0, "stage buffers must stay 16-byte aligned");
static_assert(TILE_D <= TILE_BUF, "row results reuse a col stage");

// padded index of the product array: one pad word per 16, which makes the
// thread-per-row pass bank-conflict free for rows of 16 (and light otherwise)
__device__ __forceinline__ int pidx(int j) { return j + (j >> 4); }

struct TileView {
  int64_t e0;
  int r0, rend, r1, cnt;
};

__device__ __forceinline__ TileView view(const TileDesc& d) {
  TileView v;
  v.e0 = d.e0;
  v.r0 = d.r0;
  v.cnt = (int)(d.packed & 0x3fffu);
  v.rend = v.r0 + (int)((d.packed >> 14) & 0x3fffu);
  v.r1 = v.rend + (int)((d.packed >> 28) & 1u);
  return v;
}

__device__ __forceinline__ void issue_panel_tile(const TileView& v,
                                                 const int32_t* __restrict__ col,
                                                 const float* __restrict__ val, PanelSmem& S,
                                                 int s, uint64_t pol) {
  const int64_t a0 = v.e0 & ~3ll, a1 = (v.e0 + v.cnt + 3) & ~3ll;
  const uint32_t bytes = (uint32_t)((a1 - a0) * 4);
  mbar_expect_tx(&S.bar[s], 2 * bytes);
  if (bytes) {
    bulk_g2s(S.col[s], col + a0, bytes, &S.bar[s], pol);
    bulk_g2s(S.val[s], val + a0, bytes, &S.bar[s], pol);
  }
}

template <typename OT, bool SS>
__global__ void __launch_bounds__(PT_THREADS, 2)
    k_panel(const OT* __restrict__ rp, const int32_t* __restrict__ col,
            const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
            const TileDesc* __restrict__ desc, int64_t K, int64_t diag, int64_t xlen,
            int use_win_i, const double* __restrict__ ss_in,
            int evict_first) {
  constexpr int SEGW = 1;  // window advance prefetched per thread (512 floats)
  constexpr int RPF = 1;   // row pointers prefetched per thread
  extern __shared__ __align__(16) unsigned char smraw[];
  PanelSmem& S = *reinterpret_cast<PanelSmem*>(smraw);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int64_t k0 = (K * (int64_t)blockIdx.x) / gridDim.x;
  const int64_t k1 = (K * (int64_t)(blockIdx.x + 1)) / gridDim.x;
  if (k0 >= k1) return;
  const bool use_win = use_win_i != 0;
  const int xl = (int)xlen, dg = (int)diag;  // columns are int32 (n < 2^31)
  const float alpha = alpha_of(ss_in);
  uint64_t pol = 0;
  TileView v = view(desc[k0]);
  TileView vn = v;
  if (k0 + 1 < k1) vn = view(desc[k0 + 1]);
  if (tid == 0) {
    pol = l2_policy(evict_first);
    for (int s = 0; s < PT_STAGES; ++s) mbar_init(&S.bar[s], 1);
    fence_mbar_init();
    issue_panel_tile(v, col, val, S, 0, pol);
  }
  // initial window [whi(k0) - XWIN, whi(k0))
  int whi = 0;
  if (use_win) {
    const int h = v.r1 + dg + XLEAD;
    whi = h < xl ? h : xl;
    for (int u = tid; u < XWIN; u += PT_THREADS) {
      const int c = whi - XWIN + u;
      if (c >= 0) S.win[c & (XWIN - 1)] = __ldg(x + c);
    }
  }
  __syncthreads();
  float* __restrict__ pr = S.prod;
  float* __restrict__ win = S.win;
  int s = 0;
  uint32_t ph = 0;
  for (int64_t t = k0; t < k1; ++t) {
    const bool has_next = t + 1 < k1;
    if (tid == 0) {
      S.mid_n = 0;
      if (has_next) {  // the other stage held tile t-1, finished before the last barrier
        fence_proxy_async();
        issue_panel_tile(vn, col, val, S, s ^ 1, pol);
      }
    }
    const int nr = v.rend - v.r0;
    // row pointers of this tile (prefetch)
    OT rb[RPF], re[RPF];
#pragma unroll
    for (int u = 0; u < RPF; ++u) {
      const int q = tid + u * PT_THREADS;
      rb[u] = q < nr ? rp[v.r0 + q] : (OT)0;
      re[u] = q < nr ? rp[v.r0 + q + 1] : (OT)0;
    }
    // window of this tile: [vlo, whi); warp 0 prefetches the advance for t+1
    const int vlo = whi - XWIN > 0 ? whi - XWIN : 0;
    const uint32_t span = use_win ? (uint32_t)(whi - vlo) : 0u;
    int whi_next = whi, seg_lo = whi;
    float segv[SEGW];
    if (use_win && has_next) {
      const int h = vn.r1 + dg + XLEAD;
      whi_next = h < xl ? h : xl;
      seg_lo = whi_next - whi > XWIN ? whi_next - XWIN : whi;
#pragma unroll
      for (int u = 0; u < SEGW; ++u) {
        const int c = seg_lo + tid + PT_THREADS * u;
        segv[u] = c < whi_next ? __ldg(x + c) : 0.f;
      }
    }
    mbar_wait(&S.bar[s], ph);
    const int cnt = v.cnt, sh = (int)(v.e0 & 3);
    const int32_t* __restrict__ cs = S.col[s] + sh;
    const float* __restrict__ vs = S.val[s] + sh;
    // products p_j = val_j * x[col_j] (fp32, rounded once); window hits from smem
    int j = tid;
    for (; j + 3 * PT_THREADS < cnt; j += 4 * PT_THREADS) {
      int c[4];
      float xv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) c[u] = cs[j + u * PT_THREADS];
#pragma unroll
      for (int u = 0; u < 4; ++u)
        xv[u] = (uint32_t)(c[u] - vlo) < span ? win[c[u] & (XWIN - 1)] : __ldg(x + c[u]);
      const int pj = pidx(j);  // pidx(j + 512u) = pidx(j) + 544u
#pragma unroll
      for (int u = 0; u < 4; ++u) pr[pj + 544 * u] = __fmul_rn(vs[j + u * PT_THREADS], xv[u]);
    }
    for (; j < cnt; j += PT_THREADS) {
      const int c = cs[j];
      const float xv = (uint32_t)(c - vlo) < span ? win[c & (XWIN - 1)] : __ldg(x + c);
      pr[pidx(j)] = __fmul_rn(vs[j], xv);
    }
    __syncthreads();
    // advance the window to tile t+1 (tile t no longer reads it)
    if (use_win && has_next) {
#pragma unroll
      for (int u = 0; u < SEGW; ++u) {
        const int c = seg_lo + tid + PT_THREADS * u;
        if (c < whi_next) win[c & (XWIN - 1)] = segv[u];
      }
      for (int c = seg_lo + PT_THREADS * SEGW + tid; c < whi_next; c += PT_THREADS)
        win[c & (XWIN - 1)] = __ldg(x + c);
    }
    whi = whi_next;
    float* res = reinterpret_cast<float*>(S.col[s]);  // col of this stage is dead now
    // short rows: thread per row, sequential (canonical W = 1)
    auto row_pass = [&](int q, OT p0, OT p1) {
      const int b = (int)((int64_t)p0 - v.e0);
      const int L = (int)(p1 - p0);
      if (L <= SHORT_MAX) {
        float acc = 0.f;
        int jj = b;
        const float* P = pr + pidx(b);
        for (int w = 0; w < L; ++w) {
          acc = __fadd_rn(acc, *P);
          ++jj;
          P += 1 + ((jj & 15) == 0);
        }
        res[q] = acc;
      } else if (L <= WARP_MAX) {  // longer rows belong to k_cta_rows / k_hub_chunk
        S.mid[atomicAdd(&S.mid_n, 1)] = q;
      }
    };
#pragma unroll
    for (int u = 0; u < RPF; ++u) {
      const int q = tid + u * PT_THREADS;
      if (q < nr) row_pass(q, rb[u], re[u]);
    }
    for (int q = tid + RPF * PT_THREADS; q < nr; q += PT_THREADS)
      row_pass(q, rp[v.r0 + q], rp[v.r0 + q + 1]);
    __syncthreads();
    // medium rows: warp per row (canonical W = 32)
    const int nmid = S.mid_n;
    for (int m = warp; m < nmid; m += PT_THREADS / 32) {
      const int q = S.mid[m];
      const int64_t p0 = (int64_t)rp[v.r0 + q];
      const int b = (int)(p0 - v.e0);
      const int L = (int)((int64_t)rp[v.r0 + q + 1] - p0);
      float acc = 0.f;
      for (int u = lane; u < L; u += 32) acc = __fadd_rn(acc, pr[pidx(b + u)]);
      acc = warp_tree(acc);
      if (lane == 0) res[q] = acc;
    }
    __syncthreads();
    auto emit = [&](int q, OT p0, OT p1) {
      if ((int64_t)(p1 - p0) > WARP_MAX) return;  // written by k_cta_rows / k_hub_fix
      const float o = __fmul_rn(res[q], alpha);
      y[v.r0 + q] = o;
    };
#pragma unroll
    for (int u = 0; u < RPF; ++u) {
      const int q = tid + u * PT_THREADS;
      if (q < nr) emit(q, rb[u], re[u]);
    }
    for (int q = tid + RPF * PT_THREADS; q < nr; q += PT_THREADS)
      emit(q, rp[v.r0 + q], rp[v.r0 + q + 1]);
    __syncthreads();
    v = vn;
    if (t + 2 < k1) vn = view(desc[t + 2]);
    s ^= 1;
    if (s == 0) ph ^= 1u;
  }
}

// ------------------------------------------------------------- long rows
// Strided partial sum of the entries t0, t0 + S, t0 + 2S, ... < L of a row
// (S = 32: a lane of the warp-per-row sum; S = 256: a thread of the CTA sum),
// UNR entries in flight.  PIPE: software-pipelined, the col / val of the next
// UNR entries are loaded before the x gathers of the current ones are
// consumed, so an iteration costs one memory round trip (the gathers), not
// two -- what a latency-bound launch needs (k_small: RMAT-16 16.3 -> 14.2 us,
// r68/r69) and what the one-CTA-per-row / per-chunk kernels gain from (r76,
// Kronecker-28 serialised: k_cta_rows 2.79 -> 2.71 ms, k_hub_chunk 3.11 ->
// 3.05 ms); the warp rows keep the plain loop (r69: pipelined, 4 % slower).
// The ragged end is guarded: a slot past the row has v = x = 0 and adds +0,
// which leaves s unchanged (s starts at +0 and is never -0), so the
// association is exactly t0, t0 + S, t0 + 2S, ... for every UNR and PIPE.
template <int SM, int S, int UNR, bool PIPE>
__device__ __forceinline__ float strided_sum(const int32_t* __restrict__ cc,
                                             const float* __restrict__ vv,
                                             const float* __restrict__ x, int64_t t0, int64_t L,
                                             uint64_t pol) {
  float s = 0.f;
  if constexpr (!PIPE) {  // stream, then gather, per iteration (same association)
    for (int64_t t = t0; t < L; t += S * UNR) {
      int c[UNR];
      float v[UNR], xv[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) {
        const bool pu = t + S * u < L;
        c[u] = pu ? lds<SM>(cc + t + S * u, pol) : 0;
        v[u] = pu ? lds<SM>(vv + t + S * u, pol) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < UNR; ++u) xv[u] = (t + S * u < L) ? gx(x, c[u]) : 0.f;
#pragma unroll
      for (int u = 0; u < UNR; ++u) s = __fadd_rn(s, __fmul_rn(v[u], xv[u]));
    }
  } else {
    int c[UNR];
    float v[UNR];
#pragma unroll
    for (int u = 0; u < UNR; ++u) {
      const bool pu = t0 + S * u < L;
      c[u] = pu ? lds<SM>(cc + t0 + S * u, pol) : 0;
      v[u] = pu ? lds<SM>(vv + t0 + S * u, pol) : 0.f;
    }
    for (int64_t t = t0; t < L; t += S * UNR) {
      float xv[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) xv[u] = (t + S * u < L) ? gx(x, c[u]) : 0.f;
      const int64_t tn = t + S * UNR;
      int cn[UNR];
      float vn[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) {
        const bool pu = tn + S * u < L;
        cn[u] = pu ? lds<SM>(cc + tn + S * u, pol) : 0;
        vn[u] = pu ? lds<SM>(vv + tn + S * u, pol) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < UNR; ++u) s = __fadd_rn(s, __fmul_rn(v[u], xv[u]));
#pragma unroll
      for (int u = 0; u < UNR; ++u) {
        c[u] = cn[u];
        v[u] = vn[u];
      }
    }
  }
  return s;
}

// canonical W = 32 sum of row r (32 strided partials + xor tree), valid in
// every lane
template <int SM, int UNR = 4, bool PIPE = false>
__device__ __forceinline__ float warp_row_sum_bl(const int32_t* __restrict__ col,
                                                 const float* __restrict__ val,
                                                 const float* __restrict__ x, int64_t b, int L,
                                                 int lane, uint64_t pol) {
  return warp_tree(strided_sum<SM, 32, UNR, PIPE>(col + b, val + b, x, lane, L, pol));
}

template <typename OT, int SM, int UNR = 4, bool PIPE = false>
__device__ __forceinline__ float warp_row_sum(const OT* __restrict__ rp,
                                              const int32_t* __restrict__ col,
                                              const float* __restrict__ val,
                                              const float* __restrict__ x, int r, int lane,
                                              uint64_t pol) {
  const int64_t b = (int64_t)rp[r];
  return warp_row_sum_bl<SM, UNR, PIPE>(col, val, x, b, (int)((int64_t)rp[r + 1] - b), lane, pol);
}

// (holding it to 32 registers for 8 CTAs per SM cost 4 % on Kronecker-28, r69)
template <typename OT, bool SS, int SM, int UNR = 4>
__global__ void __launch_bounds__(256)
    k_warp_rows(const OT* __restrict__ rp, const int32_t* __restrict__ col,
                const float* __restrict__ val, const float* __restrict__ x,
                float* __restrict__ y, const int32_t* __restrict__ rows, int64_t nrows,
                const double* __restrict__ ss_in, const YDst dst) {
  const int lane = threadIdx.x & 31;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float alpha = alpha_of(ss_in);
  const uint64_t pol = stream_policy<SM>();
  for (int64_t q = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; q < nrows; q += W) {
    const int r = rows[q];
    const float s = warp_row_sum<OT, SM, UNR>(rp, col, val, x, r, lane, pol);
    if (lane == 0) {
      const float v = __fmul_rn(s, alpha);
      store_y<SS>(y, dst, r, v);
    }
  }
  fence_bcast<SS>(dst);
}

// canonical W = 256 sum of entries [b, b + L) of a row
template <int SM, int UNR = 4, bool PIPE = false>
__device__ __forceinline__ float cta_sum256(const int32_t* __restrict__ col,
                                            const float* __restrict__ val,
                                            const float* __restrict__ x, int64_t b, int64_t L,
                                            float* red) {
  const int tid = threadIdx.x;
  const uint64_t pol = stream_policy<SM>();
  const float s = strided_sum<SM, 256, UNR, PIPE>(col + b, val + b, x, tid, L, pol);
  red[tid] = s;
  __syncthreads();
#pragma unroll
  for (int o = 128; o >= 32; o >>= 1) {
    if (tid < o) red[tid] = __fadd_rn(red[tid], red[tid + o]);
    __syncthreads();
  }
  float r = 0.f;
  if (tid < 32) r = warp_tree(red[tid]);
  return r;  // valid in thread 0
}

template <typename OT, bool SS, int SM, int UNR = 4>
__global__ void __launch_bounds__(256)
    k_cta_rows(const OT* __restrict__ rp, const int32_t* __restrict__ col,
               const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
               const int32_t* __restrict__ rows, const double* __restrict__ ss_in,
               const YDst dst) {
  __shared__ float red[256];
  const int r = rows[blockIdx.x];
  const int64_t b = (int64_t)rp[r], L = (int64_t)rp[r + 1] - b;
  const float s = cta_sum256<SM, UNR, true>(col, val, x, b, L, red);
  if (threadIdx.x == 0) {
    const float v = __fmul_rn(s, alpha_of(ss_in));
    store_y<SS>(y, dst, r, v);
    fence_bcast<SS>(dst);
  }
}

template <typename OT, int SM, int UNR = 4>
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
  const float s = cta_sum256<SM, UNR, true>(col, val, x, b, m, red);
  if (threadIdx.x == 0) part[c] = (double)s;
}

template <bool SS>
__global__ void k_hub_fix(const int32_t* __restrict__ hub_rows, const int32_t* __restrict__ choff,
                          int64_t nh, const double* __restrict__ part,
                          const double* __restrict__ ss_in, float* __restrict__ y,
                          const YDst dst) {
  const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (h >= nh) return;
  double acc = 0.0;
  for (int c = choff[h]; c < choff[h + 1]; ++c) acc += part[c];
  const float v = __fmul_rn((float)acc, alpha_of(ss_in));
  store_y<SS>(y, dst, hub_rows[h], v);
  fence_bcast<SS>(dst);
}

__device__ __forceinline__ double block_sum_1024(double acc, double* wss) {
  acc = warp_sum_d(acc);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane == 0) wss[w] = acc;
  __syncthreads();
  double s = 0.0;
  if (threadIdx.x == 0)
    for (int i = 0; i < 32; ++i) s += wss[i];
  return s;  // valid in thread 0
}

__global__ void __launch_bounds__(1024)
    k_ss_final(const double* __restrict__ part, int64_t np, double* __restrict__ out) {
  __shared__ double wss[32];
  double acc = 0.0;
  for (int64_t i = threadIdx.x; i < np; i += 1024) acc += part[i];
  const double s = block_sum_1024(acc, wss);
  if (threadIdx.x == 0) *out = s;
}

// Power-iteration norm (reading c22): sum of y^2 in fp64 over this rank's y
// slice in fixed segments of SS_ROWS rows (one CTA each: strided per thread,
// then a fixed tree), then the segment sums in order -- the association
// depends only on the row count, never on the grid or the row classes, so
// the norm is bitwise repeatable.  One coalesced read of y (4 B per row)
// replaces round 1's fp64 partial per row / warp stored by the SpMV kernels,
// whose scattered 8-byte stores cost the step ~0.7 ms on Kronecker-28 (r72).
constexpr int64_t SS_ROWS = 16384;

__global__ void __launch_bounds__(1024)
    k_ss_y(const float* __restrict__ y, int64_t n, double* __restrict__ part) {
  __shared__ double wss[32];
  const int64_t v0 = (int64_t)blockIdx.x * SS_ROWS, v1 = min(n, v0 + SS_ROWS);
  double acc = 0.0;
  for (int64_t v = v0 + threadIdx.x; v < v1; v += 1024) {
    const double t = (double)y[v];
    acc += t * t;
  }
  const double sblk = block_sum_1024(acc, wss);
  if (threadIdx.x == 0) part[blockIdx.x] = sblk;
}

void ss_reduce_y(spmv_plan_s* p, const float* y, double* out, cudaStream_t s) {
  const int64_t np = std::max<int64_t>(1, (p->nrows + SS_ROWS - 1) / SS_ROWS);
  k_ss_y<<<(unsigned)np, 1024, 0, s>>>(y, p->nrows, p->d_ss_part);
  k_ss_final<<<1, 1024, 0, s>>>(p->d_ss_part, np, out);
}

int g_num_sms = 0;

int num_sms(int dev) {
  if (!g_num_sms) cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
  return g_num_sms > 0 ? g_num_sms : 148;
}

// cudaFuncSetAttribute acts on the current device, so the max-dynamic-smem
// opt-in is remembered per (kernel instantiation, device), thread-safely
template <auto K>
void max_dyn_smem(int bytes, int device) {
  static std::atomic<uint64_t> done{0};
  const uint64_t bit = 1ull << (device & 63);
  if (done.load(std::memory_order_acquire) & bit) return;
  SPMV_CUDA(cudaFuncSetAttribute(K, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
  done.fetch_or(bit, std::memory_order_release);
}

template <typename OT, bool SS>
void launch_panel(spmv_plan_s* p, const float* x, float* y, const double* ss_in, cudaStream_t s) {
  constexpr size_t smem = sizeof(PanelSmem);
  max_dyn_smem<k_panel<OT, SS>>((int)smem, p->device);
  static int per_sm = 0;
  if (!per_sm) {
    SPMV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_panel<OT, SS>, PT_THREADS,
                                                            smem));
    if (per_sm < 1) per_sm = 1;
  }
  const int64_t cap = (int64_t)num_sms(p->device) * per_sm;
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min(p->K, cap));
  const int use_win = p->opts.smem_window ? 1 : 0;
  k_panel<OT, SS><<<grid, PT_THREADS, smem, s>>>((const OT*)p->d_rp, p->d_col, p->d_val, x, y,
                                                 p->d_desc, p->K, p->y_offset, p->x_len, use_win,
                                                 ss_in, p->opts.evict_first);
}

// --------------------------------------------------------- lane-per-row
// k_lane (variant 0, default): lane per row for rows with L <= 32, canonical
// W = 1 (sequential), grid-stride over 256-row blocks (CTA i takes blocks i,
// i + G, ...).  A lane streams its row in 8-entry, 32-byte-aligned chunks with
// sm_100 256-bit loads (LDG.E.NA.256: one full sector per lane, not allocated
// in L1), and gathers x with L1-allocating loads: community order
// puts a block's columns on few lines, which L1 and L2 keep on chip.  Rows
// with L > 32 are skipped here and load-balanced over their own kernels
// (k_warp_rows over the plan's mid list, k_cta_rows, k_hub_*).
// Design note (profiles/r01_summary.md, r26): a persistent variant with a
// sliding shared-memory x window, one barrier per block and evict_first
// stream hints ran 1.25x slower than this plain form on SBM 4M/64M.
constexpr int LN_THREADS = 256;
constexpr int MID_STREAM_DEFAULT = 0;  // stream-load mode of the MID / CTA / hub kernels (lds)
constexpr int LN_CTAS_PER_SM = 32;  // grid = min(blocks, SMs x this)

// 256-bit streaming loads of one 8-entry chunk, not allocated in L1.
// ef != 0 adds the L2::evict_first qualifier.  A chunk shared with a
// neighbouring row (the first / last chunk of a row) is read twice, by two
// lanes at different times; evicting it first would make the second read a
// DRAM refetch (measured: 2.3x DRAM traffic on the 27-point stencil), so
// EF mode 2 loads a row's FIRST chunk normally and the rest evict_first: a
// chunk shared by rows r and r + 1 is read first by lane r + 1 (as its first
// chunk, kept) and last by lane r (its last chunk, then marked evict_first).
template <int EF>
__device__ __forceinline__ void ld_v8_stream(const int32_t* p, int (&r)[8]) {
  if constexpr (EF == 1)
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
__device__ __forceinline__ void ld_v8_stream(const float* p, float (&r)[8]) {
  if constexpr (EF == 1)
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

// sequential (canonical W = 1) sum of a row of L <= SHORT_MAX entries
// starting at a, streamed in 8-entry, 32-byte-aligned chunks.  Every slot of
// a chunk holds a valid column of some row (or the zero tail padding), so its
// x read is always safe; a slot outside [a, a + L) has its x replaced by 0, so
// it contributes v * 0 = +-0 and leaves the sum unchanged (it starts at +0 and
// is never -0) -- exact for a finite neighbouring value v.  When the plan
// holds a non-finite value (EF & 4, detected at permute time) the value is
// masked as well (0 * 0 = +0), so an Inf / NaN never leaks into a neighbouring
// row (Alg. 1).  The value mask costs 9 % on C2 whichever way it is written
// (r62/r63: 0.0964 vs 0.0883 ms), hence the two variants.  EF & 8 (plan
// decision, lane_pred): the x of a foreign slot is not gathered at all -- the
// same sum, fewer L1 wavefronts where rows straddle chunks (stencil).
template <typename OT, int EF>
__device__ __forceinline__ float lane_row_sum(const int32_t* __restrict__ col,
                                              const float* __restrict__ val,
                                              const float* __restrict__ x, OT a, int L) {
  float res = 0.f;
  const int32_t* cp = col + (a & ~(OT)7);
  const float* vp = val + (a & ~(OT)7);
  const int lo = (int)(a & 7), hi = lo + L;
#pragma unroll 2
  for (int k = 0; k < hi; k += 8) {
    int cc[8];
    float vv[8];
    if ((EF & 3) == 2 && k == 0) {  // (warp-uniform: every lane starts at k = 0)
      ld_v8_stream<0>(cp + k, cc);
      ld_v8_stream<0>(vp + k, vv);
    } else {
      ld_v8_stream<(EF & 3) == 0 ? 0 : 1>(cp + k, cc);
      ld_v8_stream<(EF & 3) == 0 ? 0 : 1>(vp + k, vv);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const bool in = k + i >= lo && k + i < hi;
      float xv;
      if constexpr ((EF & 8) != 0)  // plan decision: no gather for a foreign slot
        xv = in ? gx(x, cc[i]) : 0.f;
      else  // branch-free: every slot gathered (valid column), foreign ones zeroed
        xv = gx(x, cc[i]);
      if constexpr ((EF & 4) != 0)  // the plan holds a non-finite value: 0 * 0 = +0
        res = __fadd_rn(res, __fmul_rn(in ? vv[i] : 0.f, in ? xv : 0.f));
      else  // finite values: v * 0 = +-0 exactly (the faster schedule, r62)
        res = __fadd_rn(res, __fmul_rn(vv[i], in ? xv : 0.f));
    }
  }
  return res;
}


// minBlocksPerSM = 1 lets ptxas keep both chunks and all 16 gathers of a
// 16-entry row in flight per lane (64 registers, 4 CTAs/SM); capping registers
// for more CTAs measured 20-40 % slower
// SS (the power-iteration step) needs 72 registers unbounded, which drops to
// 3 CTAs per SM and costs 22 % (r66: 4.45 vs 3.64 ms on C5): both variants
// are held to 64 registers, 4 CTAs per SM
template <typename OT, bool SS, int EF>
__global__ void __launch_bounds__(LN_THREADS, SS ? 4 : 1)
    k_lane(const OT* __restrict__ rp, const int32_t* __restrict__ col,
           const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
           int64_t nrows, const double* __restrict__ ss_in,
           const YDst dst) {
  const int tid = threadIdx.x;
  const int64_t NB = (nrows + LN_THREADS - 1) / LN_THREADS;
  const float alpha = alpha_of(ss_in);
  // row pointers are loaded one block iteration ahead
  OT a_n = 0, e_n = 0;
  {
    const int64_t r = (int64_t)blockIdx.x * LN_THREADS + tid;
    if (r < nrows) {
      a_n = rp[r];
      e_n = rp[r + 1];
    }
  }
  for (int64_t blk = blockIdx.x; blk < NB; blk += gridDim.x) {
    const int64_t r = blk * LN_THREADS + tid;
    const OT a = a_n, e = e_n;
    {
      const int64_t rn = r + (int64_t)gridDim.x * LN_THREADS;
      if (rn < nrows) {
        a_n = rp[rn];
        e_n = rp[rn + 1];
      }
    }
    float res = 0.f;
    bool mine = false;
    if (r < nrows) {
      const int L = (int)(e - a);
      if (L <= SHORT_MAX) {  // longer rows: k_warp_rows / k_cta_rows / k_hub_*
        mine = true;
        // Every slot of a chunk holds a valid column of some row (or the zero
        // tail padding), so its x read is always safe; a slot outside [a, e)
        // contributes the product +0 (selected, not computed: a neighbouring
        // row's Inf / NaN value never reaches this row, Alg. 1), which leaves
        // res unchanged (it starts at +0 and is never -0).
        res = lane_row_sum<OT, EF>(col, val, x, a, L);
      }
    }
    if (mine) store_y<SS>(y, dst, r, __fmul_rn(res, alpha));
  }
  fence_bcast<SS>(dst);
}

// Small plans (no hub rows, few entries): every row class in ONE launch, no
// fork / join -- CTA i < B_lane computes the 256-row lane block i, the next
// B_mid CTAs eight MID rows each (warp per row, rows with L <= MID_WIDE), the
// next n_wide CTAs one wide MID row each (L > MID_WIDE), the last n_cta CTAs
// one CTA row each.  Same per-row association as the separate kernels
// (bitwise equal y); launch and dependent-load latency dominate such plans
// (RMAT-16: 8 MB), so the long rows' loads are all put in flight at once: a
// wide MID row's 256 threads each form up to eight products p_e = v_e * x_e
// (fp32, rounded once, as the warp sum does) into shared memory, then lane j
// of warp 0 adds p_j, p_{j+32}, ... in that order -- exactly the W = 32
// strided association of warp_row_sum -- and the xor tree.
template <typename OT, bool SS, int EF, int SM>
__global__ void __launch_bounds__(LN_THREADS)
    k_small(const OT* __restrict__ rp, const int32_t* __restrict__ col,
            const float* __restrict__ val, const float* __restrict__ x, float* __restrict__ y,
            int64_t nrows, const int32_t* __restrict__ mid_rows, int64_t n_mid,
            const int32_t* __restrict__ mid_wide, int64_t n_wide,
            const int32_t* __restrict__ cta_rows, int64_t B_lane, int64_t B_mid,
            const double* __restrict__ ss_in, const YDst dst) {
  __shared__ float red[256];
  __shared__ float prod[WARP_MAX];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const float alpha = alpha_of(ss_in);
  // the long rows (wide MID, CTA rows) are dispatched first: blocks
  // [0, n_long) take roles B_lane + B_mid + ..., so the critical path starts
  // in the first wave instead of after the lane and MID blocks
  const int64_t tail0 = B_lane + B_mid, n_long = (int64_t)gridDim.x - tail0;
  const int64_t blk = (int64_t)blockIdx.x < n_long ? tail0 + blockIdx.x : blockIdx.x - n_long;
  const uint64_t pol = stream_policy<SM>();
  if (blk < B_lane) {  // block-uniform branches
    const int64_t r = blk * LN_THREADS + tid;
    if (r < nrows) {
      const OT a = rp[r];
      const int L = (int)(rp[r + 1] - a);
      if (L <= SHORT_MAX)
        store_y<SS>(y, dst, r, __fmul_rn(lane_row_sum<OT, EF>(col, val, x, a, L), alpha));
    }
  } else if (blk < B_lane + B_mid) {
    const int64_t q = (blk - B_lane) * 8 + warp;
    if (q < n_mid) {
      const int r = mid_rows[q];
      const int64_t b = (int64_t)rp[r];
      const int L = (int)((int64_t)rp[r + 1] - b);
      if (L <= MID_WIDE) {  // (wide rows: their own CTA below)
        const float s = warp_row_sum_bl<SM, 8, true>(col, val, x, b, L, lane, pol);
        if (lane == 0) store_y<SS>(y, dst, r, __fmul_rn(s, alpha));
      }
    }
  } else if (blk < B_lane + B_mid + n_wide) {
    const int64_t q = mid_wide[blk - B_lane - B_mid];
    const int r = mid_rows[q];
    const int64_t b = (int64_t)rp[r];
    const int L = (int)((int64_t)rp[r + 1] - b);  // MID_WIDE < L <= WARP_MAX
    constexpr int PER = WARP_MAX / LN_THREADS;       // 8 entries per thread
    int c[PER];
    float v[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int e = tid + LN_THREADS * k;
      c[k] = e < L ? lds<SM>(col + b + e, pol) : 0;
      v[k] = e < L ? lds<SM>(val + b + e, pol) : 0.f;
    }
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int e = tid + LN_THREADS * k;
      if (e < L) prod[e] = __fmul_rn(v[k], gx(x, c[k]));
    }
    __syncthreads();
    if (warp == 0) {
      float s = 0.f;
      for (int j0 = lane; j0 < L; j0 += 32 * 8) {  // 8 products read ahead, added in order
        float pv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) pv[u] = j0 + 32 * u < L ? prod[j0 + 32 * u] : 0.f;
#pragma unroll
        for (int u = 0; u < 8; ++u) s = __fadd_rn(s, pv[u]);
      }
      s = warp_tree(s);
      if (lane == 0) store_y<SS>(y, dst, r, __fmul_rn(s, alpha));
    }
  } else {
    const int64_t i = blk - B_lane - B_mid - n_wide;
    const int r = cta_rows[i];
    const int64_t b = (int64_t)rp[r], L = (int64_t)rp[r + 1] - b;
    const float s = cta_sum256<SM, 8, true>(col, val, x, b, L, red);
    if (tid == 0) store_y<SS>(y, dst, r, __fmul_rn(s, alpha));
  }
  fence_bcast<SS>(dst);
}

template <typename OT, bool SS, int EF>
void launch_lane_t(spmv_plan_s* p, const float* x, float* y, const double* ss_in, cudaStream_t s,
                   const YDst& dst) {
  // grid-stride with ~8 CTAs per resident slot (measured better than one
  // persistent wave on SBM, RMAT-26 and the stencil: r29, profiles/)
  int per_sm = LN_CTAS_PER_SM;
  if (const char* e = getenv("SPMV_LANE_CTAS")) per_sm = std::max(1, atoi(e));  // dev knob
  const int64_t NB = (p->nrows + LN_THREADS - 1) / LN_THREADS;
  const int64_t cap = (int64_t)num_sms(p->device) * per_sm;
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min(NB, cap));
  k_lane<OT, SS, EF><<<grid, LN_THREADS, 0, s>>>((const OT*)p->d_rp, p->d_col, p->d_val, x, y,
                                                   p->nrows, ss_in, dst);
}

}  // namespace

int lane_ef_mode(const spmv_plan_s* p) {
  return p->opts.evict_first && p->stream_ef ? 1 : 0;
}

int lane_pred_mode(const spmv_plan_s* p) {
  if (const char* e = getenv("SPMV_LANE_PRED")) return atoi(e) != 0;  // dev knob (A/B)
  return p->lane_pred ? 1 : 0;
}

namespace {

template <typename OT, bool SS>
void launch_lane(spmv_plan_s* p, const float* x, float* y, const double* ss_in, cudaStream_t s,
                 const YDst& dst) {
  // stream policy (plan decision): evict_first on every chunk when no 8-entry
  // chunk is shared by two rows (1), else none (0); 2 (first chunk of a row
  // normal, the rest evict_first) via the SPMV_LANE_EF dev knob
  int ef = lane_ef_mode(p);
  if (const char* e = getenv("SPMV_LANE_EF")) ef = std::min(2, std::max(0, atoi(e)));  // dev knob
  const int m = (p->val_nonfinite ? 4 : 0) | (lane_pred_mode(p) ? 8 : 0);
#define SPMV_LANE_M(M)                                                        \
  do {                                                                        \
    if (ef == 1) launch_lane_t<OT, SS, 1 | (M)>(p, x, y, ss_in, s, dst);      \
    else if (ef == 2) launch_lane_t<OT, SS, 2 | (M)>(p, x, y, ss_in, s, dst); \
    else launch_lane_t<OT, SS, 0 | (M)>(p, x, y, ss_in, s, dst);              \
  } while (0)
  if (m == 12) SPMV_LANE_M(12);
  else if (m == 8) SPMV_LANE_M(8);
  else if (m == 4) SPMV_LANE_M(4);
  else SPMV_LANE_M(0);
#undef SPMV_LANE_M
}

// Row-class kernels other than the short-row one: MID rows (warp per row),
// CTA rows, hub chunks + fixup, on the two plan-owned streams s1 / s2.
template <typename OT, bool SS, int SM>
void launch_rows_t(spmv_plan_s* p, const float* x, float* y, const double* ss_in, cudaStream_t s1,
                   cudaStream_t s2, bool lane_mode, const YDst& dst) {
  const OT* rp = (const OT*)p->d_rp;
  const int32_t* col = p->d_col;
  const int64_t nw = lane_mode ? p->n_mid : p->n_warp;
  const int32_t* wr = lane_mode ? p->d_mid_rows : p->d_warp_rows;
  if (nw) {
    const unsigned g = (unsigned)std::min<int64_t>((nw + 7) / 8, (int64_t)num_sms(p->device) * 16);
    k_warp_rows<OT, SS, SM><<<g, 256, 0, s1>>>(rp, col, p->d_val, x, y, wr, nw, ss_in, dst);
  }
  if (p->n_cta)
    k_cta_rows<OT, SS, SM><<<(unsigned)p->n_cta, 256, 0, s2>>>(rp, col, p->d_val, x, y,
                                                              p->d_cta_rows, ss_in, dst);
  if (p->n_chunks) {
    k_hub_chunk<OT, SM><<<(unsigned)p->n_chunks, 256, 0, s2>>>(
        rp, col, p->d_val, x, p->d_chunk_row, p->d_chunk_idx, p->d_chunk_part);
    const unsigned g = (unsigned)((p->n_hub + 127) / 128);
    k_hub_fix<SS><<<g, 128, 0, s2>>>(p->d_hub_rows, p->d_hub_choff, p->n_hub, p->d_chunk_part,
                                      ss_in, y, dst);
  }
}

template <typename OT, bool SS>
void launch_rows(spmv_plan_s* p, const float* x, float* y, const double* ss_in, cudaStream_t s1,
                 cudaStream_t s2, bool lane_mode, const YDst& dst) {
  int sm = MID_STREAM_DEFAULT;
  if (const char* e = getenv("SPMV_MID_STREAM")) sm = std::min(2, std::max(0, atoi(e)));  // dev knob
  if (sm == 1) launch_rows_t<OT, SS, 1>(p, x, y, ss_in, s1, s2, lane_mode, dst);
  else if (sm == 2) launch_rows_t<OT, SS, 2>(p, x, y, ss_in, s1, s2, lane_mode, dst);
  else launch_rows_t<OT, SS, 0>(p, x, y, ss_in, s1, s2, lane_mode, dst);
}

// plans run by k_small: lane variant, no hub rows (their fp64 fixup is a
// second kernel), MID or CTA rows present (else k_lane is one launch anyway),
// at most SMALL_NNZ entries (launch / fork-join bound); SPMV_SMALL=0/1 dev knob
constexpr int64_t SMALL_NNZ = int64_t(1) << 24;
bool small_plan(const spmv_plan_s* p) {
  if (p->n_chunks || !(p->n_mid || p->n_cta)) return false;
  if (const char* e = getenv("SPMV_SMALL")) return atoi(e) != 0;
  return p->nnz_local <= SMALL_NNZ;
}

template <typename OT>
void exec_typed(spmv_plan_s* p, const float* x, float* y, const double* ss_in, double* ss_out,
                cudaStream_t s, const YDst& dst) {
  const bool SS = ss_out != nullptr;
  const bool lane_mode = p->opts.variant != 1;
  const int64_t nw = lane_mode ? p->n_mid : p->n_warp;
  // The row classes write disjoint rows of y and only read x: the warp-row
  // kernel and the CTA/hub kernels run on two plan-owned streams concurrently
  // with the short-row kernel (fork/join by events; CUDA-graph capturable).
  // The fork is recorded before (early, default) or after the short-row
  // launch (SPMV_FORK_EARLY=0: the other classes start when it has finished).
  if (lane_mode && small_plan(p)) {  // one launch for every row class
    const int64_t B_lane = (p->nrows + LN_THREADS - 1) / LN_THREADS, B_mid = (p->n_mid + 7) / 8;
    const unsigned g = (unsigned)(B_lane + B_mid + p->n_mid_wide + p->n_cta);
    const OT* rp = (const OT*)p->d_rp;
    constexpr int SM = MID_STREAM_DEFAULT;
#define SPMV_SMALL_ARGS                                                                      \
  rp, p->d_col, p->d_val, x, y, p->nrows, p->d_mid_rows, p->n_mid, p->d_mid_wide, p->n_mid_wide,  \
      p->d_cta_rows, B_lane, B_mid,                                                                \
      ss_in, dst
    const int ef = (lane_ef_mode(p) == 1 ? 1 : 0) | (p->val_nonfinite ? 4 : 0) |
                   (lane_pred_mode(p) ? 8 : 0);
#define SPMV_SMALL_EF(SSV)                                                                 \
  do {                                                                                     \
    switch (ef) {                                                                          \
      case 1: k_small<OT, SSV, 1, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break;   \
      case 4: k_small<OT, SSV, 4, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break;   \
      case 5: k_small<OT, SSV, 5, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break;   \
      case 8: k_small<OT, SSV, 8, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break;   \
      case 9: k_small<OT, SSV, 9, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break;   \
      case 12: k_small<OT, SSV, 12, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break; \
      case 13: k_small<OT, SSV, 13, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS); break; \
      default: k_small<OT, SSV, 0, SM><<<g, LN_THREADS, 0, s>>>(SPMV_SMALL_ARGS);         \
    }                                                                                      \
  } while (0)
    if (SS) {
      SPMV_SMALL_EF(true);
      ss_reduce_y(p, dst.n ? dst.p[p->rank] : y, ss_out, s);
    } else {
      SPMV_SMALL_EF(false);
    }
#undef SPMV_SMALL_EF
#undef SPMV_SMALL_ARGS
    SPMV_LAUNCH_CHECK();
    return;
  }
  cudaStream_t s1 = s, s2 = s;
  const bool conc = p->conc && (nw > 0 || p->n_cta > 0 || p->n_chunks > 0);
  bool early = true;
  if (const char* e = getenv("SPMV_FORK_EARLY")) early = atoi(e) != 0;  // dev knob
  auto fork = [&]() {
    SPMV_CUDA(cudaEventRecord(p->ev_fork, s));
    s1 = p->aux[0];
    s2 = p->aux[1];
    SPMV_CUDA(cudaStreamWaitEvent(s1, p->ev_fork, 0));
    SPMV_CUDA(cudaStreamWaitEvent(s2, p->ev_fork, 0));
  };
  if (conc && early) fork();
  if (lane_mode) {
    if (p->nrows) {
      if (SS) launch_lane<OT, true>(p, x, y, ss_in, s, dst);
      else launch_lane<OT, false>(p, x, y, ss_in, s, dst);
    }
  } else if (p->K) {
    if (SS) launch_panel<OT, true>(p, x, y, ss_in, s);
    else launch_panel<OT, false>(p, x, y, ss_in, s);
  }
  if (conc && !early) fork();
  {
    if (SS) launch_rows<OT, true>(p, x, y, ss_in, s1, s2, lane_mode, dst);
    else launch_rows<OT, false>(p, x, y, ss_in, s1, s2, lane_mode, dst);
  }
  if (conc) {
    SPMV_CUDA(cudaEventRecord(p->ev_join[0], s1));
    SPMV_CUDA(cudaEventRecord(p->ev_join[1], s2));
    SPMV_CUDA(cudaStreamWaitEvent(s, p->ev_join[0], 0));
    SPMV_CUDA(cudaStreamWaitEvent(s, p->ev_join[1], 0));
  }
  if (SS) ss_reduce_y(p, dst.n ? dst.p[p->rank] : y, ss_out, s);
  SPMV_LAUNCH_CHECK();
}

// The persisting window on x_B[0:H) pays only when the prefix is HOT: its
// columns read at least WIN_HOT times as often as an average column (the hub
// group of a power-law graph under RABBIT++; not the 98.7 % "hubs" of a
// stencil, r57: 7.11 ms with the window vs 6.68 without).  Its size is capped
// at half the L2: the whole prefix pinned (83 MB on Kronecker-28) starves the
// rest of the step (r56/r57: 24.5 -> 21.0 ms).
constexpr double WIN_HOT = 2.0;
constexpr double WIN_L2_FRAC = 0.5;

void set_window_one(spmv_plan_s* p, const float* x, cudaStream_t s, int slot) {
  if (p->win_ptr == (const void*)x && p->win_stream[slot] == s) return;
  int maxwin = 0, maxpers = 0;
  cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, p->device);
  cudaDeviceGetAttribute(&maxpers, cudaDevAttrMaxPersistingL2CacheSize, p->device);
  int64_t want = p->H;
  if (const char* e = getenv("SPMV_WIN_ALL")) if (atoi(e)) want = p->x_len;  // dev knob
  if (const char* e = getenv("SPMV_WIN_COLS")) want = std::min<int64_t>(p->x_len, atoll(e));  // dev knob
  int64_t bytes = std::min<int64_t>(want * 4, (int64_t)maxwin);
  bytes = std::min<int64_t>(bytes, (int64_t)maxpers);
  double hit = p->opts.l2_hit_ratio;
  {
    double frac = WIN_L2_FRAC;
    if (const char* e = getenv("SPMV_WIN_FRAC")) frac = atof(e);  // dev knob
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, p->device);
    if (l2 > 0) bytes = std::min<int64_t>(bytes, (int64_t)(frac * l2));
  }
  // spmv_iterate reads x from two buffers in turn: both windows must fit the
  // persisting carve-out at once, or each step evicts the other's lines
  // (r74: the same step time as one full-size window, within noise)
  if (p->win_alternating) bytes = std::min<int64_t>(bytes, (int64_t)maxpers / 2);
  if (const char* e = getenv("SPMV_WIN_HIT")) hit = std::min(1.0, std::max(0.0, atof(e)));  // dev knob
  if (bytes <= 0) return;
  size_t cur = 0;
  cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
  if ((int64_t)cur < bytes) {
    if (!p->l2_limit_raised) {
      p->l2_limit_before = cur;
      p->l2_limit_raised = true;
    }
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)bytes);
  }
  cudaStreamAttrValue v{};
  v.accessPolicyWindow.base_ptr = (void*)x;
  v.accessPolicyWindow.num_bytes = (size_t)bytes;
  v.accessPolicyWindow.hitRatio = (float)hit;
  v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
  v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
  if (cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  if (p->win_ptr != (const void*)x) {
    p->win_stream[0] = p->win_stream[1] = p->win_stream[2] = nullptr;
    p->win_ptr = x;
  }
  p->win_stream[slot] = s;
  p->l2_window_bytes = bytes;
}


bool window_pays(const spmv_plan_s* p) {
  if (p->H <= 0 || p->n <= 0 || p->nnz <= 0) return false;
  if (const char* e = getenv("SPMV_WIN_FORCE")) return atoi(e) != 0;  // dev knob
  const double hot = (double)p->H_nnz / (double)p->H, avg = (double)p->nnz / (double)p->n;
  return hot >= WIN_HOT * avg;
}

void set_window(spmv_plan_s* p, const float* x, cudaStream_t s) {
  if (!p->opts.l2_window || !window_pays(p) || s == nullptr) return;
  set_window_one(p, x, s, 0);
  if (p->conc) {
    set_window_one(p, x, p->aux[0], 1);
    set_window_one(p, x, p->aux[1], 2);
  }
}

// lazily create the plan's two auxiliary streams and events (on the plan's
// device); concurrency is off if that fails or SPMV_CONCURRENT=0 (dev knob)
void ensure_aux(spmv_plan_s* p) {
  if (p->conc_init) return;
  p->conc_init = true;
  p->conc = false;
  if (const char* e = getenv("SPMV_L2_FETCH")) {  // dev knob: L2 miss fetch granularity (B)
    cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)atoi(e));
    cudaGetLastError();
  }
  if (const char* e = getenv("SPMV_CONCURRENT")) if (!atoi(e)) return;
  // the MID-row stream (aux 0, the longest kernel of a step) at the highest
  // priority, so its CTAs are dispatched ahead of the CTA / hub rows' (r86:
  // RMAT-26 4.35 vs 4.39 ms in 3 of 3 pairs, Kronecker-28 unchanged)
  int lo = 0, hi = 0;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  for (int i = 0; i < 2; ++i) {
    if (cudaStreamCreateWithPriority(&p->aux[i], cudaStreamNonBlocking, i == 0 ? hi : 0) !=
            cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_join[i], cudaEventDisableTiming) != cudaSuccess) {
      cudaGetLastError();
      return;
    }
  }
  if (cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  p->conc = true;
}

}  // namespace

void exec_streams(spmv_plan_s* p) { ensure_aux(p); }

int exec_launches(const spmv_plan_s* p, bool ss) {
  const bool lane_mode = p->opts.variant != 1;
  const int longk = (p->n_cta ? 1 : 0) + (p->n_chunks ? 2 : 0);
  if (lane_mode && small_plan(p)) return 1 + (ss ? 2 : 0);
  return (lane_mode ? (p->nrows ? 1 : 0) + (p->n_mid ? 1 : 0)
                    : (p->K ? 1 : 0) + (p->n_warp ? 1 : 0)) +
         longk + (ss ? 2 : 0);
}

void exec(spmv_plan_s* p, const float* x, float* y, const double* ss_in, double* ss_out,
          cudaStream_t s, float* const* bcast, int nbcast) {
  if (!p->permuted) SPMV_FAIL(SPMV_ESTATE, "spmv_exec before spmv_permute");
  if (ss_in && ss_in == ss_out) SPMV_FAIL(SPMV_EINVAL, "sumsq_in and sumsq_out alias");
  YDst dst{};
  if (nbcast) {
    if (nbcast < 0 || nbcast > 8) SPMV_FAIL(SPMV_EINVAL, "bcast: 1..8 destination buffers");
    if (!ss_out) SPMV_FAIL(SPMV_EINVAL, "bcast needs sumsq_out (exec_scaled)");
    if (p->opts.variant == 1)
      SPMV_FAIL(SPMV_EUNSUPPORTED, "bcast: lane-mode kernels only (variant 0)");
    for (int k = 0; k < nbcast; ++k) {
      if (!bcast[k]) SPMV_FAIL(SPMV_EINVAL, "bcast: NULL destination");
      dst.p[k] = bcast[k] + p->y_offset;
    }
    dst.n = nbcast;
    if (ss_out && p->rank >= nbcast)
      SPMV_FAIL(SPMV_EINVAL, "bcast: x_next[rank] must be this rank's own buffer (the norm reads it)");
  }
  ensure_aux(p);
  set_window(p, x, s);
  if (p->off64) exec_typed<int64_t>(p, x, y, ss_in, ss_out, s, dst);
  else exec_typed<int32_t>(p, x, y, ss_in, ss_out, s, dst);
}

}  // namespace spmv
