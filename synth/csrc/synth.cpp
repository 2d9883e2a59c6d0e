// synth: seeded, counter-based synthetic sparse-matrix generators.
//
// Input generators only: this file holds none of the method's arithmetic (no
// SpMV, no permutation of a matrix, no reordering).  It is shared by the
// oracle tests and the CUDA-path tests/bench, which is the one thing the two
// sides are allowed to share.
//
// Every random draw is a pure function of (seed, counter) through splitmix64's
// finaliser, so this C++ file and the numpy reference in synth/gen.py produce
// bit-identical matrices (tests/test_synth.py checks it).
//
//   mix64(z)      = splitmix64 finaliser
//   h1(s, a)      = mix64(s + G * (a + 1)),  G = 0x9E3779B97F4A7C15
//   h2(s, a, b)   = h1(h1(s, a), b)
//   sym(h)        = (h >> 40) * 2^-23 - 1        in [-1, 1), exact in fp32
//   pos(h)        = ((h >> 40) + 1) * 2^-24      in (0, 1],  exact in fp32
//
// Workload shapes follow SURVEY.md §8(d) (RMAT / Graph500 Kronecker, planted
// SBM, 27-point stencil), the synthetic stand-ins for the paper's corpus
// (§III).
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <omp.h>

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}
inline uint64_t h1(uint64_t s, uint64_t a) { return mix64(s + kGolden * (a + 1)); }
inline uint64_t h2(uint64_t s, uint64_t a, uint64_t b) { return h1(h1(s, a), b); }
inline float sym_f32(uint64_t h) { return (float)((double)(h >> 40) * (1.0 / 8388608.0) - 1.0); }
inline float pos_f32(uint64_t h) { return (float)((double)((h >> 40) + 1) * (1.0 / 16777216.0)); }

// Bijection on [0, 2^k): 4 rounds of (odd multiply + add) mod 2^k and a
// xor-shift; each step is invertible mod 2^k.
struct Bij {
  int k = 0;
  uint64_t mask = 0, mul[4] = {0, 0, 0, 0}, add[4] = {0, 0, 0, 0};
  int shift = 1;
  Bij(int k_, uint64_t seed) : k(k_) {
    mask = (k >= 64) ? ~0ull : ((1ull << k) - 1);
    shift = (k + 1) / 2;
    if (shift < 1) shift = 1;
    for (int r = 0; r < 4; ++r) {
      mul[r] = (h1(seed, 2 * r) | 1ull) & mask;
      add[r] = h1(seed, 2 * r + 1) & mask;
    }
  }
  inline uint64_t operator()(uint64_t v) const {
    if (k == 0) return 0;
    for (int r = 0; r < 4; ++r) {
      v = (v * mul[r] + add[r]) & mask;
      v ^= v >> shift;
    }
    return v;
  }
};

// Cycle-walking bijection on [0, n).
struct Scramble {
  int64_t n;
  Bij b;
  static int bits(int64_t n) {
    int k = 0;
    while ((1ll << k) < n) ++k;
    return k;
  }
  Scramble(int64_t n_, uint64_t seed) : n(n_), b(bits(n_), seed) {}
  inline int64_t operator()(int64_t v) const {
    uint64_t u = (uint64_t)v;
    do { u = b(u); } while ((int64_t)u >= n);
    return (int64_t)u;
  }
};

inline uint64_t thr53(double p) { return (uint64_t)(p * 9007199254740992.0); }

struct Csr {
  int64_t n = 0, nnz = 0;
  int64_t* row_ptr = nullptr;
  int32_t* col = nullptr;
  float* val = nullptr;
};

void exclusive_scan(const int64_t* in, int64_t* out, int64_t n) {
  // out[0..n], out[n] = total; simple two-level parallel scan
  int nt = omp_get_max_threads();
  std::vector<int64_t> part(nt + 1, 0);
#pragma omp parallel num_threads(nt)
  {
    int t = omp_get_thread_num(), T = omp_get_num_threads();
    int64_t lo = n * t / T, hi = n * (t + 1) / T, s = 0;
    for (int64_t i = lo; i < hi; ++i) s += in[i];
    part[t + 1] = s;
#pragma omp barrier
#pragma omp single
    for (int i = 1; i <= T; ++i) part[i] += part[i - 1];
    int64_t acc = part[t];
    for (int64_t i = lo; i < hi; ++i) { out[i] = acc; acc += in[i]; }
  }
  out[n] = n > 0 ? out[n - 1] + in[n - 1] : 0;
}

void fill_values(Csr& m, int valmode, uint64_t seed_v) {
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t i = 0; i < m.n; ++i)
    for (int64_t k = m.row_ptr[i]; k < m.row_ptr[i + 1]; ++k) {
      uint64_t h = h2(seed_v, (uint64_t)i, (uint64_t)m.col[k]);
      m.val[k] = valmode == 0 ? sym_f32(h) : valmode == 1 ? pos_f32(h) : 1.0f;
    }
}

// rows given as (row, col) pairs produced twice by a functor; builds a
// deduplicated, column-sorted CSR.
template <class Gen>
int build_from_edges(int64_t n, int64_t E, const Gen& gen, Csr& m) {
  std::vector<uint32_t> cnt(n, 0);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < E; ++e) {
    int64_t r, c;
    gen(e, r, c);
    __atomic_fetch_add(&cnt[r], 1u, __ATOMIC_RELAXED);
  }
  std::vector<int64_t> cnt64(n), off(n + 1);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) cnt64[i] = cnt[i];
  exclusive_scan(cnt64.data(), off.data(), n);
  int32_t* tmp = (int32_t*)malloc(sizeof(int32_t) * (size_t)std::max<int64_t>(E, 1));
  if (!tmp) return 1;
  std::vector<int64_t> cur(off.begin(), off.end() - 1);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < E; ++e) {
    int64_t r, c;
    gen(e, r, c);
    int64_t p = __atomic_fetch_add(&cur[r], (int64_t)1, __ATOMIC_RELAXED);
    tmp[p] = (int32_t)c;
  }
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    int32_t* b = tmp + off[i];
    int32_t* e = tmp + off[i + 1];
    std::sort(b, e);
    cnt64[i] = std::unique(b, e) - b;
  }
  m.n = n;
  m.row_ptr = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  if (!m.row_ptr) { free(tmp); return 1; }
  exclusive_scan(cnt64.data(), m.row_ptr, n);
  m.nnz = m.row_ptr[n];
  m.col = (int32_t*)malloc(sizeof(int32_t) * (size_t)std::max<int64_t>(m.nnz, 1));
  m.val = (float*)malloc(sizeof(float) * (size_t)std::max<int64_t>(m.nnz, 1));
  if (!m.col || !m.val) { free(tmp); return 1; }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t i = 0; i < n; ++i)
    memcpy(m.col + m.row_ptr[i], tmp + off[i], sizeof(int32_t) * (size_t)cnt64[i]);
  free(tmp);
  return 0;
}

}  // namespace

extern "C" {

typedef struct {
  int64_t n, nnz;
  int64_t* row_ptr;
  int32_t* col;
  float* val;
} synth_csr;

static void to_out(const Csr& m, synth_csr* out) {
  out->n = m.n;
  out->nnz = m.nnz;
  out->row_ptr = m.row_ptr;
  out->col = m.col;
  out->val = m.val;
}

uint64_t synth_h1(uint64_t s, uint64_t a) { return h1(s, a); }
uint64_t synth_h2(uint64_t s, uint64_t a, uint64_t b) { return h2(s, a, b); }

void synth_free(synth_csr* m) {
  if (!m) return;
  free(m->row_ptr);
  free(m->col);
  free(m->val);
  m->row_ptr = nullptr;
  m->col = nullptr;
  m->val = nullptr;
}

// RMAT / Graph500 Kronecker.  Edge e in [0, ef * 2^scale): level l picks a
// quadrant with u = h2(seed, e, l) >> 11 against thresholds a, a+b, a+b+c
// (most significant bit first).  scramble != 0 applies the bijection
// Scramble(2^scale, seed_scr) to both endpoints (Graph500's vertex scramble).
// Duplicates are merged, self-loops kept.  valmode: 0 sym, 1 pos, 2 ones.
int synth_rmat(int scale, int64_t edge_factor, uint64_t seed, double a, double b,
               double c, int scramble, uint64_t seed_scr, int valmode,
               uint64_t seed_v, synth_csr* out) {
  if (scale < 0 || scale > 31 || edge_factor < 0 || !out) return 1;
  const int64_t n = 1ll << scale;
  const int64_t E = edge_factor << scale;
  const uint64_t t1 = thr53(a), t2 = thr53(a + b), t3 = thr53(a + b + c);
  Scramble scr(n, seed_scr);
  auto gen = [&](int64_t e, int64_t& r, int64_t& cc) {
    uint64_t he = h1(seed, (uint64_t)e);
    uint64_t rr = 0, c2 = 0;
    for (int l = 0; l < scale; ++l) {
      uint64_t u = h1(he, (uint64_t)l) >> 11;
      uint64_t rb = u >= t2;
      uint64_t cb = (u >= t1 && u < t2) || (u >= t3);
      rr |= rb << (scale - 1 - l);
      c2 |= cb << (scale - 1 - l);
    }
    if (scramble) { rr = scr((int64_t)rr); c2 = scr((int64_t)c2); }
    r = (int64_t)rr;
    cc = (int64_t)c2;
  };
  Csr m;
  if (build_from_edges(n, E, gen, m)) return 2;
  fill_values(m, valmode, seed_v);
  to_out(m, out);
  return 0;
}

// Planted-community SBM: n_comm communities of comm_size nodes (planted ids),
// every row exactly `deg` distinct columns; candidate k of planted row p:
// hA = h2(seed, p, 2k), hB = h2(seed, p, 2k+1); in-community iff
// (hA >> 11) < p_in * 2^53, column = c*comm_size + hB % comm_size (in) or
// hB % N (out); rejected if already drawn.  Labels then scrambled by
// Scramble(N, seed_scr) (scramble != 0): row s(p) holds columns s(q).
int synth_sbm(int64_t n_comm, int64_t comm_size, int deg, double p_in, uint64_t seed,
              int scramble, uint64_t seed_scr, int valmode, uint64_t seed_v,
              synth_csr* out) {
  const int64_t n = n_comm * comm_size;
  if (n <= 0 || deg <= 0 || deg > comm_size || !out) return 1;
  Scramble scr(n, seed_scr);
  const uint64_t tin = thr53(p_in);
  Csr m;
  m.n = n;
  m.nnz = n * deg;
  m.row_ptr = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  m.col = (int32_t*)malloc(sizeof(int32_t) * (size_t)m.nnz);
  m.val = (float*)malloc(sizeof(float) * (size_t)m.nnz);
  if (!m.row_ptr || !m.col || !m.val) return 2;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i <= n; ++i) m.row_ptr[i] = i * deg;
#pragma omp parallel
  {
    std::vector<int64_t> cols(deg);
#pragma omp for schedule(static)
    for (int64_t p = 0; p < n; ++p) {
      const int64_t cb = (p / comm_size) * comm_size;
      int got = 0;
      for (uint64_t k = 0; got < deg; ++k) {
        uint64_t hA = h2(seed, (uint64_t)p, 2 * k), hB = h2(seed, (uint64_t)p, 2 * k + 1);
        int64_t q = ((hA >> 11) < tin) ? cb + (int64_t)(hB % (uint64_t)comm_size)
                                      : (int64_t)(hB % (uint64_t)n);
        bool dup = false;
        for (int t = 0; t < got; ++t) dup |= cols[t] == q;
        if (!dup) cols[got++] = q;
      }
      int64_t row = scramble ? scr(p) : p;
      for (int t = 0; t < deg; ++t) cols[t] = scramble ? scr(cols[t]) : cols[t];
      std::sort(cols.begin(), cols.end());
      for (int t = 0; t < deg; ++t) m.col[row * deg + t] = (int32_t)cols[t];
    }
  }
  fill_values(m, valmode, seed_v);
  to_out(m, out);
  return 0;
}

// 27-point stencil on an nx^3 grid, lexicographic id g = (z*nx + y)*nx + x.
// periodic != 0 wraps neighbours (27-regular); otherwise out-of-grid
// neighbours are dropped (Dirichlet).  relabel != 0: node g gets label
// Scramble(N, seed_scr)(g).
int synth_stencil27(int64_t nx, int periodic, int relabel, uint64_t seed_scr,
                    int valmode, uint64_t seed_v, synth_csr* out) {
  if (nx <= 0 || !out) return 1;
  const int64_t n = nx * nx * nx;
  if (n > (int64_t)INT32_MAX) return 1;
  Scramble scr(n, seed_scr);
  std::vector<int32_t> lab(n), inv(n);
#pragma omp parallel for schedule(static)
  for (int64_t g = 0; g < n; ++g) lab[g] = (int32_t)(relabel ? scr(g) : g);
#pragma omp parallel for schedule(static)
  for (int64_t g = 0; g < n; ++g) inv[lab[g]] = (int32_t)g;
  auto nbrs = [&](int64_t g, int32_t* outc) {
    int64_t x = g % nx, y = (g / nx) % nx, z = g / (nx * nx);
    int cnt = 0;
    for (int dz = -1; dz <= 1; ++dz)
      for (int dy = -1; dy <= 1; ++dy)
        for (int dx = -1; dx <= 1; ++dx) {
          int64_t X = x + dx, Y = y + dy, Z = z + dz;
          if (periodic) {
            X = (X + nx) % nx; Y = (Y + nx) % nx; Z = (Z + nx) % nx;
          } else if (X < 0 || Y < 0 || Z < 0 || X >= nx || Y >= nx || Z >= nx) {
            continue;
          }
          outc[cnt++] = lab[(Z * nx + Y) * nx + X];
        }
    return cnt;
  };
  std::vector<int64_t> len(n);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    int32_t tmp[27];
    int cnt = nbrs(inv[i], tmp);
    std::sort(tmp, tmp + cnt);
    len[i] = std::unique(tmp, tmp + cnt) - tmp;  // periodic nx<3 may repeat
  }
  Csr m;
  m.n = n;
  m.row_ptr = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  if (!m.row_ptr) return 2;
  exclusive_scan(len.data(), m.row_ptr, n);
  m.nnz = m.row_ptr[n];
  m.col = (int32_t*)malloc(sizeof(int32_t) * (size_t)std::max<int64_t>(m.nnz, 1));
  m.val = (float*)malloc(sizeof(float) * (size_t)std::max<int64_t>(m.nnz, 1));
  if (!m.col || !m.val) return 2;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    int32_t tmp[27];
    int cnt = nbrs(inv[i], tmp);
    std::sort(tmp, tmp + cnt);
    cnt = std::unique(tmp, tmp + cnt) - tmp;
    memcpy(m.col + m.row_ptr[i], tmp, sizeof(int32_t) * cnt);
  }
  fill_values(m, valmode, seed_v);
  to_out(m, out);
  return 0;
}

// Dense vector: x[i] = sym/pos/ones of h1(seed_x, i).
void synth_vector(int64_t n, uint64_t seed_x, int mode, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    uint64_t h = h1(seed_x, (uint64_t)i);
    out[i] = mode == 0 ? sym_f32(h) : mode == 1 ? pos_f32(h) : 1.0f;
  }
}

// The cycle-walking bijection table s(0..n-1) (e.g. SBM planted labels).
void synth_scramble(int64_t n, uint64_t seed_scr, int64_t* out) {
  Scramble scr(n, seed_scr);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = scr(i);
}

// Uniformly random permutation by the same bijection (used for RANDOM
// relabelling of inputs that are not produced by a generator here).
int synth_threads(void) { return omp_get_max_threads(); }

}  // extern "C"
