// spmv_reorder: host reordering (input preparation, timed separately).
//
// RABBIT (PAPER.md:86 §IV-A, :130 §V-A; Rabbit Order, ref [1] PAPER.md:259):
// modularity-maximising incremental aggregation, then community members get
// consecutive IDs by a DFS of the merge dendrogram.  The paper gives no
// algorithm; the deterministic reading (DESIGN.md
// §Readings) is implemented here sequentially so that it is reproducible bit
// for bit:
//   S = Bp + Bp^T over the off-diagonal 0/1 pattern; visit vertices in
//   ascending (deg, id); for u: aggregate u's S-row with the lists of the
//   children merged so far, map neighbours to their union-find roots, sum
//   weights per root, drop u; dQ' = 2m w_uv - tot_u tot_v (exact __int128);
//   merge into argmax (ties -> smallest root) iff dQ' > 0; else top level.
//   IDs: pre-order DFS from each top-level root in append order, children
//   in merge order.
// RABBIT++ (§VI-A): insular nodes (all S-neighbours in the
// same top-level community) grouped last, non-insular hubs (colcount*N > NZ)
// grouped first, RABBIT's relative order kept inside each group.
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <chrono>
#include <cmath>
#include <cstring>
#include <memory>
#include <numeric>
#include <stdexcept>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/spmv.h"

namespace spmv {
void set_error(const std::string& m);
}

namespace {

bool verbose() {
  static int v = -1;
  if (v < 0) v = getenv("SPMV_REORDER_VERBOSE") ? 1 : 0;
  return v == 1;
}

void phase(const char* what, std::chrono::steady_clock::time_point& t) {
  auto now = std::chrono::steady_clock::now();
  if (verbose())
    fprintf(stderr, "[spmv_reorder] %-14s %8.3f s\n", what,
            std::chrono::duration<double>(now - t).count());
  t = now;
}

struct Sym {  // S = Bp + Bp^T in CSR, weights 1 or 2
  int64_t n = 0;
  std::vector<int64_t> ptr;
  std::unique_ptr<int32_t[]> idx;  // uninitialised allocations: filled in parallel
  std::unique_ptr<uint8_t[]> w;
};

void scan_inplace(std::vector<int64_t>& v) {  // exclusive, v has n+1 slots
  int64_t acc = 0;
  for (auto& x : v) {
    int64_t t = x;
    x = acc;
    acc += t;
  }
}

// parallel exclusive scan of cnt[0..n) into out[0..n], out[n] = total
void scan_par(const int64_t* cnt, int64_t* out, int64_t n) {
  const int T = omp_get_max_threads();
  std::vector<int64_t> part(T + 1, 0);
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num(), TT = omp_get_num_threads();
    const int64_t lo = n * t / TT, hi = n * (t + 1) / TT;
    int64_t s = 0;
    for (int64_t i = lo; i < hi; ++i) s += cnt[i];
    part[t + 1] = s;
#pragma omp barrier
#pragma omp single
    for (int k = 1; k <= TT; ++k) part[k] += part[k - 1];
    int64_t a = part[t];
    for (int64_t i = lo; i < hi; ++i) {
      const int64_t c = cnt[i];
      out[i] = a;
      a += c;
    }
  }
  out[n] = part[T];
}

// S = Bp + Bp^T (reading c5).  Bp: per row sorted unique off-diagonal columns.
// Bp^T without random atomics: a stable radix partition of the (column, row)
// pairs into 2^16-column buckets (threads own contiguous row ranges, so each
// bucket receives its pairs in ascending row order), then a stable counting
// sort by column inside each bucket -- every transposed row comes out sorted.
// Rows of Bp and Bp^T are then merged; an entry present in both gets weight 2.
Sym symmetrize(int64_t n, const int64_t* rp, const int32_t* col) {
  const int64_t nnz = rp[n];
  std::unique_ptr<int32_t[]> bidx(new int32_t[std::max<int64_t>(nnz, 1)]);
  std::vector<int64_t> bl(n + 1, 0);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    int32_t* b = bidx.get() + rp[i];
    int64_t m = 0;
    bool sorted = true;
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k)
      if (col[k] != i) {
        if (m && col[k] <= b[m - 1]) sorted = false;
        b[m++] = col[k];
      }
    if (!sorted) {
      std::sort(b, b + m);
      m = std::unique(b, b + m) - b;
    }
    bl[i] = m;
  }
  constexpr int SHIFT = 16;
  const int64_t NB = (n >> SHIFT) + 1;
  const int T = omp_get_max_threads();
  // row ranges of the threads, balanced by entries
  std::vector<int64_t> rlo(T + 1, n);
  rlo[0] = 0;
  for (int t = 1; t < T; ++t)
    rlo[t] = std::lower_bound(rp, rp + n + 1, nnz * t / T) - rp;
  for (int t = 1; t <= T; ++t) rlo[t] = std::max(rlo[t], rlo[t - 1]);
  std::vector<int64_t> cnt((size_t)T * NB, 0);  // [t][bucket]
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    int64_t* c = cnt.data() + (size_t)t * NB;
    for (int64_t i = rlo[t]; i < rlo[t + 1]; ++i)
      for (int64_t k = 0; k < bl[i]; ++k) c[bidx[rp[i] + k] >> SHIFT]++;
  }
  // bucket-major offsets: off[b][t]
  std::vector<int64_t> off((size_t)NB * T + 1);
  {
    int64_t a = 0;
    for (int64_t b = 0; b < NB; ++b)
      for (int t = 0; t < T; ++t) {
        off[(size_t)b * T + t] = a;
        a += cnt[(size_t)t * NB + b];
      }
    off[(size_t)NB * T] = a;
  }
  const int64_t nt = off[(size_t)NB * T];
  std::unique_ptr<uint64_t[]> pairs(new uint64_t[std::max<int64_t>(nt, 1)]);  // col << 32 | row
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    std::vector<int64_t> cur(NB);
    for (int64_t b = 0; b < NB; ++b) cur[b] = off[(size_t)b * T + t];
    for (int64_t i = rlo[t]; i < rlo[t + 1]; ++i)
      for (int64_t k = 0; k < bl[i]; ++k) {
        const uint32_t j = (uint32_t)bidx[rp[i] + k];
        pairs[cur[j >> SHIFT]++] = ((uint64_t)j << 32) | (uint32_t)i;
      }
  }
  std::vector<int64_t> tptr(n + 1, 0);
  std::unique_ptr<int32_t[]> tidx(new int32_t[std::max<int64_t>(nt, 1)]);
#pragma omp parallel
  {
    std::vector<int64_t> cc((size_t)1 << SHIFT);
#pragma omp for schedule(dynamic, 1)
    for (int64_t b = 0; b < NB; ++b) {
      const int64_t p0 = off[(size_t)b * T], p1 = off[(size_t)(b + 1) * T];
      const int64_t j0 = b << SHIFT, j1 = std::min<int64_t>(n, (b + 1) << SHIFT);
      std::fill(cc.begin(), cc.begin() + (j1 - j0), 0);
      for (int64_t q = p0; q < p1; ++q) cc[(pairs[q] >> 32) - j0]++;
      int64_t a = p0;
      for (int64_t j = j0; j < j1; ++j) {
        tptr[j] = a;
        const int64_t c = cc[j - j0];
        cc[j - j0] = a;
        a += c;
      }
      for (int64_t q = p0; q < p1; ++q) {
        const uint64_t e = pairs[q];
        tidx[cc[(e >> 32) - j0]++] = (int32_t)(uint32_t)e;
      }
    }
  }
  tptr[n] = nt;
  pairs.reset();
  // merge row i of Bp and Bp^T
  Sym S;
  S.n = n;
  S.ptr.assign(n + 1, 0);
  std::vector<int64_t> len(n);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    const int32_t *a = bidx.get() + rp[i], *ae = a + bl[i];
    const int32_t *b = tidx.get() + tptr[i], *be = tidx.get() + tptr[i + 1];
    int64_t m = 0;
    while (a < ae || b < be) {
      if (b == be || (a < ae && *a < *b)) ++a;
      else if (a == ae || *b < *a) ++b;
      else { ++a; ++b; }
      ++m;
    }
    len[i] = m;
  }
  scan_par(len.data(), S.ptr.data(), n);
  const int64_t ns = S.ptr[n];
  S.idx.reset(new int32_t[std::max<int64_t>(ns, 1)]);
  S.w.reset(new uint8_t[std::max<int64_t>(ns, 1)]);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    const int32_t *a = bidx.get() + rp[i], *ae = a + bl[i];
    const int32_t *b = tidx.get() + tptr[i], *be = tidx.get() + tptr[i + 1];
    int64_t o = S.ptr[i];
    while (a < ae || b < be) {
      if (b == be || (a < ae && *a < *b)) { S.idx[o] = *a++; S.w[o++] = 1; }
      else if (a == ae || *b < *a) { S.idx[o] = *b++; S.w[o++] = 1; }
      else { S.idx[o] = *a; S.w[o++] = 2; ++a; ++b; }
    }
  }
  return S;
}

struct __attribute__((packed)) Edge {  // 12 bytes: aggregated lists dominate host memory
  int32_t v;
  int64_t w;
};

struct MergeRec {  // one merge of the dendrogram: child u into root v, exact gain dQ'
  int32_t u, v;
  __int128 dq;
};

struct Rabbit {
  std::vector<int32_t> perm, comm;
  int64_t two_m = 0, n_merges = 0, n_top = 0, n_deferred = 0, n_retries = 0;
  bool parallel = false;
  std::vector<MergeRec> log;  // filled when requested (SPMV_REORDER_LOG)
};

// ascending (deg, id) order of the vertices (reading c7): a stable counting
// sort, in parallel -- threads own contiguous id ranges, per-thread histograms
// of degrees below 2^16 are scanned degree-major, so ids stay ascending inside
// each degree; the few larger degrees are sorted by (deg, id) and go last
std::vector<int64_t> degree_order(const std::vector<int64_t>& deg) {
  const int64_t n = (int64_t)deg.size();
  constexpr int64_t DB = 1 << 16;
  const int T = omp_get_max_threads();
  std::vector<int64_t> order(n);
  std::vector<int64_t> h((size_t)T * DB, 0);  // [t][d]
  std::vector<std::vector<int64_t>> big(T);
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    const int64_t lo = n * t / T, hi = n * (t + 1) / T;
    int64_t* ht = h.data() + (size_t)t * DB;
    for (int64_t v = lo; v < hi; ++v) {
      if (deg[v] < DB) ht[deg[v]]++;
      else big[t].push_back(v);
    }
#pragma omp barrier
#pragma omp single
    {
      int64_t a = 0;
      for (int64_t d = 0; d < DB; ++d)
        for (int k = 0; k < T; ++k) {
          const int64_t c = h[(size_t)k * DB + d];
          h[(size_t)k * DB + d] = a;
          a += c;
        }
      std::vector<int64_t> bg;
      for (auto& b : big) bg.insert(bg.end(), b.begin(), b.end());
      std::sort(bg.begin(), bg.end(), [&](int64_t x, int64_t y) {
        return deg[x] != deg[y] ? deg[x] < deg[y] : x < y;
      });
      for (int64_t v : bg) order[a++] = v;
    }
    for (int64_t v = lo; v < hi; ++v)
      if (deg[v] < DB) order[ht[deg[v]]++] = v;
  }
  return order;
}

// pre-order DFS of the dendrogram (reading c10): roots in `top` order,
// children in merge order
// The trees are independent: their sizes (one counting DFS each, in
// parallel) give every root its first ID by a prefix sum, then each tree is
// numbered in parallel -- the same IDs as one sequential pass.
void dendrogram_ids(const std::vector<int32_t>& top, const std::vector<int32_t>& first_child,
                    const std::vector<int32_t>& next_sib, Rabbit& R, int64_t n) {
  R.perm.assign(n, -1);
  R.comm.assign(n, -1);
  const int64_t nt = (int64_t)top.size();
  std::vector<int64_t> size(nt + 1, 0);
#pragma omp parallel
  {
    std::vector<int32_t> st;
#pragma omp for schedule(dynamic, 1024)
    for (int64_t t = 0; t < nt; ++t) {
      int64_t m = 0;
      st.push_back(top[t]);
      while (!st.empty()) {
        const int32_t x = st.back();
        st.pop_back();
        ++m;
        for (int32_t c = first_child[x]; c != -1; c = next_sib[c]) st.push_back(c);
      }
      size[t] = m;
    }
  }
  scan_inplace(size);
#pragma omp parallel
  {
    std::vector<int32_t> st;
#pragma omp for schedule(dynamic, 1024)
    for (int64_t t = 0; t < nt; ++t) {
      const int32_t r = top[t];
      int32_t nxt = (int32_t)size[t];
      st.push_back(r);
      while (!st.empty()) {
        const int32_t x = st.back();
        st.pop_back();
        R.perm[x] = nxt++;
        R.comm[x] = r;
        const size_t mark = st.size();
        for (int32_t c = first_child[x]; c != -1; c = next_sib[c]) st.push_back(c);
        std::reverse(st.begin() + mark, st.end());
      }
    }
  }
  R.n_top = nt;
}

Rabbit rabbit_detect(const Sym& S, bool want_log) {
  const int64_t n = S.n;
  std::vector<int64_t> deg(n);
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < n; ++v) {
    int64_t d = 0;
    for (int64_t k = S.ptr[v]; k < S.ptr[v + 1]; ++k) d += S.w[k];
    deg[v] = d;
  }
  int64_t two_m = 0;
  for (int64_t v = 0; v < n; ++v) two_m += deg[v];
  const std::vector<int64_t> order = degree_order(deg);
  std::vector<int32_t> parent(n);
  std::iota(parent.begin(), parent.end(), 0);
  auto find = [&](int32_t v) {
    int32_t r = v;
    while (parent[r] != r) r = parent[r];
    while (parent[v] != r) {
      int32_t nx = parent[v];
      parent[v] = r;
      v = nx;
    }
    return r;
  };
  std::vector<int64_t> tot(deg);
  std::vector<int32_t> first_child(n, -1), last_child(n, -1), next_sib(n, -1);
  std::vector<std::vector<Edge>> agg(n);
  std::vector<int64_t> acc(n, 0);
  std::vector<int32_t> touched;
  std::vector<int32_t> top;
  Rabbit R;
  R.two_m = two_m;
  for (int64_t oi = 0; oi < n; ++oi) {
    const int32_t u = (int32_t)order[oi];
    touched.clear();
    auto add = [&](int32_t w, int64_t wt) {
      int32_t r = find(w);
      if (r == u) return;
      if (acc[r] == 0) touched.push_back(r);
      acc[r] += wt;
    };
    // the loop is memory-latency bound (random parent / acc accesses):
    // prefetch the union-find entry of a neighbour PF iterations ahead
    constexpr int PF = 16;
    {
      const int64_t k0 = S.ptr[u], k1 = S.ptr[u + 1];
      for (int64_t k = k0; k < k1; ++k) {
        if (k + PF < k1) __builtin_prefetch(&parent[S.idx[k + PF]]);
        add(S.idx[k], S.w[k]);
      }
    }
    for (int32_t c = first_child[u]; c != -1; c = next_sib[c]) {
      const std::vector<Edge>& L = agg[c];
      const size_t m = L.size();
      for (size_t i = 0; i < m; ++i) {
        if (i + PF < m) __builtin_prefetch(&parent[L[i + PF].v]);
        add(L[i].v, L[i].w);
      }
      std::vector<Edge>().swap(agg[c]);
    }
    if (oi + 1 < n) {  // next vertex's row and union-find entry
      const int32_t un = (int32_t)order[oi + 1];
      __builtin_prefetch(&S.idx[S.ptr[un]]);
      __builtin_prefetch(&first_child[un]);
    }
    int32_t best = -1;
    __int128 bestdq = 0;
    for (int32_t r : touched) {
      __int128 dq = (__int128)two_m * acc[r] - (__int128)tot[u] * tot[r];
      if (best == -1 || dq > bestdq || (dq == bestdq && r < best)) {
        best = r;
        bestdq = dq;
      }
    }
    if (best != -1 && bestdq > 0) {
      parent[u] = best;
      tot[best] += tot[u];
      if (last_child[best] == -1) first_child[best] = u;
      else next_sib[last_child[best]] = u;
      last_child[best] = u;
      agg[u].reserve(touched.size());
      for (int32_t r : touched) agg[u].push_back({r, acc[r]});
      R.n_merges++;
      if (want_log) R.log.push_back({u, best, bestdq});
    } else {
      top.push_back(u);
    }
    for (int32_t r : touched) acc[r] = 0;
  }
  dendrogram_ids(top, first_child, next_sib, R, n);
  return R;
}

// ------------------------------------------------ concurrent merges (f4)
// Rabbit Order's parallel incremental aggregation (ref [1], PAPER.md:259;
// SURVEY §8(f4)): threads take vertices in the same ascending (deg, id) order
// (dynamic chunks) and run the sequential step on each, with three states in
// tot[] besides a community's total degree:
//   PROC    u is being aggregated: nothing merges into u meanwhile, so u's
//           children (all merged before) are final;
//   MLOCK   short critical section of a merge into v;
//   MERGED  u is no longer a root.
// A merge u -> v locks v (CAS from a valid total), recomputes the EXACT
// weight w(C_u, C_v) from u's aggregated list with the current union-find
// roots (v's community cannot change under the lock, u's cannot change while
// PROC), and merges only if dQ' = 2m w - tot_u tot_v > 0 -- so every recorded
// gain is the exact change of Q'/2 and Q'_final - Q'_init = 2 sum dQ' holds.
// A target that is being processed (PROC) defers u; deferred vertices are
// processed sequentially afterwards, in order.  The result depends on thread
// timing (not bit-exact with the oracle); tests check it by these invariants.
struct HashAcc {  // per-thread (root -> summed weight) map, open addressing
  std::vector<int32_t> key;
  std::vector<int64_t> val;
  std::vector<uint32_t> used;
  uint32_t mask = 0;
  static size_t cap_for(size_t expect) {
    size_t cap = 64;
    while (cap < 2 * expect) cap <<= 1;
    return cap;
  }
  void prepare(size_t expect) {  // capacity for `expect` keys (grows further on demand)
    const size_t cap = cap_for(expect);
    if (cap > key.size()) rehash(cap);
  }
  void rehash(size_t cap) {
    std::vector<int32_t> k2(cap, -1);
    std::vector<int64_t> v2(cap, 0);
    std::vector<uint32_t> u2;
    u2.reserve(used.size());
    const uint32_t m2 = (uint32_t)(cap - 1);
    for (uint32_t h : used) {
      uint32_t g = ((uint32_t)key[h] * 2654435761u) & m2;
      while (k2[g] != -1) g = (g + 1) & m2;
      k2[g] = key[h];
      v2[g] = val[h];
      u2.push_back(g);
    }
    key.swap(k2);
    val.swap(v2);
    used.swap(u2);
    mask = m2;
  }
  inline void add(int32_t r, int64_t w) {
    if (2 * (used.size() + 1) > key.size()) rehash(cap_for(used.size() + 1) * 2);
    uint32_t h = ((uint32_t)r * 2654435761u) & mask;
    while (key[h] != -1 && key[h] != r) h = (h + 1) & mask;
    if (key[h] == -1) {
      key[h] = r;
      used.push_back(h);
    }
    val[h] += w;
  }
  void clear() {
    for (uint32_t h : used) {
      key[h] = -1;
      val[h] = 0;
    }
    used.clear();
  }
  void release() {  // give a huge table back after a hub
    std::vector<int32_t>().swap(key);
    std::vector<int64_t>().swap(val);
    std::vector<uint32_t>().swap(used);
    mask = 0;
  }
};

Rabbit rabbit_detect_par(const Sym& S, bool want_log) {
  const int64_t n = S.n;
  constexpr int64_t PROC = -1, MLOCK = -2, MERGED = -3;
  auto tp = std::chrono::steady_clock::now();
  std::vector<int64_t> deg(n);
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < n; ++v) {
    int64_t d = 0;
    for (int64_t k = S.ptr[v]; k < S.ptr[v + 1]; ++k) d += S.w[k];
    deg[v] = d;
  }
  int64_t two_m = 0;
#pragma omp parallel for reduction(+ : two_m) schedule(static)
  for (int64_t v = 0; v < n; ++v) two_m += deg[v];
  const std::vector<int64_t> order = degree_order(deg);
  std::vector<int64_t> pos(n);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) pos[order[i]] = i;
  std::unique_ptr<std::atomic<int64_t>[]> tot(new std::atomic<int64_t>[n]);
  std::unique_ptr<std::atomic<int32_t>[]> parent(new std::atomic<int32_t>[n]);
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < n; ++v) {
    tot[v].store(deg[v], std::memory_order_relaxed);
    parent[v].store((int32_t)v, std::memory_order_relaxed);
  }
  // written only under the target's MLOCK (or by u's own thread while PROC)
  std::vector<int32_t> first_child(n, -1), last_child(n, -1), next_sib(n, -1);
  std::vector<std::vector<Edge>> agg(n);
  auto find = [&](int32_t v) {  // path halving; concurrent shortcuts stay valid
    for (;;) {
      const int32_t p = parent[v].load(std::memory_order_acquire);
      if (p == v) return v;
      const int32_t g = parent[p].load(std::memory_order_acquire);
      if (g != p) parent[v].store(g, std::memory_order_relaxed);
      v = g;
    }
  };
  const int T = omp_get_max_threads();
  std::vector<std::vector<int32_t>> deferred(T);
  std::vector<std::vector<MergeRec>> logs(T);
  std::vector<int64_t> merges(T, 0), retries(T, 0);
  std::vector<HashAcc> Hs(T), Hsmall(T);  // small: vertices with short lists (cache-resident)
  phase("par:setup", tp);

  auto expected = [&](int32_t u) {
    size_t e = (size_t)(S.ptr[u + 1] - S.ptr[u]);
    for (int32_t c = first_child[u]; c != -1; c = next_sib[c]) e += agg[c].size();
    return e;
  };
  // u's aggregated list: its S-row and its children's lists, neighbours
  // mapped to their current roots, weights summed per root, u dropped
  auto aggregate = [&](int32_t u, HashAcc& H, std::vector<Edge>& tl) {
    H.prepare(std::min<size_t>(expected(u), (size_t)1 << 20));
    for (int64_t k = S.ptr[u]; k < S.ptr[u + 1]; ++k) {
      const int32_t r = find(S.idx[k]);
      if (r != u) H.add(r, S.w[k]);
    }
    for (int32_t c = first_child[u]; c != -1; c = next_sib[c])
      for (const Edge& e : agg[c]) {
        const int32_t r = find(e.v);
        if (r != u) H.add(r, e.w);
      }
    tl.clear();
    for (uint32_t h : H.used) tl.push_back({H.key[h], H.val[h]});
    H.clear();
    if (H.key.size() > ((size_t)1 << 22)) H.release();
  };
  // the same list with every thread (the tail phase, where the hubs with the
  // largest aggregated lists come last and nothing else runs): chunks of the
  // S-row and child lists hashed per thread, then a group-by on root % T
  std::vector<std::vector<Edge>> parts((size_t)T * T), outs(T);
  auto aggregate_all = [&](int32_t u, std::vector<Edge>& tl) {
    struct Seg { int32_t c; int64_t b, e; };  // c = -1: S-row of u
    std::vector<Seg> segs;
    constexpr int64_t CH = 1 << 15;
    for (int64_t b = S.ptr[u]; b < S.ptr[u + 1]; b += CH)
      segs.push_back({-1, b, std::min<int64_t>(b + CH, S.ptr[u + 1])});
    for (int32_t c = first_child[u]; c != -1; c = next_sib[c])
      for (int64_t b = 0; b < (int64_t)agg[c].size(); b += CH)
        segs.push_back({c, b, std::min<int64_t>(b + CH, (int64_t)agg[c].size())});
    const size_t ex = expected(u);
#pragma omp parallel num_threads(T)
    {
      const int t = omp_get_thread_num();
      HashAcc& H = Hs[t];
      H.prepare(std::min<size_t>(ex / T + 1024, (size_t)1 << 24));
#pragma omp for schedule(dynamic, 1)
      for (int64_t q = 0; q < (int64_t)segs.size(); ++q) {
        const Seg& g = segs[q];
        if (g.c < 0) {
          for (int64_t k = g.b; k < g.e; ++k) {
            const int32_t r = find(S.idx[k]);
            if (r != u) H.add(r, S.w[k]);
          }
        } else {
          const Edge* L = agg[g.c].data();
          for (int64_t k = g.b; k < g.e; ++k) {
            const int32_t r = find(L[k].v);
            if (r != u) H.add(r, L[k].w);
          }
        }
      }
      for (uint32_t h : H.used) parts[(size_t)t * T + (uint32_t)H.key[h] % (uint32_t)T].push_back({H.key[h], H.val[h]});
      H.clear();
#pragma omp barrier
      size_t m = 0;
      for (int t2 = 0; t2 < T; ++t2) m += parts[(size_t)t2 * T + t].size();
      H.prepare(std::min<size_t>(m, (size_t)1 << 24));
      for (int t2 = 0; t2 < T; ++t2) {
        for (const Edge& e : parts[(size_t)t2 * T + t]) H.add(e.v, e.w);
        std::vector<Edge>().swap(parts[(size_t)t2 * T + t]);
      }
      outs[t].clear();
      for (uint32_t h : H.used) outs[t].push_back({H.key[h], H.val[h]});
      H.clear();
      if (H.key.size() > ((size_t)1 << 24)) H.release();
    }
    tl.clear();
    for (int t = 0; t < T; ++t) tl.insert(tl.end(), outs[t].begin(), outs[t].end());
  };

  // one step of the sequential reading on u.  mode 0: concurrent (returns
  // false when u is deferred: its target is being processed, or u's
  // aggregated list is large enough to deserve every thread later); mode 1:
  // nothing else runs (no recheck needed); mode 2: as 1, aggregated with
  // every thread
  // postponed with every thread: lists of more than 1/(32 T) of all entries
  // (smaller ones are cheaper on one thread while the others work)
  const size_t BIG = std::max<size_t>((size_t)1 << 16, (size_t)(two_m / (32 * (int64_t)T)));
  std::vector<std::vector<int32_t>> bigs(T);
  auto step = [&](int32_t u, HashAcc& H, std::vector<Edge>& tl, int tid, int mode) -> bool {
    int64_t tu;
    for (;;) {  // PROC-lock u (it may be the target of a short merge section)
      tu = tot[u].load(std::memory_order_acquire);
      if (tu == MLOCK) continue;
      if (tot[u].compare_exchange_weak(tu, PROC, std::memory_order_acq_rel)) break;
    }
    if (mode == 0 && expected(u) > BIG) {
      tot[u].store(tu, std::memory_order_release);
      bigs[tid].push_back(u);
      return false;
    }
    auto free_children = [&]() {
      for (int32_t c = first_child[u]; c != -1; c = next_sib[c]) std::vector<Edge>().swap(agg[c]);
    };
    for (int attempt = 0;; ++attempt) {
      if (mode == 2) aggregate_all(u, tl);
      else aggregate(u, expected(u) <= 1024 ? Hsmall[tid] : H, tl);
      int32_t best = -1;
      __int128 bestdq = 0;
      int64_t bestw = 0;
      for (const Edge& e : tl) {
        const int64_t tr = tot[e.v].load(std::memory_order_acquire);
        if (tr < 0) continue;  // being processed / locked / merged meanwhile
        const __int128 dq = (__int128)two_m * e.w - (__int128)tu * tr;
        if (best == -1 || dq > bestdq || (dq == bestdq && e.v < best)) {
          best = e.v;
          bestdq = dq;
          bestw = e.w;
        }
      }
      if (best == -1 || bestdq <= 0) {
        free_children();
        tot[u].store(tu, std::memory_order_release);
        return true;
      }
      if (mode != 0) {  // exclusive: the aggregation is current, the gain exact
        const int64_t tv = tot[best].load(std::memory_order_relaxed);
        agg[u] = tl;
        if (last_child[best] == -1) first_child[best] = u;
        else next_sib[last_child[best]] = u;
        last_child[best] = u;
        parent[u].store(best, std::memory_order_relaxed);
        tot[u].store(MERGED, std::memory_order_relaxed);
        tot[best].store(tv + tu, std::memory_order_relaxed);
        merges[tid]++;
        if (want_log) logs[tid].push_back({u, best, (__int128)two_m * bestw - (__int128)tu * tv});
        free_children();
        return true;
      }
      // exact w(C_u, C_v) against a snapshot tv of the target's total.  tot
      // only grows with merges into v (and turns MERGED when v itself merges),
      // so a CAS that still finds tv proves C_v is the community w was
      // computed against; the critical section is then just the bookkeeping.
      int outcome = 0;  // 0: re-aggregate, 1: merged, 2: defer, 3: no gain
      agg[u] = tl;      // published with the merge (read by v's processor later)
      for (int k = 0; k < 16 && outcome == 0; ++k) {
        int64_t tv = tot[best].load(std::memory_order_acquire);
        while (tv == MLOCK) tv = tot[best].load(std::memory_order_acquire);
        if (tv == PROC) { outcome = 2; break; }
        if (tv == MERGED) break;
        int64_t w = 0;
        for (const Edge& e : tl)
          if (find(e.v) == best) w += e.w;
        const __int128 dq = (__int128)two_m * w - (__int128)tu * tv;
        if (dq <= 0) { outcome = 3; break; }
        int64_t expect = tv;
        if (!tot[best].compare_exchange_strong(expect, MLOCK, std::memory_order_acq_rel)) {
          retries[tid]++;
          continue;
        }
        if (last_child[best] == -1) first_child[best] = u;
        else next_sib[last_child[best]] = u;
        last_child[best] = u;
        parent[u].store(best, std::memory_order_release);
        tot[u].store(MERGED, std::memory_order_release);
        tot[best].store(tv + tu, std::memory_order_release);
        merges[tid]++;
        if (want_log) logs[tid].push_back({u, best, dq});
        outcome = 1;
      }
      if (outcome == 1) {
        free_children();
        return true;
      }
      std::vector<Edge>().swap(agg[u]);
      if (outcome == 2 || attempt >= 3) {
        if (outcome == 3) {  // the best gain vanished: u stays top level
          free_children();
          tot[u].store(tu, std::memory_order_release);
            return true;
        }
        tot[u].store(tu, std::memory_order_release);
        deferred[tid].push_back(u);
        return false;
      }
      retries[tid]++;
    }
  };

  // every vertex in parallel (large aggregations postponed), then the
  // deferred ones in processing order: the large ones with every thread
#pragma omp parallel num_threads(T)
  {
    const int tid = omp_get_thread_num();
    std::vector<Edge> tl;
#pragma omp for schedule(dynamic, 256)
    for (int64_t oi = 0; oi < n; ++oi) step((int32_t)order[oi], Hs[tid], tl, tid, 0);
  }
  phase("par:merges", tp);
  Rabbit R;
  R.parallel = true;
  R.two_m = two_m;
  {
    std::vector<int32_t> rest;
    for (auto& d : deferred) rest.insert(rest.end(), d.begin(), d.end());
    R.n_deferred = (int64_t)rest.size();
    for (auto& d : bigs) rest.insert(rest.end(), d.begin(), d.end());
    std::sort(rest.begin(), rest.end(), [&](int32_t a, int32_t b) { return pos[a] < pos[b]; });
    std::vector<Edge> tl;
    double t_all = 0, t_one = 0;
    int64_t n_all = 0;
    for (int32_t u : rest) {
      const bool all = expected(u) > BIG;
      auto t0 = std::chrono::steady_clock::now();
      step(u, Hs[0], tl, 0, all ? 2 : 1);
      const double dt = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
      if (all) { t_all += dt; n_all++; } else t_one += dt;
    }
    if (verbose())
      fprintf(stderr, "[spmv_reorder] deferred: %lld (%lld large, %.3f s), others %.3f s\n",
              (long long)rest.size(), (long long)n_all, t_all, t_one);
  }
  phase("par:tail", tp);
  for (int t = 0; t < T; ++t) {
    R.n_merges += merges[t];
    R.n_retries += retries[t];
  }
  if (want_log)
    for (auto& l : logs) R.log.insert(R.log.end(), l.begin(), l.end());
  // top level = the vertices still roots, in processing order (the
  // sequential reading's append order): a parallel compaction of `order`
  std::vector<int32_t> top;
  {
    const int TT = omp_get_max_threads();
    std::vector<int64_t> cnt(TT + 1, 0);
#pragma omp parallel num_threads(TT)
    {
      const int t = omp_get_thread_num();
      const int64_t lo = n * t / TT, hi = n * (t + 1) / TT;
      int64_t c = 0;
      for (int64_t i = lo; i < hi; ++i) c += tot[order[i]].load(std::memory_order_relaxed) != MERGED;
      cnt[t + 1] = c;
#pragma omp barrier
#pragma omp single
      {
        for (int k = 1; k <= TT; ++k) cnt[k] += cnt[k - 1];
        top.resize(cnt[TT]);
      }
      int64_t o = cnt[t];
      for (int64_t i = lo; i < hi; ++i)
        if (tot[order[i]].load(std::memory_order_relaxed) != MERGED) top[o++] = (int32_t)order[i];
    }
  }
  phase("par:top", tp);
#pragma omp parallel for schedule(dynamic, 65536)
  for (int64_t v = 0; v < n; ++v) std::vector<Edge>().swap(agg[v]);
  std::vector<std::vector<Edge>>().swap(agg);
  phase("par:free", tp);
  dendrogram_ids(top, first_child, next_sib, R, n);
  phase("par:dfs", tp);
  return R;
}

inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}

void random_order(int64_t n, uint64_t seed, int32_t* perm) {
  std::vector<int32_t> p(n);
  std::iota(p.begin(), p.end(), 0);
  for (int64_t i = n - 1; i > 0; --i) {
    uint64_t h = mix64(seed + 0x9E3779B97F4A7C15ull * (uint64_t)(i + 1));
    int64_t j = (int64_t)(h % (uint64_t)(i + 1));
    std::swap(p[i], p[j]);
  }
  std::memcpy(perm, p.data(), sizeof(int32_t) * n);
}

}  // namespace

static thread_local std::vector<int32_t> g_last_comm;

namespace {
struct DetectCache {
  bool valid = false;
  uint64_t key = 0;
  int64_t n = -1, nnz = -1;
  Rabbit R;
  bool logged = false;
  std::vector<uint8_t> ins;
  double seconds_detect = 0, seconds_build = 0, largest = 0, qnum = 0, q = 0, insularity = 0;
};
thread_local DetectCache g_cache;

struct InputCache {  // validation + skew + column counts + hub flags of the last input
  bool valid = false;
  uint64_t key = 0;
  int64_t n = -1, nnz = -1, nh = 0;
  double skew = 0;
  std::vector<int64_t> colcnt;
  std::vector<uint8_t> hub;
};
thread_local InputCache g_input;

uint64_t input_key(int64_t n, int64_t nnz, const int64_t* rp, const int32_t* col) {
  uint64_t a = 0, b = 0;
#pragma omp parallel for reduction(+ : a) schedule(static)
  for (int64_t i = 0; i <= n; ++i) a += mix64((uint64_t)rp[i] * 0x9E3779B97F4A7C15ull + (uint64_t)i);
#pragma omp parallel for reduction(+ : b) schedule(static)
  for (int64_t k = 0; k < nnz; ++k) b += mix64(((uint64_t)(uint32_t)col[k] << 32) ^ (uint64_t)k);
  return mix64(a ^ mix64(b) ^ (uint64_t)n * 31 ^ (uint64_t)nnz);
}
}  // namespace

extern "C" spmv_status spmv_reorder(int64_t n, int64_t nnz, const int64_t* rp, const int32_t* col,
                                    int method, uint64_t seed, int32_t* perm_out,
                                    spmv_reorder_stats_t* st) {
  nvtxRangePushA("spmv_reorder");
  struct Pop {
    ~Pop() { nvtxRangePop(); }
  } pop_;
  try {
    auto t0 = std::chrono::steady_clock::now();
    const bool par = (method & SPMV_REORDER_PARALLEL) != 0;
    const bool want_log = (method & SPMV_REORDER_LOG) != 0;
    method &= 0xff;
    if (n < 0 || nnz < 0 || !rp || (nnz && !col) || (n && !perm_out)) {
      spmv::set_error("spmv_reorder: bad argument");
      return SPMV_EINVAL;
    }
    if (n > (int64_t)INT32_MAX - 1) {
      spmv::set_error("spmv_reorder: n must fit int32");
      return SPMV_EUNSUPPORTED;
    }
    if (rp[0] != 0 || rp[n] != nnz) {
      spmv::set_error("spmv_reorder: row_ptr inconsistent with nnz");
      return SPMV_EINVAL;
    }
    // validation, skew, column counts and hub flags depend on the input only:
    // kept per thread for the next call on the same matrix (a bench orders one
    // matrix several ways)
    const uint64_t key = input_key(n, nnz, rp, col);
    auto tp = std::chrono::steady_clock::now();
    spmv_reorder_stats_t S0;
    std::memset(&S0, 0, sizeof(S0));
    InputCache& IC = g_input;
    if (!(IC.valid && IC.key == key && IC.n == n && IC.nnz == nnz)) {
      IC.valid = false;
      IC.skew = 0.0;
      int64_t bad_rp = 0, bad_col = 0;
#pragma omp parallel for schedule(static) reduction(+ : bad_rp)
      for (int64_t i = 0; i < n; ++i) bad_rp += rp[i + 1] < rp[i];
      if (bad_rp) {
        spmv::set_error("spmv_reorder: row_ptr not monotone");
        return SPMV_EINVAL;
      }
#pragma omp parallel for schedule(static) reduction(+ : bad_col)
      for (int64_t k = 0; k < nnz; ++k) bad_col += col[k] < 0 || col[k] >= n;
      if (bad_col) {
        spmv::set_error("spmv_reorder: column out of range");
        return SPMV_EINVAL;
      }
      phase("validate", tp);
      // skew: top ceil(0.1 N) row lengths / NZ
      {
        // exact: lengths below 2^16 by a histogram (per thread, merged), the few
        // longer ones sorted; the top ceil(0.1 N) taken from the longest down
        const int64_t top = (int64_t)std::ceil(0.1 * (double)n);
        if (top > 0 && n > 0) {
          constexpr int64_t HB = 1 << 16;
          std::vector<int64_t> hist(HB, 0);
          std::vector<int64_t> longl;
#pragma omp parallel
          {
            std::vector<int64_t> h(HB, 0);
            std::vector<int64_t> lg;
#pragma omp for schedule(static) nowait
            for (int64_t i = 0; i < n; ++i) {
              const int64_t L = rp[i + 1] - rp[i];
              if (L < HB) h[L]++;
              else lg.push_back(L);
            }
#pragma omp critical
            {
              for (int64_t b = 0; b < HB; ++b) hist[b] += h[b];
              longl.insert(longl.end(), lg.begin(), lg.end());
            }
          }
          std::sort(longl.begin(), longl.end(), std::greater<int64_t>());
          int64_t left = top, s = 0;
          for (size_t q = 0; q < longl.size() && left > 0; ++q, --left) s += longl[q];
          for (int64_t b = HB - 1; b >= 0 && left > 0; --b) {
            const int64_t take = std::min(left, hist[b]);
            s += take * b;
            left -= take;
          }
          IC.skew = nnz ? (double)s / (double)nnz : 0.0;
        }
      }
      // in-degree (column counts, diagonal and duplicates included: reading c13)
      std::vector<int64_t> colcnt(n, 0);
#pragma omp parallel for schedule(static)
      for (int64_t k = 0; k < nnz; ++k) __atomic_fetch_add(&colcnt[col[k]], (int64_t)1, __ATOMIC_RELAXED);
      std::vector<uint8_t> hub(n);
      int64_t nh = 0;
#pragma omp parallel for schedule(static) reduction(+ : nh)
      for (int64_t v = 0; v < n; ++v) {
        hub[v] = (__int128)colcnt[v] * n > (__int128)nnz;
        nh += hub[v];
      }
      IC.nh = nh;
      IC.colcnt.swap(colcnt);
      IC.hub.swap(hub);
      IC.key = key;
      IC.n = n;
      IC.nnz = nnz;
      IC.valid = true;
      phase("skew+colcnt", tp);
    }
    S0.skew = IC.skew;
    S0.n_hubs = IC.nh;
    const std::vector<int64_t>& colcnt = IC.colcnt;
    const std::vector<uint8_t>& hub = IC.hub;

    if (method == SPMV_ORDER_ORIGINAL) {
      for (int64_t i = 0; i < n; ++i) perm_out[i] = (int32_t)i;
    } else if (method == SPMV_ORDER_RANDOM) {
      random_order(n, seed, perm_out);
    } else if (method == SPMV_ORDER_DEGSORT) {
      std::vector<int32_t> seq(n);
      std::iota(seq.begin(), seq.end(), 0);
      std::stable_sort(seq.begin(), seq.end(),
                       [&](int32_t a, int32_t b) { return colcnt[a] > colcnt[b]; });
      for (int64_t i = 0; i < n; ++i) perm_out[seq[i]] = (int32_t)i;
    } else if ((method >= SPMV_ORDER_RABBIT && method <= SPMV_ORDER_HUBGROUP) ||
               method == SPMV_ORDER_HUBSORT_ONLY) {
      // community detection is shared by RABBIT and every RABBIT++ variant:
      // reuse the last detection on this thread when the input is identical
      double reused_s = 0;  // detection reused from the cache: charged to this call too
      if (!(g_cache.valid && g_cache.key == key && g_cache.n == n && g_cache.nnz == nnz &&
            g_cache.R.parallel == par && (!want_log || g_cache.logged))) {
        g_cache.valid = false;
        const auto tb = std::chrono::steady_clock::now();
        Sym S = symmetrize(n, rp, col);
        phase("symmetrize", tp);
        auto td = std::chrono::steady_clock::now();
        g_cache.R = par ? rabbit_detect_par(S, want_log) : rabbit_detect(S, want_log);
        g_cache.logged = want_log;
        g_cache.seconds_detect =
            std::chrono::duration<double>(std::chrono::steady_clock::now() - td).count();
        phase("detect+dfs", tp);
        Rabbit& R = g_cache.R;
        // community sizes
        {
          std::vector<int64_t> sz(n, 0);
          const Rabbit& Rr = R;
#pragma omp parallel for schedule(static)
          for (int64_t v = 0; v < n; ++v) __atomic_fetch_add(&sz[Rr.comm[v]], (int64_t)1, __ATOMIC_RELAXED);
          int64_t mx = 0;
#pragma omp parallel for reduction(max : mx) schedule(static)
          for (int64_t v = 0; v < n; ++v) mx = std::max(mx, sz[v]);
          g_cache.largest = n ? (double)mx / (double)n : 0.0;
        }
        // modularity Q' = sum_c (2m in_c - tot_c^2) and insular flags
        g_cache.ins.assign(n, 1);
        {
          // per-vertex sums in parallel, per-community accumulation in order
          std::vector<int64_t> vin(n), vtot(n);
          uint8_t* insp = g_cache.ins.data();  // g_cache is thread_local: no access in the region
          const Rabbit& Rr = R;
#pragma omp parallel for schedule(dynamic, 4096)
          for (int64_t v = 0; v < n; ++v) {
            const int32_t c = Rr.comm[v];
            int64_t a = 0, t = 0;
            uint8_t ins = 1;
            for (int64_t k = S.ptr[v]; k < S.ptr[v + 1]; ++k) {
              t += S.w[k];
              if (Rr.comm[S.idx[k]] == c) a += S.w[k];
              else ins = 0;
            }
            vin[v] = a;
            vtot[v] = t;
            insp[v] = ins;
          }
          // per-community sums fit int64 (each <= 2m); Q' itself needs int128
          std::vector<int64_t> inc(n, 0), totc(n, 0);
#pragma omp parallel for schedule(static)
          for (int64_t v = 0; v < n; ++v) {
            __atomic_fetch_add(&inc[Rr.comm[v]], vin[v], __ATOMIC_RELAXED);
            __atomic_fetch_add(&totc[Rr.comm[v]], vtot[v], __ATOMIC_RELAXED);
          }
          const int T = omp_get_max_threads();
          std::vector<__int128> qt(T, 0);
#pragma omp parallel num_threads(T)
          {
            __int128 a = 0;
#pragma omp for schedule(static)
            for (int64_t c = 0; c < n; ++c)
              if (totc[c] || inc[c]) a += (__int128)R.two_m * inc[c] - (__int128)totc[c] * totc[c];
            qt[omp_get_thread_num()] = a;
          }
          __int128 q = 0;
          for (int t = 0; t < T; ++t) q += qt[t];
          g_cache.qnum = (double)q;
          g_cache.q = R.two_m ? (double)q / ((double)R.two_m * (double)R.two_m) : 0.0;
        }
        // insularity over distinct off-diagonal pairs of A (reading c12)
        {
          int64_t intra = 0, total = 0;
#pragma omp parallel reduction(+ : intra, total)
          {
            std::vector<int32_t> tmp;
#pragma omp for schedule(dynamic, 4096)
            for (int64_t i = 0; i < n; ++i) {
              tmp.assign(col + rp[i], col + rp[i + 1]);
              if (!std::is_sorted(tmp.begin(), tmp.end())) std::sort(tmp.begin(), tmp.end());
              tmp.erase(std::unique(tmp.begin(), tmp.end()), tmp.end());
              for (int32_t j : tmp)
                if (j != i) {
                  total++;
                  intra += R.comm[j] == R.comm[i];
                }
            }
          }
          g_cache.insularity = total ? (double)intra / (double)total : 1.0;
        }
        phase("stats", tp);
        g_cache.key = key;
        g_cache.n = n;
        g_cache.nnz = nnz;
        g_cache.valid = true;
        g_cache.seconds_build =
            std::chrono::duration<double>(std::chrono::steady_clock::now() - tb).count();
      } else {
        reused_s = g_cache.seconds_build;
      }
      t0 -= std::chrono::duration_cast<std::chrono::steady_clock::duration>(
          std::chrono::duration<double>(reused_s));
      const Rabbit& R = g_cache.R;
      const std::vector<uint8_t>& ins = g_cache.ins;
      S0.seconds_detect = g_cache.seconds_detect;
      S0.two_m = R.two_m;
      S0.n_merges = R.n_merges;
      S0.n_deferred = R.n_deferred;
      S0.parallel = R.parallel ? 1 : 0;
      S0.n_communities = R.n_top;
      S0.largest_comm_frac = g_cache.largest;
      S0.modularity_num = g_cache.qnum;
      S0.modularity = g_cache.q;
      S0.insularity = g_cache.insularity;
      {
        int64_t ni = 0;
        for (int64_t v = 0; v < n; ++v) ni += ins[v];
        S0.insular_frac = n ? (double)ni / (double)n : 0.0;
        S0.n_insular = ni;
      }
      if (method == SPMV_ORDER_RABBIT) {
        std::memcpy(perm_out, R.perm.data(), sizeof(int32_t) * n);
      } else {
        std::vector<int32_t> seq(n);
        for (int64_t v = 0; v < n; ++v) seq[R.perm[v]] = (int32_t)v;
        std::vector<int32_t> out;
        out.reserve(n);
        auto take = [&](auto pred) {
          for (int32_t v : seq)
            if (pred(v)) out.push_back(v);
        };
        if (method == SPMV_ORDER_RABBITPP || method == SPMV_ORDER_HUBSORT) {
          take([&](int32_t v) { return !ins[v] && hub[v]; });
          S0.n_group0 = (int64_t)out.size();
          if (method == SPMV_ORDER_HUBSORT)
            std::stable_sort(out.begin(), out.end(),
                             [&](int32_t a, int32_t b) { return colcnt[a] > colcnt[b]; });
          take([&](int32_t v) { return !ins[v] && !hub[v]; });
          take([&](int32_t v) { return (bool)ins[v]; });
        } else if (method == SPMV_ORDER_INSULAR) {
          take([&](int32_t v) { return !ins[v]; });
          take([&](int32_t v) { return (bool)ins[v]; });
        } else {  // HUBGROUP only / HUBSORT only (no insular grouping)
          take([&](int32_t v) { return (bool)hub[v]; });
          S0.n_group0 = (int64_t)out.size();
          if (method == SPMV_ORDER_HUBSORT_ONLY)
            std::stable_sort(out.begin(), out.end(),
                             [&](int32_t a, int32_t b) { return colcnt[a] > colcnt[b]; });
          take([&](int32_t v) { return !hub[v]; });
        }
        for (int64_t i = 0; i < n; ++i) perm_out[out[i]] = (int32_t)i;
      }
      g_last_comm = R.comm;
    } else {
      spmv::set_error("spmv_reorder: unknown method");
      return SPMV_EINVAL;
    }
    S0.seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (st) *st = S0;
    return SPMV_OK;
  } catch (const std::bad_alloc&) {
    spmv::set_error("spmv_reorder: out of host memory");
    return SPMV_ENOMEM;
  } catch (...) {
    spmv::set_error("spmv_reorder: internal error");
    return SPMV_EINVAL;
  }
}

extern "C" spmv_status spmv_reorder_last_merges(int64_t cap, int32_t* child, int32_t* parent,
                                                int64_t* dq, int64_t* count_out) {
  if (!count_out || (cap > 0 && (!child || !parent || !dq))) {
    spmv::set_error("spmv_reorder_last_merges: bad argument");
    return SPMV_EINVAL;
  }
  if (!g_cache.valid || !g_cache.logged) {
    spmv::set_error("spmv_reorder_last_merges: no logged RABBIT detection on this thread");
    return SPMV_ESTATE;
  }
  const std::vector<MergeRec>& L = g_cache.R.log;
  *count_out = (int64_t)L.size();
  for (int64_t i = 0; i < std::min<int64_t>(cap, (int64_t)L.size()); ++i) {
    if (L[i].dq > (__int128)INT64_MAX || L[i].dq < (__int128)INT64_MIN) {
      spmv::set_error("spmv_reorder_last_merges: gain exceeds int64");
      return SPMV_EUNSUPPORTED;
    }
    child[i] = L[i].u;
    parent[i] = L[i].v;
    dq[i] = (int64_t)L[i].dq;
  }
  return SPMV_OK;
}

extern "C" spmv_status spmv_reorder_last_comm(int64_t n, int32_t* comm_out) {
  if ((int64_t)g_last_comm.size() != n || (n && !comm_out)) {
    spmv::set_error("spmv_reorder_last_comm: no RABBIT result of this size on this thread");
    return SPMV_EINVAL;
  }
  std::memcpy(comm_out, g_last_comm.data(), sizeof(int32_t) * n);
  return SPMV_OK;
}
