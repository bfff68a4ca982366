// nm_reorder: the SGRP heuristic of PAPER.md §4 (Alg. 1-3), deterministic and bit-identical
// to the CPU oracle under the readings of DESIGN.md §3.  Runs on the host (the greedy Stage-2
// is inherently sequential: every recorded pair changes which positions are still fresh);
// the per-row counting loops are OpenMP-parallel.  Works on the graph in its original labels
// through perm / iperm instead of materialising B = P A P^T.
#include <algorithm>
#include <chrono>
#include <cstdint>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <vector>

#include "nm_internal.h"

#ifdef _OPENMP
#include <omp.h>
#endif

namespace nm {
namespace {

struct Graph {
  int64_t n = 0;
  const int64_t* rp = nullptr;
  const int32_t* ci = nullptr;
  int64_t deg(int64_t v) const { return rp[v + 1] - rp[v]; }
};

// rank of b in the binary reflected Gray order = inverse Gray code (reading #1)
inline int64_t hamming_rank(uint64_t b) {
  uint64_t h = b;
  for (int sh = 1; sh < 64; sh <<= 1) h ^= h >> sh;
  return (int64_t)h;
}

// Per-row segment histogram of B row p: sorted (segment, bits) pairs.
struct RowSegs {
  std::vector<int64_t> seg;
  std::vector<uint32_t> bits;
  std::vector<int32_t> cnt;
};

inline void row_segments(const Graph& g, const std::vector<int32_t>& perm, const std::vector<int32_t>& iperm,
                         int64_t p, int M, std::vector<int32_t>& scratch, RowSegs& out) {
  const int32_t u = perm[p];
  scratch.clear();
  for (int64_t k = g.rp[u]; k < g.rp[u + 1]; ++k) scratch.push_back(iperm[g.ci[k]]);
  std::sort(scratch.begin(), scratch.end());
  out.seg.clear();
  out.bits.clear();
  out.cnt.clear();
  for (size_t i = 0; i < scratch.size();) {
    const int64_t s = scratch[i] / M;
    uint32_t b = 0;
    int c = 0;
    while (i < scratch.size() && scratch[i] / M == s) {
      b |= 1u << (M - 1 - (scratch[i] - s * M));  // first column of the segment -> MSB
      ++c;
      ++i;
    }
    out.seg.push_back(s);
    out.bits.push_back(b);
    out.cnt.push_back(c);
  }
}

// omega and PScore (horizontal constraint, L203 / L396)
int64_t omega_pscore(const Graph& g, const std::vector<int32_t>& perm, const std::vector<int32_t>& iperm, int N,
                     int M, std::vector<int32_t>* pscore) {
  const int64_t S = (g.n + M - 1) / M;
  if (pscore) pscore->assign(S, 0);
  int64_t omega = 0;
#pragma omp parallel reduction(+ : omega)
  {
    std::vector<int32_t> scratch;
    RowSegs rs;
#pragma omp for schedule(dynamic, 256)
    for (int64_t p = 0; p < g.n; ++p) {
      row_segments(g, perm, iperm, p, M, scratch, rs);
      for (size_t j = 0; j < rs.seg.size(); ++j)
        if (rs.cnt[j] > N) {
          ++omega;
          if (pscore) {
#pragma omp atomic
            (*pscore)[rs.seg[j]] += 1;
          }
        }
    }
  }
  return omega;
}

// MBscore: meta-blocks (V rows x M columns) with more than k = 4 distinct nonzero columns
int64_t mbscore(const Graph& g, const std::vector<int32_t>& perm, const std::vector<int32_t>& iperm, int V,
                int M) {
  const int64_t P = (g.n + V - 1) / V;
  int64_t mb = 0;
#pragma omp parallel reduction(+ : mb)
  {
    std::vector<int32_t> cols;
#pragma omp for schedule(dynamic, 64)
    for (int64_t r = 0; r < P; ++r) {
      cols.clear();
      const int64_t r1 = std::min<int64_t>(g.n, (r + 1) * (int64_t)V);
      for (int64_t p = r * (int64_t)V; p < r1; ++p) {
        const int32_t u = perm[p];
        for (int64_t k = g.rp[u]; k < g.rp[u + 1]; ++k) cols.push_back(iperm[g.ci[k]]);
      }
      std::sort(cols.begin(), cols.end());
      cols.erase(std::unique(cols.begin(), cols.end()), cols.end());
      for (size_t i = 0; i < cols.size();) {
        const int64_t s = cols[i] / M;
        int d = 0;
        while (i < cols.size() && cols[i] / M == s) { ++d; ++i; }
        if (d > 4) ++mb;
      }
    }
  }
  return mb;
}

void invert(const std::vector<int32_t>& perm, std::vector<int32_t>& iperm) {
  iperm.resize(perm.size());
  for (size_t p = 0; p < perm.size(); ++p) iperm[perm[p]] = (int32_t)p;
}

// ---- Stage-1: one sort (Alg. 2 lines 4-13) ------------------------------------------------
void stage1_sort(const Graph& g, std::vector<int32_t>& perm, std::vector<int32_t>& iperm, int N, int M) {
  const int64_t n = g.n, S = (n + M - 1) / M;
  // key of row p: pairs (sgn(c)*(S-s), c) for its nonzero codes in ascending s, then (0,0)
  std::vector<int64_t> koff(n + 1, 0);
  std::vector<std::vector<int64_t>> keys(n);
#pragma omp parallel
  {
    std::vector<int32_t> scratch;
    RowSegs rs;
#pragma omp for schedule(dynamic, 256)
    for (int64_t p = 0; p < n; ++p) {
      row_segments(g, perm, iperm, p, M, scratch, rs);
      std::vector<int64_t>& k = keys[p];
      k.clear();
      k.reserve(2 * rs.seg.size() + 2);
      for (size_t j = 0; j < rs.seg.size(); ++j) {
        const int64_t h = hamming_rank(rs.bits[j]);
        const int64_t c = (rs.cnt[j] > N) ? -h : h;  // negated when violating N:M (L313-319)
        if (c == 0) continue;
        k.push_back((c > 0 ? 1 : -1) * (S - rs.seg[j]));
        k.push_back(c);
      }
      k.push_back(0);
      k.push_back(0);
    }
  }
  std::vector<int64_t> order(n);
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(), [&](int64_t a, int64_t b) {
    return std::lexicographical_compare(keys[a].begin(), keys[a].end(), keys[b].begin(), keys[b].end());
  });
  std::vector<int32_t> np(n);
  for (int64_t p = 0; p < n; ++p) np[p] = perm[order[p]];
  perm.swap(np);
  invert(perm, iperm);
}

// ---- Stage-2 (Alg. 3) ----------------------------------------------------------------------
struct SegCount {
  // dense per-vertex counters with a touched list: cnt[w] = #vertices of the segment adjacent to w
  std::vector<int32_t> cnt;
  std::vector<int32_t> touched;
  std::vector<int32_t> mark;  // gain_table's N(x) marker (stamped, per counter owner)
  int32_t stamp = 0;
  void init(int64_t n) {
    cnt.assign(n, 0);
    mark.assign(n, 0);
    stamp = 0;
  }
  void build(const Graph& g, const std::vector<int32_t>& perm, int64_t seg, int M) {
    clear();
    for (int64_t q = seg * M; q < std::min<int64_t>(g.n, seg * M + M); ++q) {
      const int32_t x = perm[q];
      for (int64_t k = g.rp[x]; k < g.rp[x + 1]; ++k) {
        const int32_t w = g.ci[k];
        if (cnt[w] == 0) touched.push_back(w);
        cnt[w]++;
      }
    }
  }
  void clear() {
    for (int32_t w : touched) cnt[w] = 0;
    touched.clear();
  }
};

struct Pair {
  bool found = false;
  int64_t g = 0, gp = 0, gt = 0, u = -1, v = -1;
};

// gains of swapping positions u (segment p) and v (segment t), w.r.t. the pass-start order
inline void gains(const Graph& g, const std::vector<int32_t>& perm, const SegCount& cp, const SegCount& ct, int N,
                  int64_t u, int64_t v, int64_t* gp, int64_t* gt) {
  const int32_t x = perm[u], y = perm[v];
  int64_t a = g.rp[x], ae = g.rp[x + 1], b = g.rp[y], be = g.rp[y + 1];
  int64_t sp = 0, st = 0;
  while (a < ae || b < be) {
    int32_t w;
    int d;
    if (b >= be || (a < ae && g.ci[a] < g.ci[b])) { w = g.ci[a++]; d = -1; }
    else if (a >= ae || g.ci[b] < g.ci[a]) { w = g.ci[b++]; d = +1; }
    else { ++a; ++b; continue; }
    const int c1 = cp.cnt[w], c2 = ct.cnt[w];
    sp += (c1 > N) - (c1 + d > N);
    st += (c2 > N) - (c2 - d > N);
  }
  *gp = sp;
  *gt = st;
}

bool all_used(const std::vector<uint8_t>& used, int64_t seg, int M, int64_t n) {
  for (int64_t q = seg * M; q < std::min<int64_t>(n, seg * M + M); ++q)
    if (!used[q]) return false;
  return true;
}

// Gain table of a (primary p, target t) pair: (gp, gt) of every position pair (u, v) of the
// two segments w.r.t. the pass-start order (swap_cands = GetCandidates(prim, targ), Alg. 3 lines 11-14, L459-462).  The gains do not
// depend on which positions are already used, so a table can be computed ahead of the
// sequential pick (and in parallel with other targets' tables) without changing the result.
void gain_table(const Graph& g, const std::vector<int32_t>& perm, const SegCount& cp, SegCount& ct, int N,
                int M, int64_t p, int64_t t, const std::vector<uint8_t>& used, int64_t* tab /* [M*M*2] */) {
  // Same sums as gains(): a column w adjacent to x only contributes the d = -1 terms, one
  // adjacent to y only the d = +1 terms, a common one nothing.  Per u the x-only sums over
  // N(x) are formed once with N(x) marked; per v a walk of N(y) moves the common columns out
  // of them and adds the y-only ones (one pass over N(y) instead of a merge per pair).
  // Positions already used are never picked again (used only grows): their entries are skipped.
  const int64_t ue = std::min<int64_t>(g.n, p * M + M), ve = std::min<int64_t>(g.n, t * M + M);
  for (int64_t u = p * M; u < ue; ++u) {
    if (used[u]) continue;
    const int32_t x = perm[u];
    if (++ct.stamp == INT32_MAX) {
      std::fill(ct.mark.begin(), ct.mark.end(), 0);
      ct.stamp = 1;
    }
    const int32_t sx = ct.stamp;
    int64_t Sp = 0, St = 0;
    for (int64_t k = g.rp[x]; k < g.rp[x + 1]; ++k) {
      const int32_t w = g.ci[k];
      ct.mark[w] = sx;
      const int c1 = cp.cnt[w], c2 = ct.cnt[w];
      Sp += (c1 > N) - (c1 - 1 > N);
      St += (c2 > N) - (c2 + 1 > N);
    }
    for (int64_t v = t * M; v < ve; ++v) {
      if (used[v]) continue;
      const int32_t y = perm[v];
      int64_t sp = Sp, st = St;
      for (int64_t k = g.rp[y]; k < g.rp[y + 1]; ++k) {
        const int32_t w = g.ci[k];
        const int c1 = cp.cnt[w], c2 = ct.cnt[w];
        if (ct.mark[w] == sx) {
          sp -= (c1 > N) - (c1 - 1 > N);
          st -= (c2 > N) - (c2 + 1 > N);
        } else {
          sp += (c1 > N) - (c1 + 1 > N);
          st += (c2 > N) - (c2 - 1 > N);
        }
      }
      int64_t* e = tab + 2 * ((u - p * M) * M + (v - t * M));
      e[0] = sp;
      e[1] = st;
    }
  }
}

// freshtop (Alg. 3): the best fresh (u, v) pair over a precomputed table; scan u-major in
// position order, strict ">" so ties keep the smallest (u, v) (reading #18)
Pair pick_from_table(const int64_t* tab, int64_t n, int M, int64_t p, int64_t t, const std::vector<uint8_t>& used,
                     bool need_positive) {
  Pair best;
  for (int64_t u = p * M; u < std::min<int64_t>(n, p * M + M); ++u) {
    if (used[u]) continue;
    for (int64_t v = t * M; v < std::min<int64_t>(n, t * M + M); ++v) {
      if (used[v]) continue;
      const int64_t* e = tab + 2 * ((u - p * M) * M + (v - t * M));
      const int64_t gg = e[0] + e[1];
      if (need_positive && gg <= 0) continue;
      if (!best.found || gg > best.g) {
        best.found = true;
        best.g = gg;
        best.gp = e[0];
        best.gt = e[1];
        best.u = u;
        best.v = v;
      }
    }
  }
  return best;
}

// dev != nullptr: the gain tables come from the device (s2dev_tables, reorder_gpu.cu) -- the
// same integer sums, so the picks and the resulting order are identical to the host tables'
int64_t stage2(const Graph& g, std::vector<int32_t>& perm, std::vector<int32_t>& iperm, int N, int M,
               int maxiter, int gain_rule, int64_t* max_pairs, S2DeviceTables* dev, nm_status* err) {
  *err = NM_OK;
  const int64_t n = g.n, S = (n + M - 1) / M;
  int64_t passes = 0;
  std::vector<int32_t> pscore;
  std::vector<int64_t> est(S);
  std::vector<uint8_t> inI(S), used(n);
  SegCount cp, ct;
  cp.init(n);
  ct.init(n);
  std::vector<int64_t> su, sv, tb, tabs;
#ifdef _OPENMP
  const int nthr = std::max(1, std::min(omp_get_max_threads(), 16));
#else
  const int nthr = 1;
#endif
  std::vector<SegCount> cts(nthr);  // per-thread target counters for the parallel tables
  for (SegCount& c : cts) c.init(n);
  for (int it = 0; it <= maxiter; ++it) {
    omega_pscore(g, perm, iperm, N, M, &pscore);
    std::vector<int64_t> I;
    for (int64_t s = 0; s < S; ++s)
      if (pscore[s] > 0) I.push_back(s);
    if (I.empty()) break;
    std::stable_sort(I.begin(), I.end(), [&](int64_t a, int64_t b) { return pscore[a] > pscore[b]; });
    for (int64_t s = 0; s < S; ++s) { est[s] = pscore[s]; inI[s] = 0; }
    for (int64_t s : I) inI[s] = 1;
    std::fill(used.begin(), used.end(), 0);
    su.clear();
    sv.clear();
    if (dev && (*err = s2dev_set_perm(dev, perm.data())) != NM_OK) return passes;
    if (I.size() == 1) {
      const int64_t p = I[0];
      if (S == 1) break;
      int64_t t = -1, tn = 0;
      for (int64_t s = 0; s < S; ++s) {  // the sparsest other segment (reading #16)
        if (s == p) continue;
        int64_t z = 0;
        for (int64_t q = s * M; q < std::min<int64_t>(n, s * M + M); ++q) z += g.deg(perm[q]);
        if (t < 0 || z < tn) { t = s; tn = z; }
      }
      std::vector<int64_t> tab(2 * (size_t)M * M);
      if (dev) {
        if ((*err = s2dev_tables(dev, p, &t, 1, N, tab.data())) != NM_OK) return passes;
      } else {
        cp.build(g, perm, p, M);
        ct.build(g, perm, t, M);
        gain_table(g, perm, cp, ct, N, M, p, t, used, tab.data());
      }
      int64_t npairs = 0;
      for (;;) {
        Pair pr = pick_from_table(tab.data(), n, M, p, t, used, true);  // "beneficial" swaps
        if (!pr.found) break;
        su.push_back(pr.u);
        sv.push_back(pr.v);
        ++npairs;
        used[pr.u] = used[pr.v] = 1;
        est[p] -= pr.gp;
        if (est[p] <= 0 || all_used(used, p, M, n)) break;
      }
      *max_pairs = std::max(*max_pairs, npairs);
    } else {
      size_t head = 0;
      int64_t live = (int64_t)I.size();
      while (live > 1) {
        while (!inI[I[head]]) ++head;
        const int64_t p = I[head++];
        inI[p] = 0;
        --live;
        // the targets are the live entries of I after the primary, walked lazily: only the
        // target being picked can leave I, so this equals a snapshot taken when p is popped
        if (!dev) cp.build(g, perm, p, M);
        int64_t npairs = 0;
        // targets in batches: their gain tables in parallel, the picks in target order.  Only
        // the target being picked can leave I, so the batch's membership filter is final.
        size_t k = head, batch = (size_t)std::max(4, M);  // about the targets a primary needs (<= M pairs)
        bool stop = false;
        while (!stop && k < I.size()) {
          tb.clear();
          for (; k < I.size() && tb.size() < batch; ++k)
            if (inI[I[k]]) tb.push_back(I[k]);
          batch = std::min<size_t>(batch * 2, 256);
          if (tabs.size() < tb.size() * 2 * M * M) tabs.resize(tb.size() * 2 * M * M);
          const int64_t nb = (int64_t)tb.size();
          if (dev) {
            if ((*err = s2dev_tables(dev, p, tb.data(), (int)nb, N, tabs.data())) != NM_OK) return passes;
          }
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthr) if (nb > 1 && !dev)
          for (int64_t b = 0; b < (dev ? 0 : nb); ++b) {
#ifdef _OPENMP
            SegCount& c = cts[omp_get_thread_num()];
#else
            SegCount& c = cts[0];
#endif
            c.build(g, perm, tb[b], M);
            gain_table(g, perm, cp, c, N, M, p, tb[b], used, tabs.data() + (size_t)b * 2 * M * M);
            c.clear();
          }
          for (int64_t b = 0; b < nb; ++b) {
            const int64_t t = tb[b];
            Pair pr = pick_from_table(tabs.data() + (size_t)b * 2 * M * M, n, M, p, t, used, gain_rule == 1);
            if (!pr.found) continue;
            su.push_back(pr.u);
            sv.push_back(pr.v);
            ++npairs;
            used[pr.u] = used[pr.v] = 1;
            est[p] -= pr.gp;
            est[t] -= pr.gt;
            if (est[t] <= 0) { inI[t] = 0; --live; }
            if (est[p] <= 0 || all_used(used, p, M, n)) { stop = true; break; }
          }
        }
        *max_pairs = std::max(*max_pairs, npairs);
      }
      ct.clear();
    }
    cp.clear();
    if (su.empty()) break;
    for (size_t k = 0; k < su.size(); ++k) std::swap(perm[su[k]], perm[sv[k]]);
    invert(perm, iperm);
    ++passes;
  }
  return passes;
}

}  // namespace
}  // namespace nm

using namespace nm;

namespace nm {
namespace {

// The two steps of Alg. 1 that have a GPU version (Stage-1 sort and the counts); Stage-2
// stays on the host (its greedy is sequential in the recorded pairs).
struct Backend {
  virtual ~Backend() {}
  virtual S2DeviceTables* stage2_tables(int /*M*/, nm_status* st) { *st = NM_OK; return nullptr; }
  virtual nm_status stage1(std::vector<int32_t>& perm, std::vector<int32_t>& iperm, int N, int M) = 0;
  virtual nm_status counts(const std::vector<int32_t>& perm, const std::vector<int32_t>& iperm, int V, int N,
                           int M, int64_t* w, int64_t* mb) = 0;
};

struct HostBackend : Backend {
  const Graph& g;
  explicit HostBackend(const Graph& g_) : g(g_) {}
  nm_status stage1(std::vector<int32_t>& perm, std::vector<int32_t>& iperm, int N, int M) override {
    stage1_sort(g, perm, iperm, N, M);
    return NM_OK;
  }
  nm_status counts(const std::vector<int32_t>& perm, const std::vector<int32_t>& iperm, int V, int N, int M,
                   int64_t* w, int64_t* mb) override {
    *w = omega_pscore(g, perm, iperm, N, M, nullptr);
    *mb = mbscore(g, perm, iperm, V, M);
    return NM_OK;
  }
};

#ifndef NM_S2_DEVICE_TABLES
#define NM_S2_DEVICE_TABLES 0
#endif
// Stage-1 sort (reorder_gpu.cu) and omega / MBscore (counts.cu) on the device
struct DeviceBackend : Backend {
  const DevCsr& d;
  cudaStream_t s;
  int32_t* dperm = nullptr;
  S2DeviceTables* s2 = nullptr;
  int s2_M = 0;
  DeviceBackend(const DevCsr& d_, cudaStream_t s_) : d(d_), s(s_) {}
  ~DeviceBackend() override {
    if (dperm) cudaFree(dperm);
    s2dev_destroy(s2);
  }
  // The device gain tables are bit-identical to the host's but measured SLOWER on B200 (C3
  // 1:2:4, one Alg. 1 iteration: 87.7 s vs 28.7 s; banded n = 2^20: 3.27 s vs 0.71 s,
  // profiles/r02_reorder_timing.jsonl): the per-batch scatter / gain / clear launches and the
  // table read-back cost more than the host's OpenMP tables.  Compiled in with
  // -DNM_S2_DEVICE_TABLES=1 for measurement; the default uses the host tables.
  S2DeviceTables* stage2_tables(int M, nm_status* st) override {
    *st = NM_OK;
    if (!NM_S2_DEVICE_TABLES) return nullptr;
    if (s2 && s2_M != M) {
      s2dev_destroy(s2);
      s2 = nullptr;
    }
    if (!s2) {
      *st = s2dev_create(d, M, 256, s, &s2);  // 256 = the largest target batch of stage2()
      s2_M = M;
    }
    return s2;
  }
  nm_status upload(const std::vector<int32_t>& perm) {
    if (!dperm) NM_CUDA(cudaMalloc(&dperm, sizeof(int32_t) * d.n));
    NM_CUDA(cudaMemcpyAsync(dperm, perm.data(), sizeof(int32_t) * d.n, cudaMemcpyHostToDevice, s));
    return NM_OK;
  }
  nm_status stage1(std::vector<int32_t>& perm, std::vector<int32_t>& iperm, int N, int M) override {
    nm_status st = upload(perm);
    if (st == NM_OK) st = stage1_sort_dev(d, dperm, N, M, s);
    if (st != NM_OK) return st;
    NM_CUDA(cudaMemcpyAsync(perm.data(), dperm, sizeof(int32_t) * d.n, cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    invert(perm, iperm);
    return NM_OK;
  }
  nm_status counts(const std::vector<int32_t>& perm, const std::vector<int32_t>&, int V, int N, int M,
                   int64_t* w, int64_t* mb) override {
    nm_status st = upload(perm);
    if (st != NM_OK) return st;
    return count_violations_dev(d, dperm, V, N, M, w, mb, nullptr, s);
  }
};

#define NM_TRY(x)                   \
  do {                              \
    nm_status s_ = (x);             \
    if (s_ != NM_OK) return s_;     \
  } while (0)

// Alg. 1 on a validated host graph: perm_out receives the (keep-best) order.
nm_status reorder_core(const Graph& g, Backend& be, int V, int N, int M, const nm_reorder_opts& o,
                       int32_t* perm_out, nm_reorder_stats* st) {
  auto t0 = std::chrono::steady_clock::now();
  const int64_t n = g.n;
  std::vector<int32_t> perm(n), iperm(n), best;
  std::iota(perm.begin(), perm.end(), 0);
  iperm = perm;
  nm_reorder_stats stats;
  memset(&stats, 0, sizeof(stats));
  int64_t w = 0, mb = 0;
  NM_TRY(be.counts(perm, iperm, V, N, M, &w, &mb));
  stats.omega_init = w;
  stats.mb_init = mb;
  int64_t best_score = w + mb;
  best = perm;
  int64_t it = 0;
  double t_s1 = 0, t_s2 = 0;  // NM_REORDER_TRACE=1: per-stage wall time on stderr
  auto now = [] { return std::chrono::steady_clock::now(); };
  auto secs = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
    return std::chrono::duration<double>(b - a).count();
  };
  while ((w > 0 || mb > 0) && it <= o.max_outer) {
    int64_t mb1 = mb, w1 = 0;
    auto ta = now();
    for (int i1 = 0; mb1 > 0 && i1 <= o.max_stage1; ++i1) {  // Alg. 2
      NM_TRY(be.stage1(perm, iperm, N, M));
      stats.stage1_iters++;
      NM_TRY(be.counts(perm, iperm, V, N, M, &w1, &mb1));
    }
    auto tb = now();
    nm_status s2st = NM_OK;
    S2DeviceTables* dev = be.stage2_tables(M, &s2st);
    NM_TRY(s2st);
    stats.stage2_passes +=
        stage2(g, perm, iperm, N, M, o.max_stage2, o.gain_rule, &stats.max_pairs_per_primary, dev, &s2st);
    NM_TRY(s2st);
    t_s1 += secs(ta, tb);
    t_s2 += secs(tb, now());
    ++it;
    NM_TRY(be.counts(perm, iperm, V, N, M, &w, &mb));
    if (o.keep_best && w + mb < best_score) {
      best_score = w + mb;
      best = perm;
    }
  }
  stats.outer_iters = it;
  const std::vector<int32_t>& res = o.keep_best ? best : perm;
  memcpy(perm_out, res.data(), sizeof(int32_t) * n);
  invert(res, iperm);
  NM_TRY(be.counts(res, iperm, V, N, M, &stats.omega_final, &stats.mb_final));
  stats.seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  if (const char* tr = getenv("NM_REORDER_TRACE"))
    if (tr[0] == '1')
      fprintf(stderr, "nm_reorder trace: stage1(+MB counts) %.3f s, stage2 %.3f s, total %.3f s\n", t_s1, t_s2,
              stats.seconds);
  if (st) *st = stats;
  return NM_OK;
}

struct HostGraph {
  int64_t* rp = nullptr;
  int32_t* ci = nullptr;
  Graph g;
  ~HostGraph() { free(rp); free(ci); }
  nm_status load(const nm_csr* A) {
    nm_status s = host_csr(A, &rp, &ci);
    if (s != NM_OK) return s;
    s = validate_csr_host(A->n, rp, ci, true);
    if (s != NM_OK) return s;
    g.n = A->n;
    g.rp = rp;
    g.ci = ci;
    return NM_OK;
  }
};

nm_status check_graph_arg(const nm_csr* A) {
  if (A->n <= 0) return fail(NM_ERR_INVALID_ARG, "empty graph");
  if (A->n >= ((int64_t)1 << 31)) return fail(NM_ERR_UNSUPPORTED, "n >= 2^31");
  return NM_OK;
}

}  // namespace
}  // namespace nm

static nm_status reorder_host_impl(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                                   int32_t* perm_out, nm_reorder_stats* st) {
  if (!A || !perm_out) return fail(NM_ERR_INVALID_ARG, "nm_reorder: NULL argument");
  if (V < 1 || N < 1 || M <= N) return fail(NM_ERR_INVALID_ARG, "nm_reorder: need V >= 1, 1 <= N < M");
  if (M > 32) return fail(NM_ERR_UNSUPPORTED, "nm_reorder: M > 32");
  nm_status s = check_graph_arg(A);
  if (s != NM_OK) return s;
  nm_reorder_opts o = {10, 10, 10, 0, 1};
  if (opts) o = *opts;
  HostGraph hg;
  s = hg.load(A);
  if (s != NM_OK) return s;
  HostBackend be(hg.g);
  return reorder_core(hg.g, be, V, N, M, o, perm_out, st);
}

static nm_status reorder_gpu_impl(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                                  int32_t* perm_out, nm_reorder_stats* st, void* stream) {
  if (!A || !perm_out) return fail(NM_ERR_INVALID_ARG, "nm_reorder_gpu: NULL argument");
  if (V < 1 || N < 1 || M <= N) return fail(NM_ERR_INVALID_ARG, "nm_reorder_gpu: need V >= 1, 1 <= N < M");
  if (M > 32) return fail(NM_ERR_UNSUPPORTED, "nm_reorder_gpu: M > 32");
  nm_status s = check_graph_arg(A);
  if (s != NM_OK) return s;
  nm_reorder_opts o = {10, 10, 10, 0, 1};
  if (opts) o = *opts;
  HostGraph hg;  // Stage-2 walks the host copy
  s = hg.load(A);
  if (s != NM_OK) return s;
  cudaStream_t cs = (cudaStream_t)stream;
  DevCsr d;
  nm_csr pattern = *A;
  pattern.val = nullptr;  // the reorder needs the pattern only
  s = upload_csr(&pattern, NM_F16, &d, cs);
  if (s != NM_OK) return s;
  // the per-iteration scratch of Stage-1 and the counts comes from a private stream-ordered
  // pool, kept reserved between iterations and destroyed at the end of the call
  int dev = 0;
  NM_CUDA(cudaGetDevice(&dev));
  ScopedPool pool;
  NM_TRY(pool.init(dev));
  {
    DeviceBackend be(d, cs);
    s = reorder_core(hg.g, be, V, N, M, o, perm_out, st);
  }
  cudaStreamSynchronize(cs);
  return s;
}

static nm_status select_pattern_impl(const nm_csr* A, int max_M, int max_V, const nm_reorder_opts* opts,
                                     int32_t* perm_out, int* V_out, int* M_out, nm_reorder_stats* st) {
  if (!A || !perm_out || !V_out || !M_out) return fail(NM_ERR_INVALID_ARG, "nm_select_pattern: NULL argument");
  if (max_M < 4 || max_M > 32 || max_V < 1) return fail(NM_ERR_INVALID_ARG, "nm_select_pattern: need 4 <= max_M <= 32, max_V >= 1");
  nm_status s = check_graph_arg(A);
  if (s != NM_OK) return s;
  nm_reorder_opts o = {10, 10, 10, 0, 1};
  if (opts) o = *opts;
  HostGraph hg;
  s = hg.load(A);
  if (s != NM_OK) return s;
  const int64_t n = hg.g.n;
  std::vector<int32_t> cand(n);
  nm_reorder_stats cst;
  // 1:2:M with M = 4, 8, ... while the graph can be reordered to conform ...
  int bestV = 1, bestM = 4;
  nm_reorder_stats first;
  HostBackend be(hg.g);
  NM_TRY(reorder_core(hg.g, be, 1, 2, 4, o, perm_out, &first));
  if (st) *st = first;
  if (first.omega_final == 0 && first.mb_final == 0) {
    for (int M = 8; M <= max_M; M *= 2) {
      NM_TRY(reorder_core(hg.g, be, 1, 2, M, o, cand.data(), &cst));
      if (cst.omega_final != 0 || cst.mb_final != 0) break;
      bestM = M;
      memcpy(perm_out, cand.data(), sizeof(int32_t) * n);
      if (st) *st = cst;
    }
    // ... then V:2:M with V = 2, 4, ..., max_V "in a similar manner" (doubling)
    for (int V = 2; V <= max_V; V *= 2) {
      NM_TRY(reorder_core(hg.g, be, V, 2, bestM, o, cand.data(), &cst));
      if (cst.omega_final != 0 || cst.mb_final != 0) break;
      bestV = V;
      memcpy(perm_out, cand.data(), sizeof(int32_t) * n);
      if (st) *st = cst;
    }
  }
  *V_out = bestV;
  *M_out = bestM;
  return NM_OK;
}

extern "C" nm_status nm_reorder(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                                int32_t* perm_out, nm_reorder_stats* st) {
  return guarded("nm_reorder", [&] { return reorder_host_impl(A, V, N, M, opts, perm_out, st); });
}

extern "C" nm_status nm_reorder_gpu(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                                    int32_t* perm_out, nm_reorder_stats* st, void* stream) {
  return guarded("nm_reorder_gpu", [&] { return reorder_gpu_impl(A, V, N, M, opts, perm_out, st, stream); });
}

extern "C" nm_status nm_select_pattern(const nm_csr* A, int max_M, int max_V, const nm_reorder_opts* opts,
                                       int32_t* perm_out, int* V_out, int* M_out, nm_reorder_stats* st) {
  return guarded("nm_select_pattern",
                 [&] { return select_pattern_impl(A, max_M, max_V, opts, perm_out, V_out, M_out, st); });
}
