/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY (the CPU oracle).
 *
 * Plain, slow, obviously correct CPU implementation of what the hot path of
 *   J.-A. Chen, H.-H. Sung, R. Zhang, A. Li, X. Shen, "Accelerating GNNs on GPU Sparse
 *   Tensor Cores through N:M Sparsity-Oriented Graph Reordering", PPoPP'25
 * computes.  "PAPER.md:Lxxx" below cites the line of the paper text (with the section,
 * algorithm or table it sits in); "reading #k" cites DESIGN.md's list of readings where the
 * paper is silent, garbled or ambiguous.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ppopp_chensz0s25_b200/csrc) and includes nothing from it.
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"):
 *   or_hamming_code / or_position_code -- worked values PAPER.md:L286-319, brute-force minimal
 *       cumulative-Hamming orders, reflected-Gray construction.
 *   or_counts (omega, PScore, MBscore) -- brute force on dense matrices in Python.
 *   or_reorder / or_stage2_trace -- Figure-1 fixture F1 (unique answer), four hand-derived
 *       Stage-2 passes (tests/golden/s2_fixture_{a,b,c,d}.txt: priority order, gain tables,
 *       recorded pairs of both branches of Alg. 3; 13 oracle mutants killed,
 *       tools/oracle_mutants.py), brute-force optimum bound on tiny graphs, invariants
 *       (bijection, keep-best, <= M pairs per primary).
 *   or_pack_* -- unpack(pack)+residual == B bitwise, conforming => empty residual, F1 nibbles.
 *   or_spmm_f64 -- dense numpy A@X on small cases; closed forms (identity, all-ones).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define OR_K 4 /* k of the vertical constraint: "4 by default" (Fig. 2 table) */

/* ------------------------------------------------------------------------------------- */
/* Hamming position code (§4.2)                                        */
/* ------------------------------------------------------------------------------------- */

/* Rank of the bit string b in the Hamming-distance order of all strings of its length.
 * The Hamming-distance order the paper uses ({00,01,11,10} for 2 digits, L294-296) is the
 * binary reflected Gray code, whose i-th element is i ^ (i>>1); the rank of b is therefore
 * the inverse Gray code b ^ b>>1 ^ b>>2 ^ ... (reading #1). */
int64_t or_hamming_code(uint64_t b) {
  uint64_t h = 0;
  while (b) { h ^= b; b >>= 1; }
  return (int64_t)h;
}

static int popc64(uint64_t x) { int c = 0; while (x) { c += (int)(x & 1u); x >>= 1; } return c; }

/* Position code with the horizontal-violation negation (L313-319, Alg. 2 lines 8-10 at L344-346). */
int64_t or_position_code(uint64_t b, int N) {
  int64_t h = or_hamming_code(b);
  return popc64(b) > N ? -h : h;
}

/* ------------------------------------------------------------------------------------- */
/* B = P A P^T in new labels (Fig. 1 caption L38; L130-137)                               */
/* perm[p] = old vertex at new position p; B[p][q] = A[perm[p]][perm[q]].                 */
/* ------------------------------------------------------------------------------------- */

typedef struct { int64_t n; int64_t* rp; int32_t* ci; int64_t* src; } or_csr; /* src: index into A's arrays */

static int cmp64(const void* a, const void* b) {
  int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
  return (x > y) - (x < y);
}

static void csr_free(or_csr* B) { free(B->rp); free(B->ci); free(B->src); }

static int cmp_i32(const void* a, const void* b) {
  int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
  return (x > y) - (x < y);
}

/* Builds B with sorted columns; src[k] = position in A's col/val arrays of entry k of B. */
static int build_B(int64_t n, const int64_t* rp, const int32_t* ci, const int32_t* perm, or_csr* B) {
  int32_t* iperm = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int64_t nnz = rp[n];
  B->n = n;
  B->rp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  B->ci = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  B->src = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nnz > 0 ? nnz : 1));
  for (int64_t p = 0; p < n; ++p) iperm[perm ? perm[p] : p] = (int32_t)p;
  B->rp[0] = 0;
  for (int64_t p = 0; p < n; ++p) {
    int32_t u = perm ? perm[p] : (int32_t)p;
    B->rp[p + 1] = B->rp[p] + (rp[u + 1] - rp[u]);
  }
  /* pairs (new col, src) sorted by new col: encode as int64 col<<32 | local, sort per row */
  for (int64_t p = 0; p < n; ++p) {
    int32_t u = perm ? perm[p] : (int32_t)p;
    int64_t d = rp[u + 1] - rp[u];
    int64_t* tmp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(d > 0 ? d : 1));
    for (int64_t k = 0; k < d; ++k) tmp[k] = ((int64_t)iperm[ci[rp[u] + k]] << 32) | k;
    qsort(tmp, (size_t)d, sizeof(int64_t), cmp64);
    for (int64_t k = 0; k < d; ++k) {
      B->ci[B->rp[p] + k] = (int32_t)(tmp[k] >> 32);
      B->src[B->rp[p] + k] = rp[u] + (tmp[k] & 0xFFFFFFFF);
    }
    free(tmp);
  }
  free(iperm);
  return 0;
}

/* Validation: square CSR with sorted, duplicate-free, in-range columns; symmetric pattern.
 * returns 0 ok, 1 bad csr, 2 not symmetric. */
int or_validate(int64_t n, const int64_t* rp, const int32_t* ci) {
  if (rp[0] != 0) return 1;
  for (int64_t i = 0; i < n; ++i) {
    if (rp[i + 1] < rp[i]) return 1;
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      if (ci[k] < 0 || ci[k] >= n) return 1;
      if (k > rp[i] && ci[k] <= ci[k - 1]) return 1;
    }
  }
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      int32_t j = ci[k];
      /* binary search i in row j */
      int64_t lo = rp[j], hi = rp[j + 1] - 1, found = 0;
      while (lo <= hi) {
        int64_t mid = (lo + hi) / 2;
        if (ci[mid] == i) { found = 1; break; }
        if (ci[mid] < i) lo = mid + 1; else hi = mid - 1;
      }
      if (!found) return 2;
    }
  return 0;
}

/* ------------------------------------------------------------------------------------- */
/* Violation counts: omega (L203), PScore (L396), MBscore (L382, Fig. 3 caption L370)      */
/* ------------------------------------------------------------------------------------- */

/* M-bit string of row i of B over segment s: first column of the segment -> MSB
 * (Listing 1: val = (val << 1) | bit over i = 0..M-1; reading #2). */
static uint64_t seg_bits(const or_csr* B, int64_t i, int64_t s, int M) {
  uint64_t b = 0;
  int64_t lo = s * M, hi = s * M + M;
  for (int64_t k = B->rp[i]; k < B->rp[i + 1]; ++k) {
    int64_t q = B->ci[k];
    if (q >= lo && q < hi) b |= (uint64_t)1 << (M - 1 - (q - lo));
  }
  return b;
}

/* Number of nonzeros of row i of B in segment s (c_s(i) of DESIGN.md). */
static int seg_count(const or_csr* B, int64_t i, int64_t s, int M) {
  int c = 0;
  int64_t lo = s * M, hi = s * M + M;
  for (int64_t k = B->rp[i]; k < B->rp[i + 1]; ++k) {
    int64_t q = B->ci[k];
    if (q >= lo && q < hi) ++c;
  }
  return c;
}

/* omega = #segment vectors with more than N nonzeros; pscore[s] = the same count restricted
 * to segment s; mb = #meta-blocks (V rows x M columns) with more than k=4 distinct nonzero
 * columns (vertical constraint, reading #5). */
static void counts_B(const or_csr* B, int V, int N, int M, int64_t* omega, int64_t* mb,
                     int32_t* pscore) {
  int64_t n = B->n, S = (n + M - 1) / M;
  int64_t w = 0, m = 0;
  if (pscore) memset(pscore, 0, sizeof(int32_t) * (size_t)S);
  for (int64_t i = 0; i < n; ++i) {
    /* walk the sorted row, one segment at a time */
    int64_t k = B->rp[i];
    while (k < B->rp[i + 1]) {
      int64_t s = B->ci[k] / M;
      int c = 0;
      while (k < B->rp[i + 1] && B->ci[k] / M == s) { ++c; ++k; }
      if (c > N) { ++w; if (pscore) pscore[s] += 1; }
    }
  }
  int64_t P = (n + V - 1) / V;
  for (int64_t r = 0; r < P; ++r) {
    int64_t r0 = r * V, r1 = r0 + V < n ? r0 + V : n;
    int64_t cnt = B->rp[r1] - B->rp[r0];
    int32_t* cols = (int32_t*)malloc(sizeof(int32_t) * (size_t)(cnt > 0 ? cnt : 1));
    memcpy(cols, B->ci + B->rp[r0], sizeof(int32_t) * (size_t)cnt);
    qsort(cols, (size_t)cnt, sizeof(int32_t), cmp_i32);
    int64_t k = 0;
    while (k < cnt) {
      int64_t s = cols[k] / M;
      int distinct = 0;
      int32_t last = -1;
      while (k < cnt && cols[k] / M == s) {
        if (cols[k] != last) { ++distinct; last = cols[k]; }
        ++k;
      }
      if (distinct > OR_K) ++m;
    }
    free(cols);
  }
  *omega = w;
  *mb = m;
}

int or_counts(int64_t n, const int64_t* rp, const int32_t* ci, const int32_t* perm, int V, int N,
              int M, int64_t* omega, int64_t* mb, int32_t* pscore) {
  or_csr B;
  build_B(n, rp, ci, perm, &B);
  counts_B(&B, V, N, M, omega, mb, pscore);
  csr_free(&B);
  return 0;
}

/* ------------------------------------------------------------------------------------- */
/* Stage-1 (Alg. 2; steps (i)-(v) L374-382)                                     */
/* ------------------------------------------------------------------------------------- */

typedef struct { int64_t* key; int64_t len; int64_t row; } s1_key; /* key = pairs flattened */

static int cmp_s1(const void* a, const void* b) {
  const s1_key* x = (const s1_key*)a;
  const s1_key* y = (const s1_key*)b;
  int64_t L = x->len < y->len ? x->len : y->len;
  for (int64_t i = 0; i < L; ++i) {
    if (x->key[i] != y->key[i]) return x->key[i] < y->key[i] ? -1 : 1;
  }
  if (x->len != y->len) return x->len < y->len ? -1 : 1;
  return (x->row > y->row) - (x->row < y->row); /* stable: ties keep current position */
}

/* One Stage-1 sort: Vec[i][s] = position code of row i's segment s (Alg. 2 lines 4-10);
 * rows sorted ascending by the lexicographic order of their code vectors (line 11,
 * reading #6).  The dense vector is compared through the equivalent sparse key
 * [(sgn(c)*(S-s), c) for nonzero c, ascending s] ++ [(0,0)] (zero codes are "left out of
 * the sorting", L384; tests pin the equivalence against dense comparison). */
static void stage1_sort(const or_csr* B, int N, int M, int32_t* perm) {
  int64_t n = B->n, S = (n + M - 1) / M;
  s1_key* keys = (s1_key*)malloc(sizeof(s1_key) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) {
    /* distinct segments of row i, ascending */
    int64_t deg = B->rp[i + 1] - B->rp[i];
    keys[i].key = (int64_t*)malloc(sizeof(int64_t) * (size_t)(2 * deg + 2));
    keys[i].row = i;
    int64_t L = 0, k = B->rp[i];
    while (k < B->rp[i + 1]) {
      int64_t s = B->ci[k] / M;
      while (k < B->rp[i + 1] && B->ci[k] / M == s) ++k;
      uint64_t b = seg_bits(B, i, s, M);
      int64_t c = or_position_code(b, N);
      int64_t sg = c > 0 ? 1 : (c < 0 ? -1 : 0);
      if (c != 0) { keys[i].key[L++] = sg * (S - s); keys[i].key[L++] = c; }
    }
    keys[i].key[L++] = 0;
    keys[i].key[L++] = 0;
    keys[i].len = L;
  }
  qsort(keys, (size_t)n, sizeof(s1_key), cmp_s1);
  int32_t* np_ = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t p = 0; p < n; ++p) np_[p] = perm[keys[p].row]; /* perm <- perm[order] */
  memcpy(perm, np_, sizeof(int32_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i) free(keys[i].key);
  free(keys);
  free(np_);
}

/* ------------------------------------------------------------------------------------- */
/* Stage-2 (Alg. 3; details (i)-(v) L402-413, footnote L440)                    */
/* ------------------------------------------------------------------------------------- */

typedef struct {
  int found;
  int64_t g, gp, gt;
  int64_t u, v;
} or_pair;

/* Gain of swapping positions u (segment p) and v (segment t) w.r.t. the pass-start B
 * (reading #14).  Swapping u<->v maps every row i to a row whose count in segment p is
 * c_p(i) + d_i and in t is c_t(i) - d_i, d_i = [B[i][v]!=0] - [B[i][u]!=0]; the row
 * relabelling itself does not change any count.  gp / gt = drop in #violating vectors. */
static void swap_gain(const or_csr* B, int N, int M, int64_t p, int64_t t, int64_t u,
                      int64_t v, int64_t* gp, int64_t* gt) {
  int64_t a = B->rp[u], ae = B->rp[u + 1], b = B->rp[v], be = B->rp[v + 1];
  int64_t sp = 0, st = 0;
  /* merge N(u) and N(v) (B symmetric: column u's rows == row u's columns) */
  while (a < ae || b < be) {
    int64_t i;
    int d;
    if (b >= be || (a < ae && B->ci[a] < B->ci[b])) { i = B->ci[a]; d = -1; ++a; }
    else if (a >= ae || B->ci[b] < B->ci[a]) { i = B->ci[b]; d = +1; ++b; }
    else { ++a; ++b; continue; } /* neighbour of both: d = 0 */
    int cp = seg_count(B, i, p, M), ct = seg_count(B, i, t, M);
    sp += (cp > N) - (cp + d > N);
    st += (ct > N) - (ct - d > N);
  }
  *gp = sp;
  *gt = st;
}

/* freshtop(): the fresh (not yet recorded) pair with the largest gain g = gp + gt; ties ->
 * smallest u, then smallest v (reading #18).  need_positive restricts to g > 0. */
static or_pair freshtop(const or_csr* B, int N, int M, int64_t p, int64_t t, const uint8_t* used,
                        int need_positive) {
  or_pair best = {0, 0, 0, 0, -1, -1};
  int64_t n = B->n;
  for (int64_t u = p * M; u < p * M + M && u < n; ++u) {
    if (used[u]) continue;
    for (int64_t v = t * M; v < t * M + M && v < n; ++v) {
      if (used[v]) continue;
      int64_t gp, gt;
      swap_gain(B, N, M, p, t, u, v, &gp, &gt);
      int64_t g = gp + gt;
      if (need_positive && g <= 0) continue;
      if (!best.found || g > best.g) {
        best.found = 1; best.g = g; best.gp = gp; best.gt = gt; best.u = u; best.v = v;
      }
    }
  }
  return best;
}

typedef struct { int64_t seg; int64_t score; } or_item;

static int cmp_item(const void* a, const void* b) {
  const or_item* x = (const or_item*)a;
  const or_item* y = (const or_item*)b;
  if (x->score != y->score) return x->score > y->score ? -1 : 1; /* PScore descending */
  return (x->seg > y->seg) - (x->seg < y->seg);                  /* then id ascending */
}

static int all_positions_used(const uint8_t* used, int64_t seg, int M, int64_t n) {
  for (int64_t u = seg * M; u < seg * M + M && u < n; ++u)
    if (!used[u]) return 0;
  return 1;
}

/* Scratch of one Stage-2 pass, sized for n vertices / S segments. */
typedef struct {
  int32_t* pscore; int64_t* est; uint8_t* inI; uint8_t* used; or_item* I; int64_t* snap;
} s2_scratch;

/* One Stage-2 pass (Alg. 3 lines 1-23) over the pass-start matrix B: records the swap
 * pairs (u, v) -- and the (primary, target) segments they were chosen for -- in the order
 * Alg. 3 records them.  Returns the number of recorded pairs, or -1 when the pass stops
 * before recording ("I" empty, or a single segment in the whole matrix). */
static int64_t stage2_pass(const or_csr* B, int N, int M, int gain_rule, s2_scratch* w,
                           int64_t* su, int64_t* sv, int64_t* sp, int64_t* st,
                           int64_t* max_pairs_per_primary) {
  int64_t n = B->n, S = (n + M - 1) / M;
  int64_t wv, mbv;
  counts_B(B, 1, N, M, &wv, &mbv, w->pscore);              /* GetPScoreList (line 1/29) */
  int64_t nI = 0;
  for (int64_t s = 0; s < S; ++s)
    if (w->pscore[s] > 0) { w->I[nI].seg = s; w->I[nI].score = w->pscore[s]; ++nI; } /* line 2/30 */
  if (nI == 0) return -1;
  qsort(w->I, (size_t)nI, sizeof(or_item), cmp_item);
  for (int64_t s = 0; s < S; ++s) { w->est[s] = w->pscore[s]; w->inI[s] = 0; }
  for (int64_t k = 0; k < nI; ++k) w->inI[w->I[k].seg] = 1;
  memset(w->used, 0, (size_t)n);
  int64_t nS = 0;
  if (nI == 1) {
    /* line 6: beneficial swaps with the sparsest segment (L402 (ii), reading #16) */
    int64_t p = w->I[0].seg;
    if (S == 1) return -1;
    int64_t t = -1, tn = 0;
    for (int64_t s = 0; s < S; ++s) {
      if (s == p) continue;
      int64_t z = 0;
      for (int64_t q = s * M; q < s * M + M && q < n; ++q) z += B->rp[q + 1] - B->rp[q];
      if (t < 0 || z < tn) { t = s; tn = z; }
    }
    int64_t npairs = 0;
    for (;;) {
      or_pair pr = freshtop(B, N, M, p, t, w->used, 1);
      if (!pr.found) break;
      su[nS] = pr.u; sv[nS] = pr.v; sp[nS] = p; st[nS] = t; ++nS; ++npairs;
      w->used[pr.u] = w->used[pr.v] = 1;
      w->est[p] -= pr.gp;
      if (w->est[p] <= 0 || all_positions_used(w->used, p, M, n)) break;
    }
    if (npairs > *max_pairs_per_primary) *max_pairs_per_primary = npairs;
  } else {
    int64_t head = 0;
    while (1) {
      /* |I| > 1 ?  count live entries from head */
      int64_t live = 0;
      for (int64_t k = head; k < nI; ++k) live += w->inI[w->I[k].seg];
      if (live <= 1) break;
      while (!w->inI[w->I[head].seg]) ++head;
      int64_t p = w->I[head].seg; /* line 9: I.pop() */
      w->inI[p] = 0;
      ++head;
      int64_t ns = 0;
      for (int64_t k = head; k < nI; ++k) if (w->inI[w->I[k].seg]) w->snap[ns++] = w->I[k].seg;
      int64_t npairs = 0;
      for (int64_t k = 0; k < ns; ++k) { /* line 10: targets in priority order */
        int64_t t = w->snap[k];
        if (!w->inI[t]) continue;
        or_pair pr = freshtop(B, N, M, p, t, w->used, gain_rule == 1);
        if (!pr.found) continue;
        su[nS] = pr.u; sv[nS] = pr.v; sp[nS] = p; st[nS] = t; ++nS; ++npairs; /* line 15 */
        w->used[pr.u] = w->used[pr.v] = 1;
        w->est[p] -= pr.gp;                             /* line 16 */
        w->est[t] -= pr.gt;                             /* line 17 */
        if (w->est[t] <= 0) w->inI[t] = 0;              /* lines 18-19 */
        if (w->est[p] <= 0 || all_positions_used(w->used, p, M, n)) break; /* lines 20-22 */
      }
      if (npairs > *max_pairs_per_primary) *max_pairs_per_primary = npairs;
    }
  }
  return nS;
}

static int s2_alloc(int64_t n, int M, s2_scratch* w, int64_t** bufs, int nbufs) {
  int64_t S = (n + M - 1) / M;
  size_t Sz = (size_t)(S > 0 ? S : 1), nz = (size_t)(n > 0 ? n : 1);
  w->pscore = (int32_t*)malloc(sizeof(int32_t) * Sz);
  w->est = (int64_t*)malloc(sizeof(int64_t) * Sz);
  w->inI = (uint8_t*)malloc(Sz);
  w->used = (uint8_t*)malloc(nz);
  w->I = (or_item*)malloc(sizeof(or_item) * Sz);
  w->snap = (int64_t*)malloc(sizeof(int64_t) * Sz);
  for (int k = 0; k < nbufs; ++k) bufs[k] = (int64_t*)malloc(sizeof(int64_t) * nz);
  return 0;
}

static void s2_free(s2_scratch* w, int64_t** bufs, int nbufs) {
  free(w->pscore); free(w->est); free(w->inI); free(w->used); free(w->I); free(w->snap);
  for (int k = 0; k < nbufs; ++k) free(bufs[k]);
}

/* One Stage-2 run (up to MAXITER2+1 passes).  Returns #passes that applied swaps;
 * *max_pairs_per_primary receives the largest number of pairs one primary recorded. */
static int stage2(int64_t n, const int64_t* rp, const int32_t* ci, int N, int M, int maxiter,
                  int gain_rule, int32_t* perm, int64_t* max_pairs_per_primary) {
  s2_scratch w;
  int64_t* b[4];
  s2_alloc(n, M, &w, b, 4);
  int passes = 0;
  for (int it = 0; it <= maxiter; ++it) {
    or_csr B;
    build_B(n, rp, ci, perm, &B);
    int64_t nS = stage2_pass(&B, N, M, gain_rule, &w, b[0], b[1], b[2], b[3], max_pairs_per_primary);
    csr_free(&B);
    if (nS <= 0) break;                 /* nothing recorded: the state is unchanged */
    for (int64_t k = 0; k < nS; ++k) {  /* lines 24-27: apply the recorded swaps together */
      int32_t tmp = perm[b[0][k]];
      perm[b[0][k]] = perm[b[1][k]];
      perm[b[1][k]] = tmp;
    }
    ++passes;
  }
  s2_free(&w, b, 4);
  return passes;
}

/* Trace of ONE Stage-2 pass from perm (for the hand-derived pins, tests/golden/s2_*.txt):
 * pairs_out[4k..4k+3] = (primary segment, target segment, u, v) of the k-th recorded pair
 * (u, v = positions of the pass-start order), in recording order.  pairs_out holds room for
 * n pairs.  Returns the number of pairs, -1 when the pass stops before recording. */
int64_t or_stage2_trace(int64_t n, const int64_t* rp, const int32_t* ci, const int32_t* perm, int N,
                        int M, int gain_rule, int64_t* pairs_out) {
  s2_scratch w;
  int64_t* b[4];
  s2_alloc(n, M, &w, b, 4);
  or_csr B;
  build_B(n, rp, ci, perm, &B);
  int64_t mp = 0;
  int64_t nS = stage2_pass(&B, N, M, gain_rule, &w, b[0], b[1], b[2], b[3], &mp);
  for (int64_t k = 0; k < nS; ++k) {
    pairs_out[4 * k] = b[2][k]; pairs_out[4 * k + 1] = b[3][k];
    pairs_out[4 * k + 2] = b[0][k]; pairs_out[4 * k + 3] = b[1][k];
  }
  csr_free(&B);
  s2_free(&w, b, 4);
  return nS;
}

/* ------------------------------------------------------------------------------------- */
/* Alg. 1 (L248-260): repeat Stage-1, Stage-2 while violations remain                    */
/* ------------------------------------------------------------------------------------- */

typedef struct {
  int max_outer, max_stage1, max_stage2; /* MAXITER = 10 (L496), reading #8 */
  int gain_rule;                         /* 0 = paper (any gain, footnote L440); 1 = positive */
  int keep_best;                         /* reading #17 */
} or_opts;

typedef struct {
  int64_t omega_init, omega_final, mb_init, mb_final;
  int64_t outer_iters, stage1_iters, stage2_passes, max_pairs_per_primary;
} or_stats;

int or_reorder(int64_t n, const int64_t* rp, const int32_t* ci, int V, int N, int M,
               const or_opts* o, int32_t* perm_out, or_stats* st) {
  int32_t* perm = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int32_t* best = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t p = 0; p < n; ++p) perm[p] = (int32_t)p;
  int64_t w, mb;
  or_counts(n, rp, ci, perm, V, N, M, &w, &mb, NULL);
  memset(st, 0, sizeof(*st));
  st->omega_init = w; st->mb_init = mb;
  int64_t best_score = w + mb;
  memcpy(best, perm, sizeof(int32_t) * (size_t)n);
  int64_t it = 0;
  while ((w > 0 || mb > 0) && it <= o->max_outer) {
    /* Stage-1 (Alg. 2): while MBscore > 0 and iter <= MAXITER */
    int64_t mb1 = mb;
    for (int i1 = 0; mb1 > 0 && i1 <= o->max_stage1; ++i1) {
      or_csr B;
      build_B(n, rp, ci, perm, &B);
      stage1_sort(&B, N, M, perm);
      csr_free(&B);
      st->stage1_iters++;
      int64_t w1;
      or_counts(n, rp, ci, perm, V, N, M, &w1, &mb1, NULL);
    }
    st->stage2_passes += stage2(n, rp, ci, N, M, o->max_stage2, o->gain_rule, perm,
                                &st->max_pairs_per_primary);
    ++it;
    or_counts(n, rp, ci, perm, V, N, M, &w, &mb, NULL);
    if (o->keep_best && w + mb < best_score) {
      best_score = w + mb;
      memcpy(best, perm, sizeof(int32_t) * (size_t)n);
    }
  }
  st->outer_iters = it;
  if (o->keep_best) memcpy(perm_out, best, sizeof(int32_t) * (size_t)n);
  else memcpy(perm_out, perm, sizeof(int32_t) * (size_t)n);
  or_counts(n, rp, ci, perm_out, V, N, M, &st->omega_final, &st->mb_final, NULL);
  free(perm); free(best);
  return 0;
}

/* ------------------------------------------------------------------------------------- */
/* Canonical V:N:M packing (reading #19; SPTC form of L492)                                */
/* Panels of Vp rows, segments of Mp columns, k = 4 selected columns per meta-block,       */
/* <= 2 kept values per row (N = 2), 2-bit indices, residual CSR for everything else.      */
/* ------------------------------------------------------------------------------------- */

/* Selected offsets of one meta-block: the 4 offsets with the largest column counts, ties to
 * the smaller offset, returned ascending; Mp == 4 selects {0,1,2,3}. */
static void select4(const int* cnt, int Mp, uint8_t* sel) {
  int chosen[64] = {0};
  if (Mp == 4) { for (int j = 0; j < 4; ++j) sel[j] = (uint8_t)j; return; }
  int picks[4];
  for (int k = 0; k < 4; ++k) {
    int bj = -1;
    for (int j = 0; j < Mp; ++j) {
      if (chosen[j]) continue;
      if (bj < 0 || cnt[j] > cnt[bj]) bj = j;
    }
    chosen[bj] = 1;
    picks[k] = bj;
  }
  /* ascending */
  for (int a = 0; a < 4; ++a)
    for (int b = a + 1; b < 4; ++b)
      if (picks[b] < picks[a]) { int t = picks[a]; picks[a] = picks[b]; picks[b] = t; }
  for (int k = 0; k < 4; ++k) sel[k] = (uint8_t)picks[k];
}

int or_pack_fill(int64_t n, const int64_t* rp, const int32_t* ci, const uint16_t* val16,
                 uint16_t one_bits, const int32_t* perm, int Vp, int Mp, int tau, int64_t* n_mb_out,
                 int64_t* res_nnz_out, int64_t* panel_ptr, int32_t* mb_seg, uint8_t* sel_out,
                 uint8_t* nib_out, uint16_t* vals_out, int64_t* res_rp, int32_t* res_ci,
                 uint16_t* res_val);

/* Counts the packed sizes: number of meta-blocks and residual nonzeros. */
int or_pack_count(int64_t n, const int64_t* rp, const int32_t* ci, const int32_t* perm, int Vp,
                  int Mp, int tau, int64_t* n_mb, int64_t* res_nnz) {
  return or_pack_fill(n, rp, ci, NULL, 0, perm, Vp, Mp, tau, n_mb, res_nnz, NULL, NULL, NULL, NULL,
                      NULL, NULL, NULL, NULL);
}

/* Fills the canonical arrays (any output may be NULL to skip it):
 *   panel_ptr [P+1]       first meta-block of each panel
 *   mb_seg    [n_mb]      segment id of each meta-block (ascending within a panel)
 *   sel       [n_mb*4]    selected offsets
 *   nib       [n_mb*Vp]   per row of the panel: idx0 | idx1<<2
 *   vals      [n_mb*Vp*2] 16-bit value bits of the two slots
 *   res_rp [n+1], res_ci, res_val: residual CSR (new labels, ascending columns)
 * val16 holds the 16-bit bits of A's values (NULL -> one_bits for every entry).
 * tau (hybrid split, reading #27; not in the paper): a meta-block whose rows would
 * keep fewer than tau values in total is not emitted -- all its entries go to the residual.
 * tau = 0 is the plain canonical form. */
int or_pack_fill(int64_t n, const int64_t* rp, const int32_t* ci, const uint16_t* val16,
                 uint16_t one_bits, const int32_t* perm, int Vp, int Mp, int tau, int64_t* n_mb_out,
                 int64_t* res_nnz_out, int64_t* panel_ptr, int32_t* mb_seg, uint8_t* sel_out,
                 uint8_t* nib_out, uint16_t* vals_out, int64_t* res_rp, int32_t* res_ci,
                 uint16_t* res_val) {
  or_csr B;
  build_B(n, rp, ci, perm, &B);
  int64_t P = (n + Vp - 1) / Vp;
  int64_t mbk = 0, rk = 0;
  uint8_t* keep = (uint8_t*)calloc((size_t)(B.rp[n] > 0 ? B.rp[n] : 1), 1); /* 1 = packed */
  if (panel_ptr) panel_ptr[0] = 0;
  for (int64_t r = 0; r < P; ++r) {
    int64_t r0 = r * Vp, r1 = r0 + Vp < n ? r0 + Vp : n;
    /* distinct segments of the panel, ascending */
    int64_t cnt = B.rp[r1] - B.rp[r0];
    int32_t* segs = (int32_t*)malloc(sizeof(int32_t) * (size_t)(cnt > 0 ? cnt : 1));
    for (int64_t k = 0; k < cnt; ++k) segs[k] = B.ci[B.rp[r0] + k] / Mp;
    qsort(segs, (size_t)cnt, sizeof(int32_t), cmp_i32);
    int64_t nseg = 0;
    for (int64_t k = 0; k < cnt; ++k)
      if (k == 0 || segs[k] != segs[k - 1]) segs[nseg++] = segs[k];
    for (int64_t z = 0; z < nseg; ++z) {
      int64_t s = segs[z];
      int colcnt[64] = {0};
      for (int64_t i = r0; i < r1; ++i)
        for (int64_t k = B.rp[i]; k < B.rp[i + 1]; ++k)
          if (B.ci[k] / Mp == s) colcnt[B.ci[k] - s * Mp]++;
      uint8_t sel[4];
      select4(colcnt, Mp, sel);
      if (tau > 0) {
        /* values the block would keep: per row min(2, entries in the selected columns) */
        int64_t kept_total = 0;
        for (int64_t i = r0; i < r1; ++i) {
          int nk = 0;
          for (int j = 0; j < 4; ++j) {
            int64_t col = s * Mp + sel[j];
            if (col >= n) continue;
            for (int64_t k = B.rp[i]; k < B.rp[i + 1]; ++k)
              if (B.ci[k] == col) ++nk;
          }
          kept_total += nk < 2 ? nk : 2;
        }
        if (kept_total < tau) continue; /* whole block -> residual */
      }
      if (mb_seg) mb_seg[mbk] = (int32_t)s;
      if (sel_out) memcpy(sel_out + mbk * 4, sel, 4);
      for (int64_t li = 0; li < Vp; ++li) {
        int64_t i = r0 + li;
        int kept_j[2] = {-1, -1};
        int64_t kept_k[2] = {-1, -1};
        int nk = 0;
        if (i < r1) {
          for (int j = 0; j < 4; ++j) {
            int64_t col = s * Mp + sel[j];
            if (col >= n) continue;
            for (int64_t k = B.rp[i]; k < B.rp[i + 1]; ++k)
              if (B.ci[k] == col) {
                if (nk < 2) { kept_j[nk] = j; kept_k[nk] = k; keep[k] = 1; }
                ++nk;
              }
          }
        }
        uint8_t nb;
        uint16_t v0 = 0, v1 = 0;
#define VAL(k) (val16 ? val16[B.src[k]] : one_bits)
        if (nk >= 2) { nb = (uint8_t)(kept_j[0] | (kept_j[1] << 2)); v0 = VAL(kept_k[0]); v1 = VAL(kept_k[1]); }
        else if (nk == 1 && kept_j[0] < 3) { nb = (uint8_t)(kept_j[0] | (3 << 2)); v0 = VAL(kept_k[0]); }
        else if (nk == 1) { nb = (uint8_t)(0 | (3 << 2)); v1 = VAL(kept_k[0]); }
        else { nb = (uint8_t)(0 | (1 << 2)); }
#undef VAL
        if (nib_out) nib_out[mbk * Vp + li] = nb;
        if (vals_out) { vals_out[(mbk * Vp + li) * 2] = v0; vals_out[(mbk * Vp + li) * 2 + 1] = v1; }
      }
      ++mbk;
    }
    if (panel_ptr) panel_ptr[r + 1] = mbk;
    free(segs);
  }
  /* residual: every entry of B that no slot kept */
  if (res_rp) res_rp[0] = 0;
  for (int64_t i = 0; i < n; ++i) {
    for (int64_t k = B.rp[i]; k < B.rp[i + 1]; ++k) {
      if (keep[k]) continue;
      if (res_ci) res_ci[rk] = B.ci[k];
      if (res_val) res_val[rk] = val16 ? val16[B.src[k]] : one_bits;
      ++rk;
    }
    if (res_rp) res_rp[i + 1] = rk;
  }
  *n_mb_out = mbk;
  *res_nnz_out = rk;
  free(keep);
  csr_free(&B);
  return 0;
}

/* ------------------------------------------------------------------------------------- */
/* fp64 SpMM: the exact result the method reaches, Y = A X (lossless, L128, L560)          */
/* ------------------------------------------------------------------------------------- */

/* Y[i][f] = sum_k val[k] * X[ci[k]][f];  E[i][f] = sum_k |val[k]| * |X[ci[k]][f]|.
 * val NULL -> 1.0.  X row-major with leading dimension ldx, Y/E with F columns.
 * nthreads > 1 parallelises over rows (OpenMP); returns the thread count used. */
int or_spmm_f64(int64_t n_rows, const int64_t* rp, const int32_t* ci, const double* val,
                const double* X, int64_t ldx, int F, double* Y, double* E, int nthreads) {
  int used = 1;
#ifdef _OPENMP
  if (nthreads > 1) {
    omp_set_num_threads(nthreads);
#pragma omp parallel
    {
#pragma omp single
      used = omp_get_num_threads();
    }
  }
#pragma omp parallel for schedule(dynamic, 64) if (nthreads > 1)
#endif
  for (int64_t i = 0; i < n_rows; ++i) {
    double* y = Y + i * F;
    double* e = E ? E + i * F : NULL;
    for (int f = 0; f < F; ++f) { y[f] = 0.0; if (e) e[f] = 0.0; }
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      double a = val ? val[k] : 1.0;
      const double* x = X + (int64_t)ci[k] * ldx;
      for (int f = 0; f < F; ++f) {
        y[f] += a * x[f];
        if (e) e[f] += (a < 0 ? -a : a) * (x[f] < 0 ? -x[f] : x[f]);
      }
    }
  }
  (void)nthreads;
  return used;
}

/* Rows-sampled variant for full-size parity: Y[r] for r in rows[0..nr). */
int or_spmm_rows_f64(int64_t nr, const int64_t* rows, const int64_t* rp, const int32_t* ci,
                     const double* val, const double* X, int64_t ldx, int F, double* Y, double* E) {
  for (int64_t z = 0; z < nr; ++z) {
    int64_t i = rows[z];
    double* y = Y + z * F;
    double* e = E ? E + z * F : NULL;
    for (int f = 0; f < F; ++f) { y[f] = 0.0; if (e) e[f] = 0.0; }
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      double a = val ? val[k] : 1.0;
      const double* x = X + (int64_t)ci[k] * ldx;
      for (int f = 0; f < F; ++f) {
        y[f] += a * x[f];
        if (e) e[f] += (a < 0 ? -a : a) * (x[f] < 0 ? -x[f] : x[f]);
      }
    }
  }
  return 0;
}

/* One Stage-1 sort step (Alg. 2 lines 4-13) applied to perm_in, for the key-order pin. */
int or_stage1_once(int64_t n, const int64_t* rp, const int32_t* ci, const int32_t* perm_in,
                   int N, int M, int32_t* perm_out) {
  or_csr B;
  build_B(n, rp, ci, perm_in, &B);
  memcpy(perm_out, perm_in, sizeof(int32_t) * (size_t)n);
  stage1_sort(&B, N, M, perm_out);
  csr_free(&B);
  return 0;
}
