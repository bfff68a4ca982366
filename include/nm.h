/*
 * nm.h -- C ABI of libnm, the B200-native (sm_100a) hot path of
 *   Chen, Sung, Zhang, Li, Shen, "Accelerating GNNs on GPU Sparse Tensor Cores through N:M
 *   Sparsity-Oriented Graph Reordering", PPoPP'25   ("PAPER.md:Lxxx" = line of the paper text).
 *
 * The method (§3, §4): reorder the vertices of a graph so that
 * the symmetric adjacency matrix B = P A P^T meets the V:N:M structured-sparsity pattern of
 * sparse tensor cores "as much as possible" (SGRP, L188-199), pack it into the SPTC form
 * (compressed values + 2-bit metadata + per-meta-block column indices, L492), and run the
 * aggregation SpMM Y = B (P X) on sparse tensor cores (L182, L492).  This library adds a
 * residual CSR for whatever still violates the pattern, so the result is always lossless
 * (L128: reordering "does not cause any accuracy loss").
 *
 * Conventions (all entry points):
 *  - Every function returns nm_status; no exception or longjmp crosses the ABI.  On error
 *    the out-parameters are left untouched and nm_last_error() (thread-local) says why.
 *  - perm[p] = old vertex id placed at new position p (the paper's phi' as a list, Alg. 1
 *    output L255).  B[p][q] = A[perm[p]][perm[q]];  (P X)[p] = X[perm[p]]  (Fig. 1 caption
 *    L38: "the corresponding rows in the dense matrix ... must be swapped too").
 *  - Graphs are CSR: rowptr int64[n+1], col int32[nnz], columns sorted ascending, no
 *    duplicates, symmetric pattern (undirected graph, L188), self-loops allowed.
 *  - Ownership: the caller owns every array it passes (graph, perm, X, Y, W, bias) and every
 *    output buffer; the library owns nm_packed (device memory on the device current at pack
 *    time) until nm_packed_free.
 *  - Streams: `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    Device-side calls are stream-ordered and asynchronous unless stated otherwise.
 *  - There is no CPU fallback: without a usable sm_100 device the device entry points
 *    return NM_ERR_CUDA.
 */
#ifndef NM_H_
#define NM_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define NM_API __attribute__((visibility("default")))
#else
#define NM_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  NM_OK = 0,
  NM_ERR_INVALID_ARG = 1,  /* NULL pointer, negative size, bad flag combination            */
  NM_ERR_UNSUPPORTED = 2,  /* V, N, M, F or dtype outside the supported set (see below)     */
  NM_ERR_BAD_CSR = 3,      /* rowptr not monotone, column out of range, unsorted or dup     */
  NM_ERR_NOT_SYMMETRIC = 4,/* pattern of A is not symmetric                                 */
  NM_ERR_CUDA = 5,         /* CUDA runtime/driver error (message in nm_last_error)          */
  NM_ERR_OOM = 6           /* device or host allocation failed                              */
} nm_status;

typedef enum { NM_F16 = 0, NM_BF16 = 1, NM_F32 = 2 } nm_dtype;

/* A square sparse matrix in CSR form.  `val` (length nnz, dtype val_dtype) may be NULL,
 * meaning every stored entry is 1.0 (binary adjacency, L484).  on_device = 1 when the three
 * arrays are device pointers, 0 for host pointers. */
typedef struct {
  int64_t n, nnz;
  const int64_t* rowptr;
  const int32_t* col;
  const void* val;
  nm_dtype val_dtype;
  int on_device;
} nm_csr;

/* Reordering options (Alg. 1-3).  Zero-initialise and set what you need, or pass NULL for
 * the defaults {10, 10, 10, 0, 1}. */
typedef struct {
  int max_outer;   /* Alg. 1 loop cap ("max. iteration", L256; MAXITER = 10, L496)        */
  int max_stage1;  /* Alg. 2 MAXITER (L336)                                                */
  int max_stage2;  /* Alg. 3 MAXITER (L451)                                                */
  int gain_rule;   /* 0 = paper: freshtop() takes the best fresh pair whatever its gain
                      (footnote L440); 1 = only pairs with positive gain                   */
  int keep_best;   /* 1 = return the visited order with the fewest violations (never worse
                      than the input order); 0 = return the last order (literal Alg. 1)    */
} nm_reorder_opts;

typedef struct {
  int64_t omega_init, omega_final; /* #segment vectors violating N:M (omega, L203)         */
  int64_t mb_init, mb_final;       /* #meta-blocks violating the vertical constraint (MBscore, L382) */
  int64_t outer_iters, stage1_iters, stage2_passes;
  int64_t max_pairs_per_primary;   /* <= M by construction (L562-569)                      */
  double seconds;
} nm_reorder_stats;

/* ---------------------------------------------------------------------------------------
 * nm_reorder -- the SGRP heuristic (Alg. 1: repeat Stage-1 (Alg. 2, vertical
 * constraint, Hamming position codes + sort, L366-384) and Stage-2 (Alg. 3, horizontal
 * constraint, greedy pair swaps, L386-422) while violations remain).  Deterministic; the
 * permutation is bit-identical to the CPU oracle's (DESIGN.md §3 readings).
 *   A        : input graph (host or device CSR), symmetric pattern.
 *   V, N, M  : pattern; V >= 1, 1 <= N < M <= 32.
 *   perm_out : host int32[n], caller-allocated; receives perm.
 *   st       : optional statistics.
 * Synchronous.  Errors: INVALID_ARG, UNSUPPORTED (M > 32), BAD_CSR, NOT_SYMMETRIC, OOM, CUDA.
 * ------------------------------------------------------------------------------------- */
NM_API nm_status nm_reorder(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                     int32_t* perm_out, nm_reorder_stats* st);

/* nm_reorder_gpu -- nm_reorder with Stage-1 (Alg. 2 lines 4-13: Hamming position codes of
 * every (row, segment) of B, L339-346 / Listing 1, and the stable lexicographic row
 * sort, L366-384) and the omega / MBscore counts (L203, L382) run on the current CUDA device
 * (the paper's SOGRE is a GPU library, L484).  Stage-2 (Alg. 3) stays on
 * the host: its greedy is sequential in the recorded pairs, and its M x M gain tables are
 * computed in parallel batches with OpenMP (a device version of the tables, bit-identical,
 * is built with -DNM_S2_DEVICE_TABLES=1 but measured slower on B200).  The
 * permutation is bit-identical to nm_reorder's and to the CPU oracle's.
 *   A, V, N, M, opts, perm_out, st : as nm_reorder (A host or device CSR; perm_out host).
 *   stream : cudaStream_t the device work is ordered on (NULL = legacy default stream).
 * Synchronous on return.  Device memory: ~ 60 bytes per stored entry + 60 per vertex, from a
 * private stream-ordered pool created and destroyed by the call (the device's default pool is
 * not touched).  Errors: as nm_reorder, plus CUDA / OOM. */
NM_API nm_status nm_reorder_gpu(const nm_csr* A, int V, int N, int M, const nm_reorder_opts* opts,
                                int32_t* perm_out, nm_reorder_stats* st, void* stream);

/* nm_select_pattern -- the paper's best-V:N:M search (§5): reorder for 1:2:M
 * with M = 4, 8, ... (<= max_M) while the reordered graph conforms (omega = MBscore = 0),
 * then for V:2:M with V = 2, 4, ... (<= max_V, "V going from 1 to 32 in a similar manner")
 * while it conforms.  Returns the last conforming pattern (1:2:4 if none conforms) in
 * *V_out / *M_out, its order in perm_out (host int32[n]) and its statistics.  Synchronous. */
NM_API nm_status nm_select_pattern(const nm_csr* A, int max_M, int max_V, const nm_reorder_opts* opts,
                                   int32_t* perm_out, int* V_out, int* M_out, nm_reorder_stats* st);

/* nm_score_patterns -- best-V:N:M selection scored by the packed form:
 * nm_select_pattern keeps the last pattern the reordered graph CONFORMS to (L496, L655); this
 * scores what the SpMM would move.  For each candidate (V[i], M[i]), N = 2: nm_reorder_gpu with
 * opts, nm_pack_auto for F (Vp auto), score = nm_pack_auto's time model of that pack (ns,
 * DESIGN.md §6).  scores (double[ncand]), n_chunks / residual_nnz (int64[ncand]): host, nullable.
 * *best = index of the lowest score (ties: the earlier candidate), perm_out (host int32[n]) its
 * permutation.  Synchronous.  Errors: as nm_reorder_gpu and nm_pack_hybrid. */
NM_API nm_status nm_score_patterns(const nm_csr* A, int ncand, const int* V, const int* M, int F, nm_dtype dtype,
                                   const nm_reorder_opts* opts, void* stream, double* scores,
                                   int64_t* n_chunks, int64_t* residual_nnz, int* best, int32_t* perm_out);

/* nm_count_violations -- omega (L203), MBscore (L382) and optionally PScore per segment
 * (L396) of B = P A P^T, computed on the GPU.  perm: host int32[n] or NULL (identity).
 * pscore: host int32[ceil(n/M)] or NULL.  Synchronous. */
NM_API nm_status nm_count_violations(const nm_csr* A, const int32_t* perm, int V, int N, int M,
                              int64_t* omega, int64_t* mbscore, int32_t* pscore);

/* ---------------------------------------------------------------------------------------
 * Packed V:N:M matrix (the SPTC form of L492).  Rows of B are grouped in
 * panels of Vp rows (the V-row meta-block height, L194); columns in segments of Mp columns,
 * Mp = 4 when V == 1 (2:4 at
 * V = 1) and Mp = M otherwise; per non-empty (panel, segment) meta-block the k = 4 columns
 * with the most nonzeros are selected (vertical constraint, L226-227) and each row keeps
 * its first <= 2 nonzeros among them (N = 2, horizontal constraint L229-230) as two 16-bit
 * values plus a 4-bit index pair.  Everything else goes to a residual CSR.  Device memory
 * holds the MMA-native image consumed by nm_spmm (tcgen05.mma.sp operands).
 * Supported: N = 2; M in {4, 8, 16}; any V >= 1 (V = 1 -> Mp = 4); Vp in {16, 32, 64, 128}
 * (0 = auto: V when V is 16, 32 or 64, else 128); dtype NM_F16 or NM_BF16 (values are rounded
 * from val_dtype to dtype).  The tensor-core kernel always runs M = 128 MMAs over 128-row
 * kernel panels; at Vp < 128 a kernel panel's chunks hold the meta-blocks of its 128 / Vp
 * canonical panels (in canonical order), each k-group carrying the values of one panel's rows
 * and no-value nibbles in the others, so a V:2:M conforming matrix (V = Vp) packs with an
 * empty residual.
 * ------------------------------------------------------------------------------------- */
typedef struct nm_packed nm_packed;

/* Packs rows [0, n) of B = P A P^T.  perm: host int32[n] (NULL = identity).
 * The call blocks until the pack is complete; the handle is then immutable. */
NM_API nm_status nm_pack(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                  nm_dtype dtype, void* stream, nm_packed** out);

/* Packs only rows [row_begin, row_end) of B (a row shard for multi-GPU runs); row_begin
 * must be a multiple of Vp.  Columns still range over all n vertices. */
NM_API nm_status nm_pack_rows(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                       nm_dtype dtype, int64_t row_begin, int64_t row_end, void* stream,
                       nm_packed** out);

/* General form.  flags:
 *   0                      -- operands in permuted order: nm_spmm reads PX = P X (n rows) and
 *                             writes Yp rows 0..(row_end-row_begin) (rows of B).
 *   NM_PACK_ORIGINAL_ORDER -- the permutation is folded into the operand indices: nm_spmm
 *                             reads X in the ORIGINAL vertex order (gathering row perm[q] for
 *                             column q of B) and writes Y in the original order, row
 *                             perm[p] for each packed row p of B, into an n-row buffer.
 *                             Y = A X for those rows without separate permute/unpermute
 *                             passes (Fig. 1 caption L38 realised inside the SpMM).
 * The canonical export is identical in both modes. */
#define NM_PACK_ORIGINAL_ORDER 1
NM_API nm_status nm_pack_ex(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                            nm_dtype dtype, int64_t row_begin, int64_t row_end, int flags,
                            void* stream, nm_packed** out);

/* nm_pack_hybrid -- nm_pack_ex plus the hybrid split (reading #27; not in the
 * paper, an extension of the lossless residual): meta-blocks are formed and their columns
 * selected exactly as above, then every meta-block whose rows would keep fewer than `tau`
 * values in total (sum over its Vp rows of min(2, entries in its 4 selected columns)) is not
 * emitted and ALL of its entries go to the residual CSR.  tau = 0 is nm_pack_ex (plain
 * canonical form); tau >= 1 never changes Y, only which kernel computes each product.
 * Motivation: with 128-row panels a scattered graph yields meta-blocks that fill ~1 of their
 * 256 value slots, which the CSR path moves with fewer bytes.  Errors as nm_pack_ex, plus
 * INVALID_ARG for tau < 0.  Blocks until the pack is complete. */
NM_API nm_status nm_pack_hybrid(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                                nm_dtype dtype, int64_t row_begin, int64_t row_end, int flags,
                                int tau, void* stream, nm_packed** out);

/* nm_pack_auto -- nm_pack_hybrid at the tau that minimises the library's SpMM time model for F
 * feature columns: the matrix is packed at tau in {0, 2, 4, t/2, t, 3t/2, 2t} (t =
 * nm_hybrid_tau(F)) and each pack scored as n_chunks * (0.28 + 0.0075 F) + residual_nnz *
 * 0.00016 F + residual_items * 0.0024 F (ns; per-chunk, per-value and per-work-item costs
 * fitted to B200 measurements of the two kernels).  The per-item term is what
 * keeps structured (banded) graphs, whose thin blocks scatter over many rows, at tau = 0.
 * The best pack is returned in *out, its tau in *tau_out (nullable); ties keep the smaller
 * tau.  Errors as nm_pack_hybrid.  Blocks until done. */
NM_API nm_status nm_pack_auto(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp, nm_dtype dtype,
                              int64_t row_begin, int64_t row_end, int flags, int F, void* stream,
                              nm_packed** out, int* tau_out);

/* nm_hybrid_tau -- the tau nm_pack_hybrid should use for an SpMM with F feature columns: the
 * break-even number of kept values at which a meta-block's share of a tensor-core chunk costs
 * as much time as the same values in the residual CSR, from a model fitted to B200
 * measurements: ceil((0.28 + 0.0075 F) / (8 * 0.00016 F)), i.e. 8 at F = 128,
 * 7 at F = 256.  Returns 0 for F < 1. */
NM_API int nm_hybrid_tau(int F);

/* Sizes: #meta-blocks, #values kept in MMA slots, #residual nonzeros, device bytes held,
 * #K=32 chunks (8 meta-blocks each, padded per panel).  Any pointer may be NULL. */
NM_API nm_status nm_packed_info(const nm_packed* P, int64_t* n_mb, int64_t* packed_nnz,
                         int64_t* residual_nnz, int64_t* device_bytes, int64_t* n_chunks);

/* All sizes of a packed matrix (superset of nm_packed_info).  image_bytes = the compressed
 * chunk records of the compressed-record kernel, full_image_bytes = the full
 * records of the default kernel (4736 B per K = 32 chunk); residual_items = work items of the
 * residual SpMM (<= 256 nonzeros each), residual_split_rows = rows cut into several. */
typedef struct {
  int64_t n, row_begin, row_end, n_panels /* 128-row kernel panels */, n_mb, n_chunks, packed_nnz, residual_nnz;
  int64_t image_bytes, device_bytes, residual_items, residual_split_rows;
  int32_t V, M, Mp, Vp, tau, flags;
  int64_t full_image_bytes;  /* full MMA-operand records (what the default kernel streams) */
  int64_t gather_rows;       /* X rows the tensor-core part gathers (non-empty selected columns) */
} nm_packed_stat;
NM_API nm_status nm_packed_stats(const nm_packed* P, nm_packed_stat* st);

/* Copies the canonical form back to host arrays (caller-allocated, sizes from
 * nm_packed_info; rows = row_end - row_begin, panels = ceil(rows / Vp)):
 *   panel_ptr int64[panels+1], mb_seg int32[n_mb], sel uint8[n_mb*4] (ascending offsets),
 *   nib uint8[n_mb*Vp] (idx0 | idx1 << 2 per row of the meta-block's panel),
 *   vals uint16[n_mb*Vp*2] (16-bit value bits of the two slots),
 *   res_rowptr int64[rows+1], res_col int32[residual_nnz], res_val uint16[residual_nnz].
 * Any pointer may be NULL to skip that array.  Synchronous. */
NM_API nm_status nm_export_canonical(const nm_packed* P, int64_t* panel_ptr, int32_t* mb_seg,
                              uint8_t* sel, uint8_t* nib, uint16_t* vals, int64_t* res_rowptr,
                              int32_t* res_col, uint16_t* res_val);

NM_API void nm_packed_free(nm_packed* P);

/* ---------------------------------------------------------------------------------------
 * Row permutation of a dense matrix (Fig. 1 caption L38).  Device pointers, row-major,
 * leading dimension ld (elements), F columns, n rows; dtype of X/Y elements.
 *   nm_permute_rows   : PX[p] = X[perm[p]]      (X -> permuted order)
 *   nm_unpermute_rows : Y[perm[p]] = Yp[p]      (permuted order -> original order)
 * perm_dev: device int32[n].  In-place (X == PX) is not allowed. */
NM_API nm_status nm_permute_rows(const void* X, void* PX, const int32_t* perm_dev, int64_t n, int F,
                          int64_t ld, nm_dtype dtype, void* stream);
NM_API nm_status nm_unpermute_rows(const void* Yp, void* Y, const int32_t* perm_dev, int64_t n, int F,
                            int64_t ld, nm_dtype dtype, void* stream);

/* ---------------------------------------------------------------------------------------
 * nm_spmm -- Yp = B[rows of P] * PX on sparse tensor cores (tcgen05.mma.sp.kind::f16,
 * fp32 accumulation in tensor memory) plus the residual CSR (CUDA cores), i.e. exactly
 * (P A P^T)(P X) for the packed rows (the aggregation SpMM of L182, L492).
 *   PX : device, n x F, leading dimension ldx (elements), dtype of the pack, permuted order.
 *        ldx must be a multiple of 8 (16-byte rows) and below 2^31.
 *   Yp : device fp32, (row_end-row_begin) x F, leading dimension ldy; overwritten.
 *   F  : 1 <= F <= 4096.
 * Stream-ordered, asynchronous.  Errors: INVALID_ARG, UNSUPPORTED, CUDA. */
NM_API nm_status nm_spmm(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy,
                  int F, void* stream);

/* Same as nm_spmm, but only the tensor-core part (no residual) or only the residual part
 * (adds into Yp).  For profiling and tests. */
NM_API nm_status nm_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy,
                       int F, void* stream);
NM_API nm_status nm_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                           int64_t ldy, int F, void* stream);

/* nm_spmm_sptc_format -- nm_spmm_sptc with an explicit choice of the tensor-core kernel, for
 * profiling and A/B measurement:
 *   format 0 = the pack's choice (what nm_spmm runs), 1 = full-record kernel (one bulk copy of
 *   the MMA operands per K = 32 chunk, no expansion), 2 = compressed-record kernel (HBM holds
 *   only the non-empty (row, meta-block) slots; loader warps expand them in shared memory).
 * Both compute the same Yp (bitwise: identical operands and MMA order).  Errors as nm_spmm,
 * plus INVALID_ARG for another format. */
NM_API nm_status nm_spmm_sptc_format(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                                     int64_t ldy, int F, int format, void* stream);

/* ---------------------------------------------------------------------------------------
 * nm_gcn_layer -- one GCN layer (Eq. 1): Hout = act(Ahat (H W) + bias).
 *   Ahat : packed normalised adjacency in permuted order (P Ahat P^T, pack flags 0), rows
 *          [row_begin, row_end) of it (a row shard for multi-GPU runs);
 *   H    : device [n x F_in] (all vertices, permuted order), dtype of the pack, ld = F_in;
 *   W    : device [F_in x F_out] same dtype, row-major;  bias: device fp32[F_out] or NULL;
 *   Hout : device [(row_end-row_begin) x F_out] same dtype (the shard's rows).
 *   flags: NM_RELU; order NM_LINEAR_FIRST (default, GCN "aggregates after its linear layer",
 *          L564) / NM_AGG_FIRST / NM_ORDER_AUTO (aggregate first iff F_out > F_in).
 *   ws   : device workspace of at least nm_gcn_workspace_bytes(n, F_in, F_out) bytes.
 * F_in and F_out must be multiples of 8.  The dense products run on cuBLASLt (plain library
 * GEMMs, fp32 accumulation); the aggregation on nm_spmm.  Stream-ordered.
 * ------------------------------------------------------------------------------------- */
#define NM_RELU 1
#define NM_LINEAR_FIRST 0
#define NM_AGG_FIRST 2
#define NM_ORDER_AUTO 4
NM_API size_t nm_gcn_workspace_bytes(int64_t n, int F_in, int F_out);
NM_API nm_status nm_gcn_layer(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                       void* Hout, int F_in, int F_out, int flags, void* ws, size_t ws_bytes,
                       void* stream);

/* nm_gcn_layer_bcast -- nm_gcn_layer whose output rows go straight into n_dst (1..16) buffers:
 * dst is a HOST array of device pointers, each a row-major [* x F_out] buffer of the pack's
 * dtype, 16-byte aligned; the layer's rows [0, row_end-row_begin) are stored at rows
 * [dst_row0, dst_row0 + rows) of every dst[i] by the fused bias + activation + down-convert
 * kernel.  This is the all-gather of the row-sharded multi-GPU GCN (PAPER.md
 * L426) fused into the layer's last kernel: on one node dst[] holds every rank's
 * peer-mapped (NVLink, symmetric-memory) copy of the next layer's operand, so the rows reach
 * each GPU from this kernel's 16-byte stores instead of a separate collective.  The caller
 * orders the ranks (a barrier after the layer, before anyone reads the buffers).  Stream-
 * ordered.  Errors: as nm_gcn_layer, plus INVALID_ARG for a bad destination list. */
NM_API nm_status nm_gcn_layer_bcast(const nm_packed* Ahat, const void* H, const void* W, const float* bias,
                                    void* const* dst, int n_dst, int64_t dst_row0, int F_in, int F_out,
                                    int flags, void* ws, size_t ws_bytes, void* stream);

/* nm_gcn_layer_backward -- gradients of nm_gcn_layer (linear-first or aggregate-first give the
 * same Z = Ahat (H W) + b), SURVEY §8(f) item 4:
 *   dZ = dHout * act'(Z) (ReLU: Hout > 0), db = column sums of dZ, dT = Ahat^T dZ = Ahat dZ
 *   (Ahat symmetric: the reorder keeps the adjacency symmetric, PAPER.md L69-79 / L725, so the
 *   same pack serves the backward aggregation), dW = H^T dT, dH = dT W^T.
 *   Ahat : the whole matrix (row_begin 0, row_end n) packed in permuted order (flags 0).
 *   H    : n x F_in, W : F_in x F_out, Hout / dHout : n x F_out -- device, row-major, dtype of
 *          the pack (16-bit), permuted vertex order.
 *   dH   : n x F_in 16-bit (nullable: skipped), dW : F_in x F_out fp32, db : F_out fp32
 *          (nullable).  dT is rounded to 16-bit once before the two GEMMs (cuBLASLt, fp32
 *          accumulation).
 *   flags: NM_RELU or 0.  ws: nm_gcn_backward_workspace_bytes(n, F_in, F_out) bytes.
 *   Stream-ordered.  Errors: INVALID_ARG, UNSUPPORTED (row shard, fused-order pack, F not a
 *   multiple of 8), CUDA. */
NM_API size_t nm_gcn_backward_workspace_bytes(int64_t n, int F_in, int F_out);
NM_API nm_status nm_gcn_layer_backward(const nm_packed* Ahat, const void* H, const void* W, const void* Hout,
                                       const void* dHout, void* dH, float* dW, float* db, int F_in, int F_out,
                                       int flags, void* ws, size_t ws_bytes, void* stream);

/* ------------------------------------------------------------------------------------- */
/* ---------------------------------------------------------------------------------------
 * The other GNN aggregations the paper evaluates (Table 3 "SGC",
 * "SAGE", "Cheb"), on the same packed SpMM.  All need a pack of ALL rows (row_begin = 0,
 * row_end = n); SAGE and Cheb a pack in permuted order (flags 0).  16-bit operands in the pack
 * dtype, fp32 accumulation.  F_in / F_out multiples of 8.  Stream-ordered.
 *
 * nm_sgc_propagate -- SGC's propagation Y = Ahat^K X (K >= 1 SpMM hops).  X: n x F (ldx,
 *   ldx % 8 == 0), Y: fp32 n x F (ldy); Y16: optional 16-bit copy of Y (ld = ldx) or NULL.  The
 *   operand of hop k+1 is hop k's fp32 result rounded to the pack dtype.  Chains in the pack's
 *   order (original order for NM_PACK_ORIGINAL_ORDER packs).  ws: nm_sgc_workspace_bytes.
 * nm_sage_layer -- GraphSAGE, mean aggregator:
 *   Hout = act([H | Amean H] [W_self; W_neigh] + bias), Amean = the pack of D^-1 A (row-
 *   normalised values, supplied by the caller).  H: n x F_in; W_*: F_in x F_out; bias fp32 or
 *   NULL; Hout: n x F_out.  flags: NM_RELU or 0.  ws: nm_sage_workspace_bytes.
 * nm_cheb_layer -- Chebyshev convolution of order K:
 *   Hout = act(sum_{k<K} T_k W_k + bias), T_0 = H, T_1 = Lhat H, T_k = 2 Lhat T_{k-1} - T_{k-2}
 *   (each T_k rounded to the pack dtype), Lhat = the caller's scaled Laplacian pack (e.g.
 *   -D^-1/2 A D^-1/2 for lambda_max = 2).  W: (K F_in) x F_out, W_0 on top.  ws:
 *   nm_cheb_workspace_bytes.
 * Errors: INVALID_ARG (NULL, sizes, workspace), UNSUPPORTED (row-sharded / fused-order pack,
 * F not a multiple of 8), CUDA. */
NM_API size_t nm_sgc_workspace_bytes(int64_t n, int F);
NM_API nm_status nm_sgc_propagate(const nm_packed* Ahat, const void* X, int64_t ldx, float* Y, int64_t ldy,
                                  void* Y16, int F, int K, void* ws, size_t ws_bytes, void* stream);
NM_API size_t nm_sage_workspace_bytes(int64_t n, int F_in, int F_out);
NM_API nm_status nm_sage_layer(const nm_packed* Amean, const void* H, const void* W_self, const void* W_neigh,
                               const float* bias, void* Hout, int F_in, int F_out, int flags, void* ws,
                               size_t ws_bytes, void* stream);
NM_API size_t nm_cheb_workspace_bytes(int64_t n, int F_in, int F_out, int K);
NM_API nm_status nm_cheb_layer(const nm_packed* Lhat, const void* H, const void* W, const float* bias, void* Hout,
                               int F_in, int F_out, int K, int flags, void* ws, size_t ws_bytes, void* stream);

NM_API const char* nm_status_string(nm_status s);
NM_API const char* nm_last_error(void);   /* thread-local detail of the last failure on this thread */
NM_API int nm_version(void);              /* ABI version, currently 1 */

#ifdef __cplusplus
}
#endif
#endif /* NM_H_ */
