/*
 * et.h — C ABI of the B200-native (sm_100a) hot path of E.T. (Chen et al., SC'21,
 * "E.T.: Re-Thinking Self-Attention for Transformer Models on GPUs"; PAPER.md below).
 *
 * The library computes the forward pass of a post-LN Transformer encoder whose
 * Q/K/V/O and FFN weights are pruned with tensor tiles (§4.2) or
 * rows (line 171, §4.1), with the on-the-fly attention operator (line 99-113, §3.1) in a
 * short- and a long-sequence form (line 133-147, §3.2) and the scale moved before Q.K^T
 * (line 159, §3.3).
 *
 * Conventions (all entry points):
 *   - Every function returns et_status; no exception crosses the ABI.  et_last_error() returns
 *     a thread-local message describing the last failure of the calling thread.
 *   - All arguments are validated before anything is launched.  Launch errors are reported as
 *     ET_ERR_CUDA; asynchronous device faults surface at the caller's next synchronisation.
 *   - Device pointers are plain CUDA device pointers allocated BY THE CALLER (the library never
 *     allocates device memory).  Work is enqueued on the caller's stream; nothing synchronises
 *     the device except et_prune_pack (documented below).  The forward entry points are
 *     CUDA-graph capturable.
 *   - Matrices are row-major.  Weights are [out, in]; Y = X . W^T (§2.1).
 *   - Activations X / out are [batch * seq_len, d_model]; token t = b * seq_len + s.
 *   - Tensor-core operands must be 16-byte aligned (TMA); ET_ERR_INVALID_ARG otherwise.
 *   - Thread-safe and reentrant: no mutable global state beyond the error string and a
 *     lazily-initialised, read-only kernel attribute cache.
 */
#ifndef ET_H_
#define ET_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  ET_OK = 0,
  ET_ERR_INVALID_ARG = 1,  /* bad shape / pointer / enum / alignment */
  ET_ERR_UNSUPPORTED = 2,  /* valid request this build does not implement (message says which) */
  ET_ERR_WORKSPACE = 3,    /* workspace too small (query the *_workspace_size function) */
  ET_ERR_CUDA = 4,         /* a CUDA runtime / launch error */
  ET_ERR_NCCL = 5,         /* reserved for the head-parallel collective */
  ET_ERR_INTERNAL = 6
} et_status;

/* Storage dtypes.  FP16 / BF16: the tcgen05 tensor-core path (FP32 accumulation, reading C-9).
 * FP32: the validation build (BASELINE configs[0]): every step in FP32 FMA on the CUDA cores
 * (the 1e-5 gate; one-pass TF32 tensor-core math misses it), packed FP32 tiles row-major, 1 KB. */
typedef enum { ET_FP16 = 0, ET_BF16 = 1, ET_FP32 = 2 } et_dtype;

/* Pruning patterns (§4.1-4.2; attention-aware assignment line 107, 317). */
typedef enum { ET_PRUNE_NONE = 0, ET_PRUNE_TILE = 1, ET_PRUNE_ROW = 2, ET_PRUNE_COL = 3 } et_pattern;

/* Attention operator form (§3.2, switch at a length threshold line 244).
 * ET_ATTN_SHORT_GENERIC: the short form through its generic kernel even where the specialised
 * S <= 128, d_k = 64 kernel applies (test hook: both kernels are checked against the oracle). */
typedef enum { ET_ATTN_AUTO = 0, ET_ATTN_SHORT = 1, ET_ATTN_LONG = 2, ET_ATTN_SHORT_GENERIC = 3 } et_attn_mode;

/* FFN activation ("an activation layer"; GELU(erf) for BERT, ReLU otherwise). */
typedef enum { ET_ACT_GELU_ERF = 0, ET_ACT_RELU = 1 } et_act;

const char* et_last_error(void);
const char* et_version(void);

/* ------------------------------------------------------------------------------------------
 * Packed pruned weight.  Produced by et_prune_pack; consumed by the forward entry points.
 * All pointer fields are device memory allocated by the caller with the sizes returned by
 * et_prune_pack_query.  Fields:
 *   pattern, dtype, rows (= out), cols (= in), tile_r, tile_c       as requested
 *   group_rows   ROW only: rows are padded per group of group_rows original rows (one attention
 *                head: d_k) to a multiple of 16 so that every head's V width is MMA-aligned
 *                (reading C-5); 0 = one group.
 *   nnz          kept units: tiles (TILE) / rows (ROW) / columns (COL); filled by et_prune_pack
 *   rows_padded  ROW: packed row count (sum over groups of round_up(kept_g, 16)); TILE: rows
 *   mask         bitmap over units, ceil(T/32) uint32 words, unit t at bit t%32 of word t/32,
 *                1 = kept.  TILE: t = i*(cols/tile_c) + j.  ROW: t = row.  BIT-EXACT contract.
 *   idx          TILE: CSR col_idx[nnz] (ascending within each tile row).  ROW/COL: kept
 *                row/column indices [nnz], ascending.  BIT-EXACT contract.
 *   row_ptr      TILE: CSR row_ptr[rows/tile_r + 1] (BIT-EXACT contract).  ROW: the uniform
 *                tile CSR of the dense packed matrix [rows_padded/16 + 1].
 *   tile_col     tile column of every packed tile, in values order [ntiles].
 *   row_map      ROW: [rows_padded] original row of each packed row, -1 for padding.  TILE: unused.
 *   kparts       number of K parts of at most 768 columns (48 tile columns) each: ceil(cols/768).
 *   part_row_ptr [kparts][tile_rows + 1]: packed tiles of K part z and tile row i are
 *                values[part_row_ptr[z][i] .. part_row_ptr[z][i+1]) (for kparts == 1 this is the
 *                CSR row_ptr).  Lets split-K GEMM CTAs stream their tiles contiguously.
 *   values       the kept 16x16 tiles in (K part, tile row, tile column) order, each 512 bytes (16-bit dtypes) in the
 *                tcgen05 K-major no-swizzle core-matrix layout: element (n, k) of a tile at byte
 *                (n/8)*256 + (k/8)*128 + (n%8)*16 + (k%8)*2.  Only for tile_r = tile_c = 16 and
 *                FP16/BF16; may be NULL otherwise (mask / index only).
 * ------------------------------------------------------------------------------------------ */
typedef struct {
  et_pattern pattern;
  et_dtype dtype;
  int32_t rows, cols, tile_r, tile_c, group_rows;
  int32_t nnz;
  int32_t rows_padded;
  int32_t ntiles;   /* number of packed tiles (TILE: nnz; ROW: rows_padded/16 * cols/16) */
  int32_t kparts;
  uint32_t* mask;
  int32_t* idx;
  int32_t* row_ptr;
  int32_t* tile_col;     /* in values order */
  int32_t* row_map;
  int32_t* part_row_ptr;
  void* values;
} et_packed_weight;

/* Host-only size query (no CUDA call).  Returns worst-case buffer sizes for et_prune_pack.
 *   ratio in [0, 1]; n_prune = floor(ratio * T + 0.5) units are pruned (reading C-2).
 *   rows % tile_r == 0 and cols % tile_c == 0 required (TILE), else ET_ERR_INVALID_ARG.
 *   nnz_out: exact kept count (= T - n_prune, or popcount of mask_in when host_mask_in given).
 * Any output pointer may be NULL. */
et_status et_prune_pack_query(int32_t rows, int32_t cols, et_dtype dtype, et_pattern pattern, double ratio,
                              int32_t tile_r, int32_t tile_c, int32_t group_rows, const uint32_t* host_mask_in,
                              int32_t* nnz_out, size_t* mask_bytes, size_t* idx_bytes, size_t* rowptr_bytes,
                              size_t* tilecol_bytes, size_t* rowmap_bytes, size_t* partrowptr_bytes,
                              size_t* values_bytes, size_t* workspace_bytes);

/* Prune and pack one weight matrix (§4.2 step (v) 1-4; line 171 §4.1):
 * squared l2 norm per unit accumulated in FP64 in a fixed order (tile: a outer, b inner),
 * rank by (score, linear index), prune the lowest n_prune, emit mask / index / packed values.
 *   W_dev        device [rows, cols] in dtype
 *   mask_in_dev  optional device bitmap (same format as out->mask) fixing the kept set
 *   out          caller-filled buffers (sizes from the query); on return out->nnz,
 *                out->rows_padded and out->ntiles are set.
 * Deterministic.  SYNCHRONISES `stream` before returning (it is an offline, once-per-weight
 * step; the counts are needed on the host). */
et_status et_prune_pack(const void* W_dev, int32_t rows, int32_t cols, et_dtype dtype, et_pattern pattern,
                        double ratio, int32_t tile_r, int32_t tile_c, int32_t group_rows,
                        const uint32_t* mask_in_dev, et_packed_weight* out, void* workspace,
                        size_t workspace_bytes, void* stream);

/* Expand a packed weight back to a dense [rows, cols] matrix W' = mask (.) W (test hook; used
 * to check values bit-exactly).  dense_out: device [rows, cols] in the packed dtype. */
et_status et_unpack(const et_packed_weight* w, void* dense_out, void* stream);

/* Column gather for column pruning with X_adjusted (§4.1, Fig. 5(b)):
 *   out[r, j] = in[r * ld_in + idx[j]]   for j < nk;   out[r, j] = 0 for nk <= j < nk_pad
 * The column-pruned linear layer is X_adjusted . W_pruned^T: gather the kept columns of W once
 * (W_pruned = condensed [rows, nk_pad] weight, then packed as a dense tile weight with ratio 0) and
 * the kept columns of X per call (X_adjusted [M, nk_pad]); padded columns are zero on both sides,
 * so the product is exact.  idx_dev: device int32 [nk], the kept column indices (out->idx of an
 * ET_PRUNE_COL et_prune_pack, ascending).  in: device [rows, ld_in]; out: device [rows, nk_pad],
 * 16-byte aligned; dtype FP16/BF16 (bits moved as-is) or FP32.  nk_pad % 8 == 0 (FP32: % 4 == 0)
 * else ET_ERR_INVALID_ARG; idx values outside [0, ld_in) are undefined behaviour.  Stream-ordered,
 * graph capturable, no allocation. */
et_status et_gather_cols(const void* in, int32_t rows, int32_t ld_in, const int32_t* idx_dev, int32_t nk,
                         int32_t nk_pad, et_dtype dtype, void* out, void* stream);

/* ------------------------------------------------------------------------------------------
 * Tile-sparse linear layer (test hook + building block):
 *   Y[M, N] = epilogue(X[M, K] . W'^T + b)         N = w->rows (ROW: rows_padded), K = w->cols
 * Skips pruned tiles (one tcgen05.mma per kept 16x16 tile).  epilogue:
 *   ET_EPI_BIAS        Y = acc + b                              (out dtype = X dtype)
 *   ET_EPI_BIAS_SCALE  Y = (acc + b) * scale for columns < scale_cols, acc + b otherwise
 *                      (the 1/sqrt(d_k) of Q moved before Q.K^T, line 159 §3.3)
 *   ET_EPI_BIAS_GELU / ET_EPI_BIAS_RELU  Y = act(acc + b)
 *   ET_EPI_F32         Y = acc (fp32, no bias) — partial sums for a LayerNorm epilogue
 *   ET_EPI_PART16      Y = acc rounded to X's dtype (no bias) — 16-bit partial sums (FP16 path)
 * ET_EPI_F32 / ET_EPI_PART16 with K > 768: Y is [ceil(K/768)][M, N], one split-K partial per plane.
 * X: [M, K] fp16/bf16, M % 128 == 0 not required (rows are masked).  b: [N] in X's dtype or NULL. */
typedef enum { ET_EPI_BIAS = 0, ET_EPI_BIAS_SCALE = 1, ET_EPI_BIAS_GELU = 2, ET_EPI_BIAS_RELU = 3, ET_EPI_F32 = 4,
               ET_EPI_PART16 = 5 } et_epilogue;

et_status et_linear_fwd(const et_packed_weight* w, const void* X, int32_t M, const void* bias, et_epilogue epi,
                        float scale, int32_t scale_cols, void* Y, void* stream);

/* Residual + LayerNorm: out = LN(sum_p part[p] + bias + resid) * gamma + beta
 *   part: nparts x [M, N] in part_dtype (FP32, or dtype for 16-bit partials); bias [N] (dtype) or NULL; resid [M, N] in resid_dtype or NULL;
 *   gamma/beta fp32 [N]; out_act [M, N] in act_dtype (GEMM operand copy) and/or out_resid
 *   [M, N] in resid_dtype (either may be NULL).  Biased variance (reading C-11). */
et_status et_layernorm_fwd(const void* part, et_dtype part_dtype, int32_t nparts, int32_t M, int32_t N,
                           const void* bias, et_dtype dtype, const void* resid, et_dtype resid_dtype,
                           const float* gamma, const float* beta, float eps, void* out_act, void* out_resid,
                           void* stream);

/* ------------------------------------------------------------------------------------------
 * Attention descriptor.
 *   batch, seq_len, heads, d_model   problem statement (d_k = d_model / H)
 *   dtype        storage dtype of activations and weights (FP16 / BF16; FP32 = validation build)
 *   lengths_dev  device int32 [batch], valid length per sequence, 1 <= len <= seq_len; keys
 *                j >= len are masked (probability exactly 0, line 73; reading C-7).  NULL = all.
 *   causal       nonzero: also mask j > i (the triangular mask of line 73)
 *   mode         short / long / auto (auto: short while seq_len <= et_attn_short_max())
 *   head_begin, head_end   head range computed by this call ([0, H) normally; a sub-range
 *                [h0, h1) in head-parallel mode, see et_attention_fwd (Eq. 4).
 * ------------------------------------------------------------------------------------------ */
typedef struct {
  int32_t batch, seq_len, heads, d_model;
  et_dtype dtype;
  const int32_t* lengths_dev;
  int32_t causal;
  et_attn_mode mode;
  int32_t head_begin, head_end;
} et_attn_desc;

/* Largest seq_len served by the short (score row resident in TMEM) form. */
int32_t et_attn_short_max(int32_t d_k);

/* Attention core (steps 2-6 of Fig. 3(a)):
 *   Z_h = softmax(mask(Q_h . K_h^T * scale)) . V_h      for h in [head_begin, head_end)
 * qkv: [batch*seq_len, ld_qkv] (16-byte aligned rows) holding Q_h at column q_off + h*d_k and K_h at
 * k_off + h*d_k.  V_h starts at column v_off + v_col[h] and is v_width[h] wide (device int32 [H];
 * NULL => v_col[h] = h*d_k, v_width[h] = d_k); v_width_max bounds v_width (multiple of 16, <= d_k).
 * `scale` multiplies the scores: pass 1 when Q was already scaled by 1/sqrt(d_k) (the reordering
 * of line 159, §3.3).  Z: [batch*seq_len, ld_z]; head h's column c goes to Z column h*d_k + c, or
 * to z_map[v_col[h] + c] when z_map (device int32 over the packed V columns, -1 = skip) is given
 * (row-pruned W_V, line 171).  Rows >= len_b of a sequence are computed like any other query.
 * The seq x seq score matrix never leaves TMEM / registers. */
et_status et_attn_core_fwd(const et_attn_desc* desc, const void* qkv, int32_t ld_qkv, int32_t q_off, int32_t k_off,
                           int32_t v_off, const int32_t* v_col, const int32_t* v_width, int32_t v_width_max,
                           float scale, void* Z, int32_t ld_z, const int32_t* z_map, void* stream);

/* Paper-literal partial on-the-fly attention (§3.2 "partial OTF", Fig. 8 line
 * 236; the switch at sequence length 224, line 244) — the design the fused short / long forms of
 * et_attn_core_fwd replace, kept to measure that trade-off on B200:
 *   kernel A   S_h = Q_h . K_h^T for h in [head_begin, head_end), written to `scores` as 16-bit
 *              (desc->dtype; the paper's pure FP16, line 157-159 — pass Q pre-scaled by 1/sqrt(d_k));
 *   kernel B   per query row i: mask (keys j >= len_b; j > i if causal), softmax(scale * S_h[i, :])
 *              two-pass exact over the stored row, P rounded to 16 bit, Z_h[i] = (P . V_h) / rowsum.
 * qkv, q_off, k_off, v_off, Z, ld_z: as et_attn_core_fwd with dense V (v_col = v_width = z_map = NULL):
 * head h reads columns q_off + h*d_k ..., writes Z columns (h - head_begin)*d_k ....
 * Requirements: dtype FP16 / BF16, d_k 64 or 128, seq_len % 8 == 0, 16-byte aligned qkv / Z rows
 * (ET_ERR_UNSUPPORTED / ET_ERR_INVALID_ARG otherwise).
 * scores: caller-owned device buffer of et_attn_partial_scores_bytes() bytes, 16-byte aligned,
 * layout [batch][head_end - head_begin][seq_len][round_up(seq_len, 8)] 16-bit; score blocks of keys
 * >= len_b (and above the diagonal when causal) are not written.  ET_ERR_WORKSPACE if too small.
 * Two launches on `stream`, graph capturable, no allocation. */
et_status et_attn_partial_scores_bytes(const et_attn_desc* desc, size_t* bytes);
et_status et_attn_partial_fwd(const et_attn_desc* desc, const void* qkv, int32_t ld_qkv, int32_t q_off,
                              int32_t k_off, int32_t v_off, float scale, void* Z, int32_t ld_z, void* scores,
                              size_t scores_bytes, void* stream);

/* Self-attention block (Fig. 3(a) steps 1-7, Eq. 3-4):
 *   out = SelfAttn(X)                  if ln_gamma == NULL
 *   out = LN(X + SelfAttn(X))          otherwise (post-LN, line 75)
 * wq, wk, wo: TILE (or NONE packed as all-kept TILE); wv: TILE or ROW (attention-aware,
 * line 107/317).  Biases in dtype; ln params fp32.  X, out: [batch*seq_len, d_model] in dtype.
 *
 * Head-parallel mode (desc->head_begin/head_end = [h0, h1) != [0, H); Megatron-style split of
 * Eq. 4: Output = sum_h Z_h . W_O,h^T, so each rank computes the sum over its heads and
 * an all-reduce(sum) over ranks gives the full output).  The weights are either
 *   (a) the FULL packed matrices (wq->rows == d_model): the library projects only the range's tile
 *       rows of W_Q / W_K / W_V (a ROW-pruned W_V is projected whole; its per-head packed windows
 *       are located on the device) and runs W_O over a full-width Z that is zero outside the range;
 *       h0*d_k and (h1-h0)*d_k must be multiples of 16 (ET_ERR_UNSUPPORTED otherwise); or
 *   (b) the caller's slices: wq, wk, wv the rank's ROW slices [(h1-h0)*d_k, d_model] of the full
 *       matrices (rows h0*d_k ..), wo its COLUMN slice [d_model, (h1-h0)*d_k] (columns h0*d_k ..),
 *       each packed with mask_in = the full matrix's mask restricted to the slice, so the kept set
 *       is the one the whole-matrix ranking chose (pruning is per matrix, C-3); bq, bk, bv the
 *       matching slices of the biases;
 *   bo          the full [d_model] bias in both cases;
 *   ln_gamma    must be NULL (residual + LN follow the all-reduce: et_layernorm_fwd);
 *   out         FP32 [batch*seq_len, d_model] (reading C-21: FP32 partials) =
 *               sum_{h in [h0,h1)} Z_h W_O,h^T  + b_O (only if h0 == 0)
 *               + sum over this rank's pruned V features f of W_O[:, f] b_V[f] (ROW W_V, C-6).
 * Errors: ET_ERR_INVALID_ARG for slice shapes that do not match the range or a non-NULL gamma. */
et_status et_attention_workspace_size(const et_attn_desc* desc, const et_packed_weight* wv, size_t* bytes);
et_status et_attention_fwd(const et_attn_desc* desc, const void* X, const et_packed_weight* wq,
                           const et_packed_weight* wk, const et_packed_weight* wv, const et_packed_weight* wo,
                           const void* bq, const void* bk, const void* bv, const void* bo, const float* ln_gamma,
                           const float* ln_beta, float ln_eps, void* out, void* workspace, size_t ws_bytes,
                           void* stream);

/* ------------------------------------------------------------------------------------------
 * Pre-computed linear transformation operator (§3.1 Eq. 4-5, Fig. 3(b)):
 *   Output = sum_h S_h . X . (W_V,h^T . W_O,h^T) + b'
 * with the pattern the paper pairs with it (line 107, 317): W_Q / W_K tile-pruned, W_O ROW-pruned
 * (kept output features `kept`, ascending, n_kept of them), W_V dense.
 *
 * et_precompute_vo (offline, once per layer; line 129): Wvo_out device [heads*Dv, d_model] in dtype,
 *   Dv = round_up(n_kept, 16): row h*Dv + j (j < n_kept) = sum_f W_O[kept[j], h*d_k + f] W_V[h*d_k + f, :]
 *   (FP32 accumulation of the stored values, rounded once), rows j >= n_kept zero;
 *   bias_out (optional) device [d_model]: b'[o] = b_O[o] + sum_f W_O[o, f] b_V[f] for kept o, b_O[o]
 *   otherwise (S_h rows sum to 1, so b_V passes through W_O unchanged; reading C-6).
 *   Wv, Wo: dense device [d_model, d_model]; bv, bo: [d_model] or NULL.  Pack Wvo_out with
 *   et_prune_pack(ET_PRUNE_TILE, ratio 0) for et_attention_pre_fwd.
 * et_attention_pre_fwd: out = SelfAttn(X) (ln_gamma NULL) or LN(X + SelfAttn(X)), X / out [M, d] in
 *   desc->dtype; wq, wk TILE packed [d, d]; wvo the packed Wvo_out; bq, bk [d]; bias_fold = b'.
 *   The head sum runs on the tensor core inside the attention kernel (heads of a group accumulate in
 *   one TMEM accumulator); groups of heads leave partial planes that the LayerNorm step adds.
 *   Full head range, FP16 / BF16, d_k 64 or 128, seq_len <= 128, d_model <= 4096 (ET_ERR_UNSUPPORTED
 *   otherwise).  Workspace from et_attention_pre_workspace_size.  Stream-ordered, capturable. */
et_status et_precompute_vo(const void* Wv, const void* Wo, const void* bv, const void* bo, const int32_t* kept_dev,
                           int32_t n_kept, int32_t heads, int32_t d_model, et_dtype dtype, void* Wvo_out,
                           void* bias_out, void* stream);
et_status et_attention_pre_workspace_size(const et_attn_desc* desc, int32_t n_kept, size_t* bytes);
et_status et_attention_pre_fwd(const et_attn_desc* desc, const void* X, const et_packed_weight* wq,
                               const et_packed_weight* wk, const et_packed_weight* wvo, const int32_t* kept_dev,
                               int32_t n_kept, const void* bq, const void* bk, const void* bias_fold,
                               const float* ln_gamma, const float* ln_beta, float ln_eps, void* out, void* workspace,
                               size_t ws_bytes, void* stream);

/* One encoder layer's parameters.  Weights packed; biases in the storage dtype; LN fp32.
 * Attention-aware layers (row-pruned W_V, PAPER.md line 107 / 317) may carry the layer data that
 * depends only on the weights, computed once by et_vprep: v_col / v_width [heads] (each head's packed
 * V columns), bv_packed [wv.rows_padded] (b_V of the kept rows, 0 in padding rows) and bo_folded [d]
 * (b_O' = b_O + sum over pruned V features f of W_O'[:, f] b_V[f], reading C-6), all device memory
 * in the storage dtype (int32 for the column tables).  All four NULL (or a tile-pruned W_V): the
 * forward computes them on its stream every call (three extra launches per layer). */
typedef struct {
  et_packed_weight wq, wk, wv, wo, w1, w2;
  const void *bq, *bk, *bv, *bo, *b1, *b2;
  const float *ln1_g, *ln1_b, *ln2_g, *ln2_b;
  const int32_t *v_col, *v_width;
  const void *bv_packed, *bo_folded;
} et_layer;

/* et_vprep: the attention-aware layer data of et_layer (above) for a row-pruned W_V (packed with
 * group_rows = d_model / heads) and its W_O; bv / bo [d] in dtype (bo may be NULL: b_O' is then the
 * fold alone).  Outputs caller-allocated device memory: v_col, v_width [heads] int32, bv_packed
 * [wv->rows_padded] and bo_folded [d_model] in dtype.  Stream-ordered; ET_ERR_INVALID_ARG for a
 * tile-pruned W_V or mismatched shapes. */
et_status et_vprep(const et_packed_weight* wv, const et_packed_weight* wo, const void* bv, const void* bo,
                   int32_t heads, int32_t d_model, et_dtype dtype, int32_t* v_col, int32_t* v_width,
                   void* bv_packed, void* bo_folded, void* stream);

/* Post-LN encoder stack:  for each layer:
 *   Y1 = LN(X + SelfAttn(X));  U = act(Y1 W1'^T + b1);  Y2 = LN(Y1 + U W2'^T + b2).
 * X, out: [batch*seq_len, d_model] in resid_dtype (FP32, or equal to desc->dtype; reading C-22);
 * GEMM operands in desc->dtype.  layers_host: host array of num_layers et_layer.  X and out
 * may alias.  No host synchronisation; CUDA-graph capturable.  Full head range only
 * (ET_ERR_UNSUPPORTED otherwise): a head-parallel layer is et_attention_fwd on the rank's head range
 * (full weights or the rank's slices), an all-reduce of the FP32 partials by the caller's process
 * group, then et_layernorm_fwd. */
et_status et_encoder_workspace_size(const et_attn_desc* desc, int32_t num_layers, int32_t d_ff,
                                    et_dtype resid_dtype, const et_layer* layers_host, size_t* bytes);
et_status et_encoder_fwd(const et_attn_desc* desc, int32_t num_layers, int32_t d_ff, et_act act, float ln_eps,
                         et_dtype resid_dtype, const et_layer* layers_host, const void* X, void* out,
                         void* workspace, size_t ws_bytes, void* stream);

/* CUDA-graph plan of one et_encoder_fwd call (the paper's model is a fixed stack of layers run
 * again and again on new inputs of the same shape): the whole forward
 * (12 layers x 7 kernels for BERT-base) is captured once and replayed with one launch, removing
 * the host-side launch cost that otherwise exceeds the device time at small batches.
 *   et_encoder_graph_create: same arguments as et_encoder_fwd; captures on a private stream
 *     (thread-local capture mode) and instantiates.  Every pointer (X, out, workspace, the layers'
 *     device buffers, desc->lengths_dev) is baked into the graph: later launches read and write
 *     the same addresses, so the caller keeps them alive and refills X in place.  If tracing is
 *     enabled (et_trace_begin) during creation, the trace events are captured too and every
 *     launch re-records them (et_trace_get then reports the most recent launch).
 *   et_graph_launch: enqueue one replay on `stream`.
 *   et_graph_destroy: free the host-side graph objects (NULL is allowed).
 * Errors: the et_encoder_fwd validation errors; ET_ERR_CUDA if capture or instantiation fails. */
typedef struct et_graph et_graph;
et_status et_encoder_graph_create(const et_attn_desc* desc, int32_t num_layers, int32_t d_ff, et_act act,
                                  float ln_eps, et_dtype resid_dtype, const et_layer* layers_host, const void* X,
                                  void* out, void* workspace, size_t ws_bytes, et_graph** graph);
et_status et_graph_launch(et_graph* graph, void* stream);
et_status et_graph_destroy(et_graph* graph);

/* ------------------------------------------------------------------------------------------
 * Tracing (calling thread only; diagnostics, not part of the metric): while enabled, every kernel
 * the forward entry points launch (or capture into a graph) is given one slot of two uint64 in
 * `dev_slots` (caller-allocated device memory, 2 * capacity entries).  Thread 0 of each CTA of
 * that kernel folds %globaltimer (ns) into slot[0] with atomicMin when it starts and
 * ~%globaltimer into slot[1] with atomicMin when it ends, so the caller must fill the slots with
 * all-one bytes (e.g. cudaMemsetAsync(dev_slots, 0xFF, ...)) before every traced run.  The slot
 * then holds the kernel's device span: first CTA start to last CTA end.  Launches beyond
 * `capacity` are not traced.
 * ------------------------------------------------------------------------------------------ */
typedef enum {
  ET_K_QKV = 0, ET_K_ATTN = 1, ET_K_OPROJ = 2, ET_K_LN1 = 3, ET_K_FFN1 = 4, ET_K_FFN2 = 5, ET_K_LN2 = 6,
  ET_K_AUX = 7
} et_kernel_kind;
et_status et_trace_begin(int32_t capacity, unsigned long long* dev_slots);
/* Stop assigning slots; *n_launches = number of traced launches. */
et_status et_trace_end(int32_t* n_launches);
/* Traced launch i (after synchronising the stream): its kind and device milliseconds (reads the
 * slot with a synchronous cudaMemcpy).  ET_ERR_INVALID_ARG if i is out of range or unwritten. */
et_status et_trace_get(int32_t i, int32_t* kind, float* ms);
/* Number of library kernels launched by this thread since process start (launch accounting). */
int64_t et_launch_count(void);

/* Diagnostics (tcgen05 / TMA probes, profiles/r01/M1_tcgen05_probe.md, profiles/r02/) live in a
 * separate libet_diag.so built from paper_conf_sc_chenhplg0d021_b200/diag/ (not part of this ABI). */

#ifdef __cplusplus
}
#endif
#endif /* ET_H_ */
