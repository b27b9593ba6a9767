// C-ABI entry points of libet.so (include/et.h).  Host code only: argument validation, workspace
// carving and kernel launches on the caller's stream.
#include <cuda_runtime.h>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "internal.h"

namespace et {

static thread_local std::string g_err;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
}

et_status fail(et_status s, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

// ---------------------------------------------------------------- tracing
// Device-side trace: every traced launch gets a slot of two u64 in caller memory; thread 0 of each
// CTA folds %globaltimer into slot[0] with atomicMin at its start and ~%globaltimer into slot[1]
// with atomicMin at its end (both start from all-ones), so slot = (first CTA start, last CTA end).
struct Trace {
  bool on = false;
  int capacity = 0, n = 0;
  unsigned long long* slots = nullptr;
  std::vector<int> kind;
};
static thread_local Trace g_trace;
static thread_local long long g_launches = 0;

void count_launch() { ++g_launches; }
void add_launches(long long n) { g_launches += n; }
long long launch_count() { return g_launches; }

unsigned long long* trace_slot(int kind) {
  Trace& t = g_trace;
  if (!t.on || t.n >= t.capacity) return nullptr;
  t.kind[t.n] = kind;
  return t.slots + 2 * (size_t)t.n++;
}

static bool valid_dtype(et_dtype d) { return d == ET_FP16 || d == ET_BF16 || d == ET_FP32; }

static int units_of(int rows, int cols, et_pattern pat, int r, int c) {
  if (pat == ET_PRUNE_TILE) return (rows / r) * (cols / c);
  if (pat == ET_PRUNE_ROW) return rows;
  return cols;
}

static int n_pruned(double ratio, int units) { return (int)std::floor(ratio * (double)units + 0.5); }

}  // namespace et

using namespace et;

extern "C" {

const char* et_last_error(void) { return g_err.c_str(); }
const char* et_version(void) { return "et-b200 0.1 (sm_100a)"; }

et_status et_trace_begin(int32_t capacity, unsigned long long* dev_slots) {
  if (capacity < 1 || !dev_slots) return fail(ET_ERR_INVALID_ARG, "et_trace_begin: capacity < 1 or null slots");
  g_trace.on = true;
  g_trace.capacity = capacity;
  g_trace.n = 0;
  g_trace.slots = dev_slots;
  g_trace.kind.assign(capacity, 0);
  return ET_OK;
}

et_status et_trace_end(int32_t* n_launches) {
  g_trace.on = false;
  if (n_launches) *n_launches = g_trace.n;
  return ET_OK;
}

et_status et_trace_get(int32_t i, int32_t* kind, float* ms) {
  if (i < 0 || i >= g_trace.n || !g_trace.slots) return fail(ET_ERR_INVALID_ARG, "et_trace_get: index out of range");
  if (kind) *kind = g_trace.kind[i];
  if (ms) {
    unsigned long long s[2];
    cudaError_t e = cudaMemcpy(s, g_trace.slots + 2 * (size_t)i, sizeof(s), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return fail(ET_ERR_CUDA, "et_trace_get: %s", cudaGetErrorString(e));
    const unsigned long long t0 = s[0], t1 = ~s[1];
    if (s[0] == ~0ull || s[1] == ~0ull || t1 < t0) return fail(ET_ERR_INVALID_ARG, "et_trace_get: slot %d not written", i);
    *ms = (float)((double)(t1 - t0) * 1e-6);
  }
  return ET_OK;
}

int64_t et_launch_count(void) { return g_launches; }

et_status et_prune_pack_query(int32_t rows, int32_t cols, et_dtype dtype, et_pattern pattern, double ratio,
                              int32_t tile_r, int32_t tile_c, int32_t group_rows, const uint32_t* host_mask_in,
                              int32_t* nnz_out, size_t* mask_bytes, size_t* idx_bytes, size_t* rowptr_bytes,
                              size_t* tilecol_bytes, size_t* rowmap_bytes, size_t* partrowptr_bytes,
                              size_t* values_bytes, size_t* workspace_bytes) {
  if (rows <= 0 || cols <= 0) return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: empty matrix");
  if (!valid_dtype(dtype)) return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: bad dtype");
  if (pattern == ET_PRUNE_NONE) {
    pattern = ET_PRUNE_TILE;
    ratio = 0.0;
  }
  if (pattern != ET_PRUNE_TILE && pattern != ET_PRUNE_ROW && pattern != ET_PRUNE_COL)
    return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: bad pattern");
  if (!(ratio >= 0.0 && ratio <= 1.0)) return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: ratio not in [0,1]");
  if (tile_r <= 0 || tile_c <= 0 || rows % tile_r || cols % tile_c)
    return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: tile %dx%d does not divide %dx%d", tile_r, tile_c, rows,
                cols);
  if (pattern == ET_PRUNE_ROW && group_rows > 0 && rows % group_rows)
    return fail(ET_ERR_INVALID_ARG, "et_prune_pack_query: group_rows must divide rows");
  const int units = units_of(rows, cols, pattern, tile_r, tile_c);
  int nnz = units - n_pruned(ratio, units);
  if (host_mask_in) {
    nnz = 0;
    for (int t = 0; t < units; ++t) nnz += (host_mask_in[t >> 5] >> (t & 31)) & 1u;
  }
  const int groups = pattern == ET_PRUNE_ROW ? (group_rows > 0 ? rows / group_rows : 1) : 1;
  const int q16 = cols / 16;
  int tile_rows_max, tiles_max;
  if (pattern == ET_PRUNE_TILE) {
    tile_rows_max = rows / tile_r;
    tiles_max = units;
  } else if (pattern == ET_PRUNE_ROW) {
    int pr = nnz + 15 * groups;
    const int cap = groups * (((rows / groups) + 15) / 16 * 16);
    if (pr > cap) pr = cap;
    pr = (pr + 15) / 16 * 16;
    tile_rows_max = pr / 16;
    tiles_max = tile_rows_max * q16;
  } else {
    tile_rows_max = 0;
    tiles_max = 0;
  }
  const int kparts = (cols / 16 + 47) / 48;
  if (nnz_out) *nnz_out = nnz;
  if (mask_bytes) *mask_bytes = (size_t)((units + 31) / 32) * 4;
  if (idx_bytes) *idx_bytes = (size_t)(units > 0 ? units : 1) * 4;
  if (rowptr_bytes) *rowptr_bytes = (size_t)(tile_rows_max + 1) * 4;
  if (tilecol_bytes) *tilecol_bytes = (size_t)(tiles_max > 0 ? tiles_max : 1) * 4 + 16;   // +16: aligned bulk reads
  if (rowmap_bytes) *rowmap_bytes = pattern == ET_PRUNE_ROW ? (size_t)tile_rows_max * 16 * 4 : 4;
  if (partrowptr_bytes) *partrowptr_bytes = (size_t)kparts * (tile_rows_max + 1) * 4;
  const bool has_values = tile_r == 16 && tile_c == 16 && pattern != ET_PRUNE_COL && cols % 16 == 0;
  // 16-bit tiles: 512 B in the tcgen05 core-matrix layout; FP32 tiles: 1 KB row-major (simt32.cu)
  if (values_bytes) *values_bytes = has_values ? (size_t)(tiles_max > 0 ? tiles_max : 1) * 256 * dtype_size(dtype) : 0;
  if (workspace_bytes) *workspace_bytes = prune_workspace_bytes(rows, cols, pattern, tile_r, tile_c);
  return ET_OK;
}

et_status et_prune_pack(const void* W_dev, int32_t rows, int32_t cols, et_dtype dtype, et_pattern pattern,
                        double ratio, int32_t tile_r, int32_t tile_c, int32_t group_rows,
                        const uint32_t* mask_in_dev, et_packed_weight* out, void* workspace,
                        size_t workspace_bytes, void* stream) {
  if (!W_dev || !out || !workspace) return fail(ET_ERR_INVALID_ARG, "et_prune_pack: null pointer");
  if (pattern == ET_PRUNE_NONE) {
    pattern = ET_PRUNE_TILE;
    ratio = 0.0;
  }
  ET_TRY(et_prune_pack_query(rows, cols, dtype, pattern, ratio, tile_r, tile_c, group_rows, nullptr, nullptr,
                             nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr));
  if (out->values && !aligned16(out->values)) return fail(ET_ERR_INVALID_ARG, "et_prune_pack: values not 16B aligned");
  if (out->values && (pattern == ET_PRUNE_TILE || pattern == ET_PRUNE_ROW) && (cols % 16 || !aligned16(W_dev)))
    return fail(ET_ERR_INVALID_ARG, "et_prune_pack: W must be 16B aligned with cols % 16 == 0");
  out->pattern = pattern;
  out->dtype = dtype;
  out->rows = rows;
  out->cols = cols;
  out->tile_r = tile_r;
  out->tile_c = tile_c;
  out->group_rows = group_rows;
  PruneArgs a{W_dev, rows, cols, dtype, pattern, tile_r, tile_c, group_rows,
              n_pruned(ratio, units_of(rows, cols, pattern, tile_r, tile_c)), mask_in_dev};
  return prune_pack_run(a, out, workspace, workspace_bytes, static_cast<cudaStream_t>(stream));
}

et_status et_unpack(const et_packed_weight* w, void* dense_out, void* stream) {
  if (!w || !dense_out) return fail(ET_ERR_INVALID_ARG, "et_unpack: null pointer");
  return unpack_run(w, dense_out, static_cast<cudaStream_t>(stream));
}

et_status et_gather_cols(const void* in, int32_t rows, int32_t ld_in, const int32_t* idx_dev, int32_t nk,
                         int32_t nk_pad, et_dtype dtype, void* out, void* stream) {
  if (rows < 0 || nk < 0 || nk_pad < nk || ld_in < 0) return fail(ET_ERR_INVALID_ARG, "et_gather_cols: bad sizes");
  if (!valid_dtype(dtype)) return fail(ET_ERR_INVALID_ARG, "et_gather_cols: bad dtype");
  const int V = dtype == ET_FP32 ? 4 : 8;
  if (nk_pad % V) return fail(ET_ERR_INVALID_ARG, "et_gather_cols: nk_pad must be a multiple of %d", V);
  if (rows == 0 || nk_pad == 0) return ET_OK;
  if (!in || !out || (nk > 0 && !idx_dev)) return fail(ET_ERR_INVALID_ARG, "et_gather_cols: null pointer");
  if (!aligned16(out)) return fail(ET_ERR_INVALID_ARG, "et_gather_cols: out not 16B aligned");
  return gather_cols_run(in, rows, ld_in, idx_dev, nk, nk_pad, dtype, out, static_cast<cudaStream_t>(stream));
}

static et_status segment_from(const et_packed_weight* w, const void* bias, GemmSegment* sg, int out_col) {
  if (!w->values || !w->part_row_ptr || !w->tile_col)
    return fail(ET_ERR_INVALID_ARG, "packed weight has no values / part_row_ptr / tile_col");
  if (w->tile_r != 16 || w->tile_c != 16) return fail(ET_ERR_UNSUPPORTED, "GEMM needs 16x16 tiles");
  if (w->pattern != ET_PRUNE_TILE && w->pattern != ET_PRUNE_ROW)
    return fail(ET_ERR_UNSUPPORTED, "GEMM: pattern %d not supported (column pruning is NEXT-3)", (int)w->pattern);
  sg->row_ptr = w->part_row_ptr;
  sg->tile_col = w->tile_col;
  sg->values = w->values;
  sg->bias = bias;
  sg->tile_rows = (w->pattern == ET_PRUNE_TILE ? w->rows : w->rows_padded) / 16;
  sg->out_col = out_col;
  sg->scale = 1.0f;
  sg->apply_scale = 0;
  return ET_OK;
}

et_status et_linear_fwd(const et_packed_weight* w, const void* X, int32_t M, const void* bias, et_epilogue epi,
                        float scale, int32_t scale_cols, void* Y, void* stream) {
  if (!w || !X || !Y) return fail(ET_ERR_INVALID_ARG, "et_linear_fwd: null pointer");
  if (M < 0) return fail(ET_ERR_INVALID_ARG, "et_linear_fwd: M < 0");
  if (!aligned16(Y)) return fail(ET_ERR_INVALID_ARG, "et_linear_fwd: Y not 16B aligned");
  GemmArgs a{};
  a.X = X;
  a.M = M;
  a.K = w->cols;
  a.ldx = w->cols;
  a.k0 = 0;
  a.dtype = w->dtype;
  a.nseg = 1;
  ET_TRY(segment_from(w, bias, &a.seg[0], 0));
  const int N = a.seg[0].tile_rows * 16;
  if (epi == ET_EPI_BIAS_SCALE) {
    if (scale_cols % 16 != 0 && scale_cols != N)
      return fail(ET_ERR_UNSUPPORTED, "et_linear_fwd: scale_cols must be a multiple of 16");
    // split into two segments sharing the weight: [0, scale_cols) scaled, the rest not
    if (scale_cols > 0 && scale_cols < N) {
      a.seg[1] = a.seg[0];
      a.nseg = 2;
      a.seg[0].tile_rows = scale_cols / 16;
      a.seg[0].apply_scale = 1;
      a.seg[0].scale = scale;
      // the second segment starts at tile row scale_cols/16: offset the row pointer arrays
      a.seg[1].row_ptr = a.seg[0].row_ptr + scale_cols / 16;
      a.seg[1].tile_rows = N / 16 - scale_cols / 16;
      a.seg[1].out_col = scale_cols;
      a.seg[1].bias = bias ? static_cast<const uint8_t*>(bias) + (size_t)scale_cols * dtype_size(w->dtype) : nullptr;
      if (w->kparts > 1) return fail(ET_ERR_UNSUPPORTED, "et_linear_fwd: scaled epilogue with K > 768");
    } else if (scale_cols >= N) {
      a.seg[0].apply_scale = 1;
      a.seg[0].scale = scale;
    }
  }
  a.kpart_tiles = 48;
  a.Y = Y;
  a.ldy = N;
  a.epi = epi;
  return gemm_run(a, static_cast<cudaStream_t>(stream));
}

et_status et_layernorm_fwd(const void* part, et_dtype part_dtype, int32_t nparts, int32_t M, int32_t N,
                           const void* bias, et_dtype dtype, const void* resid, et_dtype resid_dtype,
                           const float* gamma, const float* beta, float eps, void* out_act, void* out_resid,
                           void* stream) {
  if (!part || nparts < 1 || (gamma == nullptr) != (beta == nullptr))
    return fail(ET_ERR_INVALID_ARG, "et_layernorm_fwd: bad arguments");
  LnArgs a{part, nparts, M, N, bias, dtype, resid, resid_dtype, gamma, beta, eps, out_act, out_resid, nullptr,
           part_dtype};
  return layernorm_run(a, static_cast<cudaStream_t>(stream));
}

int32_t et_attn_short_max(int32_t d_k) { return attn_short_max(d_k); }

}  // extern "C"
