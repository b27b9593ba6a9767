// Internal host-side declarations shared by the C-ABI implementation (api.cu) and the kernel
// launch wrappers (kernels/*.cu).  Not part of the public ABI.
#pragma once
#include <cuda_runtime.h>
#include <utility>
#include <cstdlib>
#include <cstdarg>
#include <cstdint>
#include <cstddef>

#include "et.h"

namespace et {

// thread-local error message (et_last_error)
void set_error(const char* fmt, ...);
et_status fail(et_status s, const char* fmt, ...);

#define ET_TRY(expr)                 \
  do {                               \
    et_status _s = (expr);           \
    if (_s != ET_OK) return _s;      \
  } while (0)

#define ET_CUDA(expr)                                                                              \
  do {                                                                                             \
    cudaError_t _e = (expr);                                                                       \
    if (_e != cudaSuccess)                                                                         \
      return ::et::fail(ET_ERR_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e), __FILE__, \
                        __LINE__);                                                                 \
  } while (0)

inline size_t dtype_size(et_dtype d) { return d == ET_FP32 ? 4 : 2; }
inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }
inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

// ---------------------------------------------------------------- prune / pack (kernels/prune_pack.cu)
struct PruneArgs {
  const void* W;
  int rows, cols;
  et_dtype dtype;
  et_pattern pattern;
  int tile_r, tile_c, group_rows;
  int n_prune;
  const uint32_t* mask_in;
};
size_t prune_workspace_bytes(int rows, int cols, et_pattern pattern, int tile_r, int tile_c);
// Runs the whole pack on `stream`; writes counts (nnz, rows_padded) to host via a sync.
et_status prune_pack_run(const PruneArgs& a, et_packed_weight* out, void* ws, size_t ws_bytes, cudaStream_t stream);
et_status unpack_run(const et_packed_weight* w, void* dense, cudaStream_t stream);

// ---------------------------------------------------------------- tile-sparse GEMM (kernels/tsgemm.cu)
// A segment of output tile-rows backed by one packed weight (QKV fuses three segments).
struct GemmSegment {
  const int32_t* row_ptr;   // tile CSR of the packed weight
  const int32_t* tile_col;  // tile column per packed tile
  const void* values;       // packed tiles
  const void* bias;         // [seg_rows] in dtype, or nullptr
  int tile_rows;            // number of 16-row tile rows in this segment
  int rp_stride;            // row_ptr entries between K parts (0: tile_rows + 1; a row slice of a larger
                            // packed weight passes row_ptr + first row and the weight's tile rows + 1)
  int out_col;              // first output column of the segment in Y
  float scale;              // epilogue scale for ET_EPI_BIAS_SCALE (applied if apply_scale)
  int apply_scale;
};
struct GemmArgs {
  const void* X;            // [M, ldx] in dtype; columns [k0, k0 + K) are the GEMM's K range
  int M, K, ldx, k0;
  et_dtype dtype;
  GemmSegment seg[3];
  int nseg;
  int kpart_tiles;          // split-K: number of 16-wide K tiles per part (K/16 = no split)
  void* Y;                  // output [M, ldy] (dtype) or fp32 partials [nparts][M, ldy]
  int ldy;
  et_epilogue epi;
  unsigned long long* ts;   // trace slot or nullptr
};
et_status gemm_run(const GemmArgs& a, cudaStream_t stream);
// FFN1 -> FFN2 in one launch when FFN1's pieces coincide with FFN2's K parts (kernels/tsgemm.cu)
bool gemm_ffn_applies(const GemmArgs& f1, const GemmArgs& f2);
et_status gemm_ffn_run(const GemmArgs& f1, const GemmArgs& f2, cudaStream_t stream);
// FP32 validation build (kernels/simt32.cu): CUDA-core FP32 FMA, same arguments
et_status gemm32_run(const GemmArgs& a, cudaStream_t stream);

// ---------------------------------------------------------------- LayerNorm (kernels/layernorm.cu)
struct LnArgs {
  const void* part;         // [nparts][M][N] partial sums in part_dtype (FP32 or the operand dtype)
  int nparts, M, N;
  const void* bias;
  et_dtype dtype;
  const void* resid;
  et_dtype resid_dtype;
  const float* gamma;
  const float* beta;
  float eps;
  void* out_act;
  void* out_resid;
  unsigned long long* ts;   // trace slot or nullptr
  et_dtype part_dtype;
};
et_status layernorm_run(const LnArgs& a, cudaStream_t stream);

// ---------------------------------------------------------------- attention (kernels/attention.cu)
struct AttnArgs {
  const void* qkv;
  int ld_qkv, q_off, k_off, v_off;
  const int32_t* v_col;     // [H] or nullptr
  const int32_t* v_width;   // [H] or nullptr
  void* Z;
  int ld_z;
  const int32_t* z_map;     // [packed V width] or nullptr
  const int32_t* lengths;   // [B] or nullptr
  int batch, seq_len, heads, d_k, head_begin, head_end;
  int causal;
  int long_form;
  int v_width_max;          // upper bound of the per-head V width (multiple of 16)
  float scale;
  et_dtype dtype;
  unsigned long long* ts;   // trace slot or nullptr
  int z_clear;              // z_map mode: Z columns no kept V feature maps to must be zero afterwards
                            // (attention_run zero-fills whole head windows or memsets Z; one place decides)
  int generic;              // force the generic short-form kernel (ET_ATTN_SHORT_GENERIC test hook)
  int vtab_static;          // v_col / v_width are layer weights (not written by a predecessor kernel)
};
et_status attention_run(const AttnArgs& a, cudaStream_t stream);
et_status attention32_run(const AttnArgs& a, cudaStream_t stream);
// seq_len <= 128, d_k = 64, dense V: the 3-CTAs-per-SM kernel (kernels/attention128.cu)
bool attention128_applies(const AttnArgs& a);
et_status attention128_run(const AttnArgs& a, cudaStream_t stream);
int attn_short_max(int d_k);
// split-K epilogue for K > 768 (kernels/aux.cu): Y = epi(sum of FP32 planes + bias) * scale per segment
struct SplitKSegs {
  int n;
  int col0[3];
  const void* bias[3];
  float scale[3];
};
et_status splitk_reduce_run(const float* part, int nparts, int M, int N, const SplitKSegs& segs, int act,
                            et_dtype dtype, void* Y, int ldy, cudaStream_t stream);
// pre-computed linear transformation (kernels/attention_pre.cu; Eq. 5)
struct VoPrep {
  const void* wv;           // [d, d] dense W_V (dtype)
  const void* wo;           // [d, d] W_O (dtype; rows outside `kept` are treated as pruned)
  const void* bv;           // [d] or nullptr
  const void* bo;           // [d] or nullptr
  const int32_t* kept;      // [n_kept] ascending kept W_O rows
  int n_kept, heads, d_model;
  et_dtype dtype;
  void* wvo_out;            // [heads * Dv, d]
  void* bias_out;           // [d] or nullptr
};
et_status vo_precompute_run(const VoPrep& v, cudaStream_t stream);
struct PreArgs {
  const void* qkv;          // [M, ld_qkv]: Q~ at q_off, K at k_off, X W_VO,h at vo_off + h Dv
  int ld_qkv, q_off, k_off, vo_off;
  int batch, seq_len, heads, d_k, d, Dv, groups;
  const int32_t* lengths;
  const int32_t* kept;
  int n_kept;
  void* planes;             // [groups][M][d] in part_dtype
  et_dtype part_dtype;
  int causal;
  float scale;
  et_dtype dtype;
  unsigned long long* ts;
};
int attention_pre_groups(int batch, int heads, int Dv);
et_status attention_pre_run(const PreArgs& a, cudaStream_t stream);
// paper-literal partial OTF (kernels/attention_partial.cu): S = Q K^T materialised in 16 bit,
// then mask + softmax + x V per row
size_t attention_partial_scores_bytes(int batch, int seq_len, int heads);
et_status attention_partial_run(const AttnArgs& a, void* scores, size_t scores_bytes, cudaStream_t stream);

// ---------------------------------------------------------------- small helpers (kernels/layernorm.cu)
et_status cast_run(const void* src, et_dtype sdt, void* dst, et_dtype ddt, size_t n, cudaStream_t stream);
// attention-aware (row-pruned W_V) layer data: per-head packed V columns / widths, the packed
// V bias, and the folded output bias b_O' = b_O + sum_{f pruned} W_O'[:, f] b_V[f] (reading C-6)
struct VPrep {
  const et_packed_weight* wv;
  const et_packed_weight* wo;
  const void* bv;
  const void* bo;
  int heads, d_k;
  int f_begin, f_end;  // pruned V features folded into b_O': f in [f_begin, f_end) (the call's heads)
  et_dtype dtype;
  int32_t* v_col;      // out [H]
  int32_t* v_width;    // out [H]
  void* bv_packed;     // out [rows_padded]
  void* bo_folded;     // out [d]
};
et_status vprep_run(const VPrep& v, cudaStream_t stream);

// column pruning (kernels/colgather.cu): Out[r, j] = In[r, idx[j]] (j < nk), 0 for nk <= j < nk_pad
et_status gather_cols_run(const void* in, int rows, int ld_in, const int32_t* idx, int nk, int nk_pad, et_dtype dt,
                          void* out, cudaStream_t stream);

// ---------------------------------------------------------------- tracing (api.cu)
// Record a mark of `kind` on `stream` if tracing is enabled; counts one kernel launch.
unsigned long long* trace_slot(int kind);

// Launch with programmatic stream serialisation (PDL): the kernel may begin while the previous
// kernel on the stream finishes; it must call pdl_wait() (ptx.cuh) before touching global data.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t stream,
                       Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}
// The same with a thread-block cluster of (cluster_x, 1, 1) CTAs (grid.x must be a multiple).
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl_cluster(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t stream,
                               unsigned cluster_x, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  attr[1].id = cudaLaunchAttributeClusterDimension;
  attr[1].val.clusterDim.x = cluster_x;
  attr[1].val.clusterDim.y = 1;
  attr[1].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}   // device slot of the next traced launch, or nullptr
void count_launch();
void add_launches(long long n);
long long launch_count();

}  // namespace et
