// Small helper kernels of the encoder path:
//   * cast: residual-stream dtype <-> GEMM operand dtype (reading C-22: FP32 residual stream);
//   * vprep: attention-aware layers (W_V row pruned, PAPER.md line 107 / 171 / 317): per-head packed
//     V column offsets and widths, the packed V bias, and the folded output bias
//     b_O' = b_O + sum_{f pruned} W_O'[:, f] b_V[f]  — a pruned V feature f has V[:, f] = b_V[f] and,
//     since every softmax row sums to 1, Z[:, f] = b_V[f] exactly (reading C-6).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {
namespace {

__device__ __forceinline__ float ldf(const void* p, et_dtype dt, size_t i) {
  if (dt == ET_FP32) return static_cast<const float*>(p)[i];
  if (dt == ET_BF16) return __bfloat162float(static_cast<const __nv_bfloat16*>(p)[i]);
  return __half2float(static_cast<const __half*>(p)[i]);
}
__device__ __forceinline__ void stf(void* p, et_dtype dt, size_t i, float v) {
  if (dt == ET_FP32) static_cast<float*>(p)[i] = v;
  else if (dt == ET_BF16) static_cast<__nv_bfloat16*>(p)[i] = __float2bfloat16_rn(v);
  else static_cast<__half*>(p)[i] = __float2half_rn(v);
}

__global__ void cast_kernel(const void* __restrict__ src, et_dtype sdt, void* __restrict__ dst, et_dtype ddt,
                            size_t n) {
  const size_t i0 = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) * 4;
  for (size_t i = i0; i < n && i < i0 + 4; ++i) stf(dst, ddt, i, ldf(src, sdt, i));
}

// single thread: per-head segments of the packed (padded) V rows
__global__ void vprep_heads_kernel(const int32_t* __restrict__ idx, int nnz, int heads, int d_k,
                                   int32_t* __restrict__ v_col, int32_t* __restrict__ v_width) {
  if (threadIdx.x || blockIdx.x) return;
  int k = 0, start = 0;
  for (int h = 0; h < heads; ++h) {
    int cnt = 0;
    while (k < nnz && idx[k] / d_k == h) {
      ++cnt;
      ++k;
    }
    const int pad = (cnt + 15) / 16 * 16;
    v_col[h] = start;
    v_width[h] = pad;
    start += pad;
  }
}

__global__ void vprep_bias_kernel(const int32_t* __restrict__ row_map, int rows_padded, const void* __restrict__ bv,
                                  et_dtype dt, void* __restrict__ bv_packed) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= rows_padded) return;
  const int r = row_map[i];
  stf(bv_packed, dt, i, r >= 0 ? ldf(bv, dt, r) : 0.f);
}

// one thread per output feature i of W_O (tile pruned): walk the kept tiles of its tile row in a
// fixed order (deterministic), add W_O'[i, f] * b_V[f] for every pruned V feature f.
__global__ void vprep_fold_kernel(const uint8_t* __restrict__ wo_values, const int32_t* __restrict__ wo_prp,
                                  const int32_t* __restrict__ wo_tile_col, int wo_tile_rows, int kparts,
                                  const uint32_t* __restrict__ wv_mask, const void* __restrict__ bv,
                                  const void* __restrict__ bo, et_dtype dt, int d, void* __restrict__ bo_folded) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= d) return;
  const int ti = i >> 4, n = i & 15;
  double acc = 0.0;
  for (int z = 0; z < kparts; ++z) {
    const int32_t* rp = wo_prp + z * (wo_tile_rows + 1);
    for (int t = rp[ti]; t < rp[ti + 1]; ++t) {
      const int j = wo_tile_col[t];
      const uint8_t* tile = wo_values + (size_t)t * 256 * (dt == ET_FP32 ? 4 : 2);
      for (int k = 0; k < 16; ++k) {
        const int f = j * 16 + k;
        if ((wv_mask[f >> 5] >> (f & 31)) & 1u) continue;   // kept V feature: no fold
        float w;
        if (dt == ET_FP32) {   // FP32 tiles: row-major (simt32.cu)
          w = *reinterpret_cast<const float*>(tile + n * 64 + k * 4);
        } else {
          const uint16_t raw = *reinterpret_cast<const uint16_t*>(tile + (n >> 3) * 256 + (k >> 3) * 128 + (n & 7) * 16 + (k & 7) * 2);
          w = dt == ET_BF16 ? __bfloat162float(__ushort_as_bfloat16(raw)) : __half2float(__ushort_as_half(raw));
        }
        acc += (double)w * (double)ldf(bv, dt, f);
      }
    }
  }
  stf(bo_folded, dt, i, (float)((bo ? (double)ldf(bo, dt, i) : 0.0) + acc));   // bo NULL: fold only (head-parallel rank)
}

}  // namespace

et_status cast_run(const void* src, et_dtype sdt, void* dst, et_dtype ddt, size_t n, cudaStream_t stream) {
  if (n == 0) return ET_OK;
  const size_t threads = 256, per = threads * 4;
  cast_kernel<<<(unsigned)((n + per - 1) / per), (unsigned)threads, 0, stream>>>(src, sdt, dst, ddt, n);
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

et_status vprep_run(const VPrep& v, cudaStream_t stream) {
  if (v.wv->pattern != ET_PRUNE_ROW) return fail(ET_ERR_INTERNAL, "vprep: W_V is not row pruned");
  if (v.wo->pattern != ET_PRUNE_TILE) return fail(ET_ERR_UNSUPPORTED, "vprep: W_O must be tile pruned");
  vprep_heads_kernel<<<1, 32, 0, stream>>>(v.wv->idx, v.wv->nnz, v.heads, v.d_k, v.v_col, v.v_width);
  count_launch();
  ET_CUDA(cudaGetLastError());
  if (v.wv->rows_padded > 0) {
    vprep_bias_kernel<<<(v.wv->rows_padded + 255) / 256, 256, 0, stream>>>(v.wv->row_map, v.wv->rows_padded, v.bv,
                                                                           v.dtype, v.bv_packed);
    count_launch();
    ET_CUDA(cudaGetLastError());
  }
  const int d = v.wo->rows;
  vprep_fold_kernel<<<(d + 127) / 128, 128, 0, stream>>>(static_cast<const uint8_t*>(v.wo->values),
                                                         v.wo->part_row_ptr, v.wo->tile_col, v.wo->rows / 16,
                                                         v.wo->kparts, v.wv->mask, v.bv, v.bo, v.dtype, d,
                                                         v.bo_folded);
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

}  // namespace et
