// Small helper kernels of the encoder path:
//   * cast: residual-stream dtype <-> GEMM operand dtype (reading C-22: FP32 residual stream);
//   * vprep: attention-aware layers (W_V row pruned, PAPER.md line 107 / 171 / 317): per-head packed
//     V column offsets and widths, the packed V bias, and the folded output bias
//     b_O' = b_O + sum_{f pruned} W_O'[:, f] b_V[f]  — a pruned V feature f has V[:, f] = b_V[f] and,
//     since every softmax row sums to 1, Z[:, f] = b_V[f] exactly (reading C-6).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <algorithm>
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

// per-head segments of the packed (padded) V rows: thread h counts head h's kept rows from the row
// bitmap (popcount over bits [h d_k, (h+1) d_k)), pads it to 16, and sums the padded widths of the
// heads before it.  No serial pointer chase (a single-thread walk over idx cost one dependent global
// load per kept row, ~30 us per forward on C2).
__global__ void vprep_heads_kernel(const uint32_t* __restrict__ mask, int heads, int d_k,
                                   int32_t* __restrict__ v_col, int32_t* __restrict__ v_width) {
  extern __shared__ int32_t s_pad[];
  for (int h = threadIdx.x; h < heads; h += blockDim.x) {
    const int b0 = h * d_k, b1 = b0 + d_k;
    int cnt = 0;
    for (int w = b0 >> 5; w <= (b1 - 1) >> 5; ++w) {
      uint32_t m = __ldg(mask + w);
      const int lo = max(b0 - w * 32, 0), hi = min(b1 - w * 32, 32);   // bits [lo, hi) of word w
      if (hi < 32) m &= (1u << hi) - 1u;
      m &= ~((1u << lo) - 1u);
      cnt += __popc(m);
    }
    s_pad[h] = (cnt + 15) / 16 * 16;
  }
  __syncthreads();
  for (int h = threadIdx.x; h < heads; h += blockDim.x) {
    int start = 0;
    for (int k = 0; k < h; ++k) start += s_pad[k];
    v_col[h] = start;
    v_width[h] = s_pad[h];
  }
}

__global__ void vprep_bias_kernel(const int32_t* __restrict__ row_map, int rows_padded, const void* __restrict__ bv,
                                  et_dtype dt, void* __restrict__ bv_packed) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= rows_padded) return;
  const int r = row_map[i];
  stf(bv_packed, dt, i, r >= 0 ? ldf(bv, dt, r) : 0.f);
}

// one warp per output feature i of W_O (tile pruned): the lanes stride over the (kept tile, k) pairs of
// its tile row (every K part), add W_O'[i, f] * b_V[f] for every pruned V feature f in FP64, and
// combine in a fixed butterfly (deterministic).  (One thread per feature walking the row serially
// was the longest kernel of a C2 forward: 27 us on 4 SMs.)
__global__ void vprep_fold_kernel(const uint8_t* __restrict__ wo_values, const int32_t* __restrict__ wo_prp,
                                  const int32_t* __restrict__ wo_tile_col, int wo_tile_rows, int kparts,
                                  const uint32_t* __restrict__ wv_mask, int f0, int f1, const void* __restrict__ bv,
                                  const void* __restrict__ bo, et_dtype dt, int d, void* __restrict__ bo_folded) {
  const int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (i >= d) return;
  const int ti = i >> 4, n = i & 15;
  double acc = 0.0;
  for (int z = 0; z < kparts; ++z) {
    const int32_t* rp = wo_prp + z * (wo_tile_rows + 1);
    const int t0 = rp[ti], ne = (rp[ti + 1] - t0) * 16;
    for (int e = lane; e < ne; e += 32) {
      const int t = t0 + (e >> 4), k = e & 15;
      const int f = wo_tile_col[t] * 16 + k;
      if (f < f0 || f >= f1 || ((wv_mask[f >> 5] >> (f & 31)) & 1u)) continue;   // kept / other heads: no fold
      const uint8_t* tile = wo_values + (size_t)t * 256 * (dt == ET_FP32 ? 4 : 2);
      float w;
      if (dt == ET_FP32) {   // FP32 tiles: row-major (simt32.cu)
        w = *reinterpret_cast<const float*>(tile + n * 64 + k * 4);
      } else {   // 16-bit tiles: tcgen05 core-matrix layout
        const uint16_t raw = *reinterpret_cast<const uint16_t*>(tile + (n >> 3) * 256 + (k >> 3) * 128 + (n & 7) * 16 + (k & 7) * 2);
        w = dt == ET_BF16 ? __bfloat162float(__ushort_as_bfloat16(raw)) : __half2float(__ushort_as_half(raw));
      }
      acc += (double)w * (double)ldf(bv, dt, f);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane == 0)   // bo NULL: fold only (head-parallel rank)
    stf(bo_folded, dt, i, (float)((bo ? (double)ldf(bo, dt, i) : 0.0) + acc));
}


// Split-K epilogue for K > 768 (one TMEM-resident A part holds 768 columns): Y = epi(sum_p part[p] + b)
// in the operand dtype.  Segment s covers output columns [col0, col0 + ncols) with its own bias and
// Q-scale; GELU (reading C-12: the erf form, here evaluated with erff) / ReLU as the GEMM epilogue.
__global__ void splitk_reduce_kernel(const float* __restrict__ part, int nparts, int M, int N, SplitKSegs segs,
                                     int act, et_dtype dtype, void* __restrict__ Y, int ldy) {
  const int n8 = N / 8;
  const size_t total = (size_t)M * n8;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total; i += (size_t)gridDim.x * blockDim.x) {
    const int m = (int)(i / n8), c = (int)(i % n8) * 8;
    float v[8];
    const float* src = part + (size_t)m * N + c;
    {
      const float4 a = *reinterpret_cast<const float4*>(src), b = *reinterpret_cast<const float4*>(src + 4);
      v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
    }
    for (int p = 1; p < nparts; ++p) {
      const float* q = src + (size_t)p * M * N;
      const float4 a = *reinterpret_cast<const float4*>(q), b = *reinterpret_cast<const float4*>(q + 4);
      v[0] += a.x; v[1] += a.y; v[2] += a.z; v[3] += a.w; v[4] += b.x; v[5] += b.y; v[6] += b.z; v[7] += b.w;
    }
    int s = 0;
    while (s + 1 < segs.n && c >= segs.col0[s + 1]) ++s;
    const void* bias = segs.bias[s];
    const float scale = segs.scale[s];
    for (int u = 0; u < 8; ++u) {
      float x = v[u];
      if (bias) x += dtype == ET_BF16 ? __bfloat162float(static_cast<const __nv_bfloat16*>(bias)[c - segs.col0[s] + u])
                                      : __half2float(static_cast<const __half*>(bias)[c - segs.col0[s] + u]);
      if (act == 1) x = 0.5f * x * (1.0f + erff(x * 0.70710678118654752f));
      else if (act == 2) x = fmaxf(x, 0.0f);
      v[u] = x * scale;
    }
    uint4 o;
    uint32_t* ow = reinterpret_cast<uint32_t*>(&o);
    for (int u = 0; u < 4; ++u) {
      if (dtype == ET_BF16) {
        __nv_bfloat162 h = __floats2bfloat162_rn(v[2 * u], v[2 * u + 1]);
        ow[u] = *reinterpret_cast<uint32_t*>(&h);
      } else {
        __half2 h = __floats2half2_rn(v[2 * u], v[2 * u + 1]);
        ow[u] = *reinterpret_cast<uint32_t*>(&h);
      }
    }
    *reinterpret_cast<uint4*>(static_cast<uint16_t*>(Y) + (size_t)m * ldy + c) = o;
  }
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
  const int ht = v.heads < 1024 ? (v.heads + 31) / 32 * 32 : 1024;
  vprep_heads_kernel<<<1, ht, v.heads * sizeof(int32_t), stream>>>(v.wv->mask, v.heads, v.d_k, v.v_col,
                                                                  v.v_width);
  count_launch();
  ET_CUDA(cudaGetLastError());
  if (v.wv->rows_padded > 0) {
    vprep_bias_kernel<<<(v.wv->rows_padded + 255) / 256, 256, 0, stream>>>(v.wv->row_map, v.wv->rows_padded, v.bv,
                                                                           v.dtype, v.bv_packed);
    count_launch();
    ET_CUDA(cudaGetLastError());
  }
  const int d = v.wo->rows;
  vprep_fold_kernel<<<(d + 3) / 4, 128, 0, stream>>>(static_cast<const uint8_t*>(v.wo->values),
                                                         v.wo->part_row_ptr, v.wo->tile_col, v.wo->rows / 16,
                                                         v.wo->kparts, v.wv->mask, v.f_begin, v.f_end, v.bv, v.bo,
                                                         v.dtype, d,
                                                         v.bo_folded);
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

et_status splitk_reduce_run(const float* part, int nparts, int M, int N, const SplitKSegs& segs, int act,
                            et_dtype dtype, void* Y, int ldy, cudaStream_t stream) {
  if (N % 8 || (ldy * 2) % 16 || !aligned16(Y)) return fail(ET_ERR_INVALID_ARG, "split-K reduce: 16-byte rows required");
  const size_t total = (size_t)M * (N / 8);
  const int grid = (int)std::min<size_t>((total + 255) / 256, 148 * 8);
  splitk_reduce_kernel<<<grid, 256, 0, stream>>>(part, nparts, M, N, segs, act, dtype, Y, ldy);
  ET_CUDA(cudaGetLastError());
  count_launch();
  return ET_OK;
}

}  // namespace et
