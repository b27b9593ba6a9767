// Residual add + LayerNorm epilogue of the attention block and of the FFN (PAPER.md line 75,
// §2.1: "A layer normalization is applied after self-attention and MLP respectively, whose input
// will be added by the input of the module").  Also reduces the fp32 split-K partial sums of the
// preceding tile-sparse GEMM:
//   v = sum_p part[p] + bias + resid;  out = (v - mean) / sqrt(var + eps) * gamma + beta
// (biased variance, reading C-11).  HBM/L2-bound: one warp per row, 16-byte vector accesses,
// the row kept in registers (two-pass mean / variance without re-reading memory).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {
namespace {

constexpr int kMaxChunks = 16;  // N <= 16 * 128 = 2048

__device__ __forceinline__ float4 ld_act4(const void* p, et_dtype dt, size_t idx) {
  if (dt == ET_FP32) return *reinterpret_cast<const float4*>(static_cast<const float*>(p) + idx);
  const uint2 u = *reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(p) + idx);
  float2 a, b;
  if (dt == ET_BF16) {
    a = unpack2<true>(u.x);
    b = unpack2<true>(u.y);
  } else {
    a = unpack2<false>(u.x);
    b = unpack2<false>(u.y);
  }
  return make_float4(a.x, a.y, b.x, b.y);
}
__device__ __forceinline__ void st_act4(void* p, et_dtype dt, size_t idx, float4 v) {
  if (dt == ET_FP32) {
    *reinterpret_cast<float4*>(static_cast<float*>(p) + idx) = v;
    return;
  }
  uint2 u;
  if (dt == ET_BF16) {
    u.x = pack2<true>(v.x, v.y);
    u.y = pack2<true>(v.z, v.w);
  } else {
    u.x = pack2<false>(v.x, v.y);
    u.y = pack2<false>(v.z, v.w);
  }
  *reinterpret_cast<uint2*>(static_cast<uint16_t*>(p) + idx) = u;
}

__global__ void __launch_bounds__(256) layernorm_kernel(const LnArgs a) {
  const int warp_g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (warp_g >= a.M) return;
  const int nch = (a.N + 127) / 128;
  const size_t row = (size_t)warp_g * a.N;
  float4 v[kMaxChunks];
  float s = 0.f;
#pragma unroll
  for (int c = 0; c < kMaxChunks; ++c) {
    v[c] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (c < nch && c * 128 + lane * 4 < a.N) {
      const int col = c * 128 + lane * 4;
      float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int pidx = 0; pidx < a.nparts; ++pidx) {
        const float4 t = *reinterpret_cast<const float4*>(a.part + (size_t)pidx * a.M * a.N + row + col);
        x.x += t.x; x.y += t.y; x.z += t.z; x.w += t.w;
      }
      if (a.bias) {
        const float4 b = ld_act4(a.bias, a.dtype, col);
        x.x += b.x; x.y += b.y; x.z += b.z; x.w += b.w;
      }
      if (a.resid) {
        const float4 r = ld_act4(a.resid, a.resid_dtype, row + col);
        x.x += r.x; x.y += r.y; x.z += r.z; x.w += r.w;
      }
      v[c] = x;
      s += x.x + x.y + x.z + x.w;
    }
  }
  if (a.gamma == nullptr) {   // no normalisation: out = sum(part) + bias (+ resid)
#pragma unroll
    for (int c = 0; c < kMaxChunks; ++c) {
      if (c < nch && c * 128 + lane * 4 < a.N) {
        const int col = c * 128 + lane * 4;
        if (a.out_act) st_act4(a.out_act, a.dtype, row + col, v[c]);
        if (a.out_resid) st_act4(a.out_resid, a.resid_dtype, row + col, v[c]);
      }
    }
    return;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / a.N;
  float q = 0.f;
#pragma unroll
  for (int c = 0; c < kMaxChunks; ++c) {
    if (c < nch && c * 128 + lane * 4 < a.N) {
      const float dx = v[c].x - mean, dy = v[c].y - mean, dz = v[c].z - mean, dw = v[c].w - mean;
      q += dx * dx + dy * dy + dz * dz + dw * dw;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float rstd = rsqrtf(q / a.N + a.eps);
#pragma unroll
  for (int c = 0; c < kMaxChunks; ++c) {
    if (c < nch && c * 128 + lane * 4 < a.N) {
      const int col = c * 128 + lane * 4;
      const float4 gm = *reinterpret_cast<const float4*>(a.gamma + col);
      const float4 bt = *reinterpret_cast<const float4*>(a.beta + col);
      const float4 y = make_float4((v[c].x - mean) * rstd * gm.x + bt.x, (v[c].y - mean) * rstd * gm.y + bt.y,
                                   (v[c].z - mean) * rstd * gm.z + bt.z, (v[c].w - mean) * rstd * gm.w + bt.w);
      if (a.out_act) st_act4(a.out_act, a.dtype, row + col, y);
      if (a.out_resid) st_act4(a.out_resid, a.resid_dtype, row + col, y);
    }
  }
}

}  // namespace

et_status layernorm_run(const LnArgs& a, cudaStream_t stream) {
  if (a.N % 4 || a.N > 128 * kMaxChunks)
    return fail(ET_ERR_UNSUPPORTED, "LayerNorm: N must be a multiple of 4 and <= 2048 (got %d)", a.N);
  if (a.M <= 0) return ET_OK;
  const int threads = 256;
  const int blocks = (a.M * 32 + threads - 1) / threads;
  layernorm_kernel<<<blocks, threads, 0, stream>>>(a);
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

}  // namespace et
