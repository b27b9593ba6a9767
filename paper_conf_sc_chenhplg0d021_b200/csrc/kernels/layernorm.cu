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
#include <cstdlib>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {
namespace {


template <int DT>
__device__ __forceinline__ float4 ld_act4(const void* p, size_t idx) {
  constexpr et_dtype dt = (et_dtype)DT;
  if constexpr (dt == ET_FP32) return *reinterpret_cast<const float4*>(static_cast<const float*>(p) + idx);
  const uint2 u = *reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(p) + idx);
  float2 a, b;
  if constexpr (dt == ET_BF16) {
    a = unpack2<true>(u.x);
    b = unpack2<true>(u.y);
  } else {
    a = unpack2<false>(u.x);
    b = unpack2<false>(u.y);
  }
  return make_float4(a.x, a.y, b.x, b.y);
}
template <int DT>
__device__ __forceinline__ void st_act4(void* p, size_t idx, float4 v) {
  constexpr et_dtype dt = (et_dtype)DT;
  if constexpr (dt == ET_FP32) {
    *reinterpret_cast<float4*>(static_cast<float*>(p) + idx) = v;
    return;
  }
  uint2 u;
  if constexpr (dt == ET_BF16) {
    u.x = pack2<true>(v.x, v.y);
    u.y = pack2<true>(v.z, v.w);
  } else {
    u.x = pack2<false>(v.x, v.y);
    u.y = pack2<false>(v.z, v.w);
  }
  *reinterpret_cast<uint2*>(static_cast<uint16_t*>(p) + idx) = u;
}

// One warp per row; NCH = ceil(N / 128) chunks of 4 columns per lane, NP split-K partial inputs.
// All loads of the row are issued before any arithmetic so each warp has NCH * (NP + 2) 16/8-byte
// requests in flight (the kernel is latency-bound otherwise).
template <int NCH, int NP, int DT, int RT, bool P16>
__device__ __forceinline__ void layernorm_row(const LnArgs& a) {
  const int row_i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (row_i >= a.M) return;
  const size_t row = (size_t)row_i * a.N;
  float4 part[NP][NCH];
  float4 bias[NCH], res[NCH];
  bool ok[NCH];
  // Every load is unconditional (out-of-range lanes and absent operands read a valid dummy address
  // and are masked afterwards): predicated "x = ok ? load : 0" loads make the compiler zero the
  // destination first and serialise the row's loads behind each other's latency.
  const bool has_bias = a.bias != nullptr, has_res = a.resid != nullptr;
  const void* bias_p = has_bias ? a.bias : a.part;
  const void* res_p = has_res ? a.resid : a.part;   // (dummy addresses: masked below)
#pragma unroll
  for (int c = 0; c < NCH; ++c) ok[c] = c * 128 + lane * 4 < a.N;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int col = ok[c] ? c * 128 + lane * 4 : 0;
#pragma unroll
    for (int q = 0; q < NP; ++q)
      if constexpr (P16) {   // 16-bit partial sums in the operand dtype (FP16 path, reading C-9)
        const uint2 u = __ldcs(reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(a.part) +
                                                               (size_t)q * a.M * a.N + row + col));
        const float2 lo = unpack2<DT == ET_BF16>(u.x), hi = unpack2<DT == ET_BF16>(u.y);
        part[q][c] = make_float4(lo.x, lo.y, hi.x, hi.y);
      } else {
        part[q][c] = __ldcs(reinterpret_cast<const float4*>(static_cast<const float*>(a.part) +
                                                            (size_t)q * a.M * a.N + row + col));
      }
    bias[c] = ld_act4<DT>(bias_p, has_bias ? col : 0);
    res[c] = ld_act4<RT>(res_p, has_res ? row + col : 0);
  }
  // masking by a bit AND, not by multiplying with 0 (a dummy read may hold an Inf / NaN bit
  // pattern, e.g. FP32 partials reinterpreted as 16-bit pairs, and 0 * Inf = NaN) and not by a
  // select (the compiler turns "load; select" into a predicated load and serialises the row)
  auto sel4 = [](bool keep, float4 v) {
    const uint32_t m = keep ? 0xffffffffu : 0u;
    return make_float4(__uint_as_float(__float_as_uint(v.x) & m), __uint_as_float(__float_as_uint(v.y) & m),
                       __uint_as_float(__float_as_uint(v.z) & m), __uint_as_float(__float_as_uint(v.w) & m));
  };
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
#pragma unroll
    for (int q = 0; q < NP; ++q) part[q][c] = sel4(ok[c], part[q][c]);
    bias[c] = sel4(ok[c] && has_bias, bias[c]);
    res[c] = sel4(ok[c] && has_res, res[c]);
  }
  float4 v[NCH];
  float s = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    float4 x = part[0][c];
#pragma unroll
    for (int q = 1; q < NP; ++q) {
      x.x += part[q][c].x; x.y += part[q][c].y; x.z += part[q][c].z; x.w += part[q][c].w;
    }
    x.x += bias[c].x + res[c].x; x.y += bias[c].y + res[c].y;
    x.z += bias[c].z + res[c].z; x.w += bias[c].w + res[c].w;
    v[c] = x;
    s += x.x + x.y + x.z + x.w;
  }
  if (a.gamma == nullptr) {   // no normalisation: out = sum(part) + bias (+ resid)
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
      if (!ok[c]) continue;
      const int col = c * 128 + lane * 4;
      if (a.out_act) st_act4<DT>(a.out_act, row + col, v[c]);
      if (a.out_resid) st_act4<RT>(a.out_resid, row + col, v[c]);
    }
    return;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / a.N;
  float q2 = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    if (!ok[c]) continue;
    const float dx = v[c].x - mean, dy = v[c].y - mean, dz = v[c].z - mean, dw = v[c].w - mean;
    q2 += dx * dx + dy * dy + dz * dz + dw * dw;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) q2 += __shfl_xor_sync(0xffffffffu, q2, o);
  const float rstd = rsqrtf(q2 / a.N + a.eps);
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    if (!ok[c]) continue;
    const int col = c * 128 + lane * 4;
    const float4 gm = __ldg(reinterpret_cast<const float4*>(a.gamma + col));
    const float4 bt = __ldg(reinterpret_cast<const float4*>(a.beta + col));
    const float4 y = make_float4((v[c].x - mean) * rstd * gm.x + bt.x, (v[c].y - mean) * rstd * gm.y + bt.y,
                                 (v[c].z - mean) * rstd * gm.z + bt.z, (v[c].w - mean) * rstd * gm.w + bt.w);
    if (a.out_act) st_act4<DT>(a.out_act, row + col, y);
    if (a.out_resid) st_act4<RT>(a.out_resid, row + col, y);
  }
}

// 8 columns per lane per chunk (N % 8 == 0): one 16-byte access per 16-bit operand and chunk
// (two for FP32), NCH8 = ceil(N / 256) chunks (3 for d = 768): half the memory instructions of the
// 4-wide form and twice the bytes per request — the kernel is latency / L2 bound.
template <int DT>
__device__ __forceinline__ void ld8(const void* p, size_t idx, float (&v)[8]) {
  if constexpr ((et_dtype)DT == ET_FP32) {
    const float4 a = *reinterpret_cast<const float4*>(static_cast<const float*>(p) + idx);
    const float4 b = *reinterpret_cast<const float4*>(static_cast<const float*>(p) + idx + 4);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
  } else {
    const uint4 u = *reinterpret_cast<const uint4*>(static_cast<const uint16_t*>(p) + idx);
    const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = unpack2<(et_dtype)DT == ET_BF16>(w[i]);
      v[2 * i] = f.x;
      v[2 * i + 1] = f.y;
    }
  }
}
template <int DT>
__device__ __forceinline__ void st8(void* p, size_t idx, const float (&v)[8]) {
  if constexpr ((et_dtype)DT == ET_FP32) {
    *reinterpret_cast<float4*>(static_cast<float*>(p) + idx) = make_float4(v[0], v[1], v[2], v[3]);
    *reinterpret_cast<float4*>(static_cast<float*>(p) + idx + 4) = make_float4(v[4], v[5], v[6], v[7]);
  } else {
    constexpr bool bf = (et_dtype)DT == ET_BF16;
    *reinterpret_cast<uint4*>(static_cast<uint16_t*>(p) + idx) =
        make_uint4(pack2<bf>(v[0], v[1]), pack2<bf>(v[2], v[3]), pack2<bf>(v[4], v[5]), pack2<bf>(v[6], v[7]));
  }
}

template <int NCH, int NP, int DT, int RT, bool P16>
__device__ __forceinline__ void layernorm_row8(const LnArgs& a) {
  const int row_i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (row_i >= a.M) return;
  const size_t row = (size_t)row_i * a.N;
  const bool has_bias = a.bias != nullptr, has_res = a.resid != nullptr;
  const void* bias_p = has_bias ? a.bias : a.part;   // dummy addresses for absent operands: the loads
  const void* res_p = has_res ? a.resid : a.part;    // stay unconditional, the values are discarded
  float v[NCH][8];
  // up to 16 (chunk, partial) pairs: every partial of the row in registers before any arithmetic
  // (loads in flight); wider rows or more partials (d_model 2048, d_ff 4096: Fig. 9) fold the
  // partials chunk by chunk (register budget)
  constexpr int NPR = NCH * NP <= 16 ? NP : 1;
  float part[NPR][NCH][8], bias[NCH][8], res[NCH][8];
  bool ok[NCH];
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    ok[c] = c * 256 + lane * 8 < a.N;
    const int col = ok[c] ? c * 256 + lane * 8 : 0;
#pragma unroll
    for (int q = 0; q < NP; ++q) {
      const size_t off = (size_t)q * a.M * a.N + row + col;
      float t[8];
      if constexpr (P16) ld8<DT>(a.part, off, t);
      else ld8<ET_FP32>(a.part, off, t);
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        if constexpr (NPR == NP) part[q][c][e] = t[e];
        else part[0][c][e] = q == 0 ? t[e] : part[0][c][e] + t[e];
      }
    }
    ld8<DT>(bias_p, has_bias ? col : 0, bias[c]);
    ld8<RT>(res_p, has_res ? row + col : 0, res[c]);
  }
  float s = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      float x = part[0][c][e];
#pragma unroll
      for (int q = 1; q < NPR; ++q) x += part[q][c][e];
      // absent operands / out-of-range lanes masked by a bit AND (see layernorm_row)
      x += __uint_as_float(__float_as_uint(bias[c][e]) & (has_bias ? 0xffffffffu : 0u));
      x += __uint_as_float(__float_as_uint(res[c][e]) & (has_res ? 0xffffffffu : 0u));
      v[c][e] = __uint_as_float(__float_as_uint(x) & (ok[c] ? 0xffffffffu : 0u));
      s += v[c][e];
    }
  }
  if (a.gamma == nullptr) {   // no normalisation: out = sum(part) + bias (+ resid)
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
      if (!ok[c]) continue;
      const int col = c * 256 + lane * 8;
      if (a.out_act) st8<DT>(a.out_act, row + col, v[c]);
      if (a.out_resid) st8<RT>(a.out_resid, row + col, v[c]);
    }
    return;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / a.N;
  float q2 = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c)
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      const float dx = ok[c] ? v[c][e] - mean : 0.f;
      q2 += dx * dx;
    }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) q2 += __shfl_xor_sync(0xffffffffu, q2, o);
  const float rstd = rsqrtf(q2 / a.N + a.eps);
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    if (!ok[c]) continue;
    const int col = c * 256 + lane * 8;
    float g[8], b[8], y[8];
    ld8<ET_FP32>(a.gamma, col, g);
    ld8<ET_FP32>(a.beta, col, b);
#pragma unroll
    for (int e = 0; e < 8; ++e) y[e] = (v[c][e] - mean) * rstd * g[e] + b[e];
    if (a.out_act) st8<DT>(a.out_act, row + col, y);
    if (a.out_resid) st8<RT>(a.out_resid, row + col, y);
  }
}

template <int NCH, int NP, int DT, int RT, bool P16>
__global__ void __launch_bounds__(512) layernorm_kernel(const LnArgs a) {
  pdl_trigger();
  pdl_wait();
  trace_cta_start(a.ts);
  if constexpr (NCH < 0) layernorm_row8<-NCH, NP, DT, RT, P16>(a);   // NCH < 0: 8-wide form, -NCH chunks
  else layernorm_row<NCH, NP, DT, RT, P16>(a);
  if (a.ts != nullptr) {
    __syncthreads();
    trace_cta_end(a.ts);
  }
}

template <int NCH, int DT, int RT, bool P16>
et_status launch_np(const LnArgs& a, cudaStream_t stream) {
  // rows per CTA (one warp each): 128 threads = 4 rows (256 / 512 measured no faster, round 1)
  constexpr int threads = 128;
  const int blocks = (a.M * 32 + threads - 1) / threads;
  cudaError_t e = cudaSuccess;
  switch (a.nparts) {
    case 1: e = launch_pdl(layernorm_kernel<NCH, 1, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
    case 2: e = launch_pdl(layernorm_kernel<NCH, 2, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
    case 3: e = launch_pdl(layernorm_kernel<NCH, 3, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
    case 4: e = launch_pdl(layernorm_kernel<NCH, 4, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
    default:
      if constexpr (NCH < 0) {   // 8-wide form only: more K parts (K > 3072)
        switch (a.nparts) {
          case 5: e = launch_pdl(layernorm_kernel<NCH, 5, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
          case 6: e = launch_pdl(layernorm_kernel<NCH, 6, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
          case 7: e = launch_pdl(layernorm_kernel<NCH, 7, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
          case 8: e = launch_pdl(layernorm_kernel<NCH, 8, DT, RT, P16>, dim3(blocks), dim3(threads), 0, stream, a); break;
          default: return fail(ET_ERR_UNSUPPORTED, "LayerNorm: up to 8 partial inputs (got %d)", a.nparts);
        }
        break;
      }
      return fail(ET_ERR_UNSUPPORTED, "LayerNorm: up to 4 partial inputs with N %% 8 != 0 (got %d)", a.nparts);
  }
  ET_CUDA(e);
  count_launch();
  return ET_OK;
}

template <int NCH>
et_status launch_dt(const LnArgs& a, cudaStream_t stream) {
  const int dt = a.dtype, rt = a.resid ? a.resid_dtype : (a.out_resid ? a.resid_dtype : a.dtype);
  if (a.part_dtype != ET_FP32 && a.part_dtype != a.dtype)
    return fail(ET_ERR_UNSUPPORTED, "LayerNorm: partial sums must be FP32 or the operand dtype");
  const bool p16 = a.part_dtype != ET_FP32;
  if (dt == ET_FP16 && rt == ET_FP16)
    return p16 ? launch_np<NCH, ET_FP16, ET_FP16, true>(a, stream) : launch_np<NCH, ET_FP16, ET_FP16, false>(a, stream);
  if (dt == ET_FP16 && rt == ET_FP32)
    return p16 ? launch_np<NCH, ET_FP16, ET_FP32, true>(a, stream) : launch_np<NCH, ET_FP16, ET_FP32, false>(a, stream);
  if (dt == ET_BF16 && rt == ET_BF16)
    return p16 ? launch_np<NCH, ET_BF16, ET_BF16, true>(a, stream) : launch_np<NCH, ET_BF16, ET_BF16, false>(a, stream);
  if (dt == ET_BF16 && rt == ET_FP32)
    return p16 ? launch_np<NCH, ET_BF16, ET_FP32, true>(a, stream) : launch_np<NCH, ET_BF16, ET_FP32, false>(a, stream);
  if (dt == ET_FP32 && rt == ET_FP32 && !p16)   // FP32 validation build
    return launch_np<NCH, ET_FP32, ET_FP32, false>(a, stream);
  return fail(ET_ERR_UNSUPPORTED, "LayerNorm: dtype pair (%d, %d) not supported", dt, rt);
}

}  // namespace

et_status layernorm_run(const LnArgs& a, cudaStream_t stream) {
  if (a.N % 4 || a.N > 256 * 8 || (a.N > 128 * 8 && a.N % 8))
    return fail(ET_ERR_UNSUPPORTED, "LayerNorm: N must be a multiple of 4 and <= 1024, or of 8 and <= 2048 (got %d)", a.N);
  if (a.M <= 0) return ET_OK;
  // 8-wide form (16-byte accesses) whenever N % 8 == 0 (up to 8 partial inputs); the 4-wide form
  // for N % 8 == 4
  if (a.N % 8 == 0 && a.nparts <= 8) {
    switch ((a.N + 255) / 256) {
      case 1: return launch_dt<-1>(a, stream);
      case 2: return launch_dt<-2>(a, stream);
      case 3: return launch_dt<-3>(a, stream);
      case 4: return launch_dt<-4>(a, stream);
      case 5: case 6: return launch_dt<-6>(a, stream);
      default: return launch_dt<-8>(a, stream);
    }
  }
  switch ((a.N + 127) / 128) {
    case 1: return launch_dt<1>(a, stream);
    case 2: return launch_dt<2>(a, stream);
    case 3: return launch_dt<3>(a, stream);
    case 4: return launch_dt<4>(a, stream);
    case 5: return launch_dt<5>(a, stream);
    case 6: return launch_dt<6>(a, stream);
    case 7: return launch_dt<7>(a, stream);
    default: return launch_dt<8>(a, stream);
  }
}

}  // namespace et
