// FP32 validation build (BASELINE.json configs[0], C1: "FP32"; north_star: "1e-5 for an FP32
// validation build"; reading C-9 / SURVEY §7 H8: one-pass TF32 tensor-core math misses 1e-5, so
// this path is plain FP32 FMA on the CUDA cores).  Same operations, arguments and layouts as the
// tcgen05 path it stands in for (kernels/tsgemm.cu, kernels/attention*.cu):
//   * tile-sparse linear layer (§4.2): one CTA per (tile row, 64-token
//     block, K part); the CTA walks the kept tiles of its tile row in ascending column order (the
//     packed CSR), pruned tiles cost nothing.  FP32 tiles are packed row-major (element (n, k) at
//     byte n*64 + k*4, 1 KB per tile; kernels/prune_pack.cu).  Epilogues as the tcgen05 kernel:
//     bias, Q scale 1/sqrt(d_k) before the store (line 159), GELU(erf) (accurate erff), ReLU, or
//     the raw split-K partial plane.
//   * on-the-fly attention (line 97-113 §3.1): one warp per query row; the score row lives in
//     shared memory (as in the paper's OTF kernel, Eq. 6), masked keys get probability exactly 0,
//     max-subtracted softmax with accurate expf, deferred 1/sum normalisation (line 361).  The
//     seq x seq matrix never reaches global memory.
// Not a performance path: C1 is launch-latency bound.
#include <cuda_runtime.h>
#include <cstdint>
#include <cmath>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {
namespace {

constexpr int kTok = 64;   // tokens per CTA

struct G32Params {
  const float* X;
  int M, ldx, Kp, kparts, K;
  int nseg;
  int row_begin[4];          // first global tile row of each segment (prefix sums)
  const int32_t* prp[3];     // part_row_ptr [kparts][tile_rows + 1]
  const int32_t* tile_col[3];
  const float* values[3];
  const float* bias[3];
  int tile_rows[3], rp_stride[3], out_col[3];
  float scale[3];
  int apply_scale[3];
  float* Y;
  int ldy;
  long long part_stride;
  int epi;
  unsigned long long* ts;
};

__global__ void __launch_bounds__(256) gemm32_kernel(const G32Params p) {
  __shared__ float sw[16][17];        // W tile (n, k), padded
  __shared__ float sx[kTok][17];      // X block (token, k), padded
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  const int gr = blockIdx.x;          // global tile row
  int s = 0;
  while (s + 1 < p.nseg && gr >= p.row_begin[s + 1]) ++s;
  const int i = gr - p.row_begin[s];
  const int m0 = blockIdx.y * kTok, z = blockIdx.z;
  const int n = threadIdx.x & 15, tg = threadIdx.x >> 4;   // feature n, tokens tg*4 .. tg*4+3
  const int32_t* rp = p.prp[s] + (size_t)z * p.rp_stride[s];
  float acc[4] = {0.f, 0.f, 0.f, 0.f};
  for (int t = rp[i]; t < rp[i + 1]; ++t) {
    const int j = p.tile_col[s][t];                        // global tile column (K part z's range)
    const float* wt = p.values[s] + (size_t)t * 256;
    __syncthreads();
    sw[threadIdx.x >> 4][threadIdx.x & 15] = wt[threadIdx.x];
    for (int e = threadIdx.x; e < kTok * 16; e += 256) {
      const int r = e >> 4, k = e & 15, m = m0 + r;
      sx[r][k] = m < p.M ? p.X[(size_t)m * p.ldx + j * 16 + k] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      const float w = sw[n][k];
#pragma unroll
      for (int r = 0; r < 4; ++r) acc[r] = fmaf(sx[tg * 4 + r][k], w, acc[r]);
    }
  }
  const int col = p.out_col[s] + i * 16 + n;
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const int m = m0 + tg * 4 + r;
    if (m >= p.M) continue;
    float v = acc[r];
    if (p.epi == ET_EPI_F32) {
      p.Y[(size_t)z * p.part_stride + (size_t)m * p.ldy + col] = v;
      continue;
    }
    if (p.bias[s]) v += p.bias[s][i * 16 + n];
    if (p.epi == ET_EPI_BIAS_SCALE && p.apply_scale[s]) v *= p.scale[s];
    if (p.epi == ET_EPI_BIAS_GELU) v = 0.5f * v * (1.0f + erff(v * 0.70710678118654752f));
    if (p.epi == ET_EPI_BIAS_RELU) v = fmaxf(v, 0.0f);
    p.Y[(size_t)m * p.ldy + col] = v;
  }
  if (p.ts != nullptr) {
    __syncthreads();
    trace_cta_end(p.ts);
  }
}

struct A32Params {
  const float* qkv;
  int ld_qkv, q_off, k_off, v_off;
  const int32_t* v_col;
  const int32_t* v_width;
  float* Z;
  int ld_z;
  const int32_t* z_map;
  const int32_t* lengths;
  int S, d_k, head_begin, causal;
  float scale;
  unsigned long long* ts;
};

// grid (ceil(S / 4), heads in range, batch), 4 warps, one query row per warp
__global__ void __launch_bounds__(128) attn32_kernel(const A32Params p) {
  extern __shared__ float sm32[];
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int i = blockIdx.x * 4 + warp;           // query row
  const int h = p.head_begin + blockIdx.y, b = blockIdx.z;
  float* srow = sm32 + (size_t)warp * p.S;       // this warp's score row
  float* qrow = sm32 + (size_t)4 * p.S + warp * 128;
  if (i < p.S) {
    const int len = p.lengths ? p.lengths[b] : p.S;
    const int kend = p.causal ? min(len, i + 1) : len;   // keys [0, kend) are unmasked (reading C-7)
    const size_t tok0 = (size_t)b * p.S;
    const float* q = p.qkv + (tok0 + i) * p.ld_qkv + p.q_off + h * p.d_k;
    for (int c = lane; c < p.d_k; c += 32) qrow[c] = q[c];
    __syncwarp();
    float mx = -INFINITY;
    for (int j = lane; j < kend; j += 32) {
      const float* k = p.qkv + (tok0 + j) * p.ld_qkv + p.k_off + h * p.d_k;
      float s = 0.f;
      for (int c = 0; c < p.d_k; ++c) s = fmaf(qrow[c], k[c], s);
      s *= p.scale;
      srow[j] = s;
      mx = fmaxf(mx, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    float sum = 0.f;
    for (int j = lane; j < kend; j += 32) {
      const float e = expf(srow[j] - mx);
      srow[j] = e;
      sum += e;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    __syncwarp();
    const int vc = p.v_col ? p.v_col[h] : h * p.d_k;
    const int vw = p.v_width ? p.v_width[h] : p.d_k;
    const float inv = 1.0f / sum;
    for (int c = lane; c < vw; c += 32) {
      const float* v = p.qkv + tok0 * p.ld_qkv + p.v_off + vc + c;
      float acc = 0.f;
      for (int j = 0; j < kend; ++j) acc = fmaf(srow[j], v[(size_t)j * p.ld_qkv], acc);
      const int zc = p.z_map ? p.z_map[vc + c] : h * p.d_k + c;
      if (zc >= 0) p.Z[(tok0 + i) * p.ld_z + zc] = acc * inv;
    }
  }
  if (p.ts != nullptr) {
    __syncthreads();
    trace_cta_end(p.ts);
  }
}

}  // namespace

et_status gemm32_run(const GemmArgs& a, cudaStream_t stream) {
  const int kparts = (a.K + 767) / 768;
  if (kparts > 1 && a.epi != ET_EPI_F32)
    return fail(ET_ERR_UNSUPPORTED, "FP32 linear: K > 768 needs the partial-sum (split-K) epilogue");
  if (a.epi == ET_EPI_PART16) return fail(ET_ERR_INVALID_ARG, "FP32 linear: 16-bit partials");
  if (a.K % 16) return fail(ET_ERR_UNSUPPORTED, "FP32 linear: K must be a multiple of 16");
  if (a.M <= 0) return ET_OK;
  G32Params p{};
  p.X = static_cast<const float*>(a.X) + a.k0;
  p.M = a.M;
  p.ldx = a.ldx;
  p.K = a.K;
  p.Kp = kparts > 1 ? 768 : a.K;
  p.kparts = kparts;
  p.nseg = a.nseg;
  int rows = 0;
  for (int s = 0; s < a.nseg; ++s) {
    p.row_begin[s] = rows;
    rows += a.seg[s].tile_rows;
    p.prp[s] = a.seg[s].row_ptr;
    p.tile_col[s] = a.seg[s].tile_col;
    p.values[s] = static_cast<const float*>(a.seg[s].values);
    p.bias[s] = static_cast<const float*>(a.seg[s].bias);
    p.tile_rows[s] = a.seg[s].tile_rows;
    p.rp_stride[s] = a.seg[s].rp_stride ? a.seg[s].rp_stride : a.seg[s].tile_rows + 1;
    p.out_col[s] = a.seg[s].out_col;
    p.scale[s] = a.seg[s].scale;
    p.apply_scale[s] = a.seg[s].apply_scale;
  }
  p.row_begin[a.nseg] = rows;
  p.Y = static_cast<float*>(a.Y);
  p.ldy = a.ldy;
  p.part_stride = (long long)a.M * a.ldy;
  p.epi = a.epi;
  p.ts = a.ts;
  if (rows == 0) return ET_OK;
  dim3 grid(rows, (a.M + kTok - 1) / kTok, kparts);
  ET_CUDA(launch_pdl(gemm32_kernel, grid, dim3(256), 0, stream, p));
  count_launch();
  return ET_OK;
}

et_status attention32_run(const AttnArgs& a, cudaStream_t stream) {
  if (a.d_k > 128 || a.d_k <= 0) return fail(ET_ERR_UNSUPPORTED, "FP32 attention: d_k <= 128 (got %d)", a.d_k);
  if (a.batch <= 0 || a.seq_len <= 0 || a.head_end <= a.head_begin) return ET_OK;
  const size_t smem = (size_t)4 * a.seq_len * 4 + 4 * 128 * 4;
  if (smem > 227 * 1024) return fail(ET_ERR_UNSUPPORTED, "FP32 attention: seq_len %d too long", a.seq_len);
  static cudaError_t attr = cudaFuncSetAttribute(attn32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                 227 * 1024);
  ET_CUDA(attr);
  A32Params p{};
  p.qkv = static_cast<const float*>(a.qkv);
  p.ld_qkv = a.ld_qkv;
  p.q_off = a.q_off;
  p.k_off = a.k_off;
  p.v_off = a.v_off;
  p.v_col = a.v_col;
  p.v_width = a.v_width;
  p.Z = static_cast<float*>(a.Z);
  p.ld_z = a.ld_z;
  p.z_map = a.z_map;
  p.lengths = a.lengths;
  p.S = a.seq_len;
  p.d_k = a.d_k;
  p.head_begin = a.head_begin;
  p.causal = a.causal;
  p.scale = a.scale;
  p.ts = a.ts;
  dim3 grid((a.seq_len + 3) / 4, a.head_end - a.head_begin, a.batch);
  ET_CUDA(launch_pdl(attn32_kernel, grid, dim3(128), smem, stream, p));
  count_launch();
  return ET_OK;
}

}  // namespace et
