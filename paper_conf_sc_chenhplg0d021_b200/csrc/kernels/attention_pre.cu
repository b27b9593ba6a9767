// Pre-computed linear transformation operator (§3.1 Eq. 4-5, Fig. 3(b);
// SURVEY §8(f) NEXT-1):
//   Output = sum_h S_h . (X . W_VO,h) + b'      W_VO,h = W_V,h^T . W_O,h^T  (offline, d x d per head)
// with the attention-aware pattern of the pre-computed design (line 107, 317): W_O row-pruned, W_V
// dense, so every W_VO,h keeps the same d' output features (the kept rows of W_O) and the projection
// X . [||_h W_VO,h] is a dense [M, H*Dv] GEMM (Dv = d' rounded up to 16; the tile GEMM with a
// ratio-0 packed weight).  The constant b_V folds into b' = b_O + W_O' b_V (rows of S_h sum to 1).
//
// Two kernels here:
//   vo_precompute_kernel — the offline product W_VO (FP32 accumulation of the stored 16-bit
//     operands, rounded once) and the bias fold b';
//   attn_pre_kernel — steps 2-6 + 8 of Fig. 3(b) for seq_len <= 128: per (sequence, head group,
//     column chunk) CTA, for each head of the group: S = Q~_h K_h^T into TMEM (tcgen05), one thread
//     per query row takes max / exp / sum with the exponentials held in registers, writes the
//     NORMALISED P_h (16-bit) over the scores (heads are summed, so the normalisation cannot be
//     deferred as in the per-head forms), and the MMA warp accumulates P_h . (X W_VO,h) of every head
//     of the group into ONE TMEM accumulator (Eq. 5's sum over h, step 8, on the tensor core).
//     The group's sum leaves as one [M, d] partial plane (kept columns scattered through the row
//     map, pruned columns 0); the LayerNorm kernel adds the G planes, b' and the residual.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <mutex>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {

et_status make_tmap_2d(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                       uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows, bool swizzle128);

namespace {

__device__ __forceinline__ float to_f32(__half x) { return __half2float(x); }
__device__ __forceinline__ float to_f32(__nv_bfloat16 x) { return __bfloat162float(x); }
template <typename T> __device__ __forceinline__ T from_f32(float x);
template <> __device__ __forceinline__ __half from_f32<__half>(float x) { return __float2half_rn(x); }
template <> __device__ __forceinline__ __nv_bfloat16 from_f32<__nv_bfloat16>(float x) { return __float2bfloat16_rn(x); }

// ----------------------------------------------------------------- offline: W_VO and b'
// Wvo[h*Dv + j, k] = sum_{f < d_k} W_O[kept[j], h*d_k + f] * W_V[h*d_k + f, k]   (j < n_kept; else 0)
template <typename T>
__global__ void vo_precompute_kernel(const T* __restrict__ Wv, const T* __restrict__ Wo, const int32_t* __restrict__ kept,
                                     int n_kept, int heads, int d, int Dv, T* __restrict__ Wvo) {
  const int dk = d / heads;
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  const int row = blockIdx.y;   // h * Dv + j
  const int h = row / Dv, j = row % Dv;
  if (k >= d) return;
  float acc = 0.f;
  if (j < n_kept) {
    const int o = kept[j];
    for (int f = 0; f < dk; ++f)
      acc = fmaf(to_f32(Wo[(size_t)o * d + h * dk + f]), to_f32(Wv[(size_t)(h * dk + f) * d + k]), acc);
  }
  Wvo[(size_t)row * d + k] = from_f32<T>(acc);
}

// b'[o] = b_O[o] + sum_f W_O'[o, f] b_V[f], W_O' = W_O with the rows outside `kept` zeroed
template <typename T>
__global__ void bias_fold_kernel(const T* __restrict__ Wo, const T* __restrict__ bv, const T* __restrict__ bo,
                                 const int32_t* __restrict__ kept, int n_kept, int d, T* __restrict__ bout) {
  const int o = blockIdx.x * blockDim.x + threadIdx.x;
  if (o >= d) return;
  int lo = 0, hi = n_kept;   // kept is ascending
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (kept[mid] < o) lo = mid + 1; else hi = mid;
  }
  float acc = bo ? to_f32(bo[o]) : 0.f;
  if (bv && lo < n_kept && kept[lo] == o)
    for (int f = 0; f < d; ++f) acc = fmaf(to_f32(Wo[(size_t)o * d + f]), to_f32(bv[f]), acc);
  bout[o] = from_f32<T>(acc);
}

// ----------------------------------------------------------------- attention, Eq. 5 form
constexpr int kMaxD = 4096;      // d_model bound of the shared inverse row map
constexpr int kThreads = 160;   // warp 0: TMA + MMA issue; warps 1-4: softmax / epilogue (row = lane quarter)

struct PreParams {
  int S, d, dk, Dv;            // d_model, head width, packed VO width per head
  int q_off, k_off, vo_off;    // qkv' columns: Q_h at q_off + h d_k, K_h at k_off + h d_k, VO_h at vo_off + h Dv
  int G, nchunks;              // head groups (grid.y), 256-column chunks of Dv (grid.x)
  int heads;
  const int32_t* lengths;
  const int32_t* kept;         // [n_kept] ascending original output feature of packed column j
  int n_kept;
  void* planes;                // [G][M][d] partial planes (part dtype)
  int part_f32;
  size_t plane_elems;          // M * d
  int causal;
  float scale_log2;
  int box_rows;                // TMA box rows: min(128, tokens)
  int stages;                  // load stages (1 or 2)
  uint32_t qk_bytes, v_bytes;  // one stage: Q + K tiles, VO chunk tiles
  unsigned long long* ts;
};

template <bool kBF16, int kDK>
__global__ void __launch_bounds__(kThreads, 1) attn_pre_kernel(const __grid_constant__ CUtensorMap tmap,
                                                               const __grid_constant__ PreParams p) {
  constexpr int kT = kDK / 64;                  // 64-column SWIZZLE_128B boxes per Q / K tile
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t stage_bytes = p.qk_bytes + p.v_bytes;
  __shared__ uint64_t ld_full[2], ld_free[2], s_full, p_full, o_full;
  __shared__ uint32_t tslot;
  __shared__ int16_t s_inv[kMaxD];   // packed VO column of output feature o, -1 if W_O row o is pruned
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int chunk = blockIdx.x, g = blockIdx.y, b = blockIdx.z;
  const int h0 = g * p.heads / p.G, h1 = (g + 1) * p.heads / p.G, nh = h1 - h0;
  const int c0 = chunk * 256;
  const int Dc = min(256, p.Dv - c0);          // this CTA's packed VO columns [c0, c0 + Dc)
  const int row0 = b * p.S;
  const int nvbox = (Dc + 63) / 64;

  if (p.box_rows < 128) {
    // fewer than 128 tokens in the batch: rows the TMA box leaves untouched must be finite zeros
    for (int i = threadIdx.x; i < (int)(p.stages * stage_bytes / 16); i += blockDim.x)
      reinterpret_cast<uint4*>(smem)[i] = make_uint4(0u, 0u, 0u, 0u);
    fence_proxy_async_smem();
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&ld_full[i], 1);
      mbar_init(&ld_free[i], 1);
    }
    mbar_init(&s_full, 1);
    mbar_init(&p_full, 4);
    mbar_init(&o_full, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc<512>(&tslot);
  pdl_trigger();
  pdl_wait();
  for (int o = threadIdx.x; o < p.d; o += blockDim.x) {   // rank of o in the ascending kept list
    int lo = 0, hi = p.n_kept;
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (__ldg(p.kept + mid) < o) lo = mid + 1; else hi = mid;
    }
    s_inv[o] = (int16_t)((lo < p.n_kept && __ldg(p.kept + lo) == o) ? lo : -1);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tslot;   // S / P at [0, 128), O at [128, 128 + Dc)

  if (warp == 0) {
    auto load = [&](int i) {   // head h0 + i into stage i % stages
      const int st = i % p.stages, h = h0 + i;
      uint8_t* base = smem + st * stage_bytes;
      mbar_expect_tx(&ld_full[st], (uint32_t)(2 * kT + nvbox) * p.box_rows * 128);
      for (int t = 0; t < kT; ++t) {
        tma_load_2d(base + t * 16384, &tmap, &ld_full[st], p.q_off + h * kDK + t * 64, row0);
        tma_load_2d(base + (kT + t) * 16384, &tmap, &ld_full[st], p.k_off + h * kDK + t * 64, row0);
      }
      for (int t = 0; t < nvbox; ++t)
        tma_load_2d(base + p.qk_bytes + t * 16384, &tmap, &ld_full[st], p.vo_off + h * p.Dv + c0 + t * 64, row0);
    };
    if (lane == 0) {
      tma_prefetch_desc(&tmap);
      if (p.ts != nullptr) atomicMin(p.ts, globaltimer_ns());
      for (int i = 0; i < p.stages && i < nh; ++i) load(i);
    }
    __syncwarp();
    const uint32_t idesc_s = make_idesc_f16(128, 128, kBF16 ? 1 : 0, 0, 0);
    const uint32_t idesc_o = make_idesc_f16(128, Dc, kBF16 ? 1 : 0, 0, 1);   // VO MN-major
    for (int i = 0; i < nh; ++i) {
      const int st = i % p.stages;
      const uint32_t base = smem_u32(smem + st * stage_bytes);
      mbar_wait_warp(&ld_full[st], (i / p.stages) & 1);
      tc_fence_after();
#pragma unroll
      for (int ks = 0; ks < kDK / 16; ++ks) {
        const uint32_t off = (ks >> 2) * 16384 + (ks & 3) * 32;
        mma_ss_warp(tb, make_sdesc(base + off, 16, 1024, kLayoutSW128),
                    make_sdesc(base + kT * 16384 + off, 16, 1024, kLayoutSW128), idesc_s, ks > 0);
      }
      mma_commit_warp(&s_full);
      mbar_wait_warp(&p_full, i & 1);
      tc_fence_after();
      const uint32_t vb = base + p.qk_bytes;
#pragma unroll
      for (int ks = 0; ks < 8; ++ks)   // 128 keys = 8 x K16; P packed in TMEM columns [8 ks, 8 ks + 8)
        mma_ts_warp(tb + 128, tb + ks * 8, make_sdesc(vb + ks * 2048, 16384, 1024, kLayoutSW128), idesc_o,
                    (i > 0 || ks > 0) ? 1u : 0u);
      mma_commit_warp(&ld_free[st]);
      // the next S overwrites P and the next load this stage: both wait for these MMAs
      mbar_wait_warp(&ld_free[st], (i / p.stages) & 1);
      if (lane == 0 && i + p.stages < nh) load(i + p.stages);
      __syncwarp();
    }
    mma_commit_warp(&o_full);
  } else {
    const int quarter = warp & 3, r = quarter * 32 + lane;
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    const int len = p.lengths ? p.lengths[b] : p.S;   // after pdl_wait
    int kend = len;
    if (p.causal) kend = min(kend, r + 1);
    const bool full = kend >= 128;
    const float sl2 = p.scale_log2;
    for (int i = 0; i < nh; ++i) {
      mbar_wait_warp(&s_full, i & 1);
      tc_fence_after();
      float e[128];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        uint32_t v[32];
        tmem_ld32(tb + lane_off + c * 32, v);
        tmem_ld_wait();
#pragma unroll
        for (int t = 0; t < 32; ++t) e[c * 32 + t] = __uint_as_float(v[t]);
      }
      float m = -INFINITY;
#pragma unroll
      for (int t = 0; t < 128; ++t)
        if (full || t < kend) m = fmaxf(m, e[t]);
      const float mb = m * sl2;
      float l = 0.f;
#pragma unroll
      for (int t = 0; t < 128; ++t) {
        float x;
        asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(x) : "f"(fmaf(e[t], sl2, -mb)));
        e[t] = (full || t < kend) ? x : 0.f;
        l += e[t];
      }
      const float inv = 1.f / l;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        uint32_t pk[16];
#pragma unroll
        for (int t = 0; t < 32; t += 2) pk[t >> 1] = pack2<kBF16>(e[c * 32 + t] * inv, e[c * 32 + t + 1] * inv);
        tmem_st16(tb + lane_off + c * 16, pk);
      }
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full);
    }
    // ---- epilogue: the group's sum of heads, kept columns scattered to their output features
    mbar_wait_warp(&o_full, 0);
    tc_fence_after();
    // stage this warp's 32 rows of O (fp32) in shared memory (the load stages are free now)
    const int pitch = Dc + 4;   // floats; +4 keeps the row-per-lane stores off one bank
    float* stg = reinterpret_cast<float*>(smem) + (size_t)quarter * 32 * pitch;
    for (int c = 0; c < Dc; c += 32) {
      uint32_t v[32];
      tmem_ld32(tb + lane_off + 128 + c, v);
      tmem_ld_wait();
#pragma unroll
      for (int t = 0; t < 32; t += 4)
        if (c + t < Dc)
          *reinterpret_cast<float4*>(stg + lane * pitch + c + t) =
              make_float4(__uint_as_float(v[t]), __uint_as_float(v[t + 1]), __uint_as_float(v[t + 2]),
                          __uint_as_float(v[t + 3]));
    }
    __syncwarp();
    // warp-cooperative row writes: lane covers 8 consecutive output features (s_inv: packed column)
    const int d = p.d;
    for (int rr = 0; rr < 32; ++rr) {
      const int row = quarter * 32 + rr;
      if (row >= p.S) break;
      const float* src = stg + rr * pitch;
      const size_t obase = (size_t)g * p.plane_elems + (size_t)(row0 + row) * d;
      for (int o8 = lane * 8; o8 < d; o8 += 256) {
        float val[8];
        bool own[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int j = s_inv[o8 + u];
          own[u] = j >= 0 ? (j >= c0 && j < c0 + Dc) : chunk == 0;
          val[u] = (j >= c0 && j < c0 + Dc) ? src[j - c0] : 0.f;
        }
        if (p.nchunks == 1) {
          if (p.part_f32) {
            float* dst = static_cast<float*>(p.planes) + obase + o8;
            *reinterpret_cast<float4*>(dst) = make_float4(val[0], val[1], val[2], val[3]);
            *reinterpret_cast<float4*>(dst + 4) = make_float4(val[4], val[5], val[6], val[7]);
          } else {
            *reinterpret_cast<uint4*>(static_cast<uint16_t*>(p.planes) + obase + o8) =
                make_uint4(pack2<kBF16>(val[0], val[1]), pack2<kBF16>(val[2], val[3]), pack2<kBF16>(val[4], val[5]),
                           pack2<kBF16>(val[6], val[7]));
          }
        } else {
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            if (!own[u]) continue;
            if (p.part_f32) {
              static_cast<float*>(p.planes)[obase + o8 + u] = val[u];
            } else {
              const uint32_t w = pack2<kBF16>(val[u], 0.f);
              static_cast<uint16_t*>(p.planes)[obase + o8 + u] = (uint16_t)(w & 0xffffu);
            }
          }
        }
      }
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  trace_cta_end(p.ts);
  if (warp == 0) {
    __syncwarp();
    tc_fence_after();
    tmem_dealloc<512>(tb);
  }
}

template <bool kBF16, int kDK>
et_status launch_pre(const CUtensorMap& tm, const PreParams& prm, dim3 grid, size_t smem, cudaStream_t stream) {
  auto kern = attn_pre_kernel<kBF16, kDK>;
  static std::once_flag once;
  static cudaError_t err = cudaSuccess;
  std::call_once(once, [&] { err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                         (int)(227 * 1024 - sizeof(int16_t) * kMaxD - 256)); });
  ET_CUDA(err);
  ET_CUDA(launch_pdl(kern, grid, dim3(kThreads), smem, stream, tm, prm));
  count_launch();
  return ET_OK;
}

}  // namespace

et_status vo_precompute_run(const VoPrep& v, cudaStream_t stream) {
  const int d = v.d_model, Dv = (v.n_kept + 15) / 16 * 16;
  if (v.n_kept < 0 || v.n_kept > d) return fail(ET_ERR_INVALID_ARG, "precompute: n_kept out of range");
  if (v.n_kept == 0) {   // every W_O row pruned: W_VO is empty, b' = b_O
    if (v.bias_out && v.bo) ET_CUDA(cudaMemcpyAsync(v.bias_out, v.bo, (size_t)d * dtype_size(v.dtype), cudaMemcpyDeviceToDevice, stream));
    else if (v.bias_out) ET_CUDA(cudaMemsetAsync(v.bias_out, 0, (size_t)d * dtype_size(v.dtype), stream));
    return ET_OK;
  }
  dim3 grid((d + 127) / 128, v.heads * Dv);
  if (v.dtype == ET_BF16) {
    using T = __nv_bfloat16;
    vo_precompute_kernel<T><<<grid, 128, 0, stream>>>(static_cast<const T*>(v.wv), static_cast<const T*>(v.wo), v.kept,
                                                      v.n_kept, v.heads, d, Dv, static_cast<T*>(v.wvo_out));
    if (v.bias_out)
      bias_fold_kernel<T><<<(d + 127) / 128, 128, 0, stream>>>(static_cast<const T*>(v.wo), static_cast<const T*>(v.bv),
                                                               static_cast<const T*>(v.bo), v.kept, v.n_kept, d,
                                                               static_cast<T*>(v.bias_out));
  } else {
    using T = __half;
    vo_precompute_kernel<T><<<grid, 128, 0, stream>>>(static_cast<const T*>(v.wv), static_cast<const T*>(v.wo), v.kept,
                                                      v.n_kept, v.heads, d, Dv, static_cast<T*>(v.wvo_out));
    if (v.bias_out)
      bias_fold_kernel<T><<<(d + 127) / 128, 128, 0, stream>>>(static_cast<const T*>(v.wo), static_cast<const T*>(v.bv),
                                                               static_cast<const T*>(v.bo), v.kept, v.n_kept, d,
                                                               static_cast<T*>(v.bias_out));
  }
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

int attention_pre_groups(int batch, int heads, int Dv) {
  const int nchunks = (Dv + 255) / 256;
  int G = (148 + batch * nchunks - 1) / (batch * nchunks);   // about one wave of CTAs
  return std::max(1, std::min(G, std::min(heads, 4)));   // the LayerNorm kernel sums up to 4 planes
}

et_status attention_pre_run(const PreArgs& a, cudaStream_t stream) {
  if (a.dtype != ET_FP16 && a.dtype != ET_BF16) return fail(ET_ERR_UNSUPPORTED, "pre-computed operator: FP16 / BF16");
  if (a.d_k != 64 && a.d_k != 128) return fail(ET_ERR_UNSUPPORTED, "pre-computed operator: d_k 64 or 128");
  if (a.d > kMaxD) return fail(ET_ERR_UNSUPPORTED, "pre-computed operator: d_model <= %d", kMaxD);
  if (a.seq_len > 128) return fail(ET_ERR_UNSUPPORTED, "pre-computed operator: seq_len <= 128 (one key block)");
  if (a.Dv % 16 || a.Dv <= 0) return fail(ET_ERR_INVALID_ARG, "pre-computed operator: Dv must be a positive multiple of 16");
  if (!aligned16(a.qkv) || (a.ld_qkv * 2) % 16 || !aligned16(a.planes) || a.d % 8)
    return fail(ET_ERR_INVALID_ARG, "pre-computed operator: 16-byte aligned rows required");
  const uint64_t rows = (uint64_t)a.batch * a.seq_len;
  const uint32_t box_rows = rows < 128 ? (uint32_t)rows : 128u;
  CUtensorMap tm;
  ET_TRY(make_tmap_2d(&tm, a.qkv, a.dtype, rows, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64, box_rows, true));
  PreParams prm{};
  prm.S = a.seq_len;
  prm.d = a.d;
  prm.dk = a.d_k;
  prm.Dv = a.Dv;
  prm.q_off = a.q_off;
  prm.k_off = a.k_off;
  prm.vo_off = a.vo_off;
  prm.heads = a.heads;
  prm.G = a.groups;
  prm.nchunks = (a.Dv + 255) / 256;
  prm.lengths = a.lengths;
  prm.kept = a.kept;
  prm.n_kept = a.n_kept;
  prm.planes = a.planes;
  prm.part_f32 = a.part_dtype == ET_FP32 ? 1 : 0;
  prm.plane_elems = rows * (uint64_t)a.d;
  prm.causal = a.causal;
  prm.scale_log2 = a.scale * 1.4426950408889634f;
  prm.box_rows = (int)box_rows;
  prm.ts = a.ts;
  const int Dc = std::min(256, a.Dv);
  prm.qk_bytes = 2u * (a.d_k / 64) * 16384u;
  prm.v_bytes = (uint32_t)((Dc + 63) / 64) * 16384u;
  const size_t staging = (size_t)128 * (Dc + 4) * 4;
  const size_t stage = prm.qk_bytes + prm.v_bytes;
  prm.stages = (2 * stage <= 208 * 1024) ? 2 : 1;
  const size_t smem = 1024 + std::max(prm.stages * stage, staging);
  if (smem > 227 * 1024 - sizeof(int16_t) * kMaxD - 256) return fail(ET_ERR_UNSUPPORTED, "pre-computed operator: shared memory");
  dim3 grid(prm.nchunks, a.groups, a.batch);
  const bool bf = a.dtype == ET_BF16;
  if (a.d_k == 64) return bf ? launch_pre<true, 64>(tm, prm, grid, smem, stream) : launch_pre<false, 64>(tm, prm, grid, smem, stream);
  return bf ? launch_pre<true, 128>(tm, prm, grid, smem, stream) : launch_pre<false, 128>(tm, prm, grid, smem, stream);
}

}  // namespace et
