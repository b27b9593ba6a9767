// Paper-literal "partial OTF" attention (§3.2, Fig. 8 at line 236; the switch at
// seq 224, line 244): for long sequences the paper breaks steps 3 (Q.K^T) and 6 (x V) out of the
// on-the-fly operator —
//   kernel A: the outer-product GEMM  S = Q~_h K_h^T  over the whole GPU, written to global memory
//             (16-bit: the paper's "pure FP16", line 157-159; Q~ is pre-scaled by 1/sqrt(d_k), the
//             reordering that keeps FP16 scores from overflowing), then a global synchronisation
//             (the kernel boundary);
//   kernel B: steps 4-6 per row — mask (keys j >= len_b, j > i if causal), exact two-pass row softmax
//             over the stored scores, P = exp(S - max) rounded to 16 bit, Z = (P V_h) / rowsum.
// SURVEY §8(f) NEXT-2.  This is the baseline the repo's long form (attention.cu kLong: S x S never in
// HBM) replaces; it exists to reproduce the paper's Fig. 8 trade-off on B200 (tools/sweeps.py M3).
// Both kernels run on tcgen05: A is one M=128, N=128, K=d_k MMA chain per (query block, key block);
// B streams 64-key blocks of P (written by the softmax threads into SWIZZLE_128B shared memory) and
// V (TMA, MN-major) into an M=128, N=d_k accumulation in TMEM.  Dense V only (row-pruned V: the
// short / long forms).
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

struct PParams {
  int S, H, head_begin, nh;   // nh = heads in the call
  int q_off, k_off, v_off;
  const int32_t* lengths;
  uint16_t* scores;           // [B * nh][S][ld_s] 16-bit
  int ld_s;
  void* Z;
  int ld_z;
  int causal;
  float scale_log2;
  int box_rows;               // Q / K box rows (min(128, tokens))
  int vbox_rows;              // V box rows (min(64, tokens))
  unsigned long long* ts;
};

__device__ __forceinline__ float ex2p(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// ----------------------------------------------------------------- kernel A: S = Q~ K^T to global
template <bool kBF16, int kDK>
__global__ void __launch_bounds__(128, 1) qkt_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ PParams p) {
  constexpr int kTiles = kDK / 64;
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  const int qb = blockIdx.x, kb = blockIdx.y, bh = blockIdx.z;
  const int b = bh / p.nh, h = p.head_begin + bh % p.nh;
  const int len = p.lengths ? p.lengths[b] : p.S;
  // blocks kernel B never reads: keys past the valid length, or above the diagonal when causal
  if (kb * 128 >= len || (p.causal && kb > qb)) {
    trace_cta_end(p.ts);
    return;
  }
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = smem + kTiles * 16384;
  __shared__ uint64_t full, done;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&full, 1);
    mbar_init(&done, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc<128>(&tslot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tslot;
  const int row0 = b * p.S;
  if (warp == 0) {
    if (lane == 0) {
      const uint32_t tile = (uint32_t)p.box_rows * 128;
      mbar_expect_tx(&full, 2 * kTiles * tile);
      for (int t = 0; t < kTiles; ++t) {
        tma_load_2d(sQ + t * 16384, &tmap, &full, p.q_off + h * kDK + t * 64, row0 + qb * 128);
        tma_load_2d(sK + t * 16384, &tmap, &full, p.k_off + h * kDK + t * 64, row0 + kb * 128);
      }
    }
    mbar_wait_warp(&full, 0);
    tc_fence_after();
    const uint32_t idesc = make_idesc_f16(128, 128, kBF16 ? 1 : 0, 0, 0);
#pragma unroll
    for (int ks = 0; ks < kDK / 16; ++ks) {
      const uint32_t off = (ks >> 2) * 16384 + (ks & 3) * 32;
      mma_ss_warp(tb, make_sdesc(smem_u32(sQ) + off, 16, 1024, kLayoutSW128),
                  make_sdesc(smem_u32(sK) + off, 16, 1024, kLayoutSW128), idesc, ks > 0);
    }
    mma_commit_warp(&done);
  }
  mbar_wait_warp(&done, 0);
  tc_fence_after();
  // each thread: its query row's 128 scores -> 16-bit -> global (256 contiguous bytes per row)
  const int qi = qb * 128 + warp * 32 + lane;
  uint16_t* dst = p.scores + ((size_t)bh * p.S + qi) * p.ld_s + kb * 128;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    uint32_t v[32];
    tmem_ld32(tb + ((uint32_t)(warp * 32) << 16) + c * 32, v);
    tmem_ld_wait();
    if (qi < p.S) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int k = kb * 128 + c * 32 + u * 8;
        if (k < p.S)   // S % 8 == 0: whole 16-byte groups
          *reinterpret_cast<uint4*>(dst + c * 32 + u * 8) =
              make_uint4(pack2<kBF16>(__uint_as_float(v[8 * u]), __uint_as_float(v[8 * u + 1])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 2]), __uint_as_float(v[8 * u + 3])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 4]), __uint_as_float(v[8 * u + 5])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 6]), __uint_as_float(v[8 * u + 7])));
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  trace_cta_end(p.ts);
  if (warp == 0) tmem_dealloc<128>(tb);
}

// ----------------------------------------------------------------- kernel B: mask, softmax, x V
// warps 0-3: one query row per thread (TMEM lane = row); warp 4: MMA issuer + TMEM owner; warp 5:
// TMA producer of the V blocks.  64-key blocks, P and V double-buffered.
template <bool kBF16, int kDK>
__global__ void __launch_bounds__(192, 1) softmax_pv_kernel(const __grid_constant__ CUtensorMap tmap_v,
                                                            const __grid_constant__ PParams p) {
  constexpr int kVT = kDK / 64;              // 64-wide column tiles of a V block
  constexpr int kVBytes = kVT * 64 * 128;    // 64 keys x d_k 16-bit (MN-major, SWIZZLE_128B)
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sP = smem;                        // 2 x 16 KB: 128 rows x 64 keys, K-major SWIZZLE_128B
  uint8_t* sV = smem + 2 * 16384;            // 2 x kVBytes
  __shared__ uint64_t p_full[2], p_free[2], v_full[2], v_free[2], o_full;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int qb = blockIdx.x, bh = blockIdx.y;
  const int b = bh / p.nh, h = p.head_begin + bh % p.nh;
  const int S = p.S;
  const int len = p.lengths ? p.lengths[b] : S;
  int kmax = len;
  if (p.causal) kmax = min(kmax, qb * 128 + 128);
  const int nkb = (kmax + 63) / 64;
  const int row0 = b * S;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&p_full[i], 4);
      mbar_init(&p_free[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_free[i], 1);
    }
    mbar_init(&o_full, 1);
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<(kDK <= 32 ? 32 : kDK)>(&tslot);
  if (p.vbox_rows < 64) {
    // fewer than 64 tokens in the whole batch (one key block): the V rows the box does not cover
    // must be finite zeros, not stale shared memory (P is 0 there, but 0 x NaN is NaN)
    for (int i = threadIdx.x; i < kVBytes / 16; i += blockDim.x)
      reinterpret_cast<uint4*>(sV)[i] = make_uint4(0u, 0u, 0u, 0u);
    fence_proxy_async_smem();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tslot;

  if (warp == 5) {
    if (lane == 0) {
      const uint32_t box = (uint32_t)p.vbox_rows * 128u;   // 64 keys (fewer if the batch is shorter) x 64 columns
      for (int j = 0; j < nkb; ++j) {
        const int st = j & 1;
        if (j >= 2) mbar_wait(&v_free[st], ((j >> 1) - 1) & 1);
        mbar_expect_tx(&v_full[st], kVT * box);
        for (int t = 0; t < kVT; ++t)
          tma_load_2d(sV + st * kVBytes + t * 8192, &tmap_v, &v_full[st], p.v_off + h * kDK + t * 64, row0 + j * 64);
      }
    }
  } else if (warp == 4) {
    const uint32_t idesc = make_idesc_f16(128, kDK, kBF16 ? 1 : 0, 0, 1);   // P K-major, V MN-major
    for (int j = 0; j < nkb; ++j) {
      const int st = j & 1;
      mbar_wait_warp(&p_full[st], (j >> 1) & 1);
      mbar_wait_warp(&v_full[st], (j >> 1) & 1);
      tc_fence_after();
      const uint32_t pu = smem_u32(sP + st * 16384), vu = smem_u32(sV + st * kVBytes);
#pragma unroll
      for (int ks = 0; ks < 4; ++ks)   // 64 keys = 4 x K16; V: 16 keys = 16 rows x 128 B = 2048 B
        mma_ss_warp(tb, make_sdesc(pu + ks * 32, 16, 1024, kLayoutSW128),
                    make_sdesc(vu + ks * 2048, 8192, 1024, kLayoutSW128), idesc, (j > 0 || ks > 0) ? 1u : 0u);
      mma_commit_warp(&p_free[st]);
      mma_commit_warp(&v_free[st]);
    }
    mma_commit_warp(&o_full);
  } else {
    const int r = warp * 32 + lane, qi = qb * 128 + r;
    int kend = len;
    if (p.causal) kend = min(kend, qi + 1);
    const uint16_t* srow = p.scores + ((size_t)bh * S + min(qi, S - 1)) * p.ld_s;
    const float sl2 = p.scale_log2;
    // pass 1: row max over the valid keys (stored 16-bit scores, read 8 at a time)
    float m = -INFINITY;
    for (int k = 0; k < kend; k += 8) {
      const uint4 w = __ldg(reinterpret_cast<const uint4*>(srow + k));
      const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 f = unpack2<kBF16>(ww[i]);
        if (k + 2 * i < kend) m = fmaxf(m, f.x);
        if (k + 2 * i + 1 < kend) m = fmaxf(m, f.y);
      }
    }
    const float mb = m * sl2;
    float l = 0.f;
    // pass 2: P = exp(S - max) per 64-key block into the shared-memory A operand
    for (int j = 0; j < nkb; ++j) {
      const int st = j & 1;
      if (j >= 2) mbar_wait(&p_free[st], ((j >> 1) - 1) & 1);
      uint8_t* prow = sP + st * 16384 + r * 128;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int k = j * 64 + u * 8;
        uint4 w = make_uint4(0u, 0u, 0u, 0u);
        if (k < kend) w = __ldg(reinterpret_cast<const uint4*>(srow + k));
        const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
        uint32_t pk[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 f = unpack2<kBF16>(ww[i]);
          const float p0 = k + 2 * i < kend ? ex2p(f.x * sl2 - mb) : 0.f;
          const float p1 = k + 2 * i + 1 < kend ? ex2p(f.y * sl2 - mb) : 0.f;
          l += p0 + p1;
          pk[i] = pack2<kBF16>(p0, p1);
        }
        *reinterpret_cast<uint4*>(prow + ((u ^ (r & 7)) << 4)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[st]);
    }
    // Z = O / l (deferred normalisation, line 361)
    mbar_wait_warp(&o_full, 0);
    tc_fence_after();
    const float inv = l > 0.f ? 1.f / l : 0.f;
    using T = typename std::conditional<kBF16, __nv_bfloat16, __half>::type;
#pragma unroll
    for (int c = 0; c < kDK; c += 32) {
      uint32_t v[32];
      tmem_ld32(tb + ((uint32_t)(warp * 32) << 16) + c, v);
      tmem_ld_wait();
      if (qi < S) {
        T* z = static_cast<T*>(p.Z) + (size_t)(row0 + qi) * p.ld_z + (h - p.head_begin) * kDK + c;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          *reinterpret_cast<uint4*>(z + 8 * u) =
              make_uint4(pack2<kBF16>(__uint_as_float(v[8 * u]) * inv, __uint_as_float(v[8 * u + 1]) * inv),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 2]) * inv, __uint_as_float(v[8 * u + 3]) * inv),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 4]) * inv, __uint_as_float(v[8 * u + 5]) * inv),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 6]) * inv, __uint_as_float(v[8 * u + 7]) * inv));
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  trace_cta_end(p.ts);
  if (warp == 4) tmem_dealloc<(kDK <= 32 ? 32 : kDK)>(tb);
}

template <bool kBF16, int kDK>
et_status launch_partial(const CUtensorMap& tm, const CUtensorMap& tv, const PParams& prm, int batch,
                         unsigned long long* ts_a, cudaStream_t stream) {
  const size_t smem_a = 1024 + 2 * (kDK / 64) * 16384;
  const size_t smem_b = 1024 + 2 * 16384 + 2 * (kDK / 64) * 8192;
  static std::once_flag once;
  static cudaError_t err = cudaSuccess;
  std::call_once(once, [&] {
    err = cudaFuncSetAttribute(qkt_kernel<kBF16, kDK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_a);
    if (err == cudaSuccess)
      err = cudaFuncSetAttribute(softmax_pv_kernel<kBF16, kDK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_b);
  });
  ET_CUDA(err);
  const int nqb = (prm.S + 127) / 128;
  PParams pa = prm;
  pa.ts = ts_a;
  ET_CUDA(launch_pdl(qkt_kernel<kBF16, kDK>, dim3(nqb, nqb, batch * prm.nh), dim3(128), smem_a, stream, tm, pa));
  count_launch();
  ET_CUDA(launch_pdl(softmax_pv_kernel<kBF16, kDK>, dim3(nqb, batch * prm.nh), dim3(192), smem_b, stream, tv, prm));
  count_launch();
  return ET_OK;
}

}  // namespace

size_t attention_partial_scores_bytes(int batch, int seq_len, int heads) {
  const size_t ld = (size_t)(seq_len + 7) / 8 * 8;
  return (size_t)batch * heads * seq_len * ld * 2;
}

et_status attention_partial_run(const AttnArgs& a, void* scores, size_t scores_bytes, cudaStream_t stream) {
  if (a.dtype != ET_FP16 && a.dtype != ET_BF16)
    return fail(ET_ERR_UNSUPPORTED, "partial OTF attention: FP16 / BF16 (the paper's 16-bit scores)");
  if (a.d_k != 64 && a.d_k != 128) return fail(ET_ERR_UNSUPPORTED, "partial OTF attention: d_k 64 or 128");
  if (a.v_col || a.v_width || a.z_map)
    return fail(ET_ERR_UNSUPPORTED, "partial OTF attention: dense V only (row-pruned V: short / long forms)");
  if (a.seq_len % 8) return fail(ET_ERR_UNSUPPORTED, "partial OTF attention: seq_len must be a multiple of 8");
  const int nh = a.head_end - a.head_begin;
  if (a.batch <= 0 || nh <= 0) return ET_OK;
  if (scores_bytes < attention_partial_scores_bytes(a.batch, a.seq_len, nh) || !aligned16(scores))
    return fail(ET_ERR_WORKSPACE, "partial OTF attention: score buffer too small / unaligned");
  if (!aligned16(a.qkv) || (a.ld_qkv * 2) % 16 || !aligned16(a.Z) || (a.ld_z * 2) % 16)
    return fail(ET_ERR_INVALID_ARG, "partial OTF attention: 16-byte aligned QKV / Z rows required");
  const uint64_t rows = (uint64_t)a.batch * a.seq_len;
  const uint32_t box_rows = rows < 128 ? (uint32_t)rows : 128u;
  CUtensorMap tm, tv;
  ET_TRY(make_tmap_2d(&tm, a.qkv, a.dtype, rows, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64, box_rows, true));
  ET_TRY(make_tmap_2d(&tv, a.qkv, a.dtype, rows, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64, rows < 64 ? (uint32_t)rows : 64u, true));
  PParams prm{};
  prm.S = a.seq_len;
  prm.H = a.heads;
  prm.head_begin = a.head_begin;
  prm.nh = nh;
  prm.q_off = a.q_off;
  prm.k_off = a.k_off;
  prm.v_off = a.v_off;
  prm.lengths = a.lengths;
  prm.scores = static_cast<uint16_t*>(scores);
  prm.ld_s = (a.seq_len + 7) / 8 * 8;
  prm.Z = a.Z;
  prm.ld_z = a.ld_z;
  prm.causal = a.causal;
  prm.scale_log2 = a.scale * 1.4426950408889634f;
  prm.box_rows = (int)box_rows;
  prm.vbox_rows = rows < 64 ? (int)rows : 64;
  prm.ts = a.ts;
  const bool bf = a.dtype == ET_BF16;
  if (a.d_k == 64)
    return bf ? launch_partial<true, 64>(tm, tv, prm, a.batch, a.ts, stream)
              : launch_partial<false, 64>(tm, tv, prm, a.batch, a.ts, stream);
  return bf ? launch_partial<true, 128>(tm, tv, prm, a.batch, a.ts, stream)
            : launch_partial<false, 128>(tm, tv, prm, a.batch, a.ts, stream);
}

}  // namespace et
