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
et_status make_tmap_3d_ld(CUtensorMap* tm, void* base, et_dtype dtype, uint64_t cols, uint64_t rows, uint64_t planes,
                          uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows);

namespace {

struct PParams {
  int S, H, head_begin, nh;   // nh = heads in the call
  int q_off, k_off, v_off;
  const int32_t* lengths;
  int ld_s;                   // row pitch of the [B * nh][S][ld_s] 16-bit score buffer (tensor map)
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
// One CTA per (128-query block, batch x head): Q resident in shared memory, K blocks of 128 keys
// streamed through a TMA ring, two 128-column TMEM accumulators so the epilogue of key block kb
// overlaps the MMAs of kb + 1, and the 16-bit score tile leaving through shared memory by TMA
// store (whole 128-byte lines; rows / keys past seq_len are clipped by the tensor map).
// warp 0: TMA producer, warp 1: MMA issuer + TMEM owner, warps 2-5: epilogue (TMEM lane quarter w%4).
template <int kDK> struct QktCfg {
  static constexpr int kTiles = kDK / 64;               // 64-column SWIZZLE_128B boxes per operand
  static constexpr int kOpBytes = kTiles * 16384;       // one 128-row Q or K block
  static constexpr int kKS = kDK == 64 ? 4 : 2;         // K ring stages (one CTA per SM; 2 stages measured slower)
  static constexpr int kStage = 32768;                  // one 128 x 128 16-bit score tile (two boxes)
  static constexpr int kSmem = 1024 + kOpBytes * (1 + kKS) + 2 * kStage;
};

template <bool kBF16, int kDK>
__global__ void __launch_bounds__(192, 1) qkt_kernel(const __grid_constant__ CUtensorMap tmap,
                                                     const __grid_constant__ CUtensorMap tmap_s,
                                                     const __grid_constant__ PParams p) {
  using C = QktCfg<kDK>;
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  const int qb = blockIdx.x, bh = blockIdx.y;
  const int b = bh / p.nh, h = p.head_begin + bh % p.nh;
  const int len = p.lengths ? p.lengths[b] : p.S;
  // key blocks kernel B reads: keys < len, and <= the block's last query when causal
  int nkb = (len + 127) / 128;
  if (p.causal) nkb = min(nkb, qb + 1);
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = smem + C::kOpBytes;
  uint8_t* sO = sK + C::kKS * C::kOpBytes;
  __shared__ uint64_t q_full, k_full[C::kKS], k_free[C::kKS], acc_full[2], acc_free[2];
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&q_full, 1);
    for (int i = 0; i < C::kKS; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_free[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_free[i], 4);
    }
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<256>(&tslot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tslot;
  const int row0 = b * p.S;
  const uint32_t op_tx = (uint32_t)C::kTiles * p.box_rows * 128;
  if (warp == 0) {
    if (lane == 0) {
      mbar_expect_tx(&q_full, op_tx);
      for (int t = 0; t < C::kTiles; ++t)
        tma_load_2d(sQ + t * 16384, &tmap, &q_full, p.q_off + h * kDK + t * 64, row0 + qb * 128);
      for (int kb = 0; kb < nkb; ++kb) {
        const int st = kb % C::kKS;
        if (kb >= C::kKS) mbar_wait(&k_free[st], ((kb / C::kKS) - 1) & 1);
        mbar_expect_tx(&k_full[st], op_tx);
        for (int t = 0; t < C::kTiles; ++t)
          tma_load_2d(sK + st * C::kOpBytes + t * 16384, &tmap, &k_full[st], p.k_off + h * kDK + t * 64,
                      row0 + kb * 128);
      }
    }
  } else if (warp == 1) {
    const uint32_t idesc = make_idesc_f16(128, 128, kBF16 ? 1 : 0, 0, 0);
    mbar_wait_warp(&q_full, 0);
    for (int kb = 0; kb < nkb; ++kb) {
      const int st = kb % C::kKS, a = kb & 1;
      if (kb >= 2) mbar_wait_warp(&acc_free[a], ((kb >> 1) - 1) & 1);
      mbar_wait_warp(&k_full[st], (kb / C::kKS) & 1);
      tc_fence_after();
      const uint32_t qu = smem_u32(sQ), ku = smem_u32(sK + st * C::kOpBytes);
#pragma unroll
      for (int ks = 0; ks < kDK / 16; ++ks) {
        const uint32_t off = (ks >> 2) * 16384 + (ks & 3) * 32;
        mma_ss_warp(tb + a * 128, make_sdesc(qu + off, 16, 1024, kLayoutSW128),
                    make_sdesc(ku + off, 16, 1024, kLayoutSW128), idesc, ks > 0);
      }
      mma_commit_warp(&k_free[st]);
      mma_commit_warp(&acc_full[a]);
    }
  } else {
    const int q = warp & 3, r = q * 32 + lane;
    const bool leader = warp == 2 && lane == 0;
    for (int kb = 0; kb < nkb; ++kb) {
      const int a = kb & 1;
      uint8_t* stg = sO + a * C::kStage;
      if (leader) bulk_wait_group_read<1>();   // the store issued from this buffer two tiles ago has read it
      named_bar_sync(1, 128);
      mbar_wait(&acc_full[a], (kb >> 1) & 1);
      tc_fence_after();
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        uint32_t v[32];
        tmem_ld32(tb + a * 128 + ((uint32_t)(q * 32) << 16) + c * 32, v);
        tmem_ld_wait();
        uint8_t* rowp = stg + (c >> 1) * 16384 + r * 128;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int unit = (c & 1) * 4 + u;
          *reinterpret_cast<uint4*>(rowp + ((unit ^ (r & 7)) << 4)) =
              make_uint4(pack2<kBF16>(__uint_as_float(v[8 * u]), __uint_as_float(v[8 * u + 1])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 2]), __uint_as_float(v[8 * u + 3])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 4]), __uint_as_float(v[8 * u + 5])),
                         pack2<kBF16>(__uint_as_float(v[8 * u + 6]), __uint_as_float(v[8 * u + 7])));
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free[a]);
      fence_proxy_async_smem();
      named_bar_sync(1, 128);
      if (leader) {
        tma_store_3d(&tmap_s, stg, kb * 128, qb * 128, bh);
        tma_store_3d(&tmap_s, stg + 16384, kb * 128 + 64, qb * 128, bh);
        bulk_commit_group();
      }
    }
    if (leader) bulk_wait_group<0>();
  }
  tc_fence_before();
  __syncthreads();
  trace_cta_end(p.ts);
  if (warp == 1) tmem_dealloc<256>(tb);
}

// ----------------------------------------------------------------- kernel B: mask, softmax, x V
// One CTA per (128-query block, batch x head).  The block's score rows stream through a TMA ring of
// 128 x 64-key tiles twice: pass 0 takes the row maxima, pass 1 (key blocks in reverse) turns each tile into P = exp(S - max)
// IN PLACE (same SWIZZLE_128B layout: the tile is then the K-major A operand) and the MMA warp
// accumulates P . V_block into TMEM.  The second pass hits L2 (a CTA's rows: 128 x seq_len x 2 B).
// warps 0-3: one query row per thread (TMEM lane = row); warp 4: MMA issuer + TMEM owner + releaser
// of pass-0 tiles; warp 5: TMA producer (score tiles, and in pass 1 the V blocks).
template <int kDK> struct PvCfg {
  static constexpr int kSS = 3;                       // score ring stages (16 KB each; d_k 64: 3 CTAs per SM)
  static constexpr int kVT = kDK / 64;                // 64-wide column tiles of a V block
  static constexpr int kVBytes = kVT * 64 * 128;      // 64 keys x d_k 16-bit (MN-major, SWIZZLE_128B)
  static constexpr int kSmem = 1024 + kSS * 16384 + 2 * kVBytes;
};

template <bool kBF16, int kDK>
__global__ void __launch_bounds__(192, 1) softmax_pv_kernel(const __grid_constant__ CUtensorMap tmap_s,
                                                            const __grid_constant__ CUtensorMap tmap_v,
                                                            const __grid_constant__ PParams p) {
  using C = PvCfg<kDK>;
  pdl_trigger();
  pdl_wait();
  trace_cta_start(p.ts);
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sS = smem;                        // kSS x (128 rows x 64 keys), K-major SWIZZLE_128B
  uint8_t* sV = smem + C::kSS * 16384;       // 2 x kVBytes
  __shared__ uint64_t s_full[C::kSS], s_free[C::kSS], p_full[C::kSS], v_full[2], v_free[2], o_full;
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
    for (int i = 0; i < C::kSS; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&s_free[i], 1);
      mbar_init(&p_full[i], 4);
    }
    for (int i = 0; i < 2; ++i) {
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
    for (int i = threadIdx.x; i < C::kVBytes / 16; i += blockDim.x)
      reinterpret_cast<uint4*>(sV)[i] = make_uint4(0u, 0u, 0u, 0u);
    fence_proxy_async_smem();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tslot;
  const int ni = 2 * nkb;   // pass 0: it = j, pass 1: it = nkb + j

  if (warp == 5) {
    if (lane == 0) {
      const uint32_t vbox = (uint32_t)p.vbox_rows * 128u;
      for (int it = 0; it < ni; ++it) {
        // pass 1 walks the key blocks backwards: the tiles pass 0 read last are still in L2
        const int st = it % C::kSS, j = it < nkb ? it : ni - 1 - it;
        if (it >= C::kSS) mbar_wait(&s_free[st], ((it / C::kSS) - 1) & 1);
        mbar_expect_tx(&s_full[st], 16384u);
        tma_load_3d(sS + st * 16384, &tmap_s, &s_full[st], j * 64, qb * 128, bh);
        if (it >= nkb) {
          const int jj = it - nkb, vs = jj & 1;   // jj: pass-1 step
          if (jj >= 2) mbar_wait(&v_free[vs], ((jj >> 1) - 1) & 1);
          mbar_expect_tx(&v_full[vs], C::kVT * vbox);
          for (int t = 0; t < C::kVT; ++t)
            tma_load_2d(sV + vs * C::kVBytes + t * 8192, &tmap_v, &v_full[vs], p.v_off + h * kDK + t * 64,
                        row0 + j * 64);
        }
      }
    }
  } else if (warp == 4) {
    const uint32_t idesc = make_idesc_f16(128, kDK, kBF16 ? 1 : 0, 0, 1);   // P K-major, V MN-major
    for (int it = 0; it < ni; ++it) {
      const int st = it % C::kSS;
      mbar_wait_warp(&p_full[st], (it / C::kSS) & 1);
      if (it < nkb) {   // pass 0: the softmax warps have read the tile
        if (lane == 0) mbar_arrive(&s_free[st]);
        __syncwarp();
        continue;
      }
      const int j = it - nkb, vs = j & 1;   // pass-1 step (key block nkb - 1 - j)
      mbar_wait_warp(&v_full[vs], (j >> 1) & 1);
      tc_fence_after();
      const uint32_t pu = smem_u32(sS + st * 16384), vu = smem_u32(sV + vs * C::kVBytes);
#pragma unroll
      for (int ks = 0; ks < 4; ++ks)   // 64 keys = 4 x K16; V: 16 keys = 16 rows x 128 B = 2048 B
        mma_ss_warp(tb, make_sdesc(pu + ks * 32, 16, 1024, kLayoutSW128),
                    make_sdesc(vu + ks * 2048, 8192, 1024, kLayoutSW128), idesc, (j > 0 || ks > 0) ? 1u : 0u);
      mma_commit_warp(&s_free[st]);
      mma_commit_warp(&v_free[vs]);
    }
    mma_commit_warp(&o_full);
  } else {
    const int r = warp * 32 + lane, qi = qb * 128 + r;
    int kend = len;
    if (p.causal) kend = min(kend, qi + 1);
    const float sl2 = p.scale_log2;
    using T2 = typename std::conditional<kBF16, __nv_bfloat162, __half2>::type;
    // pass 0: row max over the valid keys (packed 16-bit max; masking only in the tile holding kend)
    T2 m2;
    {
      const uint32_t ninf = kBF16 ? 0xFF80FF80u : 0xFC00FC00u;
      m2 = *reinterpret_cast<const T2*>(&ninf);
    }
    for (int j = 0; j < nkb; ++j) {
      const int it = j, st = it % C::kSS;
      mbar_wait(&s_full[st], (it / C::kSS) & 1);
      const uint8_t* rowp = sS + st * 16384 + r * 128;
      const int k0 = j * 64;
      if (k0 + 64 <= kend) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const uint4 w = *reinterpret_cast<const uint4*>(rowp + ((u ^ (r & 7)) << 4));
          m2 = __hmax2(m2, __hmax2(__hmax2(*reinterpret_cast<const T2*>(&w.x), *reinterpret_cast<const T2*>(&w.y)),
                                   __hmax2(*reinterpret_cast<const T2*>(&w.z), *reinterpret_cast<const T2*>(&w.w))));
        }
      } else if (k0 < kend) {
        float mf = -INFINITY;
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const uint4 w = *reinterpret_cast<const uint4*>(rowp + ((u ^ (r & 7)) << 4));
          const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float2 f = unpack2<kBF16>(ww[i]);
            const int k = k0 + u * 8 + 2 * i;
            if (k < kend) mf = fmaxf(mf, f.x);
            if (k + 1 < kend) mf = fmaxf(mf, f.y);
          }
        }
        const uint32_t mp = pack2<kBF16>(mf, mf);   // exact: mf is a 16-bit value
        m2 = __hmax2(m2, *reinterpret_cast<const T2*>(&mp));
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[st]);
    }
    float m;
    {
      const uint32_t mu = *reinterpret_cast<const uint32_t*>(&m2);
      const float2 mf = unpack2<kBF16>(mu);
      m = fmaxf(mf.x, mf.y);
    }
    const float mb = m * sl2;
    float l = 0.f;
    // pass 1: P = exp(S - max) in place, 16-bit, K-major A operand of P . V
    for (int jj = 0; jj < nkb; ++jj) {
      const int it = nkb + jj, st = it % C::kSS, j = nkb - 1 - jj;
      mbar_wait(&s_full[st], (it / C::kSS) & 1);
      uint8_t* rowp = sS + st * 16384 + r * 128;
      const int k0 = j * 64;
      const bool full = k0 + 64 <= kend;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        uint4* cell = reinterpret_cast<uint4*>(rowp + ((u ^ (r & 7)) << 4));
        const uint4 w = *cell;
        const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
        uint32_t pk[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 f = unpack2<kBF16>(ww[i]);
          const int k = k0 + u * 8 + 2 * i;
          float p0 = ex2p(f.x * sl2 - mb), p1 = ex2p(f.y * sl2 - mb);
          if (!full) {
            p0 = k < kend ? p0 : 0.f;
            p1 = k + 1 < kend ? p1 : 0.f;
          }
          pk[i] = pack2<kBF16>(p0, p1);
          // the row sum takes P as rounded, so that Z = (P . V) / l normalises what the MMA used
          const float2 pr = unpack2<kBF16>(pk[i]);
          l += pr.x + pr.y;
        }
        *cell = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[st]);
    }
    // Z = O / l (deferred normalisation, line 361)
    mbar_wait_warp(&o_full, 0);
    tc_fence_after();
    const float inv = 1.f / l;
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
et_status launch_partial(const CUtensorMap& tm, const CUtensorMap& ts, const CUtensorMap& tv, const PParams& prm,
                         int batch, cudaStream_t stream) {
  const size_t smem_a = QktCfg<kDK>::kSmem, smem_b = PvCfg<kDK>::kSmem;
  static std::once_flag once;
  static cudaError_t err = cudaSuccess;
  std::call_once(once, [&] {
    err = cudaFuncSetAttribute(qkt_kernel<kBF16, kDK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_a);
    if (err == cudaSuccess)
      err = cudaFuncSetAttribute(softmax_pv_kernel<kBF16, kDK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_b);
  });
  ET_CUDA(err);
  const int nqb = (prm.S + 127) / 128;
  ET_CUDA(launch_pdl(qkt_kernel<kBF16, kDK>, dim3(nqb, batch * prm.nh), dim3(192), smem_a, stream, tm, ts, prm));
  count_launch();
  ET_CUDA(launch_pdl(softmax_pv_kernel<kBF16, kDK>, dim3(nqb, batch * prm.nh), dim3(192), smem_b, stream, ts, tv, prm));
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
  prm.ld_s = (a.seq_len + 7) / 8 * 8;
  prm.Z = a.Z;
  prm.ld_z = a.ld_z;
  prm.causal = a.causal;
  prm.scale_log2 = a.scale * 1.4426950408889634f;
  prm.box_rows = (int)box_rows;
  prm.vbox_rows = rows < 64 ? (int)rows : 64;
  prm.ts = a.ts;
  CUtensorMap ts;
  ET_TRY(make_tmap_3d_ld(&ts, scores, a.dtype, (uint64_t)a.seq_len, (uint64_t)a.seq_len, (uint64_t)a.batch * nh,
                         (uint64_t)prm.ld_s, 64, 128));
  const bool bf = a.dtype == ET_BF16;
  if (a.d_k == 64)
    return bf ? launch_partial<true, 64>(tm, ts, tv, prm, a.batch, stream)
              : launch_partial<false, 64>(tm, ts, tv, prm, a.batch, stream);
  return bf ? launch_partial<true, 128>(tm, ts, tv, prm, a.batch, stream)
            : launch_partial<false, 128>(tm, ts, tv, prm, a.batch, stream);
}

}  // namespace et
