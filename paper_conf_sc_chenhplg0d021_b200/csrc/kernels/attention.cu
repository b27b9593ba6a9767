// On-the-fly attention operator on tcgen05 (§3.1, Fig. 3(a) steps 2-6):
//   per (sequence b, head h, 128-query block):  S = Q~_h K_h^T  (Q~ pre-scaled by 1/sqrt(d_k), the
//   reordering of line 159 §3.3), mask (keys j >= len_b, and j > i if causal: probability exactly 0,
//   line 73), row softmax, Z_h = P V_h with the normalisation deferred to the end (line 361).
// The seq x seq score matrix never leaves TMEM / registers (the point of OTF: no intermediate
// result written to or read from global memory, line 99, 109).
//
// Two forms (line 133-147 §3.2: the sequence-length-aware switch):
//   short (kLong = false, seq_len <= 256): the whole score row of every query lives in TMEM
//     (S: up to 256 fp32 columns), exact two-pass softmax over it, one P.V accumulation over all keys
//     — the paper's OTF operator with the row tile kept on chip (Eq. 6's budget becomes TMEM).
//   long (kLong = true): K/V streamed in 128-key blocks (double-buffered S in TMEM, TMA ring),
//     online softmax (running max m, running sum l, O rescaled by exp(m_old - m_new)); the
//     per-block P.V result is accumulated in registers.  Replaces the paper's "partial OTF"
//     (QK^T materialised in global memory) — S x S never touches HBM.
// Roles: warp 0 TMA producer, warp 1 MMA issuer (+ TMEM owner), warps 2-5 softmax / epilogue with
// one thread per query row (thread t of warp w owns TMEM lane 32*(w%4) + t: row statistics need no
// shuffles).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <mutex>
#include <type_traits>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {

et_status make_tmap_2d(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                       uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows, bool swizzle128);

namespace {

constexpr int kThreads = 192;
constexpr float kLog2e = 1.4426950408889634f;

struct AParams {
  int S, H, head_begin;
  int q_off, k_off, v_off;
  const int32_t* v_col;     // [H] or null
  const int32_t* v_width;   // [H] or null
  const int32_t* z_map;     // [packed V width] destination column of each packed V column (-1 = skip) or null
  const int32_t* lengths;   // [B] or null
  void* Z;
  int ld_z;
  int causal;
  int dv_max;               // MMA N for P.V (multiple of 16, <= kDK)
  float scale_log2;         // scale * log2(e)
  int box_rows;             // TMA box height: min(128, total rows)
};

template <int kDK>
struct Cfg {
  static constexpr int kTiles = kDK / 64;            // 64-wide SW128 tiles per 128-row operand
  static constexpr int kOpBytes = 128 * kDK * 2;     // one 128-row Q / K / V block
};

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

template <bool kBF16, int kDK, bool kLong>
__global__ void __launch_bounds__(kThreads, 1) attn_kernel(const __grid_constant__ CUtensorMap tmap,
                                                           const __grid_constant__ AParams p) {
  using C = Cfg<kDK>;
  constexpr int kStages = 2;   // K/V ring (the short form holds its <= 2 blocks resident)
  if (p.v_width && p.v_width[p.head_begin + blockIdx.y] == 0) return;   // every V feature of the head pruned
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + C::kOpBytes;                       // kStages x K block
  uint8_t* sV = sK + kStages * C::kOpBytes;             // kStages x V block
  uint64_t* bars = reinterpret_cast<uint64_t*>(sV + kStages * C::kOpBytes);
  uint64_t* q_full = bars + 0;
  uint64_t* kv_full = bars + 1;       // [2]
  uint64_t* kv_empty = bars + 3;      // [2]
  uint64_t* s_full = bars + 5;        // [2]
  uint64_t* s_free = bars + 7;        // [2]
  uint64_t* p_full = bars + 9;        // [2]
  uint64_t* o_full = bars + 11;
  uint64_t* o_free = bars + 12;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 13);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int qb = blockIdx.x;
  const int h = p.head_begin + blockIdx.y;
  const int b = blockIdx.z;
  const int S = p.S;
  const int len = p.lengths ? p.lengths[b] : S;
  // keys needed by this query block: [0, kmax)
  int kmax = len;
  if (p.causal) kmax = min(kmax, qb * 128 + 128);
  const int nkb = (kmax + 127) / 128;
  const int row0 = b * S;   // first token row of this sequence
  const int qcol = p.q_off + h * kDK, kcol = p.k_off + h * kDK;
  const int vcol = p.v_off + (p.v_col ? p.v_col[h] : h * kDK);
  const int vw = p.v_width ? p.v_width[h] : kDK;
  const int dvn = p.dv_max;   // P.V MMA N

  // TMEM columns
  constexpr int kS = 0;                    // S: [0, 256) (short: all blocks; long: 2 buffers)
  constexpr int kP = 256;                  // P: [256, 384) fp16 pairs, 64 columns per 128 keys
  constexpr int kO = 384;                  // O: [384, 384 + dv)

  if (p.box_rows < 128) {
    // tiny problem: the TMA box covers fewer than 128 rows; zero the V staging so that the rows
    // it leaves untouched are finite (P = 0 there, but 0 * NaN would poison O)
    for (int i = threadIdx.x; i < 2 * C::kOpBytes / 16; i += blockDim.x)
      reinterpret_cast<uint4*>(sV)[i] = make_uint4(0, 0, 0, 0);
    fence_proxy_async_smem();
  }
  if (threadIdx.x == 0) {
    mbar_init(q_full, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
      mbar_init(&s_full[i], 1);
      mbar_init(&s_free[i], 4);
      mbar_init(&p_full[i], 4);
    }
    mbar_init(o_full, 1);
    mbar_init(o_free, 4);
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;

  if (warp == 0) {
    // ================= TMA producer: Q once, then K/V blocks through a 2-stage ring
    if (lane == 0) {
      tma_prefetch_desc(&tmap);
      const uint32_t tile_bytes = (uint32_t)p.box_rows * 128;   // one 64-column tile
      mbar_expect_tx(q_full, tile_bytes * C::kTiles);
      for (int t = 0; t < C::kTiles; ++t)
        tma_load_2d(sQ + t * 16384, &tmap, q_full, qcol + t * 64, row0 + qb * 128);
      for (int j = 0; j < nkb; ++j) {
        const int st = j & 1;
        if (j >= 2) mbar_wait(&kv_empty[st], ((j >> 1) - 1) & 1);
        mbar_expect_tx(&kv_full[st], 2 * tile_bytes * C::kTiles);
        for (int t = 0; t < C::kTiles; ++t) {
          tma_load_2d(sK + st * C::kOpBytes + t * 16384, &tmap, &kv_full[st], kcol + t * 64, row0 + j * 128);
          tma_load_2d(sV + st * C::kOpBytes + t * 16384, &tmap, &kv_full[st], vcol + t * 64, row0 + j * 128);
        }
      }
    }
  } else if (warp == 1) {
    // ================= MMA issuer (whole warp runs the loop; one elected lane issues)
    const uint32_t idesc_s = make_idesc_f16(128, 128, kBF16 ? 1 : 0, 0, 0);          // Q.K^T, N = 128 keys
    const uint32_t idesc_o = make_idesc_f16(128, dvn, kBF16 ? 1 : 0, 0, 1);          // P.V, V MN-major
    const uint32_t q_u = smem_u32(sQ);
    auto issue_qk = [&](int j, uint32_t s_col) {
      const uint32_t k_u = smem_u32(sK + (j & 1) * C::kOpBytes);
#pragma unroll
      for (int ks = 0; ks < kDK / 16; ++ks) {
        const uint32_t off = (ks >> 2) * 16384 + (ks & 3) * 32;
        mma_ss_warp(tbase + s_col, make_sdesc(q_u + off, 16, 1024, kLayoutSW128),
                    make_sdesc(k_u + off, 16, 1024, kLayoutSW128), idesc_s, ks > 0);
      }
    };
    auto issue_pv = [&](int j, uint32_t p_col, bool acc_first) {
      const uint32_t v_u = smem_u32(sV + (j & 1) * C::kOpBytes);
#pragma unroll
      for (int ks = 0; ks < 8; ++ks)   // 128 keys = 8 x K16; V MN-major SW128: 16 rows = 2048 B
        mma_ts_warp(tbase + kO, tbase + p_col + ks * 8, make_sdesc(v_u + ks * 2048, 16384, 1024, kLayoutSW128),
                    idesc_o, (acc_first || ks > 0) ? 1u : 0u);
    };
    mbar_wait_warp(q_full, 0);
    tc_fence_after();
    if constexpr (!kLong) {
      // short form: all score blocks, then one P.V chain over all keys
      for (int j = 0; j < nkb; ++j) {
        mbar_wait_warp(&kv_full[j], 0);
        tc_fence_after();
        issue_qk(j, kS + j * 128);
      }
      mma_commit_warp(&s_full[0]);
      mbar_wait_warp(&p_full[0], 0);
      tc_fence_after();
      for (int j = 0; j < nkb; ++j) issue_pv(j, kP + j * 64, j > 0);
      mma_commit_warp(o_full);
    } else {
      // long form: S double buffer; QK(j+1) overlaps softmax(j)
      for (int j = 0; j < nkb; ++j) {
        if (j == 0) {
          mbar_wait_warp(&kv_full[0], 0);
          tc_fence_after();
          issue_qk(0, kS);
          mma_commit_warp(&s_full[0]);
        }
        if (j + 1 < nkb) {
          const int jn = j + 1, bn = jn & 1;
          if (jn >= 2) mbar_wait_warp(&s_free[bn], ((jn >> 1) - 1) & 1);
          mbar_wait_warp(&kv_full[bn], (jn >> 1) & 1);
          tc_fence_after();
          issue_qk(jn, kS + bn * 128);
          mma_commit_warp(&s_full[bn]);
        }
        mbar_wait_warp(&p_full[j & 1], (j >> 1) & 1);
        if (j >= 1) mbar_wait_warp(o_free, (j - 1) & 1);
        tc_fence_after();
        issue_pv(j, kP + (j & 1) * 64, false);
        mma_commit_warp(o_full);
        mma_commit_warp(&kv_empty[j & 1]);
      }
    }
  } else {
    // ================= softmax / epilogue: one thread per query row
    const int quarter = warp & 3;
    const int r = quarter * 32 + lane;          // row within the block = TMEM lane
    const int qi = qb * 128 + r;                // query index within the sequence
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    int kend = len;                             // valid keys: [0, kend)
    if (p.causal) kend = min(kend, qi + 1);
    const float sl2 = p.scale_log2;
    float o[kLong ? kDK : 1];
#pragma unroll
    for (int c = 0; c < (kLong ? kDK : 1); ++c) o[c] = 0.f;
    float l = 0.f;

    if constexpr (!kLong) {
      mbar_wait_warp(&s_full[0], 0);
      tc_fence_after();
      // pass 1: row max over valid keys
      float m = -INFINITY;
      for (int j = 0; j < nkb; ++j) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t v[32];
          tmem_ld32(tbase + lane_off + kS + j * 128 + c * 32, v);
          tmem_ld_wait();
#pragma unroll
          for (int t = 0; t < 32; ++t) {
            const int key = j * 128 + c * 32 + t;
            if (key < kend) m = fmaxf(m, __uint_as_float(v[t]));
          }
        }
      }
      // pass 2: p = exp(s - m) (0 for masked keys), row sum, P -> TMEM (16-bit pairs)
      const float mb = m * sl2;
      for (int j = 0; j < nkb; ++j) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t v[32];
          tmem_ld32(tbase + lane_off + kS + j * 128 + c * 32, v);
          tmem_ld_wait();
          uint32_t pk[16];
#pragma unroll
          for (int t = 0; t < 32; t += 2) {
            const int key = j * 128 + c * 32 + t;
            const float p0 = key < kend ? ex2(__uint_as_float(v[t]) * sl2 - mb) : 0.f;
            const float p1 = key + 1 < kend ? ex2(__uint_as_float(v[t + 1]) * sl2 - mb) : 0.f;
            l += p0 + p1;
            pk[t >> 1] = pack2<kBF16>(p0, p1);
          }
          tmem_st16(tbase + lane_off + kP + j * 64 + c * 16, pk);
        }
      }
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[0]);
      mbar_wait_warp(o_full, 0);
      tc_fence_after();
    } else {
      float m = -INFINITY;
      for (int j = 0; j < nkb; ++j) {
        const int bj = j & 1;
        mbar_wait_warp(&s_full[bj], (j >> 1) & 1);
        tc_fence_after();
        // pass A: block max over valid keys (S read from TMEM, not kept in registers)
        float mblk = -INFINITY;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t v[32];
          tmem_ld32(tbase + lane_off + kS + bj * 128 + c * 32, v);
          tmem_ld_wait();
#pragma unroll
          for (int t = 0; t < 32; ++t)
            if (j * 128 + c * 32 + t < kend) mblk = fmaxf(mblk, __uint_as_float(v[t]));
        }
        const float m_new = fmaxf(m, mblk);
        const float alpha = (m == -INFINITY) ? 0.f : ex2((m - m_new) * sl2);
        const float mb = m_new * sl2;
        float lsum = 0.f;
        // pass B: p = exp(s - m_new) -> P(j) in TMEM buffer j&1 (its previous reader PV(j-2)
        // completed before o_full(j-1) was observed)
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t v[32];
          tmem_ld32(tbase + lane_off + kS + bj * 128 + c * 32, v);
          tmem_ld_wait();
          uint32_t pk[16];
#pragma unroll
          for (int t = 0; t < 32; t += 2) {
            const int key = j * 128 + c * 32 + t;
            const float p0 = key < kend ? ex2(__uint_as_float(v[t]) * sl2 - mb) : 0.f;
            const float p1 = key + 1 < kend ? ex2(__uint_as_float(v[t + 1]) * sl2 - mb) : 0.f;
            lsum += p0 + p1;
            pk[t >> 1] = pack2<kBF16>(p0, p1);
          }
          tmem_st16(tbase + lane_off + kP + bj * 64 + c * 16, pk);
        }
        tmem_st_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&s_free[bj]);   // S(j) consumed: its buffer may take QK(j+2)
          mbar_arrive(&p_full[bj]);
        }
        l = l * alpha + lsum;
        m = m_new;
        // O += P(j) V(j), rescaled
        mbar_wait_warp(o_full, j & 1);
        tc_fence_after();
#pragma unroll
        for (int c = 0; c < kDK; c += 32) {
          if (c < dvn) {
            uint32_t v[32];
            tmem_ld32(tbase + lane_off + kO + c, v);
            tmem_ld_wait();
#pragma unroll
            for (int t = 0; t < 32; ++t) o[c + t] = o[c + t] * alpha + __uint_as_float(v[t]);
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(o_free);
      }
    }

    // ---- epilogue: Z = O / l in 32-column chunks.  The TMEM loads are warp-collective
    // (.sync.aligned) and stay outside the per-row condition; only the stores are predicated on
    // the row lying inside the sequence.
    {
      using T = typename std::conditional<kBF16, __nv_bfloat16, __half>::type;
      const bool store = qi < S;
      const float inv = 1.0f / l;
      T* zrow = static_cast<T*>(p.Z) + (size_t)(row0 + qi) * p.ld_z;
      const int vloc = p.v_col ? p.v_col[h] : h * kDK;        // packed V column of this head
      const int32_t* zm = p.z_map ? p.z_map + vloc : nullptr;  // scatter map (row-pruned W_V)
      T* z = zrow + h * kDK;
#pragma unroll
      for (int c0 = 0; c0 < kDK; c0 += 32) {
        if (c0 < vw) {
          float x[32];
          if constexpr (kLong) {
#pragma unroll
            for (int t = 0; t < 32; ++t) x[t] = o[c0 + t];
          } else {
            uint32_t v[32];
            tmem_ld32(tbase + lane_off + kO + c0, v);
            tmem_ld_wait();
#pragma unroll
            for (int t = 0; t < 32; ++t) x[t] = __uint_as_float(v[t]);
          }
          if (!store) {
          } else if (zm) {
#pragma unroll
            for (int t = 0; t < 32; ++t)
              if (c0 + t < vw) {
                const int dst = zm[c0 + t];
                if (dst >= 0) {
                  if constexpr (kBF16) zrow[dst] = __float2bfloat16_rn(x[t] * inv);
                  else zrow[dst] = __float2half_rn(x[t] * inv);
                }
              }
          } else if ((vw & 7) == 0) {
#pragma unroll
            for (int t = 0; t < 32; t += 8) {
              if (c0 + t < vw) {
                uint4 u;
                u.x = pack2<kBF16>(x[t] * inv, x[t + 1] * inv);
                u.y = pack2<kBF16>(x[t + 2] * inv, x[t + 3] * inv);
                u.z = pack2<kBF16>(x[t + 4] * inv, x[t + 5] * inv);
                u.w = pack2<kBF16>(x[t + 6] * inv, x[t + 7] * inv);
                *reinterpret_cast<uint4*>(z + c0 + t) = u;
              }
            }
          } else {
#pragma unroll
            for (int t = 0; t < 32; ++t)
              if (c0 + t < vw) {
                if constexpr (kBF16) z[c0 + t] = __float2bfloat16_rn(x[t] * inv);
                else z[c0 + t] = __float2half_rn(x[t] * inv);
              }
          }
        }
      }
    }
  }

  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    __syncwarp();
    tc_fence_after();
    tmem_dealloc<512>(tbase);
  }
}

template <bool kBF16, int kDK, bool kLong>
et_status launch(const CUtensorMap& tm, const AParams& prm, dim3 grid, cudaStream_t stream) {
  auto kern = attn_kernel<kBF16, kDK, kLong>;
  const size_t smem = 1024 + (size_t)(1 + 2 * 2) * Cfg<kDK>::kOpBytes + 256;
  static std::once_flag once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(once, [&] { attr_err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); });
  ET_CUDA(attr_err);
  kern<<<grid, kThreads, smem, stream>>>(tm, prm);
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

}  // namespace

int attn_short_max(int d_k) { return (d_k == 64 || d_k == 128) ? 256 : 0; }

et_status attention_run(const AttnArgs& a, cudaStream_t stream) {
  if (a.dtype == ET_FP32) return fail(ET_ERR_UNSUPPORTED, "attention: FP32 not implemented in this build");
  if (a.d_k != 64 && a.d_k != 128) return fail(ET_ERR_UNSUPPORTED, "attention: d_k must be 64 or 128 (got %d)", a.d_k);
  if (a.v_width_max <= 0 || a.v_width_max > a.d_k || a.v_width_max % 16)
    return fail(ET_ERR_INVALID_ARG, "attention: V width must be a multiple of 16 and <= d_k");
  if (!a.long_form && a.seq_len > 256) return fail(ET_ERR_UNSUPPORTED, "attention: short form needs seq_len <= 256");
  if (a.batch <= 0 || a.seq_len <= 0 || a.head_end <= a.head_begin) return ET_OK;
  if (!aligned16(a.qkv) || (a.ld_qkv * 2) % 16) return fail(ET_ERR_INVALID_ARG, "attention: QKV not 16B aligned");
  CUtensorMap tm;
  const uint32_t box_rows = (uint64_t)a.batch * a.seq_len < 128 ? (uint32_t)(a.batch * a.seq_len) : 128u;
  ET_TRY(make_tmap_2d(&tm, a.qkv, a.dtype, (uint64_t)a.batch * a.seq_len, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64,
                      box_rows, true));
  AParams prm{};
  prm.S = a.seq_len;
  prm.H = a.heads;
  prm.head_begin = a.head_begin;
  prm.q_off = a.q_off;
  prm.k_off = a.k_off;
  prm.v_off = a.v_off;
  prm.v_col = a.v_col;
  prm.v_width = a.v_width;
  prm.z_map = a.z_map;
  prm.lengths = a.lengths;
  prm.Z = a.Z;
  prm.ld_z = a.ld_z;
  prm.causal = a.causal;
  prm.dv_max = a.v_width_max;
  prm.scale_log2 = a.scale * kLog2e;
  const long long rows = (long long)a.batch * a.seq_len;
  prm.box_rows = rows < 128 ? (int)rows : 128;
  dim3 grid((a.seq_len + 127) / 128, a.head_end - a.head_begin, a.batch);
  const bool bf = a.dtype == ET_BF16;
  if (a.d_k == 64) {
    if (a.long_form) return bf ? launch<true, 64, true>(tm, prm, grid, stream) : launch<false, 64, true>(tm, prm, grid, stream);
    return bf ? launch<true, 64, false>(tm, prm, grid, stream) : launch<false, 64, false>(tm, prm, grid, stream);
  }
  if (a.long_form) return bf ? launch<true, 128, true>(tm, prm, grid, stream) : launch<false, 128, true>(tm, prm, grid, stream);
  return bf ? launch<true, 128, false>(tm, prm, grid, stream) : launch<false, 128, false>(tm, prm, grid, stream);
}

}  // namespace et
