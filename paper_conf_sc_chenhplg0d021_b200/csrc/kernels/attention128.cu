// On-the-fly attention for short sequences (seq_len <= 128, d_k = 64): the BERT-base / C3 shape.
// Same operator as attention.cu's short form (§3.1, Fig. 3(a) steps 2-6, with
// the 1/sqrt(d_k) scale already applied to Q, line 159 §3.3, and the normalisation deferred to the
// end, line 361), specialised so that THREE CTAs share an SM instead of two:
//   * one thread per query row (4 softmax warps, TMEM lane quarter = warp % 4): the whole 128-key
//     score row is owned by one thread, so P can overwrite the scores it was computed from;
//   * TMEM 128 columns: S = Q K^T in [0, 128) (fp32), P written back in place as 16-bit pairs in
//     [0, 64) (pass 2 writes columns [16c, 16c+16) only after reading [32c, 32c+32)), O = P V in
//     [64, 128) (scores there are dead once every row has produced its P);
//   * shared memory 64 KB: Q, K, V (one 128 x 64 SWIZZLE_128B tile each) + Z staging.
// The score matrix never leaves TMEM / registers.  Roles: warp 0 issues the TMA loads and the two
// MMA chains (one elected lane), warps 1-4 run the softmax and the epilogue.
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

constexpr int kThreads = 160;           // warp 0 control, warps 1-4 softmax / epilogue
constexpr int kTile = 128 * 64 * 2;     // one 128-row x 64-column 16-bit operand (SWIZZLE_128B)
constexpr int kStageWarp = 32 * 128;    // Z staging: 32 rows x 64 columns x 2 B per softmax warp
constexpr size_t kSmem = 1024 + 3 * kTile + 4 * kStageWarp + 128;
constexpr float kLog2e = 1.4426950408889634f;

struct A128Params {
  int S, head_begin;
  int q_off, k_off, v_off;
  const int32_t* lengths;   // [B] or null
  void* Z;
  int ld_z;
  int causal;
  float scale_log2;         // scale * log2(e)
  int box_rows;             // TMA box height: min(128, total rows)
  int tma_store;            // Z through TMA stores (seq_len % 32 == 0)
  unsigned long long* ts;   // trace slot or nullptr
};

__device__ __forceinline__ float ex2f(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

template <bool kBF16>
__global__ void __launch_bounds__(kThreads, 3) attn128_kernel(const __grid_constant__ CUtensorMap tmap,
                                                              const __grid_constant__ CUtensorMap tmap_z,
                                                              const __grid_constant__ A128Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + kTile;
  uint8_t* sV = sK + kTile;
  uint8_t* sStage = sV + kTile;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sStage + 4 * kStageWarp);
  uint64_t* qk_full = bars + 0;
  uint64_t* v_full = bars + 1;
  uint64_t* s_full = bars + 2;
  uint64_t* p_full = bars + 3;
  uint64_t* o_full = bars + 4;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 5);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int h = p.head_begin + blockIdx.x;
  const int b = blockIdx.y;
  const int S = p.S;
  const int row0 = b * S;   // first token row of this sequence

  if (p.box_rows < 128) {
    // tiny problem: the TMA box covers fewer than 128 rows; zero V so the rows it leaves untouched
    // are finite (their P is 0, but 0 * NaN would poison O)
    for (int i = threadIdx.x; i < kTile / 16; i += blockDim.x) reinterpret_cast<uint4*>(sV)[i] = make_uint4(0, 0, 0, 0);
    fence_proxy_async_smem();
  }
  if (threadIdx.x == 0) {
    mbar_init(qk_full, 1);
    mbar_init(v_full, 1);
    mbar_init(s_full, 1);
    mbar_init(p_full, 4);
    mbar_init(o_full, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc<128>(tmem_slot);
  pdl_trigger();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;

  if (warp == 0) {
    // ================= loads + MMA issue
    if (lane == 0) {
      tma_prefetch_desc(&tmap);
      pdl_wait();   // QKV of the predecessor is visible from here
      if (p.ts != nullptr) atomicMin(p.ts, globaltimer_ns());
      const uint32_t tile_bytes = (uint32_t)p.box_rows * 128;
      mbar_expect_tx(qk_full, 2 * tile_bytes);
      tma_load_2d(sQ, &tmap, qk_full, p.q_off + h * 64, row0);
      tma_load_2d(sK, &tmap, qk_full, p.k_off + h * 64, row0);
      mbar_expect_tx(v_full, tile_bytes);
      tma_load_2d(sV, &tmap, v_full, p.v_off + h * 64, row0);
    }
    __syncwarp();
    const uint32_t idesc_s = make_idesc_f16(128, 128, kBF16 ? 1 : 0, 0, 0);   // S = Q K^T, N = 128 keys
    const uint32_t idesc_o = make_idesc_f16(128, 64, kBF16 ? 1 : 0, 0, 1);    // O = P V, V MN-major
    mbar_wait_warp(qk_full, 0);
    tc_fence_after();
    const uint32_t q_u = smem_u32(sQ), k_u = smem_u32(sK), v_u = smem_u32(sV);
#pragma unroll
    for (int ks = 0; ks < 4; ++ks)   // d_k = 64 = 4 x K16; K-major SW128: 16 columns = 32 B
      mma_ss_warp(tbase, make_sdesc(q_u + ks * 32, 16, 1024, kLayoutSW128), make_sdesc(k_u + ks * 32, 16, 1024, kLayoutSW128),
                  idesc_s, ks > 0);
    mma_commit_warp(s_full);
    mbar_wait_warp(p_full, 0);
    mbar_wait_warp(v_full, 0);
    tc_fence_after();
#pragma unroll
    for (int ks = 0; ks < 8; ++ks)   // 128 keys = 8 x K16; P packed in TMEM columns [8 ks, 8 ks + 8)
      mma_ts_warp(tbase + 64, tbase + ks * 8, make_sdesc(v_u + ks * 2048, 16384, 1024, kLayoutSW128), idesc_o,
                  ks > 0 ? 1u : 0u);
    mma_commit_warp(o_full);
  } else {
    // ================= softmax / epilogue: thread = query row r (TMEM lane r)
    const int quarter = warp & 3;
    const int r = quarter * 32 + lane;
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    const int len = p.lengths ? p.lengths[b] : S;
    int kend = len;                              // valid keys [0, kend)
    if (p.causal) kend = min(kend, r + 1);
    const float sl2 = p.scale_log2;
    mbar_wait_warp(s_full, 0);
    tc_fence_after();
    // pass 1: row maximum over the valid keys (8 independent partial maxima: no 128-long chain;
    // rows with every key valid skip the per-key predicate)
    const bool full = kend >= 128;
    float mx8[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) mx8[i] = -INFINITY;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      uint32_t v[32];
      tmem_ld32(tbase + lane_off + c * 32, v);
      tmem_ld_wait();
      if (full) {
#pragma unroll
        for (int t = 0; t < 32; ++t) mx8[t & 7] = fmaxf(mx8[t & 7], __uint_as_float(v[t]));
      } else {
#pragma unroll
        for (int t = 0; t < 32; ++t)
          if (c * 32 + t < kend) mx8[t & 7] = fmaxf(mx8[t & 7], __uint_as_float(v[t]));
      }
    }
    const float m = fmaxf(fmaxf(fmaxf(mx8[0], mx8[1]), fmaxf(mx8[2], mx8[3])),
                          fmaxf(fmaxf(mx8[4], mx8[5]), fmaxf(mx8[6], mx8[7])));
    const float mb = m * sl2;
    // pass 2: p = 2^(s log2e - m log2e) (exactly 0 for masked keys), row sum (4 packed partial
    // sums), P in place; the exponent arguments two at a time (FFMA2)
    uint64_t ls4[4] = {0ull, 0ull, 0ull, 0ull};
    const uint64_t sl2x2 = f2pk(sl2, sl2), nmb2 = f2pk(-mb, -mb);
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      uint32_t v[32];
      tmem_ld32(tbase + lane_off + c * 32, v);
      tmem_ld_wait();
      uint32_t pk[16];
#pragma unroll
      for (int t = 0; t < 32; t += 2) {
        const float2 x = f2upk(ffma2(f2pk(__uint_as_float(v[t]), __uint_as_float(v[t + 1])), sl2x2, nmb2));
        float p0 = ex2f(x.x), p1 = ex2f(x.y);
        if (!full) {
          p0 = c * 32 + t < kend ? p0 : 0.f;
          p1 = c * 32 + t + 1 < kend ? p1 : 0.f;
        }
        ls4[(t >> 1) & 3] = fadd2(ls4[(t >> 1) & 3], f2pk(p0, p1));
        pk[t >> 1] = pack2<kBF16>(p0, p1);
      }
      tmem_st16(tbase + lane_off + c * 16, pk);
    }
    const float2 la = f2upk(fadd2(fadd2(ls4[0], ls4[1]), fadd2(ls4[2], ls4[3])));
    const float l = la.x + la.y;
    tmem_st_wait();
    tc_fence_before();
    __syncwarp();
    if (lane == 0) mbar_arrive(p_full);
    mbar_wait_warp(o_full, 0);
    tc_fence_after();
    // epilogue: Z = O / l, 64 columns of row r
    const float inv = 1.0f / l;
    uint32_t o[64];
    tmem_ld32(tbase + lane_off + 64, *reinterpret_cast<uint32_t(*)[32]>(o));
    tmem_ld32(tbase + lane_off + 96, *reinterpret_cast<uint32_t(*)[32]>(o + 32));
    tmem_ld_wait();
    const bool tma_warp = p.tma_store && quarter * 32 < S;   // all 32 rows of this warp in the sequence
    if (tma_warp) {
      uint8_t* st = sStage + (warp - 1) * kStageWarp;
      // 128-byte rows, SWIZZLE_128B: 16-byte unit c of row i at c ^ (i % 8)
#pragma unroll
      for (int ch = 0; ch < 8; ++ch) {
        const float* x = reinterpret_cast<const float*>(o) + ch * 8;
        *reinterpret_cast<uint4*>(st + lane * 128 + ((ch ^ (lane & 7)) << 4)) =
            make_uint4(pack2<kBF16>(x[0] * inv, x[1] * inv), pack2<kBF16>(x[2] * inv, x[3] * inv),
                       pack2<kBF16>(x[4] * inv, x[5] * inv), pack2<kBF16>(x[6] * inv, x[7] * inv));
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
        tma_store_2d(&tmap_z, st, h * 64, row0 + quarter * 32);
        bulk_commit_group();
        bulk_wait_group<0>();
      }
    } else if (r < S) {
      uint16_t* z = static_cast<uint16_t*>(p.Z) + (size_t)(row0 + r) * p.ld_z + h * 64;
#pragma unroll
      for (int t = 0; t < 64; t += 8) {
        const float* x = reinterpret_cast<const float*>(o) + t;
        *reinterpret_cast<uint4*>(z + t) =
            make_uint4(pack2<kBF16>(x[0] * inv, x[1] * inv), pack2<kBF16>(x[2] * inv, x[3] * inv),
                       pack2<kBF16>(x[4] * inv, x[5] * inv), pack2<kBF16>(x[6] * inv, x[7] * inv));
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
    tmem_dealloc<128>(tbase);
  }
}

template <bool kBF16>
et_status launch128(const CUtensorMap& tm, const CUtensorMap& tz, const A128Params& prm, dim3 grid,
                    cudaStream_t stream) {
  auto kern = attn128_kernel<kBF16>;
  static std::once_flag once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(once, [&] { attr_err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem); });
  ET_CUDA(attr_err);
  ET_CUDA(launch_pdl(kern, grid, dim3(kThreads), kSmem, stream, tm, tz, prm));
  count_launch();
  return ET_OK;
}

}  // namespace

bool attention128_applies(const AttnArgs& a) {
  return !a.long_form && a.d_k == 64 && a.seq_len <= 128 && a.v_col == nullptr && a.v_width == nullptr &&
         a.z_map == nullptr && a.v_width_max == 64 && a.dtype != ET_FP32;
}

et_status attention128_run(const AttnArgs& a, cudaStream_t stream) {
  const uint64_t rows = (uint64_t)a.batch * a.seq_len;
  const uint32_t box_rows = rows < 128 ? (uint32_t)rows : 128u;
  CUtensorMap tm, tz;
  ET_TRY(make_tmap_2d(&tm, a.qkv, a.dtype, rows, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64, box_rows, true));
  A128Params prm{};
  prm.S = a.seq_len;
  prm.head_begin = a.head_begin;
  prm.q_off = a.q_off;
  prm.k_off = a.k_off;
  prm.v_off = a.v_off;
  prm.lengths = a.lengths;
  prm.Z = a.Z;
  prm.ld_z = a.ld_z;
  prm.causal = a.causal;
  prm.scale_log2 = a.scale * kLog2e;
  prm.box_rows = (int)box_rows;
  prm.ts = a.ts;
  prm.tma_store = (a.seq_len % 32 == 0 && rows >= 32 && aligned16(a.Z) && (a.ld_z * 2) % 16 == 0) ? 1 : 0;
  if (prm.tma_store) {
    ET_TRY(make_tmap_2d(&tz, a.Z, a.dtype, rows, (uint64_t)a.ld_z, (uint64_t)a.ld_z, 64, 32, true));
  } else {
    tz = tm;   // unused
  }
  dim3 grid(a.head_end - a.head_begin, a.batch);
  return a.dtype == ET_BF16 ? launch128<true>(tm, tz, prm, grid, stream) : launch128<false>(tm, tz, prm, grid, stream);
}

}  // namespace et
