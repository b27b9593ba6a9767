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

#ifdef ET_TIMELINE
__device__ unsigned long long g_attn_tl[64];
__device__ __forceinline__ unsigned long long gtime_a() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define ET_TLA(slot)                                                                                  \
  do {                                                                                                \
    if (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0) g_attn_tl[(slot)] = gtime_a();          \
  } while (0)
extern "C" int et_diag_attn_timeline(unsigned long long* host_out) {
  return cudaMemcpyFromSymbol(host_out, g_attn_tl, sizeof(g_attn_tl)) == cudaSuccess ? 0 : 4;
}
#else
#define ET_TLA(slot) do {} while (0)
#endif

et_status make_tmap_2d(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                       uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows, bool swizzle128);
et_status make_tmap_2d_sw64(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                            uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows);

namespace {

constexpr int kThreads = 320;   // warp 0 TMA, warp 1 MMA + TMEM, warps 2-9 softmax / epilogue
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
  int tma_store;            // Z written through TMA stores (dense V layout, seq_len % 32 == 0)
  int z_stage;              // z_map scatter staged in shared memory, stored as 16-byte row windows
  int z_fill_empty;         // (with z_stage) a head with no kept V feature writes zeros over its Z window
  int vtab_static;          // v_col / v_width are layer weights (et_vprep at pack time): read before the grid wait
  unsigned long long* ts;   // trace slot or nullptr
};

template <int kDK>
struct Cfg {
  static constexpr int kTiles = kDK / 64;            // 64-wide SW128 tiles per 128-row operand
  static constexpr int kOpBytes = 128 * kDK * 2;     // one 128-row Q / K / V block
  static constexpr int kHalf = kDK / 2;              // O columns per softmax thread
  static constexpr int kStageBytes = 32 * kHalf * 2; // per softmax warp: 32 rows x kHalf fp16
};
// K/V ring depth: the short form holds all (<= 2) key blocks; the long form streams them through 4
// stages at d_k = 64 (the K/V load of block j+4 overlaps three blocks of work; with 2 stages the
// load of block j+2 could only start once P.V(j) had completed), 2 at d_k = 128 (shared memory)
template <bool kLong, int kDK> constexpr int kv_stages() { return (kLong && kDK == 64) ? 4 : 2; }
template <bool kLong, int kDK> constexpr size_t attn_smem_bytes() {
  return 1024 + (size_t)(1 + 2 * kv_stages<kLong, kDK>()) * Cfg<kDK>::kOpBytes + 8 * Cfg<kDK>::kStageBytes + 2048 + 256;
}

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

template <int kCols>
__device__ __forceinline__ void tmem_alloc_n(uint32_t* slot) { tmem_alloc<kCols>(slot); }

// kNKB: score blocks resident in TMEM (short form: 1 => seq_len <= 128, 2 => <= 256; long form: the
// two S buffers).  TMEM: S [0, 128 kNKB), P [128 kNKB, 192 kNKB), O [192 kNKB, 192 kNKB + kDK).
template <bool kBF16, int kDK, bool kLong, int kNKB>
__global__ void __launch_bounds__(kThreads, kLong ? 1 : 2) attn_kernel(const __grid_constant__ CUtensorMap tmap,
                                                           const __grid_constant__ CUtensorMap tmap_z,
                                                           const __grid_constant__ AParams p) {
  using C = Cfg<kDK>;
  constexpr int kKV = kv_stages<kLong, kDK>();
  constexpr int kS = 0, kP = 128 * kNKB, kO = 192 * kNKB;
  constexpr uint32_t kCols = (kO + kDK) <= 256 ? 256u : 512u;
  pdl_trigger();
  // attention-aware head tables: both loads issued together (one latency, not two in series); when
  // they are layer weights (computed at pack time) they are read before the grid-dependency wait, so
  // their latency overlaps the predecessor instead of sitting in front of every CTA's work
  const int hh = p.head_begin + blockIdx.y;
  int vloc = hh * kDK, vw = kDK;
  if (p.vtab_static) {
    if (p.v_col) vloc = __ldg(p.v_col + hh);
    if (p.v_width) vw = __ldg(p.v_width + hh);
  }
  pdl_wait();   // QKV (and per-forward head tables) of the predecessors are visible from here
  trace_cta_start(p.ts);
  if (!p.vtab_static) {
    if (p.v_col) vloc = __ldg(p.v_col + hh);     // packed V column of this head
    if (p.v_width) vw = __ldg(p.v_width + hh);
  }
  if (vw == 0) {   // every V feature of the head pruned: Z = 0 there (reading C-6: b_V folded into b_O')
    if (p.z_fill_empty) {   // the staged path writes every other head's whole window: no Z memset needed
      using T0 = typename std::conditional<kBF16, __nv_bfloat16, __half>::type;
      const int q0 = blockIdx.x * 128, nrow = min(128, p.S - q0);
      constexpr int kU = kDK / 8;
      for (int i = threadIdx.x; i < nrow * kU; i += blockDim.x)
        *reinterpret_cast<uint4*>(static_cast<T0*>(p.Z) + (size_t)(blockIdx.z * p.S + q0 + i / kU) * p.ld_z +
                                  (hh - p.head_begin) * kDK + (i % kU) * 8) = make_uint4(0, 0, 0, 0);
    }
    trace_cta_end(p.ts);
    return;
  }
  extern __shared__ uint8_t smem_raw[];
  // 1024-byte aligned, derived from smem_raw by pointer arithmetic so the compiler keeps the shared
  // address space (an integer round trip would turn every access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + C::kOpBytes;                // kKV x K block
  uint8_t* sV = sK + kKV * C::kOpBytes;          // kKV x V block
  uint8_t* sStage = sV + kKV * C::kOpBytes;      // 8 x epilogue staging
  float* xmax = reinterpret_cast<float*>(sStage + 8 * C::kStageBytes);   // [2][128] row-max halves
  float* xsum = xmax + 256;                                               // [2][128] row-sum halves
  uint64_t* bars = reinterpret_cast<uint64_t*>(xsum + 256);
  uint64_t* q_full = bars + 0;
  uint64_t* kv_full = bars + 1;              // [kKV]
  uint64_t* kv_empty = bars + 1 + kKV;       // [kKV]
  uint64_t* s_full = bars + 1 + 2 * kKV;     // [2]
  uint64_t* s_free = s_full + 2;             // [2]
  uint64_t* p_full = s_full + 4;             // [2]
  uint64_t* o_full = s_full + 6;
  uint64_t* o_free = s_full + 7;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(s_full + 8);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int qb = blockIdx.x;
  const int h = p.head_begin + blockIdx.y;
  const int b = blockIdx.z;
  const int S = p.S;
  const int len = p.lengths ? p.lengths[b] : S;
  int kmax = len;                                  // keys needed by this query block: [0, kmax)
  if (p.causal) kmax = min(kmax, qb * 128 + 128);
  const int nkb = (kmax + 127) / 128;
  const int row0 = b * S;                          // first token row of this sequence
  const int qcol = p.q_off + h * kDK, kcol = p.k_off + h * kDK;
  const int vcol = p.v_off + vloc;
  const int dvn = p.dv_max;                        // P.V MMA N

  if (p.box_rows < 128) {
    // tiny problem: the TMA box covers fewer than 128 rows; zero the V staging so that the rows
    // it leaves untouched are finite (P = 0 there, but 0 * NaN would poison O)
    for (int i = threadIdx.x; i < kKV * C::kOpBytes / 16; i += blockDim.x)
      reinterpret_cast<uint4*>(sV)[i] = make_uint4(0, 0, 0, 0);
    fence_proxy_async_smem();
  }
  if (threadIdx.x == 0) {
    mbar_init(q_full, 1);
    for (int i = 0; i < kKV; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&s_free[i], 8);
      mbar_init(&p_full[i], 8);
    }
    mbar_init(o_full, 1);
    mbar_init(o_free, 8);
    fence_mbar_init();
  }
  if (threadIdx.x == 0) ET_TLA(0);
  if (warp == 1) tmem_alloc<kCols>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;
  if (threadIdx.x == 0) ET_TLA(1);

  if (warp == 0) {
    // ================= TMA producer: Q once, then K/V blocks through a 2-stage ring
    if (lane == 0) {
      tma_prefetch_desc(&tmap);
      const uint32_t tile_bytes = (uint32_t)p.box_rows * 128;   // one 64-column tile
      mbar_expect_tx(q_full, tile_bytes * C::kTiles);
      for (int t = 0; t < C::kTiles; ++t)
        tma_load_2d(sQ + t * 16384, &tmap, q_full, qcol + t * 64, row0 + qb * 128);
      for (int j = 0; j < nkb; ++j) {
        const int st = j % kKV;
        if (j >= kKV) mbar_wait(&kv_empty[st], ((j / kKV) - 1) & 1);
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
      const uint32_t k_u = smem_u32(sK + (j % kKV) * C::kOpBytes);
#pragma unroll
      for (int ks = 0; ks < kDK / 16; ++ks) {
        const uint32_t off = (ks >> 2) * 16384 + (ks & 3) * 32;
        mma_ss_warp(tbase + s_col, make_sdesc(q_u + off, 16, 1024, kLayoutSW128),
                    make_sdesc(k_u + off, 16, 1024, kLayoutSW128), idesc_s, ks > 0);
      }
    };
    auto issue_pv = [&](int j, uint32_t p_col, bool acc_first) {
      const uint32_t v_u = smem_u32(sV + (j % kKV) * C::kOpBytes);
#pragma unroll
      for (int ks = 0; ks < 8; ++ks)   // 128 keys = 8 x K16; V MN-major SW128: 16 rows = 2048 B
        mma_ts_warp(tbase + kO, tbase + p_col + ks * 8, make_sdesc(v_u + ks * 2048, 16384, 1024, kLayoutSW128),
                    idesc_o, (acc_first || ks > 0) ? 1u : 0u);
    };
    mbar_wait_warp(q_full, 0);
    tc_fence_after();
    if (lane == 0) ET_TLA(2);
    if constexpr (!kLong) {
      // short form: every score block, then one P.V chain over all keys
      for (int j = 0; j < nkb; ++j) {
        mbar_wait_warp(&kv_full[j], 0);
        tc_fence_after();
        issue_qk(j, kS + j * 128);
      }
      mma_commit_warp(&s_full[0]);
      if (lane == 0) ET_TLA(3);
      mbar_wait_warp(&p_full[0], 0);
      tc_fence_after();
      if (lane == 0) ET_TLA(4);
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
          mbar_wait_warp(&kv_full[jn % kKV], (jn / kKV) & 1);
          tc_fence_after();
          issue_qk(jn, kS + bn * 128);
          mma_commit_warp(&s_full[bn]);
        }
        mbar_wait_warp(&p_full[j & 1], (j >> 1) & 1);
        tc_fence_after();
        issue_pv(j, kP + (j & 1) * 64, j > 0);   // O accumulates in TMEM (rescaled there when needed)
        mma_commit_warp(o_full);
        mma_commit_warp(&kv_empty[j % kKV]);
      }
    }
  } else {
    // ================= softmax / epilogue: two threads per query row, each owning 64 of every
    // 128 keys (and half of the O columns); row max / sum halves meet in shared memory
    const int sw = warp - 2;                     // 0..7
    const int half = sw >> 2;                    // key / O-column half
    const int quarter = warp & 3;                // TMEM lane quarter this warp may access
    const int r = quarter * 32 + lane;           // query row within the block = TMEM lane
    const int qi = qb * 128 + r;                 // query index within the sequence
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    int kend = len;                              // valid keys: [0, kend)
    if (p.causal) kend = min(kend, qi + 1);
    const float sl2 = p.scale_log2;
    float lpart = 0.f;                           // this half's share of the row sum

    if constexpr (!kLong) {
      mbar_wait_warp(&s_full[0], 0);
      tc_fence_after();
      if (threadIdx.x == 64) ET_TLA(5);
      float m = -INFINITY;
      for (int j = 0; j < nkb; ++j) {
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          uint32_t v[32];
          const int k0 = j * 128 + half * 64 + c * 32;
          tmem_ld32(tbase + lane_off + kS + k0, v);
          tmem_ld_wait();
#pragma unroll
          for (int t = 0; t < 32; ++t)
            if (k0 + t < kend) m = fmaxf(m, __uint_as_float(v[t]));
        }
      }
      xmax[half * 128 + r] = m;
      named_bar_sync(1, 256);
      m = fmaxf(m, xmax[(half ^ 1) * 128 + r]);
      const float mb = m * sl2;
      for (int j = 0; j < nkb; ++j) {
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          uint32_t v[32];
          const int k0 = j * 128 + half * 64 + c * 32;
          tmem_ld32(tbase + lane_off + kS + k0, v);
          tmem_ld_wait();
          uint32_t pk[16];
#pragma unroll
          for (int t = 0; t < 32; t += 2) {
            const float p0 = k0 + t < kend ? ex2(__uint_as_float(v[t]) * sl2 - mb) : 0.f;
            const float p1 = k0 + t + 1 < kend ? ex2(__uint_as_float(v[t + 1]) * sl2 - mb) : 0.f;
            lpart += p0 + p1;
            pk[t >> 1] = pack2<kBF16>(p0, p1);
          }
          tmem_st16(tbase + lane_off + kP + j * 64 + half * 32 + c * 16, pk);
        }
      }
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[0]);
      if (threadIdx.x == 64) ET_TLA(6);
      mbar_wait_warp(o_full, 0);
      tc_fence_after();
      if (threadIdx.x == 64) ET_TLA(7);
    } else {
      // Per 128-key block: the half-row of scores is read from TMEM ONCE into registers (the S
      // buffer is released at once for QK(j+2)), max and exp2 come from the registers.  O stays in
      // TMEM and accumulates across blocks; it is rescaled there only when a row's running max grows
      // by more than 2^8 in exp2 units (otherwise the stale max is kept: p <= 2^8, exact in the
      // final O / l since l uses the same max — lazy rescaling as in FlashAttention-4).
      constexpr float kRescale = 8.0f;
      float m = -INFINITY;                       // max used for this row's exponentials so far
      for (int j = 0; j < nkb; ++j) {
        const int bj = j & 1;
        mbar_wait_warp(&s_full[bj], (j >> 1) & 1);
        tc_fence_after();
        uint32_t sv0[32], sv1[32];
        tmem_ld32(tbase + lane_off + kS + bj * 128 + half * 64, sv0);
        tmem_ld32(tbase + lane_off + kS + bj * 128 + half * 64 + 32, sv1);
        tmem_ld_wait();
        auto sv = [&](int t) { return t < 32 ? sv0[t] : sv1[t - 32]; };
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&s_free[bj]);   // S(j) is in registers: its buffer may take QK(j+2)
        const int kb = j * 128 + half * 64;        // first key of this thread's half block
        const bool full = kb + 64 <= kend;         // no masked key in this half block
        // 8 independent partial maxima / sums: the reductions are not one 64-long dependency chain
        float mx8[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) mx8[i] = -INFINITY;
        if (full) {
#pragma unroll
          for (int t = 0; t < 64; ++t) mx8[t & 7] = fmaxf(mx8[t & 7], __uint_as_float(sv(t)));
        } else {
#pragma unroll
          for (int t = 0; t < 64; ++t)
            if (kb + t < kend) mx8[t & 7] = fmaxf(mx8[t & 7], __uint_as_float(sv(t)));
        }
        float mblk = fmaxf(fmaxf(fmaxf(mx8[0], mx8[1]), fmaxf(mx8[2], mx8[3])),
                           fmaxf(fmaxf(mx8[4], mx8[5]), fmaxf(mx8[6], mx8[7])));
        xmax[half * 128 + r] = mblk;
        named_bar_sync(1, 256);
        mblk = fmaxf(mblk, xmax[(half ^ 1) * 128 + r]);
        named_bar_sync(2, 256);   // both halves read xmax before it is rewritten for the next block
        float alpha = 1.0f;
        if (mblk > m && (m == -INFINITY || (mblk - m) * sl2 > kRescale)) {
          alpha = (m == -INFINITY) ? 0.f : ex2((m - mblk) * sl2);
          m = mblk;
        }
        // PV(j-1) must be complete before O is rescaled and before P buffer bj (read by PV(j-2))
        // is overwritten (in-order completion: o_full phase j-1 covers both)
        if (j >= 1) {
          mbar_wait_warp(o_full, (j - 1) & 1);
          tc_fence_after();
          if (__any_sync(0xffffffffu, alpha != 1.0f)) {   // warp-collective TMEM read-modify-write
#pragma unroll
            for (int c = 0; c < C::kHalf; c += 32) {
              if (half * C::kHalf + c < dvn) {
                uint32_t ov[32];
                tmem_ld32(tbase + lane_off + kO + half * C::kHalf + c, ov);
                tmem_ld_wait();
#pragma unroll
                for (int t = 0; t < 32; ++t) ov[t] = __float_as_uint(__uint_as_float(ov[t]) * alpha);
                tmem_st32(tbase + lane_off + kO + half * C::kHalf + c, ov);
              }
            }
          }
        }
        const float mb = (m == -INFINITY) ? 0.f : m * sl2;
        uint64_t ls4[4] = {0ull, 0ull, 0ull, 0ull};   // 4 packed FP32x2 partial sums
        const uint64_t sl2x2 = f2pk(sl2, sl2), nmb2 = f2pk(-mb, -mb);
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          uint32_t pk[16];
#pragma unroll
          for (int t = 0; t < 32; t += 2) {
            const int key = kb + c * 32 + t;
            const float2 x = f2upk(ffma2(f2pk(__uint_as_float(sv(c * 32 + t)), __uint_as_float(sv(c * 32 + t + 1))),
                                         sl2x2, nmb2));   // s * scale * log2 e - m * scale * log2 e
            float p0 = ex2(x.x), p1 = ex2(x.y);
            if (!full) {
              p0 = key < kend ? p0 : 0.f;
              p1 = key + 1 < kend ? p1 : 0.f;
            }
            ls4[(t >> 1) & 3] = fadd2(ls4[(t >> 1) & 3], f2pk(p0, p1));
            pk[t >> 1] = pack2<kBF16>(p0, p1);
          }
          tmem_st16(tbase + lane_off + kP + bj * 64 + half * 32 + c * 16, pk);
        }
        const float2 la = f2upk(fadd2(fadd2(ls4[0], ls4[1]), fadd2(ls4[2], ls4[3])));
        const float lsum = la.x + la.y;
        tmem_st_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&p_full[bj]);
        lpart = lpart * alpha + lsum;
      }
      mbar_wait_warp(o_full, (nkb - 1) & 1);   // the last P.V: O is final in TMEM
      tc_fence_after();
    }

    // ---- epilogue: Z = O / l.  l = both halves' sums (exchanged through shared memory).  The TMEM
    // loads are warp-collective and stay outside any per-row condition.
    xsum[half * 128 + r] = lpart;
    named_bar_sync(1, 256);
    const float inv = 1.0f / (lpart + xsum[(half ^ 1) * 128 + r]);
    using T = typename std::conditional<kBF16, __nv_bfloat16, __half>::type;
    const bool store = qi < S;
    // TMA path: this warp's 32 rows all lie inside the sequence (S % 32 == 0, so a warp's rows are
    // either all valid or all beyond the sequence — those must not be written at all)
    const bool tma_warp = p.tma_store && (qb * 128 + quarter * 32 < S);
    const int ccol0 = half * C::kHalf;           // first O column of this thread
    // attention-aware Z (z_map, row-pruned V): the head's kept columns scatter into its kDK-wide
    // window of Z.  Staged: the window of all 128 rows is built in the (now idle) Q buffer —
    // zero-filled, 16-byte unit u of row r at u ^ (r % 8) — then stored as whole 16-byte units by
    // consecutive threads (a direct scatter wrote 2-byte elements, one row per lane: 32 lines per
    // store instruction).  Every MMA has completed (O is final), so sQ is free.
    const bool zst = p.z_map && p.z_stage;
    const int etid = sw * 32 + lane;             // 0..255 over the softmax / epilogue warps
    int zwb = 0;                                 // first Z column of this head's window
    if (zst) {
      zwb = (__ldg(p.z_map + vloc) / kDK) * kDK;  // a head's first packed V column is a kept feature
      for (int i = etid; i < C::kOpBytes / 16; i += 256) reinterpret_cast<uint4*>(sQ)[i] = make_uint4(0, 0, 0, 0);
      named_bar_sync(1, 256);
    }
    uint8_t* st = sStage + sw * C::kStageBytes;  // 32 rows x kHalf fp16, 64-byte rows (SWIZZLE_64B)
    T* zrow = static_cast<T*>(p.Z) + (size_t)(row0 + qi) * p.ld_z;
#pragma unroll
    for (int c0 = 0; c0 < C::kHalf; c0 += 32) {
      if (ccol0 + c0 < vw) {
        float x[32];
        {
          uint32_t v[32];
          tmem_ld32(tbase + lane_off + kO + ccol0 + c0, v);
          tmem_ld_wait();
#pragma unroll
          for (int t = 0; t < 32; ++t) x[t] = __uint_as_float(v[t]);
        }
        if (tma_warp) {
          // 32 columns = 64 bytes per row: 4 x 16-byte chunks, SWIZZLE_64B position c ^ ((row >> 1) & 3)
#pragma unroll
          for (int ch = 0; ch < 4; ++ch) {
            const uint4 u = make_uint4(pack2<kBF16>(x[8 * ch] * inv, x[8 * ch + 1] * inv),
                                       pack2<kBF16>(x[8 * ch + 2] * inv, x[8 * ch + 3] * inv),
                                       pack2<kBF16>(x[8 * ch + 4] * inv, x[8 * ch + 5] * inv),
                                       pack2<kBF16>(x[8 * ch + 6] * inv, x[8 * ch + 7] * inv));
            *reinterpret_cast<uint4*>(st + (c0 / 32) * 2048 + lane * 64 + ((ch ^ ((lane >> 1) & 3)) << 4)) = u;
          }
        } else if (zst) {
          const int32_t* zm = p.z_map + vloc + ccol0 + c0;
#pragma unroll
          for (int t = 0; t < 32; ++t)
            if (ccol0 + c0 + t < vw) {
              const int dst = __ldg(zm + t);
              if (dst >= 0) {
                const int j = dst - zwb;
                T* e = reinterpret_cast<T*>(sQ + r * (kDK * 2) + (((j >> 3) ^ (r & 7)) << 4) + (j & 7) * 2);
                if constexpr (kBF16) *e = __float2bfloat16_rn(x[t] * inv);
                else *e = __float2half_rn(x[t] * inv);
              }
            }
        } else if (store && !p.tma_store) {
          if (p.z_map) {
            const int32_t* zm = p.z_map + vloc + ccol0 + c0;
#pragma unroll
            for (int t = 0; t < 32; ++t)
              if (ccol0 + c0 + t < vw) {
                const int dst = zm[t];
                if (dst >= 0) {
                  if constexpr (kBF16) zrow[dst] = __float2bfloat16_rn(x[t] * inv);
                  else zrow[dst] = __float2half_rn(x[t] * inv);
                }
              }
          } else {
            T* z = zrow + h * kDK + ccol0 + c0;
#pragma unroll
            for (int t = 0; t < 32; t += 8)
              if (ccol0 + c0 + t < vw)
                *reinterpret_cast<uint4*>(z + t) = make_uint4(
                    pack2<kBF16>(x[t] * inv, x[t + 1] * inv), pack2<kBF16>(x[t + 2] * inv, x[t + 3] * inv),
                    pack2<kBF16>(x[t + 4] * inv, x[t + 5] * inv), pack2<kBF16>(x[t + 6] * inv, x[t + 7] * inv));
          }
        }
      }
    }
    if (zst) {
      named_bar_sync(1, 256);
      constexpr int kU = kDK / 8;                // 16-byte units per row window
      for (int i = etid; i < 128 * kU; i += 256) {
        const int r2 = i / kU, u = i % kU;
        if (qb * 128 + r2 < S)
          *reinterpret_cast<uint4*>(static_cast<T*>(p.Z) + (size_t)(row0 + qb * 128 + r2) * p.ld_z + zwb + u * 8) =
              *reinterpret_cast<const uint4*>(sQ + r2 * (kDK * 2) + ((u ^ (r2 & 7)) << 4));
      }
    }
    if (tma_warp) {
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
#pragma unroll
        for (int c0 = 0; c0 < C::kHalf; c0 += 32)
          tma_store_2d(&tmap_z, st + (c0 / 32) * 2048, h * kDK + ccol0 + c0, row0 + qb * 128 + quarter * 32);
        bulk_commit_group();
        bulk_wait_group<0>();
      }
    }
    if (threadIdx.x == 64) ET_TLA(8);
  }

  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) ET_TLA(9);
  trace_cta_end(p.ts);
  if (warp == 1) {
    __syncwarp();
    tc_fence_after();
    tmem_dealloc<kCols>(tbase);
  }
}

template <bool kBF16, int kDK, bool kLong, int kNKB>
et_status launch(const CUtensorMap& tm, const CUtensorMap& tz, const AParams& prm, dim3 grid, cudaStream_t stream) {
  auto kern = attn_kernel<kBF16, kDK, kLong, kNKB>;
  const size_t smem = attn_smem_bytes<kLong, kDK>();
  static std::once_flag once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(once, [&] { attr_err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); });
  ET_CUDA(attr_err);
  ET_CUDA(launch_pdl(kern, grid, dim3(kThreads), smem, stream, tm, tz, prm));
  count_launch();
  return ET_OK;
}

}  // namespace

int attn_short_max(int d_k) { return (d_k == 64 || d_k == 128) ? 256 : 0; }

// z_map mode with z_clear: Z columns that no kept V feature maps to must read as zero afterwards.
// Decided here, next to the kernel choice: the 16-bit generic kernel's staged Z path writes every
// head's whole window (zeros included; heads with no kept feature zero theirs, z_fill_empty), any
// other path gets a memset of Z first.
static bool z_staged(const AttnArgs& a) {
  return a.dtype != ET_FP32 && a.z_map != nullptr && aligned16(a.Z) && (a.ld_z * 2) % 16 == 0;
}

et_status attention_run(const AttnArgs& a, cudaStream_t stream) {
  if (a.z_map != nullptr && a.z_clear && !z_staged(a) && a.batch > 0 && a.seq_len > 0)
    ET_CUDA(cudaMemsetAsync(a.Z, 0, (size_t)a.batch * a.seq_len * a.ld_z * dtype_size(a.dtype), stream));
  if (a.dtype == ET_FP32) return attention32_run(a, stream);   // FP32 validation build (CUDA cores)
  if (a.d_k != 64 && a.d_k != 128) return fail(ET_ERR_UNSUPPORTED, "attention: d_k must be 64 or 128 (got %d)", a.d_k);
  if (a.v_width_max <= 0 || a.v_width_max > a.d_k || a.v_width_max % 16)
    return fail(ET_ERR_INVALID_ARG, "attention: V width must be a multiple of 16 and <= d_k");
  if (!a.long_form && a.seq_len > 256) return fail(ET_ERR_UNSUPPORTED, "attention: short form needs seq_len <= 256");
  if (a.batch <= 0 || a.seq_len <= 0 || a.head_end <= a.head_begin) return ET_OK;
  if (!aligned16(a.qkv) || (a.ld_qkv * 2) % 16) return fail(ET_ERR_INVALID_ARG, "attention: QKV not 16B aligned");
  if (attention128_applies(a) && !a.generic) return attention128_run(a, stream);
  const uint64_t rows = (uint64_t)a.batch * a.seq_len;
  const uint32_t box_rows = rows < 128 ? (uint32_t)rows : 128u;
  CUtensorMap tm, tz;
  ET_TRY(make_tmap_2d(&tm, a.qkv, a.dtype, rows, (uint64_t)a.ld_qkv, (uint64_t)a.ld_qkv, 64, box_rows, true));
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
  prm.box_rows = (int)box_rows;
  prm.ts = a.ts;
  // TMA stores of Z: dense per-head V, every 32-row group inside one sequence, Z 16-byte aligned
  prm.tma_store = (a.z_map == nullptr && a.v_width == nullptr && a.seq_len % 32 == 0 && rows >= 32 &&
                   aligned16(a.Z) && (a.ld_z * 2) % 16 == 0) ? 1 : 0;
  prm.z_stage = z_staged(a) ? 1 : 0;
  prm.z_fill_empty = prm.z_stage && a.z_clear;
  prm.vtab_static = a.vtab_static;
  if (prm.tma_store) {
    ET_TRY(make_tmap_2d_sw64(&tz, a.Z, a.dtype, rows, (uint64_t)a.ld_z, (uint64_t)a.ld_z, 32, 32));
  } else {
    tz = tm;   // unused
  }
  dim3 grid((a.seq_len + 127) / 128, a.head_end - a.head_begin, a.batch);
  const bool bf = a.dtype == ET_BF16;
  const bool lf = a.long_form;
  const int nkb1 = a.seq_len <= 128;
  if (a.d_k == 64) {
    if (lf) return bf ? launch<true, 64, true, 2>(tm, tz, prm, grid, stream) : launch<false, 64, true, 2>(tm, tz, prm, grid, stream);
    if (nkb1) return bf ? launch<true, 64, false, 1>(tm, tz, prm, grid, stream) : launch<false, 64, false, 1>(tm, tz, prm, grid, stream);
    return bf ? launch<true, 64, false, 2>(tm, tz, prm, grid, stream) : launch<false, 64, false, 2>(tm, tz, prm, grid, stream);
  }
  if (lf) return bf ? launch<true, 128, true, 2>(tm, tz, prm, grid, stream) : launch<false, 128, true, 2>(tm, tz, prm, grid, stream);
  if (nkb1) return bf ? launch<true, 128, false, 1>(tm, tz, prm, grid, stream) : launch<false, 128, false, 1>(tm, tz, prm, grid, stream);
  return bf ? launch<true, 128, false, 2>(tm, tz, prm, grid, stream) : launch<false, 128, false, 2>(tm, tz, prm, grid, stream);
}

}  // namespace et
