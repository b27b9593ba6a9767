// Tile-sparse linear layer on tcgen05 (§4.2: tensor-tile pruning keeps or
// drops whole 16x16 tiles; line 252: tile-pruned linear vs dense GEMM).
//
//   Y[m, n] = epilogue( sum over KEPT tiles (i, j) of X[m, 16j:16j+16] . W'[16i:16i+16, 16j:16j+16]^T )
//
// One tcgen05.mma (M=128 tokens, N=16 features, K=16) per kept tile; pruned tiles cost nothing.
// Design (measured in profiles/r01/M1_tcgen05_probe.md and the cycle timelines of profiles/r01):
//   * the activation block (128 tokens x K<=768) lives in TMEM as the MMA A operand ("TS" MMA).
//     With A in shared memory every N=16 MMA re-reads 4 KB of A and the kernel is capped near 20 %
//     of peak by smem bandwidth.  Fill: TMA (SWIZZLE_128B) -> smem -> registers of the 24 MMA /
//     epilogue warps (idle during the prologue) -> tcgen05.st.
//   * one unified shared-memory ring (9 or 11 slots of 16 KB) carries first the A chunks (all in flight at once: the
//     prologue is bound by L2 bandwidth, not by ring depth) and then the packed tiles (512 B each,
//     contiguous per (K part, tile row), 1-D bulk copies of 32 tiles + their column indices).
//   * 8 MMA warps, one accumulator (16 TMEM columns) each, so 8 independent accumulation chains are
//     in flight (one warp can only issue an MMA every ~60 cycles; 8 warps saturate the pipe).  A
//     warp prepares its next row (barrier waits, tile columns, descriptors) before waiting for its
//     accumulator to drain, so only the MMA issue sits on the accumulator's critical path.
//   * four epilogue groups of 4 warps (one per TMEM lane quarter) each drain a pair of accumulators
//     (32 columns) with one tcgen05.ld, release them, then apply bias / Q-scale / GELU / ReLU in FP32
//     (packed FP32x2 arithmetic) and store through swizzled staging + TMA stores.  (With two groups
//     of quads the epilogue arithmetic paced the whole kernel.)
//   * warp 24 issues every load and owns the TMEM allocation.
// Grid: x = piece (a tile-row range of one segment), y = 128-token block, z = K part (split-K,
// fp32 partial outputs, reduced by the LayerNorm kernel).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <mutex>
#include <type_traits>
#include <algorithm>

#include "../internal.h"
#include "../ptx.cuh"

namespace et {

#ifdef ET_TIMELINE
// Debug builds only: %clock64 stamps (SM cycles) of CTA (0, 0, 0) of the most recent launch.
//   slot 0: start; 1: metadata staged; 14: last load issued; 16 + 24*w + 3*k + {0,1,2}: MMA warp w,
//   round k: accumulator free / first MMA / commit; 208 + 40*g + 5*k + {0,1,2,3}: epilogue group g,
//   round k: pair complete / drained / math done / stores issued; 500: end.
__device__ unsigned long long g_timeline[512];
// per-CTA (start, end) %globaltimer and SM id of the most recent launch (debug builds)
__device__ unsigned long long g_cta_span[2048][3];
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
  return t;
}
#define ET_TL(slot)                                                              \
  do {                                                                           \
    if (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0 && (slot) < 512) g_timeline[(slot)] = gtime(); \
  } while (0)
// earliest stamp wins (slots 400..511 are reset to all-ones at kernel start)
#define ET_TL_MIN(slot)                                                          \
  do {                                                                           \
    if (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0) atomicMin(&g_timeline[(slot)], gtime()); \
  } while (0)
#define ET_TL_RESET()                                                            \
  do {                                                                           \
    if (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0 && threadIdx.x < 112) g_timeline[400 + threadIdx.x] = ~0ull; \
  } while (0)
#else
#define ET_TL(slot) do {} while (0)
#define ET_TL_MIN(slot) do {} while (0)
#define ET_TL_RESET() do {} while (0)
#endif

namespace {

constexpr int kMaxPieces = 64;

// Unified staging ring: the A chunks of the K part (128 rows x 64 K, SWIZZLE_128B) come first in the
// load sequence, then the tile chunks (32 packed tiles each).  Every A load is in flight at once during
// the prologue (the whole ring is free then), and the slots are reused for tiles as soon as the
// fill warps have moved their A chunk into TMEM.
constexpr int kMaxSlots = 11;
constexpr int kSlotBytes = 16384;
constexpr int kChunkTiles = 32;  // tiles per tile chunk (16 KB)
constexpr int kMaxKChunks = 12;  // K <= 768 per part
constexpr int kMaxBChunks = 192; // tile chunks per CTA (one single-use full barrier each)
constexpr int kMaxRows = 256;    // tile rows per CTA (row pointers staged in smem)
constexpr int kMaxBiasRows = 128; // tile rows per CTA of a bias epilogue (FP32 bias staged in smem)
constexpr int kAccCol = 384;     // first accumulator column (A uses [0, Kp/2) <= 384)
constexpr int kAcc = 8;          // accumulators (16 TMEM columns each): a round = 8 tile rows
// Warp roles: MMA warps [0, MW) own kAcc / MW accumulators each (accumulator a holds tile rows a,
// a + 8, a + 16, ...); epilogue warps [MW, MW + 4 EG) form EG groups of 4 (one warp per TMEM lane
// quarter), group g draining accumulator pairs ("pair slots" j = g, g + EG, ...; pair slot j = tile
// rows 2j, 2j + 1); warp MW + 4 EG loads (A by TMA, tiles by bulk copy) and owns TMEM.  Measured
// on C3's FFN1 (GELU): 8 / 4 = 15.2 us, 8 MMA warps / 5 groups = 15.6 us, 4 / 6 = 17.9 us — its
// epilogue is throughput-bound (MUFU / FMA / TMEM reads), not short of warps, so every epilogue
// uses 8 / 4.  A pair slot's completion is signalled on its own single-use barrier (slot_full[j]):
// with the roles configurable a group may wait on round k + 1 of a pair before round k completed,
// which a parity wait on a per-accumulator barrier cannot tell apart.
template <int kEpi> struct Roles {
  static constexpr int MW = 8;
  static constexpr int EG = 4;
  static constexpr int EW = 4 * EG;
  static constexpr int WP = MW + EW;
  static constexpr int threads = (WP + 1) * 32;
};

struct SegDev {
  const int32_t* prp;       // part_row_ptr [kparts][rp_stride] (+ the segment's first row)
  const int32_t* tile_col;  // values order
  const uint8_t* values;
  const void* bias;
  int tile_rows, rp_stride;
  int out_col;
  float scale;
  int apply_scale;
};
// A piece = the tile rows one CTA computes: rows [i0, i1) of segment `seg` (seg1 == seg), or - when
// it spans two output-contiguous segments (seg1 == seg + 1, e.g. the Q|K|V projection) - rows
// [i0, rows(seg)) of `seg` followed by rows [0, i1) of `seg1` ("part A" and "part B").
struct Piece {
  int16_t seg, seg1;
  int16_t i0, i1;
};
struct Params {
  int M, K, Kp, kparts;   // Kp = 768 (K part width); the last part may be shorter
  int box_rows;           // TMA box height: min(128, M) (a box may not exceed the tensor)
  const uint8_t* X;       // activation block base (K offset k0 folded in)
  long long ldx_bytes;    // X row pitch in bytes
  int nseg;
  SegDev seg[3];
  int npieces;
  Piece piece[kMaxPieces];
  void* Y;
  int ldy;
  long long part_stride;   // elements between split-K partial outputs (fp32 epilogue)
  unsigned long long* ts;  // trace slot or nullptr
};

struct __align__(16) Barriers {
  // single-use barriers per A chunk / tile chunk (a warp may run laps ahead of a slot's reuse, and a
  // parity wait on a reused barrier cannot tell those phases apart)
  uint64_t xfull[kMaxKChunks];   // A load #s landed in its slot (TMA transaction bytes)
  uint64_t xfree[kMaxKChunks];   // A load #s read out of its slot (4 fill warps)
  uint64_t a_all;                // the whole A block is in TMEM (4 fill warps x nk chunks)
  uint64_t slot_full[kMaxRows / 2], acc_empty[kAcc];   // per pair slot (single use) / per accumulator
  uint64_t bfull[kMaxBChunks];
  alignas(16) int tcol[kMaxSlots][kChunkTiles + 4];   // bulk-copy destination (16-byte aligned): tile columns
  int rptr[kMaxRows + 1];        // this CTA's row pointers, relative to its first tile
  alignas(16) float bias_f[kMaxBiasRows * 16];   // this CTA's bias slice, FP32 (converted once)
  uint32_t tmem_base;
  uint32_t pair_done[kMaxRows / 64];   // bit j: pair slot j's MMAs observed complete (its tiles are free)
  int tcoff[kMaxSlots];          // per slot: offset of the chunk's first column index in tcol[slot]
  int a_end;                     // end (relative tile index) of part A's last row
};

// Per epilogue: staging per epilogue warp (32 rows x 32 columns: 128 B rows in FP32, 64 B in 16-bit)
// and as many ring slots as the rest of the 227 KB allows (9 with FP32 staging, 11 with 16-bit).
// (Round 1's O-projection + LayerNorm fused over a 4-CTA cluster with an FP32 stash measured 12.2 us
// against 11.5 us unfused and was removed in round 2.)
template <int kEpi> struct Smem {
  static constexpr size_t kStageWarp = kEpi == ET_EPI_F32 ? 4096 : 2048;
  static constexpr size_t kStage = (size_t)Roles<kEpi>::EW * kStageWarp;
  static constexpr int kSlots = kEpi == ET_EPI_F32 ? 9 : 11;
  static constexpr size_t kRing = (size_t)kSlots * kSlotBytes;
  static constexpr size_t kBytes = 1024 + kRing + kStage + sizeof(Barriers);
  static_assert(kBytes <= 232448, "shared memory budget");
  static_assert(kSlots <= kMaxSlots, "slot metadata");
};

// GELU(x) = x Phi(x) = 0.5 x (1 + erf(x / sqrt 2)) (reading C-12), evaluated as
//   GELU(x) = max(x, 0) + nu e,   nu = -min(|x|, 4 sqrt 2),   e = 0.5 erfc(-nu / sqrt 2) = 2^(nu R(nu) - 1)
// (x >= 0: x (1 - e); x < 0: x e).  With g(t) = -log2 erfc(t) ~ t q(t), q a degree-4 polynomial
// fitted on t in [0, 4] (tools/fit_gelu.py), R(nu) = q(-nu / sqrt 2) / sqrt 2 (coefficients
// transformed exactly; the clamp moves to |x| = 4 sqrt 2, where |nu e| < 5e-8): |GELU error| <= 1.6e-6
// (float32 emulation of this code against the float64 erf form), below FP16/BF16 output resolution
// for |GELU| > 4e-3.  Degree 4 instead of 5: one packed FMA less per pair — FFN1 15.3 -> 14.7 us per
// C3 layer (A/B on one box), the epilogue being issue-bound.  (ex2.approx.f16x2 on the pair - half
// the MUFU ops, two more conversions - measured slower: FFN1 14.4 -> 15.1 us, profiles/r02.)  Two elements at a time: one FMNMX per
// element for nu (the -|x| operand modifier), 6 packed FP32x2 FMAs and two MUFU.EX2 per pair.
__device__ __forceinline__ void gelu_erf2(float& x0, float& x1) {
  const uint64_t nu = f2pk(fmaxf(-fabsf(x0), -5.65685424949238f), fmaxf(-fabsf(x1), -5.65685424949238f));
  uint64_t q = ffma2(f2pk(5.281529925e-4f, 5.281529925e-4f), nu, f2pk(7.4382414e-3f, 7.4382414e-3f));
  q = ffma2(q, nu, f2pk(5.263240325e-2f, 5.263240325e-2f));
  q = ffma2(q, nu, f2pk(-0.4592077305f, -0.4592077305f));
  q = ffma2(q, nu, f2pk(1.151100645f, 1.151100645f));
  const float2 y = f2upk(ffma2(nu, q, f2pk(-1.0f, -1.0f)));   // nu R(nu) - 1
  float e0, e1;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e0) : "f"(y.x));
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e1) : "f"(y.y));
  const float2 g = f2upk(ffma2(nu, f2pk(e0, e1), f2pk(fmaxf(x0, 0.0f), fmaxf(x1, 0.0f))));
  x0 = g.x;
  x1 = g.y;
}

// epilogues that write raw accumulators (no bias) as split-K partial planes [kparts][M][ldy]
constexpr bool is_partial(int e) { return e == ET_EPI_F32 || e == ET_EPI_PART16; }

// Accumulator hand-off waits (MMA warp <- epilogue drain, epilogue <- MMA commit).  -DET_GEMM_SPIN:
// spin without the suspend-time hint (a parked waiter's wake-up sits on the round's critical path).
#ifdef ET_GEMM_SPIN
#define GEMM_HANDOFF_WAIT(b, ph) mbar_wait_fast_warp((b), (ph))
#else
#define GEMM_HANDOFF_WAIT(b, ph) mbar_wait_warp((b), (ph))
#endif

// One GEMM (a piece bx of token block by, K part bz) on a CTA whose TMEM is allocated (bar.tmem_base):
// the kernel below runs one; tsgemm_ffn_kernel runs FFN1 piece c and then FFN2 K part c of the same
// token block in one CTA.  Ends with every store of the GEMM complete and a CTA barrier.
template <int kEpi, bool kBF16>
__device__ __forceinline__ void gemm_body(const CUtensorMap& tmap_x, const CUtensorMap& tmap_y, const Params& p,
                                          const int bx, const int by, const int bz, uint8_t* smem) {
  uint8_t* ring = smem;
  using SM = Smem<kEpi>;
  constexpr int kSlots = SM::kSlots;
  uint8_t* sStage = smem + SM::kRing;
  Barriers& bar = *reinterpret_cast<Barriers*>(smem + SM::kRing + SM::kStage);


  constexpr int kMmaWarps = Roles<kEpi>::MW, kEpiGroups = Roles<kEpi>::EG, kEpiWarps = Roles<kEpi>::EW;
  constexpr int kWarpP = Roles<kEpi>::WP, kFillSets = kWarpP / 4;
  constexpr int kAPW = kAcc / kMmaWarps;   // accumulators per MMA warp
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const Piece pc = p.piece[bx];
  const bool two = pc.seg1 != pc.seg;
  const SegDev& sa = p.seg[pc.seg];
  const SegDev& sb = p.seg[pc.seg1];
  const int m0 = by * 128;
  const int z = bz;
  const int nk = min(p.Kp, p.K - z * p.Kp) / 64;   // A chunks (64 K each) of this K part
  const int rowsA = (two ? sa.tile_rows : pc.i1) - pc.i0, rowsB = two ? pc.i1 : 0;
  const int32_t* rpa = sa.prp + (size_t)z * sa.rp_stride;
  const int32_t* rpb = sb.prp + (size_t)z * sb.rp_stride;
  const int pbA = rpa[pc.i0], peA = rpa[pc.i0 + rowsA];     // part A's packed tiles [pbA, peA)
  const int pbB = two ? rpb[0] : 0, peB = two ? rpb[rowsB] : 0;
  const int nchA = (peA - pbA + kChunkTiles - 1) / kChunkTiles;   // part B starts on a fresh tile chunk
  const int nchunks = nchA + (peB - pbB + kChunkTiles - 1) / kChunkTiles;
  const int nrows = rowsA + rowsB;
  const int nrounds = (nrows + kAcc - 1) / kAcc;   // row t: accumulator t % 8, round t / 8
  const int npairs_all = (nrows + 1) / 2;          // pair slots

  // A chunks are loaded in K order (the first round's MMAs follow the fill chunk by chunk).
  // ET_GEMM_A_ROT: rotate the order per piece instead (CTAs of one token block start a quarter of
  // the block apart) — measured no faster: the L2 serves the sharing CTAs well (profiles/r01).
#ifdef ET_GEMM_A_ROT
  const int a_rot = (bx & 3) * (nk >> 2);
#else
  constexpr int a_rot = 0;
#endif
  auto a_chunk = [&](int sq) { return sq + a_rot < nk ? sq + a_rot : sq + a_rot - nk; };
  // Ring positions: position s uses slot s % kSlots and recycles position s - kSlots; the A chunks
  // come first (positions 0 .. nk - 1), then the tile chunks.  (-DET_GEMM_T0_EARLY, the first tile
  // chunk moved ahead of the A chunks that do not fit the ring, measured slower: every GEMM
  // +0.5-0.7 us on C3, profiles/r02/ab_gemm_t0_early.txt; removed.)
  auto pos_t = [&](int c) { return nk + c; };
  // position -> load: >= 0 A chunk (load order index), < 0 tile chunk -(c + 1)
  auto at_pos = [&](int s) { return s < nk ? s : -(s - nk + 1); };
  // The producer issues the A loads that need no slot recycling (positions < kSlots) before the
  // block-wide setup: they depend only on the launch geometry, while the setup waits on global loads
  // of the weight's row pointers (measured ~1-1.5k cycles at kernel start, profiles/r02).
  const int n_early = min(nk, kSlots);
  if (warp == kWarpP && lane == 0) {
    for (int i = 0; i < kMaxKChunks; ++i) {
      mbar_init(&bar.xfull[i], 1);
      mbar_init(&bar.xfree[i], 4);
    }
    mbar_init(&bar.a_all, 4 * nk);
    fence_mbar_init();
    tma_prefetch_desc(&tmap_x);
    pdl_wait();
    if (p.ts != nullptr) atomicMin(p.ts, globaltimer_ns());   // trace: this CTA's work starts
    for (int s = 0; s < n_early; ++s) {
      mbar_expect_tx(&bar.xfull[s], p.box_rows * 128);
      tma_load_2d(ring + s * kSlotBytes, &tmap_x, &bar.xfull[s], z * p.Kp + a_chunk(s) * 64, m0);
    }
  }
  if (threadIdx.x == 0) ET_TL(0);
  ET_TL_RESET();
#ifdef ET_TIMELINE
  const unsigned cta_lin = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  if (threadIdx.x == 0 && cta_lin < 2048) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    g_cta_span[cta_lin][0] = globaltimer_ns();
    g_cta_span[cta_lin][2] = smid;
  }
#endif
  if (threadIdx.x == 0) {
    if (nchunks > kMaxBChunks || nrows > kMaxRows || (!is_partial(kEpi) && nrows > kMaxBiasRows))
      __trap();   // host sizes pieces so this cannot happen
    for (int i = 0; i < kAcc; ++i) mbar_init(&bar.acc_empty[i], 4);
    for (int j = 0; j < npairs_all; ++j)   // one commit per row (MMA warps) or per pair (epilogue-issued)
      mbar_init(&bar.slot_full[j], min(2, nrows - 2 * j));
    for (int i = 0; i < nchunks; ++i) mbar_init(&bar.bfull[i], 1);
    for (int i = 0; i < kMaxRows / 64; ++i) bar.pair_done[i] = 0u;
    fence_mbar_init();
  }
  // stage the per-CTA row pointers once (static weight metadata, not written by any predecessor, so
  // this overlaps the previous kernel's tail under PDL).  Everything the predecessor produces (A,
  // and a bias it may have computed) is read only after pdl_wait(): by the producer before its
  // first load and by the epilogue warps before they stage the bias.
  for (int i = threadIdx.x; i <= nrows; i += blockDim.x)
    bar.rptr[i] = i < rowsA ? rpa[pc.i0 + i] - pbA
                            : (two ? nchA * kChunkTiles + rpb[i - rowsA] - pbB : peA - pbA);
  if (threadIdx.x == 0) bar.a_end = two ? peA - pbA : 0x7fffffff;
  pdl_trigger();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = bar.tmem_base;
  if (threadIdx.x == 0) ET_TL(1);
  // end of local row t's tiles (part A's last row ends before the padding to part B's first chunk)
  auto rend = [&](int t) { return t == rowsA - 1 ? min(bar.a_end, bar.rptr[t + 1]) : bar.rptr[t + 1]; };

  // One tile row's MMA chain into accumulator `acc` (warp-collective; one elected lane issues).  The
  // row's tiles lie in chunks [q0 / 32, (q1 - 1) / 32]; a segment = the row's tiles inside one chunk:
  // wait for the chunk once, read the tile columns lane-parallel, issue the MMAs from register
  // broadcasts.  The first segment is prepared BEFORE `before_issue` (the accumulator hand-off), so
  // the barrier / shared-memory / shuffle latency stays off the accumulator's critical path.
  const uint32_t idesc = make_idesc_f16(128, 16, kBF16 ? 1 : 0, 0, 0);
  const uint32_t ring_u32 = smem_u32(ring);
  const int kbase = z * 48;   // first tile column of this K part
  auto issue_row = [&](int t, int acc, int k, int& cur_chunk, auto&& before_issue) {
    const uint32_t d_tmem = tbase + kAccCol + acc * 16;
    const int q0 = bar.rptr[t], q1 = rend(t);   // this row's tiles, relative to the CTA's stream
    int qb = q0, qe = q0, n = 0, mycol = 0;
    uint32_t acol = 0, blo = 0, bhi = 0;
    auto prep = [&]() {
      const int c = qb / kChunkTiles;
      qe = min(q1, (c + 1) * kChunkTiles);
      if (c != cur_chunk) {
        mbar_wait_warp(&bar.bfull[c], 0);
        if (lane == 0 && c < 40) ET_TL_MIN(400 + c);   // first time any issuer saw tile chunk c (debug)
        cur_chunk = c;
        tc_fence_after();
      }
      const int slot = pos_t(c) % kSlots;
      const int coff = two ? bar.tcoff[slot] : (pbA + c * kChunkTiles) & 3;
      n = qe - qb;
      mycol = lane < n ? bar.tcol[slot][coff + (qb % kChunkTiles) + lane] - kbase : 0;
      // B descriptor of tile u: start address field advances by 512 B / 16 = 32 per tile
      const uint64_t bd0 = make_sdesc(ring_u32 + slot * kSlotBytes + (qb % kChunkTiles) * 512, 128, 256,
                                      kLayoutNone);
      blo = (uint32_t)bd0;
      bhi = (uint32_t)(bd0 >> 32);
      acol = tbase + (uint32_t)(mycol * 8);   // this lane's tile: its A columns
    };
    if (qb < q1) prep();
    before_issue();
    if (lane == 0 && warp < kMmaWarps && k < 8) ET_TL(16 + 24 * warp + 3 * k);
    while (qb < q1) {
      int u = 0;
      for (; u + 4 <= n; u += 4) {
        if (lane == 0 && warp < kMmaWarps && k < 8 && qb + u == q0) ET_TL(16 + 24 * warp + 3 * k + 1);
        mma_ts_warp_x4(d_tmem, __shfl_sync(0xffffffffu, acol, u), __shfl_sync(0xffffffffu, acol, u + 1),
                       __shfl_sync(0xffffffffu, acol, u + 2), __shfl_sync(0xffffffffu, acol, u + 3),
                       blo + 32 * u, blo + 32 * (u + 1), blo + 32 * (u + 2), blo + 32 * (u + 3), bhi, idesc,
                       (qb + u) != q0);
      }
      for (; u < n; ++u) {
        const uint32_t a = __shfl_sync(0xffffffffu, acol, u);
        mma_ts_warp_nc(d_tmem, a, ((uint64_t)bhi << 32) | (blo + 32 * u), idesc, (qb + u) != q0);
      }
      qb = qe;
      if (qb < q1) prep();
    }
  };

  if (warp < kWarpP) {
    // A fill, smem ring -> TMEM through registers: chunk j is moved by the four warps of set j % 6,
    // warp w taking TMEM lane quarter w % 4 (its 32 token rows); lane i reads its row's 128 bytes from
    // the SWIZZLE_128B chunk (16-byte unit c of row r sits at unit c ^ (r % 8): conflict-free) and
    // one tcgen05.st.32x32b.x32 writes 32 packed columns.
    const int q = warp & 3;
    const int rr = q * 32 + lane;
    const uint32_t tq = tbase + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
    for (int sq = warp >> 2; sq < nk; sq += kFillSets) {   // load sequence position sq holds chunk j
      const int j = a_chunk(sq);
      mbar_wait_warp(&bar.xfull[sq], 0);
      const uint8_t* rowp = ring + (sq % kSlots) * kSlotBytes + rr * 128;
      uint32_t v[32];
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const uint4 u = *reinterpret_cast<const uint4*>(rowp + ((c ^ (rr & 7)) << 4));
        v[4 * c] = u.x; v[4 * c + 1] = u.y; v[4 * c + 2] = u.z; v[4 * c + 3] = u.w;
      }
      fence_proxy_async_smem();   // these generic-proxy reads precede the async-proxy refill of the slot
      __syncwarp();
      if (lane == 0) mbar_arrive(&bar.xfree[sq]);   // the producer may reuse the slot
      tmem_st32(tq + j * 32, v);
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&bar.a_all);
      if (lane == 0 && q == 0) ET_TL(2 + sq);
    }
  }

  if (warp == kWarpP) {
    // ===================== producer: A chunks (TMA) then tile chunks (bulk copies) through the ring.
    // Slot reuse: an A slot once its chunk was read out; a tile slot once every tile row touching
    // the old chunk completed its MMAs (row-granular; epilogue group g publishes rows_seen[g], its
    // rows being 8k + 2g + {0, 1}).  A row spans at most 3 tile chunks < kSlots, so the producer
    // never waits for a row that itself needs the chunk being loaded.
    if (lane == 0) {
      const int kx0 = z * p.Kp;
      int tl = 0;   // last local row that starts before the end of the tile chunk being recycled
      int pdone = 0;   // pair slots [0, pdone) known complete
      const int nseq = nk + nchunks;
      for (int s = n_early; s < nseq; ++s) {   // positions < n_early: issued before the setup
        const int slot = s % kSlots;
        const int prev = s - kSlots;
        if (prev >= 0) {
          const int lp = at_pos(prev);
          if (lp >= 0) {
            mbar_wait(&bar.xfree[lp], 0);
          } else {
            const int end_rel = (-lp) * kChunkTiles;   // tile chunk -lp - 1 ends here
            while (tl + 1 < nrows && bar.rptr[tl + 1] < end_rel) ++tl;
            // pair slots 0 .. tl / 2 (rows 0 .. tl) observed complete
            while (pdone <= (tl >> 1)) {
              while (!((ld_acquire_shared_u32(&bar.pair_done[pdone >> 5]) >> (pdone & 31)) & 1u)) {}
              ++pdone;
            }
          }
        }
        uint8_t* dst = ring + slot * kSlotBytes;
        const int ls = at_pos(s);
        if (ls >= 0) {
          mbar_expect_tx(&bar.xfull[ls], p.box_rows * 128);
          tma_load_2d(dst, &tmap_x, &bar.xfull[ls], kx0 + a_chunk(ls) * 64, m0);
        } else {
          const int c = -ls - 1;
          const bool inB = c >= nchA;
          const SegDev& sx = inB ? sb : sa;
          const int cc = inB ? c - nchA : c, pbx = inB ? pbB : pbA, pex = inB ? peB : peA;
          const int nt = min(kChunkTiles, pex - pbx - cc * kChunkTiles);
          // tile columns: copy from the 16-byte aligned start at or below the chunk's first entry
          // (tile_col is allocated with 16 bytes of slack, et_prune_pack_query)
          const int first = pbx + cc * kChunkTiles, off = first & 3;
          const int col_bytes = ((off + nt) * 4 + 15) & ~15;
          bar.tcoff[slot] = off;   // published by the expect_tx arrive (release) below
          mbar_expect_tx(&bar.bfull[c], nt * 512 + col_bytes);
          bulk_load(dst, sx.values + (size_t)first * 512, nt * 512, &bar.bfull[c]);
          bulk_load(&bar.tcol[slot][0], sx.tile_col + (first - off), col_bytes, &bar.bfull[c]);
        }
      }
      ET_TL(14);
    }
  } else if (warp < kMmaWarps) {
    // ===================== MMA warps: warp w issues the chains of tile rows w, w+8, w+16, ...
    // (Round 2 measured the alternative of the epilogue groups issuing their accumulator pair's next
    // chains right after draining it - a named barrier instead of the mbarrier hand-off: 29.1k / 34.9k
    // seq/s with one / two issuing warps per group against 41.1k, profiles/r02/ab_gemm_epilogue_issue.txt:
    // issue and epilogue math serialise on the same warps.)
    {
      int cur_chunk = -1;         // tile chunk whose full barrier was last waited
      // one wait for the whole A block (a wait on a completed mbarrier still costs ~100-300 cycles
      // of this warp's issue: per-chunk waits made the first round 2-3x slower than the others; round 2
      // re-measured lazy per-chunk spin waits - MMAs issued while the A block still arrives - at +0.9 us
      // per GEMM, profiles/r02/ab_gemm_a_progressive.txt: the MMA warps are also fill warps)
      mbar_wait_warp(&bar.a_all, 0);
      tc_fence_after();
      for (int kk = 0; kk < nrounds * kAPW; ++kk) {
        const int k = kk / kAPW;                     // round
        const int acc = warp + (kk % kAPW) * kMmaWarps;   // accumulator (rows in increasing order)
        const int t = k * kAcc + acc;
        if (t >= nrows) break;
        issue_row(t, acc, k, cur_chunk, [&]() {   // the epilogue group must have read the previous row
          if (k > 0) {
            GEMM_HANDOFF_WAIT(&bar.acc_empty[acc], (k - 1) & 1);
            tc_fence_after();
          }
        });
        mma_commit_warp(&bar.slot_full[t >> 1]);   // fires when this row's MMAs are complete
        if (lane == 0 && k < 8) ET_TL(16 + 24 * warp + 3 * k + 2);
      }
    }
  } else {
    // ===================== epilogue warps: group g drains the accumulators of MMA warps 2g, 2g+1
    const int ew = warp - kMmaWarps;
    if constexpr (!is_partial(kEpi)) {   // bias slice of this CTA's rows (16-bit pairs)
      pdl_wait();
      for (int i = ew * 32 + lane; i < nrows * 8; i += kEpiWarps * 32) {
        const int t = i >> 3;
        const uint32_t* bsrc = static_cast<const uint32_t*>(t < rowsA ? sa.bias : sb.bias);
        const int row = t < rowsA ? pc.i0 + t : t - rowsA;
        const float2 f = unpack2<kBF16>(bsrc ? __ldg(bsrc + (size_t)row * 8 + (i & 7)) : 0u);
        *reinterpret_cast<float2*>(&bar.bias_f[2 * i]) = f;
      }
      named_bar_sync(1, kEpiWarps * 32);
    }
    const int g = ew >> 2;
    const int quarter = warp & 3;               // TMEM lane quarter this warp may access
    uint8_t* st = sStage + ew * SM::kStageWarp;
    // Per round: wait for the group's 2 accumulators (rows 8k + 2g + a), read their 32 columns with
    // one TMEM load, release them to the MMA warps, THEN do the bias / activation / store math (so
    // an MMA warp never waits for another row's epilogue arithmetic).
    for (int jp = g, it = 0; jp < npairs_all; jp += kEpiGroups, ++it) {
      const int k = jp >> 2, pidx = jp & 3;   // round, pair within the round (accumulators 2p, 2p+1)
      const int t0 = 2 * jp;                  // first row of the pair
      const int na = min(2, nrows - t0);
      uint32_t r[32];
      (void)k;
      GEMM_HANDOFF_WAIT(&bar.slot_full[jp], 0);   // single-use: both rows' MMAs complete
      if (quarter == 0 && lane == 0 && it < 8 && g < 4) ET_TL(208 + 40 * g + 5 * it);
      tc_fence_after();
      if (quarter == 0 && lane == 0)   // the pair's MMAs are complete: their tiles are free
        atom_or_release_shared(&bar.pair_done[jp >> 5], 1u << (jp & 31));
      tmem_ld32(tbase + kAccCol + pidx * 32 + ((uint32_t)(quarter * 32) << 16), r);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0)
        for (int a = 0; a < na; ++a) mbar_arrive(&bar.acc_empty[pidx * 2 + a]);
      if (quarter == 0 && lane == 0 && it < 8 && g < 4) ET_TL(208 + 40 * g + 5 * it + 1);
      if (quarter > 0 && lane == 0 && it < 4 && g == 0) ET_TL(386 + 4 * (quarter - 1) + it);   // debug
      // math: bias / scale / activation on the pair's 32 columns of this thread's token row
      float v[32];
#pragma unroll
      for (int a = 0; a < 2; ++a) {
        const int t = t0 + min(a, na - 1);
        // a row with no kept tile was never written: its accumulator is zero (output = epi(bias))
        const bool empty_row = a >= na || rend(t) == bar.rptr[t];
        const float4* bt = reinterpret_cast<const float4*>(&bar.bias_f[(is_partial(kEpi) ? 0 : t) * 16]);
        float sc = 1.0f;
        if constexpr (kEpi == ET_EPI_BIAS_SCALE) {
          const SegDev& st_seg = t < rowsA ? sa : sb;
          if (st_seg.apply_scale) sc = st_seg.scale;
        }
        if (empty_row) {   // rare (no kept tile in the row): a branch, not 16 selects per row
          asm volatile("" ::: "memory");
#pragma unroll
          for (int c = 0; c < 16; ++c) r[a * 16 + c] = 0u;
        }
#pragma unroll
        for (int c = 0; c < 16; c += 2) {
          float x0 = __uint_as_float(r[a * 16 + c]);
          float x1 = __uint_as_float(r[a * 16 + c + 1]);
          if constexpr (!is_partial(kEpi)) {
            const float4 b4 = bt[c / 4];   // broadcast LDS.128, shared by every thread of the group
            const float2 bb = (c & 2) ? make_float2(b4.z, b4.w) : make_float2(b4.x, b4.y);
            uint64_t xx = fadd2(f2pk(x0, x1), f2pk(bb.x, bb.y));
            if constexpr (kEpi == ET_EPI_BIAS_SCALE) xx = fmul2(xx, f2pk(sc, sc));
            const float2 xf = f2upk(xx);
            x0 = xf.x;
            x1 = xf.y;
            if constexpr (kEpi == ET_EPI_BIAS_GELU) {
              gelu_erf2(x0, x1);
            } else if constexpr (kEpi == ET_EPI_BIAS_RELU) {
              x0 = fmaxf(x0, 0.0f);
              x1 = fmaxf(x1, 0.0f);
            }
          }
          v[a * 16 + c] = x0;
          v[a * 16 + c + 1] = x1;
        }
      }
      if (quarter == 0 && lane == 0 && it < 8 && g < 4) ET_TL(208 + 40 * g + 5 * it + 2);
      // store: registers -> this warp's 32-row staging tile -> one TMA tensor store (clipped at M by
      // the tensor map).  fp32: 128-byte rows, SWIZZLE_128B (unit c of row r at c ^ (r % 8));
      // 16-bit: 64-byte rows, SWIZZLE_64B (unit c of row r at c ^ ((r / 2) % 4)); both conflict-free.
      // output columns: segments of a two-part piece are output-contiguous (checked on the host)
      const int col0 = t0 < rowsA ? sa.out_col + (pc.i0 + t0) * 16 : sb.out_col + (t0 - rowsA) * 16;
      const int row0 = m0 + quarter * 32;
#ifdef ET_GEMM_DIRECT_ST
      constexpr bool kDirect = true;
#else
      constexpr bool kDirect = false;
#endif
      if (na == 2 && !kDirect) {
        if (lane == 0) bulk_wait_group_read<0>();   // the previous store finished reading the staging tile
        __syncwarp();
        if constexpr (kEpi == ET_EPI_F32) {
#pragma unroll
          for (int ch = 0; ch < 8; ++ch) {
            const float* f = v + ch * 4;
            *reinterpret_cast<uint4*>(st + lane * 128 + ((ch ^ (lane & 7)) << 4)) =
                make_uint4(__float_as_uint(f[0]), __float_as_uint(f[1]), __float_as_uint(f[2]), __float_as_uint(f[3]));
          }
        } else {
#pragma unroll
          for (int ch = 0; ch < 4; ++ch) {
            const float* f = v + ch * 8;
            *reinterpret_cast<uint4*>(st + lane * 64 + ((ch ^ ((lane >> 1) & 3)) << 4)) =
                make_uint4(pack2<kBF16>(f[0], f[1]), pack2<kBF16>(f[2], f[3]), pack2<kBF16>(f[4], f[5]),
                           pack2<kBF16>(f[6], f[7]));
          }
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          if constexpr (is_partial(kEpi)) tma_store_3d(&tmap_y, st, col0, row0, z);
          else tma_store_2d(&tmap_y, st, col0, row0);
          bulk_commit_group();
        }
      } else {
        // direct stores (-DET_GEMM_DIRECT_ST: every pair; otherwise a lone last row of the piece, so
        // nothing is written into the neighbouring piece's or segment's columns): 16 columns per row
        const int row = row0 + lane;
        if (row < p.M) {
#pragma unroll
          for (int a = 0; a < 2; ++a) {
            if (a >= na) break;
            const float* va = v + 16 * a;
            if constexpr (kEpi == ET_EPI_F32) {
              float* y = static_cast<float*>(p.Y) + (size_t)z * p.part_stride + (size_t)row * p.ldy + col0 + 16 * a;
#pragma unroll
              for (int c = 0; c < 16; c += 4)
                *reinterpret_cast<float4*>(y + c) = make_float4(va[c], va[c + 1], va[c + 2], va[c + 3]);
            } else {
              uint16_t* y = static_cast<uint16_t*>(p.Y) + (kEpi == ET_EPI_PART16 ? (size_t)z * p.part_stride : 0) +
                            (size_t)row * p.ldy + col0 + 16 * a;
              *reinterpret_cast<uint4*>(y) = make_uint4(pack2<kBF16>(va[0], va[1]), pack2<kBF16>(va[2], va[3]),
                                                        pack2<kBF16>(va[4], va[5]), pack2<kBF16>(va[6], va[7]));
              *reinterpret_cast<uint4*>(y + 8) = make_uint4(pack2<kBF16>(va[8], va[9]), pack2<kBF16>(va[10], va[11]),
                                                            pack2<kBF16>(va[12], va[13]), pack2<kBF16>(va[14], va[15]));
            }
          }
        }
      }
      if (quarter == 0 && lane == 0 && it < 8 && g < 4) ET_TL(208 + 40 * g + 5 * it + 3);
    }
  }
  if (warp >= kMmaWarps && warp < kWarpP && lane == 0) bulk_wait_group<0>();   // epilogue stores done
  __syncwarp();   // the producer warp: lane 0 ran the loop alone; reconverge before the block barrier
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) ET_TL(500);
#ifdef ET_TIMELINE
  if (threadIdx.x == 0 && cta_lin < 2048) g_cta_span[cta_lin][1] = globaltimer_ns();
#endif
  trace_cta_end(p.ts);
}

template <int kEpi, bool kBF16>
__global__ void __launch_bounds__(Roles<kEpi>::threads, 1) tsgemm_kernel(const __grid_constant__ CUtensorMap tmap_x,
                                                             const __grid_constant__ CUtensorMap tmap_y,
                                                             const __grid_constant__ Params p) {
  extern __shared__ uint8_t smem_raw[];
  // 1024-byte aligned, derived from smem_raw by pointer arithmetic so the compiler keeps the shared
  // address space (an integer round trip would turn every access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  Barriers& bar = *reinterpret_cast<Barriers*>(smem + Smem<kEpi>::kRing + Smem<kEpi>::kStage);
  const int warp = threadIdx.x >> 5;
  if (warp == Roles<kEpi>::WP) tmem_alloc<512>(&bar.tmem_base);   // published by gemm_body's first barrier
  gemm_body<kEpi, kBF16>(tmap_x, tmap_y, p, blockIdx.x, blockIdx.y, blockIdx.z, smem);
  if (warp == Roles<kEpi>::WP) {
    __syncwarp();
    tc_fence_after();
    tmem_dealloc<512>(bar.tmem_base);   // .sync.aligned: the whole warp, converged
  }
}

// FFN1 -> FFN2 in one CTA (NEXT-4's FFN fusion without a cross-CTA exchange): FFN1's piece c of a
// token block is the tile-row range [48c, 48c + 48) of W_1, i.e. exactly the 768 U columns that form
// FFN2's K part c, so the CTA that produced them runs FFN2's K part c next.  U still goes through L2
// (the CTA's own TMA stores, complete at the end of phase 1, read back by phase 2's TMA loads), but the
// FFN2 kernel boundary - launch, prologue, the wait for FFN1's slowest CTA - disappears.
template <int kEpi1, int kEpi2, bool kBF16>
__global__ void __launch_bounds__(Roles<kEpi1>::threads, 1) tsgemm_ffn_kernel(const __grid_constant__ CUtensorMap tmx1,
                                                                  const __grid_constant__ CUtensorMap tmy1,
                                                                  const __grid_constant__ CUtensorMap tmx2,
                                                                  const __grid_constant__ CUtensorMap tmy2,
                                                                  const __grid_constant__ Params p1,
                                                                  const __grid_constant__ Params p2) {
  static_assert(Smem<kEpi1>::kRing == Smem<kEpi2>::kRing && Smem<kEpi1>::kStage == Smem<kEpi2>::kStage,
                "both phases share one shared-memory layout");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  Barriers& bar = *reinterpret_cast<Barriers*>(smem + Smem<kEpi1>::kRing + Smem<kEpi1>::kStage);
  const int warp = threadIdx.x >> 5;
  if (warp == Roles<kEpi1>::WP) tmem_alloc<512>(&bar.tmem_base);
  gemm_body<kEpi1, kBF16>(tmx1, tmy1, p1, blockIdx.x, blockIdx.y, 0, smem);
  // phase 1's U stores are complete (bulk wait + barrier at the end of gemm_body); order them before
  // phase 2's loads of the same bytes, and every phase-1 tcgen05 op before phase 2 refills TMEM
  asm volatile("fence.proxy.async.global;" ::: "memory");
  __threadfence();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  gemm_body<kEpi2, kBF16>(tmx2, tmy2, p2, 0, blockIdx.y, blockIdx.x, smem);
  if (warp == Roles<kEpi1>::WP) {
    __syncwarp();
    tc_fence_after();
    tmem_dealloc<512>(bar.tmem_base);
  }
}

// ---------------------------------------------------------------- host side
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(ptr);
  });
  return fn;
}

template <int kEpi, bool kBF16>
et_status launch_typed(const CUtensorMap& tm, const CUtensorMap& tmy, const Params& prm, dim3 grid,
                       cudaStream_t stream) {
  auto kern = tsgemm_kernel<kEpi, kBF16>;
  static std::once_flag once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(once, [&] {
    attr_err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Smem<kEpi>::kBytes);
  });
  ET_CUDA(attr_err);
  ET_CUDA(launch_pdl(kern, grid, dim3(Roles<kEpi>::threads), Smem<kEpi>::kBytes, stream, tm, tmy, prm));
  count_launch();
  return ET_OK;
}

}  // namespace

et_status make_tmap_2d(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                       uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows, bool swizzle128) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {ld_elems * dtype_size(dtype)};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUtensorMapDataType dt = dtype == ET_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                           : dtype == ET_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                              : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  CUresult r = enc(tm, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return ET_OK;
}

et_status make_tmap_2d_sw64(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                            uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {ld_elems * dtype_size(dtype)};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUtensorMapDataType dt = dtype == ET_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  CUresult r = enc(tm, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled (sw64) failed (%d)", (int)r);
  return ET_OK;
}

// [planes][rows][cols] tensor (fp32: SWIZZLE_128B, box 32 cols = 128 B; 16-bit: SWIZZLE_64B, 32 cols = 64 B)
et_status make_tmap_3d(CUtensorMap* tm, void* base, et_dtype dtype, uint64_t cols, uint64_t rows, uint64_t planes,
                       uint32_t box_cols, uint32_t box_rows) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  const uint64_t es = dtype_size(dtype);
  cuuint64_t dims[3] = {cols, rows, planes};
  cuuint64_t strides[2] = {cols * es, cols * rows * es};
  cuuint32_t box[3] = {box_cols, box_rows, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUtensorMapDataType dt = dtype == ET_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                           : dtype == ET_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                              : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  CUresult r = enc(tm, dt, 3, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   es == 4 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled (3d) failed (%d)", (int)r);
  return ET_OK;
}

// [planes][rows][cols] 16-bit tensor with a row pitch of ld_elems (>= cols), SWIZZLE_128B boxes of
// box_cols (64) x box_rows; elements outside [cols, rows] read as zero and are dropped on stores
// (the partial-OTF score matrix, kernels/attention_partial.cu).
et_status make_tmap_3d_ld(CUtensorMap* tm, void* base, et_dtype dtype, uint64_t cols, uint64_t rows, uint64_t planes,
                          uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  const uint64_t es = dtype_size(dtype);
  cuuint64_t dims[3] = {cols, rows, planes};
  cuuint64_t strides[2] = {ld_elems * es, ld_elems * rows * es};
  cuuint32_t box[3] = {box_cols, box_rows, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUtensorMapDataType dt = dtype == ET_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  CUresult r = enc(tm, dt, 3, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(ET_ERR_CUDA, "cuTensorMapEncodeTiled (3d, ld) failed (%d)", (int)r);
  return ET_OK;
}

// Launch plan of one tile GEMM: parameters, tensor maps and grid.  force_pieces > 0 replaces the
// piece planner with that many equal tile-row pieces of the (single) segment (the FFN fusion needs
// FFN1's pieces to coincide with FFN2's K parts).  *np_out = 0: nothing to launch (M == 0).
static et_status build_gemm(const GemmArgs& a, Params& prm, CUtensorMap& tm, CUtensorMap& tmy, dim3& grid,
                            int force_pieces, int* np_out) {
  *np_out = 0;
  if (a.K % 64) return fail(ET_ERR_UNSUPPORTED, "tile GEMM: K must be a multiple of 64 (got %d)", a.K);
  if (!aligned16(a.X) || (a.ldx * 2) % 16 || (a.k0 * 2) % 16)
    return fail(ET_ERR_INVALID_ARG, "tile GEMM: X must be 16-byte aligned with 16-byte row pitch");
  const int kparts = (a.K + 767) / 768;
  if (kparts > 1 && a.epi != ET_EPI_F32 && a.epi != ET_EPI_PART16)
    return fail(ET_ERR_UNSUPPORTED, "tile GEMM: K > 768 needs a partial-sum (split-K) epilogue");
  if (a.M <= 0) return ET_OK;

  prm = Params{};
  prm.M = a.M;
  prm.K = a.K;
  prm.box_rows = a.M < 128 ? a.M : 128;
  prm.X = static_cast<const uint8_t*>(a.X) + (size_t)a.k0 * 2;
  prm.ldx_bytes = (long long)a.ldx * 2;
  prm.Kp = kparts > 1 ? 768 : a.K;
  prm.kparts = kparts;
  prm.nseg = a.nseg;
  prm.Y = a.Y;
  prm.ldy = a.ldy;
  prm.part_stride = (long long)a.M * a.ldy;
  prm.ts = a.ts;
  const int mblocks = (a.M + 127) / 128;
  int total_rows = 0;
  for (int s = 0; s < a.nseg; ++s) total_rows += a.seg[s].tile_rows;
  // pieces: one wave of CTAs over the 148 SMs (a nearly empty second wave would double the time)
  const int target_ctas = 148;
  int pieces_total = target_ctas / (mblocks * kparts);
  if (pieces_total < 1) pieces_total = 1;
  if (pieces_total < a.nseg) pieces_total = a.nseg;
  for (int s = 0; s < a.nseg; ++s) {
    const GemmSegment& gs = a.seg[s];
    prm.seg[s].prp = gs.row_ptr;
    prm.seg[s].tile_col = gs.tile_col;
    prm.seg[s].values = static_cast<const uint8_t*>(gs.values);
    prm.seg[s].bias = gs.bias;
    prm.seg[s].tile_rows = gs.tile_rows;
    prm.seg[s].rp_stride = gs.rp_stride ? gs.rp_stride : gs.tile_rows + 1;
    prm.seg[s].out_col = gs.out_col;
    prm.seg[s].scale = gs.scale;
    prm.seg[s].apply_scale = gs.apply_scale;
  }
  const int kt = std::min(a.K, 768) / 16;   // tile columns per K part (bound on tiles per row)
  const int max_rows = is_partial(a.epi) ? kMaxRows : kMaxBiasRows;
  auto fits = [&](int rows) { return rows <= max_rows && (long long)rows * kt + kChunkTiles <= (long long)kMaxBChunks * kChunkTiles; };
  int np = 0;
  // Output-contiguous segments (Q|K|V): plan the pieces over the concatenated tile rows, so the CTA
  // count is set by the total rows rather than rounded per segment (4 pieces of 36 rows instead of
  // 3 of 48 for BERT-base); a piece may straddle one segment boundary.
  bool contiguous = a.nseg > 1;
  for (int s = 1; s < a.nseg; ++s)
    contiguous = contiguous && a.seg[s].out_col == a.seg[s - 1].out_col + a.seg[s - 1].tile_rows * 16;
  if (contiguous) {
    int start[4] = {0, 0, 0, 0};
    for (int s = 0; s < a.nseg; ++s) start[s + 1] = start[s] + a.seg[s].tile_rows;
    const int q4 = (total_rows + 3) / 4;
    int ps = std::max(1, std::min(pieces_total, q4));
    bool ok = false;
    for (; ps <= q4 && !ok; ++ps) {
      ok = true;
      np = 0;
      for (int k = 0; k < ps && ok; ++k) {
        const int g0 = std::min(total_rows, 4 * (int)((long long)q4 * k / ps));
        const int g1 = std::min(total_rows, 4 * (int)((long long)q4 * (k + 1) / ps));
        if (g1 <= g0) continue;
        int s0 = 0;
        while (g0 >= start[s0 + 1]) ++s0;
        int s1 = s0;
        while (g1 > start[s1 + 1]) ++s1;
        if (s1 > s0 + 1 || !fits(g1 - g0) || np >= kMaxPieces) {
          ok = false;
          break;
        }
        prm.piece[np].seg = (int16_t)s0;
        prm.piece[np].seg1 = (int16_t)s1;
        prm.piece[np].i0 = (int16_t)(g0 - start[s0]);
        prm.piece[np].i1 = (int16_t)(g1 - start[s1]);
        ++np;
      }
    }
    if (!ok) contiguous = false;
  }
  if (force_pieces > 0) {
    if (a.nseg != 1 || a.seg[0].tile_rows % force_pieces || force_pieces > kMaxPieces ||
        !fits(a.seg[0].tile_rows / force_pieces))
      return fail(ET_ERR_INTERNAL, "tile GEMM: forced piece plan does not fit");
    const int R = a.seg[0].tile_rows / force_pieces;
    np = 0;
    for (int k = 0; k < force_pieces; ++k) {
      prm.piece[np].seg = prm.piece[np].seg1 = 0;
      prm.piece[np].i0 = (int16_t)(k * R);
      prm.piece[np].i1 = (int16_t)((k + 1) * R);
      ++np;
    }
  } else if (!contiguous) {
    np = 0;
    for (int s = 0; s < a.nseg; ++s) {
      const GemmSegment& gs = a.seg[s];
      int ps = (int)(((long long)pieces_total * gs.tile_rows * 2 + (total_rows > 0 ? total_rows : 1)) /
                     (2LL * (total_rows > 0 ? total_rows : 1)));   // rounded
      ps = std::max(1, std::min(ps, std::max(1, gs.tile_rows / 8)));
      const int q4 = (gs.tile_rows + 3) / 4;
      for (;;) {   // each piece's tile stream must fit the per-CTA chunk / row budgets
        bool ok = true;
        for (int k = 0; k < ps && ok; ++k)
          ok = fits(std::min(gs.tile_rows, 4 * (int)((long long)q4 * (k + 1) / ps)) -
                    std::min(gs.tile_rows, 4 * (int)((long long)q4 * k / ps)));
        if (ok || ps >= q4) break;
        ++ps;
      }
      ps = std::min(ps, q4);   // no empty pieces
      for (int k = 0; k < ps; ++k) {
        if (np >= kMaxPieces) return fail(ET_ERR_INTERNAL, "tile GEMM: too many pieces");
        prm.piece[np].seg = prm.piece[np].seg1 = (int16_t)s;
        // piece boundaries on multiples of 4 tile rows (an epilogue pair never straddles two CTAs)
        prm.piece[np].i0 = (int16_t)std::min(gs.tile_rows, 4 * (int)((long long)q4 * k / ps));
        prm.piece[np].i1 = (int16_t)std::min(gs.tile_rows, 4 * (int)((long long)q4 * (k + 1) / ps));
        ++np;
      }
    }
  }
  prm.npieces = np;
  // the K offset k0 is folded into the base address
  ET_TRY(make_tmap_2d(&tm, static_cast<const uint8_t*>(a.X) + (size_t)a.k0 * 2, a.dtype, (uint64_t)a.M,
                      (uint64_t)a.K, (uint64_t)a.ldx, 64, (uint32_t)prm.box_rows, true));
  // output tensor map: [M, ldy] in the operand dtype, box 32 cols x 32 rows (one epilogue warp's
  // staging tile, SWIZZLE_64B); fp32 partials: [kparts, M, ldy], box 32 x 32 x 1 (SWIZZLE_128B).
  if (a.epi == ET_EPI_F32 || a.epi == ET_EPI_PART16) {
    ET_TRY(make_tmap_3d(&tmy, a.Y, a.epi == ET_EPI_F32 ? ET_FP32 : a.dtype, (uint64_t)a.ldy, (uint64_t)a.M,
                        (uint64_t)kparts, 32, a.M < 32 ? (uint32_t)a.M : 32u));
  } else {
    ET_TRY(make_tmap_2d_sw64(&tmy, a.Y, a.dtype, (uint64_t)a.M, (uint64_t)a.ldy, (uint64_t)a.ldy, 32,
                             a.M < 32 ? (uint32_t)a.M : 32u));
  }
  grid = dim3(np, mblocks, kparts);
  *np_out = np;
  return ET_OK;
}

et_status gemm_run(const GemmArgs& a, cudaStream_t stream) {
  if (a.dtype == ET_FP32) return gemm32_run(a, stream);   // FP32 validation build (CUDA cores)
  Params prm;
  CUtensorMap tm, tmy;
  dim3 grid;
  int np = 0;
  ET_TRY(build_gemm(a, prm, tm, tmy, grid, 0, &np));
  if (np == 0) return ET_OK;
  const bool bf = a.dtype == ET_BF16;
  switch ((int)a.epi) {
    case ET_EPI_BIAS: return bf ? launch_typed<ET_EPI_BIAS, true>(tm, tmy, prm, grid, stream)
                                : launch_typed<ET_EPI_BIAS, false>(tm, tmy, prm, grid, stream);
    case ET_EPI_BIAS_SCALE: return bf ? launch_typed<ET_EPI_BIAS_SCALE, true>(tm, tmy, prm, grid, stream)
                                      : launch_typed<ET_EPI_BIAS_SCALE, false>(tm, tmy, prm, grid, stream);
    case ET_EPI_BIAS_GELU: return bf ? launch_typed<ET_EPI_BIAS_GELU, true>(tm, tmy, prm, grid, stream)
                                     : launch_typed<ET_EPI_BIAS_GELU, false>(tm, tmy, prm, grid, stream);
    case ET_EPI_BIAS_RELU: return bf ? launch_typed<ET_EPI_BIAS_RELU, true>(tm, tmy, prm, grid, stream)
                                     : launch_typed<ET_EPI_BIAS_RELU, false>(tm, tmy, prm, grid, stream);
    case ET_EPI_F32: return bf ? launch_typed<ET_EPI_F32, true>(tm, tmy, prm, grid, stream)
                               : launch_typed<ET_EPI_F32, false>(tm, tmy, prm, grid, stream);
    case ET_EPI_PART16: return bf ? launch_typed<ET_EPI_PART16, true>(tm, tmy, prm, grid, stream)
                                  : launch_typed<ET_EPI_PART16, false>(tm, tmy, prm, grid, stream);
    default: break;
  }
  return fail(ET_ERR_INVALID_ARG, "tile GEMM: bad epilogue %d", (int)a.epi);
}

// FFN1 -> FFN2 in one launch (tsgemm_ffn_kernel).  Applies when FFN1 has one segment with K <= 768
// and a 16-bit bias + activation epilogue, FFN2 writes 16-bit split-K partial planes over K = FFN1's
// output width, and FFN1 split into FFN2's K parts (768 output columns = 48 tile rows each) gives at
// least 96 CTAs (C3: 4 pieces x 32 token blocks; C4 / C5: many waves).
bool gemm_ffn_applies(const GemmArgs& f1, const GemmArgs& f2) {
  if (f1.dtype == ET_FP32 || f1.dtype != f2.dtype || f1.nseg != 1 || f2.nseg != 1 || f1.M != f2.M) return false;
  if (f1.K > 768 || (f1.epi != ET_EPI_BIAS_GELU && f1.epi != ET_EPI_BIAS_RELU) || f2.epi != ET_EPI_PART16) return false;
  if (f2.X != f1.Y || f2.ldx != f1.ldy || f2.k0 != 0 || f2.K != f1.seg[0].tile_rows * 16 || f2.K % 768) return false;
  const int kparts = f2.K / 768, mblocks = (f1.M + 127) / 128;
  // no upper bound: the phases of a CTA depend on nothing outside it, so any number of waves works
  // (and there U_c is read back while still in L2 instead of after the whole U left it)
  return kparts * mblocks >= 96 && f1.seg[0].tile_rows == kparts * 48;
}

et_status gemm_ffn_run(const GemmArgs& f1, const GemmArgs& f2, cudaStream_t stream) {
  if (!gemm_ffn_applies(f1, f2)) return fail(ET_ERR_INTERNAL, "FFN fusion does not apply");
  Params p1, p2;
  CUtensorMap tx1, ty1, tx2, ty2;
  dim3 g1, g2;
  int np1 = 0, np2 = 0;
  ET_TRY(build_gemm(f1, p1, tx1, ty1, g1, f2.K / 768, &np1));
  ET_TRY(build_gemm(f2, p2, tx2, ty2, g2, 1, &np2));
  if (np1 == 0) return ET_OK;
  if ((int)g1.x != (int)g2.z || g1.y != g2.y || g2.x != 1) return fail(ET_ERR_INTERNAL, "FFN fusion: plans differ");
  const bool bf = f1.dtype == ET_BF16;
  auto go = [&](auto kern) -> et_status {
    static std::once_flag once;
    static cudaError_t attr_err = cudaSuccess;
    std::call_once(once, [&] {
      attr_err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)Smem<ET_EPI_PART16>::kBytes);
    });
    ET_CUDA(attr_err);
    ET_CUDA(launch_pdl(kern, g1, dim3(Roles<ET_EPI_PART16>::threads), Smem<ET_EPI_PART16>::kBytes, stream, tx1, ty1,
                       tx2, ty2, p1, p2));
    count_launch();
    return ET_OK;
  };
  if (f1.epi == ET_EPI_BIAS_GELU)
    return bf ? go(tsgemm_ffn_kernel<ET_EPI_BIAS_GELU, ET_EPI_PART16, true>)
              : go(tsgemm_ffn_kernel<ET_EPI_BIAS_GELU, ET_EPI_PART16, false>);
  return bf ? go(tsgemm_ffn_kernel<ET_EPI_BIAS_RELU, ET_EPI_PART16, true>)
            : go(tsgemm_ffn_kernel<ET_EPI_BIAS_RELU, ET_EPI_PART16, false>);
}

#ifdef ET_TIMELINE
extern "C" int et_diag_gemm_cta_spans(unsigned long long* host_out) {
  return cudaMemcpyFromSymbol(host_out, g_cta_span, sizeof(g_cta_span)) == cudaSuccess ? 0 : 4;
}
extern "C" int et_diag_gemm_timeline(unsigned long long* host_out) {
  return cudaMemcpyFromSymbol(host_out, g_timeline, sizeof(g_timeline)) == cudaSuccess ? 0 : 4;
}
#endif

}  // namespace et
