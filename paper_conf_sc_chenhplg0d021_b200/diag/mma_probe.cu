// M1 diagnostic: tcgen05.mma shape/operand-source probe.
//
// Computes D[128 x N] = iters * (A[128 x 64] . B^T) with one CTA per SM and reports the cycles
// the single issuing thread needed, for
//   a_mode 0: A from shared memory (SS), K-major SWIZZLE_128B
//   a_mode 1: A from TMEM (TS), loaded row-per-lane with tcgen05.st
// and B in shared memory as
//   b_mode 0: K-major SWIZZLE_128B                                   (B given as [N, 64])
//   b_mode 1: K-major no-swizzle core matrices, one 16-wide K slice per block, LBO=128 SBO=256
//             -- exactly the packed 16x16 weight-tile layout of the tile-sparse GEMM ([N, 64])
//   b_mode 2: MN-major SWIZZLE_128B, N % 64 == 0 (the V operand of P.V)  (B given as [64, N])
// It validates the descriptor / TMEM conventions used by the real kernels and measures whether
// N=16 MMAs (one per 16x16 tile) reach the tcgen05 floor of 8 cycles.
#include <cuda_runtime.h>
#include <cstdint>
#include "ptx.cuh"

namespace et {

__global__ void __launch_bounds__(512, 1)
mma_probe_kernel(const __half* __restrict__ A, const __half* __restrict__ B, float* __restrict__ D, int N,
                 int a_mode, int b_mode, int iters, int n_acc, int issue_mode, long long* __restrict__ cycles) {
  extern __shared__ uint8_t smem_raw[];
  // 1024-byte aligned, derived from smem_raw by pointer arithmetic so the compiler keeps the shared
  // address space (an integer round trip would turn every access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;                // 16 KB
  uint8_t* sB = smem + 16384;        // up to 32 KB
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem_base_s;

  const int t = threadIdx.x;
  const int warp = t >> 5;

  // ---- fill A (K-major SW128): row t, 16-byte chunk c -> t*128 + ((c ^ (t&7)) * 16)
  if (t < 128) {
    const uint4* src = reinterpret_cast<const uint4*>(A + t * 64);
    for (int c = 0; c < 8; ++c)
      *reinterpret_cast<uint4*>(sA + t * 128 + ((c ^ (t & 7)) << 4)) = src[c];
  }
  // ---- fill B
  if (b_mode == 0) {
    for (int n = t; n < N; n += blockDim.x) {
      const uint4* src = reinterpret_cast<const uint4*>(B + n * 64);
      for (int c = 0; c < 8; ++c)
        *reinterpret_cast<uint4*>(sB + n * 128 + ((c ^ (n & 7)) << 4)) = src[c];
    }
  } else if (b_mode == 1) {
    for (int n = t; n < N; n += blockDim.x) {
      for (int k8 = 0; k8 < 8; ++k8) {   // 8 halves per 16-byte core-matrix row
        const int s = k8 >> 1, kh = k8 & 1;
        uint8_t* dst = sB + s * (N * 32) + (n >> 3) * 256 + kh * 128 + (n & 7) * 16;
        *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(B + n * 64 + k8 * 8);
      }
    }
  } else {
    // B given as [64 (k), N]; atom a = n/64 is a 64 x 128B block at a*8192
    for (int idx = t; idx < 64 * (N / 8); idx += blockDim.x) {
      const int k = idx / (N / 8), cc = idx % (N / 8);
      const int a = cc >> 3, c = cc & 7;
      uint8_t* dst = sB + a * 8192 + (k >> 3) * 1024 + (k & 7) * 128 + ((c ^ (k & 7)) << 4);
      *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(B + k * N + cc * 8);
    }
  }
  fence_proxy_async_smem();   // generic-proxy smem writes -> visible to the tensor core (async proxy)

  if (warp == 0) tmem_alloc<512>(&tmem_base_s);
  if (t == 0) {
    mbar_init(&bar, issue_mode >= 100 ? issue_mode - 100 : (issue_mode >= 2 ? issue_mode : 1));
    fence_mbar_init();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tmem_base_s;
  const uint32_t a_col = 448;

  __shared__ uint64_t cpbar;
  if (a_mode == 2) {
    // A via tcgen05.cp from the K-major SW128 smem copy: 4 x (128 rows x 16 halves) -> 4 x 8 columns
    if (t == 0) {
      mbar_init(&cpbar, 1);
      fence_mbar_init();
      long long c0 = clock64();
      for (int s = 0; s < 4; ++s)
        tmem_cp_128x256b(tbase + a_col + s * 8, make_sdesc(smem_u32(sA) + s * 32, 16, 1024, kLayoutSW128));
      mma_commit(&cpbar);
      mbar_wait(&cpbar, 0);
      if (blockIdx.x == 0) cycles[gridDim.x] = clock64() - c0;
    }
  }
  if (issue_mode >= 100 && warp < 4) {   // shared-accumulator mode: pre-zero D (this warp's lanes)
    uint32_t zr[16];
    for (int i = 0; i < 16; ++i) zr[i] = 0u;
    for (int c = 0; c < N * n_acc; c += 16) tmem_st16(tbase + ((uint32_t)(warp * 32) << 16) + c, zr);
    tmem_st_wait();
  }
  if (a_mode == 1 && warp < 4) {
    // A row t -> TMEM lane t, columns [256, 288): 2 halves per 32-bit column, low half = even k
    uint32_t r[32];
    const uint32_t* src = reinterpret_cast<const uint32_t*>(A + t * 64);
    for (int i = 0; i < 32; ++i) r[i] = src[i];
    tmem_st32(tbase + ((uint32_t)(warp * 32) << 16) + a_col, r);
    tmem_st_wait();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();

  // issue_mode 0: thread 0; 1: warp 0; k >= 2: warps [0, k) each issue accumulators a = w (mod k)
  const int nissue = issue_mode >= 100 ? issue_mode - 100 : issue_mode;
  const bool issuer = issue_mode == 0 ? (t == 0) : issue_mode == 1 ? (warp == 0) : (warp < nissue);
  if (issuer) {
    const uint32_t idesc = make_idesc_f16(128, N, 0, 0, b_mode == 2 ? 1 : 0);
    uint64_t adesc[4], bdesc[4];
    for (int s = 0; s < 4; ++s) {
      adesc[s] = make_sdesc(smem_u32(sA) + s * 32, 16, 1024, kLayoutSW128);
      if (b_mode == 0) bdesc[s] = make_sdesc(smem_u32(sB) + s * 32, 16, 1024, kLayoutSW128);
      else if (b_mode == 1) bdesc[s] = make_sdesc(smem_u32(sB) + s * N * 32, 128, 256, kLayoutNone);
      else bdesc[s] = make_sdesc(smem_u32(sB) + s * 2048, 8192, 1024, kLayoutSW128);
    }
    // issue_mode 2: warp w issues accumulators a = w, w+4, ... (n_acc % 4 == 0)
    const int a0 = issue_mode >= 2 ? warp : 0, astep = issue_mode >= 2 ? issue_mode : 1;
    long long t0 = clock64();
    if (issue_mode >= 100) {
      const int a = warp % n_acc;
      for (int it = 0; it < iters; ++it)
#pragma unroll
        for (int s = 0; s < 4; ++s) mma_ts_warp(tbase + a * N, tbase + a_col + s * 8, bdesc[s], idesc, 1u);
      mma_commit_warp(&bar);
    } else if (issue_mode == 0) {
      if (a_mode != 0) {
        for (int it = 0; it < iters; ++it)
#pragma unroll
          for (int s = 0; s < 4; ++s)
            for (int a = 0; a < n_acc; ++a)
              mma_ts(tbase + a * N, tbase + a_col + s * 8, bdesc[s], idesc, (it | s) != 0);
      } else {
        for (int it = 0; it < iters; ++it)
#pragma unroll
          for (int s = 0; s < 4; ++s)
            for (int a = 0; a < n_acc; ++a)
              mma_ss(tbase + a * N, adesc[s], bdesc[s], idesc, (it | s) != 0);
      }
      mma_commit(&bar);
    } else {
      if (a_mode != 0) {
        for (int it = 0; it < iters; ++it)
#pragma unroll
          for (int s = 0; s < 4; ++s)
            for (int a = a0; a < n_acc; a += astep)
              mma_ts_warp(tbase + a * N, tbase + a_col + s * 8, bdesc[s], idesc, (it | s) != 0);
      } else {
        for (int it = 0; it < iters; ++it)
#pragma unroll
          for (int s = 0; s < 4; ++s)
            for (int a = a0; a < n_acc; a += astep)
              mma_ss_warp(tbase + a * N, adesc[s], bdesc[s], idesc, (it | s) != 0);
      }
      mma_commit_warp(&bar);
    }
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    if (t == 0) cycles[blockIdx.x] = t1 - t0;
  }
  __syncwarp();
  mbar_wait(&bar, 0);
  tc_fence_after();

  // read D back: warp w owns lanes [32w, 32w+32)
  if (blockIdx.x == 0 && warp < 4) {
    for (int j = 0; j < N * n_acc; j += 16) {
      uint32_t r[16];
      tmem_ld16(tbase + ((uint32_t)(warp * 32) << 16) + j, r);
      tmem_ld_wait();
      for (int i = 0; i < 16; ++i) D[t * N * n_acc + j + i] = __uint_as_float(r[i]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512>(tbase);
}

}  // namespace et

extern "C" int et_diag_mma_probe(const void* A, const void* B, float* D, int N, int a_mode, int b_mode,
                                 int iters, int n_acc, int issue_mode, long long* cycles, int grid, void* stream) {
  if (N < 16 || N > 256 || N % 16) return 1;
  if (n_acc < 1 || N * n_acc > (a_mode != 0 ? 448 : 512)) return 1;
  if (b_mode == 2 && N % 64) return 1;
  if (b_mode == 2 && N > 128) return 1;
  if (issue_mode >= 2 && issue_mode < 100 && (n_acc % issue_mode || issue_mode > 16)) return 1;
  if (issue_mode >= 100 && (issue_mode - 100 > 16 || (issue_mode - 100) % n_acc)) return 1;
  const size_t smem = 16384 + 32768 + 1024;
  cudaFuncSetAttribute(et::mma_probe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  et::mma_probe_kernel<<<grid, 512, smem, (cudaStream_t)stream>>>(
      (const __half*)A, (const __half*)B, D, N, a_mode, b_mode, iters, n_acc, issue_mode, cycles);
  return cudaGetLastError() == cudaSuccess ? 0 : 4;
}
