// M1b diagnostic (round 2): can ONE warp keep the tensor pipe busy with N=16 TS MMAs when the MMAs
// go to many independent accumulators (K-outer issue order), and how fast does the activation block
// reach TMEM (tcgen05.cp from a SWIZZLE_128B shared-memory chunk vs registers + tcgen05.st)?
//
//   mode 0: issue throughput.  `nw` warps; warp w issues n_mma MMAs (M=128, N=16, K=16, A in TMEM)
//           round-robin over its accumulators a = w, w + nw, ... < n_acc, four MMAs (four different
//           accumulators) per elect.  One commit per warp at the end.
//   mode 1: tcgen05.cp throughput: n_chunks x (4 x 128x256b) of the same 16 KB SW128 chunk into a
//           ring of 4 TMEM slots (32 columns each), one commit at the end.
//   mode 2: streaming (the K-outer GEMM pattern): one warp, per chunk c: 4 cps into slot c % 4,
//           then mpc MMAs into distinct accumulators reading that slot (tile column s = u % 4).
//   mode 3: register-path fill: 4 warps move n_chunks chunks smem -> registers -> tcgen05.st.
// Cycles: clock64 on thread 0 between a CTA barrier before the work and the completion of the
// last commit; grid = one CTA per SM.
#include <cuda_runtime.h>
#include <cstdint>
#include "ptx.cuh"

namespace et {

__device__ __forceinline__ void mma_ts_warp_x4d(uint32_t d0, uint32_t d1, uint32_t d2, uint32_t d3, uint32_t a0,
                                                uint32_t a1, uint32_t a2, uint32_t a3, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n .reg .pred e;\n .reg .b32 rx;\n"
      " elect.sync rx|e, 0xffffffff;\n"
      " @e tcgen05.mma.cta_group::1.kind::f16 [%0], [%4], %8, %9, 1;\n"
      " @e tcgen05.mma.cta_group::1.kind::f16 [%1], [%5], %8, %9, 1;\n"
      " @e tcgen05.mma.cta_group::1.kind::f16 [%2], [%6], %8, %9, 1;\n"
      " @e tcgen05.mma.cta_group::1.kind::f16 [%3], [%7], %8, %9, 1;\n}\n" ::"r"(d0),
      "r"(d1), "r"(d2), "r"(d3), "r"(a0), "r"(a1), "r"(a2), "r"(a3), "l"(b), "r"(idesc));
}
__device__ __forceinline__ void tmem_cp4_warp(uint32_t t, uint64_t s0, uint64_t s1, uint64_t s2, uint64_t s3) {
  asm volatile(
      "{\n .reg .pred e;\n .reg .b32 rx;\n"
      " elect.sync rx|e, 0xffffffff;\n"
      " @e tcgen05.cp.cta_group::1.128x256b [%0], %1;\n"
      " @e tcgen05.cp.cta_group::1.128x256b [%2], %3;\n"
      " @e tcgen05.cp.cta_group::1.128x256b [%4], %5;\n"
      " @e tcgen05.cp.cta_group::1.128x256b [%6], %7;\n}\n" ::"r"(t),
      "l"(s0), "r"(t + 8), "l"(s1), "r"(t + 16), "l"(s2), "r"(t + 24), "l"(s3)
      : "memory");
}

__global__ void __launch_bounds__(512, 1)
mma_probe2_kernel(const __half* __restrict__ A, const __half* __restrict__ B, float* __restrict__ D, int mode, int nw,
                  int n_acc, int n_mma, int n_chunks, int mpc, long long* __restrict__ cycles) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;            // 16 KB: A chunk, 128 rows x 64 K, SW128
  uint8_t* sB = smem + 16384;    // one 16x16 tile, core-matrix no-swizzle (512 B)
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem_base_s;
  const int t = threadIdx.x, warp = t >> 5;
  if (t < 128) {
    const uint4* src = reinterpret_cast<const uint4*>(A + t * 64);
    for (int c = 0; c < 8; ++c) *reinterpret_cast<uint4*>(sA + t * 128 + ((c ^ (t & 7)) << 4)) = src[c];
  }
  if (t < 16) {   // B tile [16 n][16 k]: element (n, k) at (n/8)*256 + (k/8)*128 + (n%8)*16 + (k%8)*2
    for (int k8 = 0; k8 < 2; ++k8)
      *reinterpret_cast<uint4*>(sB + (t >> 3) * 256 + k8 * 128 + (t & 7) * 16) =
          *reinterpret_cast<const uint4*>(B + t * 16 + k8 * 8);
  }
  fence_proxy_async_smem();
  if (warp == 0) tmem_alloc<512>(&tmem_base_s);
  if (t == 0) {
    mbar_init(&bar, (mode == 0 || mode >= 4) ? nw : (mode == 3 ? 4 : 1));
    fence_mbar_init();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tmem_base_s;
  constexpr uint32_t kAslot = 384;   // A ring: 4 slots x 32 columns at [384, 512)
  // zero the accumulators (lanes of warps 0-3)
  if (warp < 4) {
    uint32_t zr[16];
    for (int i = 0; i < 16; ++i) zr[i] = 0u;
    for (int c = 0; c < 384; c += 16) tmem_st16(tb + ((uint32_t)(warp * 32) << 16) + c, zr);
    // modes 0, 4, 5: A at slot 0 via registers (rows of sA, unswizzled)
    if (mode == 0 || mode >= 4) {
      uint32_t r[32];
      const int rr = warp * 32 + (t & 31);
      for (int c = 0; c < 8; ++c) {
        const uint4 u = *reinterpret_cast<const uint4*>(sA + rr * 128 + ((c ^ (rr & 7)) << 4));
        r[4 * c] = u.x; r[4 * c + 1] = u.y; r[4 * c + 2] = u.z; r[4 * c + 3] = u.w;
      }
      tmem_st32(tb + ((uint32_t)(warp * 32) << 16) + kAslot, r);
    }
    tmem_st_wait();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t idesc = make_idesc_f16(128, 16, 0, 0, 0);
  const uint64_t bdesc = make_sdesc(smem_u32(sB), 128, 256, kLayoutNone);
  long long t0 = clock64();
  if (mode == 0) {
    if (warp < nw) {
      // accumulators of this warp: w, w + nw, ... ; MMA u goes to the (u % na)-th of them
      const int na = (n_acc - warp + nw - 1) / nw;
      int u = 0;
      int ai = 0;
      for (; u + 4 <= n_mma; u += 4) {
        uint32_t d[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          d[i] = tb + (uint32_t)((warp + nw * ai) * 16);
          ai = ai + 1 == na ? 0 : ai + 1;
        }
        mma_ts_warp_x4d(d[0], d[1], d[2], d[3], tb + kAslot, tb + kAslot + 8, tb + kAslot + 16, tb + kAslot + 24,
                        bdesc, idesc);
      }
      mma_commit_warp(&bar);
    }
  } else if (mode == 1) {
    if (warp == 0) {
      for (int c = 0; c < n_chunks; ++c) {
        const uint32_t slot = tb + kAslot + (uint32_t)((c & 3) * 32);
        tmem_cp4_warp(slot, make_sdesc(smem_u32(sA), 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 32, 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 64, 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 96, 16, 1024, kLayoutSW128));
      }
      mma_commit_warp(&bar);
    }
  } else if (mode == 2) {
    if (warp == 0) {
      int ai = 0;
      for (int c = 0; c < n_chunks; ++c) {
        const uint32_t slot = tb + kAslot + (uint32_t)((c & 3) * 32);
        tmem_cp4_warp(slot, make_sdesc(smem_u32(sA), 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 32, 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 64, 16, 1024, kLayoutSW128),
                      make_sdesc(smem_u32(sA) + 96, 16, 1024, kLayoutSW128));
        for (int u = 0; u + 4 <= mpc; u += 4) {
          uint32_t d[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            d[i] = tb + (uint32_t)(ai * 16);
            ai = ai + 1 == n_acc ? 0 : ai + 1;
          }
          mma_ts_warp_x4d(d[0], d[1], d[2], d[3], slot, slot + 8, slot + 16, slot + 24, bdesc, idesc);
        }
      }
      mma_commit_warp(&bar);
    }
  } else if (mode == 4 || mode == 5) {
    // the tile GEMM's issue pattern: per-warp lists of (D, A, B lo, accumulate) in shared memory,
    // broadcast LDS.128 + four MMAs per elect (mode 4), or the same values kept in registers and
    // broadcast with shuffles (mode 5); nw warps, n_mma MMAs each, distinct B tiles per MMA
    __shared__ uint4 lst[16][32];
    if (warp < nw) {
      const uint32_t bhi = (uint32_t)(bdesc >> 32), blo = (uint32_t)bdesc;
      const int na = (n_acc - warp + nw - 1) / nw;
      uint4 mine;
      {
        const int ai = (t & 31) % na;
        mine = make_uint4(tb + (uint32_t)((warp + nw * ai) * 16), tb + kAslot + (uint32_t)(((t & 31) & 3) * 8), blo, 1u);
      }
      lst[warp][t & 31] = mine;
      __syncwarp();
      for (int u0 = 0; u0 < n_mma; u0 += 32) {
        if (mode == 4) {
          for (int u = 0; u + 4 <= 32 && u0 + u + 4 <= n_mma; u += 4) {
            const uint4* l = lst[warp];
            asm volatile(
                "{\n .reg .pred e, p0, p1, p2, p3;\n .reg .b32 rx;\n .reg .b64 q0, q1, q2, q3;\n"
                " elect.sync rx|e, 0xffffffff;\n"
                " setp.ne.b32 p0, %12, 0;\n setp.ne.b32 p1, %13, 0;\n setp.ne.b32 p2, %14, 0;\n setp.ne.b32 p3, %15, 0;\n"
                " mov.b64 q0, {%8, %16};\n mov.b64 q1, {%9, %16};\n mov.b64 q2, {%10, %16};\n mov.b64 q3, {%11, %16};\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%0], [%4], q0, %17, p0;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%1], [%5], q1, %17, p1;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%2], [%6], q2, %17, p2;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%3], [%7], q3, %17, p3;\n}\n" ::"r"(l[u].x),
                "r"(l[u + 1].x), "r"(l[u + 2].x), "r"(l[u + 3].x), "r"(l[u].y), "r"(l[u + 1].y), "r"(l[u + 2].y),
                "r"(l[u + 3].y), "r"(l[u].z), "r"(l[u + 1].z), "r"(l[u + 2].z), "r"(l[u + 3].z), "r"(l[u].w),
                "r"(l[u + 1].w), "r"(l[u + 2].w), "r"(l[u + 3].w), "r"(bhi), "r"(idesc));
          }
        } else {
          for (int u = 0; u + 4 <= 32 && u0 + u + 4 <= n_mma; u += 4) {
            uint32_t d[4], a[4], b[4], f[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              d[i] = __shfl_sync(0xffffffffu, mine.x, u + i);
              a[i] = __shfl_sync(0xffffffffu, mine.y, u + i);
              b[i] = __shfl_sync(0xffffffffu, mine.z, u + i);
              f[i] = __shfl_sync(0xffffffffu, mine.w, u + i);
            }
            asm volatile(
                "{\n .reg .pred e, p0, p1, p2, p3;\n .reg .b32 rx;\n .reg .b64 q0, q1, q2, q3;\n"
                " elect.sync rx|e, 0xffffffff;\n"
                " setp.ne.b32 p0, %12, 0;\n setp.ne.b32 p1, %13, 0;\n setp.ne.b32 p2, %14, 0;\n setp.ne.b32 p3, %15, 0;\n"
                " mov.b64 q0, {%8, %16};\n mov.b64 q1, {%9, %16};\n mov.b64 q2, {%10, %16};\n mov.b64 q3, {%11, %16};\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%0], [%4], q0, %17, p0;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%1], [%5], q1, %17, p1;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%2], [%6], q2, %17, p2;\n"
                " @e tcgen05.mma.cta_group::1.kind::f16 [%3], [%7], q3, %17, p3;\n}\n" ::"r"(d[0]),
                "r"(d[1]), "r"(d[2]), "r"(d[3]), "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]),
                "r"(b[2]), "r"(b[3]), "r"(f[0]), "r"(f[1]), "r"(f[2]), "r"(f[3]), "r"(bhi), "r"(idesc));
          }
        }
      }
      mma_commit_warp(&bar);
    }
  } else if (mode == 3) {
    if (warp < 4) {
      const int rr = warp * 32 + (t & 31);
      for (int c = 0; c < n_chunks; ++c) {
        uint32_t r[32];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const uint4 u = *reinterpret_cast<const uint4*>(sA + rr * 128 + ((q ^ (rr & 7)) << 4));
          r[4 * q] = u.x; r[4 * q + 1] = u.y; r[4 * q + 2] = u.z; r[4 * q + 3] = u.w;
        }
        tmem_st32(tb + ((uint32_t)(warp * 32) << 16) + kAslot + (uint32_t)((c & 3) * 32), r);
      }
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if ((t & 31) == 0) mbar_arrive(&bar);
    }
  }
  mbar_wait(&bar, 0);
  long long t1 = clock64();
  if (t == 0) cycles[blockIdx.x] = t1 - t0;
  tc_fence_after();
  // read back: accumulators [0, 384) (modes 0, 2) or the A ring (modes 1, 3), CTA 0 only
  if (blockIdx.x == 0 && warp < 4) {
    for (int j = 0; j < 512; j += 16) {
      uint32_t r[16];
      tmem_ld16(tb + ((uint32_t)(warp * 32) << 16) + j, r);
      tmem_ld_wait();
      for (int i = 0; i < 16; ++i) D[t * 512 + j + i] = __uint_as_float(r[i]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512>(tb);
}

}  // namespace et

extern "C" int et_diag_mma_probe2(const void* A, const void* B, float* D, int mode, int nw, int n_acc, int n_mma,
                                  int n_chunks, int mpc, long long* cycles, int grid, void* stream) {
  if (n_acc < 1 || n_acc > 24 || nw < 1 || nw > 16 || ((mode == 0 || mode >= 4) && n_mma % 4) || (mode == 2 && mpc % 4)) return 1;
  const size_t smem = 16384 + 512 + 1024;
  cudaFuncSetAttribute(et::mma_probe2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  et::mma_probe2_kernel<<<grid, 512, smem, (cudaStream_t)stream>>>((const __half*)A, (const __half*)B, D, mode, nw,
                                                                  n_acc, n_mma, n_chunks, mpc, cycles);
  return cudaGetLastError() == cudaSuccess ? 0 : 4;
}
