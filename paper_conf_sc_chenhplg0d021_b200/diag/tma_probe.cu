// Diagnostic (not part of the metric): how fast can 128 CTAs pull the activation block of the tile
// GEMM (128 rows x 768 K fp16 = 192 KB per CTA, 4 CTAs per token block) out of L2?
//   mode 0: every CTA loads its block itself (unicast, the shipped GEMM);
//   mode 1: clusters of 4 CTAs (the 4 pieces of one token block): CTA r loads chunks j = r (mod 4)
//           and multicasts each to all 4 (TMA .multicast::cluster);
//   mode 2: unicast, but every CTA reads a distinct block (no sharing at all).
// Result: device time per launch (host events), written by the caller's timing loop.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "internal.h"
#include "ptx.cuh"

namespace et {
et_status make_tmap_2d(CUtensorMap* tm, const void* base, et_dtype dtype, uint64_t rows, uint64_t cols,
                       uint64_t ld_elems, uint32_t box_cols, uint32_t box_rows, bool swizzle128);
namespace {

__device__ __forceinline__ void tma_load_2d_mc(void* smem_dst, const void* tmap, uint64_t* bar, int32_t c0, int32_t c1,
                                               uint16_t mask) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%2, "
      "%3}], [%4], %5;" ::"r"(smem_u32(smem_dst)),
      "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "h"(mask)
      : "memory");
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

template <int kMode>
__global__ void __launch_bounds__(128, 1) tma_probe_kernel(const __grid_constant__ CUtensorMap tm, int nchunks,
                                                           unsigned long long* out_cycles) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ uint64_t full;
  const int mblk = kMode == 2 ? blockIdx.x : blockIdx.x / 4;
  if (threadIdx.x == 0) {
    mbar_init(&full, 1);
    fence_mbar_init();
  }
  if constexpr (kMode == 1) cluster_sync(); else __syncthreads();
  const long long t0 = clock64();
  if (threadIdx.x == 0) {
    mbar_expect_tx(&full, (uint32_t)nchunks * 16384u);
    if constexpr (kMode == 1) {
      const int r = (int)cluster_rank();
      for (int j = r; j < nchunks; j += 4) tma_load_2d_mc(smem + j * 16384, &tm, &full, j * 64, mblk * 128, 0xF);
    } else {
      for (int j = 0; j < nchunks; ++j) tma_load_2d(smem + j * 16384, &tm, &full, j * 64, mblk * 128);
    }
    mbar_wait(&full, 0);
    out_cycles[blockIdx.x] = (unsigned long long)(clock64() - t0);
  }
  if constexpr (kMode == 1) cluster_sync();   // no CTA exits while a peer may still multicast into it
}

}  // namespace
}  // namespace et

using namespace et;

extern "C" int et_diag_tma_probe(const void* src, int rows, int cols, int mode, int grid, int nchunks,
                                 unsigned long long* out_cycles, void* stream) {
  CUtensorMap tm;
  if (make_tmap_2d(&tm, src, ET_FP16, (uint64_t)rows, (uint64_t)cols, (uint64_t)cols, 64, 128, true) != ET_OK) return 1;
  const size_t smem = 1024 + (size_t)nchunks * 16384;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(128);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 4;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = mode == 1 ? 1 : 0;
  cudaError_t e;
  if (mode == 0) {
    cudaFuncSetAttribute(tma_probe_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    e = cudaLaunchKernelEx(&cfg, tma_probe_kernel<0>, tm, nchunks, out_cycles);
  } else if (mode == 1) {
    cudaFuncSetAttribute(tma_probe_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    e = cudaLaunchKernelEx(&cfg, tma_probe_kernel<1>, tm, nchunks, out_cycles);
  } else {
    cudaFuncSetAttribute(tma_probe_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    e = cudaLaunchKernelEx(&cfg, tma_probe_kernel<2>, tm, nchunks, out_cycles);
  }
  return e == cudaSuccess ? 0 : 2;
}
