// Column pruning with X_adjusted (§4.1, Fig. 5(b)): after column
// pruning only the kept input features of X meet nonzero weights, so the pruned linear layer is the
// dense product X_adjusted . W_pruned^T with X_adjusted = X[:, keep] and W_pruned = W[:, keep] (the
// condensed weight).  This kernel is the gather for both: Out[r, j] = In[r, idx[j]] for j < nk and
// 0 for nk <= j < nk_pad (zero padding to the tile GEMM's K granule; exact: padded columns meet
// padded zeros).  One 16-byte output vector per thread (8 x 16-bit or 4 x FP32 elements), rows
// contiguous so the stores coalesce; the gathered reads of a row hit the same few L2 lines.
#include <cuda_runtime.h>
#include <cstdint>

#include "../internal.h"

namespace et {
namespace {

template <typename T>
__global__ void gather_cols_kernel(const T* __restrict__ in, int rows, int ld_in, const int32_t* __restrict__ idx,
                                   int nk, int nk_pad, T* __restrict__ out) {
  constexpr int V = 16 / sizeof(T);
  const int vpr = nk_pad / V;   // vectors per output row
  const long long g = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= (long long)rows * vpr) return;
  const int r = (int)(g / vpr), j0 = (int)(g % vpr) * V;
  const T* src = in + (size_t)r * ld_in;
  union {
    uint4 u;
    T e[V];
  } pk;
#pragma unroll
  for (int v = 0; v < V; ++v) {
    const int j = j0 + v;
    pk.e[v] = j < nk ? src[__ldg(idx + j)] : T(0);
  }
  *reinterpret_cast<uint4*>(out + (size_t)r * nk_pad + j0) = pk.u;
}

}  // namespace

et_status gather_cols_run(const void* in, int rows, int ld_in, const int32_t* idx, int nk, int nk_pad, et_dtype dt,
                          void* out, cudaStream_t stream) {
  if (rows == 0 || nk_pad == 0) return ET_OK;
  const int V = dt == ET_FP32 ? 4 : 8;
  const long long n = (long long)rows * (nk_pad / V);
  const int threads = 256;
  const unsigned blocks = (unsigned)((n + threads - 1) / threads);
  if (dt == ET_FP32)
    gather_cols_kernel<float><<<blocks, threads, 0, stream>>>(static_cast<const float*>(in), rows, ld_in, idx, nk,
                                                              nk_pad, static_cast<float*>(out));
  else   // FP16 / BF16: moved as raw 16-bit patterns (bit-exact gather)
    gather_cols_kernel<uint16_t><<<blocks, threads, 0, stream>>>(static_cast<const uint16_t*>(in), rows, ld_in, idx,
                                                                 nk, nk_pad, static_cast<uint16_t*>(out));
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

}  // namespace et
