// Tensor-tile / row / column pruning and packing on the GPU (§4.2 step (v) 1-4;
// line 169-171, §4.1).  Offline, once per weight; bit-exact contract with the oracle:
//   score(unit) = sum of w^2 in FP64, fixed order (tile: a outer, b inner; row: over columns;
//   col: over rows), each add rounded (__dadd_rn of an exact square) — reading C-2;
//   rank by (score ascending, linear index ascending); the first n_prune are pruned.
// Ranking counts, for every unit, how many units precede it in that total order (no sort, so
// the result cannot depend on a sort's stability).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cstdint>

#include "../internal.h"

namespace et {
namespace {

template <typename T>
__device__ __forceinline__ double to_f64(T v);
template <>
__device__ __forceinline__ double to_f64<__half>(__half v) { return (double)__half2float(v); }
template <>
__device__ __forceinline__ double to_f64<__nv_bfloat16>(__nv_bfloat16 v) { return (double)__bfloat162float(v); }
template <>
__device__ __forceinline__ double to_f64<float>(float v) { return (double)v; }

// one thread per unit: TILE t = i*q + j; ROW t = row; COL t = col
template <typename T>
__global__ void scores_kernel(const T* __restrict__ W, int rows, int cols, int pattern, int r, int c,
                              int units, double* __restrict__ scores) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= units) return;
  double s = 0.0;
  if (pattern == ET_PRUNE_TILE) {
    const int q = cols / c;
    const int i = t / q, j = t % q;
    for (int a = 0; a < r; ++a) {
      const T* rowp = W + (size_t)(i * r + a) * cols + (size_t)j * c;
      for (int b = 0; b < c; ++b) {
        const double w = to_f64(rowp[b]);
        s = __dadd_rn(s, __dmul_rn(w, w));
      }
    }
  } else if (pattern == ET_PRUNE_ROW) {
    const T* rowp = W + (size_t)t * cols;
    for (int j = 0; j < cols; ++j) {
      const double w = to_f64(rowp[j]);
      s = __dadd_rn(s, __dmul_rn(w, w));
    }
  } else {  // COL
    for (int i = 0; i < rows; ++i) {
      const double w = to_f64(W[(size_t)i * cols + t]);
      s = __dadd_rn(s, __dmul_rn(w, w));
    }
  }
  scores[t] = s;
}

// keep[t] = rank(t) >= n_prune, rank = #{u : (s_u, u) < (s_t, t)}
__global__ void rank_kernel(const double* __restrict__ scores, int units, int n_prune,
                            const uint32_t* __restrict__ mask_in, uint8_t* __restrict__ keep) {
  constexpr int CH = 2048;
  __shared__ double sc[CH];
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (mask_in != nullptr) {
    if (t < units) keep[t] = (mask_in[t >> 5] >> (t & 31)) & 1u;
    return;
  }
  const double my = t < units ? scores[t] : 0.0;
  int cnt = 0;
  for (int base = 0; base < units; base += CH) {
    const int n = min(CH, units - base);
    __syncthreads();
    for (int u = threadIdx.x; u < n; u += blockDim.x) sc[u] = scores[base + u];
    __syncthreads();
    if (t < units) {
      for (int u = 0; u < n; ++u) {
        const double su = sc[u];
        cnt += (su < my) || (su == my && base + u < t);
      }
    }
  }
  if (t < units) keep[t] = cnt >= n_prune ? 1 : 0;
}

__global__ void bitmap_kernel(const uint8_t* __restrict__ keep, int units, uint32_t* __restrict__ mask) {
  const int w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w >= (units + 31) / 32) return;
  uint32_t v = 0;
  for (int b = 0; b < 32; ++b) {
    const int t = w * 32 + b;
    if (t < units && keep[t]) v |= 1u << b;
  }
  mask[w] = v;
}

// Sequential bookkeeping for the index structures (tiny: <= a few thousand entries).
// TILE: CSR row_ptr / col_idx (the bit-exact contract) plus the values order used by the GEMM:
// K-part-major (part z = tile columns [48z, 48z+48)), then tile row, then column, with
// part_row_ptr[z][i] and tile_col in that order.  ROW: kept indices, per-group padding, row_map
// and the dense tile grid of the packed [rows_padded, cols] matrix in the same part-major order.
// COL: kept indices only.  counts[0] = nnz, counts[1] = rows_padded, counts[2] = ntiles.
__global__ void index_kernel(const uint8_t* __restrict__ keep, int rows, int cols, int pattern, int r, int c,
                             int group_rows, int32_t* __restrict__ idx, int32_t* __restrict__ row_ptr,
                             int32_t* __restrict__ tile_col, int32_t* __restrict__ row_map,
                             int32_t* __restrict__ part_row_ptr, int32_t* __restrict__ counts) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  constexpr int kPartTiles = 48;
  if (pattern == ET_PRUNE_TILE) {
    const int p = rows / r, q = cols / c;
    int pos = 0;
    for (int i = 0; i < p; ++i) {
      if (row_ptr) row_ptr[i] = pos;
      for (int j = 0; j < q; ++j) {
        if (keep[i * q + j]) {
          if (idx) idx[pos] = j;
          ++pos;
        }
      }
    }
    if (row_ptr) row_ptr[p] = pos;
    const int kparts = (q + kPartTiles - 1) / kPartTiles;
    int vpos = 0;
    for (int z = 0; z < kparts; ++z) {
      for (int i = 0; i < p; ++i) {
        if (part_row_ptr) part_row_ptr[z * (p + 1) + i] = vpos;
        for (int j = z * kPartTiles; j < min(q, (z + 1) * kPartTiles); ++j)
          if (keep[i * q + j]) {
            if (tile_col) tile_col[vpos] = j;
            ++vpos;
          }
      }
      if (part_row_ptr) part_row_ptr[z * (p + 1) + p] = vpos;
    }
    counts[0] = pos;
    counts[1] = rows;
    counts[2] = pos;
  } else if (pattern == ET_PRUNE_ROW) {
    const int gr = group_rows > 0 ? group_rows : rows;
    const int G = rows / gr;
    int nnz = 0, pr = 0;
    for (int g = 0; g < G; ++g) {
      int cnt = 0;
      for (int i = g * gr; i < (g + 1) * gr; ++i) {
        if (keep[i]) {
          if (idx) idx[nnz] = i;
          if (row_map) row_map[pr + cnt] = i;
          ++nnz;
          ++cnt;
        }
      }
      const int pad = (cnt + 15) / 16 * 16;
      for (int k = cnt; k < pad; ++k)
        if (row_map) row_map[pr + k] = -1;
      pr += pad;
    }
    const int q = cols / 16;
    const int tr = pr / 16;
    if (row_ptr)
      for (int i = 0; i <= tr; ++i) row_ptr[i] = i * q;
    const int kparts = (q + kPartTiles - 1) / kPartTiles;
    int vpos = 0;
    for (int z = 0; z < kparts; ++z) {
      for (int i = 0; i < tr; ++i) {
        if (part_row_ptr) part_row_ptr[z * (tr + 1) + i] = vpos;
        for (int j = z * kPartTiles; j < min(q, (z + 1) * kPartTiles); ++j) {
          if (tile_col) tile_col[vpos] = j;
          ++vpos;
        }
      }
      if (part_row_ptr) part_row_ptr[z * (tr + 1) + tr] = vpos;
    }
    counts[0] = nnz;
    counts[1] = pr;
    counts[2] = tr * q;
  } else {  // COL
    int nnz = 0;
    for (int j = 0; j < cols; ++j)
      if (keep[j]) {
        if (idx) idx[nnz] = j;
        ++nnz;
      }
    counts[0] = nnz;
    counts[1] = rows;
    counts[2] = 0;
  }
}

// packed position -> tile row, by searching the part-major part_row_ptr
__device__ __forceinline__ int tile_row_of(const int32_t* __restrict__ prp, int tile_rows, int kparts, int pos) {
  int z = 0;
  while (z + 1 < kparts && prp[(z + 1) * (tile_rows + 1)] <= pos) ++z;
  const int32_t* rp = prp + z * (tile_rows + 1);
  int lo = 0, hi = tile_rows;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (rp[mid] <= pos) lo = mid;
    else hi = mid;
  }
  return lo;
}

// Copy one 16x16 tile per warp into the tcgen05 K-major no-swizzle core-matrix layout:
// element (n, k) at byte (n/8)*256 + (k/8)*128 + (n%8)*16 + (k%8)*2.  Lane l moves row n = l/2,
// k-half kh = l%2 (16 bytes).  TILE: packed tile p = (i, col_idx[p]) with i from row_ptr.
// ROW: packed tile p = (i, j) of the dense [rows_padded, cols] matrix, rows via row_map.
__global__ void pack_values_kernel(const uint16_t* __restrict__ W, int cols, int pattern,
                                   const int32_t* __restrict__ part_row_ptr, const int32_t* __restrict__ tile_col,
                                   const int32_t* __restrict__ row_map, const int32_t* __restrict__ counts,
                                   int kparts, uint8_t* __restrict__ values, int rows) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int ntiles = counts[2];
  if (warp >= ntiles) return;
  const int tile_rows = pattern == ET_PRUNE_TILE ? rows / 16 : counts[1] / 16;
  const int i = tile_row_of(part_row_ptr, tile_rows, kparts, warp);
  const int j = tile_col[warp];
  const int n = lane >> 1, kh = lane & 1;
  const int src_row = pattern == ET_PRUNE_TILE ? i * 16 + n : row_map[i * 16 + n];
  uint4 v = make_uint4(0, 0, 0, 0);
  if (src_row >= 0) v = *reinterpret_cast<const uint4*>(W + (size_t)src_row * cols + j * 16 + kh * 8);
  *reinterpret_cast<uint4*>(values + (size_t)warp * 512 + (n >> 3) * 256 + kh * 128 + (n & 7) * 16) = v;
}

// FP32 validation build: the same tile order, each tile row-major (element (n, k) at byte
// n*64 + k*4, 1 KB).  Lane l moves row n = l/2, half kh = l%2 (8 floats).
__global__ void pack_values32_kernel(const float* __restrict__ W, int cols, int pattern,
                                     const int32_t* __restrict__ part_row_ptr, const int32_t* __restrict__ tile_col,
                                     const int32_t* __restrict__ row_map, const int32_t* __restrict__ counts,
                                     int kparts, float* __restrict__ values, int rows) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int ntiles = counts[2];
  if (warp >= ntiles) return;
  const int tile_rows = pattern == ET_PRUNE_TILE ? rows / 16 : counts[1] / 16;
  const int i = tile_row_of(part_row_ptr, tile_rows, kparts, warp);
  const int j = tile_col[warp];
  const int n = lane >> 1, kh = lane & 1;
  const int src_row = pattern == ET_PRUNE_TILE ? i * 16 + n : row_map[i * 16 + n];
  float4 a = make_float4(0.f, 0.f, 0.f, 0.f), b = a;
  if (src_row >= 0) {
    const float4* s = reinterpret_cast<const float4*>(W + (size_t)src_row * cols + j * 16 + kh * 8);
    a = s[0];
    b = s[1];
  }
  float4* d = reinterpret_cast<float4*>(values + (size_t)warp * 256 + n * 16 + kh * 8);
  d[0] = a;
  d[1] = b;
}

__global__ void unpack32_kernel(const float* __restrict__ values, int cols, int pattern,
                                const int32_t* __restrict__ part_row_ptr, const int32_t* __restrict__ tile_col,
                                const int32_t* __restrict__ row_map, int ntiles, int tile_rows, int kparts,
                                float* __restrict__ dense) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (warp >= ntiles) return;
  const int i = tile_row_of(part_row_ptr, tile_rows, kparts, warp);
  const int j = tile_col[warp];
  const int n = lane >> 1, kh = lane & 1;
  const int dst_row = pattern == ET_PRUNE_TILE ? i * 16 + n : row_map[i * 16 + n];
  if (dst_row < 0) return;
  const float4* s = reinterpret_cast<const float4*>(values + (size_t)warp * 256 + n * 16 + kh * 8);
  float4* d = reinterpret_cast<float4*>(dense + (size_t)dst_row * cols + j * 16 + kh * 8);
  d[0] = s[0];
  d[1] = s[1];
}

// Inverse of pack_values_kernel: dense [rows, cols] = 0 except kept tiles / rows.
__global__ void unpack_kernel(const uint8_t* __restrict__ values, int cols, int pattern,
                              const int32_t* __restrict__ part_row_ptr, const int32_t* __restrict__ tile_col,
                              const int32_t* __restrict__ row_map, int ntiles, int tile_rows, int kparts,
                              uint16_t* __restrict__ dense) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (warp >= ntiles) return;
  const int i = tile_row_of(part_row_ptr, tile_rows, kparts, warp);
  const int j = tile_col[warp];
  const int n = lane >> 1, kh = lane & 1;
  const int dst_row = pattern == ET_PRUNE_TILE ? i * 16 + n : row_map[i * 16 + n];
  if (dst_row < 0) return;
  *reinterpret_cast<uint4*>(dense + (size_t)dst_row * cols + j * 16 + kh * 8) =
      *reinterpret_cast<const uint4*>(values + (size_t)warp * 512 + (n >> 3) * 256 + kh * 128 + (n & 7) * 16);
}

int units_of(int rows, int cols, et_pattern pattern, int r, int c) {
  if (pattern == ET_PRUNE_TILE) return (rows / r) * (cols / c);
  if (pattern == ET_PRUNE_ROW) return rows;
  return cols;
}

}  // namespace

size_t prune_workspace_bytes(int rows, int cols, et_pattern pattern, int tile_r, int tile_c) {
  const size_t units = (size_t)units_of(rows, cols, pattern, tile_r, tile_c);
  return align_up(units * sizeof(double), 256) + align_up(units, 256) + 256;
}

et_status prune_pack_run(const PruneArgs& a, et_packed_weight* out, void* ws, size_t ws_bytes, cudaStream_t stream) {
  const int units = units_of(a.rows, a.cols, a.pattern, a.tile_r, a.tile_c);
  if (ws_bytes < prune_workspace_bytes(a.rows, a.cols, a.pattern, a.tile_r, a.tile_c))
    return fail(ET_ERR_WORKSPACE, "et_prune_pack: workspace too small");
  uint8_t* base = static_cast<uint8_t*>(ws);
  double* scores = reinterpret_cast<double*>(base);
  uint8_t* keep = base + align_up((size_t)units * sizeof(double), 256);
  int32_t* counts = reinterpret_cast<int32_t*>(keep + align_up(units, 256));

  const int tb = 256;
  const int nb = (units + tb - 1) / tb;
  switch (a.dtype) {
    case ET_FP16:
      scores_kernel<__half><<<nb, tb, 0, stream>>>(static_cast<const __half*>(a.W), a.rows, a.cols, a.pattern,
                                                   a.tile_r, a.tile_c, units, scores);
  count_launch();
      break;
    case ET_BF16:
      scores_kernel<__nv_bfloat16><<<nb, tb, 0, stream>>>(static_cast<const __nv_bfloat16*>(a.W), a.rows, a.cols,
                                                          a.pattern, a.tile_r, a.tile_c, units, scores);
  count_launch();
      break;
    default:
      scores_kernel<float><<<nb, tb, 0, stream>>>(static_cast<const float*>(a.W), a.rows, a.cols, a.pattern,
                                                  a.tile_r, a.tile_c, units, scores);
  count_launch();
  }
  ET_CUDA(cudaGetLastError());
  rank_kernel<<<nb, tb, 0, stream>>>(scores, units, a.n_prune, a.mask_in, keep);
  count_launch();
  ET_CUDA(cudaGetLastError());
  if (out->mask) {
    const int words = (units + 31) / 32;
    bitmap_kernel<<<(words + 127) / 128, 128, 0, stream>>>(keep, units, out->mask);
  count_launch();
    ET_CUDA(cudaGetLastError());
  }
  index_kernel<<<1, 32, 0, stream>>>(keep, a.rows, a.cols, a.pattern, a.tile_r, a.tile_c, a.group_rows, out->idx,
                                     out->row_ptr, out->tile_col, out->row_map, out->part_row_ptr, counts);
  count_launch();
  ET_CUDA(cudaGetLastError());
  const bool pack_values = out->values != nullptr && a.tile_r == 16 && a.tile_c == 16 && a.pattern != ET_PRUNE_COL;
  const int kparts = (a.cols / 16 + 47) / 48;
  if (pack_values) {
    if (!out->tile_col || !out->part_row_ptr || (a.pattern == ET_PRUNE_ROW && !out->row_map))
      return fail(ET_ERR_INVALID_ARG, "et_prune_pack: values requested without tile_col/part_row_ptr/row_map");
    // upper bound of packed tiles for the grid; the kernel reads the exact count from counts[2]
    const int groups = a.pattern == ET_PRUNE_ROW ? (a.group_rows > 0 ? a.rows / a.group_rows : 1) : 1;
    const int max_tiles = a.pattern == ET_PRUNE_TILE ? units : ((a.rows + 15 * groups) / 16 + 1) * (a.cols / 16);
    const int threads = 256;
    const int blocks = (max_tiles * 32 + threads - 1) / threads;
    if (a.dtype == ET_FP32)
      pack_values32_kernel<<<blocks, threads, 0, stream>>>(static_cast<const float*>(a.W), a.cols, a.pattern,
                                                           out->part_row_ptr, out->tile_col, out->row_map, counts,
                                                           kparts, static_cast<float*>(out->values), a.rows);
    else
      pack_values_kernel<<<blocks, threads, 0, stream>>>(static_cast<const uint16_t*>(a.W), a.cols, a.pattern,
                                                         out->part_row_ptr, out->tile_col, out->row_map, counts,
                                                         kparts, static_cast<uint8_t*>(out->values), a.rows);
  count_launch();
    ET_CUDA(cudaGetLastError());
  }
  int32_t hc[3];
  ET_CUDA(cudaMemcpyAsync(hc, counts, sizeof(hc), cudaMemcpyDeviceToHost, stream));
  ET_CUDA(cudaStreamSynchronize(stream));
  out->nnz = hc[0];
  out->rows_padded = hc[1];
  out->ntiles = hc[2];
  out->kparts = kparts;
  return ET_OK;
}

et_status unpack_run(const et_packed_weight* w, void* dense, cudaStream_t stream) {
  if (w->values == nullptr)
    return fail(ET_ERR_UNSUPPORTED, "et_unpack: no packed values (non-16x16 tiles or column pattern)");
  ET_CUDA(cudaMemsetAsync(dense, 0, (size_t)w->rows * w->cols * dtype_size(w->dtype), stream));
  if (w->ntiles == 0) return ET_OK;
  const int threads = 256;
  const int blocks = (w->ntiles * 32 + threads - 1) / threads;
  if (w->dtype == ET_FP32) {
    unpack32_kernel<<<blocks, threads, 0, stream>>>(static_cast<const float*>(w->values), w->cols, w->pattern,
                                                    w->part_row_ptr, w->tile_col, w->row_map, w->ntiles,
                                                    w->pattern == ET_PRUNE_TILE ? w->rows / 16 : w->rows_padded / 16,
                                                    w->kparts, static_cast<float*>(dense));
    count_launch();
    ET_CUDA(cudaGetLastError());
    return ET_OK;
  }
  unpack_kernel<<<blocks, threads, 0, stream>>>(static_cast<const uint8_t*>(w->values), w->cols, w->pattern,
                                                w->part_row_ptr, w->tile_col, w->row_map, w->ntiles,
                                                w->pattern == ET_PRUNE_TILE ? w->rows / 16 : w->rows_padded / 16,
                                                w->kparts, static_cast<uint16_t*>(dense));
  count_launch();
  ET_CUDA(cudaGetLastError());
  return ET_OK;
}

}  // namespace et
