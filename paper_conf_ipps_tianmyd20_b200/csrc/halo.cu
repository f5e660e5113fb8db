// Halo pack / unpack of a sharded plan (PAPER.md L99
// §III-A.b: a partition reads the source rows of the blocks E_{k,i} that
// touch it).  Destination partitions are sharded over ranks in contiguous
// plan-row ranges; before an aggregation every rank needs the rows of other
// shards its selective edges and full-mode windows read — the planner's halo
// lists.  pack gathers this shard's rows listed for each peer (peers in rank
// order) into one contiguous send buffer; the transport (NCCL grouped
// send/recv / all-to-all over NVLink, or gloo in the CPU tests) moves the
// segments; unpack scatters the received rows into the full-height input.
// Rows are copied as `w` floats (the activation stride, pad columns
// included): bitwise copies, so a sharded aggregation reproduces the
// unsharded one bit for bit.
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"

namespace pcgcn {
namespace {

// dst[i] = src[idx[i]] (pack, idx = send rows)  or  dst[idx[i]] = src[i] (unpack)
template <bool PACK>
__global__ void __launch_bounds__(256) halo_copy_kernel(const float* __restrict__ src, int64_t lds,
                                                        float* __restrict__ dst, int64_t ldd,
                                                        const int32_t* __restrict__ idx, int64_t rows, int nvec) {
  const int64_t total = rows * nvec;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total;
       t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = t / nvec;
    const int q = int(t - i * nvec);
    const int64_t r = __ldg(idx + i);
    if (PACK) {
      reinterpret_cast<float4*>(dst + i * ldd)[q] = __ldg(reinterpret_cast<const float4*>(src + r * lds) + q);
    } else {
      reinterpret_cast<float4*>(dst + r * ldd)[q] = __ldg(reinterpret_cast<const float4*>(src + i * lds) + q);
    }
  }
}

}  // namespace

cudaError_t launch_halo_copy(bool pack, const float* src, int64_t lds, float* dst, int64_t ldd, const int32_t* idx,
                             int64_t rows, int w, cudaStream_t s) {
  if (rows <= 0) return cudaSuccess;
  const int nvec = w / 4;
  const int64_t total = rows * nvec;
  const unsigned blocks = unsigned(total / 256 + 1 < 148 * 8 ? total / 256 + 1 : 148 * 8);
  if (pack)
    halo_copy_kernel<true><<<blocks, 256, 0, s>>>(src, lds, dst, ldd, idx, rows, nvec);
  else
    halo_copy_kernel<false><<<blocks, 256, 0, s>>>(src, lds, dst, ldd, idx, rows, nvec);
  return cudaGetLastError();
}

}  // namespace pcgcn
