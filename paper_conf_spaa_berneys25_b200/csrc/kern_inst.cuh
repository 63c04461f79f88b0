// kern_inst.cuh -- explicit instantiation of the kernels for one E and the
// three block sizes; included by kern_E<E>.cu with BCF_E defined.
#pragma once
#include "bcf_kernels.cuh"
#include "bcf_launch.h"

namespace bcf {

// Opt in to > 48 KB dynamic shared memory once per (kernel, device).
template <typename K>
cudaError_t ensure_smem_attr(K kernel, size_t bytes) {
  static int done_mask = 0;  // bit per device ordinal (< 32 devices)
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (bytes <= 48 * 1024 || (__atomic_load_n(&done_mask, __ATOMIC_ACQUIRE) >> dev) & 1) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) __atomic_fetch_or(&done_mask, 1 << dev, __ATOMIC_ACQ_REL);
  return e;
}

template <int E, int U, bool PAIRS, bool CF>
cudaError_t launch_block_sort(const SortArgs& a, long long grid, cudaStream_t s) {
  constexpr size_t smem = tile_smem_bytes<E, U, PAIRS>();
  cudaError_t e = ensure_smem_attr(block_sort_kernel<E, U, PAIRS, CF>, smem);
  if (e != cudaSuccess) return e;
  block_sort_kernel<E, U, PAIRS, CF><<<(unsigned)grid, U, smem, s>>>(a);
  return cudaGetLastError();
}

template <int E, int U, bool PAIRS, bool CF, bool BDESC>
cudaError_t launch_merge(const MergeArgs& a, long long grid, cudaStream_t s) {
  constexpr size_t smem = tile_smem_bytes<E, U, PAIRS>();
  cudaError_t e = ensure_smem_attr(merge_pass_kernel<E, U, PAIRS, CF, BDESC>, smem);
  if (e != cudaSuccess) return e;
  merge_pass_kernel<E, U, PAIRS, CF, BDESC><<<(unsigned)grid, U, smem, s>>>(a);
  return cudaGetLastError();
}

template <int E, int U>
void register_eu(LaunchTable& t) {
  const int ui = u_index(U);
  t.v[E][ui][0][0] = {&launch_block_sort<E, U, false, true>, &launch_merge<E, U, false, true, true>,
                      &launch_merge<E, U, false, true, false>};
  t.v[E][ui][0][1] = {&launch_block_sort<E, U, true, true>, &launch_merge<E, U, true, true, true>,
                      &launch_merge<E, U, true, true, false>};
  t.v[E][ui][1][0] = {&launch_block_sort<E, U, false, false>, &launch_merge<E, U, false, false, false>,
                      nullptr};
}

}  // namespace bcf

#define BCF_DEFINE_REG(E)                         \
  namespace bcf {                                 \
  void register_E##E(LaunchTable& t) {            \
    register_eu<E, 128>(t);                       \
    register_eu<E, 256>(t);                       \
    register_eu<E, 512>(t);                       \
  }                                               \
  }
