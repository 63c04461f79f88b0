// bcf_launch.h -- host-side launch table over the instantiated (E, u) set.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace bcf {

struct SortArgs;
struct MergeArgs;

using BlockSortFn = cudaError_t (*)(const SortArgs&, long long grid, cudaStream_t);
using MergeFn = cudaError_t (*)(const MergeArgs&, long long grid, cudaStream_t);

struct Variant {
  BlockSortFn block_sort = nullptr;
  MergeFn merge = nullptr;        // regular pass (CF: B runs stored descending)
  MergeFn merge_table = nullptr;  // group-table pass, all runs ascending (CF)
  MergeFn merge_tma = nullptr;    // persistent TMA pass (CF, E coprime with 32); grid arg = tiles
  MergeFn merge_win = nullptr;    // the persistent window kernel itself (keys or pairs; reads src_kb/src_vb), or nullptr
  MergeFn merge_multi = nullptr;  // the window kernel running MergeArgs::npass regular passes in one launch
  BlockSortFn block_sort2 = nullptr;  // two-tile block sort (runs of 2 U E; keys-only CF, E = 31)
};

// [E][u index][algo: 0 CF, 1 baseline][pairs]
constexpr int E_MIN = 7, E_MAX = 31;
struct LaunchTable {
  Variant v[E_MAX + 1][3][2][2];
};

inline int u_index(int u) { return u == 128 ? 0 : u == 256 ? 1 : u == 512 ? 2 : -1; }

LaunchTable& launch_table();

// one registration function per E (one translation unit each, compiled in
// parallel); defined in kern_E<E>.cu
#define BCF_DECLARE_REG(E) void register_E##E(LaunchTable&);
BCF_DECLARE_REG(7)
BCF_DECLARE_REG(8)
BCF_DECLARE_REG(9)
BCF_DECLARE_REG(10)
BCF_DECLARE_REG(11)
BCF_DECLARE_REG(12)
BCF_DECLARE_REG(13)
BCF_DECLARE_REG(14)
BCF_DECLARE_REG(15)
BCF_DECLARE_REG(16)
BCF_DECLARE_REG(17)
BCF_DECLARE_REG(31)
#undef BCF_DECLARE_REG

}  // namespace bcf
