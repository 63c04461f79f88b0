// ncu counter calibration, part 2: does l1tex__data_bank_conflicts_pipe_lsu_mem_shared
// count shared-memory traffic that is NOT issued by LDS/STS instructions?
// Each case is one launch (148 CTAs x 160 threads) doing only one kind of
// shared-memory access, repeated `iters` times:
//   case 0  cp.async.bulk global->shared, 128-B aligned smem destination
//   case 1  cp.async.bulk global->shared, smem destination at +16 B (16-B aligned only)
//   case 2  cp.async.bulk shared->global, 128-B aligned smem source
//   case 3  cp.async.bulk shared->global, smem source at +16 B
//   case 4  mbarrier.try_wait spin by 128 threads on one barrier (thread 128 arrives late)
//   case 5  LDS.128 (uint4) stride-1 loads by 128 threads (4 wavefronts per instruction)
//   case 6  all-thread broadcast read of a 48-byte struct (the merge pass's WinMeta)
//   case 7  conflict-free stride-1 LDS by warps 0-3 WHILE thread 128 streams bulk
//           global->shared copies into another smem region (the merge pass's overlap)
//   case 8  conflict-free stride-1 LDS by warps 0-3 WHILE warp 4 streams LDG (L1 fills)
//   case 9  stride-31 STS by warps 0-3 (the merge pass's output staging), alone
//   case 10 stride-31 STS by warps 0-3 WHILE thread 128 streams bulk shared->global
//   case 11 stride-1 LDS by warps 0-3 WHILE thread 128 streams bulk shared->global
//   case 12 stride-31 STS by warps 0-3 WHILE thread 128 streams bulk global->shared
//   case 13 stride-31 STS by warps 0-3 WHILE warp 4 streams LDG (L1 fills)
//   case 14 stride-1 LDS by warps 0-3 WHILE warp 4 streams STG
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I<csrc> tools/ncu_calib_tma.cu
#include <cstdint>
#include <cstdio>

#include "bcf_tma.cuh"

using namespace bcf;

constexpr int BYTES = 16384;

struct Meta12 {
  long long c0;
  int a[10];
};

extern "C" __global__ void __launch_bounds__(160) calib_tma_kernel(uint32_t* gin, uint32_t* gout, int which, int iters) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ Meta12 meta;
  const int tid = threadIdx.x;
  uint32_t* s = reinterpret_cast<uint32_t*>(sm + ((which == 1 || which == 3) ? 16 : 0));
  if (tid == 0) tma::mbar_init(&bar, 1);
  if (tid < 12) reinterpret_cast<int*>(&meta)[tid] = tid;
  for (int i = tid; i < 2 * BYTES / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = i;
  tma::fence_proxy_async_smem();
  __syncthreads();
  const uint32_t* src = gin + (size_t)blockIdx.x * (BYTES / 4);
  uint32_t* dst = gout + (size_t)blockIdx.x * (BYTES / 4);
  uint32_t acc = 0;
  for (int it = 0; it < iters; ++it) {
    if (which <= 1) {
      if (tid == 0) {
        tma::mbar_expect_tx(&bar, BYTES - 16);
        tma::bulk_g2s(s, src, BYTES - 16, &bar);
        tma::mbar_arrive(&bar);
        tma::mbar_wait(&bar, it & 1);
      }
    } else if (which <= 3) {
      if (tid == 0) {
        tma::bulk_s2g(dst, s, BYTES - 16);
        tma::bulk_commit();
        tma::bulk_wait_all();
      }
    } else if (which == 4) {
      if (tid == 128) {
        long long t0 = clock64();
        while (clock64() - t0 < 2000) {
        }
        tma::mbar_arrive(&bar);
      } else if (tid < 128) {
        tma::mbar_wait(&bar, it & 1);
      }
    } else if (which == 5) {
      if (tid < 128) {
        const uint4 v = reinterpret_cast<const uint4*>(sm)[(tid + it) & 1023];
        acc += v.x ^ v.y ^ v.z ^ v.w;
      }
    } else if (which >= 9) {
      if (tid < 128) {
        uint32_t* x = reinterpret_cast<uint32_t*>(sm + BYTES);
        if (which == 11 || which == 14) {
#pragma unroll 4
          for (int q = 0; q < 64; ++q) acc += x[(tid + 32 * q + it) & 4095];
        } else {
          // thread t writes words 31 t + q (q = 0..30): a round set per q
#pragma unroll 4
          for (int q = 0; q < 31; ++q) x[(31 * tid + q + it) & 4095] = q + it;
        }
      } else if (which == 13) {
#pragma unroll 4
        for (int q = 0; q < BYTES / 4 / 32; ++q) acc += __ldg(src + (tid - 128) + 32 * q);
      } else if (which == 14) {
#pragma unroll 4
        for (int q = 0; q < BYTES / 4 / 32; ++q) dst[(tid - 128) + 32 * q] = q + it;
      } else if (tid == 128 && which != 9) {
        if (which == 12) {
          tma::mbar_expect_tx(&bar, BYTES);
          tma::bulk_g2s(sm, src, BYTES, &bar);
          tma::mbar_arrive(&bar);
          tma::mbar_wait(&bar, it & 1);
        } else {
          tma::bulk_s2g(dst, sm, BYTES);
          tma::bulk_commit();
          tma::bulk_wait_all();
        }
      }
    } else if (which == 7 || which == 8) {
      if (tid < 128) {
        const uint32_t* x = reinterpret_cast<const uint32_t*>(sm + BYTES);
#pragma unroll 4
        for (int q = 0; q < 64; ++q) acc += x[(tid + 32 * q + it) & 4095];
      } else if (which == 7) {
        if (tid == 128) {
          tma::mbar_expect_tx(&bar, BYTES);
          tma::bulk_g2s(sm, src, BYTES, &bar);
          tma::mbar_arrive(&bar);
          tma::mbar_wait(&bar, it & 1);
        }
      } else {
        const uint32_t* g = src;
#pragma unroll 4
        for (int q = 0; q < BYTES / 4 / 32; ++q) acc += __ldg(g + (tid - 128) + 32 * q);
      }
    } else {
      Meta12 m = meta;
      acc += (uint32_t)m.c0 + m.a[(it + tid) % 10];
      __syncwarp();
    }
    __syncthreads();
  }
  if (acc == 0x12345678u) gout[tid] = acc;
}

int main() {
  uint32_t *in, *out;
  const size_t words = (size_t)148 * BYTES / 4;
  cudaMalloc(&in, words * 4);
  cudaMalloc(&out, words * 4);
  cudaMemset(in, 1, words * 4);
  cudaFuncSetAttribute(calib_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * BYTES + 128);
  for (int which = 0; which <= 14; ++which) {
    calib_tma_kernel<<<148, 160, 2 * BYTES + 128>>>(in, out, which, 64);
    cudaError_t e = cudaDeviceSynchronize();
    printf("case %d: %s\n", which, cudaGetErrorString(e));
  }
  cudaFree(in);
  cudaFree(out);
  return 0;
}
