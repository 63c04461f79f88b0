// ncu counter calibration, part 3: does l1tex__data_bank_conflicts_pipe_lsu_mem_shared
// count conflict-free LDS and STS that are merely CONCURRENT (different warps
// or different CTAs of one SM), with no TMA involved?  Every access below is
// conflict-free by address (32 distinct banks per warp instruction).
//   case 0  stride-1 LDS by 4 warps, 1 CTA per SM
//   case 1  stride-31 STS by 4 warps, 1 CTA per SM
//   case 2  warps 0-1 stride-1 LDS || warps 2-3 stride-31 STS (other region), same CTA
//   case 3  case 0 with 5 CTAs per SM
//   case 4  case 1 with 5 CTAs per SM
//   case 5  5 CTAs per SM: even CTAs LDS, odd CTAs STS (concurrent across CTAs)
//   case 6  every warp alternates one LDS and one STS (other region), same CTA
//   case 7  stride-1 LDS.64 (uint2) by 4 warps (2 wavefronts per instruction)
//   case 8  warps 0-2 stride-1 LDS || warp 3 cp.async (LDGSTS) 16-byte copies into another region
//   case 9  warps 0-2 stride-31 STS || warp 3 cp.async 16-byte copies into another region
//   case 10 5 CTAs per SM touching shared memory only once at the end (CTA launch artefact?)
//   case 11 5 CTAs per SM: case 8 (cp.async || LDS) with persistent-style co-residency
//   case 12 5 CTAs per SM: even CTAs only cp.async, odd CTAs only stride-31 STS (cross-CTA)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/ncu_calib_lsu.cu -o tools/ncu_calib_lsu
#include <cstdint>
#include <cstdio>

constexpr int WORDS = 4096;

extern "C" __global__ void __launch_bounds__(128) calib_lsu_kernel(const uint32_t* __restrict__ gin, uint32_t* gout,
                                                                   int which, int iters) {
  __shared__ uint32_t a[WORDS];
  __shared__ uint32_t b[WORDS];
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  for (int i = tid; i < WORDS; i += blockDim.x) {
    a[i] = i;
    b[i] = 3 * i;
  }
  __syncthreads();
  uint32_t acc = 0;
  bool do_ld, do_st;
  switch (which) {
    case 0: case 3: do_ld = true; do_st = false; break;
    case 1: case 4: do_ld = false; do_st = true; break;
    case 2: do_ld = warp < 2; do_st = warp >= 2; break;
    case 5: do_ld = (blockIdx.x & 1) == 0; do_st = !do_ld; break;
    default: do_ld = do_st = true; break;
  }
  if (which == 10) {
    for (int it = 0; it < iters * 64; ++it) acc += __ldg(gin + ((tid + 32 * it) & 65535));
    b[tid] = acc;
    __syncthreads();
    if (acc == 0x12345678u) gout[tid] = acc + b[(tid + 1) & 127];
    return;
  }
  for (int it = 0; it < iters; ++it) {
    if (which == 8 || which == 9 || which == 11 || which == 12) {
      const bool copier = which == 12 ? (blockIdx.x & 1) == 0 : warp == 3;
      if (copier) {
        // 32 lanes x 16 B per round into region b (async, LDGSTS)
#pragma unroll 4
        for (int q = 0; q < 8; ++q) {
          const uint32_t dst = (uint32_t)__cvta_generic_to_shared(b + 4 * ((tid + 32 * q) & 1023));
          const uint32_t* src = gin + 4 * ((blockIdx.x * 256 + tid + 32 * q + it) & 16383);
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      } else if (which == 9 || which == 12) {
#pragma unroll 4
        for (int q = 0; q < 31; ++q) a[(31 * tid + q + it) & (WORDS - 1)] = q + it;
      } else {
#pragma unroll 4
        for (int q = 0; q < 64; ++q) acc += a[(tid + 32 * q + it) & (WORDS - 1)];
      }
      continue;
    }
    if (which == 7) {
#pragma unroll 4
      for (int q = 0; q < 32; ++q) {
        const uint2 v = reinterpret_cast<const uint2*>(a)[(tid + 64 * q + it) & (WORDS / 2 - 1)];
        acc += v.x ^ v.y;
      }
    } else if (which == 6) {
#pragma unroll 4
      for (int q = 0; q < 31; ++q) {
        acc += a[(tid + 32 * q + it) & (WORDS - 1)];
        b[(31 * tid + q + it) & (WORDS - 1)] = acc;
      }
    } else {
      if (do_ld) {
#pragma unroll 4
        for (int q = 0; q < 64; ++q) acc += a[(tid + 32 * q + it) & (WORDS - 1)];
      }
      if (do_st) {
#pragma unroll 4
        for (int q = 0; q < 31; ++q) b[(31 * (tid & 127) + q + it) & (WORDS - 1)] = q + it;
      }
    }
  }
  __syncthreads();
  if (acc == 0x12345678u) gout[tid] = acc + b[tid];
}

int main() {
  uint32_t *out, *in;
  cudaMalloc(&out, 1 << 20);
  cudaMalloc(&in, 1 << 20);
  cudaMemset(in, 1, 1 << 20);
  for (int which = 0; which <= 12; ++which) {
    const int ctas = ((which >= 3 && which <= 5) || which >= 10) ? 148 * 5 : 148;
    calib_lsu_kernel<<<ctas, 128>>>(in, out, which, 256);
    cudaError_t e = cudaDeviceSynchronize();
    printf("case %d: %s\n", which, cudaGetErrorString(e));
  }
  cudaFree(out);
  cudaFree(in);
  return 0;
}
