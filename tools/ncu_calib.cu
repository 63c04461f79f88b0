// ncu counter calibration for shared-memory bank conflicts:
// stride-1 LDS (0 conflicts), stride-2 (2-way), stride-32 (32-way), broadcast,
// and the CF round-set pattern (stride E = 15).  Built by tools/ncu_calib.py.
#include <cstdint>
extern "C" __global__ void calib_kernel(uint32_t* out, int stride, int iters) {
  __shared__ uint32_t s[32 * 33 * 4];
  for (int i = threadIdx.x; i < 32 * 33 * 4; i += blockDim.x) s[i] = i;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  uint32_t acc = 0;
  int idx = (lane * stride) % (32 * 33 * 4);
  for (int it = 0; it < iters; ++it) {
    acc += s[idx];
    idx = (idx + 1) % (32 * 33 * 4);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

#include <cstdio>
int main() {
  uint32_t* out;
  cudaMalloc(&out, 148 * 256 * sizeof(uint32_t));
  const int strides[] = {1, 2, 32, 0, 15};
  for (int s : strides) {
    calib_kernel<<<148, 256>>>(out, s, 64);
    cudaDeviceSynchronize();
    printf("stride %d launched\n", s);
  }
  cudaFree(out);
  return 0;
}
