// Test helper (not product code): Philox4x32-10 outputs of NVIDIA's cuRAND device implementation
// (curand_Philox4x32_10 in curand_philox4x32_x.h) for counters / a key read from stdin, so that
// tests/test_gpu_curand.py can cross-check the library's own device Philox (vs_debug_philox, R23).
#include <cstdio>
#include <vector>
#include <curand_kernel.h>

__global__ void k(int n, const uint4* c, uint2 key, uint4* o) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) o[i] = curand_Philox4x32_10(c[i], key);
}

int main() {
  int n;
  unsigned k0, k1;
  if (std::scanf("%d %u %u", &n, &k0, &k1) != 3) return 2;
  std::vector<uint4> c(n), o(n);
  for (int i = 0; i < n; ++i)
    if (std::scanf("%u %u %u %u", &c[i].x, &c[i].y, &c[i].z, &c[i].w) != 4) return 2;
  uint4 *dc, *dout;
  cudaMalloc(&dc, sizeof(uint4) * n);
  cudaMalloc(&dout, sizeof(uint4) * n);
  cudaMemcpy(dc, c.data(), sizeof(uint4) * n, cudaMemcpyHostToDevice);
  k<<<(n + 127) / 128, 128>>>(n, dc, make_uint2(k0, k1), dout);
  if (cudaMemcpy(o.data(), dout, sizeof(uint4) * n, cudaMemcpyDeviceToHost) != cudaSuccess) return 3;
  for (int i = 0; i < n; ++i) std::printf("%u %u %u %u\n", o[i].x, o[i].y, o[i].z, o[i].w);
  return 0;
}
