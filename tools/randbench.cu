// randbench.cu -- B200 memory microbenchmarks for the BFS roofline (diagnostics):
// streaming read, random 16-byte gathers (one 32-byte sector each) over arrays of several
// sizes, and random 64-bit RED.OR -- the access classes the level kernels are made of.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o randbench randbench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

__global__ void seq_read(const uint4 *p, size_t n, uint32_t *out) {
  uint32_t acc = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = __ldg(p + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678) out[0] = acc;
}

template <int U>
__global__ void rand_gather(const uint4 *p, size_t nwords, size_t per_thread, uint32_t *out, uint64_t seed) {
  uint32_t acc = 0;
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (size_t k = 0; k < per_thread; k += U) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      uint64_t h = mix(seed ^ (tid * 1000003ull + k + u));
      v[u] = __ldg(p + (h % nwords));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].w;
  }
  if (acc == 0x12345678) out[0] = acc;
}

__global__ void rand_red(unsigned long long *p, size_t nwords, size_t per_thread, uint64_t seed) {
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (size_t k = 0; k < per_thread; ++k) {
    uint64_t h = mix(seed ^ (tid * 1000003ull + k));
    atomicOr(p + (h % nwords), 1ull << (h >> 58));
  }
}

int main() {
  const size_t big = 8ull << 30;
  void *buf;
  cudaMalloc(&buf, big);
  cudaMemset(buf, 1, big);
  uint32_t *out;
  cudaMalloc(&out, 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float ms;
  // streaming
  for (int r = 0; r < 3; ++r) {
    cudaEventRecord(a);
    seq_read<<<sms * 8, 256>>>((const uint4 *)buf, big / 16, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
  }
  printf("seq_read 8 GiB: %.1f GB/s\n", big / ms / 1e6);
  const size_t sizes[] = {32ull << 20, 128ull << 20, 1ull << 30, 8ull << 30};
  for (size_t sz : sizes) {
    const size_t nthreads = (size_t)sms * 2048;
    const size_t per = 64;
    for (int r = 0; r < 2; ++r) {
      cudaEventRecord(a);
      rand_gather<8><<<nthreads / 256, 256>>>((const uint4 *)buf, sz / 16, per, out, 7 + r);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      cudaEventElapsedTime(&ms, a, b);
    }
    double n = (double)nthreads * per;
    printf("rand_gather16 over %6zu MiB: %.2f G gathers/s = %.1f GB/s of 32B sectors\n", sz >> 20,
           n / ms / 1e6, n * 32 / ms / 1e6);
  }
  for (size_t sz : sizes) {
    const size_t nthreads = (size_t)sms * 2048;
    const size_t per = 32;
    for (int r = 0; r < 2; ++r) {
      cudaEventRecord(a);
      rand_red<<<nthreads / 256, 256>>>((unsigned long long *)buf, sz / 8, per, 11 + r);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      cudaEventElapsedTime(&ms, a, b);
    }
    double n = (double)nthreads * per;
    printf("rand_red_or64 over %6zu MiB: %.2f G reds/s\n", sz >> 20, n / ms / 1e6);
  }
  cudaError_t e = cudaGetLastError();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
