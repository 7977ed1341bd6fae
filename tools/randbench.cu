// randbench.cu -- B200 memory ceilings for the BFS roofline (diagnostics, not the product):
// the access classes the level and depth kernels are made of, each timed alone with CUDA
// events (best of 3) over arrays well beyond the 126 MB L2 unless stated.
//   seq_read / seq_write / copy       streaming 16-byte accesses (the commit scan, the rows)
//   gather16 over S bytes, U in flight random 16-byte loads (one 32-byte sector each): the
//                                     bottom-up visited[w] reads, top-down pre-checks
//   gather8                           random 8-byte loads
//   red_or64 over S                   one random 64-bit RED.OR
//   red_or128 over S                  two 64-bit RED.OR on the same 16 bytes (a 128-bit
//                                     status word's top-down update)
//   st32_rows                         4-byte streaming stores, warp = 4 rows x 32 contiguous
//                                     bytes (the depth kernel's store pattern)
// Prints one JSON object (profiles/randbench.json).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/randbench tools/randbench.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

__global__ void seq_read(const uint4 *p, size_t n, uint32_t *out) {
  uint32_t acc = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = __ldcs(p + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678) out[0] = acc;
}

__global__ void seq_write(uint4 *p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    __stcs(p + i, make_uint4((uint32_t)i, 1, 2, 3));
}

__global__ void copy16(const uint4 *a, uint4 *b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    __stcs(b + i, __ldcs(a + i));
}

template <int U, typename V>
__global__ void gather(const V *p, size_t nwords, size_t per_thread, uint32_t *out, uint64_t seed) {
  uint32_t acc = 0;
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (size_t k = 0; k < per_thread; k += U) {
    V v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      uint64_t h = mix(seed ^ (tid * 1000003ull + k + u));
      v[u] = __ldg(p + (h % nwords));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= reinterpret_cast<const uint32_t *>(&v[u])[0];
  }
  if (acc == 0x12345678) out[0] = acc;
}

template <int WORDS>
__global__ void red_or(unsigned long long *p, size_t nslots, size_t per_thread, uint64_t seed) {
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (size_t k = 0; k < per_thread; ++k) {
    uint64_t h = mix(seed ^ (tid * 1000003ull + k));
    unsigned long long *q = p + (h % nslots) * WORDS;
#pragma unroll
    for (int w = 0; w < WORDS; ++w)
      asm volatile("red.global.or.b64 [%0], %1;" ::"l"(q + w), "l"(1ull << ((h >> (58 - w)) & 63)) : "memory");
  }
}

// warp = 4 rows x 32 contiguous bytes per 4-byte store instruction (rows `stride` apart)
__global__ void st32_rows(uint8_t *p, size_t rows, size_t stride) {
  const int lane = threadIdx.x & 31;
  const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nwarps = ((size_t)gridDim.x * blockDim.x) >> 5;
  const size_t colchunks = stride / 32;
  for (size_t w = warp; w < (rows / 4) * colchunks; w += nwarps) {
    const size_t rq = w / colchunks, cc = w % colchunks;
    const size_t row = rq * 4 + (lane >> 3);
    __stcs(reinterpret_cast<unsigned int *>(p + row * stride + cc * 32 + (lane & 7) * 4), (unsigned)w);
  }
}

static cudaEvent_t ea, eb;
template <typename F>
static float best3(F &&f) {
  float best = 1e30f;
  for (int r = 0; r < 3; ++r) {
    cudaEventRecord(ea);
    f(r);
    cudaEventRecord(eb);
    cudaEventSynchronize(eb);
    float ms;
    cudaEventElapsedTime(&ms, ea, eb);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  const size_t big = 8ull << 30;
  uint8_t *buf, *buf2;
  if (cudaMalloc(&buf, big) != cudaSuccess || cudaMalloc(&buf2, big) != cudaSuccess) {
    printf("{\"error\": \"alloc\"}\n");
    return 1;
  }
  cudaMemset(buf, 1, big);
  cudaMemset(buf2, 0, big);
  uint32_t *out;
  cudaMalloc(&out, 4);
  cudaEventCreate(&ea);
  cudaEventCreate(&eb);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int grid = sms * 8;
  printf("{\n \"tool\": \"tools/randbench.cu\", \"sms\": %d,\n", sms);
  float ms = best3([&](int) { seq_read<<<grid, 256>>>((const uint4 *)buf, big / 16, out); });
  printf(" \"seq_read_gbs\": %.1f,\n", big / ms / 1e6);
  ms = best3([&](int) { seq_write<<<grid, 256>>>((uint4 *)buf2, big / 16); });
  printf(" \"seq_write_gbs\": %.1f,\n", big / ms / 1e6);
  ms = best3([&](int) { copy16<<<grid, 256>>>((const uint4 *)buf, (uint4 *)buf2, big / 16); });
  printf(" \"copy_rw_gbs\": %.1f,\n", 2.0 * big / ms / 1e6);
  ms = best3([&](int) { st32_rows<<<grid, 256>>>(buf2, 4096, (size_t)2 << 20); });
  printf(" \"st32_rows_gbs\": %.1f,\n", (4096.0 * (2 << 20)) / ms / 1e6);
  const size_t sizes[] = {32ull << 20, 512ull << 20, 2ull << 30, 8ull << 30};
  const char *names[] = {"32MiB", "512MiB", "2GiB", "8GiB"};
  const size_t nthreads = (size_t)sms * 2048;
  double best_g16_big = 0;
  printf(" \"gather16_per_s\": {");
  for (int si = 0; si < 4; ++si) {
    const size_t sz = sizes[si];
    const size_t per = 64;
    double bestr = 0;
    int bu = 0;
    for (int U : {4, 8, 16}) {
      float t = best3([&](int r) {
        if (U == 4) gather<4, uint4><<<nthreads / 256, 256>>>((const uint4 *)buf, sz / 16, per, out, 7 + r);
        if (U == 8) gather<8, uint4><<<nthreads / 256, 256>>>((const uint4 *)buf, sz / 16, per, out, 7 + r);
        if (U == 16) gather<16, uint4><<<nthreads / 256, 256>>>((const uint4 *)buf, sz / 16, per, out, 7 + r);
      });
      const double rate = (double)nthreads * per / (t * 1e-3);
      if (rate > bestr) { bestr = rate; bu = U; }
    }
    if (si == 2) best_g16_big = bestr;
    printf("%s\"%s\": {\"rate\": %.4g, \"sector_gbs\": %.1f, \"useful16_gbs\": %.1f, \"U\": %d}", si ? ", " : "",
           names[si], bestr, bestr * 32 / 1e9, bestr * 16 / 1e9, bu);
  }
  printf("},\n");
  printf(" \"gather8_per_s\": {");
  for (int si = 0; si < 4; ++si) {
    const size_t sz = sizes[si];
    float t = best3([&](int r) {
      gather<8, unsigned long long><<<nthreads / 256, 256>>>((const unsigned long long *)buf, sz / 8, 64, out, 9 + r);
    });
    printf("%s\"%s\": %.4g", si ? ", " : "", names[si], (double)nthreads * 64 / (t * 1e-3));
  }
  printf("},\n");
  printf(" \"red_or64_per_s\": {");
  for (int si = 0; si < 4; ++si) {
    const size_t sz = sizes[si];
    float t = best3([&](int r) { red_or<1><<<nthreads / 256, 256>>>((unsigned long long *)buf2, sz / 8, 32, 11 + r); });
    printf("%s\"%s\": %.4g", si ? ", " : "", names[si], (double)nthreads * 32 / (t * 1e-3));
  }
  printf("},\n");
  printf(" \"red_or128_per_s\": {");
  double red128_big = 0;
  for (int si = 0; si < 4; ++si) {
    const size_t sz = sizes[si];
    float t = best3([&](int r) { red_or<2><<<nthreads / 256, 256>>>((unsigned long long *)buf2, sz / 16, 32, 13 + r); });
    const double rate = (double)nthreads * 32 / (t * 1e-3);
    if (si == 2) red128_big = rate;
    printf("%s\"%s\": %.4g", si ? ", " : "", names[si], rate);
  }
  printf("},\n");
  printf(" \"gather16_per_s_2GiB\": %.4g, \"red_or128_per_s_2GiB\": %.4g,\n", best_g16_big, red128_big);
  cudaError_t e = cudaDeviceSynchronize();
  printf(" \"status\": \"%s\"\n}\n", cudaGetErrorString(e));
  return 0;
}
