// Layout probe (diagnostic): what stmatrix.sync.aligned.m16n8.{x1,x4}.trans.shared.b8 stores
// on sm_100a.  Lane L's register r holds bytes 0x10*... = (L << 2 | b) + 64 * r; each lane's
// address is smem + 16 * L (x1: 16 B per "row" address) -- the dump shows which bytes land where.
#include <cstdio>
#include <cstdint>
__global__ void probe(uint8_t *out1, uint8_t *out4) {
  __shared__ __align__(1024) uint8_t s[8192];
  const int L = threadIdx.x;
  for (int i = L; i < 8192; i += 32) s[i] = 0xEE;
  __syncwarp();
  uint32_t r[4];
  for (int k = 0; k < 4; ++k) r[k] = ((uint32_t)((L << 2) | 0)) | ((uint32_t)((L << 2) | 1) << 8) | ((uint32_t)((L << 2) | 2) << 16) | ((uint32_t)((L << 2) | 3) << 24);
  uint32_t a1 = (uint32_t)__cvta_generic_to_shared(s + 16 * L);
  asm volatile("stmatrix.sync.aligned.m16n8.x1.trans.shared.b8 [%0], {%1};" ::"r"(a1), "r"(r[0]));
  __syncwarp();
  for (int i = L; i < 1024; i += 32) out1[i] = s[i];
  __syncwarp();
  for (int i = L; i < 8192; i += 32) s[i] = 0xEE;
  __syncwarp();
  for (int k = 0; k < 4; ++k) r[k] = (r[k] & 0x3f3f3f3fu) | (0x40404040u * (uint32_t)k);
  uint32_t a4 = (uint32_t)__cvta_generic_to_shared(s + 128 * L);
  asm volatile("stmatrix.sync.aligned.m16n8.x4.trans.shared.b8 [%0], {%1, %2, %3, %4};" ::"r"(a4), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]));
  __syncwarp();
  for (int i = L; i < 4096; i += 32) out4[i] = s[i];
}
int main() {
  uint8_t *d1, *d4;
  cudaMalloc(&d1, 1024);
  cudaMalloc(&d4, 4096);
  probe<<<1, 32>>>(d1, d4);
  uint8_t h1[1024], h4[4096];
  cudaMemcpy(h1, d1, 1024, cudaMemcpyDeviceToHost);
  cudaMemcpy(h4, d4, 4096, cudaMemcpyDeviceToHost);
  printf("x1 (lane L address = s + 16L): rows of 16 bytes, EE = untouched\n");
  for (int row = 0; row < 32; ++row) {
    printf("%3d:", row * 16);
    for (int c = 0; c < 16; ++c) printf(" %02x", h1[row * 16 + c]);
    printf("\n");
  }
  printf("x4 (lane L address = s + 128L): first 16 bytes of each 128-byte row\n");
  for (int row = 0; row < 32; ++row) {
    printf("%4d:", row * 128);
    for (int c = 0; c < 16; ++c) printf(" %02x", h4[row * 128 + c]);
    printf("\n");
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
