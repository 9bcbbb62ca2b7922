// Integer pipe microbenchmark (B200): warp-instruction throughput per SM of IMAD (reg x reg),
// VIMNMX3 (3-input min) and the expand hot-loop mix (2 IMAD : 1 VIMNMX3).
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a int_pipes.cu -o int_pipes
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_imad(uint32_t* out, int iters, uint32_t s) {
  uint32_t a[16];
  for (int i = 0; i < 16; i++) a[i] = threadIdx.x * 7u + i + s;
  const uint32_t b = s | 1u;
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < 16; i++) a[i] = a[i] * b;  // IMAD R, R, R, RZ
  }
  uint32_t x = 0;
  for (int i = 0; i < 16; i++) x ^= a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}
__global__ void k_min3(uint32_t* out, int iters, uint32_t s) {
  uint32_t a[16];
  for (int i = 0; i < 16; i++) a[i] = threadIdx.x * 7u + i + s;
  const uint32_t b = s ^ 0x1234u, c = s ^ 0x77u;
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < 16; i++) a[i] = min(min(a[i], b + (uint32_t)it), c ^ a[(i + 1) & 15]);
  }
  uint32_t x = 0;
  for (int i = 0; i < 16; i++) x ^= a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}
// hot-loop mix: per node quad, CPT=8 candidates: 32 IMAD + 16 VIMNMX3
__global__ void k_mix(uint32_t* out, int iters, uint32_t s) {
  uint32_t h[8];
  for (int c = 0; c < 8; c++) h[c] = (threadIdx.x + c) * 2654435761u + s;
  uint32_t acc = 0;
  uint32_t n0 = s, n1 = s + 1, n2 = s + 2, n3 = s + 3;
  for (int it = 0; it < iters; it++) {
    uint32_t m0 = ~0u, m1 = ~0u, m2 = ~0u, m3 = ~0u;
#pragma unroll
    for (int c = 0; c < 8; c++) {
      m0 = min(m0, n0 * h[c]);
      m1 = min(m1, n1 * h[c]);
      m2 = min(m2, n2 * h[c]);
      m3 = min(m3, n3 * h[c]);
    }
    acc += m0 ^ m1 ^ m2 ^ m3;
    n0 += 4; n1 += 4; n2 += 4; n3 += 4;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

// faithful hot loop: node quads streamed from shared memory, CPT=32 candidates in registers
__global__ void k_hot(uint32_t* out, int iters, uint32_t s) {
  __shared__ uint4 tab[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) tab[i] = make_uint4(s + 4 * i, s + 4 * i + 1, s * 3 + i, s ^ i);
  __syncthreads();
  uint32_t h[32];
  for (int c = 0; c < 32; c++) h[c] = (threadIdx.x * 32 + c) * 2654435761u + s;
  uint32_t acc = 0;
  for (int it = 0; it < iters; it++) {
    const uint4 n4 = tab[it & 255];
    uint32_t m0 = ~0u, m1 = ~0u, m2 = ~0u, m3 = ~0u;
#pragma unroll
    for (int c = 0; c < 32; c++) {
      m0 = min(m0, n4.x * h[c]);
      m1 = min(m1, n4.y * h[c]);
      m2 = min(m2, n4.z * h[c]);
      m3 = min(m3, n4.w * h[c]);
    }
    acc += __ballot_sync(0xffffffffu, m0 < 0x10000u) ^ __ballot_sync(0xffffffffu, m1 < 0x10000u) ^
           __ballot_sync(0xffffffffu, m2 < 0x10000u) ^ __ballot_sync(0xffffffffu, m3 < 0x10000u);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

// transposed hot loop: lane = node (register), candidate magics warp-uniform from constant memory
__constant__ uint32_t c_mag[4096];
__global__ void k_hotT(uint32_t* out, int iters, uint32_t s) {
  uint32_t n = threadIdx.x * 2654435761u + s;
  uint32_t acc = 0;
  for (int it = 0; it < iters; it++) {
    const int base = (it * 32) & 4095;
    uint32_t m = 0xffffffffu, m2 = 0xffffffffu;
#pragma unroll
    for (int c = 0; c < 32; c += 2) {
      m = min(m, min(n * c_mag[base + c], n * c_mag[base + c + 1]));
    }
    acc += (m < 0x10000u) << (it & 31);
    n += acc & 1;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

// transposed, 4 nodes per lane, 32 uniform magics hoisted into uniform registers
__global__ void k_hotT2(uint32_t* out, int iters, uint32_t s) {
  uint32_t n0 = threadIdx.x * 2654435761u + s, n1 = n0 + 7, n2 = n0 + 13, n3 = n0 + 29;
  uint32_t acc = 0;
  for (int it = 0; it < iters; it++) {
    uint32_t m0 = ~0u, m1 = ~0u, m2 = ~0u, m3 = ~0u;
#pragma unroll
    for (int c = 0; c < 32; c++) {
      const uint32_t mc = c_mag[c];
      m0 = min(m0, n0 * mc);
      m1 = min(m1, n1 * mc);
      m2 = min(m2, n2 * mc);
      m3 = min(m3, n3 * mc);
    }
    acc += __ballot_sync(0xffffffffu, m0 < 0x10000u) ^ __ballot_sync(0xffffffffu, m1 < 0x10000u) ^
           __ballot_sync(0xffffffffu, m2 < 0x10000u) ^ __ballot_sync(0xffffffffu, m3 < 0x10000u);
    n0 += acc & 1; n1 += acc & 2; n2 += acc & 4; n3 += acc & 8;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  uint32_t* out;
  cudaMalloc(&out, 64 << 20);
  {
    static uint32_t h[4096];
    for (int i = 0; i < 4096; i++) h[i] = 0xffffffffu / (uint32_t)(i + 1) + 1u;
    cudaMemcpyToSymbol(c_mag, h, sizeof h);
  }
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 20000;
  for (int warps = 8; warps <= 32; warps *= 2) {
    const int blocks = sms * warps / 8, threads = 256;
    for (int k = 3; k < 6; k++) {
      for (int rep = 0; rep < 2; rep++) {
        cudaEventRecord(a);
        if (k == 0) k_imad<<<blocks, threads>>>(out, iters, 3);
        if (k == 1) k_min3<<<blocks, threads>>>(out, iters, 3);
        if (k == 2) k_mix<<<blocks, threads>>>(out, iters, 3);
        if (k == 3) k_hot<<<blocks, threads>>>(out, iters / 4, 3);
        if (k == 4) k_hotT<<<blocks, threads>>>(out, iters * 4, 3);
        if (k == 5) k_hotT2<<<blocks, threads>>>(out, iters, 3);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
      }
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      // intended warp instructions per thread-iteration: imad 16, min3 16 (+16 IADD/LOP),
      // mix 32 IMAD + 16 VIMNMX3 (+ ~6 overhead)
      const double per_it = k == 0 ? 16 : k == 1 ? 16 : k == 2 ? 32 : k == 3 ? 128.0 / 4 : k == 4 ? 32.0 * 4 : 128.0;  // counted: the multiplies
      const double warp_inst = (double)blocks * threads / 32 * iters * per_it;
      printf("%s warps/SM=%d: %.3f ms  %.3f counted warp-inst per SM per cycle (clock %d kHz)\n",
             k == 0 ? "IMAD   " : k == 1 ? "VIMNMX3" : k == 2 ? "MIX(IMAD)" : k == 3 ? "HOT(IMAD)" : k == 4 ? "HOT-T(IMAD, uniform magic)" : "HOT-T2(4 nodes/lane, UR magics)", warps, ms,
             warp_inst / sms / (ms * 1e-3) / (clk * 1e3), clk);
    }
  }
  return 0;
}
