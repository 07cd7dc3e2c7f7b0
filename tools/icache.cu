// Instruction-fetch cost of cold code: one thread runs a straight-line block of N dependent
// FMAs (16 bytes of SASS each) twice in one launch; pass 1 fetches the code, pass 2 runs it
// from the instruction cache. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/icache_bin tools/icache.cu
#include <cstdio>
#include <cstdint>

template <int N>
__device__ __noinline__ float block(float x, float a, float b) {
#pragma unroll
  for (int i = 0; i < N; i++) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(x) : "f"(a), "f"(b));
  return x;
}

template <int N>
__global__ void run(float* out, long long* cyc, float a, float b) {
  if (threadIdx.x != 0) return;
  float x = out[0];
  long long t0 = clock64();
  x = block<N>(x, a, b);
  long long t1 = clock64();
  x = block<N>(x, a, b);
  long long t2 = clock64();
  out[1 + blockIdx.x] = x;
  cyc[2 * blockIdx.x] = t1 - t0;
  cyc[2 * blockIdx.x + 1] = t2 - t1;
}

template <int N>
void go(float* out, long long* cyc, int blocks) {
  for (int rep = 0; rep < 3; rep++) run<N><<<blocks, 32>>>(out, cyc, 1.0f, 0.0f);
  long long h[2];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  printf("%6d FMAs (%4d KiB of code) blocks %3d: cold pass %7lld cycles, warm pass %7lld cycles -> %.2f us per cold KiB\n",
         N, N * 16 / 1024, blocks, h[0], h[1], (h[0] - h[1]) / 1.965e3 / (N * 16 / 1024.0));
}

int main() {
  float* out;
  long long* cyc;
  cudaMalloc(&out, 4096);
  cudaMalloc(&cyc, 4096);
  cudaMemset(out, 0, 4096);
  go<256>(out, cyc, 1);
  go<1024>(out, cyc, 1);
  go<4096>(out, cyc, 1);
  go<4096>(out, cyc, 112);
  return 0;
}
