// HBM copy throughput vs number of CTAs (256 threads, 256-bit vectors, U vectors in flight
// per lane): how many CTAs a pure data-moving phase needs to saturate HBM on this GPU.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/copybw_bin tools/copybw.cu
#include <cstdio>
#include <cuda_runtime.h>
struct V32 { uint4 a, b; };
template <int U>
__global__ void __launch_bounds__(256) copyk(const V32* __restrict__ a, V32* __restrict__ c, long nvec) {
  // each CTA streams its own contiguous slab (like one interpreter thread block)
  const long per = (nvec + gridDim.x - 1) / gridDim.x;
  const long lo = per * blockIdx.x, hi = lo + per < nvec ? lo + per : nvec;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (long base = lo + (long)warp * U * 32; base + U * 32 <= hi; base += (long)nw * U * 32) {
    V32 x[U];
#pragma unroll
    for (int u = 0; u < U; u++)
      asm volatile("ld.global.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(x[u].a.x), "=r"(x[u].a.y), "=r"(x[u].a.z), "=r"(x[u].a.w), "=r"(x[u].b.x), "=r"(x[u].b.y),
                     "=r"(x[u].b.z), "=r"(x[u].b.w) : "l"(a + base + u * 32 + lane) : "memory");
#pragma unroll
    for (int u = 0; u < U; u++)
      asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(c + base + u * 32 + lane), "r"(x[u].a.x),
                   "r"(x[u].a.y), "r"(x[u].a.z), "r"(x[u].a.w), "r"(x[u].b.x), "r"(x[u].b.y), "r"(x[u].b.z), "r"(x[u].b.w)
                   : "memory");
  }
}
template <int U>
void run(const V32* a, V32* c, long nvec, int g) {
  copyk<U><<<g, 256>>>(a, c, nvec);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int i = 0; i < 5; i++) copyk<U><<<g, 256>>>(a, c, nvec);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  printf("U=%d ctas=%4d: %.0f GB/s (read+write)\n", U, g, 2.0 * nvec * 32 * 5 / (ms * 1e-3) / 1e9);
}
int main() {
  long bytes = 1L << 30, nvec = bytes / 32;
  V32 *a, *c;
  cudaMalloc(&a, bytes);
  cudaMalloc(&c, bytes);
  cudaMemset(a, 1, bytes);
  for (int g : {56, 112, 148, 224, 296, 444, 592}) {
    run<4>(a, c, nvec, g);
    run<8>(a, c, nvec, g);
  }
  return 0;
}
