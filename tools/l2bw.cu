// L2 / HBM throughput microbenchmark for the roofline of the virtual-rank interpreter.
// Persistent grid (k CTAs per SM), 256-bit loads/stores (the interpreter's vector width),
// working set of W bytes touched `passes` times; pattern 'c' = copy (1 read + 1 write per
// element), 'r' = rrs-like (2 reads + 1 write). Prints GB/s of touched bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/l2bw_bin tools/l2bw.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

struct V32 { uint4 a, b; };
__device__ __forceinline__ V32 ld(const void* p) {
  V32 v;
  asm volatile("ld.global.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v.a.x), "=r"(v.a.y), "=r"(v.a.z), "=r"(v.a.w), "=r"(v.b.x), "=r"(v.b.y), "=r"(v.b.z), "=r"(v.b.w)
               : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st(void* p, const V32& v) {
  asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v.a.x), "r"(v.a.y), "r"(v.a.z),
               "r"(v.a.w), "r"(v.b.x), "r"(v.b.y), "r"(v.b.z), "r"(v.b.w) : "memory");
}

template <int MODE>
__global__ void __launch_bounds__(256) kern(const V32* a, const V32* b, V32* c, long nvec, int passes) {
  const long tid = (long)blockIdx.x * blockDim.x + threadIdx.x, nt = (long)gridDim.x * blockDim.x;
  for (int p = 0; p < passes; p++) {
    for (long i = tid; i < nvec; i += 4 * nt) {
      V32 x[4], y[4];
#pragma unroll
      for (int u = 0; u < 4; u++)
        if (i + u * nt < nvec) {
          x[u] = ld(a + i + u * nt);
          if (MODE == 1) y[u] = ld(b + i + u * nt);
        }
#pragma unroll
      for (int u = 0; u < 4; u++)
        if (i + u * nt < nvec) {
          if (MODE == 1) x[u].a.x ^= y[u].a.x, x[u].b.y ^= y[u].b.y;
          st(c + i + u * nt, x[u]);
        }
    }
  }
}

int main(int argc, char** argv) {
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const long sizes[] = {8, 16, 24, 32, 48, 64, 96, 128, 1024};
  for (int mode = 0; mode < 2; mode++) {
    for (long mib : sizes) {
      long bytes = mib << 20;  // per stream
      long nvec = bytes / 32;
      V32 *a, *b, *c;
      cudaMalloc(&a, bytes);
      cudaMalloc(&b, bytes);
      cudaMalloc(&c, bytes);
      cudaMemset(a, 1, bytes);
      cudaMemset(b, 2, bytes);
      int passes = (int)(mib >= 1024 ? 3 : 2048 / mib);
      for (int k : {2, 4}) {
        dim3 g(nsm * k), blk(256);
        if (mode == 0) kern<0><<<g, blk>>>(a, b, c, nvec, 1);
        else kern<1><<<g, blk>>>(a, b, c, nvec, 1);
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0);
        if (mode == 0) kern<0><<<g, blk>>>(a, b, c, nvec, passes);
        else kern<1><<<g, blk>>>(a, b, c, nvec, passes);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        double touched = (double)bytes * (mode == 0 ? 2 : 3) * passes;
        printf("%s working set %4ld MiB x %d streams, %d CTA/SM: %.0f GB/s touched\n", mode == 0 ? "copy" : "rrs ",
               mib, mode == 0 ? 2 : 3, k, touched / (ms * 1e-3) / 1e9);
        fflush(stdout);
      }
      cudaFree(a);
      cudaFree(b);
      cudaFree(c);
    }
  }
  return 0;
}
