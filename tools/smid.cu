// Which SM does each CTA of a co-resident (cooperative) grid land on? Prints the SM of
// blocks 0..N-1 and how many distinct SMs the first k blocks cover.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/smid_bin tools/smid.cu
#include <cstdio>
#include <set>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(256) k(int* out) {
  if (threadIdx.x == 0) {
    int s;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    out[blockIdx.x] = s;
  }
  // keep every block resident for a while so the placement is the co-resident one
  long t0 = clock64();
  while (clock64() - t0 < 2000000) {
  }
}
int main() {
  for (int n : {224, 256, 296}) {
    int* d;
    cudaMalloc(&d, n * sizeof(int));
    void* args[] = {&d};
    cudaLaunchCooperativeKernel((void*)k, dim3(n), dim3(256), args, 0, 0);
    cudaDeviceSynchronize();
    int h[1024];
    cudaMemcpy(h, d, n * sizeof(int), cudaMemcpyDeviceToHost);
    printf("grid %d: first 40 blocks -> SM:", n);
    for (int i = 0; i < 40; i++) printf(" %d", h[i]);
    std::set<int> s;
    int cov[4] = {0, 0, 0, 0};
    for (int i = 0; i < n; i++) {
      s.insert(h[i]);
      if (i == 73) cov[0] = s.size();
      if (i == 111) cov[1] = s.size();
      if (i == 147) cov[2] = s.size();
    }
    printf("\n  distinct SMs in first 74 / 112 / 148 blocks: %d / %d / %d; total %zu\n", cov[0], cov[1], cov[2], s.size());
    cudaFree(d);
  }
  return 0;
}
