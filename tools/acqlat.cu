// Latency of the flag loads the interpreter's waits use (one thread, dependent chain of
// loads of an already-set 64-bit word): volatile, relaxed.gpu, acquire.gpu, acquire.sys,
// and a fence.acq_rel.gpu. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/acqlat_bin tools/acqlat.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint64_t ldVol(const uint64_t* p) { uint64_t v; asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint64_t ldRlx(const uint64_t* p) { uint64_t v; asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint64_t ldAcqG(const uint64_t* p) { uint64_t v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint64_t ldAcqS(const uint64_t* p) { uint64_t v; asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }

template <int K>
__global__ void probe(uint64_t* flag, uint64_t* out, int iters, uint64_t zero) {
  if (threadIdx.x != 0) return;
  uint64_t s = 0;
  const uint64_t* p = flag;
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
    uint64_t v;
    if (K == 0) v = ldVol(p);
    if (K == 1) v = ldRlx(p);
    if (K == 2) v = ldAcqG(p);
    if (K == 3) v = ldAcqS(p);
    if (K == 4) { asm volatile("fence.acq_rel.gpu;" ::: "memory"); v = ldVol(p); }
    if (K == 5) { asm volatile("fence.acq_rel.sys;" ::: "memory"); v = ldVol(p); }
    s += v;
    p = flag + (v & zero);  // dependent chain (zero == 0 at run time)
  }
  long long t1 = clock64();
  out[blockIdx.x * 2] = (uint64_t)(t1 - t0);
  out[blockIdx.x * 2 + 1] = s;
}

int main() {
  uint64_t *flag, *out;
  cudaMalloc(&flag, 4096);
  cudaMalloc(&out, 4096 * 16);
  cudaMemset(flag, 0, 4096);
  const char* names[] = {"ld.volatile", "ld.relaxed.gpu", "ld.acquire.gpu", "ld.acquire.sys", "fence.acq_rel.gpu+ld", "fence.acq_rel.sys+ld"};
  const int iters = 64;
  for (int rep = 0; rep < 2; rep++) {
    for (int k = 0; k < 6; k++) {
      for (int blocks : {1, 112}) {
        switch (k) {
          case 0: probe<0><<<blocks, 32>>>(flag, out, iters, 0); break;
          case 1: probe<1><<<blocks, 32>>>(flag, out, iters, 0); break;
          case 2: probe<2><<<blocks, 32>>>(flag, out, iters, 0); break;
          case 3: probe<3><<<blocks, 32>>>(flag, out, iters, 0); break;
          case 4: probe<4><<<blocks, 32>>>(flag, out, iters, 0); break;
          case 5: probe<5><<<blocks, 32>>>(flag, out, iters, 0); break;
        }
        uint64_t h[2];
        cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
        if (rep == 1) printf("%-22s blocks %3d: %7.1f cycles per load (%.0f ns at 1.965 GHz)\n", names[k], blocks, (double)h[0] / iters, (double)h[0] / iters / 1.965);
      }
    }
  }
  return 0;
}
