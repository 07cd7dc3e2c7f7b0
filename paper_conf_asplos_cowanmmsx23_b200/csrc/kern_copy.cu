// Copy-only interpreter instantiations (AllGather / AllToAll / custom movement programs)
// and the kernel table.
#include "interp.cuh"
#include "kernels.h"
namespace msccl {
template __global__ void mscclInterpreter<DT_U8, R_COPY>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_F16, R_COPY>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_U32, R_COPY>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_U64, R_COPY>(const __grid_constant__ KernelArgs);
const void* kernel_I8(int);
const void* kernel_U8(int);
const void* kernel_I32(int);
const void* kernel_U32(int);
const void* kernel_I64(int);
const void* kernel_U64(int);
const void* kernel_F16(int);
const void* kernel_F32(int);
const void* kernel_F64(int);
const void* kernel_BF16(int);
const void* interpreterKernel(int dtype, int op) {
  switch (dtype) {
    case DT_I8: return kernel_I8(op);
    case DT_U8: return kernel_U8(op);
    case DT_I32: return kernel_I32(op);
    case DT_U32: return kernel_U32(op);
    case DT_I64: return kernel_I64(op);
    case DT_U64: return kernel_U64(op);
    case DT_F16: return kernel_F16(op);
    case DT_F32: return kernel_F32(op);
    case DT_F64: return kernel_F64(op);
    case DT_BF16: return kernel_BF16(op);
  }
  return nullptr;
}
const void* copyKernel(int elemBytes) {
  switch (elemBytes) {
    case 1: return (const void*)mscclInterpreter<DT_U8, R_COPY>;
    case 2: return (const void*)mscclInterpreter<DT_F16, R_COPY>;
    case 4: return (const void*)mscclInterpreter<DT_U32, R_COPY>;
    case 8: return (const void*)mscclInterpreter<DT_U64, R_COPY>;
  }
  return nullptr;
}
}  // namespace msccl
