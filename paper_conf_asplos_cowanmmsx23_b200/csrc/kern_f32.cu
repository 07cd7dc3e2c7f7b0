// Interpreter instantiations for DT_F32 (see interp.cuh).
#include "interp.cuh"
namespace msccl {
template __global__ void mscclInterpreter<DT_F32, R_SUM>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_F32, R_PROD>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_F32, R_MAX>(const __grid_constant__ KernelArgs);
template __global__ void mscclInterpreter<DT_F32, R_MIN>(const __grid_constant__ KernelArgs);
const void* kernel_F32(int op) {
  switch (op) {
    case R_SUM: return (const void*)mscclInterpreter<DT_F32, R_SUM>;
    case R_PROD: return (const void*)mscclInterpreter<DT_F32, R_PROD>;
    case R_MAX: return (const void*)mscclInterpreter<DT_F32, R_MAX>;
    case R_MIN: return (const void*)mscclInterpreter<DT_F32, R_MIN>;
  }
  return nullptr;
}
}  // namespace msccl
