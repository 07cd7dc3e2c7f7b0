// Kernel table: one interpreter instantiation per (datatype, reduction op), plus
// copy-only instantiations per element size for programs without reduce instructions.
#pragma once
namespace msccl {
const void* interpreterKernel(int dtype, int op);  // op 0..3 = sum/prod/max/min
const void* copyKernel(int elemBytes);             // programs with no reduction
}  // namespace msccl
