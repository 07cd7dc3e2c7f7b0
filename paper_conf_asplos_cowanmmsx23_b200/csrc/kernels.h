// Kernel table: one interpreter instantiation per (datatype, reduction op), plus
// copy-only instantiations per element size for programs without reduce instructions.
#pragma once
namespace msccl {
// op 0..3 sum/prod/max/min; proto 0 Simple 1 LL 2 LL128; wide: the LL / LL128 build for 2 CTAs per SM
// (the default LL / LL128 build runs 1 CTA per SM: more registers, at most 148 thread blocks)
const void* interpreterKernel(int dtype, int op, int proto, bool wide = false);
const void* copyKernel(int elemBytes, int proto, bool wide = false);  // programs with no reduction
// programs with multimem ops (reading R23; Simple protocol): separate kernel variants
const void* interpreterKernelMM(int dtype, int op);
const void* copyKernelMM(int elemBytes);
}  // namespace msccl
