// sw_fill16_patch.cu -- the packed Stage-1 kernels built with magic
// instruction immediates for the gap penalties (SWB_PATCH, sw_fill16.cuh).
// Compiled to a cubin that is embedded in libcudalign_b200.so; at run time
// sw_api.cu replaces the magic immediates with the call's -G_ext / -G_first
// encodings and loads the patched image (cudaLibraryLoadData).  An add with an
// immediate reads one register instead of three, which is what the packed
// cell update is bound by.  The build compiles this file twice
// with two magic sets and requires identical SASS up to the magic words
// (tools/patch_check.py): no constant derived from a magic can hide in the code.
// The int32 kernel is not patched: its faster H form compiles to
// magic-dependent code.
#define SWB_PATCH 1
#include "sw_fill16.cuh"

namespace swb {
// the packed geometries of the variant table (sw_api.cu variant_for)
template __global__ void sw_fill16_kernel<4, 64, false, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<12, 64, false, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<14, 64, false, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<15, 64, false, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<16, 64, true, 8, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<4, 64, false, 16, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<4, 64, true, 16, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<4, 64, false, 15, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 16, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<16, 64, true, 16, false>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 17, false>(const __grid_constant__ FillArgs);
// the GEN instantiations (generic special rows): variants 0, 1, 8, 10, 13, 14
template __global__ void sw_fill16_kernel<4, 64, false, 8, false, true, true>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 8, false, true, true>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<4, 64, false, 16, false, true, true>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 16, false, true, true>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<4, 64, false, 15, false, true, true>(const __grid_constant__ FillArgs);
template __global__ void sw_fill16_kernel<8, 64, false, 17, false, true, true>(const __grid_constant__ FillArgs);
// the reverse pass (global mode), variant 10's geometry
template __global__ void sw_fill16_kernel<8, 64, false, 16, false, false>(const __grid_constant__ FillArgs);
// Stage-2 partitions (global mode with matching), variant 1's geometry
template __global__ void sw_fill16_kernel<8, 64, false, 8, false, false>(const __grid_constant__ FillArgs);
}  // namespace swb
