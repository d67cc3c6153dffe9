// globals_demo.cu -- device-global linking (the paper's __jit_register_var, PAPER.md:1
// §3.2-3.3 P@19299-21805): "references to device global variables in JIT code must be
// linked to the same memory the AOT module uses so that AOT and JIT kernels share
// state".  None of the four workloads has a __device__ global, so this kernel exists to
// exercise the mechanism: y = scale * y + bias with `scale` read from a device global,
// and the number of processed elements added to a device-global counter.
//
// Parameters (1-based): 1 y  2 n  3 bias.   Annotated: 2, 3.
// Globals: proteus_demo_scale (double), proteus_demo_count (unsigned long long [1]),
// exported from the AOT build (proteus_aot_global) and bound to JIT specializations with
// proteus_kernel_bind_global; unbound, a specialization uses its own module's copies.
#include "proteus_device.h"

__device__ double proteus_demo_scale;
__device__ unsigned long long proteus_demo_count[1];
#ifndef PROTEUS_GLOBAL_proteus_demo_scale
#define PROTEUS_GLOBAL_proteus_demo_scale proteus_demo_scale
#endif
#ifndef PROTEUS_GLOBAL_proteus_demo_count
#define PROTEUS_GLOBAL_proteus_demo_count proteus_demo_count
#endif

extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void scale_count(double* __restrict__ y, long long n_rt, double bias_rt) {
    const long long n = PROTEUS_SPEC(2, n_rt);
    const double bias = PROTEUS_SPEC(3, bias_rt);
    const double s = PROTEUS_GLOBAL_proteus_demo_scale;
    const long long stride = (long long)PROTEUS_GRIDDIM_X * PROTEUS_BLOCKDIM_X;
    unsigned long long mine = 0;
    for (long long i = (long long)blockIdx.x * PROTEUS_BLOCKDIM_X + threadIdx.x; i < n; i += stride) {
        y[i] = s * y[i] + bias;
        ++mine;
    }
    if (mine) atomicAdd(&PROTEUS_GLOBAL_proteus_demo_count[0], mine);
}
