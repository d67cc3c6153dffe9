// daxpy.cu -- the paper's running example (§3.1, Figure 2, P@12138-12857):
// y = a x + y, annotated "jit", 1, 2 (specialize on the scaling factor a and the vector
// size N).  Smoke test of the end-to-end specialization path.
#include "proteus_device.h"

extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void daxpy(double a_rt, long long n_rt, const double* __restrict__ x, double* __restrict__ y) {
    const double a = PROTEUS_SPEC(1, a_rt);
    const long long n = PROTEUS_SPEC(2, n_rt);
    const long long stride = (long long)PROTEUS_GRIDDIM_X * PROTEUS_BLOCKDIM_X;
    for (long long i = (long long)blockIdx.x * PROTEUS_BLOCKDIM_X + threadIdx.x; i < n; i += stride)
        y[i] = a * x[i] + y[i];
}
