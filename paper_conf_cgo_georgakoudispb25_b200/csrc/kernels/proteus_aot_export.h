// proteus_aot_export.h -- host glue for the nvcc (AOT, generic) build only.
// PROTEUS_AOT_EXPORT(k) defines extern "C" int proteus_aot_get_<k>(void** fn) returning
// the CUfunction of the nvcc-compiled kernel k (cudaGetFuncBySymbol), so libproteus can
// launch the generic AOT variant with cuLaunchKernel.  Never seen by NVRTC.
#pragma once
#include <cuda_runtime.h>

// PROTEUS_AOT_EXPORT_GLOBAL(g) defines extern "C" int proteus_aot_global_<g>(void** p):
// the device address of the AOT module's __device__ global g (cudaGetSymbolAddress), to
// be bound to JIT specializations (proteus_kernel_bind_global).
#define PROTEUS_AOT_EXPORT_GLOBAL(g)                                        \
    extern "C" int proteus_aot_global_##g(void** p) {                       \
        return static_cast<int>(cudaGetSymbolAddress(p, g));                \
    }

#define PROTEUS_AOT_EXPORT(k)                                               \
    extern "C" int proteus_aot_get_##k(void** fn) {                         \
        cudaFunction_t f = nullptr;                                         \
        cudaError_t e = cudaGetFuncBySymbol(&f, reinterpret_cast<const void*>(&k)); \
        *fn = reinterpret_cast<void*>(f);                                   \
        return static_cast<int>(e);                                         \
    }
