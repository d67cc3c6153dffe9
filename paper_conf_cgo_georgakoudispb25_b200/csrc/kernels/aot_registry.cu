// aot_registry.cu -- proteus_aot_function(entry, &fn): the generic (nvcc, sm_100a)
// CUfunction of each workload kernel, for proteus_register_kernel(..., generic_fn).
#include <cstring>

extern "C" {
int proteus_aot_get_daxpy(void**);
int proteus_aot_get_adam_step(void**);
int proteus_aot_get_stencil4(void**);
int proteus_aot_get_stencil4_smem(void**);
int proteus_aot_get_xs_lookup(void**);
int proteus_aot_get_micro_column(void**);

// Returns 0 on success, a cudaError_t value on a runtime failure, -1 if unknown.
int proteus_aot_function(const char* entry, void** fn) {
    struct { const char* name; int (*get)(void**); } table[] = {
        {"daxpy", proteus_aot_get_daxpy},
        {"adam_step", proteus_aot_get_adam_step},
        {"stencil4", proteus_aot_get_stencil4},
        {"stencil4_smem", proteus_aot_get_stencil4_smem},
        {"xs_lookup", proteus_aot_get_xs_lookup},
        {"micro_column", proteus_aot_get_micro_column},
    };
    for (auto& t : table)
        if (std::strcmp(t.name, entry) == 0) return t.get(fn);
    *fn = nullptr;
    return -1;
}
}
