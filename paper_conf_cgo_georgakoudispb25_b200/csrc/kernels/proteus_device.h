/* proteus_device.h -- device-side conventions of the Proteus specializer.
 *
 * Included by every workload kernel.  The nvcc AOT (generic) build sees no PROTEUS_*
 * definitions, so every macro below falls back to the runtime value: that build IS
 * the generic kernel.  For a JIT specialization libproteus prepends a prelude that
 * defines, §3.3 "Dynamic specialization" (P@21805-23412):
 *   PROTEUS_A<i>_OR(x)     -> the bit-exact literal of annotated argument i (1-based,
 *                             as annotate("jit", i, ...), P@12394)        [RCF]
 *   PROTEUS_BDX/BDY/BDZ, PROTEUS_GDX/GDY/GDZ -> the launch dimensions     [FOLD_DIMS]
 *   PROTEUS_LAUNCH_BOUNDS  -> __launch_bounds__(bx*by*bz, minBlocks)      [LB]
 * This header is embedded in libproteus and handed to NVRTC under this name.
 */
#ifndef PROTEUS_DEVICE_H
#define PROTEUS_DEVICE_H

#ifndef PROTEUS_LAUNCH_BOUNDS
#define PROTEUS_LAUNCH_BOUNDS
#endif

#define PROTEUS_CAT3_(a, b, c) a##b##c
#define PROTEUS_CAT3(a, b, c) PROTEUS_CAT3_(a, b, c)
/* value of 1-based kernel argument i: the folded literal if specialized, else x */
#define PROTEUS_SPEC(i, x) PROTEUS_CAT3(PROTEUS_A, i, _OR)(x)

#ifndef PROTEUS_A1_OR
#define PROTEUS_A1_OR(x) (x)
#endif
#ifndef PROTEUS_A2_OR
#define PROTEUS_A2_OR(x) (x)
#endif
#ifndef PROTEUS_A3_OR
#define PROTEUS_A3_OR(x) (x)
#endif
#ifndef PROTEUS_A4_OR
#define PROTEUS_A4_OR(x) (x)
#endif
#ifndef PROTEUS_A5_OR
#define PROTEUS_A5_OR(x) (x)
#endif
#ifndef PROTEUS_A6_OR
#define PROTEUS_A6_OR(x) (x)
#endif
#ifndef PROTEUS_A7_OR
#define PROTEUS_A7_OR(x) (x)
#endif
#ifndef PROTEUS_A8_OR
#define PROTEUS_A8_OR(x) (x)
#endif
#ifndef PROTEUS_A9_OR
#define PROTEUS_A9_OR(x) (x)
#endif
#ifndef PROTEUS_A10_OR
#define PROTEUS_A10_OR(x) (x)
#endif
#ifndef PROTEUS_A11_OR
#define PROTEUS_A11_OR(x) (x)
#endif
#ifndef PROTEUS_A12_OR
#define PROTEUS_A12_OR(x) (x)
#endif
#ifndef PROTEUS_A13_OR
#define PROTEUS_A13_OR(x) (x)
#endif
#ifndef PROTEUS_A14_OR
#define PROTEUS_A14_OR(x) (x)
#endif
#ifndef PROTEUS_A15_OR
#define PROTEUS_A15_OR(x) (x)
#endif
#ifndef PROTEUS_A16_OR
#define PROTEUS_A16_OR(x) (x)
#endif
#ifndef PROTEUS_A17_OR
#define PROTEUS_A17_OR(x) (x)
#endif
#ifndef PROTEUS_A18_OR
#define PROTEUS_A18_OR(x) (x)
#endif
#ifndef PROTEUS_A19_OR
#define PROTEUS_A19_OR(x) (x)
#endif
#ifndef PROTEUS_A20_OR
#define PROTEUS_A20_OR(x) (x)
#endif
#ifndef PROTEUS_A21_OR
#define PROTEUS_A21_OR(x) (x)
#endif
#ifndef PROTEUS_A22_OR
#define PROTEUS_A22_OR(x) (x)
#endif
#ifndef PROTEUS_A23_OR
#define PROTEUS_A23_OR(x) (x)
#endif
#ifndef PROTEUS_A24_OR
#define PROTEUS_A24_OR(x) (x)
#endif
#ifndef PROTEUS_A25_OR
#define PROTEUS_A25_OR(x) (x)
#endif
#ifndef PROTEUS_A26_OR
#define PROTEUS_A26_OR(x) (x)
#endif
#ifndef PROTEUS_A27_OR
#define PROTEUS_A27_OR(x) (x)
#endif
#ifndef PROTEUS_A28_OR
#define PROTEUS_A28_OR(x) (x)
#endif
#ifndef PROTEUS_A29_OR
#define PROTEUS_A29_OR(x) (x)
#endif
#ifndef PROTEUS_A30_OR
#define PROTEUS_A30_OR(x) (x)
#endif
#ifndef PROTEUS_A31_OR
#define PROTEUS_A31_OR(x) (x)
#endif
#ifndef PROTEUS_A32_OR
#define PROTEUS_A32_OR(x) (x)
#endif

#ifdef PROTEUS_BDX
#define PROTEUS_BLOCKDIM_X (PROTEUS_BDX)
#define PROTEUS_BLOCKDIM_Y (PROTEUS_BDY)
#define PROTEUS_BLOCKDIM_Z (PROTEUS_BDZ)
#define PROTEUS_GRIDDIM_X (PROTEUS_GDX)
#define PROTEUS_GRIDDIM_Y (PROTEUS_GDY)
#define PROTEUS_GRIDDIM_Z (PROTEUS_GDZ)
#else
#define PROTEUS_BLOCKDIM_X (blockDim.x)
#define PROTEUS_BLOCKDIM_Y (blockDim.y)
#define PROTEUS_BLOCKDIM_Z (blockDim.z)
#define PROTEUS_GRIDDIM_X (gridDim.x)
#define PROTEUS_GRIDDIM_Y (gridDim.y)
#define PROTEUS_GRIDDIM_Z (gridDim.z)
#endif

/* Multi-kernel sources wrap each kernel in
 *     #if PROTEUS_KERNEL_ENABLED(name) ... #endif
 * with PROTEUS_KERNEL_ENABLED defined by the including file as
 *     #if !defined(PROTEUS_SELECT_ENTRY) || defined(PROTEUS_ENTRY_name)
 * (the prelude defines PROTEUS_SELECT_ENTRY and PROTEUS_ENTRY_<launched entry>), so a
 * specialization compiles only the launched kernel; the nvcc build compiles them all. */

/* Programmatic dependent launch (sm_90+).  A kernel launched with PROTEUS_LAUNCH_PDL
 * (proteus_kernel_set_launch_attrs) may start while the previous kernel in its stream is
 * still running; it must execute PROTEUS_PDL_WAIT() -- which returns once that kernel
 * has completed and its memory is visible -- before its first global-memory access.
 * PROTEUS_PDL_TRIGGER() lets the next PDL launch in the stream begin (its blocks get
 * scheduled and run their prologue up to their own wait).  Both are no-ops for a launch
 * without the attribute, so generic and specialized builds carry them unconditionally. */
#define PROTEUS_PDL_WAIT() asm volatile("griddepcontrol.wait;" ::: "memory")
#define PROTEUS_PDL_TRIGGER() asm volatile("griddepcontrol.launch_dependents;" ::: "memory")

/* Opt-in device bounds checks (compile with -DPROTEUS_CHECK, e.g. as a kernel's NVRTC
 * options): PROTEUS_CHECK_IDX(i, n) traps unless 0 <= i < n, so an out-of-bounds index
 * fails the launch (CUDA_ERROR_LAUNCH_FAILED) instead of corrupting memory.  The GPU pool
 * refuses compute-sanitizer since r02at; tests/test_gpu_bounds.py runs every workload's
 * specialization with the checks on small ragged cases instead.  Off: no code. */
#ifdef PROTEUS_CHECK
#define PROTEUS_CHECK_IDX(i, n)                                                            \
    do {                                                                                   \
        if (!(static_cast<unsigned long long>(i) < static_cast<unsigned long long>(n)))    \
            __trap();                                                                      \
    } while (0)
#else
#define PROTEUS_CHECK_IDX(i, n) ((void)0)
#endif

/* 1 inside a JIT specialization (any mode), 0 in the nvcc generic build */
#ifndef PROTEUS_JIT
#define PROTEUS_JIT 0
#endif

#endif /* PROTEUS_DEVICE_H */
