/* proteus.h -- C ABI of libproteus, the B200 runtime-specialization library.
 *
 * The library executes GPU kernels specialized at launch time: annotated scalar
 * arguments and the launch dimensions are folded into the kernel source as
 * compile-time constants, the result is compiled once for sm_100a with NVRTC, cached
 * in memory and on disk under a hash of the specialization key, and dispatched with
 * cuLaunchKernel.  It follows PAPER.md:1 (Georgakoudis et al., "Proteus", CGO '25):
 *   annotate("jit", i1, i2, ...) with 1-based argument indices  ........ §3.1 P@12394-12699
 *   __jit_launch_kernel(module id, symbol, grid, block, shmem, stream,
 *                       annotated values)  ............................ §3.2 P@18812-19086
 *   runtime constant folding (RCF) + launch bounds (LB) ................ §3.3 P@21805-23412
 *   hash of (module id, symbol, specialized values, launch bounds),
 *   in-memory cache fed by a persistent per-file cache ................. §3.3 P@24205-26536
 * Readings where the paper is silent are listed in DESIGN.md ("Readings").
 *
 * Conventions for every entry point:
 *   - returns proteus_status; PROTEUS_OK == 0.  Nothing aborts or throws across the
 *     ABI; on failure proteus_last_error() holds a thread-local message.
 *   - thread-safe.  Strings and arrays passed in are copied; nothing passed in is
 *     retained by pointer except `generic_fn` (borrowed, must outlive the kernel)
 *     and `stream` (borrowed for the call).
 *   - device memory belongs to the caller; modules, cubins and cache files belong to
 *     the library.
 *   - the library uses the device's PRIMARY context (the one the CUDA runtime and
 *     PyTorch use) and loads libcuda.so.1 / libnvrtc.so.12 with dlopen at
 *     proteus_init, so this .so loads (and the non-launch API works) on a host
 *     without a GPU.
 */
#ifndef PROTEUS_H
#define PROTEUS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    PROTEUS_OK = 0,
    PROTEUS_E_INVALID = 1,   /* bad argument (index out of range, pointer annotated, ...) */
    PROTEUS_E_NOT_INIT = 2,  /* proteus_init not called / after proteus_finalize        */
    PROTEUS_E_CUDA = 3,      /* driver error (message has the CUresult string)           */
    PROTEUS_E_COMPILE = 4,   /* NVRTC failure and no generic fallback (message = log)    */
    PROTEUS_E_IO = 5,        /* cache directory unusable                                 */
    PROTEUS_E_NOMEM = 6
} proteus_status;

/* Kernel parameter types.  Only scalar types may be annotated (the paper folds
 * scalar arguments, P@40817).  PROTEUS_OPAQUE marks a by-value parameter of any
 * other size (e.g. a CUtensorMap); it is forwarded but never keyed or folded. */
typedef enum {
    PROTEUS_I32 = 1,
    PROTEUS_U32 = 2,
    PROTEUS_I64 = 3,
    PROTEUS_U64 = 4,
    PROTEUS_F32 = 5,
    PROTEUS_F64 = 6,
    PROTEUS_PTR = 7,
    PROTEUS_OPAQUE = 8
} proteus_type;

/* Specialization flags.  RCF/LB/FOLD_DIMS select what is folded (the paper's
 * None / LB / RCF / LB+RCF ablation, P@39538-40272; FOLD_DIMS also folds gridDim and
 * blockDim, north_star).  They and LINEINFO enter the key; DISK and TRACE do not. */
enum {
    PROTEUS_F_RCF = 1,
    PROTEUS_F_LB = 2,
    PROTEUS_F_FOLD_DIMS = 4,
    PROTEUS_F_DISK = 8,
    PROTEUS_F_TRACE = 16,
    PROTEUS_F_LINEINFO = 32, /* NVRTC -lineinfo (ncu source views); off by default: ~15% of
                                a compile.  In the key (cubins differ).  Env PROTEUS_LINEINFO=1 */
    PROTEUS_F_IR = 64        /* IR-level specialization (the paper's IR
                                folding P@21805-22851, P@26536-27018): the kernel is compiled
                                ONCE per (kernel, block dims, minBlocks) to LTO-IR with the
                                annotated values and grid dims as extern device constants;
                                each key then compiles only a constants module and links the
                                two with nvJitLink -lto, whose optimizer folds the constants.
                                Same folding as RCF/FOLD_DIMS (block dims and launch bounds
                                are literals of the kernel IR).  In the key.  A NaN annotated
                                value takes the source path.  Env PROTEUS_IR=1 */
};

typedef struct {
    int device;              /* CUDA ordinal; -1 = the calling thread's current device     */
    const char* cache_dir;   /* NULL: $PROTEUS_CACHE_DIR or ./.proteus-cache; copied         */
    unsigned flags;          /* default RCF|LB|FOLD_DIMS|DISK                               */
    int async_workers;       /* 0 = compile synchronously on a miss (the paper's behaviour)  */
    int min_blocks_per_sm;   /* launch-bounds minBlocks; paper default 1 (P@23207)          */
    /* Cache management (the paper's planned LRU + size caps, §3.4 P@26536-27373):       */
    uint64_t max_entries;    /* in-memory specializations per device; 0 = unlimited; LRU    */
    uint64_t max_disk_bytes; /* persistent cache bytes; 0 = unlimited; least-recently used  */
                             /* files (mtime, bumped on every disk hit) are deleted first   */
} proteus_config;

typedef struct proteus_kernel_s* proteus_kernel;   /* opaque; valid until proteus_finalize */

typedef struct {
    uint64_t launches;          /* proteus_launch calls that launched something             */
    uint64_t mem_hits;          /* in-memory cache hits (level 1, P@24805)                  */
    uint64_t disk_hits;         /* misses served from the persistent cache (level 2)        */
    uint64_t misses;            /* in-memory misses (= disk_hits + compiles + failures)     */
    uint64_t compiles;          /* successful NVRTC compilations                            */
    uint64_t compile_failures;
    uint64_t generic_launches;  /* launches of the AOT generic kernel (async miss/failure)  */
    uint64_t inflight;          /* async compilations queued or running now                 */
    uint64_t entries;           /* specializations resident in memory                       */
    uint64_t cubin_bytes;       /* sum of resident cubin sizes (Table 3 analogue)           */
    uint64_t disk_bytes_written;
    uint64_t disk_rejects;      /* corrupt / mismatched cache files ignored                 */
    double compile_ms_total;
    double compile_ms_max;
    double load_ms_total;       /* disk read + cuModuleLoadData                             */
    double disk_write_ms_total; /* persistent-cache writes (temp file + rename)             */
    uint64_t evictions;         /* in-memory entries evicted (LRU, max_entries)             */
    uint64_t disk_evictions;    /* cache files deleted to honour max_disk_bytes             */
    uint64_t ir_compiles;       /* PROTEUS_F_IR: kernel LTO-IR compilations (once per kernel,
                                   block dims and minBlocks, process-wide)                  */
    double ir_ms_total;         /* their NVRTC time (also counted in the compile_ms_total of
                                   the miss that triggered each)                            */
} proteus_cache_stats_t;

/* Fill *out with the defaults, then apply environment overrides:
 *   PROTEUS_CACHE_DIR, PROTEUS_DISK_CACHE=0|1, PROTEUS_ASYNC=<workers>,
 *   PROTEUS_SPECIALIZE=none|lb|rcf|all, PROTEUS_FOLD_DIMS=0|1, PROTEUS_MIN_BLOCKS=<n>,
 *   PROTEUS_TRACE=0|1 (one JSON line per miss on stderr), PROTEUS_LINEINFO=0|1,
 *   PROTEUS_IR=0|1 (IR-level specialization, PROTEUS_F_IR),
 *   PROTEUS_CACHE_MAX_ENTRIES=<n>, PROTEUS_DISK_MAX_MB=<MiB>. */
proteus_status proteus_config_default(proteus_config* out);

/* Retain the primary context of the device, open/create the cache directory, start
 * the worker pool, and warm NVRTC on a background thread.  cfg == NULL means
 * proteus_config_default().  Idempotent: a second call with the library already
 * initialised only initialises a not-yet-seen device. */
proteus_status proteus_init(const proteus_config* cfg);

/* Register a kernel (the analogue of annotate("jit", ...), P@12394).
 *   entry         extern "C" __global__ symbol in cuda_source
 *   cuda_source   NVRTC-compilable text; may #include "proteus_device.h" (embedded)
 *   options       extra NVRTC options separated by spaces (e.g. "-fmad=false"), or NULL;
 *                 they must match the options of the nvcc build of generic_fn
 *   arg_types     nargs entries, in parameter order
 *   annotated_idx n_annotated 1-based indices (<= 32) of scalar parameters to fold, in
 *                 any order; duplicates, pointers and out-of-range indices are rejected
 *                 with PROTEUS_E_INVALID
 *   generic_fn    CUfunction of the nvcc-built (AOT sm_100a) generic kernel or NULL;
 *                 launched while an async compile is in flight or if compilation fails
 * kernel_id = FNV-1a-64(source 0 entry 0 options 0 toolkit 0 arch). */
proteus_status proteus_register_kernel(const char* entry, const char* cuda_source,
                                       const char* options, const proteus_type* arg_types,
                                       int nargs, const int* annotated_idx, int n_annotated,
                                       void* generic_fn, proteus_kernel* out);

/* Per-kernel launch-bounds minBlocks hint (0 = the config's min_blocks_per_sm).  The paper
 * sets max threads per block and leaves minBlocks at 1 (P@23207); on sm_100a a larger
 * minBlocks caps registers so the specialization keeps the occupancy a latency-bound
 * kernel needs.  Part of the key.  Set before the kernel's first launch. */
proteus_status proteus_kernel_set_min_blocks(proteus_kernel k, int min_blocks);

/* Per-kernel launch attributes, applied to every later launch of k (specialized,
 * generic and proteus_launch_aot); not part of the key (the code is the same).
 *   PROTEUS_LAUNCH_PDL  programmatic dependent launch (cuLaunchKernelEx with
 *                       CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION): the
 *                       launch may begin while the previous kernel in the stream runs.
 *                       Only for kernels whose source calls PROTEUS_PDL_WAIT() before
 *                       any global-memory access (proteus_device.h); hides the launch
 *                       gap and prologue of back-to-back launches.
 * attrs with unknown bits -> PROTEUS_E_INVALID. */
enum { PROTEUS_LAUNCH_PDL = 1 };
proteus_status proteus_kernel_set_launch_attrs(proteus_kernel k, unsigned attrs);

/* Launch k (the analogue of __jit_launch_kernel, P@18812-19086).  args: nargs pointers
 * to the argument values (cuLaunchKernel convention), read only during the call.
 * stream: a CUstream / cudaStream_t (e.g. torch.cuda.current_stream().cuda_stream),
 * NULL = legacy default stream.  Asynchronous with respect to the device.
 * Hit: one hash + map lookup + cuLaunchKernel.  Miss: disk, else compile (blocking,
 * or async with the generic kernel launched meanwhile).  While an async compile of the
 * key is in flight, a launch may block the host until the GPU has completed all but the
 * last 8 generic launches of the device (or the specialization is published, which the
 * launch then uses), so a job that would be enqueued before the cubin exists still
 * switches mid-job.  Compile failure with a generic_fn: launches it, counts
 * compile_failures, returns PROTEUS_OK. */
proteus_status proteus_launch(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                              unsigned bx, unsigned by, unsigned bz, unsigned shmem_bytes,
                              void* stream, void** args);

/* Link a device global of the kernel source to existing device storage (the paper's
 * __jit_register_var + device-global linking, §3.2-3.3 P@19299-21805: JIT code must
 * refer to the SAME global as the AOT module so both share state).  Kernel-source
 * convention: the source declares the global normally and refers to it only as
 * PROTEUS_GLOBAL_<name>, defaulting to the global itself:
 *     __device__ unsigned long long hits[1];
 *     #ifndef PROTEUS_GLOBAL_hits
 *     #define PROTEUS_GLOBAL_hits hits
 *     #endif
 * A bound specialization gets
 *     #define PROTEUS_GLOBAL_<name> (*reinterpret_cast<decltype(&<name>)>(<dptr>))
 * so every use addresses dptr (typically the AOT module's storage, from
 * cudaGetSymbolAddress).  The bindings (name, address) enter the key.  name: a C
 * identifier; rebinding a name replaces its address.  Set before the kernel's first
 * launch (not synchronised with concurrent launches of k).  PROTEUS_E_INVALID for a
 * null or non-identifier argument. */
proteus_status proteus_kernel_bind_global(proteus_kernel k, const char* name, void* dptr);

/* The AOT baseline: launch k's generic_fn (the nvcc sm_100a build) directly with
 * cuLaunchKernel -- no key, no cache, no JIT.  PROTEUS_E_INVALID if k has none. */
proteus_status proteus_launch_aot(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                                  unsigned bx, unsigned by, unsigned bz, unsigned shmem_bytes,
                                  void* stream, void** args);

/* Encode a TMA tiled descriptor (a CUtensorMap, 128 bytes, written to map_out which must
 * be 64-byte aligned) with cuTensorMapEncodeTiled, for kernels that stream tiles with
 * cp.async.bulk.tensor (stencil4).  rank 1..5; dims[i] in elements, innermost first;
 * strides[i] = byte stride of dimension i+1 (rank-1 entries, multiples of 16); box[i] in
 * elements; elem_type = CUtensorMapDataType code (8 = FLOAT64).  No interleave, no
 * swizzle, L2 promotion 128 B, out-of-bounds elements read as zero.  The descriptor holds
 * `base`; the memory stays the caller's.  Pass it to the kernel as a PROTEUS_OPAQUE arg. */
proteus_status proteus_encode_tensor_map(void* map_out, int elem_type, unsigned rank,
                                         void* base, const uint64_t* dims,
                                         const uint64_t* strides, const uint32_t* box);

/* ---- peer memory for fused compute + halo kernels ---------------------------------
 * The B200-native form of the stencil's z-slab halo exchange (
 * north_star "stencil over z-slabs ... halo exchange over NVLink"): each rank's stencil
 * kernel stores its boundary planes straight into the neighbours' halo planes through
 * mapped peer memory, and the ranks order their sweeps with 32-bit flags written and
 * awaited by the GPU front end (stream memory operations), so no copy kernel or NCCL
 * call sits between two sweeps.  The paper has no multi-GPU path (it runs one GPU per
 * process, P@54134); this interface is the build's own.
 *
 * proteus_ipc_get_handle: 64-byte CUDA IPC handle (CUipcMemHandle) of the device
 *   allocation holding dptr, and *offset = dptr - allocation base.  The allocation
 *   stays the caller's (it must outlive every opened mapping).
 * proteus_ipc_open_handle: map a handle exported by ANOTHER process (same or peer GPU;
 *   peer access is enabled lazily); *base = the allocation base, so the exporter's
 *   dptr is *base + offset.  PROTEUS_E_CUDA if the driver refuses (e.g. a handle of
 *   this process).  Close with proteus_ipc_close_handle(base).
 * proteus_stream_write_u32: enqueue on `stream` a 32-bit store of `value` to dptr
 *   (local or mapped peer memory, 4-byte aligned), ordered after all prior work of the
 *   stream with a memory fence (its stores, including peer stores, are visible first).
 * proteus_stream_wait_u32: enqueue on `stream` a wait until (int32_t)(*dptr - value)
 *   >= 0; later work of the stream starts only then.  Nothing blocks the host.
 * Errors: PROTEUS_E_NOT_INIT before proteus_init, PROTEUS_E_INVALID for null or
 *   misaligned pointers, PROTEUS_E_CUDA with the driver's message otherwise. */
proteus_status proteus_ipc_get_handle(void* dptr, uint8_t* handle, uint64_t* offset);
proteus_status proteus_ipc_open_handle(const uint8_t* handle, void** base);
proteus_status proteus_ipc_close_handle(void* base);
proteus_status proteus_stream_write_u32(void* stream, void* dptr, uint32_t value);
proteus_status proteus_stream_wait_u32(void* stream, void* dptr, uint32_t value);

/* Counters of device `device` (-1 = current). */
proteus_status proteus_cache_stats(int device, proteus_cache_stats_t* out);
/* Drop the in-memory level (unloads modules; waits for in-flight compiles) and/or
 * delete this library's files from the cache directory.  Counters are reset when
 * memory != 0. */
proteus_status proteus_cache_clear(int device, int memory, int disk);
/* Block until no asynchronous compilation is queued or running. */
proteus_status proteus_wait_idle(void);
/* Join workers, unload every module, release primary contexts.  All handles die. */
proteus_status proteus_finalize(void);
const char* proteus_last_error(void);

/* ---- introspection (tests, ncu/SASS evidence, bench) ---------------------------- */
/* kernel_id, and the toolkit / arch strings that entered it. */
proteus_status proteus_kernel_info(proteus_kernel k, uint64_t* kernel_id, char* toolkit,
                                   size_t toolkit_cap, char* arch, size_t arch_cap);
/* The key bytes and hash the launch with these arguments would use (no launch). */
proteus_status proteus_key(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                           unsigned bx, unsigned by, unsigned bz, void** args,
                           uint8_t* buf, size_t cap, size_t* len, uint64_t* hash);
/* The exact NVRTC input (prelude + source) for that specialization.  With PROTEUS_F_IR:
 * the constants module, the line "//@@proteus-ir-kernel@@", then the kernel translation
 * unit (values and grid dims as extern device constants), i.e. both NVRTC inputs. */
proteus_status proteus_specialized_source(proteus_kernel k, unsigned gx, unsigned gy,
                                          unsigned gz, unsigned bx, unsigned by,
                                          unsigned bz, void** args, char* buf, size_t cap,
                                          size_t* len);
/* Start compiling (or loading from the persistent cache) the specialization that a
 * launch of these dims and args would use, on the background worker pool, and return at
 * once (the paper compiles at the first launch, P@13896-14499; this lets a program
 * overlap the compile with its own set-up).  A later proteus_launch of the same key waits
 * for it (async_workers == 0) or runs the generic kernel meanwhile (async mode).  With
 * async_workers == 0 the library starts 4 workers on the first prefetch.  No-op when the
 * specialization is already resident, compiling or failed.  proteus_wait_idle() waits
 * for every queued prefetch. */
proteus_status proteus_prefetch(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                                unsigned bx, unsigned by, unsigned bz, void** args);
/* Compile (or fetch from cache) that specialization without launching; copies the
 * cubin out (buf may be NULL to query *len) and reports the CUfunction.
 * *state: 1 = specialized cubin ready, 2 = compile failed. */
proteus_status proteus_get_specialization(proteus_kernel k, unsigned gx, unsigned gy,
                                          unsigned gz, unsigned bx, unsigned by,
                                          unsigned bz, void** args, void** fn, int* state,
                                          uint8_t* buf, size_t cap, size_t* len);

#ifdef __cplusplus
}
#endif
#endif /* PROTEUS_H */
