/* proteus_testing.h -- test hooks of libproteus (CPU-only unit tests of the cache
 * state machine).  Not part of the product API: exported by libproteus_testing.so (which
 * links libproteus.so), not by libproteus.so itself.
 *
 * The fake backend replaces NVRTC + the CUDA driver: "compiling" returns the bytes
 * "FAKECUBIN\n" followed by the exact specialized source, "loading" returns a handle,
 * and "launching" records the call.  It lets the key/cache/async logic of §3.3
 * (P@24205-26536) run on a host with no GPU.
 */
#ifndef PROTEUS_TESTING_H
#define PROTEUS_TESTING_H
#include "proteus.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Select the backend for the next proteus_init (call before it, or after
 * proteus_finalize): 0 = CUDA (default), 1 = fake, 2 = fake load/launch but the real
 * NVRTC compiler (CPU-only check that specializations compile for sm_100a). */
proteus_status proteus_testing_use_fake_backend(int enable);

/* Fault injection / timing for the fake backend:
 *   fail_compile      1 = every compile fails with a log message
 *   compile_delay_ms  each compile sleeps this long (exercises async + dedupe) */
proteus_status proteus_testing_fake_control(int fail_compile, int compile_delay_ms);
/*   load_delay_ms     each module load sleeps this long after creating the module */
proteus_status proteus_testing_fake_load_delay(int load_delay_ms);

typedef struct {
    uint64_t compiles;           /* backend compile calls                               */
    uint64_t loads;              /* backend load calls                                  */
    uint64_t spec_launches;      /* launches of loaded (specialized) functions          */
    uint64_t generic_launches;   /* launches of the registered generic_fn               */
    void* last_fn;               /* function of the last launch                          */
    unsigned last_grid[3], last_block[3], last_shmem;
    unsigned last_attrs;         /* PROTEUS_LAUNCH_* bits of the last launch             */
    uint64_t unloads;            /* backend unload calls with a module                  */
    uint64_t bad_unloads;        /* unloads of a module that was not loaded (double)    */
    uint64_t live_modules;       /* loaded and not unloaded                              */
    uint64_t ir_compiles;        /* compile_ltoir calls (PROTEUS_F_IR)                   */
    uint64_t links;              /* link_ltoir calls                                     */
} proteus_fake_counts_t;

proteus_status proteus_testing_fake_counts(proteus_fake_counts_t* out);

#ifdef __cplusplus
}
#endif
#endif
