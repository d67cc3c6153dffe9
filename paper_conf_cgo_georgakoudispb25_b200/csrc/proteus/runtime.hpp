// runtime.hpp -- internal declarations of libproteus (not installed).
//
// Layering (DESIGN.md §"Runtime"):
//   proteus.cpp   C ABI, per-device state, hit/miss state machine, async worker pool
//   key.cpp       specialization key bytes + FNV-1a-64 (§3.3 P@24205-24805)
//                 and the RCF/LB prelude with bit-exact literals (P@21805-23412)
//   disk_cache.cpp persistent level "cache-jit-<hash>" (P@25405-26536)
//   backend_cuda.cpp compile/load/launch: NVRTC + the CUDA driver via dlopen
//   ../proteus_testing/  the fake backend and the proteus_testing_* hooks: a separate
//                  library (libproteus_testing.so) that installs a backend factory
//                  through set_backend_factory(); the product library has no test code
#pragma once

#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <memory>
#include <mutex>
#include <shared_mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "proteus.h"

namespace proteus {

// ---------------------------------------------------------------- backend interface
struct LaunchDims {
    unsigned g[3];
    unsigned b[3];
    unsigned attrs = 0;   // PROTEUS_LAUNCH_* bits (not part of the key)
};

class Backend {
public:
    virtual ~Backend() = default;
    // One-time global setup (dlopen, cuInit).  Returns false + message on failure.
    virtual bool init(std::string* err) = 0;
    // Primary context of `device` (retained); device < 0 = current.
    virtual bool device_open(int device, int* ordinal, void** ctx, std::string* err) = 0;
    virtual void device_close(int ordinal, void* ctx) = 0;
    // Device of the calling thread's current context, or -1 if none.
    virtual int current_device() = 0;
    // The calling thread's current context (nullptr if none): one cheap driver call.
    virtual void* current_context() = 0;
    // Make ctx current on the calling thread (worker threads).
    virtual bool make_current(void* ctx, std::string* err) = 0;
    virtual std::string toolkit() = 0;           // e.g. "nvrtc-12.9/proteus-1/<hdr>"
    virtual std::string arch(int ordinal) = 0;   // e.g. "sm_100a"
    // Source -> cubin.  opts are complete NVRTC options; log receives diagnostics.
    virtual bool compile(const std::string& src, const std::string& name,
                         const std::vector<std::string>& opts, std::string* cubin,
                         std::string* log) = 0;
    virtual bool load(const std::string& cubin, const std::string& entry, void** module,
                      void** fn, std::string* err) = 0;
    virtual void unload(void* module) = 0;
    virtual bool launch(void* fn, const LaunchDims& d, unsigned shmem, void* stream,
                        void** args, std::string* err) = 0;
    // IR-level specialization (PROTEUS_F_IR): source -> LTO-IR (NVRTC -dlto), and LTO-IR
    // modules -> one cubin (nvJitLink -lto).  Unsupported by default.
    virtual bool compile_ltoir(const std::string& src, const std::string& name,
                               const std::vector<std::string>& opts, std::string* ir,
                               std::string* log) {
        (void)src; (void)name; (void)opts; (void)ir;
        *log = "LTO-IR compilation is not supported by this backend";
        return false;
    }
    virtual bool link_ltoir(const std::vector<const std::string*>& irs,
                            const std::vector<std::string>& opts, std::string* cubin,
                            std::string* log) {
        (void)irs; (void)opts; (void)cubin;
        *log = "nvJitLink is not supported by this backend";
        return false;
    }
    // A kernel registered with this generic (AOT) function (test backends count launches).
    virtual void note_generic(void* fn) { (void)fn; }
    // true: the backend compiles with the real NVRTC and is worth warming at init.
    virtual bool real_compiler() { return true; }
    // Optional warm-up (first NVRTC call initialises ~250 ms of state).
    virtual void warm() {}
    // Wait for all work of ctx (before unloading evicted modules).
    virtual void synchronize(void* ctx) {}
    // cuTensorMapEncodeTiled (see proteus_encode_tensor_map).
    virtual bool encode_tensor_map(void* out, int elem_type, unsigned rank, void* base,
                                   const uint64_t* dims, const uint64_t* strides,
                                   const uint32_t* box, std::string* err) = 0;
    // Peer memory for fused compute + halo kernels (proteus_ipc_*, proteus_stream_*_u32).
    // handle: 64 bytes (CUipcMemHandle) of the allocation holding dptr; *offset = dptr -
    // allocation base.  open maps a handle exported by another process (base address).
    virtual bool ipc_get_handle(void* dptr, void* handle, uint64_t* offset, std::string* err) {
        *err = "peer memory is not supported by this backend";
        return false;
    }
    virtual bool ipc_open_handle(const void* handle, void** base, std::string* err) {
        *err = "peer memory is not supported by this backend";
        return false;
    }
    virtual bool ipc_close_handle(void* base, std::string* err) {
        *err = "peer memory is not supported by this backend";
        return false;
    }
    // Events (async-compile throttle): create in the current context (nullptr when the
    // backend has none: no throttling), record on a stream, query (1 = complete, 0 = not
    // yet, -1 = error), destroy.
    virtual void* event_create() { return nullptr; }
    virtual bool event_record(void* ev, void* stream) { return false; }
    virtual int event_query(void* ev) { return 1; }
    virtual void event_destroy(void* ev) {}
    // Stream memory operations: a 32-bit write ordered after all prior work of the stream
    // (with a memory fence), and a wait until (int32_t)(*dptr - value) >= 0.
    virtual bool stream_write_u32(void* stream, void* dptr, uint32_t value, std::string* err) {
        *err = "stream memory operations are not supported by this backend";
        return false;
    }
    virtual bool stream_wait_u32(void* stream, void* dptr, uint32_t value, std::string* err) {
        *err = "stream memory operations are not supported by this backend";
        return false;
    }
};

std::unique_ptr<Backend> make_cuda_backend();
std::unique_ptr<Backend> make_nvrtc_only_backend();   // compile() only, no driver

// Backend used by the next proteus_init (nullptr = the CUDA backend).  The only hook the
// product library offers its test library (not part of the C ABI); fails once initialised.
using BackendFactory = std::unique_ptr<Backend> (*)();
bool set_backend_factory(BackendFactory f);

// ---------------------------------------------------------------- key + prelude
uint64_t fnv1a64(const void* data, size_t len, uint64_t h = 0xcbf29ce484222325ull);
// Hash of the key bytes for the in-memory map only (8 bytes per step, ~4x cheaper than the
// byte-wise FNV-1a on a ~60-100 B key); the FNV-1a-64 of the key still names the disk file.
uint64_t key_map_hash(const uint8_t* data, size_t len);
size_t type_size(proteus_type t);

struct KernelDesc {
    std::string entry, source, options;
    std::vector<proteus_type> types;
    std::vector<int> annotated;        // 0-based, ascending
    void* generic_fn = nullptr;
    int min_blocks = 0;                // launch-bounds minBlocks hint; 0 = config default
    unsigned launch_attrs = 0;         // PROTEUS_LAUNCH_* bits applied to every launch
    uint64_t version = 0;              // bumped by every change that alters the key
    // device globals linked to the AOT build's storage (proteus_kernel_bind_global),
    // sorted by name: (name, device address)
    std::vector<std::pair<std::string, uint64_t>> globals;
    uint64_t kernel_id = 0;
    std::string toolkit, arch;
};

// Key bytes of DESIGN.md §"Specialization key" into out (cleared first).
void build_key(const KernelDesc& k, unsigned key_flags, unsigned min_blocks,
               const LaunchDims& d, void** args, std::vector<uint8_t>* out);
// Literal that reproduces the value's bits exactly in CUDA C++.
std::string literal_for(proteus_type t, const void* value);
// Symbol of a specialization of `entry` in its cubin: "<entry>__jit" in the product mode,
// "<entry>__jit_<mode>" in the ablation modes (none, lb, v = values, d = dims, ...) and
// "..._ir" on the IR path; the generic AOT kernel keeps the plain name, so ncu launch
// lists tell the variants apart.
std::string jit_symbol(const std::string& entry, unsigned key_flags);
// PROTEUS_F_IR: specialized_source() returns "<constants TU>" kIrSplit "<kernel TU>".
extern const char* const kIrSplit;
// Prelude + #line + source, as handed to NVRTC.
std::string specialized_source(const KernelDesc& k, unsigned key_flags, unsigned min_blocks,
                               const LaunchDims& d, void** args);
extern const char* const kDeviceHeader;       // proteus_device.h text (embedded)
extern const char* const kDeviceHeaderName;   // "proteus_device.h"

// ---------------------------------------------------------------- persistent cache
std::string cache_file_path(const std::string& dir, uint64_t hash);
// Returns true and fills cubin if the file exists, is intact and holds exactly `key`.
// *reject is set when a file existed but was corrupt or mismatched.
bool disk_read(const std::string& dir, uint64_t hash, const std::vector<uint8_t>& key,
               std::string* cubin, bool* reject);
// Atomic write (temp file + rename).  Returns bytes written (0 on failure).
size_t disk_write(const std::string& dir, uint64_t hash, const std::vector<uint8_t>& key,
                  const std::string& cubin);
// Cross-process compile claim (ranks of one box sharing the directory): a lock file
// cache-jit-<hash>.lock created atomically with its owner's token "pid host nonce".
// disk_claim: 1 = this process compiles the key (*token set; call disk_release with it
// afterwards), 0 = another process holds a live claim, -1 = no lock could be created
// (compile anyway).  Claims of dead processes on this host are taken over at once.  disk_wait_claim: wait until the claim is released
// or goes stale or timeout_ms passes; true when the cubin file exists by then.
int disk_claim(const std::string& dir, uint64_t hash, std::string* token);
void disk_release(const std::string& dir, uint64_t hash, const std::string& token);
bool disk_wait_claim(const std::string& dir, uint64_t hash, double timeout_ms);
int disk_clear(const std::string& dir);
// Delete least-recently-used cache files (oldest mtime) until the directory holds at most
// max_bytes of cache-jit-* files; `keep` is never deleted.  Returns files deleted.
int disk_enforce_cap(const std::string& dir, uint64_t max_bytes, const std::string& keep);
bool ensure_dir(const std::string& dir, std::string* err);

}  // namespace proteus
