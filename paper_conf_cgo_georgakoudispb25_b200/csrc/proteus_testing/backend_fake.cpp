// backend_fake.cpp -- GPU-free backend for unit tests of the cache state machine, and the
// proteus_testing_* entry points (include/proteus_testing.h).  Built into
// libproteus_testing.so, which links libproteus.so and installs this backend through
// proteus::set_backend_factory(); the product library carries none of it.
//
// "compile" returns "FAKECUBIN\n" + the exact specialized source (so tests can read
// the RCF/LB prelude back), "load" hands out a heap token per module, "launch" records
// the call.  Fault injection (compile failures, compile and load latency) is driven from
// proteus_testing.h; unloads of modules that are not loaded are counted (double unload).
// Nothing here touches CUDA.
#include <chrono>
#include <cstring>
#include <mutex>
#include <set>
#include <thread>

#include "proteus_testing.h"
#include "runtime.hpp"

namespace proteus {
namespace {

std::mutex g_mu;
int g_fail_compile = 0;
int g_delay_ms = 0;
int g_load_delay_ms = 0;
proteus_fake_counts_t g_counts{};
void* g_generic = nullptr;
std::set<void*> g_live;   // loaded, not yet unloaded modules

struct FakeModule {
    std::string entry;
    char fn_token;   // address used as the CUfunction stand-in
};

class FakeBackend final : public Backend {
public:
    explicit FakeBackend(bool with_nvrtc) {
        if (with_nvrtc) nvrtc_ = make_nvrtc_only_backend();
    }
    bool init(std::string* err) override { return nvrtc_ ? nvrtc_->init(err) : true; }
    bool device_open(int device, int* ordinal, void** ctx, std::string*) override {
        *ordinal = device < 0 ? 0 : device;
        *ctx = reinterpret_cast<void*>(0x1000 + *ordinal);
        return true;
    }
    void device_close(int, void*) override {}
    int current_device() override { return 0; }
    void* current_context() override { return reinterpret_cast<void*>(0x1000); }
    bool make_current(void*, std::string*) override { return true; }
    std::string toolkit() override { return nvrtc_ ? "fake+" + nvrtc_->toolkit() : "fake"; }
    std::string arch(int) override { return "sm_100a"; }
    bool compile(const std::string& src, const std::string& name, const std::vector<std::string>& opts,
                 std::string* cubin, std::string* log) override {
        int fail, delay;
        {
            std::lock_guard<std::mutex> g(g_mu);
            ++g_counts.compiles;
            fail = g_fail_compile;
            delay = g_delay_ms;
        }
        if (delay > 0) std::this_thread::sleep_for(std::chrono::milliseconds(delay));
        if (fail) {
            *log = "fake compile failure (injected)";
            return false;
        }
        if (nvrtc_) return nvrtc_->compile(src, name, opts, cubin, log);
        std::string o;
        for (const auto& s : opts) o += s + " ";
        *cubin = "FAKECUBIN\n// opts: " + o + "\n" + src;
        log->clear();
        return true;
    }
    bool compile_ltoir(const std::string& src, const std::string& name,
                       const std::vector<std::string>& opts, std::string* ir,
                       std::string* log) override {
        {
            std::lock_guard<std::mutex> g(g_mu);
            ++g_counts.ir_compiles;
        }
        if (nvrtc_) return nvrtc_->compile_ltoir(src, name, opts, ir, log);
        *ir = "FAKEIR\n" + src;
        log->clear();
        return true;
    }
    bool link_ltoir(const std::vector<const std::string*>& irs,
                    const std::vector<std::string>& opts, std::string* cubin,
                    std::string* log) override {
        {
            std::lock_guard<std::mutex> g(g_mu);
            ++g_counts.links;
        }
        if (nvrtc_) return nvrtc_->link_ltoir(irs, opts, cubin, log);
        std::string o;
        for (const auto& x : opts) o += x + " ";
        *cubin = "FAKECUBIN\n// nvJitLink " + o + "\n";
        for (const auto* x : irs) *cubin += *x + "\n";
        log->clear();
        return true;
    }
    bool load(const std::string& cubin, const std::string& entry, void** module, void** fn,
              std::string* err) override {
        if (!nvrtc_ && cubin.compare(0, 10, "FAKECUBIN\n") != 0) {
            *err = "fake load: not a fake cubin";
            return false;
        }
        auto* m = new FakeModule{entry, 0};
        int delay;
        {
            std::lock_guard<std::mutex> g(g_mu);
            ++g_counts.loads;
            g_live.insert(m);
            delay = g_load_delay_ms;
        }
        *module = m;   // the runtime passes &entry->module: the entry holds it from here
        *fn = &m->fn_token;
        // a delay widens the window between the load and the runtime accounting it
        // (cache_clear racing a miss)
        if (delay > 0) std::this_thread::sleep_for(std::chrono::milliseconds(delay));
        return true;
    }
    void unload(void* module) override {
        if (!module) return;
        {
            std::lock_guard<std::mutex> g(g_mu);
            ++g_counts.unloads;
            if (!g_live.erase(module)) {   // double unload: never free it twice
                ++g_counts.bad_unloads;
                return;
            }
        }
        delete static_cast<FakeModule*>(module);
    }
    void note_generic(void* fn) override {
        std::lock_guard<std::mutex> g(g_mu);
        g_generic = fn;
    }
    bool real_compiler() override { return nvrtc_ != nullptr; }
    // events: launches complete instantly, so a recorded event is always complete; the
    // objects are real so the async throttle ring runs under the sanitizer stress tests
    void* event_create() override { return new std::atomic<int>(0); }
    bool event_record(void* ev, void*) override {
        static_cast<std::atomic<int>*>(ev)->fetch_add(1);
        return true;
    }
    int event_query(void* ev) override {
        return static_cast<std::atomic<int>*>(ev)->load() >= 0 ? 1 : -1;
    }
    void event_destroy(void* ev) override { delete static_cast<std::atomic<int>*>(ev); }

    bool launch(void* fn, const LaunchDims& d, unsigned shmem, void*, void**,
                std::string*) override {
        std::lock_guard<std::mutex> g(g_mu);
        if (fn == g_generic) ++g_counts.generic_launches; else ++g_counts.spec_launches;
        g_counts.last_fn = fn;
        std::memcpy(g_counts.last_grid, d.g, sizeof d.g);
        std::memcpy(g_counts.last_block, d.b, sizeof d.b);
        g_counts.last_shmem = shmem;
        g_counts.last_attrs = d.attrs;
        return true;
    }
    bool encode_tensor_map(void* out, int, unsigned rank, void* base, const uint64_t*,
                           const uint64_t*, const uint32_t*, std::string* err) override {
        if (rank < 1 || rank > 5) {
            *err = "rank must be 1..5";
            return false;
        }
        std::memset(out, 0, 128);
        std::memcpy(out, &base, sizeof base);   // recognisable stand-in
        return true;
    }
    // Peer memory on HOST memory (CPU tests of the ABI wiring): the "handle" carries the
    // pointer itself, writes store immediately, a wait that would block is an error.
    bool ipc_get_handle(void* dptr, void* handle, uint64_t* offset, std::string*) override {
        std::memset(handle, 0, 64);
        std::memcpy(handle, "FAKEIPC", 7);
        std::memcpy(static_cast<char*>(handle) + 8, &dptr, sizeof dptr);
        *offset = 0;
        return true;
    }
    bool ipc_open_handle(const void* handle, void** base, std::string* err) override {
        if (std::memcmp(handle, "FAKEIPC", 7) != 0) {
            *err = "fake ipc: not a fake handle";
            return false;
        }
        std::memcpy(base, static_cast<const char*>(handle) + 8, sizeof *base);
        return true;
    }
    bool ipc_close_handle(void*, std::string*) override { return true; }
    bool stream_write_u32(void*, void* dptr, uint32_t value, std::string*) override {
        __atomic_store_n(static_cast<uint32_t*>(dptr), value, __ATOMIC_RELEASE);
        return true;
    }
    bool stream_wait_u32(void*, void* dptr, uint32_t value, std::string* err) override {
        const uint32_t v = __atomic_load_n(static_cast<uint32_t*>(dptr), __ATOMIC_ACQUIRE);
        if (static_cast<int32_t>(v - value) >= 0) return true;
        *err = "fake stream wait would block (value " + std::to_string(v) + " < " +
               std::to_string(value) + ")";
        return false;
    }

private:
    std::unique_ptr<Backend> nvrtc_;
};

}  // namespace

std::unique_ptr<Backend> fake_plain() { return std::make_unique<FakeBackend>(false); }
std::unique_ptr<Backend> fake_nvrtc() { return std::make_unique<FakeBackend>(true); }

}  // namespace proteus

using namespace proteus;

extern "C" {

proteus_status proteus_testing_use_fake_backend(int enable) {
    if (enable < 0 || enable > 2) return PROTEUS_E_INVALID;
    const BackendFactory f = enable == 0 ? nullptr : enable == 1 ? fake_plain : fake_nvrtc;
    return set_backend_factory(f) ? PROTEUS_OK : PROTEUS_E_INVALID;
}

proteus_status proteus_testing_fake_control(int fail_compile, int compile_delay_ms) {
    std::lock_guard<std::mutex> g(g_mu);
    g_fail_compile = fail_compile;
    g_delay_ms = compile_delay_ms;
    return PROTEUS_OK;
}

proteus_status proteus_testing_fake_load_delay(int load_delay_ms) {
    std::lock_guard<std::mutex> g(g_mu);
    g_load_delay_ms = load_delay_ms;
    return PROTEUS_OK;
}

proteus_status proteus_testing_fake_counts(proteus_fake_counts_t* out) {
    if (!out) return PROTEUS_E_INVALID;
    std::lock_guard<std::mutex> g(g_mu);
    *out = g_counts;
    out->live_modules = g_live.size();
    return PROTEUS_OK;
}

}  // extern "C"
