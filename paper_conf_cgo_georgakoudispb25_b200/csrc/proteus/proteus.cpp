// proteus.cpp -- C ABI and the hit/miss state machine of libproteus.
//
// PAPER.md:1 §3.3 (P@20005-26536), redesigned for one process per B200:
//   * proteus_launch is the analogue of __jit_launch_kernel (§3.2, P@18812-19086).
//   * key -> per-device in-memory map keyed by key_map_hash (a word-wise hash of the key
//     bytes; level 1, "populated afresh at runtime", P@24805-25287) -> persistent file
//     named by FNV-1a-64 of the key (level 2, P@25287-26005; FNV is computed once, when
//     an entry is created) -> NVRTC.
//   * Unlike the paper (synchronous JIT, P@13896-14499) a miss may be compiled by a
//     background worker while the nvcc-built generic AOT sm_100a kernel runs
//     (north_star); the specialized kernel takes over once published.  Never a CPU
//     fallback.
// Hit path cost: relaunching a kernel's last specialization (per-thread memo) is a
// compare of the annotated values and dims plus one cuLaunchKernel; otherwise one key
// serialisation (~50-100 B), one key_map_hash pass, one shared-lock map probe + memcmp,
// one cuLaunchKernel.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <functional>
#include <memory>
#include <mutex>
#include <shared_mutex>
#include <sstream>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "runtime.hpp"

namespace proteus {

const char* const kDeviceHeaderName = "proteus_device.h";
const char* const kDeviceHeader =
#include "device_header.inc"
    ;

namespace {

constexpr unsigned kKeyFlagMask = PROTEUS_F_RCF | PROTEUS_F_LB | PROTEUS_F_FOLD_DIMS |
                                   PROTEUS_F_LINEINFO | PROTEUS_F_IR;
constexpr int kMaxDevices = 64;
constexpr int kMaxArgs = 64;
constexpr int kMaxAnnotated = 32;   // PROTEUS_A1_OR .. PROTEUS_A32_OR in proteus_device.h
constexpr const char* kLibTag = "proteus-2";   // 2: specializations named <entry>__jit

thread_local std::string t_err;

proteus_status fail(proteus_status s, const std::string& msg) {
    t_err = msg;
    return s;
}

double now_ms() {
    using namespace std::chrono;
    return duration<double, std::milli>(steady_clock::now().time_since_epoch()).count();
}

enum EntryState { kCompiling = 0, kReady = 1, kFailed = 2 };

// While a specialization compiles in the background (async mode), the generic kernel runs
// in its place -- but a host that enqueues a whole short job before the compile finishes
// would never switch.  So the host is kept at most this many generic launches ahead of the
// GPU (per device) until the cubin is published.
constexpr unsigned kAsyncAhead = 8;
// proteus_prefetch compiles on the worker pool; with async_workers == 0 it starts this many
constexpr size_t kPrefetchWorkers = 4;

struct Entry {
    std::vector<uint8_t> key;
    uint64_t hash = 0;    // FNV-1a-64 of the key: names the disk file (R-key-1)
    uint64_t mhash = 0;   // key_map_hash: the in-memory map's key
    std::atomic<int> state{kCompiling};
    void* module = nullptr;
    void* fn = nullptr;
    std::string cubin;   // kept for introspection (proteus_get_specialization)
    std::string log;     // compile log on failure
    std::atomic<uint64_t> last_use{0};   // LRU tick (max_entries)
    // module counted in the device's resident set (account_if_linked); only resident
    // modules are unloaded by eviction, cache_clear and finalize -- a module still being
    // loaded / accounted by its owner is the owner's to unload.  Guarded by D->mu.
    bool resident = false;
};

struct Device {
    int ordinal = -1;
    void* ctx = nullptr;
    std::shared_mutex mu;
    // Entries are shared: a thread that waits for, compiles or inspects an entry outside
    // the lock keeps it alive even if an eviction or cache_clear unlinks it meanwhile
    // (launches only ever use entries found in the map under the lock).
    std::unordered_map<uint64_t, std::vector<std::shared_ptr<Entry>>> map;
    std::mutex wait_mu;
    std::condition_variable wait_cv;
    // counters
    std::atomic<uint64_t> launches{0}, mem_hits{0}, disk_hits{0}, misses{0}, compiles{0},
        compile_failures{0}, generic_launches{0}, inflight{0}, entries{0}, cubin_bytes{0},
        disk_bytes_written{0}, disk_rejects{0}, evictions{0}, disk_evictions{0},
        ir_compiles{0};
    std::atomic<uint64_t> tick{0};
    // async-compile throttle: events recorded after the last kAsyncAhead generic launches
    std::mutex ev_mu;
    void* evs[kAsyncAhead] = {};
    bool ev_rec[kAsyncAhead] = {};
    unsigned ev_pos = 0;
    bool ev_init = false;
    // bumped (under the exclusive lock) whenever entries are removed: eviction, clear
    std::atomic<uint64_t> gen{0};
    std::mutex fmu;
    double compile_ms_total = 0, compile_ms_max = 0, load_ms_total = 0, disk_write_ms_total = 0,
           ir_ms_total = 0;

    void reset_counters() {
        for (auto* a : {&launches, &mem_hits, &disk_hits, &misses, &compiles, &compile_failures,
                        &generic_launches, &entries, &cubin_bytes, &disk_bytes_written,
                        &disk_rejects, &evictions, &disk_evictions, &ir_compiles})
            a->store(0);
        std::lock_guard<std::mutex> g(fmu);
        compile_ms_total = compile_ms_max = load_ms_total = disk_write_ms_total = ir_ms_total = 0;
    }
};

struct Job {
    Device* dev;
    const KernelDesc* k;
    std::shared_ptr<Entry> e;
    std::string src;
};

}  // namespace
}  // namespace proteus

struct proteus_kernel_s {
    proteus::KernelDesc d;
};

namespace proteus {
namespace {

struct Global {
    std::mutex mu;   // init / finalize / registration
    std::atomic<bool> initialized{false};
    BackendFactory backend_factory = nullptr;   // nullptr: CUDA (set_backend_factory)
    proteus_config cfg{};
    std::string cache_dir;
    std::unique_ptr<Backend> be;
    std::atomic<Device*> devs[kMaxDevices] = {};
    int default_device = 0;
    std::vector<std::unique_ptr<proteus_kernel_s>> kernels;
    // worker pool
    std::vector<std::thread> workers;
    std::deque<Job> q;
    std::mutex qmu;
    std::condition_variable qcv, idle_cv;
    bool stop = false;
    int busy = 0;
    std::thread warm_thread;
    // bumped by proteus_finalize: per-thread memos of Device / kernel pointers from an
    // earlier init are invalid (the addresses may be reused)
    std::atomic<uint64_t> epoch{1};
    // PROTEUS_F_IR: kernel LTO-IR per (kernel TU text + options) -- the TU holds the source,
    // block dims, minBlocks and flags, so it is the cache key; shared by all devices
    std::mutex ir_mu;
    std::unordered_map<std::string, std::shared_ptr<struct IrEntry>> ir_cache;
};

struct IrEntry {
    std::mutex mu;      // held while compiling: concurrent misses of one kernel IR wait
    bool done = false, ok = false;
    std::string ir, log;
};

Global& G() {
    static Global* g = new Global();   // never destroyed: safe at process exit
    return *g;
}

std::vector<std::string> split_opts(const std::string& s) {
    std::vector<std::string> out;
    std::istringstream is(s);
    std::string t;
    while (is >> t) out.push_back(t);
    return out;
}

std::vector<std::string> nvrtc_options(const KernelDesc& k) {
    // -lineinfo only on request (PROTEUS_F_LINEINFO, for ncu source views): it costs ~15%
    // of a compile (NVVM + ptxas, measured on stencil4_ws) and changes no instruction
    std::vector<std::string> o = {"-arch=" + k.arch, "-std=c++17", "-minimal"};
    if (G().cfg.flags & PROTEUS_F_LINEINFO) o.push_back("-lineinfo");
    for (auto& s : split_opts(k.options)) o.push_back(s);
    return o;
}

void trace(const Device* D, const KernelDesc& k, uint64_t h, const char* what, double ms) {
    if (!(G().cfg.flags & PROTEUS_F_TRACE)) return;
    std::fprintf(stderr,
                 "{\"proteus\": \"%s\", \"device\": %d, \"kernel\": \"%s\", \"hash\": \"%016llx\", "
                 "\"ms\": %.3f}\n",
                 what, D->ordinal, k.entry.c_str(), static_cast<unsigned long long>(h), ms);
}

void publish(Device* D, Entry* e, int state) {
    {
        std::lock_guard<std::mutex> g(D->wait_mu);
        e->state.store(state, std::memory_order_release);
    }
    D->wait_cv.notify_all();
}

// In-memory LRU (max_entries; the paper's planned eviction, P@26536-27373).  Launches read
// ready entries and call cuLaunchKernel under the shared lock, so once the victims are
// unlinked under the exclusive lock no thread can still be launching them; the context is
// synchronized before their modules are unloaded, so no in-flight kernel loses its code.
void evict_if_needed(Device* D, Entry* keep) {
    Global& g = G();
    const uint64_t cap = g.cfg.max_entries;
    if (!cap || D->entries.load() <= cap) return;
    std::vector<std::shared_ptr<Entry>> victims;
    {
        std::unique_lock<std::shared_mutex> lk(D->mu);
        std::vector<std::pair<uint64_t, Entry*>> ready;
        for (auto& kv : D->map)
            for (auto& e : kv.second)
                if (e.get() != keep && e->state.load() == kReady)
                    ready.emplace_back(e->last_use.load(), e.get());
        const uint64_t n = D->entries.load();
        if (n <= cap) return;
        uint64_t over = n - cap;
        std::sort(ready.begin(), ready.end(),
                  [](const std::pair<uint64_t, Entry*>& a, const std::pair<uint64_t, Entry*>& b) {
                      return a.first < b.first;
                  });
        for (size_t i = 0; i < ready.size() && over; ++i, --over) {
            Entry* v = ready[i].second;
            auto& chain = D->map[v->mhash];
            for (auto it = chain.begin(); it != chain.end(); ++it) {
                if (it->get() == v) {
                    victims.push_back(std::move(*it));
                    chain.erase(it);
                    break;
                }
            }
            if (chain.empty()) D->map.erase(v->mhash);
        }
        if (!victims.empty()) D->gen++;
    }
    if (victims.empty()) return;
    g.be->synchronize(D->ctx);
    for (auto& v : victims) {
        g.be->unload(v->module);   // victims are ready, hence resident, and now unlinked
        v->module = nullptr;
        v->resident = false;
        D->entries--;
        D->cubin_bytes -= v->cubin.size();
        D->evictions++;
    }
}

// After a successful load: if e is still in the map, count it as resident; if a
// cache_clear unlinked it meanwhile, unload the module at once (no launch can reach an
// unlinked entry) and publish it so that waiters retry through the map.  Counting under
// the exclusive lock keeps the counters consistent with a concurrent clear.
bool account_if_linked(Device* D, Entry* e, size_t cubin_bytes) {
    bool linked = false;
    {
        std::unique_lock<std::shared_mutex> lk(D->mu);
        auto it = D->map.find(e->mhash);
        if (it != D->map.end())
            for (auto& p : it->second) linked = linked || p.get() == e;
        if (linked) {
            D->entries++;
            D->cubin_bytes += cubin_bytes;
            e->resident = true;
        }
    }
    if (!linked) {
        G().be->synchronize(D->ctx);
        G().be->unload(e->module);
        e->module = nullptr;
        e->fn = nullptr;
        publish(D, e, kReady);
    }
    return linked;
}

// Disk level, else compile; then load and publish.  Runs on the launching thread
// (synchronous miss) or on a worker (async miss).  `src` is the specialized source.
// The persistent level: load the key's cubin file into e (disk hit) if it is there and
// intact.  *reject: a file existed but was corrupt or for another key.
bool load_from_disk(Device* D, const KernelDesc& k, Entry* e, bool* reject) {
    Global& g = G();
    std::string err;
    const double t0 = now_ms();
    std::string cubin;
    if (disk_read(g.cache_dir, e->hash, e->key, &cubin, reject)) {
        if (g.be->load(cubin, jit_symbol(k.entry, G().cfg.flags & kKeyFlagMask), &e->module, &e->fn, &err)) {
            const double dt = now_ms() - t0;
            {
                std::lock_guard<std::mutex> lk(D->fmu);
                D->load_ms_total += dt;
            }
            if (!account_if_linked(D, e, cubin.size())) return true;
            D->disk_hits++;
            e->cubin.swap(cubin);
            trace(D, k, e->hash, "disk_hit", dt);
            e->last_use.store(D->tick.fetch_add(1) + 1);
            publish(D, e, kReady);
            evict_if_needed(D, e);
            return true;
        }
        *reject = true;
    }
    return false;
}

// nvJitLink options equivalent to the kernel's NVRTC floating-point options (the link-time
// optimizer and ptxas run in nvJitLink, which takes 0/1 values): -fmad=false -> -fma=0,
// -ftz / -prec-div / -prec-sqrt=<b> -> <opt>=0|1, -lineinfo as it is.
std::vector<std::string> link_options(const KernelDesc& k) {
    std::vector<std::string> o = {"-arch=" + k.arch, "-lto", "-O3"};
    for (std::string x : nvrtc_options(k)) {
        if (x.rfind("--", 0) == 0) x = x.substr(1);
        const size_t eq = x.find('=');
        if (x == "-lineinfo") {
            o.push_back(x);
            continue;
        }
        if (eq == std::string::npos) continue;
        std::string name = x.substr(0, eq), val = x.substr(eq + 1);
        if (name == "-fmad") name = "-fma";
        if (name != "-fma" && name != "-ftz" && name != "-prec-div" && name != "-prec-sqrt")
            continue;
        o.push_back(name + "=" + (val == "false" || val == "0" ? "0" : "1"));
    }
    return o;
}

// The IR-level specialization (PROTEUS_F_IR): kernel TU -> LTO-IR once (cached
// process-wide), the key's constants TU -> LTO-IR, nvJitLink -lto of the two -> cubin.
bool compile_ir_path(Device* D, const KernelDesc& k, const std::string& src, size_t split,
                     std::string* cubin, std::string* log) {
    Global& g = G();
    const std::string consts = src.substr(0, split);
    const std::string ktu = src.substr(split + std::strlen(kIrSplit));
    std::vector<std::string> kopts = nvrtc_options(k);
    kopts.push_back("-dlto");
    kopts.push_back("-rdc=true");
    std::string ckey = ktu;
    for (const auto& o : kopts) ckey += '\x01' + o;
    std::shared_ptr<IrEntry> ir;
    {
        std::lock_guard<std::mutex> lk(g.ir_mu);
        auto& slot = g.ir_cache[ckey];
        if (!slot) slot = std::make_shared<IrEntry>();
        ir = slot;
    }
    {
        std::lock_guard<std::mutex> lk(ir->mu);
        if (!ir->done) {
            const double t0 = now_ms();
            ir->ok = g.be->compile_ltoir(ktu, k.entry + ".cu", kopts, &ir->ir, &ir->log);
            ir->done = true;
            D->ir_compiles++;
            std::lock_guard<std::mutex> fk(D->fmu);
            D->ir_ms_total += now_ms() - t0;
        }
    }
    if (!ir->ok) {
        *log = "kernel LTO-IR (NVRTC -dlto): " + ir->log;
        return false;
    }
    std::vector<std::string> copts = {"-arch=" + k.arch, "-std=c++17", "-minimal", "-dlto",
                                      "-rdc=true"};
    std::string cir;
    if (!g.be->compile_ltoir(consts, k.entry + "_constants.cu", copts, &cir, log)) {
        *log = "constants LTO-IR (NVRTC -dlto): " + *log;
        return false;
    }
    return g.be->link_ltoir({&ir->ir, &cir}, link_options(k), cubin, log);
}

void materialize(Device* D, const KernelDesc& k, Entry* e, const std::string& src) {
    Global& g = G();
    std::string err;
    const bool disk = (g.cfg.flags & PROTEUS_F_DISK) && !g.cache_dir.empty();
    int claim = -1;
    std::string claim_token;
    if (disk) {
        bool reject = false;
        if (load_from_disk(D, k, e, &reject)) return;
        if (reject) D->disk_rejects++;
        // Another process sharing the directory (a rank of the same job) may be compiling
        // this key right now: wait for its file instead of compiling it again.
        if (!reject && (claim = disk_claim(g.cache_dir, e->hash, &claim_token)) == 0) {
            if (disk_wait_claim(g.cache_dir, e->hash, 60000.0)) {
                bool rej2 = false;
                if (load_from_disk(D, k, e, &rej2)) return;
                if (rej2) D->disk_rejects++;
            }
            claim = disk_claim(g.cache_dir, e->hash, &claim_token);
        }
        // A claimant writes the file before it releases its claim, so a claim won just
        // after another process's release finds that process's file: check once more.
        if (claim == 1) {
            bool rej3 = false;
            if (load_from_disk(D, k, e, &rej3)) {
                disk_release(g.cache_dir, e->hash, claim_token);
                return;
            }
            if (rej3) D->disk_rejects++;
        }
    }
    const double t0 = now_ms();
    std::string cubin, log;
    const size_t ir_split = src.find(kIrSplit);
    const bool ok = ir_split != std::string::npos
                        ? compile_ir_path(D, k, src, ir_split, &cubin, &log)
                        : g.be->compile(src, k.entry + ".cu", nvrtc_options(k), &cubin, &log);
    const double cms = now_ms() - t0;
    if (!ok) {
        if (claim == 1) disk_release(g.cache_dir, e->hash, claim_token);
        e->log = "NVRTC compile of " + k.entry + " failed:\n" + log;
        D->compile_failures++;
        trace(D, k, e->hash, "compile_failed", cms);
        publish(D, e, kFailed);
        return;
    }
    {
        std::lock_guard<std::mutex> lk(D->fmu);
        D->compile_ms_total += cms;
        if (cms > D->compile_ms_max) D->compile_ms_max = cms;
    }
    D->compiles++;
    const double t1 = now_ms();
    if (!g.be->load(cubin, jit_symbol(k.entry, G().cfg.flags & kKeyFlagMask), &e->module, &e->fn, &err)) {
        if (claim == 1) disk_release(g.cache_dir, e->hash, claim_token);
        e->log = "loading the specialized cubin of " + k.entry + " failed: " + err;
        D->compile_failures++;
        publish(D, e, kFailed);
        return;
    }
    {
        std::lock_guard<std::mutex> lk(D->fmu);
        D->load_ms_total += now_ms() - t1;
    }
    if (!account_if_linked(D, e, cubin.size())) {
        if (claim == 1) disk_release(g.cache_dir, e->hash, claim_token);
        return;
    }
    if (disk) {
        const double t2 = now_ms();
        D->disk_bytes_written += disk_write(g.cache_dir, e->hash, e->key, cubin);
        if (claim == 1) disk_release(g.cache_dir, e->hash, claim_token);   // after the file is in place
        if (g.cfg.max_disk_bytes)
            D->disk_evictions += disk_enforce_cap(g.cache_dir, g.cfg.max_disk_bytes,
                                                  cache_file_path(g.cache_dir, e->hash));
        std::lock_guard<std::mutex> lk(D->fmu);
        D->disk_write_ms_total += now_ms() - t2;
    }
    e->cubin.swap(cubin);
    trace(D, k, e->hash, "compiled", cms);
    e->last_use.store(D->tick.fetch_add(1) + 1);
    publish(D, e, kReady);
    evict_if_needed(D, e);
}

void worker_main() {
    Global& g = G();
    for (;;) {
        Job job;
        {
            std::unique_lock<std::mutex> lk(g.qmu);
            g.qcv.wait(lk, [&] { return g.stop || !g.q.empty(); });
            if (g.q.empty()) return;   // stop requested and drained
            job = std::move(g.q.front());
            g.q.pop_front();
            ++g.busy;
        }
        std::string err;
        g.be->make_current(job.dev->ctx, &err);
        materialize(job.dev, *job.k, job.e.get(), job.src);
        job.dev->inflight--;
        {
            std::lock_guard<std::mutex> lk(g.qmu);
            --g.busy;
        }
        g.idle_cv.notify_all();
    }
}

void wait_idle() {
    Global& g = G();
    std::unique_lock<std::mutex> lk(g.qmu);
    g.idle_cv.wait(lk, [&] { return g.q.empty() && g.busy == 0; });
}

proteus_status open_device(int want, Device** out) {
    Global& g = G();
    std::lock_guard<std::mutex> lk(g.mu);
    int ordinal = -1;
    void* ctx = nullptr;
    std::string err;
    if (!g.be->device_open(want, &ordinal, &ctx, &err)) return fail(PROTEUS_E_CUDA, err);
    if (ordinal < 0 || ordinal >= kMaxDevices) return fail(PROTEUS_E_INVALID, "device ordinal out of range");
    Device* D = g.devs[ordinal].load();
    if (D) {
        g.be->device_close(ordinal, ctx);   // balance the extra retain
    } else {
        D = new Device();
        D->ordinal = ordinal;
        D->ctx = ctx;
        g.devs[ordinal].store(D);
    }
    *out = D;
    return PROTEUS_OK;
}

// Device of the calling thread (its current context), initialised on first use.  The
// last (context -> Device) of the thread is memoised: a hit costs one cuCtxGetCurrent.
proteus_status current_device(Device** out) {
    Global& g = G();
    thread_local struct {
        uint64_t epoch = 0;
        void* ctx = nullptr;
        Device* D = nullptr;
    } memo;
    void* ctx = g.be->current_context();
    const uint64_t ep = g.epoch.load(std::memory_order_acquire);
    if (ctx && memo.ctx == ctx && memo.epoch == ep) {
        *out = memo.D;
        return PROTEUS_OK;
    }
    int dev = g.be->current_device();
    if (dev < 0) dev = g.default_device;
    if (dev >= 0 && dev < kMaxDevices) {
        Device* D = g.devs[dev].load(std::memory_order_acquire);
        if (D) {
            if (!ctx) {
                std::string err;
                g.be->make_current(D->ctx, &err);
            } else if (ctx == D->ctx) {
                memo.epoch = ep;
                memo.ctx = ctx;
                memo.D = D;
            }
            *out = D;
            return PROTEUS_OK;
        }
    }
    return open_device(dev, out);
}

// Per-thread memo of the last in-memory hit of a kernel (direct-mapped by the kernel's
// address): a launch with the same annotated values, dims and kernel settings on the same
// Device reuses the Entry without building, hashing and looking up the key -- valid while
// the Device's removal generation is unchanged (checked under the shared lock, so the
// entry cannot be evicted during the launch).  Same entry, same counters as the full path.
struct HitMemo {
    const proteus_kernel_s* k = nullptr;
    uint64_t epoch = 0, version = 0, gen = 0;
    Device* D = nullptr;
    Entry* e = nullptr;
    unsigned dims[6] = {};
    size_t nvals = 0;
    uint8_t vals[kMaxAnnotated * 8];
};

HitMemo& hit_memo(const proteus_kernel_s* k) {
    thread_local HitMemo memo[16];
    return memo[(reinterpret_cast<uintptr_t>(k) >> 4) & 15];
}

// the raw bytes of the annotated arguments, in order
size_t annotated_bytes(const KernelDesc& kd, void** args, uint8_t* out) {
    size_t n = 0;
    for (int i : kd.annotated) {
        const size_t sz = type_size(kd.types[i]);
        std::memcpy(out + n, args[i], sz);
        n += sz;
    }
    return n;
}

Entry* find(Device* D, uint64_t h, const std::vector<uint8_t>& key) {
    auto it = D->map.find(h);
    if (it == D->map.end()) return nullptr;
    for (auto& e : it->second)
        if (e->key == key) return e.get();
    return nullptr;
}

unsigned min_blocks_of(const KernelDesc& k) {
    return static_cast<unsigned>(k.min_blocks > 0 ? k.min_blocks : G().cfg.min_blocks_per_sm);
}

bool check_dims(unsigned gx, unsigned gy, unsigned gz, unsigned bx, unsigned by, unsigned bz) {
    if (!gx || !gy || !gz || !bx || !by || !bz) return false;
    return static_cast<unsigned long long>(bx) * by * bz <= 1024ull;
}

struct Resolved {
    std::shared_ptr<Entry> e;   // keeps the entry alive while this thread uses it
    bool inserted = false;
};

std::shared_ptr<Entry> find_shared(Device* D, uint64_t h, const std::vector<uint8_t>& key) {
    auto it = D->map.find(h);
    if (it == D->map.end()) return nullptr;
    for (auto& e : it->second)
        if (e->key == key) return e;
    return nullptr;
}

// Find or insert the entry for this key (exclusive lock only on insert).
Resolved resolve(Device* D, const std::vector<uint8_t>& key, uint64_t h) {
    {
        std::shared_lock<std::shared_mutex> lk(D->mu);
        if (auto e = find_shared(D, h, key)) return {e, false};
    }
    std::unique_lock<std::shared_mutex> lk(D->mu);
    if (auto e = find_shared(D, h, key)) return {e, false};
    auto sp = std::make_shared<Entry>();
    sp->key = key;
    sp->hash = fnv1a64(key.data(), key.size());
    sp->mhash = h;
    D->map[h].push_back(sp);
    return {sp, true};
}

void wait_ready(Device* D, Entry* e) {
    std::unique_lock<std::mutex> lk(D->wait_mu);
    D->wait_cv.wait(lk, [&] { return e->state.load(std::memory_order_acquire) != kCompiling; });
}

proteus_status do_launch(Device* D, void* fn, const LaunchDims& d, unsigned shmem, void* stream,
                         void** args) {
    std::string err;
    if (!G().be->launch(fn, d, shmem, stream, args, &err)) return fail(PROTEUS_E_CUDA, err);
    D->launches++;
    return PROTEUS_OK;
}

// Async throttle, before a generic launch that stands in for entry e: wait until the
// generic launch kAsyncAhead back has completed on the GPU, or e is published.  Returns
// true when e became ready (the caller launches the specialization instead).
bool throttle_generic(Device* D, Entry* e) {
    Global& g = G();
    void* ev = nullptr;
    {
        std::lock_guard<std::mutex> lk(D->ev_mu);
        if (!D->ev_init) {
            for (auto& x : D->evs) x = g.be->event_create();   // nullptr: no throttling
            D->ev_init = true;
        }
        if (D->ev_rec[D->ev_pos]) ev = D->evs[D->ev_pos];
    }
    if (ev) {
        std::unique_lock<std::mutex> lk(D->wait_mu);   // publish() notifies wait_cv
        while (e->state.load(std::memory_order_acquire) == kCompiling &&
               g.be->event_query(ev) == 0)
            D->wait_cv.wait_for(lk, std::chrono::microseconds(20));
    }
    return e->state.load(std::memory_order_acquire) == kReady;
}

// after a generic launch on `stream`: mark it in the throttle ring
void record_generic(Device* D, void* stream) {
    std::lock_guard<std::mutex> lk(D->ev_mu);
    void* ev = D->evs[D->ev_pos];
    if (ev && G().be->event_record(ev, stream)) {
        D->ev_rec[D->ev_pos] = true;
        D->ev_pos = (D->ev_pos + 1) % kAsyncAhead;
    }
}

proteus_status launch_generic_async(Device* D, const KernelDesc& kd, const LaunchDims& d,
                                    unsigned shmem, void* stream, void** args) {
    D->generic_launches++;
    const proteus_status st = do_launch(D, kd.generic_fn, d, shmem, stream, args);
    if (st == PROTEUS_OK) record_generic(D, stream);
    return st;
}

}  // namespace
}  // namespace proteus

using namespace proteus;

extern "C" {

proteus_status proteus_config_default(proteus_config* out) {
    if (!out) return fail(PROTEUS_E_INVALID, "null config");
    out->device = -1;
    out->cache_dir = nullptr;
    out->flags = PROTEUS_F_RCF | PROTEUS_F_LB | PROTEUS_F_FOLD_DIMS | PROTEUS_F_DISK;
    out->async_workers = 0;
    out->min_blocks_per_sm = 1;
    if (const char* s = std::getenv("PROTEUS_CACHE_DIR")) out->cache_dir = s;
    if (const char* s = std::getenv("PROTEUS_DISK_CACHE")) {
        if (std::atoi(s)) out->flags |= PROTEUS_F_DISK; else out->flags &= ~PROTEUS_F_DISK;
    }
    if (const char* s = std::getenv("PROTEUS_ASYNC")) out->async_workers = std::atoi(s);
    if (const char* s = std::getenv("PROTEUS_SPECIALIZE")) {
        // none = plain JIT (the paper's "None", P@36323); rcf folds argument values and
        // launch dims; lb = launch bounds only; all = both.
        out->flags &= ~(PROTEUS_F_RCF | PROTEUS_F_LB | PROTEUS_F_FOLD_DIMS);
        if (!std::strcmp(s, "lb") || !std::strcmp(s, "all")) out->flags |= PROTEUS_F_LB;
        if (!std::strcmp(s, "rcf") || !std::strcmp(s, "all"))
            out->flags |= PROTEUS_F_RCF | PROTEUS_F_FOLD_DIMS;
        if (std::strcmp(s, "none") && std::strcmp(s, "lb") && std::strcmp(s, "rcf") &&
            std::strcmp(s, "all"))
            return fail(PROTEUS_E_INVALID, std::string("PROTEUS_SPECIALIZE must be none|lb|rcf|all, got ") + s);
    }
    if (const char* s = std::getenv("PROTEUS_FOLD_DIMS")) {
        if (std::atoi(s)) out->flags |= PROTEUS_F_FOLD_DIMS; else out->flags &= ~PROTEUS_F_FOLD_DIMS;
    }
    if (const char* s = std::getenv("PROTEUS_MIN_BLOCKS")) out->min_blocks_per_sm = std::atoi(s);
    out->max_entries = 0;
    out->max_disk_bytes = 0;
    if (const char* s = std::getenv("PROTEUS_CACHE_MAX_ENTRIES"))
        out->max_entries = std::strtoull(s, nullptr, 10);
    if (const char* s = std::getenv("PROTEUS_DISK_MAX_MB"))
        out->max_disk_bytes = std::strtoull(s, nullptr, 10) << 20;
    if (const char* s = std::getenv("PROTEUS_TRACE")) {
        if (std::atoi(s)) out->flags |= PROTEUS_F_TRACE;
    }
    if (const char* s = std::getenv("PROTEUS_LINEINFO")) {
        if (std::atoi(s)) out->flags |= PROTEUS_F_LINEINFO;
    }
    if (const char* s = std::getenv("PROTEUS_IR")) {
        if (std::atoi(s)) out->flags |= PROTEUS_F_IR; else out->flags &= ~PROTEUS_F_IR;
    }
    return PROTEUS_OK;
}

proteus_status proteus_init(const proteus_config* cfg_in) {
    Global& g = G();
    proteus_config cfg;
    if (cfg_in) {
        cfg = *cfg_in;
    } else if (proteus_status s = proteus_config_default(&cfg)) {
        return s;
    }
    if (cfg.min_blocks_per_sm < 0 || cfg.async_workers < 0 || cfg.async_workers > 64)
        return fail(PROTEUS_E_INVALID, "bad min_blocks_per_sm / async_workers");
    {
        std::lock_guard<std::mutex> lk(g.mu);
        if (!g.initialized.load()) {
            g.be = g.backend_factory ? g.backend_factory() : make_cuda_backend();
            std::string err;
            if (!g.be->init(&err)) {
                g.be.reset();
                return fail(PROTEUS_E_CUDA, err);
            }
            std::string dir = cfg.cache_dir ? cfg.cache_dir : "./.proteus-cache";
            if (cfg.flags & PROTEUS_F_DISK) {
                if (!ensure_dir(dir, &err)) {
                    g.be.reset();
                    return fail(PROTEUS_E_IO, err);
                }
            }
            g.cache_dir = dir;
            g.cfg = cfg;
            g.cfg.cache_dir = nullptr;   // the string lives in g.cache_dir
            g.stop = false;
            for (int i = 0; i < cfg.async_workers; ++i) g.workers.emplace_back(worker_main);
            if (!g.backend_factory) g.warm_thread = std::thread([] { G().be->warm(); });
            g.initialized.store(true);
        }
    }
    Device* D = nullptr;
    if (proteus_status s = open_device(cfg.device, &D)) return s;
    if (cfg.device >= 0 || g.default_device == 0) g.default_device = D->ordinal;
    return PROTEUS_OK;
}

proteus_status proteus_register_kernel(const char* entry, const char* cuda_source,
                                       const char* options, const proteus_type* arg_types,
                                       int nargs, const int* annotated_idx, int n_annotated,
                                       void* generic_fn, proteus_kernel* out) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!entry || !*entry || !cuda_source || !out) return fail(PROTEUS_E_INVALID, "null entry/source/out");
    if (nargs < 0 || nargs > kMaxArgs || (nargs && !arg_types))
        return fail(PROTEUS_E_INVALID, "nargs out of range");
    if (n_annotated < 0 || n_annotated > kMaxAnnotated || (n_annotated && !annotated_idx))
        return fail(PROTEUS_E_INVALID, "n_annotated out of range");
    auto k = std::make_unique<proteus_kernel_s>();
    KernelDesc& d = k->d;
    d.entry = entry;
    d.source = cuda_source;
    d.options = options ? options : "";
    for (int i = 0; i < nargs; ++i) {
        if (arg_types[i] < PROTEUS_I32 || arg_types[i] > PROTEUS_OPAQUE)
            return fail(PROTEUS_E_INVALID, "bad proteus_type for argument " + std::to_string(i + 1));
        d.types.push_back(arg_types[i]);
    }
    std::vector<bool> seen(nargs, false);
    for (int i = 0; i < n_annotated; ++i) {
        const int a = annotated_idx[i];
        if (a < 1 || a > nargs)
            return fail(PROTEUS_E_INVALID, "annotated index " + std::to_string(a) + " not in 1..nargs (1-based, P@12394)");
        if (a > kMaxAnnotated)
            return fail(PROTEUS_E_INVALID, "annotated index > 32 not supported");
        if (seen[a - 1]) return fail(PROTEUS_E_INVALID, "duplicate annotated index " + std::to_string(a));
        const proteus_type t = d.types[a - 1];
        if (t == PROTEUS_PTR || t == PROTEUS_OPAQUE)
            return fail(PROTEUS_E_INVALID, "annotated argument " + std::to_string(a) + " is not a scalar");
        seen[a - 1] = true;
    }
    for (int i = 0; i < nargs; ++i)
        if (seen[i]) d.annotated.push_back(i);
    d.generic_fn = generic_fn;
    if (generic_fn) g.be->note_generic(generic_fn);
    char hdr[64];
    std::snprintf(hdr, sizeof hdr, "|%s|hdr=%016llx", kLibTag,
                  static_cast<unsigned long long>(fnv1a64(kDeviceHeader, std::strlen(kDeviceHeader))));
    d.toolkit = g.be->toolkit() + hdr;
    d.arch = g.be->arch(g.default_device);
    std::string blob = d.source;
    for (const std::string* s : {&d.entry, &d.options, &d.toolkit, &d.arch}) {
        blob.push_back('\0');
        blob += *s;
    }
    d.kernel_id = fnv1a64(blob.data(), blob.size());
    std::lock_guard<std::mutex> lk(g.mu);
    *out = k.get();
    g.kernels.push_back(std::move(k));
    return PROTEUS_OK;
}

proteus_status proteus_launch(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                              unsigned bx, unsigned by, unsigned bz, unsigned shmem_bytes,
                              void* stream, void** args) {
    Global& g = G();
    if (!g.initialized.load(std::memory_order_acquire)) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k) return fail(PROTEUS_E_INVALID, "null kernel");
    if (!check_dims(gx, gy, gz, bx, by, bz)) return fail(PROTEUS_E_INVALID, "bad launch dimensions (zero, or block > 1024 threads)");
    if (!args && !k->d.types.empty()) return fail(PROTEUS_E_INVALID, "null args");
    Device* D = nullptr;
    if (proteus_status s = current_device(&D)) return s;
    const KernelDesc& kd = k->d;
    const LaunchDims dims{{gx, gy, gz}, {bx, by, bz}, kd.launch_attrs};
    const uint64_t ep = g.epoch.load(std::memory_order_acquire);
    HitMemo& m = hit_memo(k);
    uint8_t vals[kMaxAnnotated * 8];
    const size_t nvals = annotated_bytes(kd, args, vals);
    const unsigned dv[6] = {gx, gy, gz, bx, by, bz};
    const bool memo_match = m.k == k && m.epoch == ep && m.D == D &&
                            m.version == kd.version && m.nvals == nvals &&
                            std::memcmp(m.dims, dv, sizeof dv) == 0 &&
                            std::memcmp(m.vals, vals, nvals) == 0;
    if (memo_match) {   // memoised hit: no key build, hash or map lookup
        std::shared_lock<std::shared_mutex> lk(D->mu);
        Entry* e = m.e;
        if (m.gen == D->gen.load(std::memory_order_relaxed) &&
            e->state.load(std::memory_order_acquire) == kReady) {
            if (g.cfg.max_entries)
                e->last_use.store(D->tick.fetch_add(1, std::memory_order_relaxed) + 1,
                                  std::memory_order_relaxed);
            D->mem_hits++;
            return do_launch(D, e->fn, dims, shmem_bytes, stream, args);
        }
    }
    const unsigned kf = g.cfg.flags & kKeyFlagMask;
    const unsigned minb = min_blocks_of(kd);
    thread_local std::vector<uint8_t> key;
    build_key(kd, kf, minb, dims, args, &key);
    const uint64_t h = key_map_hash(key.data(), key.size());   // map key (file name: FNV)
    {   // hit path: find + launch under the shared lock (eviction takes it exclusively)
        std::shared_lock<std::shared_mutex> lk(D->mu);
        if (Entry* e = find(D, h, key)) {
            if (e->state.load(std::memory_order_acquire) == kReady) {
                if (g.cfg.max_entries)
                    e->last_use.store(D->tick.fetch_add(1, std::memory_order_relaxed) + 1,
                                      std::memory_order_relaxed);
                D->mem_hits++;
                m.k = k;
                m.epoch = ep;
                m.version = kd.version;
                m.gen = D->gen.load(std::memory_order_relaxed);
                m.D = D;
                m.e = e;
                std::memcpy(m.dims, dv, sizeof dv);
                m.nvals = nvals;
                std::memcpy(m.vals, vals, nvals);
                return do_launch(D, e->fn, dims, shmem_bytes, stream, args);
            }
        }
    }
    Resolved r = resolve(D, key, h);
    Entry* e = r.e.get();
    if (!r.inserted) {
        int st = e->state.load(std::memory_order_acquire);
        if (st == kReady)   // became ready since the probe: take the locked hit path
            return proteus_launch(k, gx, gy, gz, bx, by, bz, shmem_bytes, stream, args);
        if (st == kCompiling) {
            if (g.cfg.async_workers > 0 && kd.generic_fn) {
                if (throttle_generic(D, e))   // published while the host waited
                    return proteus_launch(k, gx, gy, gz, bx, by, bz, shmem_bytes, stream, args);
                return launch_generic_async(D, kd, dims, shmem_bytes, stream, args);
            }
            wait_ready(D, e);
            st = e->state.load(std::memory_order_acquire);
            if (st == kReady)
                return proteus_launch(k, gx, gy, gz, bx, by, bz, shmem_bytes, stream, args);
        }
        // failed specialization
        if (kd.generic_fn) {
            D->generic_launches++;
            return do_launch(D, kd.generic_fn, dims, shmem_bytes, stream, args);
        }
        return fail(PROTEUS_E_COMPILE, e->log);
    }
    // in-memory miss: this thread owns the new entry
    D->misses++;
    std::string src = specialized_source(kd, kf, minb, dims, args);
    if (g.cfg.async_workers > 0 && kd.generic_fn) {
        D->inflight++;
        {
            std::lock_guard<std::mutex> lk(g.qmu);
            g.q.push_back(Job{D, &kd, r.e, std::move(src)});
        }
        g.qcv.notify_one();
        return launch_generic_async(D, kd, dims, shmem_bytes, stream, args);
    }
    materialize(D, kd, e, src);
    if (e->state.load() == kReady) {
        {   // re-find under the shared lock: a concurrent miss may have evicted it already
            std::shared_lock<std::shared_mutex> lk(D->mu);
            Entry* f = find(D, h, key);
            if (f && f->state.load(std::memory_order_acquire) == kReady)
                return do_launch(D, f->fn, dims, shmem_bytes, stream, args);
        }
        return proteus_launch(k, gx, gy, gz, bx, by, bz, shmem_bytes, stream, args);
    }
    if (kd.generic_fn) {
        D->generic_launches++;
        return do_launch(D, kd.generic_fn, dims, shmem_bytes, stream, args);
    }
    return fail(PROTEUS_E_COMPILE, e->log);
}

proteus_status proteus_kernel_set_min_blocks(proteus_kernel k, int min_blocks) {
    if (!k || min_blocks < 0 || min_blocks > 32)
        return fail(PROTEUS_E_INVALID, "min_blocks must be 0..32");
    k->d.min_blocks = min_blocks;
    k->d.version++;
    return PROTEUS_OK;
}

proteus_status proteus_kernel_set_launch_attrs(proteus_kernel k, unsigned attrs) {
    if (!k || (attrs & ~static_cast<unsigned>(PROTEUS_LAUNCH_PDL)))
        return fail(PROTEUS_E_INVALID, "launch attrs: unknown bits (known: PROTEUS_LAUNCH_PDL)");
    k->d.launch_attrs = attrs;
    return PROTEUS_OK;
}

proteus_status proteus_kernel_bind_global(proteus_kernel k, const char* name, void* dptr) {
    if (!k || !name || !dptr) return fail(PROTEUS_E_INVALID, "null argument");
    const size_t n = std::strlen(name);
    bool ok = n > 0 && n < 128 && !(name[0] >= '0' && name[0] <= '9');
    for (size_t i = 0; ok && i < n; ++i) {
        const char c = name[i];
        ok = (c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z') || (c >= '0' && c <= '9') || c == '_';
    }
    if (!ok) return fail(PROTEUS_E_INVALID, "global name must be a C identifier (< 128 chars)");
    auto& gl = k->d.globals;
    const uint64_t a = reinterpret_cast<uint64_t>(dptr);
    bool found = false;
    for (auto& g : gl)
        if (g.first == name) {
            g.second = a;
            found = true;
        }
    if (!found) {
        if (gl.size() >= 255) return fail(PROTEUS_E_INVALID, "too many bound globals");
        gl.emplace_back(name, a);
        std::sort(gl.begin(), gl.end());
    }
    k->d.version++;   // the bindings are in the key: memoised hits of k are stale
    return PROTEUS_OK;
}

proteus_status proteus_launch_aot(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                                  unsigned bx, unsigned by, unsigned bz, unsigned shmem_bytes,
                                  void* stream, void** args) {
    Global& g = G();
    if (!g.initialized.load(std::memory_order_acquire)) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k || !k->d.generic_fn) return fail(PROTEUS_E_INVALID, "kernel has no generic (AOT) function");
    if (!check_dims(gx, gy, gz, bx, by, bz)) return fail(PROTEUS_E_INVALID, "bad launch dimensions");
    std::string err;
    if (!g.be->launch(k->d.generic_fn, LaunchDims{{gx, gy, gz}, {bx, by, bz}, k->d.launch_attrs},
                      shmem_bytes, stream, args, &err))
        return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_encode_tensor_map(void* map_out, int elem_type, unsigned rank,
                                         void* base, const uint64_t* dims,
                                         const uint64_t* strides, const uint32_t* box) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!map_out || (reinterpret_cast<uintptr_t>(map_out) & 63) || !dims || !box ||
        rank < 1 || rank > 5 || (rank > 1 && !strides))
        return fail(PROTEUS_E_INVALID, "bad tensor-map arguments (map_out must be 64-B aligned)");
    std::string err;
    if (!g.be->encode_tensor_map(map_out, elem_type, rank, base, dims, strides, box, &err))
        return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

// ---- peer memory for fused compute + halo kernels (NEXT-2) ------------------------
proteus_status proteus_ipc_get_handle(void* dptr, uint8_t* handle, uint64_t* offset) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!dptr || !handle || !offset) return fail(PROTEUS_E_INVALID, "null argument");
    Device* D = nullptr;
    if (proteus_status s = current_device(&D)) return s;
    std::string err;
    if (!g.be->ipc_get_handle(dptr, handle, offset, &err)) return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_ipc_open_handle(const uint8_t* handle, void** base) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!handle || !base) return fail(PROTEUS_E_INVALID, "null argument");
    Device* D = nullptr;
    if (proteus_status s = current_device(&D)) return s;
    std::string err;
    if (!g.be->ipc_open_handle(handle, base, &err)) return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_ipc_close_handle(void* base) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!base) return fail(PROTEUS_E_INVALID, "null argument");
    std::string err;
    if (!g.be->ipc_close_handle(base, &err)) return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_stream_write_u32(void* stream, void* dptr, uint32_t value) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!dptr || (reinterpret_cast<uintptr_t>(dptr) & 3))
        return fail(PROTEUS_E_INVALID, "flag address must be non-null and 4-byte aligned");
    std::string err;
    if (!g.be->stream_write_u32(stream, dptr, value, &err)) return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_stream_wait_u32(void* stream, void* dptr, uint32_t value) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!dptr || (reinterpret_cast<uintptr_t>(dptr) & 3))
        return fail(PROTEUS_E_INVALID, "flag address must be non-null and 4-byte aligned");
    std::string err;
    if (!g.be->stream_wait_u32(stream, dptr, value, &err)) return fail(PROTEUS_E_CUDA, err);
    return PROTEUS_OK;
}

proteus_status proteus_cache_stats(int device, proteus_cache_stats_t* out) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!out) return fail(PROTEUS_E_INVALID, "null out");
    Device* D = nullptr;
    if (device < 0) {
        if (proteus_status s = current_device(&D)) return s;
    } else {
        if (device >= kMaxDevices || !(D = g.devs[device].load()))
            return fail(PROTEUS_E_INVALID, "device not initialised");
    }
    out->launches = D->launches;
    out->mem_hits = D->mem_hits;
    out->disk_hits = D->disk_hits;
    out->misses = D->misses;
    out->compiles = D->compiles;
    out->compile_failures = D->compile_failures;
    out->generic_launches = D->generic_launches;
    out->inflight = D->inflight;
    out->entries = D->entries;
    out->cubin_bytes = D->cubin_bytes;
    out->disk_bytes_written = D->disk_bytes_written;
    out->disk_rejects = D->disk_rejects;
    std::lock_guard<std::mutex> lk(D->fmu);
    out->compile_ms_total = D->compile_ms_total;
    out->compile_ms_max = D->compile_ms_max;
    out->load_ms_total = D->load_ms_total;
    out->disk_write_ms_total = D->disk_write_ms_total;
    out->evictions = D->evictions;
    out->disk_evictions = D->disk_evictions;
    out->ir_compiles = D->ir_compiles;
    out->ir_ms_total = D->ir_ms_total;   // fmu held above
    return PROTEUS_OK;
}

proteus_status proteus_wait_idle(void) {
    if (!G().initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    wait_idle();
    return PROTEUS_OK;
}

proteus_status proteus_cache_clear(int device, int memory, int disk) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (memory) {
        wait_idle();
        for (int i = 0; i < kMaxDevices; ++i) {
            Device* D = g.devs[i].load();
            if (!D || (device >= 0 && device != i)) continue;
            std::unique_lock<std::shared_mutex> lk(D->mu);
            // kernels of these modules may still be queued on the device (launches are
            // asynchronous): drain the context before unloading, as LRU eviction does.
            // Only resident modules: an entry still compiling or loading (a synchronous
            // miss on another thread, a job queued after wait_idle) is unlinked here, and
            // its owner's account_if_linked then unloads its module itself.
            if (!D->map.empty()) g.be->synchronize(D->ctx);
            for (auto& kv : D->map)
                for (auto& e : kv.second)
                    if (e->resident) {
                        g.be->unload(e->module);
                        e->module = nullptr;
                        e->fn = nullptr;
                        e->resident = false;
                    }
            D->map.clear();
            D->gen++;
            D->reset_counters();
        }
        // the kernel LTO-IR cache of PROTEUS_F_IR is part of the in-memory level (entries
        // being compiled keep theirs alive through their shared_ptr)
        std::lock_guard<std::mutex> ik(g.ir_mu);
        g.ir_cache.clear();
    }
    if (disk) disk_clear(g.cache_dir);
    return PROTEUS_OK;
}

proteus_status proteus_finalize(void) {
    Global& g = G();
    std::lock_guard<std::mutex> lk(g.mu);
    if (!g.initialized.load()) return PROTEUS_OK;
    {
        std::lock_guard<std::mutex> qk(g.qmu);
        g.stop = true;
    }
    g.qcv.notify_all();
    g.epoch++;
    for (auto& t : g.workers) t.join();
    g.workers.clear();
    if (g.warm_thread.joinable()) g.warm_thread.join();
    for (int i = 0; i < kMaxDevices; ++i) {
        Device* D = g.devs[i].exchange(nullptr);
        if (!D) continue;
        for (auto& kv : D->map)
            for (auto& e : kv.second)
                if (e->resident) g.be->unload(e->module);
        for (void* ev : D->evs) g.be->event_destroy(ev);
        g.be->device_close(D->ordinal, D->ctx);
        delete D;
    }
    g.kernels.clear();
    g.q.clear();
    {
        std::lock_guard<std::mutex> ik(g.ir_mu);
        g.ir_cache.clear();
    }
    g.be.reset();
    g.default_device = 0;
    g.initialized.store(false);
    return PROTEUS_OK;
}

const char* proteus_last_error(void) { return t_err.c_str(); }

proteus_status proteus_kernel_info(proteus_kernel k, uint64_t* kernel_id, char* toolkit,
                                   size_t toolkit_cap, char* arch, size_t arch_cap) {
    if (!k) return fail(PROTEUS_E_INVALID, "null kernel");
    if (kernel_id) *kernel_id = k->d.kernel_id;
    if (toolkit && toolkit_cap) std::snprintf(toolkit, toolkit_cap, "%s", k->d.toolkit.c_str());
    if (arch && arch_cap) std::snprintf(arch, arch_cap, "%s", k->d.arch.c_str());
    return PROTEUS_OK;
}

proteus_status proteus_key(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                           unsigned bx, unsigned by, unsigned bz, void** args,
                           uint8_t* buf, size_t cap, size_t* len, uint64_t* hash) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k || (!args && !k->d.types.empty())) return fail(PROTEUS_E_INVALID, "null kernel/args");
    std::vector<uint8_t> key;
    build_key(k->d, g.cfg.flags & kKeyFlagMask, min_blocks_of(k->d),
              LaunchDims{{gx, gy, gz}, {bx, by, bz}}, args, &key);
    if (len) *len = key.size();
    if (hash) *hash = fnv1a64(key.data(), key.size());
    if (buf) {
        if (cap < key.size()) return fail(PROTEUS_E_INVALID, "buffer too small");
        std::memcpy(buf, key.data(), key.size());
    }
    return PROTEUS_OK;
}

proteus_status proteus_specialized_source(proteus_kernel k, unsigned gx, unsigned gy,
                                          unsigned gz, unsigned bx, unsigned by,
                                          unsigned bz, void** args, char* buf, size_t cap,
                                          size_t* len) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k || (!args && !k->d.types.empty())) return fail(PROTEUS_E_INVALID, "null kernel/args");
    const std::string s =
        specialized_source(k->d, g.cfg.flags & kKeyFlagMask, min_blocks_of(k->d),
                           LaunchDims{{gx, gy, gz}, {bx, by, bz}}, args);
    if (len) *len = s.size();
    if (buf) {
        if (cap < s.size() + 1) return fail(PROTEUS_E_INVALID, "buffer too small");
        std::memcpy(buf, s.c_str(), s.size() + 1);
    }
    return PROTEUS_OK;
}

proteus_status proteus_get_specialization(proteus_kernel k, unsigned gx, unsigned gy,
                                          unsigned gz, unsigned bx, unsigned by,
                                          unsigned bz, void** args, void** fn, int* state,
                                          uint8_t* buf, size_t cap, size_t* len) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k || (!args && !k->d.types.empty())) return fail(PROTEUS_E_INVALID, "null kernel/args");
    if (!check_dims(gx, gy, gz, bx, by, bz)) return fail(PROTEUS_E_INVALID, "bad launch dimensions");
    Device* D = nullptr;
    if (proteus_status s = current_device(&D)) return s;
    const KernelDesc& kd = k->d;
    const LaunchDims dims{{gx, gy, gz}, {bx, by, bz}};
    const unsigned kf = g.cfg.flags & kKeyFlagMask;
    const unsigned minb = min_blocks_of(kd);
    std::vector<uint8_t> key;
    build_key(kd, kf, minb, dims, args, &key);
    const uint64_t h = key_map_hash(key.data(), key.size());   // map key (file name: FNV)
    Resolved r = resolve(D, key, h);
    if (r.inserted) {
        D->misses++;
        materialize(D, kd, r.e.get(), specialized_source(kd, kf, minb, dims, args));
    } else {
        wait_ready(D, r.e.get());
    }
    const int st = r.e->state.load();
    if (state) *state = st;
    if (fn) *fn = st == kReady ? r.e->fn : nullptr;
    if (len) *len = r.e->cubin.size();
    if (buf && st == kReady) {
        if (cap < r.e->cubin.size()) return fail(PROTEUS_E_INVALID, "buffer too small");
        std::memcpy(buf, r.e->cubin.data(), r.e->cubin.size());
    }
    if (st != kReady) return fail(PROTEUS_E_COMPILE, r.e->log);
    return PROTEUS_OK;
}

proteus_status proteus_prefetch(proteus_kernel k, unsigned gx, unsigned gy, unsigned gz,
                                unsigned bx, unsigned by, unsigned bz, void** args) {
    Global& g = G();
    if (!g.initialized.load()) return fail(PROTEUS_E_NOT_INIT, "proteus_init has not been called");
    if (!k || (!args && !k->d.types.empty())) return fail(PROTEUS_E_INVALID, "null kernel/args");
    if (!check_dims(gx, gy, gz, bx, by, bz)) return fail(PROTEUS_E_INVALID, "bad launch dimensions");
    Device* D = nullptr;
    if (proteus_status s = current_device(&D)) return s;
    const KernelDesc& kd = k->d;
    const LaunchDims dims{{gx, gy, gz}, {bx, by, bz}, kd.launch_attrs};
    const unsigned kf = g.cfg.flags & kKeyFlagMask;
    const unsigned minb = min_blocks_of(kd);
    std::vector<uint8_t> key;
    build_key(kd, kf, minb, dims, args, &key);
    Resolved r = resolve(D, key, key_map_hash(key.data(), key.size()));
    if (!r.inserted) return PROTEUS_OK;   // ready, being compiled, or failed already
    D->misses++;
    std::string src = specialized_source(kd, kf, minb, dims, args);
    {   // the compile runs on the worker pool; a configuration without workers gets
        // kPrefetchWorkers of them now (they also serve later async misses)
        std::lock_guard<std::mutex> lk(g.mu);
        while (g.workers.size() < kPrefetchWorkers) g.workers.emplace_back(worker_main);
    }
    D->inflight++;
    {
        std::lock_guard<std::mutex> lk(g.qmu);
        g.q.push_back(Job{D, &kd, r.e, std::move(src)});
    }
    g.qcv.notify_one();
    return PROTEUS_OK;
}

}  // extern "C"

namespace proteus {
bool set_backend_factory(BackendFactory f) {
    Global& g = G();
    std::lock_guard<std::mutex> lk(g.mu);
    if (g.initialized.load()) return false;
    g.backend_factory = f;
    return true;
}
}  // namespace proteus
