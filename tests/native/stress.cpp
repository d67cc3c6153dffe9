// stress.cpp -- multi-threaded stress of libproteus's cache state machine on the fake
// backend, built with -fsanitize=thread (data races) or -fsanitize=address,undefined
// (memory errors) by tests/test_sanitizers_native.py (SURVEY.md §5 "Race detection /
// sanitizers": TSAN and ASAN on libproteus with the fake backend).
//
// 8 launcher threads hammer proteus_launch on 3 kernels with ~150 distinct keys (lr bit
// patterns), with async workers (generic launched while compiling, per-key dedupe), an
// in-memory LRU cap (evictions + unload after sync) and a disk cap (file deletion), while
// one thread snapshots counters and another clears the memory level now and then.  The
// counters must balance at the end; exit code 0 = consistent.
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "proteus.h"
#include "proteus_testing.h"

static const char* kSrc =
    "#include \"proteus_device.h\"\n"
    "extern \"C\" __global__ PROTEUS_LAUNCH_BOUNDS void k(double* y, float lr, int n) {\n"
    "  const float a = PROTEUS_SPEC(2, lr); const int m = PROTEUS_SPEC(3, n);\n"
    "  if (threadIdx.x < m) y[threadIdx.x] *= a; }\n";

#define CHECK(x)                                                                     \
    do {                                                                             \
        proteus_status s_ = (x);                                                     \
        if (s_ != PROTEUS_OK) {                                                      \
            std::fprintf(stderr, "%s:%d %s -> %d (%s)\n", __FILE__, __LINE__, #x,    \
                         (int)s_, proteus_last_error());                             \
            std::exit(2);                                                            \
        }                                                                            \
    } while (0)

int main(int argc, char** argv) {
    const char* dir = argc > 1 ? argv[1] : "/tmp/proteus-stress";
    const int iters = argc > 2 ? std::atoi(argv[2]) : 3000;
    CHECK(proteus_testing_use_fake_backend(1));
    CHECK(proteus_testing_fake_control(0, 1));   // 1 ms compiles: async paths overlap
    proteus_config c;
    CHECK(proteus_config_default(&c));
    c.device = 0;
    c.cache_dir = dir;
    c.async_workers = 3;
    c.max_entries = 64;
    c.max_disk_bytes = 256 * 1024;
    CHECK(proteus_init(&c));

    static char generic_token[3];
    const proteus_type types[3] = {PROTEUS_PTR, PROTEUS_F32, PROTEUS_I32};
    const int ann[2] = {2, 3};
    proteus_kernel ks[3];
    for (int i = 0; i < 3; ++i) {
        std::string opt = "-DVARIANT=" + std::to_string(i);
        CHECK(proteus_register_kernel("k", kSrc, opt.c_str(), types, 3, ann, 2,
                                      i == 2 ? nullptr : &generic_token[i], &ks[i]));
    }
    CHECK(proteus_kernel_set_min_blocks(ks[1], 2));

    std::atomic<bool> done{false};
    std::atomic<uint64_t> launched{0};
    std::vector<std::thread> th;
    for (int t = 0; t < 8; ++t) {
        th.emplace_back([&, t] {
            unsigned x = 12345u + 977u * t;
            for (int i = 0; i < iters; ++i) {
                x = x * 1664525u + 1013904223u;
                const int kk = (x >> 8) % 3;
                float lr = 1.0f + static_cast<float>((x >> 12) % 50) * 0.25f;
                int n = static_cast<int>(32 + (x >> 20) % 2 * 32);
                void* y = nullptr;
                void* args[3] = {&y, &lr, &n};
                if (i % 7 == 3)   // background compile requests racing the launches
                    CHECK(proteus_prefetch(ks[kk], 1 + (x >> 24) % 2, 1, 1, 64, 1, 1, args));
                CHECK(proteus_launch(ks[kk], 1 + (x >> 24) % 2, 1, 1, 64, 1, 1, 0, nullptr, args));
                launched.fetch_add(1, std::memory_order_relaxed);
            }
        });
    }
    std::thread stats([&] {
        while (!done.load()) {
            proteus_cache_stats_t s;
            CHECK(proteus_cache_stats(0, &s));
            // LRU keeps it near the cap (inserts by 8 launchers + 3 workers race with the
            // eviction of their victims, so a transient overshoot is allowed)
            if (s.entries > 2 * c.max_entries) {
                std::fprintf(stderr, "entries %llu over cap\n", (unsigned long long)s.entries);
                std::exit(3);
            }
            std::this_thread::sleep_for(std::chrono::microseconds(200));
        }
    });
    std::thread clearer([&] {   // clears while the launchers run
        for (int i = 0; i < 4 && !done.load(); ++i) {
            std::this_thread::sleep_for(std::chrono::milliseconds(2));
            CHECK(proteus_cache_clear(0, 1, 0));
        }
    });
    for (auto& t : th) t.join();
    clearer.join();
    // a last single-threaded stretch after every clear: all counters are fresh
    for (int i = 0; i < 400; ++i) {
        float lr = 1.0f + static_cast<float>(i % 80) * 0.25f;
        int n = 32;
        void* y = nullptr;
        void* args[3] = {&y, &lr, &n};
        CHECK(proteus_launch(ks[i % 2], 1, 1, 1, 64, 1, 1, 0, nullptr, args));
        launched.fetch_add(1, std::memory_order_relaxed);
    }
    done = true;
    stats.join();
    CHECK(proteus_wait_idle());
    proteus_cache_stats_t s;
    CHECK(proteus_cache_stats(0, &s));
    proteus_fake_counts_t f;
    CHECK(proteus_testing_fake_counts(&f));
    std::printf("launched %llu  stats: launches %llu mem_hits %llu disk_hits %llu misses %llu "
                "compiles %llu generic %llu evictions %llu disk_evictions %llu entries %llu | "
                "fake: compiles %llu spec %llu generic %llu\n",
                (unsigned long long)launched.load(), (unsigned long long)s.launches,
                (unsigned long long)s.mem_hits, (unsigned long long)s.disk_hits,
                (unsigned long long)s.misses, (unsigned long long)s.compiles,
                (unsigned long long)s.generic_launches, (unsigned long long)s.evictions,
                (unsigned long long)s.disk_evictions, (unsigned long long)s.entries,
                (unsigned long long)f.compiles, (unsigned long long)f.spec_launches,
                (unsigned long long)f.generic_launches);
    // every launch launched exactly one function (the clear resets counters, so compare
    // the backend's own counts, which are never reset)
    if (f.spec_launches + f.generic_launches != launched.load()) {
        std::fprintf(stderr, "launch accounting mismatch\n");
        return 4;
    }
    // the last stretch (after the final clear) exercised every path
    if (s.mem_hits == 0 || s.evictions == 0 || s.generic_launches == 0 || s.disk_hits == 0 ||
        s.compiles == 0) {
        std::fprintf(stderr, "a cache path was not exercised\n");
        return 6;
    }
    if (s.entries > c.max_entries) {
        std::fprintf(stderr, "entries above cap after idle\n");
        return 5;
    }
    CHECK(proteus_finalize());

    // Phase 2: the IR-level path (PROTEUS_F_IR) under the same concurrency -- the shared
    // kernel-IR cache (one LTO-IR compile per kernel/block shape, waited on by concurrent
    // misses), constants modules and links from 8 launchers and 3 workers, clears racing
    // module loads (fake load delay), then a finalize that drops the IR cache.
    CHECK(proteus_testing_fake_load_delay(1));
    c.flags |= PROTEUS_F_IR;
    CHECK(proteus_init(&c));
    for (int i = 0; i < 3; ++i) {
        std::string opt = "-DVARIANT=" + std::to_string(i);
        CHECK(proteus_register_kernel("k", kSrc, opt.c_str(), types, 3, ann, 2,
                                      i == 2 ? nullptr : &generic_token[i], &ks[i]));
    }
    proteus_fake_counts_t f0;
    CHECK(proteus_testing_fake_counts(&f0));
    std::atomic<uint64_t> launched2{0};
    th.clear();
    for (int t = 0; t < 8; ++t) {
        th.emplace_back([&, t] {
            unsigned x = 777u + 131u * t;
            for (int i = 0; i < iters / 4; ++i) {
                x = x * 1664525u + 1013904223u;
                const int kk = (x >> 8) % 3;
                float lr = 2.0f + static_cast<float>((x >> 12) % 40) * 0.5f;
                int n = 32;
                void* y = nullptr;
                void* args[3] = {&y, &lr, &n};
                CHECK(proteus_launch(ks[kk], 1 + (x >> 24) % 2, 1, 1, 64 * (1 + (x >> 28) % 2), 1,
                                     1, 0, nullptr, args));
                launched2.fetch_add(1, std::memory_order_relaxed);
            }
        });
    }
    std::thread clearer2([&] {
        for (int i = 0; i < 3; ++i) {
            std::this_thread::sleep_for(std::chrono::milliseconds(3));
            CHECK(proteus_cache_clear(0, 1, 0));
        }
    });
    for (auto& t : th) t.join();
    clearer2.join();
    CHECK(proteus_wait_idle());
    CHECK(proteus_cache_stats(0, &s));
    proteus_fake_counts_t f1;
    CHECK(proteus_testing_fake_counts(&f1));
    std::printf("IR phase: launched %llu  links %llu  ir/constants compiles %llu  "
                "bad unloads %llu  live modules %llu\n",
                (unsigned long long)launched2.load(), (unsigned long long)(f1.links - f0.links),
                (unsigned long long)(f1.ir_compiles - f0.ir_compiles),
                (unsigned long long)f1.bad_unloads, (unsigned long long)f1.live_modules);
    if (f1.links == f0.links || f1.ir_compiles == f0.ir_compiles) {
        std::fprintf(stderr, "the IR path was not exercised\n");
        return 7;
    }
    if (f1.spec_launches + f1.generic_launches - f0.spec_launches - f0.generic_launches !=
        launched2.load()) {
        std::fprintf(stderr, "IR phase: launch accounting mismatch\n");
        return 8;
    }
    if (f1.bad_unloads != 0) {
        std::fprintf(stderr, "a module was unloaded twice\n");
        return 9;
    }
    CHECK(proteus_finalize());
    CHECK(proteus_testing_fake_counts(&f1));
    if (f1.live_modules != 0) {
        std::fprintf(stderr, "modules leaked: %llu\n", (unsigned long long)f1.live_modules);
        return 10;
    }
    std::printf("stress ok\n");
    return 0;
}
