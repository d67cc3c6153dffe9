// hit_latency.cpp -- native measurement of the in-memory-hit launch path (SURVEY.md §8a
// A2-A5 + A10, CFG 5 "mem-hit latency us"): host time of one proteus_launch call that hits
// the in-memory cache (key build + FNV-1a-64 + map lookup + full-key compare +
// cuLaunchKernel) against a bare cuLaunchKernel of the same CUfunction, no Python in the
// loop.  The kernel is the paper's daxpy (Fig. 2) launched with N = 0, so the GPU does no
// work; the launch queue is drained (untimed) every 128 calls so the host never blocks
// on a full queue.  K distinct specializations (a = 1..K) are cycled to include the map
// with several entries.
//   hit_latency <daxpy.cu> [K=16] [reps=20000]  ->  one JSON line
#include <dlfcn.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <sstream>
#include <string>
#include <vector>

#include "proteus.h"

using clk = std::chrono::steady_clock;

static double pct(std::vector<double> v, double q) {
    std::sort(v.begin(), v.end());
    return v[static_cast<size_t>(q * (v.size() - 1))];
}

int main(int argc, char** argv) {
    if (argc < 2) {
        std::fprintf(stderr, "usage: hit_latency <daxpy.cu> [K] [reps]\n");
        return 2;
    }
    const int K = argc > 2 ? std::atoi(argv[2]) : 16;
    const int reps = argc > 3 ? std::atoi(argv[3]) : 20000;
    std::ifstream f(argv[1]);
    std::stringstream ss;
    ss << f.rdbuf();
    const std::string src = ss.str();

    void* cu = dlopen("libcuda.so.1", RTLD_NOW);
    if (!cu) {
        std::fprintf(stderr, "no libcuda\n");
        return 1;
    }
    using LaunchFn = int (*)(void*, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                             unsigned, void*, void**, void**);
    auto cuLaunchKernel = reinterpret_cast<LaunchFn>(dlsym(cu, "cuLaunchKernel"));
    auto cuCtxSynchronize = reinterpret_cast<int (*)()>(dlsym(cu, "cuCtxSynchronize"));

    proteus_config cfg;
    proteus_config_default(&cfg);
    cfg.device = 0;
    cfg.cache_dir = "";   // memory only
    if (proteus_init(&cfg) != PROTEUS_OK) {
        std::fprintf(stderr, "proteus_init: %s\n", proteus_last_error());
        return 1;
    }
    const proteus_type types[4] = {PROTEUS_F64, PROTEUS_I64, PROTEUS_PTR, PROTEUS_PTR};
    const int ann[2] = {1, 2};
    proteus_kernel k = nullptr;
    if (proteus_register_kernel("daxpy", src.c_str(), nullptr, types, 4, ann, 2, nullptr, &k) !=
        PROTEUS_OK) {
        std::fprintf(stderr, "register: %s\n", proteus_last_error());
        return 1;
    }
    double a = 1.0;
    long long n = 0;
    void* x = nullptr;
    void* y = nullptr;
    void* args[4] = {&a, &n, &x, &y};
    std::vector<void*> fns(K);
    auto t0 = clk::now();
    for (int i = 0; i < K; ++i) {   // compile the K specializations (misses)
        a = 1.0 + i;
        int state = 0;
        size_t len = 0;
        if (proteus_get_specialization(k, 1, 1, 1, 128, 1, 1, args, &fns[i], &state, nullptr, 0,
                                       &len) != PROTEUS_OK ||
            state != 1) {
            std::fprintf(stderr, "specialize: %s\n", proteus_last_error());
            return 1;
        }
    }
    const double compile_s = std::chrono::duration<double>(clk::now() - t0).count();
    cuCtxSynchronize();

    std::vector<double> hit, raw;
    hit.reserve(reps);
    raw.reserve(reps);
    for (int round = 0; round < 2; ++round) {   // round 0 = warm-up
        hit.clear();
        raw.clear();
        for (int r = 0; r < reps; ++r) {
            a = 1.0 + (r % K);
            auto s0 = clk::now();
            proteus_launch(k, 1, 1, 1, 128, 1, 1, 0, nullptr, args);
            auto s1 = clk::now();
            cuLaunchKernel(fns[r % K], 1, 1, 1, 128, 1, 1, 0, nullptr, args, nullptr);
            auto s2 = clk::now();
            hit.push_back(std::chrono::duration<double, std::micro>(s1 - s0).count());
            raw.push_back(std::chrono::duration<double, std::micro>(s2 - s1).count());
            if (r % 128 == 127) cuCtxSynchronize();
        }
        cuCtxSynchronize();
    }
    proteus_cache_stats_t st;
    proteus_cache_stats(0, &st);
    std::printf(
        "{\"K\": %d, \"reps\": %d, \"compile_s_total\": %.3f, \"hit_us_p50\": %.3f, "
        "\"hit_us_p10\": %.3f, \"hit_us_p90\": %.3f, \"raw_cuLaunchKernel_us_p50\": %.3f, "
        "\"raw_us_p10\": %.3f, \"raw_us_p90\": %.3f, \"hit_overhead_us_p50\": %.3f, "
        "\"mem_hits\": %llu, \"compiles\": %llu}\n",
        K, reps, compile_s, pct(hit, 0.5), pct(hit, 0.1), pct(hit, 0.9), pct(raw, 0.5),
        pct(raw, 0.1), pct(raw, 0.9), pct(hit, 0.5) - pct(raw, 0.5),
        static_cast<unsigned long long>(st.mem_hits), static_cast<unsigned long long>(st.compiles));
    proteus_finalize();
    return 0;
}
