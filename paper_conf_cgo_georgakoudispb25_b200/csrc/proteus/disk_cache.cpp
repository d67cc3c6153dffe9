// disk_cache.cpp -- the persistent cache level.
//
// PAPER.md:1 §3.3 "Code caching" (P@25405-26536): a second, persistent level "designed
// to retain objects across program runs, feeding the in-memory cache ... storing each
// JIT-optimized binary in a unique file, named cache-jit-<hash>.o"; no size limit;
// users clear it by deleting files; a source change changes the module id so stale
// entries are never hit.
//
// File cache-jit-<016x hash>.cubin (DESIGN.md §"Persistent cache"):
//   "PRTC" | u32 version=1 | u32 key_len | key bytes | u64 cubin_len |
//   u64 FNV-1a-64(cubin) | cubin bytes
// The full key is stored and compared, so a 64-bit hash collision or a truncated /
// corrupted file is detected and ignored (then recompiled and rewritten).  Writes go
// to a unique temp file in the same directory followed by rename(2), so concurrent
// processes sharing one directory never observe a partial file.
#include <dirent.h>
#include <fcntl.h>
#include <sys/stat.h>
#include <sys/types.h>
#include <unistd.h>
#include <utime.h>

#include <signal.h>

#include <algorithm>
#include <atomic>

#include <cerrno>
#include <chrono>
#include <cstdio>
#include <ctime>
#include <cstring>
#include <thread>

#include "runtime.hpp"

namespace proteus {

std::string cache_file_path(const std::string& dir, uint64_t hash) {
    char name[64];
    std::snprintf(name, sizeof name, "/cache-jit-%016llx.cubin",
                  static_cast<unsigned long long>(hash));
    return dir + name;
}

bool ensure_dir(const std::string& dir, std::string* err) {
    if (dir.empty()) return true;
    std::string cur;
    size_t pos = 0;
    while (pos != std::string::npos) {
        pos = dir.find('/', pos + 1);
        cur = dir.substr(0, pos);
        if (cur.empty()) continue;
        if (mkdir(cur.c_str(), 0775) != 0 && errno != EEXIST) {
            *err = "cannot create cache dir " + cur + ": " + std::strerror(errno);
            return false;
        }
    }
    struct stat st;
    if (stat(dir.c_str(), &st) != 0 || !S_ISDIR(st.st_mode)) {
        *err = "cache dir is not a directory: " + dir;
        return false;
    }
    return true;
}

static bool read_all(const std::string& path, std::string* out) {
    FILE* f = std::fopen(path.c_str(), "rb");
    if (!f) return false;
    std::string data;
    char buf[1 << 16];
    size_t n;
    while ((n = std::fread(buf, 1, sizeof buf, f)) > 0) data.append(buf, n);
    const bool ok = !std::ferror(f);
    std::fclose(f);
    if (ok) out->swap(data);
    return ok;
}

template <typename T>
static bool take(const std::string& s, size_t* off, T* v) {
    if (*off + sizeof(T) > s.size()) return false;
    std::memcpy(v, s.data() + *off, sizeof(T));
    *off += sizeof(T);
    return true;
}

bool disk_read(const std::string& dir, uint64_t hash, const std::vector<uint8_t>& key,
               std::string* cubin, bool* reject) {
    *reject = false;
    if (dir.empty()) return false;
    std::string data;
    if (!read_all(cache_file_path(dir, hash), &data)) return false;
    size_t off = 0;
    uint32_t version = 0, klen = 0;
    uint64_t clen = 0, csum = 0;
    *reject = true;
    if (data.size() < 4 || std::memcmp(data.data(), "PRTC", 4) != 0) return false;
    off = 4;
    if (!take(data, &off, &version) || version != 1) return false;
    if (!take(data, &off, &klen) || klen != key.size()) return false;
    if (off + klen > data.size() || std::memcmp(data.data() + off, key.data(), klen) != 0)
        return false;
    off += klen;
    if (!take(data, &off, &clen) || !take(data, &off, &csum)) return false;
    if (off + clen != data.size()) return false;
    if (fnv1a64(data.data() + off, clen) != csum) return false;
    cubin->assign(data.data() + off, clen);
    *reject = false;
    utime(cache_file_path(dir, hash).c_str(), nullptr);   // LRU: a hit is a use
    return true;
}

size_t disk_write(const std::string& dir, uint64_t hash, const std::vector<uint8_t>& key,
                  const std::string& cubin) {
    if (dir.empty()) return 0;
    const std::string path = cache_file_path(dir, hash);
    char suffix[96];
    std::snprintf(suffix, sizeof suffix, ".tmp.%d.%zx", static_cast<int>(getpid()),
                  std::hash<std::thread::id>{}(std::this_thread::get_id()));
    const std::string tmp = path + suffix;
    FILE* f = std::fopen(tmp.c_str(), "wb");
    if (!f) return 0;
    const uint32_t version = 1, klen = static_cast<uint32_t>(key.size());
    const uint64_t clen = cubin.size(), csum = fnv1a64(cubin.data(), cubin.size());
    bool ok = std::fwrite("PRTC", 1, 4, f) == 4;
    ok = ok && std::fwrite(&version, 4, 1, f) == 1;
    ok = ok && std::fwrite(&klen, 4, 1, f) == 1;
    ok = ok && std::fwrite(key.data(), 1, klen, f) == klen;
    ok = ok && std::fwrite(&clen, 8, 1, f) == 1;
    ok = ok && std::fwrite(&csum, 8, 1, f) == 1;
    ok = ok && std::fwrite(cubin.data(), 1, clen, f) == clen;
    ok = (std::fclose(f) == 0) && ok;
    if (!ok || std::rename(tmp.c_str(), path.c_str()) != 0) {
        std::remove(tmp.c_str());
        return 0;
    }
    return 4 + 4 + 4 + klen + 8 + 8 + clen;
}

// Cross-process claims (R-cache-1).  A lock file cache-jit-<hash>.lock holds its owner's
// token "pid host nonce".  It is created atomically WITH that content (written to a unique
// temp file, then link(2)ed to the lock name: fails with EEXIST if a claim exists).  A
// claim is stale when its owner is a dead process on this host (kill(pid, 0) -> ESRCH;
// detected at once), or -- for an owner on another host sharing the directory, or an
// unreadable lock -- when the lock is older than kClaimStaleS.  A stale claim is taken
// over by rename(2)ing it to a unique name (only one contender's rename succeeds, so two
// waiters never delete each other's fresh claims) and claiming again; a release deletes
// the lock only if it still holds this claim's token.
static constexpr double kClaimStaleS = 120.0;

static std::string claim_path(const std::string& dir, uint64_t hash) {
    char name[64];
    std::snprintf(name, sizeof name, "/cache-jit-%016llx.lock",
                  static_cast<unsigned long long>(hash));
    return dir + name;
}

static std::string host_name() {
    char h[256] = {};
    if (gethostname(h, sizeof h - 1) != 0) return "?";
    return h;
}

static std::string unique_suffix() {
    static std::atomic<uint64_t> n{0};
    char b[96];
    std::snprintf(b, sizeof b, ".%d.%zx.%llu", static_cast<int>(getpid()),
                  std::hash<std::thread::id>{}(std::this_thread::get_id()),
                  static_cast<unsigned long long>(n.fetch_add(1)));
    return b;
}

static bool read_small(const std::string& path, std::string* out) {
    FILE* f = std::fopen(path.c_str(), "rb");
    if (!f) return false;
    char buf[512];
    const size_t n = std::fread(buf, 1, sizeof buf - 1, f);
    std::fclose(f);
    out->assign(buf, n);
    return true;
}

static bool claim_stale(const std::string& lock) {
    struct stat st;
    if (stat(lock.c_str(), &st) != 0) return false;
    std::string tok;
    if (read_small(lock, &tok)) {
        long pid = 0;
        char host[256] = {};
        if (std::sscanf(tok.c_str(), "%ld %255s", &pid, host) == 2 && pid > 0 &&
            host_name() == host)
            return kill(static_cast<pid_t>(pid), 0) != 0 && errno == ESRCH;
    }
    return difftime(time(nullptr), st.st_mtime) > kClaimStaleS;
}

int disk_claim(const std::string& dir, uint64_t hash, std::string* token) {
    if (dir.empty()) return -1;
    const std::string lock = claim_path(dir, hash);
    char tok[400];
    std::snprintf(tok, sizeof tok, "%d %s %s\n", static_cast<int>(getpid()), host_name().c_str(),
                  unique_suffix().c_str());
    const std::string tmp = lock + ".new" + unique_suffix();
    for (int attempt = 0; attempt < 3; ++attempt) {
        FILE* f = std::fopen(tmp.c_str(), "wb");
        if (!f) return -1;
        const bool ok = std::fputs(tok, f) >= 0;
        if (std::fclose(f) != 0 || !ok) {
            std::remove(tmp.c_str());
            return -1;
        }
        const int r = link(tmp.c_str(), lock.c_str());
        const int err = errno;
        std::remove(tmp.c_str());
        if (r == 0) {
            *token = tok;
            return 1;
        }
        if (err != EEXIST) return -1;
        if (!claim_stale(lock)) return 0;
        // take the dead claimant's lock out of the way atomically, then claim again
        const std::string aside = lock + ".stale" + unique_suffix();
        if (std::rename(lock.c_str(), aside.c_str()) == 0) std::remove(aside.c_str());
    }
    return 0;
}

void disk_release(const std::string& dir, uint64_t hash, const std::string& token) {
    if (dir.empty()) return;
    const std::string lock = claim_path(dir, hash);
    std::string cur;
    if (!read_small(lock, &cur) || cur != token) return;   // no longer ours (taken over)
    const std::string aside = lock + ".rel" + unique_suffix();
    if (std::rename(lock.c_str(), aside.c_str()) != 0) return;
    std::string moved;
    if (read_small(aside, &moved) && moved != token)   // raced with a takeover + re-claim
        (void)std::rename(aside.c_str(), lock.c_str());
    else
        std::remove(aside.c_str());
}

bool disk_wait_claim(const std::string& dir, uint64_t hash, double timeout_ms) {
    const std::string lock = claim_path(dir, hash), file = cache_file_path(dir, hash);
    struct stat st;
    const auto t0 = std::chrono::steady_clock::now();
    for (;;) {
        if (stat(file.c_str(), &st) == 0) return true;
        if (stat(lock.c_str(), &st) != 0 || claim_stale(lock)) return stat(file.c_str(), &st) == 0;
        const double el = std::chrono::duration<double, std::milli>(
                              std::chrono::steady_clock::now() - t0).count();
        if (el > timeout_ms) return false;
        std::this_thread::sleep_for(std::chrono::microseconds(500));
    }
}

int disk_clear(const std::string& dir) {
    if (dir.empty()) return 0;
    DIR* d = opendir(dir.c_str());
    if (!d) return 0;
    int n = 0;
    while (dirent* e = readdir(d)) {
        if (std::strncmp(e->d_name, "cache-jit-", 10) == 0) {
            if (std::remove((dir + "/" + e->d_name).c_str()) == 0) ++n;
        }
    }
    closedir(d);
    return n;
}

int disk_enforce_cap(const std::string& dir, uint64_t max_bytes, const std::string& keep) {
    if (dir.empty() || !max_bytes) return 0;
    DIR* d = opendir(dir.c_str());
    if (!d) return 0;
    struct F {
        std::string path;
        uint64_t size;
        struct timespec mtime;
    };
    std::vector<F> files;
    uint64_t total = 0;
    while (dirent* e = readdir(d)) {
        if (std::strncmp(e->d_name, "cache-jit-", 10) != 0) continue;
        const std::string p = dir + "/" + e->d_name;
        if (p.find(".tmp.") != std::string::npos) continue;
        if (p.find(".lock") != std::string::npos) continue;   // claims and their temp names
        struct stat st;
        if (stat(p.c_str(), &st) != 0) continue;
        files.push_back({p, static_cast<uint64_t>(st.st_size), st.st_mtim});
        total += static_cast<uint64_t>(st.st_size);
    }
    closedir(d);
    if (total <= max_bytes) return 0;
    std::sort(files.begin(), files.end(), [](const F& a, const F& b) {
        return a.mtime.tv_sec != b.mtime.tv_sec ? a.mtime.tv_sec < b.mtime.tv_sec
                                                : a.mtime.tv_nsec < b.mtime.tv_nsec;
    });
    int n = 0;
    for (const F& f : files) {
        if (total <= max_bytes) break;
        if (f.path == keep) continue;
        if (std::remove(f.path.c_str()) == 0) {
            total -= f.size;
            ++n;
        }
    }
    return n;
}

}  // namespace proteus
