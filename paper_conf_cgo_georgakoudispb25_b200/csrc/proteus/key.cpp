// key.cpp -- specialization key, hash and the RCF/LB prelude.
//
// PAPER.md:1 §3.3 "Code caching" (P@24205-24805): the hash "jointly encod[es] (1) a
// unique module identifier bound to source code ..., (2) the kernel's symbol, and (3)
// the runtime values of specialized kernel arguments and launch bound values".
// Layout (DESIGN.md §"Specialization key"), all little-endian:
//   "PRTK" | u32 version=1 | u64 kernel_id | u32 flags | u32 minB | u8 n_annot |
//   n_annot x (u8 idx(1-based) | u8 type | u8 size | raw[size]) | u32 gx gy gz bx by bz
//   [ "G" | u8 n_glob | n_glob x (u8 len | name[len] | u64 device address) ]
// kernel_id (set at registration) binds (1) and (2); values are keyed by raw bits.  The
// optional G section (device globals bound with proteus_kernel_bind_global, by name)
// is present only when the kernel has bindings, so other keys are unchanged.
//
// "Dynamic specialization" (P@21805-23412): RCF replaces each use of an annotated
// argument by its runtime value; LB sets max threads per block to the launch's block
// size with minimum blocks per SM defaulting to 1.  Here both are a prelude of
// #defines ahead of the source; folded values are emitted as literals that reproduce
// the argument's bits exactly (hex-float for finite floats).
#include <cinttypes>
#include <cmath>
#include <cstdio>
#include <cstring>

#include "runtime.hpp"

namespace proteus {

uint64_t fnv1a64(const void* data, size_t len, uint64_t h) {
    const uint8_t* p = static_cast<const uint8_t*>(data);
    for (size_t i = 0; i < len; ++i) {
        h ^= p[i];
        h *= 0x100000001b3ull;
    }
    return h;
}

uint64_t key_map_hash(const uint8_t* p, size_t n) {
    uint64_t h = 0x9E3779B97F4A7C15ull ^ n;
    size_t i = 0;
    for (; i + 8 <= n; i += 8) {
        uint64_t w;
        std::memcpy(&w, p + i, 8);
        h = (h ^ w) * 0xBF58476D1CE4E5B9ull;
        h ^= h >> 31;
    }
    uint64_t t = 0;
    std::memcpy(&t, p + i, n - i);
    h = (h ^ t) * 0x94D049BB133111EBull;
    return h ^ (h >> 29);
}

size_t type_size(proteus_type t) {
    switch (t) {
        case PROTEUS_I32:
        case PROTEUS_U32:
        case PROTEUS_F32:
            return 4;
        case PROTEUS_I64:
        case PROTEUS_U64:
        case PROTEUS_F64:
        case PROTEUS_PTR:
            return 8;
        default:
            return 0;
    }
}

static inline void put_u32(std::vector<uint8_t>* o, uint32_t v) {
    for (int i = 0; i < 4; ++i) o->push_back(static_cast<uint8_t>(v >> (8 * i)));
}
static inline void put_u64(std::vector<uint8_t>* o, uint64_t v) {
    for (int i = 0; i < 8; ++i) o->push_back(static_cast<uint8_t>(v >> (8 * i)));
}

void build_key(const KernelDesc& k, unsigned key_flags, unsigned min_blocks,
               const LaunchDims& d, void** args, std::vector<uint8_t>* out) {
    out->clear();
    static const uint8_t magic[4] = {'P', 'R', 'T', 'K'};
    out->insert(out->end(), magic, magic + 4);
    put_u32(out, 1u);
    put_u64(out, k.kernel_id);
    put_u32(out, key_flags);
    put_u32(out, min_blocks);
    out->push_back(static_cast<uint8_t>(k.annotated.size()));
    for (int a : k.annotated) {
        const proteus_type t = k.types[a];
        const size_t sz = type_size(t);
        out->push_back(static_cast<uint8_t>(a + 1));
        out->push_back(static_cast<uint8_t>(t));
        out->push_back(static_cast<uint8_t>(sz));
        const uint8_t* v = static_cast<const uint8_t*>(args[a]);
        out->insert(out->end(), v, v + sz);   // host is little-endian (x86-64 / aarch64)
    }
    for (int i = 0; i < 3; ++i) put_u32(out, d.g[i]);
    for (int i = 0; i < 3; ++i) put_u32(out, d.b[i]);
    if (!k.globals.empty()) {   // the linked addresses are folded into the code: keyed
        out->push_back('G');
        out->push_back(static_cast<uint8_t>(k.globals.size()));
        for (const auto& g : k.globals) {
            out->push_back(static_cast<uint8_t>(g.first.size()));
            out->insert(out->end(), g.first.begin(), g.first.end());
            put_u64(out, g.second);
        }
    }
}

std::string literal_for(proteus_type t, const void* value) {
    char buf[96];
    switch (t) {
        case PROTEUS_F32: {
            float f;
            uint32_t u;
            std::memcpy(&f, value, 4);
            std::memcpy(&u, value, 4);
            if (std::isfinite(f))
                std::snprintf(buf, sizeof buf, "(%af)", static_cast<double>(f));
            else
                std::snprintf(buf, sizeof buf, "(__int_as_float(0x%08" PRIx32 "))", u);
            return buf;
        }
        case PROTEUS_F64: {
            double f;
            uint64_t u;
            std::memcpy(&f, value, 8);
            std::memcpy(&u, value, 8);
            if (std::isfinite(f))
                std::snprintf(buf, sizeof buf, "(%a)", f);
            else
                std::snprintf(buf, sizeof buf, "(__longlong_as_double(0x%016" PRIx64 "ll))", u);
            return buf;
        }
        case PROTEUS_I32: {
            int32_t v;
            std::memcpy(&v, value, 4);
            if (v == INT32_MIN) return "(-2147483647-1)";
            std::snprintf(buf, sizeof buf, "(%" PRId32 ")", v);
            return buf;
        }
        case PROTEUS_U32: {
            uint32_t v;
            std::memcpy(&v, value, 4);
            std::snprintf(buf, sizeof buf, "(%" PRIu32 "u)", v);
            return buf;
        }
        case PROTEUS_I64: {
            int64_t v;
            std::memcpy(&v, value, 8);
            if (v == INT64_MIN) return "(-9223372036854775807ll-1ll)";
            std::snprintf(buf, sizeof buf, "(%" PRId64 "ll)", v);
            return buf;
        }
        case PROTEUS_U64: {
            uint64_t v;
            std::memcpy(&v, value, 8);
            std::snprintf(buf, sizeof buf, "(%" PRIu64 "ull)", v);
            return buf;
        }
        default:
            return "";
    }
}

std::string jit_symbol(const std::string& entry, unsigned key_flags) {
    // the product mode (RCF + LB + FOLD_DIMS) is plain "__jit"; the ablation modes and the
    // IR path carry their mode, so an ncu launch list names every variant apart (§8d)
    const unsigned fold = key_flags & (PROTEUS_F_RCF | PROTEUS_F_LB | PROTEUS_F_FOLD_DIMS);
    std::string s = entry + "__jit";
    if (fold != (PROTEUS_F_RCF | PROTEUS_F_LB | PROTEUS_F_FOLD_DIMS)) {
        s += '_';
        if (!fold) s += "none";
        if (fold & PROTEUS_F_LB) s += "lb";
        if (fold & PROTEUS_F_RCF) s += "v";
        if (fold & PROTEUS_F_FOLD_DIMS) s += "d";
    }
    if (key_flags & PROTEUS_F_IR) s += "_ir";
    return s;
}

const char* const kIrSplit = "\n//@@proteus-ir-kernel@@\n";

namespace {

const char* ctype_of(proteus_type t) {
    switch (t) {
        case PROTEUS_I32: return "int";
        case PROTEUS_U32: return "unsigned";
        case PROTEUS_I64: return "long long";
        case PROTEUS_U64: return "unsigned long long";
        case PROTEUS_F32: return "float";
        case PROTEUS_F64: return "double";
        default: return nullptr;
    }
}

// Initializer of a constants-TU global reproducing the value's bits: finite values and
// integers as literal_for's exact literals, infinities as __builtin_huge_val[f]; false
// for NaN (no constant expression keeps a payload: that key takes the source path).
bool const_initializer(proteus_type t, const void* value, std::string* out) {
    if (t == PROTEUS_F32 || t == PROTEUS_F64) {
        double f;
        if (t == PROTEUS_F32) {
            float x;
            std::memcpy(&x, value, 4);
            f = x;
        } else {
            std::memcpy(&f, value, 8);
        }
        if (std::isnan(f)) return false;
        if (std::isinf(f)) {
            *out = std::string(f < 0 ? "-" : "") +
                   (t == PROTEUS_F32 ? "__builtin_huge_valf()" : "__builtin_huge_val()");
            return true;
        }
    }
    *out = literal_for(t, value);
    return true;
}

// The IR path's two translation units (PROTEUS_F_IR), or false when a value has no
// constant initializer.
bool ir_sources(const KernelDesc& k, unsigned key_flags, unsigned min_blocks,
                const LaunchDims& d, void** args, std::string* consts, std::string* kernel) {
    char buf[256];
    consts->clear();
    std::string& s = *kernel;
    s.clear();
    std::snprintf(buf, sizeof buf, "// proteus IR-level specialization of %s (flags=%u minB=%u)\n",
                  k.entry.c_str(), key_flags, min_blocks);
    s += buf;
    s += "#define PROTEUS_JIT 1\n#define PROTEUS_SELECT_ENTRY 1\n#define PROTEUS_ENTRY_" +
         k.entry + " 1\n";
    s += "#define " + k.entry + " " + jit_symbol(k.entry, key_flags) + "\n";
    if (key_flags & PROTEUS_F_RCF) {
        for (int a : k.annotated) {
            std::string init;
            if (!const_initializer(k.types[a], args[a], &init)) return false;
            std::snprintf(buf, sizeof buf,
                          "extern __device__ const %s proteus_a%d;\n#define PROTEUS_A%d_OR(x) "
                          "(proteus_a%d)\n", ctype_of(k.types[a]), a + 1, a + 1, a + 1);
            s += buf;
            std::snprintf(buf, sizeof buf, "extern __device__ const %s proteus_a%d = ",
                          ctype_of(k.types[a]), a + 1);
            *consts += buf + init + ";\n";
        }
    }
    if (key_flags & PROTEUS_F_FOLD_DIMS) {
        // block dims are literals of the kernel IR (launch bounds need them); grid dims are
        // constants of the key's module
        std::snprintf(buf, sizeof buf,
                      "#define PROTEUS_BDX %uu\n#define PROTEUS_BDY %uu\n#define PROTEUS_BDZ %uu\n",
                      d.b[0], d.b[1], d.b[2]);
        s += buf;
        static const char* const gn[3] = {"gdx", "gdy", "gdz"};
        static const char* const gm[3] = {"GDX", "GDY", "GDZ"};
        for (int i = 0; i < 3; ++i) {
            std::snprintf(buf, sizeof buf,
                          "extern __device__ const unsigned proteus_%s;\n#define PROTEUS_%s "
                          "(proteus_%s)\n", gn[i], gm[i], gn[i]);
            s += buf;
            std::snprintf(buf, sizeof buf, "extern __device__ const unsigned proteus_%s = %uu;\n",
                          gn[i], d.g[i]);
            *consts += buf;
        }
    }
    if (key_flags & PROTEUS_F_LB) {
        const unsigned long long threads =
            static_cast<unsigned long long>(d.b[0]) * d.b[1] * d.b[2];
        std::snprintf(buf, sizeof buf, "#define PROTEUS_LAUNCH_BOUNDS __launch_bounds__(%llu, %u)\n",
                      threads, min_blocks);
        s += buf;
    }
    for (const auto& g : k.globals) {
        std::snprintf(buf, sizeof buf,
                      "#define PROTEUS_GLOBAL_%s (*reinterpret_cast<decltype(&%s)>(0x%016llxull))\n",
                      g.first.c_str(), g.first.c_str(),
                      static_cast<unsigned long long>(g.second));
        s += buf;
    }
    std::snprintf(buf, sizeof buf, "#line 1 \"%s.cu\"\n", k.entry.c_str());
    s += buf;
    s += k.source;
    if (consts->empty()) *consts = "// no constants\n";
    return true;
}

}  // namespace

std::string specialized_source(const KernelDesc& k, unsigned key_flags, unsigned min_blocks,
                               const LaunchDims& d, void** args) {
    if (key_flags & PROTEUS_F_IR) {
        std::string consts, kernel;
        if (ir_sources(k, key_flags, min_blocks, d, args, &consts, &kernel))
            return consts + kIrSplit + kernel;
    }
    std::string s;
    s.reserve(k.source.size() + 1024);
    char buf[256];
    std::snprintf(buf, sizeof buf, "// proteus specialization of %s (flags=%u minB=%u)\n",
                  k.entry.c_str(), key_flags, min_blocks);
    s += buf;
    s += "#define PROTEUS_JIT 1\n";
    // multi-kernel sources compile only the launched entry (PROTEUS_KERNEL_ENABLED)
    s += "#define PROTEUS_SELECT_ENTRY 1\n#define PROTEUS_ENTRY_" + k.entry + " 1\n";
    // the specialization's symbol is <entry>__jit (every use of the entry's identifier
    // token is renamed alike), so profilers tell it from the generic AOT kernel <entry>
    s += "#define " + k.entry + " " + jit_symbol(k.entry, key_flags) + "\n";
    if (key_flags & PROTEUS_F_RCF) {
        for (int a : k.annotated) {
            std::snprintf(buf, sizeof buf, "#define PROTEUS_A%d_OR(x) ", a + 1);
            s += buf;
            s += literal_for(k.types[a], args[a]);
            s += "\n";
        }
    }
    if (key_flags & PROTEUS_F_FOLD_DIMS) {
        std::snprintf(buf, sizeof buf,
                      "#define PROTEUS_BDX %uu\n#define PROTEUS_BDY %uu\n#define PROTEUS_BDZ %uu\n"
                      "#define PROTEUS_GDX %uu\n#define PROTEUS_GDY %uu\n#define PROTEUS_GDZ %uu\n",
                      d.b[0], d.b[1], d.b[2], d.g[0], d.g[1], d.g[2]);
        s += buf;
    }
    if (key_flags & PROTEUS_F_LB) {
        const unsigned long long threads =
            static_cast<unsigned long long>(d.b[0]) * d.b[1] * d.b[2];
        std::snprintf(buf, sizeof buf, "#define PROTEUS_LAUNCH_BOUNDS __launch_bounds__(%llu, %u)\n",
                      threads, min_blocks);
        s += buf;
    }
    // device-global linking (the paper's __jit_register_var, P@19299-21805): every use of
    // a bound global refers to the AOT module's storage, so AOT and JIT code share state
    for (const auto& g : k.globals) {
        std::snprintf(buf, sizeof buf,
                      "#define PROTEUS_GLOBAL_%s (*reinterpret_cast<decltype(&%s)>(0x%016llxull))\n",
                      g.first.c_str(), g.first.c_str(),
                      static_cast<unsigned long long>(g.second));
        s += buf;
    }
    std::snprintf(buf, sizeof buf, "#line 1 \"%s.cu\"\n", k.entry.c_str());
    s += buf;
    s += k.source;
    return s;
}

}  // namespace proteus
