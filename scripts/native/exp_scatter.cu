// Where xs_scatter's time goes (experiment, not product code): the kernel as shipped vs
// its global atomics alone (coalesced write) vs its scattered perm writes alone (no
// atomics, hashed position) vs a warp-aggregated variant.  nvcc -arch=sm_100a -O3 -I<kernels>.
#include <cstdio>
#include <cuda_runtime.h>
#include "xs_lookup.cu"

__global__ void scatter_atomic_only(unsigned long long seed, unsigned long long L, int n_mat,
                                    const double* cum, unsigned* cursors, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        int mat;
        const int key = xs_key(seed, i, cum, n_mat, &mat);
        perm[i] = atomicAdd(&cursors[key], 1u);
    }
}

__global__ void scatter_write_only(unsigned long long seed, unsigned long long L, int n_mat,
                                   const double* cum, unsigned* cursors, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        int mat;
        const int key = xs_key(seed, i, cum, n_mat, &mat);
        const unsigned pos = (unsigned)(sm64(i) % L);
        perm[pos] = static_cast<unsigned>(i) | (static_cast<unsigned>(mat) << 28) | (key & 0);
    }
}

__global__ void key_only(unsigned long long seed, unsigned long long L, int n_mat,
                         const double* cum, unsigned* cursors, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        int mat;
        acc += xs_key(seed, i, cum, n_mat, &mat);
    }
    if (acc == 0x12345678u) perm[0] = acc;
}

__device__ __forceinline__ int key_intbin(unsigned long long seed, unsigned long long i,
                                          const double* __restrict__ cum, int n_mat) {
    const unsigned long long x = sm64(seed + (34ull << 40) + i);
    const int mat = xs_material(seed, i, cum, n_mat);
    return mat * XS_EBINS + (int)(x >> 52);   // = floor(u01(x) * 4096)
}

__constant__ unsigned long long c_thr[16];   // ceil(cum[m] * 2^53): r < cum[m] <=> k < thr[m]

__device__ __forceinline__ int key_int(unsigned long long seed, unsigned long long i, int n_mat) {
    const unsigned long long x = sm64(seed + (34ull << 40) + i);
    const unsigned long long k = sm64(seed + (35ull << 40) + i) >> 11;
    int mat = n_mat - 1;
    for (int m = n_mat - 1; m >= 0; --m)
        if (k < c_thr[m]) mat = m;
    return mat * XS_EBINS + (int)(x >> 52);
}

__global__ void key_only_intbin(unsigned long long seed, unsigned long long L, int n_mat,
                                const double* cum, unsigned* cursors, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride)
        acc += key_intbin(seed, i, cum, n_mat);
    if (acc == 0x12345678u) perm[0] = acc;
}

__global__ void key_only_int(unsigned long long seed, unsigned long long L, int n_mat,
                             const double* cum, unsigned* cursors, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride)
        acc += key_int(seed, i, n_mat);
    if (acc == 0x12345678u) perm[0] = acc;
}

__global__ void check_keys(unsigned long long seed, unsigned long long L, int n_mat,
                           const double* cum, unsigned* bad, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        int mat;
        const int k0 = xs_key(seed, i, cum, n_mat, &mat);
        if (k0 != key_intbin(seed, i, cum, n_mat) || k0 != key_int(seed, i, n_mat)) atomicAdd(bad, 1u);
    }
}

// scatter reading stored keys (written by a binning pass)
__global__ void bin_store_keys(unsigned long long seed, unsigned long long L, int n_mat,
                               const double* cum, unsigned* keys, unsigned* perm) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        int mat;
        keys[i] = xs_key(seed, i, cum, n_mat, &mat);
    }
}
__global__ void scatter_from_keys(unsigned long long seed, unsigned long long L, int n_mat,
                                  const double* keys_d, unsigned* cursors, unsigned* perm) {
    const unsigned* keys = reinterpret_cast<const unsigned*>(keys_d);
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < L; i += stride) {
        const unsigned key = __ldg(&keys[i]);
        const unsigned pos = atomicAdd(&cursors[key], 1u);
        perm[pos] = static_cast<unsigned>(i) | ((key / XS_EBINS) << 28);
    }
}

template <int U>
__global__ void scatter_unroll(unsigned long long seed, unsigned long long L, int n_mat,
                               const double* cum, unsigned* cursors, unsigned* perm) {
    // U independent atomics in flight per thread before their results are used
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < L; i += U * stride) {
        unsigned pos[U], val[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            int mat;
            const int key = xs_key(seed, i + u * stride, cum, n_mat, &mat);
            val[u] = static_cast<unsigned>(i + u * stride) | (static_cast<unsigned>(mat) << 28);
            pos[u] = atomicAdd(&cursors[key], 1u);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) perm[pos[u]] = val[u];
    }
    for (; i < L; i += stride) {
        int mat;
        const int key = xs_key(seed, i, cum, n_mat, &mat);
        perm[atomicAdd(&cursors[key], 1u)] = static_cast<unsigned>(i) | (static_cast<unsigned>(mat) << 28);
    }
}

typedef void (*K)(unsigned long long, unsigned long long, int, const double*, unsigned*, unsigned*);

int main() {
    const unsigned long long L = 10000000ull, seed = 0x5eedull;
    const int n_mat = 12, nb = n_mat * XS_EBINS;
    double hcum[16];
    for (int m = 0; m < n_mat; ++m) hcum[m] = (m + 1.0) / n_mat;
    double* cum; unsigned *counts, *cursors, *perm;
    cudaMalloc(&cum, sizeof hcum); cudaMemcpy(cum, hcum, sizeof hcum, cudaMemcpyHostToDevice);
    cudaMalloc(&counts, nb * 4); cudaMemset(counts, 0, nb * 4);
    cudaMalloc(&cursors, nb * 4); cudaMalloc(&perm, L * 4);
    cudaFuncSetAttribute(xs_bin, cudaFuncAttributeMaxDynamicSharedMemorySize, nb * 4);
    const int grid = 148 * 16, block = 128;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    unsigned long long thr[16];
    for (int m = 0; m < n_mat; ++m) thr[m] = (unsigned long long)__builtin_ceil(hcum[m] * 0x1p53);
    cudaMemcpyToSymbol(c_thr, thr, sizeof thr);
    unsigned* keys; cudaMalloc(&keys, L * 4);
    unsigned* bad; cudaMalloc(&bad, 4); cudaMemset(bad, 0, 4);
    check_keys<<<grid, block>>>(seed, L, n_mat, cum, bad, perm);
    unsigned hbad = 0; cudaMemcpy(&hbad, bad, 4, cudaMemcpyDeviceToHost);
    printf("key mismatches (int forms vs xs_key): %u\n", hbad);
    struct { const char* name; K k; } ks[] = {{"xs_scatter", (K)xs_scatter}, {"atomic_only", scatter_atomic_only},
                                              {"write_only", scatter_write_only}, {"key_only", key_only},
                                              {"key_intbin", key_only_intbin}, {"key_int", key_only_int},
                                              {"unroll2", scatter_unroll<2>}, {"unroll4", scatter_unroll<4>}};
    for (int rep = 0; rep < 2; ++rep)
        for (auto& x : ks) {
            float tot = 0;
            for (int r = 0; r < 20; ++r) {
                xs_bin<<<296, 512, nb * 4>>>(seed, L, n_mat, cum, counts);
                xs_scan<<<1, 1024>>>(n_mat, counts, cursors);
                cudaEventRecord(a);
                x.k<<<grid, block>>>(seed, L, n_mat, cum, cursors, perm);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b); tot += ms;
            }
            printf("%-12s %.1f us\n", x.name, tot / 20 * 1e3);
        }
    {   // stored keys: bin pass writes them, scatter reads them
        float t1 = 0, t2 = 0;
        for (int r = 0; r < 20; ++r) {
            xs_bin<<<296, 512, nb * 4>>>(seed, L, n_mat, cum, counts);
            xs_scan<<<1, 1024>>>(n_mat, counts, cursors);
            cudaEventRecord(a);
            bin_store_keys<<<grid, block>>>(seed, L, n_mat, cum, keys, perm);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b); t1 += ms;
            cudaEventRecord(a);
            scatter_from_keys<<<grid, block>>>(seed, L, n_mat, (const double*)keys, cursors, perm);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b); t2 += ms;
        }
        printf("store_keys   %.1f us (key + coalesced 4-B store, no histogram)\n", t1 / 20 * 1e3);
        printf("scatter_keys %.1f us\n", t2 / 20 * 1e3);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
