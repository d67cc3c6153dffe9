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

// ---- per-block cursors: block b owns lookups [b*C, (b+1)*C); shared-memory atomics only
__global__ void __launch_bounds__(1024, 1) bin_pb(unsigned long long seed, unsigned long long L, int n_mat,
                                                  const double* __restrict__ cum, unsigned* __restrict__ counts_pb) {
    extern __shared__ unsigned hist_pb[];
    unsigned* hist = hist_pb;
    const int nb = n_mat * XS_EBINS;
    for (int k = threadIdx.x; k < nb; k += blockDim.x) hist[k] = 0;
    __syncthreads();
    const unsigned long long C = (L + gridDim.x - 1) / gridDim.x;
    const unsigned long long i0 = blockIdx.x * C, i1 = min(L, i0 + C);
    for (unsigned long long i = i0 + threadIdx.x; i < i1; i += blockDim.x) {
        int mat;
        atomicAdd(&hist[xs_key(seed, i, cum, n_mat, &mat)], 1u);
    }
    __syncthreads();
    unsigned* out = counts_pb + (size_t)blockIdx.x * nb;
    for (int k = threadIdx.x; k < nb; k += blockDim.x) out[k] = hist[k];
}
// per key: exclusive prefix over blocks (to a separate array) and the key total; rows loaded
// 16 at a time so that 16 loads are in flight per thread
__global__ void colscan_pb2(int nblk, int nb, const unsigned* __restrict__ counts_pb,
                            unsigned* __restrict__ colpre, unsigned* __restrict__ totals) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nb) return;
    unsigned run = 0;
    int b = 0;
    for (; b + 16 <= nblk; b += 16) {
        unsigned c[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) c[j] = __ldg(&counts_pb[(size_t)(b + j) * nb + k]);
#pragma unroll
        for (int j = 0; j < 16; ++j) { colpre[(size_t)(b + j) * nb + k] = run; run += c[j]; }
    }
    for (; b < nblk; ++b) {
        const unsigned c = __ldg(&counts_pb[(size_t)b * nb + k]);
        colpre[(size_t)b * nb + k] = run;
        run += c;
    }
    totals[k] = run;
}
// per key: exclusive prefix over blocks (in place) and the key total
__global__ void colscan_pb(int nblk, int nb, unsigned* __restrict__ counts_pb, unsigned* __restrict__ totals) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nb) return;
    unsigned run = 0;
    for (int b = 0; b < nblk; ++b) {
        const unsigned c = counts_pb[(size_t)b * nb + k];
        counts_pb[(size_t)b * nb + k] = run;
        run += c;
    }
    totals[k] = run;
}
__global__ void __launch_bounds__(1024, 1) scatter_pb(unsigned long long seed, unsigned long long L, int n_mat,
                                                      const double* __restrict__ cum, const unsigned* __restrict__ base,
                                                      const unsigned* __restrict__ colpre, unsigned* __restrict__ perm) {
    extern __shared__ unsigned cur[];
    const int nb = n_mat * XS_EBINS;
    const unsigned* cp = colpre + (size_t)blockIdx.x * nb;
    for (int k = threadIdx.x; k < nb; k += blockDim.x) cur[k] = base[k] + cp[k];
    __syncthreads();
    const unsigned long long C = (L + gridDim.x - 1) / gridDim.x;
    const unsigned long long i0 = blockIdx.x * C, i1 = min(L, i0 + C);
    for (unsigned long long i = i0 + threadIdx.x; i < i1; i += blockDim.x) {
        int mat;
        const int key = xs_key(seed, i, cum, n_mat, &mat);
        perm[atomicAdd(&cur[key], 1u)] = static_cast<unsigned>(i) | (static_cast<unsigned>(mat) << 28);
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
    {   // per-block cursors
        const int NBLK = 148;
        unsigned *counts_pb, *totals, *base;
        cudaMalloc(&counts_pb, (size_t)NBLK * nb * 4); cudaMalloc(&totals, nb * 4); cudaMalloc(&base, nb * 4);
        cudaMemset(totals, 0, nb * 4);
        cudaFuncSetAttribute(bin_pb, cudaFuncAttributeMaxDynamicSharedMemorySize, nb * 4);
        cudaFuncSetAttribute(scatter_pb, cudaFuncAttributeMaxDynamicSharedMemorySize, nb * 4);
        float t[4] = {0, 0, 0, 0};
        cudaEvent_t e[5]; for (auto& x : e) cudaEventCreate(&x);
        for (int r = 0; r < 20; ++r) {
            cudaEventRecord(e[0]);
            bin_pb<<<NBLK, 1024, nb * 4>>>(seed, L, n_mat, cum, counts_pb);
            cudaEventRecord(e[1]);
            colscan_pb<<<(nb + 255) / 256, 256>>>(NBLK, nb, counts_pb, totals);
            cudaEventRecord(e[2]);
            xs_scan<<<1, 1024>>>(n_mat, totals, base);   // exclusive scan of the totals (zeroes totals)
            cudaEventRecord(e[3]);
            scatter_pb<<<NBLK, 1024, nb * 4>>>(seed, L, n_mat, cum, base, counts_pb, perm);
            cudaEventRecord(e[4]);
            cudaEventSynchronize(e[4]);
            for (int j = 0; j < 4; ++j) { float ms; cudaEventElapsedTime(&ms, e[j], e[j + 1]); t[j] += ms; }
        }
        unsigned* colpre; cudaMalloc(&colpre, (size_t)NBLK * nb * 4);
        float v = 0;
        for (int r = 0; r < 20; ++r) {
            bin_pb<<<NBLK, 1024, nb * 4>>>(seed, L, n_mat, cum, counts_pb);
            cudaEventRecord(e[0]);
            colscan_pb2<<<(nb + 127) / 128, 128>>>(NBLK, nb, counts_pb, colpre, totals);
            cudaEventRecord(e[1]);
            cudaEventSynchronize(e[1]);
            float ms; cudaEventElapsedTime(&ms, e[0], e[1]); v += ms;
            xs_scan<<<1, 1024>>>(n_mat, totals, base);
        }
        printf("colscan2 (16 loads in flight, separate output) %.1f us\n", v / 20 * 1e3);
        printf("per-block: bin_pb %.1f  colscan %.1f  scan %.1f  scatter_pb %.1f  total %.1f us\n",
               t[0] / 20 * 1e3, t[1] / 20 * 1e3, t[2] / 20 * 1e3, t[3] / 20 * 1e3, (t[0] + t[1] + t[2] + t[3]) / 20 * 1e3);
        // reference: the shipped bin + scan + scatter
        float u[3] = {0, 0, 0};
        for (int r = 0; r < 20; ++r) {
            cudaEventRecord(e[0]);
            xs_bin<<<296, 512, nb * 4>>>(seed, L, n_mat, cum, counts);
            cudaEventRecord(e[1]);
            xs_scan<<<1, 1024>>>(n_mat, counts, cursors);
            cudaEventRecord(e[2]);
            xs_scatter<<<grid, block>>>(seed, L, n_mat, cum, cursors, perm);
            cudaEventRecord(e[3]);
            cudaEventSynchronize(e[3]);
            for (int j = 0; j < 3; ++j) { float ms; cudaEventElapsedTime(&ms, e[j], e[j + 1]); u[j] += ms; }
        }
        printf("shipped:   bin %.1f  scan %.1f  scatter %.1f  total %.1f us\n",
               u[0] / 20 * 1e3, u[1] / 20 * 1e3, u[2] / 20 * 1e3, (u[0] + u[1] + u[2]) / 20 * 1e3);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
