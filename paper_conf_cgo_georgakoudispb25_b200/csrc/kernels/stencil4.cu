// stencil4.cu -- 13-point 4th-order 3D stencil, fp64, TMA-fed (CFG 2; SW4CK-shaped,
// PAPER.md:1 P@45192-45829, operator per DESIGN.md R-st-1):
//   interior: s1 = u[x-1]+u[x+1]+u[y-1]+u[y+1]+u[z-1]+u[z+1]  (this order)
//             s2 = same at distance 2;   w = a0 u + a1 s1 + a2 s2
//   global 2-cell Dirichlet frame: w = u.
//
// Parameters (1-based): 1 tmap(u)  2 w  3 nx  4 ny  5 nzl  6 k_begin  7 k_end  8 kg0
//                       9 nzg  10 a0  11 a1  12 a2.    Annotated: 3, 4, 5, 9, 10, 11, 12.
// tmap is a 3-D TMA descriptor (CUtensorMap, by value, __grid_constant__) over the slab u
// [nzl+4][ny][nx] fp64 with box {2*TX+4, TY*RY+4, 1}; built by proteus_encode_tensor_map.
// Slab layout as in stencil4_smem.cu: planes 0-1 / nzl+2..nzl+3 are halos, local plane kl
// has global z = kg0 + kl - 2; the kernel updates local planes [k_begin, k_end).  nx even.
//
// B200 design (HBM-bound, 16 B/point/sweep; the limiter after TMA is smem bandwidth):
//  * block = TX x TY threads over an x-y tile of (2 TX) x (TY RY) points; each thread owns
//    a 2-column x RY-row patch (double2 everywhere) and marches in z over gridDim.z chunks;
//  * one elected thread streams whole halo'd plane tiles HBM/L2 -> smem with
//    cp.async.bulk.tensor into a ring of ST_S slots completed on mbarriers (transaction
//    bytes), keeping ST_S-3 planes in flight per block;
//  * z-neighbours come from a 5-deep register queue, x/y neighbours inside the patch from
//    registers, the rest from smem with 16-B LDS: 40 B of smem reads per point (profiles/
//    r01: the 1-column version needed 56 B and was smem-bound at 82% L1 throughput);
//  * w is written once with coalesced 16-B stores (512 B per warp row).
#include "proteus_device.h"

#ifndef ST_RY
#define ST_RY 2   // rows per thread
#endif
#ifndef ST_S
#define ST_S 6    // ring slots (planes resident or in flight)
#endif
#ifndef ST_WSTORE
#define ST_WSTORE 0   // 0: st.global (write-back), 1: st.global.cs (streaming, evict-first)
#endif
#ifndef ST_L2HINT
#define ST_L2HINT 2   // TMA loads: 0 no hint, 1 evict_first, 2 evict_last (B200: 47.2 -> 46.0 us)
#endif

struct __align__(64) ProteusTmaDesc {
    unsigned long long q[16];
};

__device__ __forceinline__ unsigned smem_u32(const void* p) {
    return static_cast<unsigned>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void tma_load_plane(void* dst, const ProteusTmaDesc* map,
                                               unsigned long long* bar, int x, int y, int z) {
#if ST_L2HINT
    unsigned long long pol;
#if ST_L2HINT == 1
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
#else
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
#endif
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%3, %4, %5}], [%2], %6;" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<unsigned long long>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y), "r"(z),
        "l"(pol)
        : "memory");
#else
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<unsigned long long>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y), "r"(z)
        : "memory");
#endif
}

__device__ __forceinline__ double st4_point(double c, double xm2, double xm1, double xp1,
                                            double xp2, double ym2, double ym1, double yp1,
                                            double yp2, double zm2, double zm1, double zp1,
                                            double zp2, double a0, double a1, double a2) {
    double s1 = xm1;
    s1 = s1 + xp1;
    s1 = s1 + ym1;
    s1 = s1 + yp1;
    s1 = s1 + zm1;
    s1 = s1 + zp1;
    double s2 = xm2;
    s2 = s2 + xp2;
    s2 = s2 + ym2;
    s2 = s2 + yp2;
    s2 = s2 + zm2;
    s2 = s2 + zp2;
    return a0 * c + a1 * s1 + a2 * s2;
}

extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void stencil4(const __grid_constant__ ProteusTmaDesc tmap, double* __restrict__ w, int nx_rt,
              int ny_rt, int nzl_rt, int k_begin, int k_end, int kg0, int nzg_rt, double a0_rt,
              double a1_rt, double a2_rt) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int nx = PROTEUS_SPEC(3, nx_rt);
    const int ny = PROTEUS_SPEC(4, ny_rt);
    (void)PROTEUS_SPEC(5, nzl_rt);
    const int nzg = PROTEUS_SPEC(9, nzg_rt);
    const double a0 = PROTEUS_SPEC(10, a0_rt);
    const double a1 = PROTEUS_SPEC(11, a1_rt);
    const double a2 = PROTEUS_SPEC(12, a2_rt);
    const int TX = PROTEUS_BLOCKDIM_X;
    const int TY = PROTEUS_BLOCKDIM_Y;
    const int PW = 2 * TX + 4;             // smem plane pitch (doubles, even)
    const int PH = TY * ST_RY + 4;         // smem plane rows
    const unsigned PLANE_BYTES = static_cast<unsigned>(PW * PH) * 8u;   // one TMA box
    const int PLANE = ((PW * PH + 15) / 16) * 16;   // slot stride: 128-B aligned TMA dst
    double* ring = reinterpret_cast<double*>(smem);
    unsigned long long* bars = reinterpret_cast<unsigned long long*>(smem + ST_S * PLANE * 8);

    const int tx = threadIdx.x, ty = threadIdx.y;
    const int tid = ty * TX + tx;
    const int i0 = blockIdx.x * (2 * TX);
    const int j0 = blockIdx.y * (TY * ST_RY);
    const int i = i0 + 2 * tx;             // this thread's columns i, i+1
    const int jr0 = j0 + ty * ST_RY;       // first of this thread's rows

    // z-chunk of this block: computes planes [k0, k1), needs planes [k0-2, k1+2)
    const int nplanes = k_end - k_begin;
    const int chunk = (nplanes + PROTEUS_GRIDDIM_Z - 1) / PROTEUS_GRIDDIM_Z;
    const int k0 = k_begin + blockIdx.z * chunk;
    const int k1 = min(k0 + chunk, k_end);
    if (k0 >= k1) return;
    const int pfirst = k0 - 2;             // ring holds planes pfirst.. ; slot = (p - pfirst) % S
    const int plast = k1 + 1;              // last plane needed

    if (tid == 0) {
        for (int s = 0; s < ST_S; ++s) mbar_init(&bars[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0) {
        for (int s = 0; s < ST_S && pfirst + s <= plast; ++s) {
            mbar_expect_tx(&bars[s], PLANE_BYTES);
            tma_load_plane(ring + s * PLANE, &tmap, &bars[s], i0 - 2, j0 - 2, pfirst + s);
        }
    }

    // smem offset of this thread's first-row, first-column centre (even => 16-B aligned)
    const int cbase = (ty * ST_RY + 2) * PW + 2 * tx + 2;
    auto wait_plane = [&](int p) {
        const int n = p - pfirst;
        mbar_wait(&bars[n % ST_S], static_cast<unsigned>((n / ST_S) & 1));
        return ring + (n % ST_S) * PLANE;
    };
    auto ld2 = [](const double* p) { return *reinterpret_cast<const double2*>(p); };

    double2 q0[ST_RY], q1[ST_RY], q2[ST_RY], q3[ST_RY], q4[ST_RY];
    {
        const double* P0 = wait_plane(k0 - 2);
        const double* P1 = wait_plane(k0 - 1);
        const double* P2 = wait_plane(k0);
        const double* P3 = wait_plane(k0 + 1);
#pragma unroll
        for (int r = 0; r < ST_RY; ++r) {
            q0[r] = ld2(P0 + cbase + r * PW);
            q1[r] = ld2(P1 + cbase + r * PW);
            q2[r] = ld2(P2 + cbase + r * PW);
            q3[r] = ld2(P3 + cbase + r * PW);
        }
    }
    __syncthreads();   // slots of planes k0-2, k0-1 are free
    if (tid == 0) {
        for (int p = pfirst + ST_S; p < pfirst + ST_S + 2 && p <= plast; ++p) {
            const int s = (p - pfirst) % ST_S;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&bars[s], PLANE_BYTES);
            tma_load_plane(ring + s * PLANE, &tmap, &bars[s], i0 - 2, j0 - 2, p);
        }
    }

    const long long sxy = static_cast<long long>(nx) * ny;
    const bool xin = i < nx;                               // nx even: i+1 < nx too
    const bool xint0 = (i >= 2) && (i <= nx - 3);
    const bool xint1 = (i + 1 >= 2) && (i + 1 <= nx - 3);
    for (int k = k0; k < k1; ++k) {
        const double* Pn = wait_plane(k + 2);
#pragma unroll
        for (int r = 0; r < ST_RY; ++r) q4[r] = ld2(Pn + cbase + r * PW);
        const double* Pk = ring + ((k - pfirst) % ST_S) * PLANE;   // already waited (as k+2)
        // rows outside this thread's patch
        const double2 ym2 = ld2(Pk + cbase - 2 * PW), ym1 = ld2(Pk + cbase - PW);
        const double2 yp1 = ld2(Pk + cbase + ST_RY * PW), yp2 = ld2(Pk + cbase + (ST_RY + 1) * PW);
        const int zg = kg0 + k - 2;
        const bool zint = (zg >= 2) && (zg <= nzg - 3);
        double* wrow = w + static_cast<long long>(k) * sxy + static_cast<long long>(jr0) * nx + i;
#pragma unroll
        for (int r = 0; r < ST_RY; ++r) {
            const int j = jr0 + r;
            const double2 L = ld2(Pk + cbase + r * PW - 2);   // x-2, x-1
            const double2 R = ld2(Pk + cbase + r * PW + 2);   // x+2, x+3
            const double2 c = q2[r];
            const double2 ya1 = (r >= 1) ? q2[(r + ST_RY - 1) % ST_RY] : ym1;
            const double2 ya2 = (r >= 2) ? q2[(r + ST_RY - 2) % ST_RY] : (r == 1 ? ym1 : ym2);
            const double2 yb1 = (r + 1 < ST_RY) ? q2[(r + 1) % ST_RY] : yp1;
            const double2 yb2 = (r + 2 < ST_RY) ? q2[(r + 2) % ST_RY]
                                                : (r + 2 == ST_RY ? yp1 : yp2);
            const bool yzint = zint && j >= 2 && j <= ny - 3;
            double2 res = c;
            if (yzint && xint0)
                res.x = st4_point(c.x, L.x, L.y, c.y, R.x, ya2.x, ya1.x, yb1.x, yb2.x, q0[r].x,
                                  q1[r].x, q3[r].x, q4[r].x, a0, a1, a2);
            if (yzint && xint1)
                res.y = st4_point(c.y, L.y, c.x, R.x, R.y, ya2.y, ya1.y, yb1.y, yb2.y, q0[r].y,
                                  q1[r].y, q3[r].y, q4[r].y, a0, a1, a2);
            if (xin && j < ny)
#if ST_WSTORE == 1
                __stcs(reinterpret_cast<double2*>(wrow + static_cast<long long>(r) * nx), res);
#else
                *reinterpret_cast<double2*>(wrow + static_cast<long long>(r) * nx) = res;
#endif
        }
        __syncthreads();   // everyone is done with plane k's slot
        if (tid == 0 && k + ST_S <= plast) {
            const int s = (k - pfirst) % ST_S;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&bars[s], PLANE_BYTES);
            tma_load_plane(ring + s * PLANE, &tmap, &bars[s], i0 - 2, j0 - 2, k + ST_S);
        }
#pragma unroll
        for (int r = 0; r < ST_RY; ++r) {
            q0[r] = q1[r];
            q1[r] = q2[r];
            q2[r] = q3[r];
            q3[r] = q4[r];
        }
    }
}
