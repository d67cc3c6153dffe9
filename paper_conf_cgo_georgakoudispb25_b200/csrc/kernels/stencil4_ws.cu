// stencil4_ws.cu -- 13-point 4th-order 3D stencil, fp64, TMA-fed, warp-specialized
// (CFG 2; SW4CK-shaped, PAPER.md:1 P@45192-45829; operator per DESIGN.md R-st-1):
//   interior: s1 = u[x-1]+u[x+1]+u[y-1]+u[y+1]+u[z-1]+u[z+1]  (this order)
//             s2 = same at distance 2;   w = a0 u + a1 s1 + a2 s2
//   global 2-cell Dirichlet frame: w = u.
//
// Same parameters, annotations and slab layout as stencil4.cu (1 tmap(u)  2 w  3 nx  4 ny
// 5 nzl  6 k_begin  7 k_end  8 kg0  9 nzg  10 a0  11 a1  12 a2; annotated 3,4,5,9,10,11,12),
// so one launch helper and one TMA descriptor serve both.  Differences from stencil4.cu:
//  * block = 32 x (TY + 1) threads: warps 0..TY-1 consume (each owns WS_RY rows of a
//    64-column tile, 2 columns per lane), warp TY is the producer: one lane streams the
//    halo'd plane tiles (68 x (TY*WS_RY+4) doubles) with cp.async.bulk.tensor into a ring
//    of WS_S slots;
//  * each slot has a "full" mbarrier (TMA transaction bytes) and an "empty" mbarrier that
//    the TY consumer warps arrive on when done with the plane -- no __syncthreads in the
//    z loop, so a slow warp no longer stalls the whole block and the producer refills a
//    slot as soon as the last reader leaves it (WS_S-2 planes ahead of the slowest warp);
//  * tile rows = TY*WS_RY is free (not a power of two); the defaults (TY = 4, WS_RY = 2,
//    WS_S = 6, 4 z-chunks: 512 blocks of 64 x 8 points) are the B200 sweep's best
//    (profiles/r01/tune_ws_wide.txt; the launch helper's STENCIL_WS must match WS_RY/WS_S);
//  * u's TMA loads carry an L2::evict_last policy (WS_L2HINT=1): the 2-row/2-column halo
//    of each tile plane is re-read by the neighbouring tiles' blocks shortly after.
// The z-chunking (gridDim.z) and the arithmetic are those of stencil4.cu.
#include "proteus_device.h"

#ifndef WS_RY
#define WS_RY 2   // rows per consumer thread
#endif
#ifndef WS_S
#define WS_S 6    // ring slots
#endif
#ifndef WS_L2HINT
#define WS_L2HINT 1   // TMA loads of u: 0 no hint, 1 L2::evict_last (halo rows are re-read
                      // by the neighbouring tiles' blocks), 2 evict_first
#endif

struct __align__(64) ProteusTmaDescWs {
    unsigned long long q[16];
};

__device__ __forceinline__ unsigned ws_smem_u32(const void* p) {
    return static_cast<unsigned>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void ws_mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(ws_smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void ws_mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(ws_smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void ws_mbar_arrive(unsigned long long* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ws_smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void ws_mbar_wait(unsigned long long* bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WSWAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WSWAIT_%=;\n"
        "}\n" ::"r"(ws_smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void ws_tma_load_plane(void* dst, const ProteusTmaDescWs* map,
                                                  unsigned long long* bar, int x, int y, int z,
                                                  unsigned long long pol) {
#if WS_L2HINT
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%3, %4, %5}], [%2], %6;" ::"r"(ws_smem_u32(dst)),
        "l"(reinterpret_cast<unsigned long long>(map)), "r"(ws_smem_u32(bar)), "r"(x), "r"(y), "r"(z),
        "l"(pol)
        : "memory");
#else
    (void)pol;
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(ws_smem_u32(dst)),
        "l"(reinterpret_cast<unsigned long long>(map)), "r"(ws_smem_u32(bar)), "r"(x), "r"(y), "r"(z)
        : "memory");
#endif
}

__device__ __forceinline__ double ws_point(double c, double xm2, double xm1, double xp1,
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

// One sweep over local planes [k_begin, k_end).  P2P: the results of the owned boundary
// planes {2, 3} are also stored to peer_lo (plane nzl+2 of rank r-1's slab) and those of
// {nzl, nzl+1} to peer_hi (plane 0 of rank r+1's slab), when non-null.
template <bool P2P>
__device__ __forceinline__ void ws_sweep(const ProteusTmaDescWs& tmap, double* __restrict__ w,
                                         double* __restrict__ peer_lo,
                                         double* __restrict__ peer_hi, const int nx,
                                         const int ny, const int nzl, const int k_begin,
                                         const int k_end, const int kg0, const int nzg,
                                         const double a0, const double a1, const double a2) {
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int PW = 68;                         // smem plane pitch (doubles): 64 + 4
    const int TY = PROTEUS_BLOCKDIM_Y - 1;         // consumer warps
    const int PH = TY * WS_RY + 4;                 // smem plane rows
    const unsigned PLANE_BYTES = static_cast<unsigned>(PW * PH) * 8u;   // one TMA box
    const int PLANE = ((PW * PH + 15) / 16) * 16;  // slot stride: 128-B aligned TMA dst
    double* ring = reinterpret_cast<double*>(smem);
    unsigned long long* full = reinterpret_cast<unsigned long long*>(smem + WS_S * PLANE * 8);
    unsigned long long* empty = full + WS_S;

    const int lane = threadIdx.x, wy = threadIdx.y;
    const int i0 = blockIdx.x * 64;
    const int j0 = blockIdx.y * (TY * WS_RY);

    // z-chunk of this block: computes planes [k0, k1), needs planes [k0-2, k1+2)
    const int nplanes = k_end - k_begin;
    const int chunk = (nplanes + PROTEUS_GRIDDIM_Z - 1) / PROTEUS_GRIDDIM_Z;
    const int k0 = k_begin + blockIdx.z * chunk;
    const int k1 = min(k0 + chunk, k_end);
    if (k0 >= k1) return;
    const int pfirst = k0 - 2;   // plane p lives in slot (p - pfirst) % WS_S
    const int plast = k1 + 1;

    if (wy == 0 && lane == 0) {
        for (int s = 0; s < WS_S; ++s) {
            ws_mbar_init(&full[s], 1);
            ws_mbar_init(&empty[s], static_cast<unsigned>(TY));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    // programmatic dependent launch: the prologue above overlapped the previous sweep;
    // u (its output) may be read and w (its input) written only after it completed
    PROTEUS_PDL_WAIT();
    PROTEUS_PDL_TRIGGER();

    if (wy == TY) {   // ---------------------------------------------------- producer warp
        if (lane == 0) {
            unsigned long long pol = 0;
#if WS_L2HINT == 1
            asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
#elif WS_L2HINT == 2
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
#endif
            for (int p = pfirst; p <= plast; ++p) {
                const int n = p - pfirst, s = n % WS_S;
                if (n >= WS_S) ws_mbar_wait(&empty[s], static_cast<unsigned>((n / WS_S - 1) & 1));
                ws_mbar_expect_tx(&full[s], PLANE_BYTES);
                ws_tma_load_plane(ring + s * PLANE, &tmap, &full[s], i0 - 2, j0 - 2, p, pol);
            }
        }
        return;
    }

    // ---------------------------------------------------------------- consumer warps
    const int i = i0 + 2 * lane;           // this lane's columns i, i+1
    const int jr0 = j0 + wy * WS_RY;       // first of this thread's rows
    const int cbase = (wy * WS_RY + 2) * PW + 2 * lane + 2;   // even => 16-B aligned
    auto wait_plane = [&](int p) {
        const int n = p - pfirst;
        ws_mbar_wait(&full[n % WS_S], static_cast<unsigned>((n / WS_S) & 1));
        return ring + (n % WS_S) * PLANE;
    };
    auto release_plane = [&](int p) {
        __syncwarp();
        if (lane == 0) ws_mbar_arrive(&empty[(p - pfirst) % WS_S]);
    };
    auto ld2 = [](const double* p) { return *reinterpret_cast<const double2*>(p); };

    double2 q0[WS_RY], q1[WS_RY], q2[WS_RY], q3[WS_RY], q4[WS_RY];
    {
        const double* P0 = wait_plane(k0 - 2);
        const double* P1 = wait_plane(k0 - 1);
        const double* P2 = wait_plane(k0);
        const double* P3 = wait_plane(k0 + 1);
#pragma unroll
        for (int r = 0; r < WS_RY; ++r) {
            q0[r] = ld2(P0 + cbase + r * PW);
            q1[r] = ld2(P1 + cbase + r * PW);
            q2[r] = ld2(P2 + cbase + r * PW);
            q3[r] = ld2(P3 + cbase + r * PW);
        }
    }
    release_plane(k0 - 2);
    release_plane(k0 - 1);

    const long long sxy = static_cast<long long>(nx) * ny;
    const bool xin = i < nx;                               // nx even: i+1 < nx too
    const bool xint0 = (i >= 2) && (i <= nx - 3);
    const bool xint1 = (i + 1 >= 2) && (i + 1 <= nx - 3);
    for (int k = k0; k < k1; ++k) {
        const double* Pn = wait_plane(k + 2);
#pragma unroll
        for (int r = 0; r < WS_RY; ++r) q4[r] = ld2(Pn + cbase + r * PW);
        const double* Pk = ring + ((k - pfirst) % WS_S) * PLANE;   // already waited (as k+2)
        const double2 ym2 = ld2(Pk + cbase - 2 * PW), ym1 = ld2(Pk + cbase - PW);
        const double2 yp1 = ld2(Pk + cbase + WS_RY * PW), yp2 = ld2(Pk + cbase + (WS_RY + 1) * PW);
        double2 L[WS_RY], R[WS_RY];
#pragma unroll
        for (int r = 0; r < WS_RY; ++r) {
            L[r] = ld2(Pk + cbase + r * PW - 2);   // x-2, x-1
            R[r] = ld2(Pk + cbase + r * PW + 2);   // x+2, x+3
        }
        release_plane(k);   // every smem read of plane k is in registers now
        const int zg = kg0 + k - 2;
        const bool zint = (zg >= 2) && (zg <= nzg - 3);
        double* wrow = w + static_cast<long long>(k) * sxy + static_cast<long long>(jr0) * nx + i;
#pragma unroll
        for (int r = 0; r < WS_RY; ++r) {
            const int j = jr0 + r;
            const double2 c = q2[r];
            const double2 ya1 = (r >= 1) ? q2[(r + WS_RY - 1) % WS_RY] : ym1;
            const double2 ya2 = (r >= 2) ? q2[(r + WS_RY - 2) % WS_RY] : (r == 1 ? ym1 : ym2);
            const double2 yb1 = (r + 1 < WS_RY) ? q2[(r + 1) % WS_RY] : yp1;
            const double2 yb2 = (r + 2 < WS_RY) ? q2[(r + 2) % WS_RY]
                                                : (r + 2 == WS_RY ? yp1 : yp2);
            const bool yzint = zint && j >= 2 && j <= ny - 3;
            double2 res = c;
            if (yzint && xint0)
                res.x = ws_point(c.x, L[r].x, L[r].y, c.y, R[r].x, ya2.x, ya1.x, yb1.x, yb2.x,
                                 q0[r].x, q1[r].x, q3[r].x, q4[r].x, a0, a1, a2);
            if (yzint && xint1)
                res.y = ws_point(c.y, L[r].y, c.x, R[r].x, R[r].y, ya2.y, ya1.y, yb1.y, yb2.y,
                                 q0[r].y, q1[r].y, q3[r].y, q4[r].y, a0, a1, a2);
            if (xin && j < ny) {
                const long long off = static_cast<long long>(r) * nx;
                // the slab is [nzl + 4][ny][nx]; a thread's double2 covers columns i, i + 1
                PROTEUS_CHECK_IDX(static_cast<long long>(k) * sxy + static_cast<long long>(j) * nx + i + 1,
                                  static_cast<long long>(nzl + 4) * sxy);
                *reinterpret_cast<double2*>(wrow + off) = res;
                if (P2P) {   // the halo exchange, fused: store into the neighbour's halo
                    const long long inplane = static_cast<long long>(jr0) * nx + i + off;
                    if (k < 4 && peer_lo)
                        *reinterpret_cast<double2*>(peer_lo + (k - 2) * sxy + inplane) = res;
                    if (k >= nzl && peer_hi)
                        *reinterpret_cast<double2*>(peer_hi + (k - nzl) * sxy + inplane) = res;
                }
            }
        }
#pragma unroll
        for (int r = 0; r < WS_RY; ++r) {
            q0[r] = q1[r];
            q1[r] = q2[r];
            q2[r] = q3[r];
            q3[r] = q4[r];
        }
    }
}

#if !defined(PROTEUS_SELECT_ENTRY) || defined(PROTEUS_ENTRY_stencil4_ws)
extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void stencil4_ws(const __grid_constant__ ProteusTmaDescWs tmap, double* __restrict__ w, int nx_rt,
                 int ny_rt, int nzl_rt, int k_begin, int k_end, int kg0, int nzg_rt, double a0_rt,
                 double a1_rt, double a2_rt) {
    ws_sweep<false>(tmap, w, nullptr, nullptr, PROTEUS_SPEC(3, nx_rt), PROTEUS_SPEC(4, ny_rt),
                    PROTEUS_SPEC(5, nzl_rt), k_begin, k_end, kg0, PROTEUS_SPEC(9, nzg_rt),
                    PROTEUS_SPEC(10, a0_rt), PROTEUS_SPEC(11, a1_rt), PROTEUS_SPEC(12, a2_rt));
}
#endif

// stencil4_p2p: stencil4_ws + the z-slab halo exchange fused into the store path (NEXT-2).
// Parameters 1-12 and annotations as stencil4_ws; 13 peer_lo, 14 peer_hi (device
// pointers into the neighbours' slabs, mapped with proteus_ipc_open_handle, or null at
// the global ends).  Ordering between the ranks' sweeps is the host's (stream flags).
#if !defined(PROTEUS_SELECT_ENTRY) || defined(PROTEUS_ENTRY_stencil4_p2p)
extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void stencil4_p2p(const __grid_constant__ ProteusTmaDescWs tmap, double* __restrict__ w,
                  int nx_rt, int ny_rt, int nzl_rt, int k_begin, int k_end, int kg0, int nzg_rt,
                  double a0_rt, double a1_rt, double a2_rt, double* __restrict__ peer_lo,
                  double* __restrict__ peer_hi) {
    ws_sweep<true>(tmap, w, peer_lo, peer_hi, PROTEUS_SPEC(3, nx_rt), PROTEUS_SPEC(4, ny_rt),
                   PROTEUS_SPEC(5, nzl_rt), k_begin, k_end, kg0, PROTEUS_SPEC(9, nzg_rt),
                   PROTEUS_SPEC(10, a0_rt), PROTEUS_SPEC(11, a1_rt), PROTEUS_SPEC(12, a2_rt));
}
#endif
