// stencil4_smem.cu -- 13-point 4th-order 3D stencil, fp64 (CFG 2; SW4CK-shaped, PAPER.md:1
// P@45192-45829, operator per DESIGN.md R-st-1):
//   interior: s1 = u[x-1]+u[x+1]+u[y-1]+u[y+1]+u[z-1]+u[z+1]  (this order)
//             s2 = same at distance 2;   w = a0 u + a1 s1 + a2 s2
//   global 2-cell Dirichlet frame: w = u.
//
// Parameters (1-based): 1 u  2 w  3 nx  4 ny  5 nzl  6 k_begin  7 k_end  8 kg0  9 nzg
//                       10 a0  11 a1  12 a2.      Annotated: 3, 4, 5, 9, 10, 11, 12.
// Local slab layout (one rank of a z-slab decomposition):
//   nzl + 4 planes of ny*nx doubles, x fastest; planes 0-1 = lower halo, 2..nzl+1 owned,
//   nzl+2..nzl+3 = upper halo.  Local plane kl has global z = kg0 + kl - 2 (nzg planes
//   in total).  The kernel updates local planes [k_begin, k_end).
//
// This is the portable variant (any nx; v1 of the bench kernel, see profiles/r01): the
// TMA variant stencil4.cu needs nx*8 % 16 == 0 for its tensor map.
// Design (B200, HBM-bound at 16 B/point/sweep): block = TX x TY threads over an x-y tile,
// marching in z over a chunk of planes (gridDim.z chunks).  Each thread keeps the 5
// z-values of its column in registers (z-queue); the current plane is staged in shared
// memory with a 2-point halo so x/y neighbours come from smem; u is read from HBM once
// per point (halo reads hit L2), w written once, both coalesced (rows of 32 doubles).
#include "proteus_device.h"

extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void stencil4_smem(const double* __restrict__ u, double* __restrict__ w, int nx_rt, int ny_rt,
              int nzl_rt, int k_begin, int k_end, int kg0, int nzg_rt, double a0_rt,
              double a1_rt, double a2_rt) {
    extern __shared__ double tile[];   // (TY + 4) rows x (TX + 4) cols
    const int nx = PROTEUS_SPEC(3, nx_rt);
    const int ny = PROTEUS_SPEC(4, ny_rt);
    const int nzl = PROTEUS_SPEC(5, nzl_rt);
    const int nzg = PROTEUS_SPEC(9, nzg_rt);
    const double a0 = PROTEUS_SPEC(10, a0_rt);
    const double a1 = PROTEUS_SPEC(11, a1_rt);
    const double a2 = PROTEUS_SPEC(12, a2_rt);
    (void)nzl;
    const int TX = PROTEUS_BLOCKDIM_X;
    const int TY = PROTEUS_BLOCKDIM_Y;
    const int SW = TX + 4;   // smem row pitch
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int i = blockIdx.x * TX + tx;
    const int j = blockIdx.y * TY + ty;
    const long long sxy = (long long)nx * ny;

    // z-chunk of this block
    const int nplanes = k_end - k_begin;
    const int chunk = (nplanes + PROTEUS_GRIDDIM_Z - 1) / PROTEUS_GRIDDIM_Z;
    const int k0 = k_begin + blockIdx.z * chunk;
    const int k1 = min(k0 + chunk, k_end);
    if (k0 >= k1) return;

    const bool in = (i < nx) && (j < ny);
    const bool xy_int = (i >= 2) && (i <= nx - 3) && (j >= 2) && (j <= ny - 3);
    const long long col = (long long)j * nx + i;

    // z-queue: q0..q4 = u at planes k-2 .. k+2 of this column
    double q0 = 0, q1 = 0, q2 = 0, q3 = 0, q4 = 0;
    if (in) {
        q0 = u[(k0 - 2) * sxy + col];
        q1 = u[(k0 - 1) * sxy + col];
        q2 = u[(k0)*sxy + col];
        q3 = u[(k0 + 1) * sxy + col];
    }
    double* srow = tile + (ty + 2) * SW + (tx + 2);

    for (int k = k0; k < k1; ++k) {
        const long long pk = (long long)k * sxy;
        if (in) q4 = u[pk + 2 * sxy + col];
        // stage plane k: centre from the queue, x/y halos from global (L2)
        srow[0] = q2;
        if (tx < 2) {
            const int il = i - 2, ir = i + TX;
            srow[-2] = (il >= 0 && j < ny) ? u[pk + (long long)j * nx + il] : 0.0;
            srow[TX] = (ir < nx && j < ny) ? u[pk + (long long)j * nx + ir] : 0.0;
        }
        if (ty < 2) {
            const int jb = j - 2, jt = j + TY;
            srow[-2 * SW] = (jb >= 0 && i < nx) ? u[pk + (long long)jb * nx + i] : 0.0;
            srow[TY * SW] = (jt < ny && i < nx) ? u[pk + (long long)jt * nx + i] : 0.0;
        }
        __syncthreads();
        if (in) {
            const int zg = kg0 + k - 2;
            double r = q2;
            if (xy_int && zg >= 2 && zg <= nzg - 3) {
                double s1 = srow[-1];
                s1 = s1 + srow[1];
                s1 = s1 + srow[-SW];
                s1 = s1 + srow[SW];
                s1 = s1 + q1;
                s1 = s1 + q3;
                double s2 = srow[-2];
                s2 = s2 + srow[2];
                s2 = s2 + srow[-2 * SW];
                s2 = s2 + srow[2 * SW];
                s2 = s2 + q0;
                s2 = s2 + q4;
                r = a0 * q2 + a1 * s1 + a2 * s2;
            }
            w[pk + col] = r;
        }
        __syncthreads();
        q0 = q1;
        q1 = q2;
        q2 = q3;
        q3 = q4;
    }
}
