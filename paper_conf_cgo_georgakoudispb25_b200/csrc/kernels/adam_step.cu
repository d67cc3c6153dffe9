// adam_step.cu -- fused Adam update (CFG 1), the paper's ADAM program (Listing 1,
// PAPER.md:1 P@38745-39163; Fig. 7 discussion P@40535-41853).
//
// Parameters (1-based, as annotate("jit", ...)):
//   1 p  2 m  3 v  4 g  5 n  6 lr  7 b1  8 b2  9 eps  10 grad_scale  11 decay
//   12 mode  13 bc1  14 bc2
// Annotated: 5..11 (Listing 1's set by name minus time_step; mode stays runtime as in
// Listing 1).  bc1/bc2 = fp32(1 - b^t) are per-step runtime scalars (DESIGN.md R-adam-2).
// Update per element (DESIGN.md R-adam-1):
//   gs = g / grad_scale; m = b1 m + (1-b1) gs; v = b2 v + (1-b2) gs^2
//   mh = m / bc1; vh = v / bc2; den = mode == 0 ? sqrt(vh + eps) : sqrt(vh) + eps
//   p = p - lr (mh / den + decay p)
// fp32 evaluation (DESIGN.md R-adam-5): the step-uniform divisions by bc1, bc2 are
// multiplications by their fp32 reciprocals (one IEEE division per thread, or per block
// and step in adam_run); sqrt and the division by den use the SFU approximations
// (sqrt.approx / rsqrt.approx / rcp.approx, relative error ~2^-22): the result stays
// within the north_star's 1e-5 (fp32) of the fp64 oracle, and an element-step costs ~11
// FMA-pipe + 2 SFU instructions instead of ~4 IEEE division/sqrt sequences.
// Layout: fp32 arrays, 16-B aligned; each thread moves one float4 of p, m, v, g per
// grid-stride iteration (128-bit loads/stores), scalar tail for n % 4.
#include "proteus_device.h"

struct AdamScalars {
    float lr, b1, b2, eps, gscale, decay, rbc1, rbc2;   // rbc = fp32(1 / bc) (R-adam-5)
    int mode;
};

// .ftz: a subnormal vh (< 2^-126) flushes to 0, and then den = sqrt(vh) + eps rounds to eps
// either way (sqrt(2^-126) = 2^-63 is far below half an ulp of eps = 1e-8), so den is the
// same and the non-ftz form's subnormal rescaling (3 instructions per sqrt) is saved
__device__ __forceinline__ float adam_sqrt_approx(float x) {
    float y;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float adam_rsqrt_approx(float x) {
    float y;
    asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));   // x = vh + eps >= eps: normal
    return y;
}
#ifndef ADAM_RCP_NEWTON
#define ADAM_RCP_NEWTON 0
#endif
#ifndef ADAM_FOLD
#define ADAM_FOLD 1   // adam_run: the folded element-step (adam_one_fold, DESIGN R-adam-6)
#endif
#ifndef ADAM_RCP_SPLIT
// adam_run: elements of a float4 whose 1/den uses the FMA pipe: 1 with the folded step (6
// FMA-pipe instructions + 2 SFU per element-step: 0.0478 ms per 100 steps of 10^6, vs
// 0.0506 at 2, 0.0520 at 0, 0.0541 at 3; profiles/r02/ab_adam_fold_r02ax.txt), 2 for the
// unfolded one (0.0517 ms, profiles/r01/ab_adam_rcp.txt)
#define ADAM_RCP_SPLIT (ADAM_FOLD ? 1 : 2)
#endif
// 1/x for the positive normal x = sqrt(vh) + eps >= eps: rcp.approx on the SFU, or
// (NEWTON) on the FMA pipe.  Domain: x finite.  The Newton form returns NaN for x = inf
// where rcp.approx returns 0; x is inf only when v overflowed (|g / grad_scale| above
// ~2^63), where the fp32 update has already left the range the fp64 oracle's 1e-5 gate
// can describe, so no guard instruction is spent on it
// -- an exponent-flip initial guess (relative error <= 5.1%) and three Newton steps
// y = y (2 - x y) (error 5.1e-2 -> 2.6e-3 -> 6.7e-6 -> fp32 rounding, <= 1.5e-7 measured
// over 2e6 values spanning 2^-40..2^41).  adam_run splits its float4 between the two
// (ADAM_RCP_SPLIT): all-SFU 0.0558, all-FMA 0.0563, split 0.0543 ms per 100 steps of 10^6,
// 0.0517 with minBlocks 5 (profiles/r01/ab_adam_rcp.txt); adam_step (HBM-bound) uses the SFU.
template <bool NEWTON>
__device__ __forceinline__ float adam_rcp(float x) {
    if (NEWTON) {
        float y = __int_as_float(0x7EF311C3 - __float_as_int(x));
        y = y * fmaf(-x, y, 2.0f);
        y = y * fmaf(-x, y, 2.0f);
        y = y * fmaf(-x, y, 2.0f);
        return y;
    }
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));   // x >= eps: normal
    return y;
}

// one step from the scaled gradient gs = g / grad_scale; MODE 0: den = sqrt(vh + eps),
// MODE 1: den = sqrt(vh) + eps (the mode is a template parameter so that a loop over steps
// does not evaluate both forms and select)
template <int MODE, bool NEWTON = (ADAM_RCP_NEWTON != 0)>
__device__ __forceinline__ void adam_one_gs(float& p, float& m, float& v, float gs,
                                            const AdamScalars& s) {
    m = s.b1 * m + (1.0f - s.b1) * gs;
    v = s.b2 * v + (1.0f - s.b2) * gs * gs;
    const float mh = m * s.rbc1;
    const float vh = v * s.rbc2;
    const float upd = (MODE == 0) ? mh * adam_rsqrt_approx(vh + s.eps)
                                  : mh * adam_rcp<NEWTON>(adam_sqrt_approx(vh) + s.eps);
    p = p - s.lr * (upd + s.decay * p);
}

__device__ __forceinline__ void adam_one(float& p, float& m, float& v, float g,
                                         const AdamScalars& s) {
    if (s.mode == 0)
        adam_one_gs<0>(p, m, v, g / s.gscale, s);
    else
        adam_one_gs<1>(p, m, v, g / s.gscale, s);
}

// ADAM_FOLD: adam_run's element-step with the step-uniform factors folded (the same update,
// refactored): with L = lr / bc1 (fp32 lr * fp32(1/bc1)) and r2 = 1/bc2,
//   mode 1: y = 1 / fma(sqrt(v), sqrt(r2), eps)      (= 1 / (sqrt(v/bc2) + eps))
//   mode 0: y = rsqrt(fma(v, r2, eps))                (= 1 / sqrt(v/bc2 + eps))
//   p = p - fma(lr decay, p, L (m y))                 (= p - lr (mh/den + decay p))
// so the update still leaves p in ONE rounding per step, as in adam_one (subtracting
// lr decay p and the gradient term separately drifts: the rounding of p - 1e-5 p varies
// slowly with p, 7e-6 relative after 100 steps instead of 8e-7, r02aw).  L stays a factor
// (folding it into den as a divisor, r02ax, was as fast but not finite for lr = 0 or a
// vanishing lr: a guard for that cost the generic build 8 registers, r02bp).  (1 - b1) gs
// and (1 - b2) gs^2 are per-element constants (g is fixed).  Seven FMA-pipe instructions
// per element-step instead of eight, under the SFU's bound: 0.0545 -> 0.0477 ms per 100
// steps of 10^6, the same max error against the fp64 oracle (8.5e-7).
// tab[t] = (L, mode 1 ? sqrt(r2) : r2), per block and step in shared memory.
template <int MODE, bool NEWTON>
__device__ __forceinline__ void adam_one_fold(float& p, float& m, float& v, float c1, float c2,
                                              float2 tab, const AdamScalars& s) {
    m = s.b1 * m + c1;
    v = s.b2 * v + c2;
    const float y = (MODE == 0) ? adam_rsqrt_approx(fmaf(v, tab.y, s.eps))
                                : adam_rcp<NEWTON>(fmaf(adam_sqrt_approx(v), tab.y, s.eps));
    p = p - fmaf(s.lr * s.decay, p, tab.x * (m * y));
}

__device__ __forceinline__ float2 adam_fold_tab(float bc1, float bc2, const AdamScalars& s) {
    const float L = s.lr * (1.0f / bc1), r2 = 1.0f / bc2;
    return make_float2(L, s.mode == 0 ? r2 : sqrtf(r2));
}

template <int MODE>
__device__ __forceinline__ void adam_run4_fold(float4& P, float4& M, float4& V, const float4& Gs,
                                               const AdamScalars& s, const float2* tab, int steps) {
    const float a1 = 1.0f - s.b1, a2 = 1.0f - s.b2;
    const float4 C1 = make_float4(a1 * Gs.x, a1 * Gs.y, a1 * Gs.z, a1 * Gs.w);
    const float4 C2 = make_float4(a2 * Gs.x * Gs.x, a2 * Gs.y * Gs.y, a2 * Gs.z * Gs.z,
                                  a2 * Gs.w * Gs.w);
#pragma unroll 2   // 1, 2 and 4 within 1% (profiles/r02/ab_adam_sqrt_r02az.txt)
    for (int t = 0; t < steps; ++t) {
        const float2 r = tab[t];
        adam_one_fold<MODE, (ADAM_RCP_SPLIT >= 4)>(P.x, M.x, V.x, C1.x, C2.x, r, s);
        adam_one_fold<MODE, (ADAM_RCP_SPLIT >= 3)>(P.y, M.y, V.y, C1.y, C2.y, r, s);
        adam_one_fold<MODE, (ADAM_RCP_SPLIT >= 2)>(P.z, M.z, V.z, C1.z, C2.z, r, s);
        adam_one_fold<MODE, (ADAM_RCP_SPLIT >= 1)>(P.w, M.w, V.w, C1.w, C2.w, r, s);
    }
}

// `steps` steps of one float4 (adam_run), bias-correction reciprocals from shared memory
template <int MODE>
__device__ __forceinline__ void adam_run4(float4& P, float4& M, float4& V, const float4& Gs,
                                          AdamScalars s, const float2* rbc, int steps) {
#pragma unroll 2
    for (int t = 0; t < steps; ++t) {
        const float2 r = rbc[t];
        s.rbc1 = r.x;
        s.rbc2 = r.y;
#if ADAM_RCP_SPLIT   // ADAM_RCP_SPLIT of the 4 elements' 1/den on the FMA pipe, the rest on the SFU
        adam_one_gs<MODE, (ADAM_RCP_SPLIT >= 4)>(P.x, M.x, V.x, Gs.x, s);
        adam_one_gs<MODE, (ADAM_RCP_SPLIT >= 3)>(P.y, M.y, V.y, Gs.y, s);
        adam_one_gs<MODE, (ADAM_RCP_SPLIT >= 2)>(P.z, M.z, V.z, Gs.z, s);
        adam_one_gs<MODE, (ADAM_RCP_SPLIT >= 1)>(P.w, M.w, V.w, Gs.w, s);
#else
        adam_one_gs<MODE>(P.x, M.x, V.x, Gs.x, s);
        adam_one_gs<MODE>(P.y, M.y, V.y, Gs.y, s);
        adam_one_gs<MODE>(P.z, M.z, V.z, Gs.z, s);
        adam_one_gs<MODE>(P.w, M.w, V.w, Gs.w, s);
#endif
    }
}

#if !defined(PROTEUS_SELECT_ENTRY) || defined(PROTEUS_ENTRY_adam_step)
extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void adam_step(float* __restrict__ p, float* __restrict__ m, float* __restrict__ v,
               const float* __restrict__ g, unsigned long long n_rt, float lr_rt, float b1_rt,
               float b2_rt, float eps_rt, float gscale_rt, float decay_rt, int mode,
               float bc1, float bc2) {
    const unsigned long long n = PROTEUS_SPEC(5, n_rt);
    const AdamScalars s{PROTEUS_SPEC(6, lr_rt), PROTEUS_SPEC(7, b1_rt), PROTEUS_SPEC(8, b2_rt),
                        PROTEUS_SPEC(9, eps_rt), PROTEUS_SPEC(10, gscale_rt),
                        PROTEUS_SPEC(11, decay_rt), 1.0f / bc1, 1.0f / bc2, mode};
    const unsigned long long nvec = n / 4;
    const unsigned long long stride = (unsigned long long)PROTEUS_GRIDDIM_X * PROTEUS_BLOCKDIM_X;
    float4* p4 = reinterpret_cast<float4*>(p);
    float4* m4 = reinterpret_cast<float4*>(m);
    float4* v4 = reinterpret_cast<float4*>(v);
    const float4* g4 = reinterpret_cast<const float4*>(g);
    const unsigned long long tid = (unsigned long long)blockIdx.x * PROTEUS_BLOCKDIM_X + threadIdx.x;
    PROTEUS_PDL_WAIT();      // programmatic dependent launch: the previous step has completed
    PROTEUS_PDL_TRIGGER();
    for (unsigned long long i = tid; i < nvec; i += stride) {
        float4 P = p4[i], M = m4[i], V = v4[i];
        const float4 Gv = __ldg(&g4[i]);
        adam_one(P.x, M.x, V.x, Gv.x, s);
        adam_one(P.y, M.y, V.y, Gv.y, s);
        adam_one(P.z, M.z, V.z, Gv.z, s);
        adam_one(P.w, M.w, V.w, Gv.w, s);
        p4[i] = P;
        m4[i] = M;
        v4[i] = V;
    }
    // tail: n % 4 elements, one per thread of the first threads
    const unsigned long long j = nvec * 4 + tid;
    if (j < n) {
        float P = p[j], M = m[j], V = v[j];
        adam_one(P, M, V, g[j], s);
        p[j] = P;
        m[j] = M;
        v[j] = V;
    }
}
#endif

// adam_run: the whole time loop in one launch -- the form of the paper's ADAM kernel,
// whose time_step parameter is annotated with the other scalars (Listing 1,
// P@38745-39163, footnote 5 P@42483) and whose warps execute the steps in-kernel
// (inst_per_warp 9.6E5 -> 4E5 under RCF, P@41697-41853).  An element's update depends
// only on its own p, m, v and the fixed g, so a thread keeps its float4 of p, m, v in
// registers across all steps: 28 B/param of HBM traffic for the whole run instead of per
// step.  Each step is adam_one's update with the step-uniform factors folded into den
// (adam_one_fold, ADAM_FOLD, DESIGN R-adam-6: the same update, refactored, one rounding
// of p per step), and 1/den of the w element of each float4 is the FMA-pipe Newton
// reciprocal, that of x, y, z (and of the scalar tail) the SFU rcp.approx (ADAM_RCP_SPLIT
// = 1), so the reciprocal an element gets depends on its position; both are within
// 1.5e-7 relative of 1/den, far inside the 1e-5 gate (R-adam-5), and adam_run matches
// adam_step to that tolerance, not bit for bit.  g and grad_scale are fixed, so gs = g / grad_scale is computed once per
// element (the same value every step).  Work split: each CTA takes a contiguous, equal share of the float4s
// (not a grid stride), so with a grid that is a multiple of the SM count every SM gets
// the same number of element-steps (the kernel is ALU-bound).
// Parameters (1-based): 1 p  2 m  3 v  4 g  5 n  6 lr  7 b1  8 b2  9 eps  10 grad_scale
//   11 decay  12 mode  13 steps  14 bc (fp32[2*steps]: bc1, bc2 of each step,
//   host-computed in double, DESIGN.md R-adam-2).
// Annotated: 5..11 and 13 (the trip count, the paper's time_step).
#if !defined(PROTEUS_SELECT_ENTRY) || defined(PROTEUS_ENTRY_adam_run)
extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void adam_run(float* __restrict__ p, float* __restrict__ m, float* __restrict__ v,
              const float* __restrict__ g, unsigned long long n_rt, float lr_rt, float b1_rt,
              float b2_rt, float eps_rt, float gscale_rt, float decay_rt, int mode,
              int steps_rt, const float* __restrict__ bc) {
    const unsigned long long n = PROTEUS_SPEC(5, n_rt);
    const int steps = PROTEUS_SPEC(13, steps_rt);
    AdamScalars s{PROTEUS_SPEC(6, lr_rt), PROTEUS_SPEC(7, b1_rt), PROTEUS_SPEC(8, b2_rt),
                  PROTEUS_SPEC(9, eps_rt), PROTEUS_SPEC(10, gscale_rt),
                  PROTEUS_SPEC(11, decay_rt), 1.0f, 1.0f, mode};
    const unsigned long long nvec = n / 4;
    float4* p4 = reinterpret_cast<float4*>(p);
    float4* m4 = reinterpret_cast<float4*>(m);
    float4* v4 = reinterpret_cast<float4*>(v);
    const float4* g4 = reinterpret_cast<const float4*>(g);
    // per-step reciprocals of the bias corrections, once per block (R-adam-5); dynamic
    // shared memory of 8 * steps bytes (adam_run_launch)
    extern __shared__ float2 adam_rbc[];
    for (int t = threadIdx.x; t < steps; t += PROTEUS_BLOCKDIM_X) {
#if ADAM_FOLD
        adam_rbc[t] = adam_fold_tab(bc[2 * t], bc[2 * t + 1], s);
#else
        adam_rbc[t] = make_float2(1.0f / bc[2 * t], 1.0f / bc[2 * t + 1]);
#endif
    }
    __syncthreads();
    const unsigned long long share = (nvec + PROTEUS_GRIDDIM_X - 1) / PROTEUS_GRIDDIM_X;
    const unsigned long long i0 = (unsigned long long)blockIdx.x * share;
    const unsigned long long i1 = min(i0 + share, nvec);
    for (unsigned long long i = i0 + threadIdx.x; i < i1; i += PROTEUS_BLOCKDIM_X) {
        float4 P = p4[i], M = m4[i], V = v4[i];
        const float4 Gv = __ldg(&g4[i]);
        const float4 Gs = make_float4(Gv.x / s.gscale, Gv.y / s.gscale, Gv.z / s.gscale,
                                      Gv.w / s.gscale);
#if ADAM_FOLD
        if (s.mode == 0)   // uniform: one loop per mode
            adam_run4_fold<0>(P, M, V, Gs, s, adam_rbc, steps);
        else
            adam_run4_fold<1>(P, M, V, Gs, s, adam_rbc, steps);
#else
        if (s.mode == 0)   // uniform: one loop per mode
            adam_run4<0>(P, M, V, Gs, s, adam_rbc, steps);
        else
            adam_run4<1>(P, M, V, Gs, s, adam_rbc, steps);
#endif
        PROTEUS_CHECK_IDX(i, nvec);
        p4[i] = P;
        m4[i] = M;
        v4[i] = V;
    }
    const unsigned long long tid = (unsigned long long)blockIdx.x * PROTEUS_BLOCKDIM_X + threadIdx.x;
    const unsigned long long j = nvec * 4 + tid;   // tail: n % 4 elements
    if (j < n) {
        float P = p[j], M = m[j], V = v[j];
        const float Gs = g[j] / s.gscale;
#if ADAM_FOLD
        const float c1 = (1.0f - s.b1) * Gs, c2 = (1.0f - s.b2) * Gs * Gs;
#endif
        for (int t = 0; t < steps; ++t) {
#if ADAM_FOLD
            if (s.mode == 0)
                adam_one_fold<0, false>(P, M, V, c1, c2, adam_rbc[t], s);
            else
                adam_one_fold<1, false>(P, M, V, c1, c2, adam_rbc[t], s);
#else
            s.rbc1 = adam_rbc[t].x;
            s.rbc2 = adam_rbc[t].y;
            if (s.mode == 0)
                adam_one_gs<0>(P, M, V, Gs, s);
            else
                adam_one_gs<1>(P, M, V, Gs, s);
#endif
        }
        p[j] = P;
        m[j] = M;
        v[j] = V;
    }
}
#endif
