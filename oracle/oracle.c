/* oracle.c -- CPU oracle for the Proteus B200 hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline, --impl reference)
 * may load this.  It shares no code, header, table or constant generator with the
 * CUDA path under paper_conf_cgo_georgakoudispb25_b200/; the two are written
 * independently from the same text (PAPER.md + SURVEY.md §8c + DESIGN.md readings).
 *
 * Citations: "P@n" = /root/reference/PAPER.md line 1, character offset n.
 *
 * Pins (tests/test_oracle_*.py, all -m "not gpu"):
 *   rng / fnv1a64  : published SplitMix64 and FNV-1a-64 test vectors
 *   adam           : one step from zero moments (closed form), constant-gradient
 *                    closed form over T steps, g = 0 geometric decay
 *   stencil        : exact 12*Laplacian of integer polynomials of degree <= 5 (P1),
 *                    light-cone closed form u_T = u_0 + 0.5625 T (P2)
 *   xs             : lower index vs brute-force linear scan, grid-point / below /
 *                    above special cases, linear-in-E tables (closed form)
 *   micro          : exp_s vs fp64 exp (ulp bound), pow_s(a,1) = a, pow_s(a,.5) vs
 *                    sqrt, dry-column identity, saturation adjustment (Newton
 *                    residual), first law, Kessler autoconversion, KW78 accretion,
 *                    ground flux, sedimentation profile + top half cell, KW78 rain
 *                    evaporation rate and its caps, substep composition, water
 *                    budget (sanity); mutation-checked by scripts/mutate_oracle_micro.py
 * Parity status per function is listed in DESIGN.md §"Oracle pins".
 */
#include "oracle.h"

#include <math.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void oracle_set_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

int oracle_get_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---------------------------------------------------------------------------------
 * Counter-based generator: splitmix64 first output; rng(stream,i) =
 * splitmix64(seed + (stream << 40) + i).  Needed by the XS lookup, which draws its
 * (E, r) pair per lookup.
 * ------------------------------------------------------------------------------- */
uint64_t oracle_splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t oracle_rng(uint64_t seed, uint64_t stream, uint64_t i) {
    return oracle_splitmix64(seed + (stream << 40) + i);
}

static double u01_f64(uint64_t r) { return (double)(r >> 11) * 0x1p-53; }

/* FNV-1a 64-bit (the hash the specialization key uses; P@24205-24805 leaves the hash
 * function unspecified, reading R-key-1). */
uint64_t oracle_fnv1a64(const uint8_t* data, uint64_t len) {
    uint64_t h = 0xcbf29ce484222325ull;
    for (uint64_t i = 0; i < len; ++i) {
        h ^= data[i];
        h *= 0x100000001b3ull;
    }
    return h;
}

/* ---------------------------------------------------------------------------------
 * CFG 1: fused Adam update.  Listing 1 (P@38745-39163) gives the HeCBench prototype
 * adam(p, m, v, g, b1, b2, eps, grad_scale, step_size, time_step, vector_size, mode,
 * decay); the update rule itself is not printed in the paper, so this follows the
 * DESIGN.md reading:
 *   gs = g / grad_scale
 *   m  = b1 m + (1 - b1) gs
 *   v  = b2 v + (1 - b2) gs^2
 *   mh = m / bc1_t,  vh = v / bc2_t,   bc_t = fp32(1 - b^t) computed in double
 *   den = mode == 0 ? sqrt(vh + eps) : sqrt(vh) + eps
 *   p  = p - lr (mh / den + decay p)
 * State is kept in fp64 (the oracle's precision); scalars are the fp32 values.
 * ------------------------------------------------------------------------------- */
void oracle_adam(double* p, double* m, double* v, const double* g, uint64_t n,
                 float lr, float b1, float b2, float eps, float grad_scale, float decay,
                 int mode, int t_first, int steps) {
    const double LR = lr, B1 = b1, B2 = b2, EPS = eps, GS = grad_scale, WD = decay;
    for (int s = 0; s < steps; ++s) {
        const int t = t_first + s;
        const double bc1 = (double)(float)(1.0 - pow(B1, (double)t));
        const double bc2 = (double)(float)(1.0 - pow(B2, (double)t));
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < (int64_t)n; ++i) {
            const double gs = g[i] / GS;
            m[i] = B1 * m[i] + (1.0 - B1) * gs;
            v[i] = B2 * v[i] + (1.0 - B2) * gs * gs;
            const double mh = m[i] / bc1;
            const double vh = v[i] / bc2;
            const double den = (mode == 0) ? sqrt(vh + EPS) : sqrt(vh) + EPS;
            p[i] = p[i] - LR * (mh / den + WD * p[i]);
        }
    }
}

/* ---------------------------------------------------------------------------------
 * CFG 2: 13-point 4th-order 3D stencil (SW4CK-shaped, P@45192-45829; operator from
 * SURVEY.md §8c-2, reading R-st-1):
 *   interior (2 <= i <= nx-3, 2 <= j <= ny-3, 2 <= k <= nz-3):
 *     s1 = u[i-1] + u[i+1] + u[j-1] + u[j+1] + u[k-1] + u[k+1]   (this order)
 *     s2 = u[i-2] + u[i+2] + u[j-2] + u[j+2] + u[k-2] + u[k+2]
 *     w  = a0 u + a1 s1 + a2 s2
 *   every other point (the 2-cell Dirichlet frame): w = u.
 * index (k*ny + j)*nx + i, x fastest.
 * ------------------------------------------------------------------------------- */
void oracle_stencil_sweep(const double* u, double* w, int nx, int ny, int nz,
                          double a0, double a1, double a2) {
    const int64_t sx = 1, sy = nx, sz = (int64_t)nx * ny;
#pragma omp parallel for schedule(static)
    for (int k = 0; k < nz; ++k) {
        for (int j = 0; j < ny; ++j) {
            for (int i = 0; i < nx; ++i) {
                const int64_t c = (int64_t)k * sz + (int64_t)j * sy + i;
                const int interior = i >= 2 && i <= nx - 3 && j >= 2 && j <= ny - 3 &&
                                     k >= 2 && k <= nz - 3;
                if (!interior) {
                    w[c] = u[c];
                    continue;
                }
                double s1 = u[c - sx];
                s1 = s1 + u[c + sx];
                s1 = s1 + u[c - sy];
                s1 = s1 + u[c + sy];
                s1 = s1 + u[c - sz];
                s1 = s1 + u[c + sz];
                double s2 = u[c - 2 * sx];
                s2 = s2 + u[c + 2 * sx];
                s2 = s2 + u[c - 2 * sy];
                s2 = s2 + u[c + 2 * sy];
                s2 = s2 + u[c - 2 * sz];
                s2 = s2 + u[c + 2 * sz];
                w[c] = a0 * u[c] + a1 * s1 + a2 * s2;
            }
        }
    }
}

int oracle_stencil_run(double* a, double* b, int nx, int ny, int nz,
                       double a0, double a1, double a2, int T) {
    double* src = a;
    double* dst = b;
    for (int t = 0; t < T; ++t) {
        oracle_stencil_sweep(src, dst, nx, ny, nz, a0, a1, a2);
        double* tmp = src;
        src = dst;
        dst = tmp;
    }
    return src == a ? 0 : 1;
}

/* ---------------------------------------------------------------------------------
 * CFG 3: Monte-Carlo cross-section lookup (RSBench-shaped, P@29228, P@44652-45192;
 * pointwise-table reading SURVEY.md §8c-3, reading R-xs-*).
 * lower(e, G, E) = max{ g in [0, G-2] : e[g] <= E }, or 0 if that set is empty.
 * ------------------------------------------------------------------------------- */
int oracle_xs_lower(const double* e, int G, double E) {
    /* plain bisection on the invariant e[lo] <= E < e[hi] over candidates [0, G-2] */
    if (!(e[0] <= E)) return 0;
    int lo = 0, hi = G - 1;            /* answer in [lo, hi-1]; e[lo] <= E */
    while (hi - lo > 1) {
        const int mid = lo + (hi - lo) / 2;
        if (e[mid] <= E) lo = mid; else hi = mid;
    }
    return lo;                        /* <= G-2 because hi starts at G-1 */
}

void oracle_xs_lookup(const double* egrid, const double* recs,
                      const int* mat_nuc, const int* mat_off, const int* mat_cnt,
                      const double* conc, const double* cum, uint64_t seed,
                      uint64_t i0, uint64_t L, int n_nuc, int n_grid, int n_mat,
                      double* macro_out, uint32_t* idx_out, int32_t* mat_out) {
    (void)n_nuc;
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t q = 0; q < (int64_t)L; ++q) {
        const uint64_t i = i0 + (uint64_t)q;
        const double E = u01_f64(oracle_rng(seed, 34, i));
        const double r = u01_f64(oracle_rng(seed, 35, i));
        int mat = n_mat - 1;
        for (int mm = 0; mm < n_mat; ++mm) {
            if (r < cum[mm]) { mat = mm; break; }
        }
        double macro[5] = {0, 0, 0, 0, 0};
        uint32_t isum = 0;
        for (int t = 0; t < mat_cnt[mat]; ++t) {
            const int nuc = mat_nuc[mat_off[mat] + t];
            const double c = conc[mat_off[mat] + t];
            const double* e = egrid + (int64_t)nuc * n_grid;
            const int lo = oracle_xs_lower(e, n_grid, E);
            const int hi = lo + 1;
            const double f = (e[hi] - E) / (e[hi] - e[lo]);
            const double* rl = recs + ((int64_t)nuc * n_grid + lo) * 6;
            const double* rh = recs + ((int64_t)nuc * n_grid + hi) * 6;
            for (int ch = 0; ch < 5; ++ch) {
                const double sig = rh[1 + ch] - f * (rh[1 + ch] - rl[1 + ch]);
                macro[ch] = macro[ch] + c * sig;
            }
            isum += (uint32_t)lo;
        }
        for (int ch = 0; ch < 5; ++ch) macro_out[q * 5 + ch] = macro[ch];
        idx_out[q] = isum;
        if (mat_out) mat_out[q] = mat;
    }
}

/* ---------------------------------------------------------------------------------
 * CFG 4: column warm-rain microphysics (WSM5-shaped, P@43000-44469; the paper prints
 * no equations, so the scheme is the Kessler/Klemp-Wilhelmson warm-rain column of
 * DESIGN.md §"Microphysics spec", evaluated in reproducible fp32: every operation
 * below is one IEEE fp32 op in the written order; fma only where written.
 * ------------------------------------------------------------------------------- */

/* exp_s (DESIGN.md spec R2): Cody-Waite reduction + degree-7 Taylor in fmaf. */
static float pow2i(int e) {              /* 2^e for e in [-126, 127], built from bits */
    union { uint32_t u; float f; } c;
    c.u = (uint32_t)(e + 127) << 23;
    return c.f;
}

float oracle_exp_s(float x) {
    const float LOG2E = 0x1.715476p+0f;
    const float LN2_HI = 0x1.62e4p-1f;
    const float LN2_LO = 0x1.7f7d1cp-20f;
    if (x != x) return x;
    if (x > 88.0f) x = 88.0f;
    if (x < -103.0f) return 0.0f;
    const float n = rintf(x * LOG2E);
    float r = fmaf(-n, LN2_HI, x);
    r = fmaf(-n, LN2_LO, r);
    float q = 0x1.a01a02p-13f;              /* 1/7! */
    q = fmaf(q, r, 0x1.6c16c2p-10f);        /* 1/6! */
    q = fmaf(q, r, 0x1.111112p-7f);         /* 1/5! */
    q = fmaf(q, r, 0x1.555556p-5f);         /* 1/4! */
    q = fmaf(q, r, 0x1.555556p-3f);         /* 1/3! */
    q = fmaf(q, r, 0x1p-1f);                /* 1/2! */
    q = fmaf(q, r, 1.0f);                   /* 1/1! */
    q = fmaf(q, r, 1.0f);                   /* 1/0! */
    const int ni = (int)n;
    const int h = ni / 2;                   /* C division truncates toward zero */
    return (q * pow2i(h)) * pow2i(ni - h);
}

/* log_s (spec R2): a = m 2^ex with m in (sqrt(1/2), sqrt(2)]; atanh series in z = s^2. */
float oracle_log_s(float a) {
    const float LN2_HI = 0x1.62e4p-1f;
    const float LN2_LO = 0x1.7f7d1cp-20f;
    union { float f; uint32_t u; } c;
    c.f = a;
    int e = (int)((c.u >> 23) & 0xffu);
    int adj = 0;
    if (e == 0) {                           /* subnormal: scale by 2^24 (exact) */
        c.f = a * 0x1p24f;
        e = (int)((c.u >> 23) & 0xffu);
        adj = 24;
    }
    int ex = e - 127 - adj;
    c.u = (c.u & 0x7fffffu) | (127u << 23);  /* m in [1, 2) */
    float m = c.f;
    if (m > 0x1.6a09e6p+0f) {               /* sqrt(2) */
        m = m * 0.5f;
        ex = ex + 1;
    }
    const float s = (m - 1.0f) / (m + 1.0f);
    const float z = s * s;
    float P = 0x1.111112p-4f;               /* 1/15 */
    P = fmaf(P, z, 0x1.3b13b2p-4f);         /* 1/13 */
    P = fmaf(P, z, 0x1.745d18p-4f);         /* 1/11 */
    P = fmaf(P, z, 0x1.c71c72p-4f);         /* 1/9  */
    P = fmaf(P, z, 0x1.24924ap-3f);         /* 1/7  */
    P = fmaf(P, z, 0x1.99999ap-3f);         /* 1/5  */
    P = fmaf(P, z, 0x1.555556p-2f);         /* 1/3  */
    P = fmaf(P, z, 1.0f);                   /* 1/1  */
    const float q = (2.0f * s) * P;
    const float fe = (float)ex;
    return fmaf(fe, LN2_HI, fmaf(fe, LN2_LO, q));
}

float oracle_pow_s(float a, float b) {
    if (!(a > 0.0f)) return 0.0f;
    return oracle_exp_s(b * oracle_log_s(a));
}

/* spec max_s / min_s: explicit ternaries (return the second operand on ties), so the
 * sign of a zero result is defined by the spec, not by libm or the ISA. */
static float max_s(float a, float b) { return a > b ? a : b; }
static float min_s(float a, float b) { return a < b ? a : b; }
static float fmin3(float a, float b, float c) { return min_s(min_s(a, b), c); }

/* Exhaustive-sweep helper for the "exp_s/pow_s unit pins": the CUDA
 * side computes the same per-chunk sums independently (micro_spec_sweep). */
void oracle_spec_sweep(uint64_t start, uint64_t count, int fn, float b, uint64_t* chunk_hash) {
    const uint64_t nchunk = count / 65536u;
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t c = 0; c < (int64_t)nchunk; ++c) {
        uint64_t h = 0;
        for (uint64_t j = 0; j < 65536u; ++j) {
            const uint64_t i = start + (uint64_t)c * 65536u + j;
            const uint32_t xb = (uint32_t)i;
            float x, y;
            memcpy(&x, &xb, 4);
            if (fn == 0) y = oracle_exp_s(x);
            else if (fn == 1) y = oracle_log_s(x);
            else if (fn == 2) y = oracle_pow_s(x, b);
            else y = x / b;   /* fn 3: the spec's "/" (IEEE fp32 division, R-mp-2 R3) */
            uint32_t yb;
            memcpy(&yb, &y, 4);
            h += oracle_splitmix64((i << 32) | yb);
        }
        chunk_hash[c] = h;
    }
}

void oracle_micro(float* th, float* qv, float* qc, float* qr,
                  const float* rho, const float* pk, const float* p, float* precip,
                  uint64_t ncol, int nz, int nsub, float dt, float dz, int ncalls) {
    const float F5 = 10214784.0f;          /* fp32 of 237.3*17.27*2.5e6/1003, left to right */
#pragma omp parallel for schedule(static)
    for (int64_t col = 0; col < (int64_t)ncol; ++col) {
        float r[256], rhalf[256], pc[256], vt[256], F[256], sed[256];
        float* TH = th + col * nz;
        float* QV = qv + col * nz;
        float* QC = qc + col * nz;
        float* QR = qr + col * nz;
        const float* RHO = rho + col * nz;
        const float* PK = pk + col * nz;
        const float* P = p + col * nz;
        for (int call = 0; call < ncalls; ++call) {
            for (int k = 0; k < nz; ++k) {
                r[k] = 0.001f * RHO[k];
                rhalf[k] = sqrtf(RHO[0] / RHO[k]);
                pc[k] = 380.0f / P[k];
                vt[k] = (36.34f * oracle_pow_s(QR[k] * r[k], 0.1364f)) * rhalf[k];
            }
            const float dt0 = dt / (float)nsub;
            float prec = 0.0f;
            for (int s = 0; s < nsub; ++s) {
                prec = prec + ((RHO[0] * QR[0]) * vt[0]) / 1000.0f;
                for (int k = 0; k < nz; ++k) F[k] = (r[k] * QR[k]) * vt[k];
                for (int k = 0; k < nz - 1; ++k)
                    sed[k] = (dt0 * (F[k + 1] - F[k])) / (r[k] * dz);
                sed[nz - 1] = ((-dt0) * (QR[nz - 1] * vt[nz - 1])) / (0.5f * dz);
                for (int k = 0; k < nz; ++k) {
                    /* autoconversion + accretion */
                    const float ac = max_s(0.001f * (QC[k] - 0.001f), 0.0f);
                    const float qrprod = QC[k] - (QC[k] - dt0 * ac) /
                                         (1.0f + (dt0 * 2.2f) * oracle_pow_s(QR[k], 0.875f));
                    QC[k] = max_s(QC[k] - qrprod, 0.0f);
                    QR[k] = max_s((QR[k] + qrprod) + sed[k], 0.0f);
                    /* saturation adjustment */
                    const float T = PK[k] * TH[k];
                    const float qvs = pc[k] * oracle_exp_s((17.27f * (T - 273.0f)) / (T - 36.0f));
                    const float tm = T - 36.0f;
                    const float prod = (QV[k] - qvs) / (1.0f + (qvs * F5) / (tm * tm));
                    /* rain evaporation */
                    const float rq = r[k] * QR[k];
                    const float vent = (1.6f + 124.9f * oracle_pow_s(rq, 0.2046f)) *
                                       oracle_pow_s(rq, 0.525f);
                    /* KW78 ventilation-diffusion denominator 5.4e5 + 2.55e6/(p[mb] qvs), with
                     * 1/p[mb] = pc/3.8 (DESIGN.md R-mp-3) */
                    const float dif = (2.55e6f * pc[k]) / (3.8f * qvs) + 5.4e5f;
                    const float e1 = ((dt0 * (vent / dif)) * max_s(qvs - QV[k], 0.0f)) /
                                     (r[k] * qvs);
                    const float ern = fmin3(e1, max_s(-prod - QC[k], 0.0f), QR[k]);
                    /* state update */
                    const float cond = max_s(prod, -QC[k]);
                    TH[k] = TH[k] + (2.5e6f / (1003.0f * PK[k])) * (cond - ern);
                    QV[k] = max_s((QV[k] - cond) + ern, 0.0f);
                    QC[k] = QC[k] + cond;
                    QR[k] = QR[k] - ern;
                }
                for (int k = 0; k < nz; ++k)
                    vt[k] = (36.34f * oracle_pow_s(QR[k] * r[k], 0.1364f)) * rhalf[k];
            }
            precip[col] = prec / (float)nsub;
        }
    }
}
