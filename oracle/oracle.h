/* oracle.h -- CPU oracle for the Proteus B200 hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this library.  The product path (paper_conf_cgo_georgakoudispb25_b200/)
 * never links, imports or executes it, and shares no code with it.
 *
 * Plain, slow, obviously-correct implementations of the four workloads the runtime
 * specializer drives (BASELINE.json configs 1-4).  Built with
 * -O2 -fno-fast-math -ffp-contract=off; OpenMP only over independent units
 * (elements, z-planes, lookups, columns) so results do not depend on thread count.
 */
#ifndef PROTEUS_ORACLE_H
#define PROTEUS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

void     oracle_set_threads(int n);        /* <=0: OpenMP default */
int      oracle_get_threads(void);

uint64_t oracle_splitmix64(uint64_t x);
uint64_t oracle_rng(uint64_t seed, uint64_t stream, uint64_t i);
uint64_t oracle_fnv1a64(const uint8_t* data, uint64_t len);

/* CFG 1 fused Adam, fp64 state.  p,m,v in/out [n]; g [n] (fp32 values as double). */
void oracle_adam(double* p, double* m, double* v, const double* g, uint64_t n,
                 float lr, float b1, float b2, float eps, float grad_scale, float decay,
                 int mode, int t_first, int steps);

/* CFG 2 stencil: one sweep u -> w over the full [nz][ny][nx] fp64 field. */
void oracle_stencil_sweep(const double* u, double* w, int nx, int ny, int nz,
                          double a0, double a1, double a2);
/* T sweeps, ping-pong between a and b; returns pointer index (0: a, 1: b) of result. */
int  oracle_stencil_run(double* a, double* b, int nx, int ny, int nz,
                        double a0, double a1, double a2, int T);

/* CFG 3 cross-section lookup (L lookups starting at lookup index i0). */
int  oracle_xs_lower(const double* e, int G, double E);
void oracle_xs_lookup(const double* egrid, const double* recs,
                      const int* mat_nuc, const int* mat_off, const int* mat_cnt,
                      const double* conc, const double* cum, uint64_t seed,
                      uint64_t i0, uint64_t L, int n_nuc, int n_grid, int n_mat,
                      double* macro_out, uint32_t* idx_out, int32_t* mat_out);

/* CFG 4 column microphysics, reproducible fp32 (no contraction; spec exp_s/pow_s). */
float oracle_exp_s(float x);
float oracle_log_s(float a);
float oracle_pow_s(float a, float b);
/* Sweep of a spec routine over fp32 bit patterns [start, start+count): fn 0 exp_s(x),
 * 1 log_s(x), 2 pow_s(x, b), 3 x / b (IEEE fp32 division).  chunk_hash[c] = sum mod 2^64 over i in chunk c (65536
 * consecutive patterns) of splitmix64((i << 32) | bits(result)); count % 65536 == 0. */
void  oracle_spec_sweep(uint64_t start, uint64_t count, int fn, float b, uint64_t* chunk_hash);
void  oracle_micro(float* th, float* qv, float* qc, float* qr,
                   const float* rho, const float* pk, const float* p, float* precip,
                   uint64_t ncol, int nz, int nsub, float dt, float dz, int ncalls);

#ifdef __cplusplus
}
#endif
#endif
