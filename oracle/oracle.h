/*
 * oracle.h — fp64 CPU oracle for the seismic modeling / RTM hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_ppopp_qawasmehchc15_b200/csrc), and the CUDA path never calls it.
 *
 * Paper: Qawasmeh, Chapman, Hugues, Calandra, "GPU Technology Applied to
 * Reverse Time Migration and Seismic Modeling via OpenACC", PMAM'15.
 * Citations "P:<line>" are line numbers of /root/reference/PAPER.md; the
 * readings of passages the paper leaves open are listed in DESIGN.md §3
 * (same labels O1..O19 as SURVEY.md §8c).
 *
 * Layout: every 3D array is C order [z][y][x] (x fastest), index
 *   ((size_t)k*ny + j)*nx + i,  i = x, j = y, k = z (depth, k = 0 top).
 * All arithmetic is double precision; fp32 inputs (models, h, dt) are
 * promoted to double exactly (O17).
 */
#ifndef SEIS_ORACLE_H
#define SEIS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t nx, ny, nz;   /* grid points */
  double h, dt;         /* spacing (m), time step (s); callers pass fp32 values */
  int32_t nb;           /* absorbing-layer width in points (inside the grid); 0 = none */
  int32_t free_surface; /* elastic: traction-free top (O16); top face then has no layer */
  double pml_R;         /* target reflection coefficient (O6/O7) */
  double pml_f;         /* C-PML alpha reference frequency (Hz) (O7) */
  int32_t periodic;     /* TEST MODE (O4): periodic wrap instead of zero ghosts; needs nb = 0;
                           with free_surface the wrap is lateral (x, y) only */
  int32_t iso_pml;      /* ISO absorbing layer: 0 = damped wave (O6), 1 = split-field PML (O6b) */
} or_grid;

/* O1: 8th-order coefficient tables: c[0..4] centred 2nd derivative,
 * d[0..3] staggered 1st derivative (d[m-1] multiplies the m-th pair). */
void or_coef(double c[5], double d[4]);

/* O1: out = Lambda u (the 25-point Laplacian times h^2) with zero (or periodic) ghosts. */
void or_lap(const or_grid* g, const double* u, double* out);
/* O1: out = h * D^{+/-}_axis f   (axis 0 = x, 1 = y, 2 = z; plus = 1 for D+). */
void or_dstag(const or_grid* g, int axis, int plus, const double* f, double* out);

/* O6: isotropic damping profile eta[N] for one axis. */
void or_iso_eta(int N, int nb, double h, double vmax, double R, double* eta);
/* O7: C-PML coefficient arrays for one axis: a,b at integer nodes, ah,bh at
 * half nodes i+1/2.  lo/hi select whether the low / high face has a layer. */
void or_cpml(int N, int nb, int lo, int hi, double h, double dt, double vmax,
             double R, double f, double* a, double* b, double* ah, double* bh);

/* Injection list: n_inj points, positions pos[n_inj][3] (x,y,z), samples
 * amp[t][n_inj] addressed by the ABSOLUTE step index t (O11). */
typedef struct {
  int32_t n;
  const int32_t* pos;
  const double* amp;
} or_inj;

/* Receiver list: positions pos[nrec][3]. */
typedef struct {
  int32_t n;
  const int32_t* pos;
  int32_t component;    /* elastic only: 0 vx, 1 vy, 2 vz, 3 pressure (O13) */
} or_rec;

/* ISO (Eq 1 + O3/O6): advance (u_prev, u_cur) = (u^{n-1}, u^n) by nsteps
 * steps starting at absolute step n0; on return they hold the last two
 * levels.  seis[s][r] = u^{n0+s+1}(x_r) (O13).  Returns 0 on success.
 * w: split-field PML state (O6b, g->iso_pml = 1 and nb > 0; else ignored, may be
 * NULL): [2][3][nz][ny][nx], w[0][d] = u^{(d),n-1}, w[1][d] = u^{(d),n}, used only
 * inside the layers; updated in place like (u_prev, u_cur). */
int or_iso_run(const or_grid* g, const float* vp, double* u_prev, double* u_cur, double* w,
               int n0, int nsteps, const or_inj* inj, const or_rec* rec, double* seis);

/* ACOUSTIC (Eq 2 in 3D, O8 + O7): state p, qx, qy, qz and psi[6][N^3]
 * (psi_{p,x}, psi_{p,y}, psi_{p,z} at q nodes; psi_{q,x}, psi_{q,y}, psi_{q,z}
 * at p nodes).  seis[s][r] = p^{n0+s+1}(x_r). */
int or_ac_run(const or_grid* g, const float* vp, const float* rho, double* p,
              double* qx, double* qy, double* qz, double* psi, int n0, int nsteps,
              const or_inj* inj, const or_rec* rec, double* seis);

/* ELASTIC (Eq 3, O9 + O7 + O16): f[9][N^3] = vx, vy, vz, sxx, syy, szz,
 * sxy, sxz, syz; psi[18][N^3] (see oracle.c for the order). */
int or_el_run(const or_grid* g, const float* vp, const float* vs, const float* rho,
              double* f, double* psi, int n0, int nsteps, const or_inj* inj,
              const or_rec* rec, double* seis);

/* RTM (Alg 1; O14/O15): forward source propagation storing
 * snapshots S_j (j = snap, 2 snap, ... <= nt-1), then backward receiver
 * propagation injecting data[nt-1-m][r] at reversed step m and imaging
 * image += S_j * R.  kind 0 = ISO, 1 = ACOUSTIC, 2 = ELASTIC (imaged field:
 * pressure -(sxx+syy+szz)/3; receivers inject like the explosive source).
 * image is accumulated. */
int or_migrate(const or_grid* g, int kind, const float* vp, const float* vs, const float* rho,
               const int32_t src_pos[3], const double* src_amp, int nt,
               int nrec, const int32_t* rec_pos, const double* data, int snap,
               double* image);

#ifdef __cplusplus
}
#endif
#endif
