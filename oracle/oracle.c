/*
 * oracle.c — plain fp64 CPU oracle of the paper's hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Deliberately slow and literal:
 * plain triple loops (OpenMP over z only), every derivative evaluated
 * straight from its definition with an explicit ghost accessor, no blocking,
 * no fusion, no reordering beyond what the paper's Algorithm 1 states.
 *
 * Paper passages (P:<line> of /root/reference/PAPER.md):
 *   Eq 1  P:123-129  isotropic constant-density propagator
 *   Eq 2  P:131-142  variable-density acoustic first-order staggered system
 *   Eq 3  P:146-159  isotropic elastic velocity-stress staggered system
 *   P:175            "operators with a 3D stencil width of 8", "25 data read accesses"
 *   P:177, P:179     source injection, snapshots, standard PML (iso) / C-PML (acoustic, elastic)
 *   Alg 1 P:183-209  modeling + RTM loop order
 *   P:111            imaging condition I = sum_s sum_t S R
 *   P:352            single precision on the product side (fp64 here)
 * Readings of unstated details: DESIGN.md §3 (labels O1..O19).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

#define IDX(g, i, j, k) ((((size_t)(k)) * (size_t)(g)->ny + (size_t)(j)) * (size_t)(g)->nx + (size_t)(i))
#define NPTS(g) ((size_t)(g)->nx * (size_t)(g)->ny * (size_t)(g)->nz)

/* ---------------------------------------------------------------- O1 --- */
/* 8th-order coefficients (radius 4: "stencil width of 8").  The
 * canonical values are the fp32 roundings of the exact rationals
 *   c = [-205/72, 8/5, -1/5, 8/315, -1/560]       (centred 2nd derivative)
 *   d = [1225/1024, -245/3072, 49/5120, -5/7168]  (staggered 1st derivative)
 * promoted to double (O1, O17): the product computes in fp32 with exactly
 * these values, so oracle and product differ by arithmetic rounding only. */
static double C2[5];
static double D1[4];
static int coef_ready = 0;

static void init_coef(void) {
  if (coef_ready) return;
  C2[0] = (double)(float)(-205.0 / 72.0);
  C2[1] = (double)(float)(8.0 / 5.0);
  C2[2] = (double)(float)(-1.0 / 5.0);
  C2[3] = (double)(float)(8.0 / 315.0);
  C2[4] = (double)(float)(-1.0 / 560.0);
  D1[0] = (double)(float)(1225.0 / 1024.0);
  D1[1] = (double)(float)(-245.0 / 3072.0);
  D1[2] = (double)(float)(49.0 / 5120.0);
  D1[3] = (double)(float)(-5.0 / 7168.0);
  coef_ready = 1;
}

void or_coef(double c[5], double d[4]) {
  init_coef();
  for (int m = 0; m < 5; ++m) c[m] = C2[m];
  for (int m = 0; m < 4; ++m) d[m] = D1[m];
}

static int wrap(int i, int n) {
  i %= n;
  return i < 0 ? i + n : i;
}

/* Value of f at (i,j,k): zero outside the grid (O1), or periodic wrap (O4 test mode;
 * with a free surface the wrap is lateral only and z keeps zero ghosts below the grid). */
static double at(const or_grid* g, const double* f, int i, int j, int k) {
  if (g->periodic) {
    i = wrap(i, g->nx);
    j = wrap(j, g->ny);
    if (!g->free_surface) k = wrap(k, g->nz);
  }
  if (i < 0 || j < 0 || k < 0 || i >= g->nx || j >= g->ny || k >= g->nz) return 0.0;
  return f[IDX(g, i, j, k)];
}

static double atf(const or_grid* g, const float* f, int i, int j, int k) {
  return (double)f[IDX(g, i, j, k)];
}

/* Lambda u = 3 c0 u_i + sum_{m=1..4} c_m sum_axes (u_{i+m e} + u_{i-m e}) (O1: this
 * algebraic form is fixed; Eq 1's nabla^2 u ~= Lambda u / h^2). */
static double lap_at(const or_grid* g, const double* u, int i, int j, int k) {
  double s = 3.0 * C2[0] * at(g, u, i, j, k);
  for (int m = 1; m <= 4; ++m) {
    double t = at(g, u, i + m, j, k) + at(g, u, i - m, j, k) + at(g, u, i, j + m, k) +
               at(g, u, i, j - m, k) + at(g, u, i, j, k + m) + at(g, u, i, j, k - m);
    s += C2[m] * t;
  }
  return s;
}

/* One axis of it (O6b): L_d u = c0 u_i + sum_m c_m (u_{i+m e_d} + u_{i-m e_d});
 * Lambda = L_x + L_y + L_z. */
static double lap_axis(const or_grid* g, const double* u, int i, int j, int k, int d) {
  double s = C2[0] * at(g, u, i, j, k);
  for (int m = 1; m <= 4; ++m) {
    int e[3] = {0, 0, 0};
    e[d] = m;
    s += C2[m] * (at(g, u, i + e[0], j + e[1], k + e[2]) + at(g, u, i - e[0], j - e[1], k - e[2]));
  }
  return s;
}

void or_lap(const or_grid* g, const double* u, double* out) {
  init_coef();
#pragma omp parallel for schedule(static)
  for (int k = 0; k < g->nz; ++k)
    for (int j = 0; j < g->ny; ++j)
      for (int i = 0; i < g->nx; ++i) out[IDX(g, i, j, k)] = lap_at(g, u, i, j, k);
}

/* Staggered first derivatives (O1), times h.  Array index i of a half-node
 * field holds position i+1/2.
 *   (h D+ f)_{i+1/2} = sum_m d_m (f_{i+m}   - f_{i-m+1})
 *   (h D- g)_i       = sum_m d_m (g_{i+m-1} - g_{i-m})                        */
typedef double (*acc_fn)(const or_grid*, const double*, int, int, int);

static double dstag_at(const or_grid* g, acc_fn acc, const double* f, int axis, int plus, int i,
                       int j, int k) {
  int e[3] = {0, 0, 0};
  e[axis] = 1;
  double s = 0.0;
  for (int m = 1; m <= 4; ++m) {
    int a = plus ? m : m - 1;  /* forward offset  */
    int b = plus ? m - 1 : m;  /* backward offset */
    s += D1[m - 1] * (acc(g, f, i + a * e[0], j + a * e[1], k + a * e[2]) -
                      acc(g, f, i - b * e[0], j - b * e[1], k - b * e[2]));
  }
  return s;
}

void or_dstag(const or_grid* g, int axis, int plus, const double* f, double* out) {
  init_coef();
#pragma omp parallel for schedule(static)
  for (int k = 0; k < g->nz; ++k)
    for (int j = 0; j < g->ny; ++j)
      for (int i = 0; i < g->nx; ++i)
        out[IDX(g, i, j, k)] = dstag_at(g, at, f, axis, plus, i, j, k);
}

/* ------------------------------------------------------------ O6, O7 --- */
/* Normalised depth into the layer of a point at grid position x (may be a
 * half node), for a layer of nb points on each selected face; clipped to 1. */
static double layer_xi(double x, int N, int nb, int lo, int hi) {
  double xi = 0.0;
  if (lo && nb - x > xi) xi = nb - x;
  if (hi && x - (N - 1 - nb) > xi) xi = x - (N - 1 - nb);
  xi /= (double)nb;
  return xi > 1.0 ? 1.0 : xi;
}

/* O6: eta_d(xi) = eta_max xi^2, eta_max = 3 vmax ln(1/R) / (2 nb h). */
void or_iso_eta(int N, int nb, double h, double vmax, double R, double* eta) {
  for (int i = 0; i < N; ++i) {
    if (nb <= 0) {
      eta[i] = 0.0;
      continue;
    }
    double emax = 3.0 * vmax * log(1.0 / R) / (2.0 * nb * h);
    double xi = layer_xi((double)i, N, nb, 1, 1);
    eta[i] = emax * xi * xi;
  }
}

/* O7 (Komatitsch & Martin 2007, kappa = 1): d = d0 xi^2, alpha = pi f (1 - xi),
 * b = exp(-(d + alpha) dt), a = d (b - 1) / (d + alpha), a = 0 where d = 0.
 * "four different one-dimensional arrays with the cpml-coefficients for each
 * dimension" = a, b (integer nodes), ah, bh (half nodes). */
static void cpml_point(double xi, double d0, double f, double dt, double* a, double* b) {
  double d = d0 * xi * xi;
  double alpha = M_PI * f * (1.0 - xi);
  *b = exp(-(d + alpha) * dt);
  *a = (d > 0.0) ? d * (*b - 1.0) / (d + alpha) : 0.0;
}

void or_cpml(int N, int nb, int lo, int hi, double h, double dt, double vmax, double R, double f,
             double* a, double* b, double* ah, double* bh) {
  for (int i = 0; i < N; ++i) {
    if (nb <= 0) {
      a[i] = b[i] = ah[i] = bh[i] = 0.0;
      continue;
    }
    double d0 = 3.0 * vmax * log(1.0 / R) / (2.0 * nb * h);
    cpml_point(layer_xi((double)i, N, nb, lo, hi), d0, f, dt, &a[i], &b[i]);
    cpml_point(layer_xi((double)i + 0.5, N, nb, lo, hi), d0, f, dt, &ah[i], &bh[i]);
  }
}

static double vmax_of(const or_grid* g, const float* vp) {
  double v = 0.0;
  size_t n = NPTS(g);
  for (size_t t = 0; t < n; ++t)
    if ((double)vp[t] > v) v = (double)vp[t];
  return v;
}

static int in_grid(const or_grid* g, const int32_t* p) {
  return p[0] >= 0 && p[1] >= 0 && p[2] >= 0 && p[0] < g->nx && p[1] < g->ny && p[2] < g->nz;
}

static int check_lists(const or_grid* g, const or_inj* inj, const or_rec* rec) {
  if (g->periodic && g->nb != 0) return -1;
  if (inj)
    for (int s = 0; s < inj->n; ++s)
      if (!in_grid(g, inj->pos + 3 * s)) return -2;
  if (rec)
    for (int r = 0; r < rec->n; ++r)
      if (!in_grid(g, rec->pos + 3 * r)) return -3;
  return 0;
}

/* ---------------------------------------------------------- ISO, O3 --- */
/* Eq 1 with the damped-wave absorbing term (O6):
 *   u^{n+1} = [2u^n - (1 - eta dt) u^{n-1} + m Lambda u^n + s^n] / (1 + eta dt),
 *   m = v^2 dt^2 / h^2,  s^n = delta_{i,s} v_s^2 dt^2 w(n dt) / h^3,
 *   eta = eta_x + eta_y + eta_z.
 * With eta = 0 this is exactly Eq 1 with f^n = w(n dt) delta / h^3 (O3).
 * Step order (O2): update -> source -> gather (Alg 1).
 *
 * Split-field PML (O6b, g->iso_pml = 1; the paper's "standard PML ... in our second
 * order (isotropic) formulation", after Berenger [4]): inside the layers
 * (eta > 0) the field is the sum of three components, u = u^(x) + u^(y) + u^(z), each
 * damped along its own axis only,
 *   (d_t + eta_d)^2 u^(d) = v^2 d_d^2 u      (eta_d = eta_max xi_d^2 of O6),
 * centred in time:
 *   u^(d),n+1 = [(2 - (eta_d dt)^2) u^(d),n - (1 - eta_d dt) u^(d),n-1 + m L_d u^n] / (1 + eta_d dt),
 *   u^{n+1} = sum_d u^(d),n+1.
 * Outside the layers the update is Eq 1 as above (with eta_d = 0 the three component
 * updates sum to it).  A point source inside the layers enters the x component:
 * s^n / (1 + eta_x dt) is added to u^(x),n+1 and to u^{n+1}.                       */
int or_iso_run(const or_grid* g, const float* vp, double* u_prev, double* u_cur, double* w, int n0,
               int nsteps, const or_inj* inj, const or_rec* rec, double* seis) {
  init_coef();
  int rc = check_lists(g, inj, rec);
  if (rc) return rc;
  const double h = g->h, dt = g->dt;
  double vmax = vmax_of(g, vp);
  double* ex = (double*)malloc(sizeof(double) * g->nx);
  double* ey = (double*)malloc(sizeof(double) * g->ny);
  double* ez = (double*)malloc(sizeof(double) * g->nz);
  or_iso_eta(g->nx, g->nb, h, vmax, g->pml_R, ex);
  or_iso_eta(g->ny, g->nb, h, vmax, g->pml_R, ey);
  or_iso_eta(g->nz, g->nb, h, vmax, g->pml_R, ez);
  size_t n = NPTS(g);
  double* a = (double*)malloc(sizeof(double) * n); /* u^{n-1}, overwritten by u^{n+1} */
  double* b = (double*)malloc(sizeof(double) * n); /* u^n */
  memcpy(a, u_prev, sizeof(double) * n);
  memcpy(b, u_cur, sizeof(double) * n);
  const int spml = g->iso_pml == 1 && g->nb > 0;
  if (spml && !w) {
    free(a);
    free(b);
    free(ex);
    free(ey);
    free(ez);
    return -5;
  }
  double* wa[3]; /* u^(d),n-1 (overwritten by u^(d),n+1) */
  double* wb[3]; /* u^(d),n */
  for (int d = 0; d < 3; ++d) {
    wa[d] = spml ? w + (size_t)d * n : NULL;
    wb[d] = spml ? w + (size_t)(3 + d) * n : NULL;
  }

  for (int s = 0; s < nsteps; ++s) {
    int t = n0 + s;
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; ++k)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) {
          size_t p = IDX(g, i, j, k);
          double v = (double)vp[p];
          double m = v * v * dt * dt / (h * h);
          double eta = ex[i] + ey[j] + ez[k];
          if (spml && eta > 0.0) { /* O6b */
            const double ed[3] = {ex[i] * dt, ey[j] * dt, ez[k] * dt};
            double sum = 0.0;
            for (int d = 0; d < 3; ++d) {
              const double Ld = lap_axis(g, b, i, j, k, d);
              wa[d][p] = ((2.0 - ed[d] * ed[d]) * wb[d][p] - (1.0 - ed[d]) * wa[d][p] + m * Ld) / (1.0 + ed[d]);
              sum += wa[d][p];
            }
            a[p] = sum;
            continue;
          }
          double L = lap_at(g, b, i, j, k);
          a[p] = (2.0 * b[p] - (1.0 - eta * dt) * a[p] + m * L) / (1.0 + eta * dt);
        }
    if (inj)
      for (int r = 0; r < inj->n; ++r) {
        const int32_t* q = inj->pos + 3 * r;
        size_t p = IDX(g, q[0], q[1], q[2]);
        double v = (double)vp[p];
        double eta = ex[q[0]] + ey[q[1]] + ez[q[2]];
        const double amp = v * v * dt * dt * inj->amp[(size_t)t * inj->n + r] / (h * h * h);
        if (spml && eta > 0.0) { /* O6b: into the x component */
          const double sx = amp / (1.0 + ex[q[0]] * dt);
          a[p] += sx;
          wa[0][p] += sx;
          continue;
        }
        a[p] += amp / (1.0 + eta * dt);
      }
    if (rec && seis)
      for (int r = 0; r < rec->n; ++r) {
        const int32_t* q = rec->pos + 3 * r;
        seis[(size_t)s * rec->n + r] = a[IDX(g, q[0], q[1], q[2])];
      }
    double* tmp = a; /* logical swap of time levels */
    a = b;
    b = tmp;
    for (int d = 0; spml && d < 3; ++d) {
      tmp = wa[d];
      wa[d] = wb[d];
      wb[d] = tmp;
    }
  }
  memcpy(u_prev, a, sizeof(double) * n);
  memcpy(u_cur, b, sizeof(double) * n);
  if (spml && (nsteps & 1)) /* the caller's w[0] = level n-1, w[1] = level n */
    for (int d = 0; d < 3; ++d) {
      double* t0 = (double*)malloc(sizeof(double) * n);
      memcpy(t0, w + (size_t)d * n, sizeof(double) * n);
      memcpy(w + (size_t)d * n, w + (size_t)(3 + d) * n, sizeof(double) * n);
      memcpy(w + (size_t)(3 + d) * n, t0, sizeof(double) * n);
      free(t0);
    }
  free(a);
  free(b);
  free(ex);
  free(ey);
  free(ez);
  return 0;
}

/* ----------------------------------------------------- ACOUSTIC, O8 --- */
/* Buoyancy on the face between node i and i+1 along one axis:
 * b = 2 / (rho_i + rho_{i+1}); the last face clamps rho_{N} -> rho_{N-1} (O8). */
static double face_buoy(const or_grid* g, const float* rho, int axis, int i, int j, int k) {
  int e[3] = {0, 0, 0};
  e[axis] = 1;
  int n[3] = {g->nx, g->ny, g->nz};
  int c[3] = {i + e[0], j + e[1], k + e[2]};
  if (c[axis] >= n[axis]) c[axis] = (g->periodic && !(axis == 2 && g->free_surface)) ? 0 : n[axis] - 1;
  double r0 = atf(g, rho, i, j, k);
  double r1 = atf(g, rho, c[0], c[1], c[2]);
  return 2.0 / (r0 + r1);
}

typedef struct {
  double *a[3], *b[3], *ah[3], *bh[3];
} cpml_set;

static void cpml_alloc(const or_grid* g, double vmax, int top_layer, cpml_set* c) {
  int N[3] = {g->nx, g->ny, g->nz};
  for (int ax = 0; ax < 3; ++ax) {
    c->a[ax] = (double*)malloc(sizeof(double) * N[ax]);
    c->b[ax] = (double*)malloc(sizeof(double) * N[ax]);
    c->ah[ax] = (double*)malloc(sizeof(double) * N[ax]);
    c->bh[ax] = (double*)malloc(sizeof(double) * N[ax]);
    int lo = (ax == 2) ? top_layer : 1;
    or_cpml(N[ax], g->nb, lo, 1, g->h, g->dt, vmax, g->pml_R, g->pml_f, c->a[ax], c->b[ax],
            c->ah[ax], c->bh[ax]);
  }
}

static void cpml_free(cpml_set* c) {
  for (int ax = 0; ax < 3; ++ax) {
    free(c->a[ax]);
    free(c->b[ax]);
    free(c->ah[ax]);
    free(c->bh[ax]);
  }
}

/* Eq 2, extended to 3D with q_y, signs as printed:
 *   dp/dt = K div q + K d_t^{-1} f,   dq/dt = (1/rho) grad p,   K = rho v^2.
 * Grid (O8): p, K at (i,j,k); q_x at (i+1/2,j,k), q_y at (i,j+1/2,k), q_z at (i,j,k+1/2).
 * Leapfrog (O2):
 *   V: psi_{p,d} <- bh psi + ah D+_d p;   q_d += dt b_d (D+_d p + psi_{p,d})
 *   P: psi_{q,d} <- b psi + a D-_d q_d;   p += dt K sum_d (D-_d q_d + psi_{q,d})
 *   source p_s += dt K_s s[n] / h^3 (O11),   gather p (O13).                   */
int or_ac_run(const or_grid* g, const float* vp, const float* rho, double* p, double* qx,
              double* qy, double* qz, double* psi, int n0, int nsteps, const or_inj* inj,
              const or_rec* rec, double* seis) {
  init_coef();
  int rc = check_lists(g, inj, rec);
  if (rc) return rc;
  if (g->free_surface) return -4; /* EUNSUPPORTED in v1 (§8b) */
  const double h = g->h, dt = g->dt;
  size_t n = NPTS(g);
  cpml_set c;
  cpml_alloc(g, vmax_of(g, vp), 1, &c);
  double* q[3] = {qx, qy, qz};
  double* psi_p[3] = {psi, psi + n, psi + 2 * n};
  double* psi_q[3] = {psi + 3 * n, psi + 4 * n, psi + 5 * n};

  for (int s = 0; s < nsteps; ++s) {
    int t = n0 + s;
    /* V half-step: q^{n+1/2} from p^n */
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; ++k)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) {
          size_t o = IDX(g, i, j, k);
          int idx3[3] = {i, j, k};
          for (int ax = 0; ax < 3; ++ax) {
            double dp = dstag_at(g, at, p, ax, 1, i, j, k) / h;
            int l = idx3[ax];
            psi_p[ax][o] = c.bh[ax][l] * psi_p[ax][o] + c.ah[ax][l] * dp;
            q[ax][o] += dt * face_buoy(g, rho, ax, i, j, k) * (dp + psi_p[ax][o]);
          }
        }
    /* P half-step: p^{n+1} from q^{n+1/2} */
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; ++k)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) {
          size_t o = IDX(g, i, j, k);
          int idx3[3] = {i, j, k};
          double v = atf(g, vp, i, j, k), r = atf(g, rho, i, j, k);
          double K = r * v * v;
          double div = 0.0;
          for (int ax = 0; ax < 3; ++ax) {
            double dq = dstag_at(g, at, q[ax], ax, 0, i, j, k) / h;
            int l = idx3[ax];
            psi_q[ax][o] = c.b[ax][l] * psi_q[ax][o] + c.a[ax][l] * dq;
            div += dq + psi_q[ax][o];
          }
          p[o] += dt * K * div;
        }
    if (inj)
      for (int r = 0; r < inj->n; ++r) {
        const int32_t* qq = inj->pos + 3 * r;
        size_t o = IDX(g, qq[0], qq[1], qq[2]);
        double v = (double)vp[o], K = (double)rho[o] * v * v;
        p[o] += dt * K * inj->amp[(size_t)t * inj->n + r] / (h * h * h);
      }
    if (rec && seis)
      for (int r = 0; r < rec->n; ++r) {
        const int32_t* qq = rec->pos + 3 * r;
        seis[(size_t)s * rec->n + r] = p[IDX(g, qq[0], qq[1], qq[2])];
      }
  }
  cpml_free(&c);
  return 0;
}

/* ------------------------------------------------------ ELASTIC, O9 --- */
enum { VX, VY, VZ, SXX, SYY, SZZ, SXY, SXZ, SYZ };

/* Free-surface ghost accessors for z-derivatives above k = 0 (O16, stress
 * imaging): odd mirror for szz (integer z) and sxz/syz (half z); even mirror
 * for vx/vy (integer z) and vz (half z).  Elsewhere: zero outside the grid. */
static double acc_fs_int_odd(const or_grid* g, const double* f, int i, int j, int k) {
  if (k < 0 && g->free_surface) return -at(g, f, i, j, -k);
  return at(g, f, i, j, k);
}
static double acc_fs_half_odd(const or_grid* g, const double* f, int i, int j, int k) {
  if (k < 0 && g->free_surface) return -at(g, f, i, j, -1 - k);
  return at(g, f, i, j, k);
}
static double acc_fs_int_even(const or_grid* g, const double* f, int i, int j, int k) {
  if (k < 0 && g->free_surface) return at(g, f, i, j, -k);
  return at(g, f, i, j, k);
}
static double acc_fs_half_even(const or_grid* g, const double* f, int i, int j, int k) {
  if (k < 0 && g->free_surface) return at(g, f, i, j, -1 - k);
  return at(g, f, i, j, k);
}

/* Node value of mu with the grid-edge clamp (or periodic wrap). */
static double node_mu(const or_grid* g, const float* vs, const float* rho, int i, int j, int k) {
  if (g->periodic) {
    i = wrap(i, g->nx);
    j = wrap(j, g->ny);
  } else {
    if (i >= g->nx) i = g->nx - 1;
    if (j >= g->ny) j = g->ny - 1;
  }
  if (g->periodic && !g->free_surface) k = wrap(k, g->nz);
  else if (k >= g->nz) k = g->nz - 1;
  double s = atf(g, vs, i, j, k);
  return atf(g, rho, i, j, k) * s * s;
}

/* Edge mu: harmonic mean of the 4 adjacent node values, 0 if any is 0 (O9). */
static double edge_mu(const or_grid* g, const float* vs, const float* rho, int i, int j, int k,
                      int a1, int a2) {
  int e1[3] = {0, 0, 0}, e2[3] = {0, 0, 0};
  e1[a1] = 1;
  e2[a2] = 1;
  double m[4];
  m[0] = node_mu(g, vs, rho, i, j, k);
  m[1] = node_mu(g, vs, rho, i + e1[0], j + e1[1], k + e1[2]);
  m[2] = node_mu(g, vs, rho, i + e2[0], j + e2[1], k + e2[2]);
  m[3] = node_mu(g, vs, rho, i + e1[0] + e2[0], j + e1[1] + e2[1], k + e1[2] + e2[2]);
  double inv = 0.0;
  for (int t = 0; t < 4; ++t) {
    if (m[t] == 0.0) return 0.0;
    inv += 1.0 / m[t];
  }
  return 4.0 / inv;
}

/* Eq 3 on the Virieux grid (O9):
 *   vx (i+1/2,j,k)  vy (i,j+1/2,k)  vz (i,j,k+1/2)
 *   sxx, syy, szz, lambda, mu, rho (i,j,k)
 *   sxy (i+1/2,j+1/2,k)  sxz (i+1/2,j,k+1/2)  syz (i,j+1/2,k+1/2)
 * psi order (18): V terms  0 dx sxx, 1 dy sxy, 2 dz sxz (vx); 3 dx sxy, 4 dy syy,
 *   5 dz syz (vy); 6 dx sxz, 7 dy syz, 8 dz szz (vz);  S terms 9 dx vx, 10 dy vy,
 *   11 dz vz (normal); 12 dy vx, 13 dx vy (sxy); 14 dz vx, 15 dx vz (sxz);
 *   16 dz vy, 17 dy vz (syz).
 * Step order (O2): V -> S -> source -> free-surface fix-up -> gather.        */
int or_el_run(const or_grid* g, const float* vp, const float* vs, const float* rho, double* f,
              double* psi, int n0, int nsteps, const or_inj* inj, const or_rec* rec,
              double* seis) {
  init_coef();
  int rc = check_lists(g, inj, rec);
  if (rc) return rc;
  const double h = g->h, dt = g->dt;
  size_t n = NPTS(g);
  cpml_set c;
  cpml_alloc(g, vmax_of(g, vp), g->free_surface ? 0 : 1, &c);
  double* F[9];
  double* P[18];
  for (int t = 0; t < 9; ++t) F[t] = f + (size_t)t * n;
  for (int t = 0; t < 18; ++t) P[t] = psi + (size_t)t * n;

  for (int s = 0; s < nsteps; ++s) {
    int t = n0 + s;
    /* ---- V: v^{n+1/2} from sigma^n ---- */
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; ++k)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) {
          size_t o = IDX(g, i, j, k);
          double d;
          /* vx at (i+1/2,j,k): Dx+ sxx, Dy- sxy, Dz- sxz */
          double acc = 0.0;
          d = dstag_at(g, at, F[SXX], 0, 1, i, j, k) / h;
          P[0][o] = c.bh[0][i] * P[0][o] + c.ah[0][i] * d;
          acc += d + P[0][o];
          d = dstag_at(g, at, F[SXY], 1, 0, i, j, k) / h;
          P[1][o] = c.b[1][j] * P[1][o] + c.a[1][j] * d;
          acc += d + P[1][o];
          d = dstag_at(g, acc_fs_half_odd, F[SXZ], 2, 0, i, j, k) / h;
          P[2][o] = c.b[2][k] * P[2][o] + c.a[2][k] * d;
          acc += d + P[2][o];
          F[VX][o] += dt * face_buoy(g, rho, 0, i, j, k) * acc;
          /* vy at (i,j+1/2,k): Dx- sxy, Dy+ syy, Dz- syz */
          acc = 0.0;
          d = dstag_at(g, at, F[SXY], 0, 0, i, j, k) / h;
          P[3][o] = c.b[0][i] * P[3][o] + c.a[0][i] * d;
          acc += d + P[3][o];
          d = dstag_at(g, at, F[SYY], 1, 1, i, j, k) / h;
          P[4][o] = c.bh[1][j] * P[4][o] + c.ah[1][j] * d;
          acc += d + P[4][o];
          d = dstag_at(g, acc_fs_half_odd, F[SYZ], 2, 0, i, j, k) / h;
          P[5][o] = c.b[2][k] * P[5][o] + c.a[2][k] * d;
          acc += d + P[5][o];
          F[VY][o] += dt * face_buoy(g, rho, 1, i, j, k) * acc;
          /* vz at (i,j,k+1/2): Dx- sxz, Dy- syz, Dz+ szz */
          acc = 0.0;
          d = dstag_at(g, at, F[SXZ], 0, 0, i, j, k) / h;
          P[6][o] = c.b[0][i] * P[6][o] + c.a[0][i] * d;
          acc += d + P[6][o];
          d = dstag_at(g, at, F[SYZ], 1, 0, i, j, k) / h;
          P[7][o] = c.b[1][j] * P[7][o] + c.a[1][j] * d;
          acc += d + P[7][o];
          d = dstag_at(g, acc_fs_int_odd, F[SZZ], 2, 1, i, j, k) / h;
          P[8][o] = c.bh[2][k] * P[8][o] + c.ah[2][k] * d;
          acc += d + P[8][o];
          F[VZ][o] += dt * face_buoy(g, rho, 2, i, j, k) * acc;
        }
    /* ---- S: sigma^{n+1} from v^{n+1/2} ---- */
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; ++k)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) {
          size_t o = IDX(g, i, j, k);
          double vpv = atf(g, vp, i, j, k), vsv = atf(g, vs, i, j, k), r = atf(g, rho, i, j, k);
          double mu = r * vsv * vsv;
          double lam = r * (vpv * vpv - 2.0 * vsv * vsv);
          double l2m = lam + 2.0 * mu;
          double d;
          /* normal stresses: Dx- vx, Dy- vy, Dz- vz at (i,j,k) */
          d = dstag_at(g, at, F[VX], 0, 0, i, j, k) / h;
          P[9][o] = c.b[0][i] * P[9][o] + c.a[0][i] * d;
          double exx = d + P[9][o];
          d = dstag_at(g, at, F[VY], 1, 0, i, j, k) / h;
          P[10][o] = c.b[1][j] * P[10][o] + c.a[1][j] * d;
          double eyy = d + P[10][o];
          d = dstag_at(g, acc_fs_half_even, F[VZ], 2, 0, i, j, k) / h;
          P[11][o] = c.b[2][k] * P[11][o] + c.a[2][k] * d;
          double ezz = d + P[11][o];
          if (g->free_surface && k == 0) ezz = -lam / l2m * (exx + eyy); /* O16 surface row */
          F[SXX][o] += dt * (l2m * exx + lam * (eyy + ezz));
          F[SYY][o] += dt * (l2m * eyy + lam * (exx + ezz));
          F[SZZ][o] += dt * (l2m * ezz + lam * (exx + eyy));
          /* sxy at (i+1/2,j+1/2,k): Dy+ vx + Dx+ vy */
          double dvx, dvy;
          dvx = dstag_at(g, at, F[VX], 1, 1, i, j, k) / h;
          P[12][o] = c.bh[1][j] * P[12][o] + c.ah[1][j] * dvx;
          dvy = dstag_at(g, at, F[VY], 0, 1, i, j, k) / h;
          P[13][o] = c.bh[0][i] * P[13][o] + c.ah[0][i] * dvy;
          F[SXY][o] += dt * edge_mu(g, vs, rho, i, j, k, 0, 1) *
                       (dvx + P[12][o] + dvy + P[13][o]);
          /* sxz at (i+1/2,j,k+1/2): Dz+ vx + Dx+ vz */
          double dvz;
          dvx = dstag_at(g, acc_fs_int_even, F[VX], 2, 1, i, j, k) / h;
          P[14][o] = c.bh[2][k] * P[14][o] + c.ah[2][k] * dvx;
          dvz = dstag_at(g, at, F[VZ], 0, 1, i, j, k) / h;
          P[15][o] = c.bh[0][i] * P[15][o] + c.ah[0][i] * dvz;
          F[SXZ][o] += dt * edge_mu(g, vs, rho, i, j, k, 0, 2) *
                       (dvx + P[14][o] + dvz + P[15][o]);
          /* syz at (i,j+1/2,k+1/2): Dz+ vy + Dy+ vz */
          dvy = dstag_at(g, acc_fs_int_even, F[VY], 2, 1, i, j, k) / h;
          P[16][o] = c.bh[2][k] * P[16][o] + c.ah[2][k] * dvy;
          dvz = dstag_at(g, at, F[VZ], 1, 1, i, j, k) / h;
          P[17][o] = c.bh[1][j] * P[17][o] + c.ah[1][j] * dvz;
          F[SYZ][o] += dt * edge_mu(g, vs, rho, i, j, k, 1, 2) *
                       (dvy + P[16][o] + dvz + P[17][o]);
        }
    /* explosive source (O11): sigma_ii -= dt (lambda + 2/3 mu) s[n] / h^3 */
    if (inj)
      for (int r = 0; r < inj->n; ++r) {
        const int32_t* qq = inj->pos + 3 * r;
        size_t o = IDX(g, qq[0], qq[1], qq[2]);
        double vpv = (double)vp[o], vsv = (double)vs[o], rr = (double)rho[o];
        double mu = rr * vsv * vsv, lam = rr * (vpv * vpv - 2.0 * vsv * vsv);
        double add = dt * (lam + 2.0 / 3.0 * mu) * inj->amp[(size_t)t * inj->n + r] / (h * h * h);
        F[SXX][o] -= add;
        F[SYY][o] -= add;
        F[SZZ][o] -= add;
      }
    /* free-surface fix-up (O16): szz = 0 on the surface plane */
    if (g->free_surface)
      for (int j = 0; j < g->ny; ++j)
        for (int i = 0; i < g->nx; ++i) F[SZZ][IDX(g, i, j, 0)] = 0.0;
    if (rec && seis)
      for (int r = 0; r < rec->n; ++r) {
        const int32_t* qq = rec->pos + 3 * r;
        size_t o = IDX(g, qq[0], qq[1], qq[2]);
        double val;
        switch (rec->component) {
          case 0: val = F[VX][o]; break;
          case 1: val = F[VY][o]; break;
          case 3: val = -(F[SXX][o] + F[SYY][o] + F[SZZ][o]) / 3.0; break;
          default: val = F[VZ][o]; break;
        }
        seis[(size_t)s * rec->n + r] = val;
      }
  }
  cpml_free(&c);
  return 0;
}

/* --------------------------------------------------------- RTM, O15 --- */
/* Algorithm 1 with snapshots kept in memory (O14):
 *  forward: for n = 0..nt-1: step (source injection inside); if level n+1 is a
 *           snapshot level (multiple of snap, <= nt-1) save S_{n+1}.
 *  backward (the paper's order, imaging BEFORE the step):
 *           R = 0; for m = 0..nt-1: j = nt - m; if j is a snapshot level,
 *           image += S_j * R; step R with receiver injection of data[nt-1-m][r].
 * This pairs S_j with R^{m+1}, j = nt-1-m (O15).  ELASTIC (f3): snapshots and
 * imaging use the pressure -(sxx+syy+szz)/3; receivers inject as explosive sources. */
int or_migrate(const or_grid* g, int kind, const float* vp, const float* vs, const float* rho,
               const int32_t src_pos[3], const double* src_amp, int nt, int nrec,
               const int32_t* rec_pos, const double* data, int snap, double* image) {
  if (snap < 1 || nt < 1) return -1;
  if (kind != 0 && kind != 1 && kind != 2) return -4;
  size_t n = NPTS(g);
  int nsnap = (nt - 1) / snap;
  double* S = (double*)calloc((size_t)(nsnap > 0 ? nsnap : 1) * n, sizeof(double));
  double* back_amp = (double*)malloc(sizeof(double) * (size_t)nt * (nrec > 0 ? nrec : 1));
  for (int m = 0; m < nt; ++m)
    for (int r = 0; r < nrec; ++r)
      back_amp[(size_t)m * nrec + r] = data[(size_t)(nt - 1 - m) * nrec + r];
  or_inj src = {1, src_pos, src_amp};
  or_inj recinj = {nrec, rec_pos, back_amp};
  int rc = 0;
  double *a = (double*)calloc(n, sizeof(double)), *b = (double*)calloc(n, sizeof(double));
  double *q = NULL, *psi = NULL, *f = NULL, *w = NULL;
  if (kind == 0) w = (double*)calloc(6 * n, sizeof(double)); /* O6b split fields (if used) */
  if (kind == 1) {
    q = (double*)calloc(3 * n, sizeof(double));
    psi = (double*)calloc(6 * n, sizeof(double));
  }
  if (kind == 2) { /* elastic: 9 fields, 18 psi; imaged field = pressure -(sxx+syy+szz)/3 */
    f = (double*)calloc(9 * n, sizeof(double));
    psi = (double*)calloc(18 * n, sizeof(double));
  }
  /* forward phase */
  for (int t = 0; t < nt && !rc; ++t) {
    if (kind == 0) {
      rc = or_iso_run(g, vp, a, b, w, t, 1, &src, NULL, NULL);
    } else if (kind == 1) {
      rc = or_ac_run(g, vp, rho, b, q, q + n, q + 2 * n, psi, t, 1, &src, NULL, NULL);
    } else {
      rc = or_el_run(g, vp, vs, rho, f, psi, t, 1, &src, NULL, NULL);
      for (size_t o = 0; o < n; ++o) b[o] = -(f[3 * n + o] + f[4 * n + o] + f[5 * n + o]) / 3.0;
    }
    int j = t + 1;
    if (j % snap == 0 && j <= nt - 1) memcpy(S + (size_t)(j / snap - 1) * n, b, sizeof(double) * n);
  }
  /* backward phase: fresh zero state */
  memset(a, 0, sizeof(double) * n);
  memset(b, 0, sizeof(double) * n);
  if (kind == 0) memset(w, 0, sizeof(double) * 6 * n);
  if (kind == 1) {
    memset(q, 0, sizeof(double) * 3 * n);
    memset(psi, 0, sizeof(double) * 6 * n);
  }
  if (kind == 2) {
    memset(f, 0, sizeof(double) * 9 * n);
    memset(psi, 0, sizeof(double) * 18 * n);
  }
  for (int m = 0; m < nt && !rc; ++m) {
    int j = nt - m;
    if (j % snap == 0 && j >= snap && j <= nt - 1) {
      const double* Sj = S + (size_t)(j / snap - 1) * n;
      for (size_t o = 0; o < n; ++o) image[o] += Sj[o] * b[o]; /* P:111 zero-lag */
    }
    if (kind == 0) {
      rc = or_iso_run(g, vp, a, b, w, m, 1, &recinj, NULL, NULL);
    } else if (kind == 1) {
      rc = or_ac_run(g, vp, rho, b, q, q + n, q + 2 * n, psi, m, 1, &recinj, NULL, NULL);
    } else {
      /* receivers inject as explosive sources (O11 scaling), the imaged field is pressure */
      rc = or_el_run(g, vp, vs, rho, f, psi, m, 1, &recinj, NULL, NULL);
      for (size_t o = 0; o < n; ++o) b[o] = -(f[3 * n + o] + f[4 * n + o] + f[5 * n + o]) / 3.0;
    }
  }
  free(S);
  free(back_amp);
  free(a);
  free(b);
  free(q);
  free(psi);
  free(f);
  free(w);
  return rc;
}
