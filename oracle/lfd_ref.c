/*
 * lfd_ref.c -- plain, slow, obviously-correct CPU ORACLE of the DC-MESH LFD time step.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path (the CUDA library under
 * paper_conf_ipps_razakhllknvn24_b200/, the Python binding) may include, link, import or call
 * this file.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg use it.  It shares no code, header, table or constant generator with the CUDA path.
 *
 * Source of truth: /root/reference/PAPER.md ("P:n" = line n) and the readings R1..R22 of
 * SURVEY.md §8(c), restated in DESIGN.md §3.  Everything is FP64 / complex128, natural index
 * order, libm sin/cos/exp, no BLAS, no blocking, no fusion, single-threaded.
 *
 * Data layout (matches the paper's SoA psi[i][j][k][n], orbital fastest):
 *   psi  [ndom][nx][ny][nz][norb]   complex128 (re, im interleaved = C99 double complex)
 *   proj [ndom][nx][ny][nz][nproj]  complex128  (B = Psi_u(0), the unoccupied KS orbitals; R9)
 *   vloc [ndom][nx][ny][nz]         double      (v_loc of Eq. 5)
 *   A    [ndom][3]                  double      (A_X(alpha) of Eq. 2/5 at the step midpoint, Eq. 4)
 *   dnl  [ndom][nproj]              double      (D_u; paper: all = Delta_sci, Eq. 7-8)
 *   occ  [ndom][norb]               double      (f_s of P:44)
 * Atomic units (R1): hbar = m = e = 1, c = 137.035999084.
 *
 * Parity status of each function (see DESIGN.md §4 and tests/test_oracle_pins.py):
 *   lfd_ref_link_sweep       pinned: dense scipy expm of the link-set Hamiltonian; H_E+H_O = FD op.
 *   lfd_ref_kinetic          pinned: plane-wave closed form; O(dt^2) convergence; commutation.
 *   lfd_ref_local            pinned: product of dense expms on a tiny 3-D grid; time reversal.
 *   lfd_ref_nl_half          pinned: norm closed form; Gram closed form; BLAS (numpy) for C.
 *   lfd_ref_nl_half_exact    pinned: dense scipy expm of -i(Delta/2) B D B^H dV; projector columns get
 *                            e^{-i(Delta/2)D_u}; span(B)-orthogonal part unchanged; unitary.
 *   lfd_ref_step_exact       pinned: Gram matrix (orthonormality) conserved for D != 0; second-order
 *                            convergence to dense expm(-i T (H_FD + V + B diag(D) B^H dV)).
 *   lfd_ref_step             pinned: norm / orthonormality conservation; gauge covariance; with the
 *                            nonlocal factor ON (tests/test_oracle_pins_step.py): closed form on
 *                            projector plane waves (lambda_u f_u^2, f_u = (1-i eps D_u)/|.|) and on a
 *                            two-column mix; first-order convergence to the same dense expm.
 *   lfd_ref_nl_half_dense    pinned (tests/test_oracle_pins_dense.py): diagonal D equals lfd_ref_nl_half; a
 *                            rotated diagonal D equals the diagonal factor on rotated projectors; the step
 *                            converges (order 1) to dense expm(-i T (H_FD + V + B D B^H dV)).
 *   lfd_ref_nl_half_exact_dense pinned: dense scipy expm of -i(Delta/2) B D B^H dV on orthonormal B; the
 *                            exact dense step converges at second order to the same expm.
 *   lfd_ref_energy_nl_dense  pinned: equals <psi| B D B^H dV |psi> with dense matrices.
 *   lfd_ref_density_current  pinned: plane-wave closed forms; sum rule; J = dE_kin/dA / V.
 *   lfd_ref_energy           pinned: plane-wave closed forms (kinetic, local = f mean(v)); nonlocal on
 *                            projector columns = f D_u; O(dt^2) energy drift of the step at A = D = 0.
 *   lfd_ref_remap_occ        pinned: onto the grid basis it equals rho dV; on the t = 0 basis it gives
 *                            back f; sum rule over a complete basis.
 *   Faithfulness to the paper's own printed numbers: parity unpinned (the paper prints none).
 */
#include <complex.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define REF_C_LIGHT 137.035999084 /* R1 */
#define REF_BC_PERIODIC 0
#define REF_BC_ZERO 1

/* Mirror of the problem description (its own definition; not the product header). */
typedef struct {
  int32_t ndom;
  int32_t nx, ny, nz;
  double hx, hy, hz;
  int32_t bc;
  int32_t norb;
  int32_t nproj;
  double dt;
} lfd_ref_config;

static int ref_check(const lfd_ref_config* c) {
  if (!c || c->ndom < 1 || c->nx < 2 || c->ny < 2 || c->nz < 2 || c->norb < 1 || c->nproj < 0) return -1;
  if (!(c->hx > 0) || !(c->hy > 0) || !(c->hz > 0) || c->dt == 0.0) return -1;
  if (c->bc != REF_BC_PERIODIC && c->bc != REF_BC_ZERO) return -1;
  if (c->bc == REF_BC_PERIODIC && ((c->nx | c->ny | c->nz) & 1)) return -1; /* R8 */
  return 0;
}

/* Flat index of (ix, iy, iz) -- grid index r = ((ix*ny)+iy)*nz+iz (SoA). */
static size_t gidx(const lfd_ref_config* c, int ix, int iy, int iz) {
  return ((size_t)ix * c->ny + iy) * c->nz + iz;
}

/* ---------------------------------------------------------------------------------------------
 * Pair (2x2) block of the space-splitting propagator.  SURVEY §8(c) step 1, readings R2-R4.
 * Paper: P:80 (§III: "time step p in {Delta/2, Delta}, diagonal, upper-diagonal and
 * lower-diagonal coefficients alpha_dp, beta_l,dp, beta_u,dp"), Alg. 1 l.7 (scalar al[d][p]),
 * Alg. 3 l.11 (per-point bl[i]).
 *
 * For the link Hamiltonian L = t [[1, -e^{i theta}], [-e^{-i theta}, 1]], t = 1/(2h^2),
 * theta = a h, a = A_d / c:
 *   exp(-i tau L) = e^{-i tau t} [[cos(tau t), i sin(tau t) e^{i theta}],
 *                                 [i sin(tau t) e^{-i theta}, cos(tau t)]]
 *   => alpha = e^{-i tau t} cos(tau t),  sigma = i e^{-i tau t} sin(tau t)
 *      psi'_i  = alpha psi_i + sigma e^{+i theta} psi_i'
 *      psi'_i' = sigma e^{-i theta} psi_i + alpha psi_i'
 * A singleton (zero-BC end point without a link) gets the on-site factor e^{-i tau t}.
 * ------------------------------------------------------------------------------------------- */
typedef struct {
  double complex alpha, up, dn, onsite;
} ref_pair;

static ref_pair ref_pair_coeffs(double tau, double h, double a) {
  ref_pair p;
  double t = 1.0 / (2.0 * h * h);
  double theta = a * h;
  double complex ph = cexp(-I * tau * t);
  double complex sigma = I * ph * sin(tau * t);
  p.alpha = ph * cos(tau * t);
  p.up = sigma * cexp(I * theta);
  p.dn = sigma * cexp(-I * theta);
  p.onsite = ph;
  return p;
}

/* Apply one pair block to the link (i, i2) of a strided line. */
static void ref_apply_link(double complex* line, size_t stride, int i, int i2, const ref_pair* p) {
  double complex a = line[(size_t)i * stride];
  double complex b = line[(size_t)i2 * stride];
  line[(size_t)i * stride] = p->alpha * a + p->up * b;
  line[(size_t)i2 * stride] = p->dn * a + p->alpha * b;
}

/* One link-set sweep along a single line of n points (stride between points in complex units).
 * parity 0 = E_d: links (2m, 2m+1); parity 1 = O_d: links (2m+1, 2m+2) and, if periodic, the
 * wrap link (n-1, 0).  SURVEY §8(c) step 2, reading R5 (0-based origin, E first), R8 (BC). */
static void ref_sweep_line(double complex* line, size_t stride, int n, int bc, int parity,
                           const ref_pair* p) {
  if (parity == 0) {
    for (int i = 0; i + 1 < n; i += 2) ref_apply_link(line, stride, i, i + 1, p);
    if (n & 1) line[(size_t)(n - 1) * stride] *= p->onsite; /* only reachable with zero BC */
  } else {
    for (int i = 1; i + 1 < n; i += 2) ref_apply_link(line, stride, i, i + 1, p);
    if (bc == REF_BC_PERIODIC) {
      ref_apply_link(line, stride, n - 1, 0, p); /* wrap link, n even */
    } else {
      line[0] *= p->onsite;                                        /* point 0 has no O link */
      if ((n & 1) == 0) line[(size_t)(n - 1) * stride] *= p->onsite; /* even n: last point too */
    }
  }
}

/* Public: one E_d or O_d sweep over every line along axis d, every orbital, one domain.
 * psi: [nx][ny][nz][norb]; axis 0/1/2 = x/y/z; tau = time of this factor; a = A_d / c. */
int lfd_ref_link_sweep(const lfd_ref_config* c, double complex* psi, int axis, int parity,
                       double tau, double a) {
  if (ref_check(c) || axis < 0 || axis > 2 || (parity != 0 && parity != 1) || !psi) return -1;
  const int n[3] = {c->nx, c->ny, c->nz};
  const double h[3] = {c->hx, c->hy, c->hz};
  ref_pair p = ref_pair_coeffs(tau, h[axis], a);
  size_t stride_pts[3] = {(size_t)c->ny * c->nz, (size_t)c->nz, 1};
  size_t stride = stride_pts[axis] * (size_t)c->norb;
  int o1 = (axis + 1) % 3, o2 = (axis + 2) % 3;
  for (int j1 = 0; j1 < n[o1]; ++j1)
    for (int j2 = 0; j2 < n[o2]; ++j2)
      for (int s = 0; s < c->norb; ++s) {
        size_t base = (j1 * stride_pts[o1] + j2 * stride_pts[o2]) * (size_t)c->norb + s;
        ref_sweep_line(psi + base, stride, n[axis], c->bc, parity, &p);
      }
  return 0;
}

/* Public: K_d = E_d(tau/2) O_d(tau) E_d(tau/2), E first (R4, R5).  With tau = Delta this is the
 * paper's pair of time steps p in {Delta/2, Delta}. */
int lfd_ref_kinetic(const lfd_ref_config* c, double complex* psi, int axis, double tau, double a) {
  int e = 0;
  e |= lfd_ref_link_sweep(c, psi, axis, 0, 0.5 * tau, a);
  e |= lfd_ref_link_sweep(c, psi, axis, 1, tau, a);
  e |= lfd_ref_link_sweep(c, psi, axis, 0, 0.5 * tau, a);
  return e ? -1 : 0;
}

/* Public: local propagator of one domain, exp(-i Delta h_loc) of Eq. 6 by space
 * splitting:  Psi <- Phi . K_z K_y K_x (Phi . Psi),  Phi = e^{-i (Delta/2) v_loc}
 * (R6 direction order x, y, z; R7 Strang placement of the potential phase). A: [3] a.u. */
int lfd_ref_local(const lfd_ref_config* c, double complex* psi, const double* vloc, const double* A) {
  if (ref_check(c) || !psi || !vloc || !A) return -1;
  size_t ng = (size_t)c->nx * c->ny * c->nz;
  double half = 0.5 * c->dt;
  for (size_t r = 0; r < ng; ++r) {
    double complex phi = cexp(-I * half * vloc[r]);
    for (int s = 0; s < c->norb; ++s) psi[r * c->norb + s] *= phi;
  }
  for (int d = 0; d < 3; ++d)
    if (lfd_ref_kinetic(c, psi, d, c->dt, A[d] / REF_C_LIGHT)) return -1;
  for (size_t r = 0; r < ng; ++r) {
    double complex phi = cexp(-I * half * vloc[r]);
    for (int s = 0; s < c->norb; ++s) psi[r * c->norb + s] *= phi;
  }
  return 0;
}

/* Public: one renormalised nonlocal factor N of Eq. 6 with the scissor projector of
 * Eq. 7 in the BLASified form of Eq. 9, readings R9-R12:
 *   C_us   = dV sum_r conj(B_ru) Psi_rs                                  (first BLAS-3 call)
 *   Psi'_rs = Psi_rs - i (Delta/2) sum_u B_ru D_u C_us                   (second BLAS-3 call)
 *   Psi'_.s <- Psi'_.s * sqrt( sum_r |Psi_rs|^2 / sum_r |Psi'_rs|^2 )     (the ||.|| denominator)
 * Both norms are direct grid sums here (independent of the GPU's Gram route). */
int lfd_ref_nl_half(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                    const double* dnl) {
  if (ref_check(c) || !psi) return -1;
  if (c->nproj == 0) return 0;
  if (!proj || !dnl) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  const double dV = c->hx * c->hy * c->hz;
  const double eps = 0.5 * c->dt;
  double complex* C = calloc((size_t)np * no, sizeof(double complex));
  double* n0 = calloc((size_t)no, sizeof(double));
  double* n1 = calloc((size_t)no, sizeof(double));
  double complex* row = malloc((size_t)no * sizeof(double complex));
  if (!C || !n0 || !n1 || !row) { free(C); free(n0); free(n1); free(row); return -2; }
  for (size_t r = 0; r < ng; ++r)
    for (int s = 0; s < no; ++s) {
      double complex v = psi[r * no + s];
      n0[s] += creal(v) * creal(v) + cimag(v) * cimag(v);
    }
  for (size_t r = 0; r < ng; ++r)
    for (int u = 0; u < np; ++u) {
      double complex bc = conj(proj[r * np + u]);
      for (int s = 0; s < no; ++s) C[(size_t)u * no + s] += bc * psi[r * no + s];
    }
  for (size_t k = 0; k < (size_t)np * no; ++k) C[k] *= dV;
  for (size_t r = 0; r < ng; ++r) {
    for (int s = 0; s < no; ++s) row[s] = 0.0;
    for (int u = 0; u < np; ++u) {
      double complex b = proj[r * np + u] * dnl[u];
      for (int s = 0; s < no; ++s) row[s] += b * C[(size_t)u * no + s];
    }
    for (int s = 0; s < no; ++s) {
      double complex v = psi[r * no + s] - I * eps * row[s];
      psi[r * no + s] = v;
      n1[s] += creal(v) * creal(v) + cimag(v) * cimag(v);
    }
  }
  for (int s = 0; s < no; ++s) {
    double f = sqrt(n0[s] / n1[s]);
    for (size_t r = 0; r < ng; ++r) psi[r * no + s] *= f;
  }
  free(C); free(n0); free(n1); free(row);
  return 0;
}

/* Public: the EXACTLY UNITARY nonlocal factor, for projector
 * columns that are dV-orthonormal (dV B^H B = I). Then v_nl = B diag(D) B^H dV has the spectral form
 * sum_u D_u P_u with orthogonal projectors P_u = |B_u><B_u| dV, so the factor of Eq. 6 taken exactly
 * instead of to first order,  exp(-i (Delta/2) v_nl) = 1 + sum_u (e^{-i (Delta/2) D_u} - 1) P_u,  is
 *   C_us    = dV sum_r conj(B_ru) Psi_rs
 *   Psi'_rs = Psi_rs + sum_u B_ru (e^{-i (Delta/2) D_u} - 1) C_us
 * and needs no renormalisation (the ||.|| denominator of Eq. 6 is 1). One domain (c->ndom ignored). */
int lfd_ref_nl_half_exact(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                          const double* dnl) {
  if (ref_check(c) || !psi) return -1;
  if (c->nproj == 0) return 0;
  if (!proj || !dnl) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  const double dV = c->hx * c->hy * c->hz;
  const double eps = 0.5 * c->dt;
  double complex* C = calloc((size_t)np * no, sizeof(double complex));
  double complex* row = malloc((size_t)no * sizeof(double complex));
  if (!C || !row) { free(C); free(row); return -2; }
  for (size_t r = 0; r < ng; ++r)
    for (int u = 0; u < np; ++u) {
      double complex bc = conj(proj[r * np + u]);
      for (int s = 0; s < no; ++s) C[(size_t)u * no + s] += bc * psi[r * no + s];
    }
  for (size_t k = 0; k < (size_t)np * no; ++k) C[k] *= dV;
  for (size_t r = 0; r < ng; ++r) {
    for (int s = 0; s < no; ++s) row[s] = 0.0;
    for (int u = 0; u < np; ++u) {
      double complex b = proj[r * np + u] * (cexp(-I * eps * dnl[u]) - 1.0);
      for (int s = 0; s < no; ++s) row[s] += b * C[(size_t)u * no + s];
    }
    for (int s = 0; s < no; ++s) psi[r * no + s] += row[s];
  }
  free(C); free(row);
  return 0;
}

/* Public: nsteps LFD steps with the exactly unitary nonlocal factor (N_exact o Local o N_exact). */
int lfd_ref_step_exact(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                       const double* dnl, const double* vloc, const double* A, int nsteps) {
  if (ref_check(c) || !psi || !vloc || !A || nsteps < 0) return -1;
  if (c->nproj > 0 && (!proj || !dnl)) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  lfd_ref_config one = *c;
  one.ndom = 1;
  for (int it = 0; it < nsteps; ++it)
    for (int dm = 0; dm < c->ndom; ++dm) {
      double complex* p = psi + (size_t)dm * ng * c->norb;
      const double complex* b = proj ? proj + (size_t)dm * ng * c->nproj : NULL;
      const double* d = dnl ? dnl + (size_t)dm * c->nproj : NULL;
      int e = lfd_ref_nl_half_exact(&one, p, b, d);
      e |= lfd_ref_local(&one, p, vloc + (size_t)dm * ng, A + 3 * dm);
      e |= lfd_ref_nl_half_exact(&one, p, b, d);
      if (e) return -1;
    }
  return 0;
}

/* Public: nsteps LFD steps of Eq. 6 for every domain:
 *   Psi <- N( Local( N(Psi) ) )    (rightmost factor acts first).
 * vloc / A are held fixed over the nsteps (the caller re-sets them at each step midpoint, Eq. 4,
 * P:54, reading R15).  psi/proj/vloc/A/dnl are per-domain arrays as in the header comment. */
int lfd_ref_step(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                 const double* dnl, const double* vloc, const double* A, int nsteps) {
  if (ref_check(c) || !psi || !vloc || !A || nsteps < 0) return -1;
  if (c->nproj > 0 && (!proj || !dnl)) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  lfd_ref_config one = *c;
  one.ndom = 1;
  for (int it = 0; it < nsteps; ++it)
    for (int dm = 0; dm < c->ndom; ++dm) {
      double complex* p = psi + (size_t)dm * ng * c->norb;
      const double complex* b = proj ? proj + (size_t)dm * ng * c->nproj : NULL;
      const double* d = dnl ? dnl + (size_t)dm * c->nproj : NULL;
      int e = lfd_ref_nl_half(&one, p, b, d);
      e |= lfd_ref_local(&one, p, vloc + (size_t)dm * ng, A + 3 * dm);
      e |= lfd_ref_nl_half(&one, p, b, d);
      if (e) return -1;
    }
  return 0;
}

/* ---------------------------------------------------------------------------------------------
 * Dense Hermitian D. Eq. 5 puts the nonlocal ionic pseudopotential into
 * v_nl; in Kleinman-Bylander form it is  v_nl = sum_{u,v} |b_u> D_uv <b_v|  with a Hermitian coupling
 * matrix D (the scissor operator of Eq. 7, is the special case D = Delta_sci I). With
 * <a|b> = dV sum_r conj(a_r) b_r (R12), Eq. 9's BLASified form reads
 *   C = dV B^H Psi,   Psi' = Psi - i (Delta/2) B (D C),
 * and N of Eq. 6 renormalises each orbital to its pre-factor norm (R11). Dm: [nproj][nproj] complex,
 * row-major D[u][v], one domain. Both norms are direct grid sums.
 * ------------------------------------------------------------------------------------------- */
static void ref_project(const lfd_ref_config* c, const double complex* psi, const double complex* proj,
                        double complex* C) {
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  const double dV = c->hx * c->hy * c->hz;
  for (size_t k = 0; k < (size_t)np * no; ++k) C[k] = 0.0;
  for (size_t r = 0; r < ng; ++r)
    for (int u = 0; u < np; ++u) {
      double complex bc = conj(proj[r * np + u]);
      for (int s = 0; s < no; ++s) C[(size_t)u * no + s] += bc * psi[r * no + s];
    }
  for (size_t k = 0; k < (size_t)np * no; ++k) C[k] *= dV;
}

/* Psi += B Y (Y [nproj][norb]), the back-projection of Eq. 9. */
static void ref_backproject(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                            const double complex* Y) {
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  for (size_t r = 0; r < ng; ++r)
    for (int u = 0; u < np; ++u) {
      double complex b = proj[r * np + u];
      for (int s = 0; s < no; ++s) psi[r * no + s] += b * Y[(size_t)u * no + s];
    }
}

int lfd_ref_nl_half_dense(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                          const double complex* Dm) {
  if (ref_check(c) || !psi) return -1;
  if (c->nproj == 0) return 0;
  if (!proj || !Dm) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  const double eps = 0.5 * c->dt;
  double complex* C = malloc((size_t)np * no * sizeof(double complex));
  double complex* Y = calloc((size_t)np * no, sizeof(double complex));
  double* n0 = calloc((size_t)no, sizeof(double));
  double* n1 = calloc((size_t)no, sizeof(double));
  if (!C || !Y || !n0 || !n1) { free(C); free(Y); free(n0); free(n1); return -2; }
  for (size_t r = 0; r < ng; ++r)
    for (int s = 0; s < no; ++s) {
      double complex v = psi[r * no + s];
      n0[s] += creal(v) * creal(v) + cimag(v) * cimag(v);
    }
  ref_project(c, psi, proj, C);
  for (int u = 0; u < np; ++u)  /* Y = -i eps D C */
    for (int v = 0; v < np; ++v)
      for (int s = 0; s < no; ++s) Y[(size_t)u * no + s] += -I * eps * Dm[(size_t)u * np + v] * C[(size_t)v * no + s];
  ref_backproject(c, psi, proj, Y);
  for (size_t r = 0; r < ng; ++r)
    for (int s = 0; s < no; ++s) {
      double complex v = psi[r * no + s];
      n1[s] += creal(v) * creal(v) + cimag(v) * cimag(v);
    }
  for (int s = 0; s < no; ++s) {
    double f = sqrt(n0[s] / n1[s]);
    for (size_t r = 0; r < ng; ++r) psi[r * no + s] *= f;
  }
  free(C); free(Y); free(n0); free(n1);
  return 0;
}

/* exp(M) of an n x n complex matrix by the textbook Taylor series with scaling and squaring:
 * exp(M) = (exp(M / 2^k))^(2^k), ||M||_1 / 2^k <= 1/2, 30 Taylor terms (truncation < 1e-30). */
static int ref_expm(int n, const double complex* M, double complex* E) {
  double nrm = 0.0;
  for (int j = 0; j < n; ++j) {
    double col = 0.0;
    for (int i = 0; i < n; ++i) col += cabs(M[(size_t)i * n + j]);
    if (col > nrm) nrm = col;
  }
  int k = 0;
  while (nrm > 0.5) { nrm *= 0.5; ++k; }
  const double sc = ldexp(1.0, -k);
  double complex* T = malloc((size_t)n * n * sizeof(double complex));
  double complex* W = malloc((size_t)n * n * sizeof(double complex));
  if (!T || !W) { free(T); free(W); return -2; }
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < n; ++j) {
      E[(size_t)i * n + j] = (i == j) ? 1.0 : 0.0;
      T[(size_t)i * n + j] = (i == j) ? 1.0 : 0.0;
    }
  for (int t = 1; t <= 30; ++t) {  /* T <- T (M sc) / t ; E += T */
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) {
        double complex a = 0.0;
        for (int l = 0; l < n; ++l) a += T[(size_t)i * n + l] * M[(size_t)l * n + j] * sc;
        W[(size_t)i * n + j] = a / (double)t;
      }
    for (size_t q = 0; q < (size_t)n * n; ++q) { T[q] = W[q]; E[q] += W[q]; }
  }
  for (int it = 0; it < k; ++it) {  /* E <- E E */
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) {
        double complex a = 0.0;
        for (int l = 0; l < n; ++l) a += E[(size_t)i * n + l] * E[(size_t)l * n + j];
        W[(size_t)i * n + j] = a;
      }
    for (size_t q = 0; q < (size_t)n * n; ++q) E[q] = W[q];
  }
  free(T); free(W);
  return 0;
}

/* The exactly unitary factor with a dense Hermitian D, for dV-orthonormal projector columns: v_nl =
 * B D B^H dV acts on span(B) as the matrix D in the basis B, so exp(-i eps v_nl) = 1 + B (exp(-i eps D) - 1)
 * B^H dV:  C = dV B^H Psi,  Psi' = Psi + B ((exp(-i eps D) - I) C). No renormalisation. One domain. */
int lfd_ref_nl_half_exact_dense(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                                const double complex* Dm) {
  if (ref_check(c) || !psi) return -1;
  if (c->nproj == 0) return 0;
  if (!proj || !Dm) return -1;
  const int no = c->norb, np = c->nproj;
  const double eps = 0.5 * c->dt;
  double complex* M = malloc((size_t)np * np * sizeof(double complex));
  double complex* E = malloc((size_t)np * np * sizeof(double complex));
  double complex* C = malloc((size_t)np * no * sizeof(double complex));
  double complex* Y = calloc((size_t)np * no, sizeof(double complex));
  if (!M || !E || !C || !Y) { free(M); free(E); free(C); free(Y); return -2; }
  for (size_t q = 0; q < (size_t)np * np; ++q) M[q] = -I * eps * Dm[q];
  if (ref_expm(np, M, E)) { free(M); free(E); free(C); free(Y); return -2; }
  for (int u = 0; u < np; ++u) E[(size_t)u * np + u] -= 1.0;
  ref_project(c, psi, proj, C);
  for (int u = 0; u < np; ++u)
    for (int v = 0; v < np; ++v)
      for (int s = 0; s < no; ++s) Y[(size_t)u * no + s] += E[(size_t)u * np + v] * C[(size_t)v * no + s];
  ref_backproject(c, psi, proj, Y);
  free(M); free(E); free(C); free(Y);
  return 0;
}

/* nsteps Eq.-6 steps N o Local o N with the dense-D factor (exact != 0: the exactly unitary one) for every
 * domain; Dm [ndom][nproj][nproj]. */
int lfd_ref_step_dense(const lfd_ref_config* c, double complex* psi, const double complex* proj,
                       const double complex* Dm, const double* vloc, const double* A, int nsteps, int exact) {
  if (ref_check(c) || !psi || !vloc || !A || nsteps < 0) return -1;
  if (c->nproj > 0 && (!proj || !Dm)) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  lfd_ref_config one = *c;
  one.ndom = 1;
  for (int it = 0; it < nsteps; ++it)
    for (int dm = 0; dm < c->ndom; ++dm) {
      double complex* p = psi + (size_t)dm * ng * c->norb;
      const double complex* b = proj ? proj + (size_t)dm * ng * c->nproj : NULL;
      const double complex* d = Dm ? Dm + (size_t)dm * c->nproj * c->nproj : NULL;
      int e = exact ? lfd_ref_nl_half_exact_dense(&one, p, b, d) : lfd_ref_nl_half_dense(&one, p, b, d);
      e |= lfd_ref_local(&one, p, vloc + (size_t)dm * ng, A + 3 * dm);
      e |= exact ? lfd_ref_nl_half_exact_dense(&one, p, b, d) : lfd_ref_nl_half_dense(&one, p, b, d);
      if (e) return -1;
    }
  return 0;
}

/* Nonlocal energy with a dense D, per domain: E_nl[dm] = sum_s f_s sum_{u,v} conj(C_us) D_uv C_vs
 * (<psi_s| v_nl |psi_s>, Eq. 5 / P:63). */
int lfd_ref_energy_nl_dense(const lfd_ref_config* c, const double complex* psi, const double* occ,
                            const double complex* proj, const double complex* Dm, double* Enl) {
  if (ref_check(c) || !psi || !occ || !Enl) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  lfd_ref_config one = *c;
  one.ndom = 1;
  double complex* C = malloc(((size_t)np * no + 1) * sizeof(double complex));
  if (!C) return -2;
  for (int dm = 0; dm < c->ndom; ++dm) {
    double e = 0.0;
    if (np > 0) {
      ref_project(&one, psi + (size_t)dm * ng * no, proj + (size_t)dm * ng * np, C);
      const double complex* d = Dm + (size_t)dm * np * np;
      for (int s = 0; s < no; ++s) {
        double complex q = 0.0;
        for (int u = 0; u < np; ++u)
          for (int v = 0; v < np; ++v) q += conj(C[(size_t)u * no + s]) * d[(size_t)u * np + v] * C[(size_t)v * no + s];
        e += occ[(size_t)dm * no + s] * creal(q);
      }
    }
    Enl[dm] = e;
  }
  free(C);
  return 0;
}

/* Public: density and current of every domain (kernel 4 semantics), readings R12-R14:
 *   rho_r   = sum_s f_s |Psi_rs|^2
 *   j_d,r   = (1/h_d) sum_s f_s Im( e^{i theta_d} conj(Psi_rs) Psi_{r+e_d,s} ),  theta_d = A_d h_d / c
 *             (gauge-consistent link current of the R2 discretisation; r+e_d periodic, or
 *              j_d = 0 on the last plane for zero BC; stored at the link's left node)
 *   J_d     = (1/Ngrid) sum_r j_d,r
 * rho [ndom][ng]; j [ndom][3][ng] (may be NULL); Jmac [ndom][3] (may be NULL). */
int lfd_ref_density_current(const lfd_ref_config* c, const double complex* psi, const double* occ,
                            const double* A, double* rho, double* j, double* Jmac) {
  if (ref_check(c) || !psi || !occ || !A || !rho) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int n[3] = {c->nx, c->ny, c->nz};
  const double h[3] = {c->hx, c->hy, c->hz};
  const int no = c->norb;
  for (int dm = 0; dm < c->ndom; ++dm) {
    const double complex* p = psi + (size_t)dm * ng * no;
    const double* f = occ + (size_t)dm * no;
    for (int ix = 0; ix < c->nx; ++ix)
      for (int iy = 0; iy < c->ny; ++iy)
        for (int iz = 0; iz < c->nz; ++iz) {
          size_t r = gidx(c, ix, iy, iz);
          double acc = 0.0;
          for (int s = 0; s < no; ++s) {
            double complex v = p[r * no + s];
            acc += f[s] * (creal(v) * creal(v) + cimag(v) * cimag(v));
          }
          rho[(size_t)dm * ng + r] = acc;
        }
    double Jsum[3] = {0.0, 0.0, 0.0};
    for (int d = 0; d < 3; ++d) {
      double complex eth = cexp(I * (A[3 * dm + d] / REF_C_LIGHT) * h[d]);
      for (int ix = 0; ix < c->nx; ++ix)
        for (int iy = 0; iy < c->ny; ++iy)
          for (int iz = 0; iz < c->nz; ++iz) {
            int q[3] = {ix, iy, iz};
            size_t r = gidx(c, ix, iy, iz);
            double val = 0.0;
            if (!(c->bc == REF_BC_ZERO && q[d] == n[d] - 1)) {
              q[d] = (q[d] + 1) % n[d];
              size_t r2 = gidx(c, q[0], q[1], q[2]);
              for (int s = 0; s < no; ++s)
                val += f[s] * cimag(eth * conj(p[r * no + s]) * p[r2 * no + s]);
              val /= h[d];
            }
            if (j) j[((size_t)dm * 3 + d) * ng + r] = val;
            Jsum[d] += val;
          }
    }
    if (Jmac)
      for (int d = 0; d < 3; ++d) Jmac[3 * dm + d] = Jsum[d] / (double)ng;
  }
  return 0;
}

/* Public (used by the current pin, R13): kinetic energy of one domain in the same
 * discretisation, E_kin = sum_s f_s dV <psi_s| sum_links L + singletons |psi_s>, where each link
 * (i, i') contributes t_d |psi_i - e^{i theta_d} psi_i'|^2 (the quadratic form of the link
 * Hamiltonian L of ref_pair_coeffs) and each zero-BC singleton contributes t_d |psi_i|^2. */
double lfd_ref_kinetic_energy(const lfd_ref_config* c, const double complex* psi, const double* occ,
                              const double* A) {
  if (ref_check(c) || !psi || !occ || !A) return NAN;
  const int n[3] = {c->nx, c->ny, c->nz};
  const double h[3] = {c->hx, c->hy, c->hz};
  const double dV = c->hx * c->hy * c->hz;
  const int no = c->norb;
  double e = 0.0;
  for (int d = 0; d < 3; ++d) {
    double t = 1.0 / (2.0 * h[d] * h[d]);
    double complex eth = cexp(I * (A[d] / REF_C_LIGHT) * h[d]);
    for (int ix = 0; ix < c->nx; ++ix)
      for (int iy = 0; iy < c->ny; ++iy)
        for (int iz = 0; iz < c->nz; ++iz) {
          int q[3] = {ix, iy, iz};
          size_t r = gidx(c, ix, iy, iz);
          for (int s = 0; s < no; ++s) {
            double complex a = psi[r * no + s];
            if (c->bc == REF_BC_ZERO && q[d] == n[d] - 1) {
              /* no link to the right; the point keeps its diagonal through the on-site half */
              e += occ[s] * dV * t * (creal(a) * creal(a) + cimag(a) * cimag(a));
              continue;
            }
            int q2[3] = {q[0], q[1], q[2]};
            q2[d] = (q2[d] + 1) % n[d];
            double complex b = psi[gidx(c, q2[0], q2[1], q2[2]) * no + s];
            double complex dlt = a - eth * b;
            e += occ[s] * dV * t * (creal(dlt) * creal(dlt) + cimag(dlt) * cimag(dlt));
            if (c->bc == REF_BC_ZERO && q[d] == 0)
              e += occ[s] * dV * t * (creal(a) * creal(a) + cimag(a) * cimag(a));
          }
        }
  }
  return e;
}

/* Public (calc_energy, P:212 / Fig. 5): energy of every domain,
 * E = sum_s f_s <psi_s| h |psi_s> with h = T(A) + v_loc + v_nl of Eq. 5:
 *   E[4*dm+0] = kinetic (lfd_ref_kinetic_energy, the FD Peierls form of the propagator),
 *   E[4*dm+1] = local   = dV sum_r v_r sum_s f_s |psi_rs|^2          (v_loc applies point by point)
 *   E[4*dm+2] = nonlocal = sum_s f_s sum_u D_u |C_us|^2,  C_us = dV sum_r conj(B_ru) psi_rs
 *               (<psi| Delta_sci sum_u |B_u><B_u| |psi>, Eq. 7 P:68 with D_u = Delta_sci; R9)
 *   E[4*dm+3] = total. proj/dnl may be NULL iff nproj == 0. */
int lfd_ref_energy(const lfd_ref_config* c, const double complex* psi, const double* occ, const double* vloc,
                   const double* A, const double complex* proj, const double* dnl, double* E) {
  if (ref_check(c) || !psi || !occ || !vloc || !A || !E) return -1;
  if (c->nproj > 0 && (!proj || !dnl)) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb, np = c->nproj;
  const double dV = c->hx * c->hy * c->hz;
  lfd_ref_config one = *c;
  one.ndom = 1;
  for (int dm = 0; dm < c->ndom; ++dm) {
    const double complex* p = psi + (size_t)dm * ng * no;
    const double* f = occ + (size_t)dm * no;
    const double* v = vloc + (size_t)dm * ng;
    double ekin = lfd_ref_kinetic_energy(&one, p, f, A + 3 * dm);
    double eloc = 0.0;
    for (size_t r = 0; r < ng; ++r) {
      double rho = 0.0;
      for (int s = 0; s < no; ++s) rho += f[s] * (creal(p[r * no + s]) * creal(p[r * no + s]) +
                                                  cimag(p[r * no + s]) * cimag(p[r * no + s]));
      eloc += v[r] * rho;
    }
    eloc *= dV;
    double enl = 0.0;
    if (np > 0) {
      const double complex* b = proj + (size_t)dm * ng * np;
      const double* d = dnl + (size_t)dm * np;
      for (int u = 0; u < np; ++u)
        for (int s = 0; s < no; ++s) {
          double complex cus = 0.0;
          for (size_t r = 0; r < ng; ++r) cus += conj(b[r * np + u]) * p[r * no + s];
          cus *= dV;
          enl += f[s] * d[u] * (creal(cus) * creal(cus) + cimag(cus) * cimag(cus));
        }
    }
    E[4 * dm + 0] = ekin;
    E[4 * dm + 1] = eloc;
    E[4 * dm + 2] = enl;
    E[4 * dm + 3] = ekin + eloc + enl;
  }
  return 0;
}

/* Public (remap_occ, P:58 / P:212): the shadow-dynamics handshake maps the
 * propagated orbitals back to occupation numbers of a reference basis (reading: the KS orbitals at
 * t = 0), out[dm][k] = sum_s f_s |<ref_k | psi_s>|^2 = sum_s f_s |dV sum_r conj(ref_rk) psi_rs|^2.
 * ref [ndom][nx][ny][nz][nref] complex128. */
int lfd_ref_remap_occ(const lfd_ref_config* c, const double complex* psi, const double* occ,
                      const double complex* ref, int nref, double* out) {
  if (ref_check(c) || !psi || !occ || !ref || nref < 1 || !out) return -1;
  const size_t ng = (size_t)c->nx * c->ny * c->nz;
  const int no = c->norb;
  const double dV = c->hx * c->hy * c->hz;
  for (int dm = 0; dm < c->ndom; ++dm) {
    const double complex* p = psi + (size_t)dm * ng * no;
    const double complex* q = ref + (size_t)dm * ng * nref;
    const double* f = occ + (size_t)dm * no;
    for (int k = 0; k < nref; ++k) {
      double acc = 0.0;
      for (int s = 0; s < no; ++s) {
        double complex ov = 0.0;
        for (size_t r = 0; r < ng; ++r) ov += conj(q[r * nref + k]) * p[r * no + s];
        ov *= dV;
        acc += f[s] * (creal(ov) * creal(ov) + cimag(ov) * cimag(ov));
      }
      out[(size_t)dm * nref + k] = acc;
    }
  }
  return 0;
}
