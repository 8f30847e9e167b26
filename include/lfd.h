/*
 * lfd.h -- C ABI of the B200-native Local Field Dynamics (LFD) step of DC-MESH.
 *
 * What the library computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n; the readings
 * R1..R22 are listed in DESIGN.md §3):
 *   One LFD/QD time step of Eq. 6 for every divide-and-conquer domain (Fig. 1):
 *       Psi <- N( Local( N(Psi) ) )
 *   * Local = exp(-i Delta h_loc) of Eq. 5 by the O(N) space-splitting stencil (P:68, P:76-80,
 *     Alg. 1-5): Psi <- Phi . K_z K_y K_x (Phi . Psi), Phi = e^{-i (Delta/2) v_loc},
 *     K_d = E_d(Delta/2) O_d(Delta) E_d(Delta/2) (2x2 pair blocks with Peierls phases for A(t); R2-R8).
 *   * N = the renormalised first-order nonlocal factor (1 - i Delta/2 v_nl)/||...|| of Eq. 6 with the
 *     scissor projector of Eq. 7, BLASified as in Eq. 9: C = dV B^H Psi,
 *     Psi <- (Psi - i (Delta/2) B diag(D) C) diag(n), n_s restoring each orbital's norm (R9-R12).
 *   * Density rho = sum_s f_s |psi_s|^2 and the gauge-consistent link current j, J (R13).
 *
 * Conventions (all entry points):
 *   - Units: atomic units, hbar = m = e = 1, c = 137.035999084 (R1).
 *   - Layout: complex128 = two doubles (re, im) interleaved; orbital index fastest, then z, y, x,
 *     then domain:  psi[dom][x][y][z][orb]  (the paper's SoA psi[i][j][k][n]).
 *     Grid index r = ((x*ny)+y)*nz+z. Orbitals are normalised as dV * sum_r |psi|^2 = 1 (R12).
 *   - Ownership: the caller owns every buffer (device buffers are typically torch tensors) and keeps
 *     the borrowed ones (psi, proj, workspace) alive until lfd_destroy. The library owns only the
 *     context struct. Small HOST arrays are copied (or captured by value) during the call.
 *   - Streams: all device work is enqueued on the context's CUDA stream, in call order. Calls return
 *     before the GPU finishes; lfd_sync() waits and reports asynchronous CUDA errors.
 *   - Errors: every call returns lfd_status. Arguments are validated before anything is enqueued and a
 *     failed call changes no state. No C++ exception crosses the ABI. lfd_last_error() gives text.
 *   - Threading: one context = one host thread + one stream. Many contexts may coexist.
 *   - There is no CPU fallback: without a usable sm_100a device, lfd_init returns LFD_ECUDA.
 */
#ifndef LFD_H_
#define LFD_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LFD_ABI_VERSION 4
#define LFD_MAX_DOMAINS 4096

typedef struct lfd_ctx lfd_ctx; /* opaque */

typedef enum {
  LFD_OK = 0,
  LFD_EINVAL = -1,       /* bad argument or configuration */
  LFD_ENOMEM = -2,       /* workspace too small / host allocation failed */
  LFD_ECUDA = -3,        /* CUDA runtime error (including no sm_100 device) */
  LFD_ESTATE = -4,       /* call not valid in the current state (e.g. use after destroy) */
  LFD_EUNSUPPORTED = -5  /* valid request this build does not implement */
} lfd_status;

typedef enum { LFD_BC_PERIODIC = 0, LFD_BC_ZERO = 1 } lfd_bc; /* reading R8 */

typedef struct {
  int32_t abi_version; /* must equal LFD_ABI_VERSION */
  int32_t ndomains;    /* same-shape DC domains batched in this context, 1..LFD_MAX_DOMAINS */
  int32_t nx, ny, nz;  /* mesh points per domain, each >= 2; even when bc == LFD_BC_PERIODIC */
  double hx, hy, hz;   /* mesh spacing [bohr], > 0 */
  int32_t bc;          /* lfd_bc */
  int32_t norb;        /* propagated KS orbitals per domain, >= 1 */
  int32_t nproj;       /* projector columns per domain, 0..2048 (0 disables the nonlocal factor) */
  int32_t nref_max;    /* max reference-basis columns for lfd_remap_occ, 0..2048 (0: max(norb, nproj)) */
  double dt;           /* Delta_QD [a.u.], finite and nonzero (negative = backward in time) */
  int32_t device;      /* CUDA device ordinal */
  int32_t flags;       /* 0 or LFD_FLAG_NO_CARRY | EXACT_NL | SP | NL_DMMA | NL_I8 | DENSE_D | NO_PDL (below) */
} lfd_config;

/* lfd_config.flags: disable the projection carry (lfd_step takes the C of each nonlocal factor that
 * directly follows another one from C_new = (C + G C') diag(n), an exact identity, instead of
 * recomputing dV B^H Psi by GEMM-1). With the flag every factor runs its GEMM-1; results agree to
 * roundoff. */
#define LFD_FLAG_NO_CARRY 1
/* lfd_config.flags: the EXACTLY UNITARY nonlocal factor instead of Eq. 6's
 * renormalised first-order one: for dV-orthonormal projector columns (dV B^H B = I, checked at lfd_init:
 * LFD_EINVAL otherwise) exp(-i (Delta/2) B diag(D) B^H dV) = 1 + B diag(e^{-i (Delta/2) D} - 1) B^H dV,
 * which keeps every orbital's norm and the orthonormality of Psi exactly (no renormalisation). */
#define LFD_FLAG_EXACT_NL 2
/* lfd_config.flags: the SP variant (the paper's SP column, and its
 * complex<float> listings): psi, proj (and lfd_remap_occ's ref) are complex64 [.. same layouts ..]
 * (two floats, 8-byte aligned). The stencil sweeps run in FP32 (three line passes); the projector GEMMs run on
 * the tcgen05 int8 tensor cores (GEMM-2: 4 balanced base-128 digits per operand; GEMM-1: 3 base-256 digits;
 * products to ~2^-22 .. 2^-27 of the row / column scales, below FP32 rounding of Psi; the default where nproj,
 * norb <= 64 and >= 65,536 points, or LFD_FLAG_NL_I8),
 * else as 3xTF32 on the warp-level mma.sync path (LFD_FLAG_NL_DMMA selects the latter); everything
 * O(nproj x norb) -- the split reduction, the Gram matrix, n_s, the carry, the energies -- runs in FP64. Results
 * agree with the FP64 path to single-precision roundoff (DESIGN.md §4 states the tolerance). */
#define LFD_FLAG_SP 4
/* lfd_config.flags: run the nonlocal GEMMs (C = dV B^H Psi; Psi <- Psi diag(n) + B C'') as
 * strict IEEE complex FP64 on the DMMA pipe (mma.sync m8n8k4) instead of the default for FP64 contexts with
 * nproj <= 64, norb <= 64 and >= 65,536 points per domain: the same products EMULATED on the tcgen05 int8
 * tensor cores -- operands split exactly into int8 digits with power-of-two row / column scales, the digit
 * pairs accumulated exactly in int32 in tensor memory, recombined in FP64 (GEMM-2: 6 balanced base-128 digits,
 * the 21 pairs i + j <= 7; GEMM-1: 5 base-256 digits, Psi's offset-binary, the 19 pairs k + i >= 3).
 * That arithmetic is narrower than an FP64 product: the truncation (digit remainders and dropped pairs) leaves
 * an error of ~2^-40 (GEMM-2) / ~2^-38 (GEMM-1) of (row scale x column scale) per output, against ~2^-53 for
 * IEEE FP64 (measured against the DMMA path in tests/test_gpu_i8.py). The nonlocal update B C'' is O(Delta Delta_sci / 2 ~ 1.4e-3) of Psi, so at the
 * paper's scissor size each factor moves Psi by ~1e-15 relative and the FP64 parity contract (1e-10 after 100
 * steps) holds; bench.py reports the strict-FP64 step (this flag) beside the default. See lfd_nl_path(). */
#define LFD_FLAG_NL_DMMA 8
/* lfd_config.flags: use the int8-digit GEMMs wherever they are supported (nproj, norb <= 64), also on small
 * grids where they are not the default (< 65,536 points per domain: set-up not amortised). */
#define LFD_FLAG_NL_I8 16

/* lfd_config.flags: a DENSE Hermitian nonlocal coupling (Eq. 5 v_nl, in
 * Kleinman-Bylander form v_nl = sum_uv |b_u> D_uv <b_v|; Eq. 7's scissor, is D = Delta_sci I): lfd_init's
 * dnl is then HOST complex128 [ndom][nproj][nproj] (row-major D[u][v], Hermitian to 1e-12 of max |D|, else
 * LFD_EINVAL), copied. The library diagonalises each D once (D = Q diag(w) Q^H, host Jacobi) and propagates
 * with the rotated projectors B Q (computed into the workspace by the FP64 GEMM-2) and diagonal couplings w --
 * the same operator B D B^H, so every path (first-order and exact factors, carry, merged sequences, energy)
 * applies unchanged. lfd_set_occupations etc. are unaffected. nproj <= 512. */
#define LFD_FLAG_DENSE_D 32

/* lfd_config.flags: launch every kernel in plain stream order, without programmatic dependent launch (PDL lets
 * a kernel's set-up overlap its predecessor's tail; the results are the same either way). For debugging and
 * measurement. */
#define LFD_FLAG_NO_PDL 64

/* Kernel classes, for lfd_profile_read(). */
typedef enum {
  LFD_K_COEF = 0,      /* a1: stencil coefficients from A(t) */
  LFD_K_PHASE = 1,     /* a2: Phi = exp(-i Delta/2 v_loc) */
  LFD_K_KIN_X = 2,     /* a6: Phi . K_x (pre-phase fused) */
  LFD_K_KIN_Y = 3,     /* a6: K_y (unfused path) */
  LFD_K_KIN_Z = 4,     /* a6: K_z . Phi (post-phase fused; unfused path) */
  LFD_K_NL_PROJ = 5,   /* a3: GEMM-1 split-K partials of C = dV B^H Psi + column norms */
  LFD_K_NL_REDUCE = 6, /* a4: fixed-order split-K reduction, C' = -i(Delta/2) D C */
  LFD_K_NL_NORM = 7,   /* a4: n_s from the Gram closed form */
  LFD_K_NL_BACK = 8,   /* a5: GEMM-2 Psi <- (Psi + B C') diag(n), in place */
  LFD_K_DENSITY = 9,   /* a7: rho, j, per-line partial J */
  LFD_K_JREDUCE = 10,  /* a7: J = mean of j (fixed order) */
  LFD_K_ENERGY = 11,   /* NEXT f-1: energy / occupation reductions (calc_energy, remap_occ) */
  LFD_K_NL_CARRY = 12, /* a3/a4: projection carry C_new = (C + G C') diag(n) (replaces GEMM-1) */
  LFD_K_KIN_YZ = 13,   /* a6: K_y K_z . Phi fused in one pass (post-phase fused) */
  LFD_K_SC = 14,       /* self-consistent step: Maxwell, potential gather, Poisson filter, v_Hxc */
  LFD_K_FFT = 15,      /* self-consistent step: cuFFT D2Z / Z2D of the Hartree solve (library kernels) */
  LFD_K_NL_BACKX = 16, /* a5 + a6: the first factor's GEMM-2 fused with Phi . K_x (int8-digit path, nx <= 80) */
  LFD_K_COUNT = 17
} lfd_kernel_id;

/* Bytes of DEVICE workspace lfd_init needs for this configuration. */
lfd_status lfd_workspace_size(const lfd_config* cfg, size_t* bytes);

/* Create a context.
 *  psi   DEVICE complex128 [ndom][nx][ny][nz][norb]; borrowed; propagated in place by lfd_step. Like the
 *        paper's GPU-resident Psi(t), it belongs to the library while the context is live: the
 *        caller may read it (after lfd_sync or in stream order) but must call lfd_psi_modified() after
 *        writing it, because the context keeps the projection C = dV B^H Psi of the last nonlocal
 *        factor for the next one (see LFD_FLAG_NO_CARRY).
 *  proj  DEVICE complex128 [ndom][nx][ny][nz][nproj]; borrowed, read-only (B = Psi_u(0), the
 *        unoccupied KS orbitals at t = 0, Eq. 7 P:68 / R9); NULL iff nproj == 0. Need not be
 *        orthonormal: the Gram matrix G = dV B^H B is computed here (on the device) and used for n_s.
 *        Must not change while the context lives: G and (default path) B's int8 digits are made here.
 *  dnl   HOST double [ndom][nproj] real couplings D_u (paper: all equal Delta_sci of Eq. 8), or with
 *        LFD_FLAG_DENSE_D complex128 [ndom][nproj][nproj] Hermitian matrices; copied. NULL iff nproj == 0.
 *  occ   HOST double [ndom][norb] occupations f_s (not clamped, R14); copied.
 *  workspace DEVICE, >= lfd_workspace_size bytes, 256-byte aligned; borrowed.
 *  stream cudaStream_t (NULL = legacy default stream); all work is ordered on it.
 * Initial state: v_loc = 0 (Phi = 1) and A = 0 until the setters are called.
 * Errors: LFD_EINVAL (bad config / pointer kind / alignment), LFD_ENOMEM (workspace too small),
 *         LFD_ECUDA (no sm_100 device or a CUDA failure). *out is set only on LFD_OK. */
lfd_status lfd_init(const lfd_config* cfg, void* psi, const void* proj, const double* dnl,
                    const double* occ, void* workspace, size_t ws_bytes, void* stream, lfd_ctx** out);

/* v_loc(r) at the step midpoint (Eq. 4; Eq. 5 v_loc), DEVICE double [ndom][nx][ny][nz]
 * [Hartree]; read in stream order (Phi is computed on the device; the buffer may be reused after the
 * call's work has run). */
lfd_status lfd_set_potential(lfd_ctx* ctx, const double* vloc);

/* As lfd_set_potential, but vloc is a HOST buffer (pinned recommended): an async H2D copy into one of two
 * workspace staging slots is enqueued on a side stream (so it overlaps the kernels already queued, e.g. the
 * previous step), and the potential-phase kernel waits for it in stream order. The host buffer must stay
 * unchanged until that copy has run (lfd_sync; callers that refill it every step double-buffer it). */
lfd_status lfd_set_potential_host(lfd_ctx* ctx, const double* vloc_host);

/* A_X(alpha)(t) at the step midpoint (Eq. 2 / Eq. 5; Eq. 4 midpoint), HOST double [ndom][3] a.u.;
 * captured by value (the coefficient table is rebuilt on the device in stream order). */
lfd_status lfd_set_vector_potential(lfd_ctx* ctx, const double* A);

/* Enqueue nsteps LFD steps (Eq. 6) with the current v_loc and A. nsteps == 0 is a no-op; < 0 EINVAL. */
lfd_status lfd_step(lfd_ctx* ctx, int32_t nsteps);

/* Enqueue the FIRST nonlocal factor of the next Eq.-6 step now (Psi <- N(Psi)). It depends only on Psi,
 * B, D and Delta -- not on v_loc or A -- so a caller can run it before the inputs of the step are known, e.g.
 * while the previous step's density is being all-gathered across ranks; the next lfd_step /
 * lfd_step_sequence then starts with the local factor. The result is bitwise that of the plain call order.
 * Until that step, Psi holds the intermediate N(Psi): lfd_density_current*, lfd_energy, lfd_remap_occ,
 * lfd_step_graph, lfd_sc_*, lfd_psi_modified and a second prologue return LFD_ESTATE. */
lfd_status lfd_step_prologue(lfd_ctx* ctx);

/* Enqueue nsteps LFD steps with one vector potential per step, A_seq HOST double [nsteps][ndom][3]
 * (captured by value; step n uses A_seq[n], Eq. 4 midpoints), and the current v_loc. The result equals
 * nsteps x (lfd_set_vector_potential(A_seq[n]); lfd_step(1)) up to roundoff: the second nonlocal
 * factor of step n and the first of step n+1 (Eq. 6; both depend only on Psi, B, D, Delta) are applied
 * as one combined factor N o N = L^2 renormalised, L^2 = I + B (2cD + c^2 D G D) B^H dV, c = -i Delta/2,
 * so a sequence costs nsteps + 1 projector GEMM pairs instead of 2 nsteps. Psi is only materialised
 * at the end. Afterwards the context's A is A_seq[nsteps-1]. */
lfd_status lfd_step_sequence(lfd_ctx* ctx, int32_t nsteps, const double* A_seq);

/* nsteps x (lfd_set_vector_potential(A_seq[n]); lfd_step(1); [density]) executed as CUDA graphs: chunks of up
 * to 32 steps are captured once (on a private stream, on first use; keyed by chunk length, the projection-carry
 * state and the outputs) and replayed with the chunk's A values uploaded to the workspace, so the host cost is
 * one graph launch per 32 steps instead of ~12 kernel launches per step (latency-bound shapes such as C1 / C3).
 * Results are bitwise those of the per-step calls (same kernels, same order).
 *  A_seq     HOST double [nsteps][ndom][3] (copied during the call), the step midpoints (Eq. 4)
 *  rho       DEVICE double [ndom][nx][ny][nz] or NULL: the density after each step (the last one remains)
 *  Jmac_seq  DEVICE double [nsteps][ndom][3] or NULL: J of every step (the current response time series)
 * Density and J use each step's own A, as lfd_density_current after that step. With lfd_profile_enable on, the
 * same kernels run eagerly (per-launch events). Afterwards the context's A is A_seq[nsteps-1]. */
lfd_status lfd_step_graph(lfd_ctx* ctx, int32_t nsteps, const double* A_seq, double* rho, double* Jmac_seq);

/* Density and current of the current Psi with the current A (kernel 4; R13):
 *  rho  DEVICE double [ndom][nx][ny][nz]          rho_r = sum_s f_s |psi_rs|^2
 *  j    DEVICE double [ndom][3][nx][ny][nz] or NULL
 *       j_d,r = (1/h_d) sum_s f_s Im(e^{i A_d h_d / c} conj(psi_rs) psi_{r+e_d,s}) (left-node link
 *       current; periodic wrap, or 0 on the last plane for zero BC). Electron-number current.
 *  Jmac DEVICE double [ndom][3] or NULL            J_d = (1/Ngrid) sum_r j_d,r
 */
lfd_status lfd_density_current(lfd_ctx* ctx, double* rho, double* j, double* Jmac);

/* As lfd_density_current, but writes each domain's core into GLOBAL-layout device arrays
 * rho_g [GX][GY][GZ] and j_g [3][GX][GY][GZ] (j_g may be NULL) at the HOST-given offsets
 * dom_offset[ndom][3]; domain cores must lie inside gdims[3] and must not overlap. Untouched global
 * points are left as they are (callers zero them; a SUM all-reduce then assembles the DC
 * recombination of rho, R18). Jmac as above (per domain, may be NULL). */
lfd_status lfd_density_current_global(lfd_ctx* ctx, double* rho_g, double* j_g, double* Jmac,
                                      const int32_t* dom_offset, const int32_t* gdims);

/* As lfd_density_current for rho and Jmac, into HOST buffers (pinned recommended) via async D2H
 * copies; read them after lfd_sync(). Either pointer may be NULL to skip it. */
lfd_status lfd_density_current_host(lfd_ctx* ctx, double* rho_host, double* Jmac_host);

/* Wait on the host until the D2H copies of an lfd_density_current_host call have landed: lag 0 = the latest
 * call, lag 1 = the one before it (its copies ran on a side stream while later work was queued: a caller that
 * double-buffers its host outputs reads step n's while step n+1 runs). LFD_EINVAL for another lag,
 * LFD_ESTATE if there is no such call; asynchronous CUDA errors as lfd_sync. */
lfd_status lfd_wait_host_outputs(lfd_ctx* ctx, int32_t lag);

/* calc_energy (Fig. 5): E[dom][4] = {kinetic, local, nonlocal,
 * total} of the current Psi with the current v_loc and A, DEVICE double, stream-ordered:
 *   kinetic  = sum_s f_s dV sum_d (1/h_d^2) sum_r [ |psi_rs|^2 - Re(e^{i theta_d} conj(psi_rs) psi_{r+e_d,s}) ]
 *              (the FD Peierls operator the propagator splits; the neighbour term is absent on the last
 *              plane for zero BC),
 *   local    = dV sum_r v_loc(r) rho(r),   nonlocal = sum_s f_s sum_u D_u |C_us|^2, C = dV B^H Psi. */
lfd_status lfd_energy(lfd_ctx* ctx, double* E);

/* remap_occ: occupations of a reference basis (e.g. the KS orbitals
 * at t = 0), occ_out[dom][k] = sum_s f_s |dV sum_r conj(ref_rk) psi_rs|^2.
 *  ref     DEVICE complex128 [ndom][nx][ny][nz][nref], 1 <= nref <= nref_max (config); read-only.
 *  occ_out DEVICE double [ndom][nref]. Stream-ordered. */
lfd_status lfd_remap_occ(lfd_ctx* ctx, const void* ref, int32_t nref, double* occ_out);

/* ---- Self-consistent LFD step (readings R23-R28 in DESIGN.md §3) -----------------
 * Eq. 5 puts the Hartree and local xc potentials of the propagated density into v_loc, A_X(alpha)
 * obeys Maxwell's equation, and each QD step is "self-consistent, time-reversible". With the
 * SC state initialised, one lfd_sc_step does, for every step n (all on the context stream):
 *   A: velocity-Verlet half kick and drift of the induced field with Jbar(t_n) (R25/R26),
 *      A_mid = A_ext(t_n + Delta/2) + (A_ind(t_n) + A_ind(t_n+1)) / 2, A_end = A_ext(t_n+1) + A_ind(t_n+1);
 *   v: v_loc = v_ion + 3/2 v_Hxc(t_n) - 1/2 v_Hxc(t_n-1) (predictor, R27);
 *   S = N(Psi(t_n)) (the first Eq.-6 nonlocal factor does not depend on v or A: applied once per step);
 *   for k = 0..n_corr: Psi <- N(Local(S)) with (v_loc, A_mid); rho, Jbar of Psi with A_end on the
 *      GLOBAL grid (domain cores, R18; SUM all-reduce over ranks when nranks > 1); v_Hxc = v_H + v_x (R23,
 *      R24; Hartree by cuFFT on the global grid); if k < n_corr: v_loc = v_ion + (v_Hxc(t_n) + v_Hxc)/2;
 *   A: second half kick with Jbar(t_n+1).
 * Afterwards the context's A (lfd_density_current) is A_end of the last step. */
#define LFD_SC_HARTREE 1 /* v_H[rho] in v_loc (R23) */
#define LFD_SC_XC 2      /* LDA exchange v_x[rho] in v_loc (R24) */
#define LFD_SC_MAXWELL 4 /* induced A_ind from the macroscopic current (R25) */

typedef struct {
  int32_t flags;            /* LFD_SC_* (0 = v_ion and A_ext only: the plain step with midpoint inputs) */
  int32_t n_corr;           /* corrector sweeps per step, 0..16 (each re-propagates Psi(t_n) once) */
  int32_t gdims[3];         /* global grid the domain cores of ALL ranks tile (periodic cell of v_H) */
  int32_t nranks, rank;     /* processes sharing the global grid (1, 0 for one process) */
  const int32_t* dom_offset; /* HOST [ndom][3] global offsets of this context's domains (copied) */
} lfd_sc_config;

/* Bytes of DEVICE workspace lfd_sc_init needs (includes a buffer of Psi's size for N(Psi(t_n)) and the cuFFT
 * work area; the library allocates nothing). */
lfd_status lfd_sc_workspace_size(const lfd_ctx* ctx, const lfd_sc_config* sc, size_t* bytes);

/* Initialise the SC state at t_0 from the current Psi: rho(t_0), Jbar(t_0) with A(t_0) = Aext0 + A_ind0,
 * v_Hxc(t_0) (= v_Hxc(t_-1)).
 *  vion    DEVICE double [ndom][nx][ny][nz] local pseudopotential (borrowed, read every step), or NULL = 0
 *  ws      DEVICE >= lfd_sc_workspace_size bytes, 256-byte aligned (borrowed until lfd_destroy)
 *  Aext0   HOST double[3]; A_ind0, Adot0 HOST double[3] or NULL (= 0)
 * With nranks == 1 the domains must tile gdims exactly; with nranks > 1 lfd_sc_comm_init must come first
 * (each rank's domains must lie inside gdims without overlap; the ranks together must tile it).
 * Errors: LFD_EINVAL (config), LFD_ENOMEM (ws too small), LFD_ESTATE (nranks > 1 without a communicator),
 * LFD_ECUDA / LFD_EUNSUPPORTED (cuFFT / NCCL failures). Calling it again re-initialises. */
lfd_status lfd_sc_init(lfd_ctx* ctx, const lfd_sc_config* sc, const double* vion, void* ws, size_t ws_bytes,
                       const double* Aext0, const double* A_ind0, const double* Adot0);

/* Enqueue nsteps self-consistent steps. Aext HOST double [2*nsteps+1][3]: A_ext at t_n, t_n + Delta/2,
 * t_n+1, ... (R28), one vector for all domains; captured by value. */
lfd_status lfd_sc_step(lfd_ctx* ctx, int32_t nsteps, const double* Aext);

/* Copy the SC state out (stream-ordered, DEVICE pointers, each may be NULL):
 *  state DEVICE double[9] = {A_ind[3], dA_ind/dt[3], Jbar[3]} at the current time,
 *  rho_g DEVICE double [GX][GY][GZ] global density, vhxc DEVICE double [GX][GY][GZ] v_Hxc(t_n). */
lfd_status lfd_sc_read(lfd_ctx* ctx, double* state, double* rho_g, double* vhxc);

/* Multi-process SC: lfd_comm_unique_id fills 128 bytes on ONE rank (broadcast them to the others, e.g.
 * with torch.distributed); every rank then calls lfd_sc_comm_init with the same bytes. The library loads
 * NCCL (libnccl.so.2) at this call and all-reduces the [rho_g | Jbar] buffer over it on the context stream.
 * LFD_EUNSUPPORTED if NCCL cannot be loaded. */
lfd_status lfd_comm_unique_id(void* id128);
lfd_status lfd_sc_comm_init(lfd_ctx* ctx, int32_t nranks, int32_t rank, const void* id128);

/* Tell the context that the caller wrote psi (drops the kept projection; the next nonlocal factor
 * recomputes C = dV B^H Psi by GEMM-1). */
lfd_status lfd_psi_modified(lfd_ctx* ctx);

/* Replace the occupations f (the QXMD<->LFD shadow-dynamics handshake). HOST [ndom][norb]. */
lfd_status lfd_set_occupations(lfd_ctx* ctx, const double* occ);

/* Change the stream used by later calls (work already enqueued stays on the old stream). */
lfd_status lfd_set_stream(lfd_ctx* ctx, void* stream);

/* Wait for all enqueued work; LFD_ECUDA if any asynchronous CUDA error occurred. */
lfd_status lfd_sync(lfd_ctx* ctx);

/* Number of kernels this context has launched so far (all classes). */
lfd_status lfd_launch_count(const lfd_ctx* ctx, uint64_t* count);

/* Which kernel runs the nonlocal GEMM-2 of this context: *path = 0 complex FP64 DMMA (mma.sync),
 * 1 int8-digit tcgen05 tensor cores, FP64 emulated (see LFD_FLAG_NL_DMMA), 2 SP 3xTF32 (LFD_FLAG_SP),
 * 3 SP on the int8-digit tcgen05 tensor cores (4 digits),
 * -1 no nonlocal factor (nproj == 0). */
lfd_status lfd_nl_path(const lfd_ctx* ctx, int32_t* path);

/* Per-kernel-class device timing with CUDA events on the context stream.
 * lfd_profile_enable(ctx, 1) starts recording an event pair around every launch;
 * lfd_profile_read() synchronises, returns accumulated milliseconds and launch counts per class
 * (arrays of LFD_K_COUNT), and resets the accumulators. enable 0 stops recording. */
lfd_status lfd_profile_enable(lfd_ctx* ctx, int32_t enable);
lfd_status lfd_profile_read(lfd_ctx* ctx, double* ms, int64_t* launches);

/* Message of the last error on this context (ctx == NULL: of the last failed lfd_init /
 * lfd_workspace_size on this thread). Never NULL. */
const char* lfd_last_error(const lfd_ctx* ctx);

/* Free the context struct (never caller memory). Waits for the context's work first. NULL is OK. */
lfd_status lfd_destroy(lfd_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* LFD_H_ */
