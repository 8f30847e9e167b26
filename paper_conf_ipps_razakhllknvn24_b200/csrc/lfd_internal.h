// lfd_internal.h -- shared (product-only) declarations of the sm_100a kernels and their launchers.
// Not part of the public ABI (include/lfd.h). Nothing here is shared with oracle/.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace lfd {

constexpr double kCLight = 137.035999084;  // R1: speed of light in atomic units

// ---- programmatic dependent launch (PDL) -----------------------------------------------------------------
// Every kernel starts with pdl_wait() (griddepcontrol.wait: returns once the previous kernel in the stream has
// completed and its writes are visible; a no-op when launched without the PDL attribute) and pdl_trigger()
// (griddepcontrol.launch_dependents: once every CTA of this grid has started, the next kernel may launch).
// So each launch, block scheduling and prologue overlaps the previous kernel's last wave, with the same
// ordering guarantees as plain stream order. LFD_PDL=0 in the environment disables the attribute.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
bool pdl_enabled();
void pdl_suspend(bool s);  // graph capture: plain stream edges (measured faster inside graphs than PDL edges)
bool pdl_suspended();
template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// Per-domain stencil/current coefficients, rebuilt on the device from A (step a1 of SURVEY §8(a)).
// For axis d and tau in {Delta/2 (p=0), Delta (p=1)} (p in {Delta_QD/2, Delta_QD}):
//   alpha = e^{-i tau t_d} cos(tau t_d), up = sigma e^{+i theta_d}, dn = sigma e^{-i theta_d},
//   onsite = e^{-i tau t_d},  sigma = i e^{-i tau t_d} sin(tau t_d),  t_d = 1/(2 h_d^2),
//   theta_d = (A_d / c) h_d.   eth[d] = e^{i theta_d} (link current phase, R13).
struct DomCoef {
  double2 alpha[3][2];
  double2 up[3][2];
  double2 dn[3][2];
  double2 onsite[3][2];
  double2 eth[3];
  double inv_h[3];
  double pad_;
  // scaled pair form (kin.cu): w_up = i tan(tau t_d) e^{+i theta_d}, w_dn = i tan(tau t_d) e^{-i theta_d},
  // rc = 1 / cos(tau t_d) (zero-BC singletons)
  double2 wu[3][2];
  double2 wd[3][2];
  double rc[3][2];
};

struct Geometry {
  int ndom, nx, ny, nz, norb, nproj, bc;
  int sp;  // 1: SP variant (complex64 Psi / B, FP32 sweeps and 3xTF32 tensor-core GEMMs), else FP64
  int i8;  // 1: GEMM-2 on the int8-digit tcgen05 path (nl_i8.cu), else DMMA / SP
  double hx, hy, hz, dt, dV;
  long long ng;  // points per domain
};

// TMA tensor map of a float64 tensor (dims innermost first, in elements; strides of dims 1.. in bytes;
// box in elements), no swizzle, zero fill out of bounds (tmap.cu).
cudaError_t encode_tmap_f64(CUtensorMap* out, int rank, const void* base, const uint64_t* dims,
                            const uint64_t* strides_bytes, const uint32_t* box);

// Any tensor map: dtype a CUtensorMapDataType, swizzle a CUtensorMapSwizzle (tmap.cu).
cudaError_t encode_tmap(CUtensorMap* out, int dtype, int rank, const void* base, const uint64_t* dims,
                        const uint64_t* strides_bytes, const uint32_t* box, int swizzle);

// ---- launchers (each returns the cudaError_t of the launch) -------------------------------------
constexpr int kCoefMaxPerLaunch = 512;
struct CoefParams {
  double A[kCoefMaxPerLaunch][3];
};
cudaError_t launch_coef(const Geometry& g, const CoefParams& p, int dom0, int count, DomCoef* coef,
                        cudaStream_t st);
cudaError_t launch_coef_dev(const Geometry& g, const double* A, DomCoef* coef, cudaStream_t st);
// Phi = e^{-i (Delta/2) v} (times sqrt(g) when the scaled pair form is used, kin.cu).
// The coefficient table of a pending lfd_set_vector_potential (up to kCoefFuse domains), computed by the phase
// kernel that runs next (one launch instead of two; count = 0: none pending).
constexpr int kCoefFuse = 8;
struct CoefFuse {
  double A[kCoefFuse][3];
  int count;
  DomCoef* coef;
};
cudaError_t launch_phase(const Geometry& g, const double* v, double2* phi, double* vcopy, bool scaled,
                         cudaStream_t st, const CoefFuse* cf = nullptr);
cudaError_t launch_phase_sp(const Geometry& g, const double* v, float2* phi, double* vcopy, bool scaled,
                            cudaStream_t st, const CoefFuse* cf = nullptr);
// True when the scaled pair form applies (cos(tau t_d) >= 1/2 for every axis and tau).
bool kin_scaled_ok(const Geometry& g);

// One pass of K_axis over every line of every domain, optionally fused with a phase multiply
// (phase_mode 1: Phi . psi before the sweep; 2: after).
cudaError_t launch_kin(const Geometry& g, double2* psi, const DomCoef* coef, const double2* phi,
                       int axis, int phase_mode, bool scaled, cudaStream_t st, const double2* src = nullptr);
// SP variant (complex64 Psi and Phi, FP32 sweeps)
// colE != nullptr (the z pass on the int8-digit path): also records each orbital's largest exponent (k_kin_yz's
// role for FP64) for the next GEMM-1
cudaError_t launch_kin_sp(const Geometry& g, float2* psi, const DomCoef* coef, const float2* phi,
                          int axis, int phase_mode, bool scaled, cudaStream_t st, const float2* src = nullptr,
                          int* colE = nullptr);

// Fused pass Psi <- Phi . K_y K_z Psi (one read + write of Psi; nz <= 80).
bool kin_yz_supported(const Geometry& g);
cudaError_t kin_yz_tensor_map(const Geometry& g, void* psi, CUtensorMap* out);
// colE != nullptr: atomicMax of the biased FP64 exponent of every output Re / Im per orbital into
// colE[dom][norb] (the per-orbital scale of the int8-digit GEMM-1, nl_i8.cu)
cudaError_t launch_kin_yz(const Geometry& g, const CUtensorMap* tmap, double2* psi, const DomCoef* coef,
                          const double2* phi, bool scaled, cudaStream_t st, int* colE = nullptr);
cudaError_t launch_kin_yz_sp(const Geometry& g, const CUtensorMap* tmap, float2* psi, const DomCoef* coef,
                             const float2* phi, bool scaled, cudaStream_t st, int* colE);
cudaError_t kin_yz_set_attributes();

// GEMM-1 split-K: part[dom][split][mrows][ncols] (complex) = sum over the split's grid rows of
// conj(A[r][m]) X[r][n]; if norms != nullptr also norms[dom][split][n] = sum |X[r][n]|^2.
// A: [dom][ng][mrows], X: [dom][ng][ncols] complex.
struct Gemm1Args {
  const double2* A;
  const double2* X;
  double2* part;
  double* norms;
  int ndom, mrows, ncols, nsplit;
  long long ng, rows_per_split;
  long long a_dom_stride, x_dom_stride;  // in complex elements
};
cudaError_t launch_gemm1(const Gemm1Args& a, cudaStream_t st);
int gemm1_smem_bytes();

// Fixed-order split reduction: out[dom][m][n] = scale * D[m] * sum_split part (D == nullptr -> 1);
// if cprime != nullptr also cprime = -i eps * out.  Column norms: s[dom][n] = scale * sum_split norms.
struct ReduceArgs {
  const double2* part;
  const double* normp;
  const double* D;  // [dom][mrows] or nullptr
  double2* out;     // [dom][mrows][ncols]
  double2* cprime;  // [dom][mrows][ncols] or nullptr
  double* s;        // [dom][ncols] or nullptr
  int ndom, mrows, ncols, nsplit;
  double scale, eps;
  const double2* W = nullptr;  // [dom][mrows]: cprime = W out instead of -i eps out (exact factor)
};
cudaError_t launch_reduce(const ReduceArgs& a, cudaStream_t st);

// n_s = sqrt( s_s / (s_s + eps^2 * (DC)_s^H G (DC)_s) )   (Gram closed form of the Eq. 6 norm, R11),
// then C'_s <- C'_s n_s in place: the GEMM-2 coefficient is always C'' = C' diag(n), so its epilogue is
// Psi n + B C'' (and the projection carry uses DC_new = n DC + D G C'').
cudaError_t launch_nlnorm(int ndom, int nproj, int norb, double eps, const double2* G,
                          const double2* DC, const double* s, double* nfac, double2* Cp, cudaStream_t st);

// Combined factor of two consecutive nonlocal halves (lfd_step_sequence): X = (2c D + c^2 D G D) C,
// nfac from the Gram closed form of ||Psi + B X||; X diag(n) is written (the GEMM-2 coefficient).
cudaError_t launch_nlmerge(int ndom, int nproj, int norb, double eps, const double2* G, const double* D,
                           const double2* DC, const double* s, double2* X, double* nfac, cudaStream_t st);

// Projection carry after a GEMM-2 Psi <- Psi diag(n) + B X'' (X'' = X diag(n)): DC <- n DC + D (G X'')
// and X <- -i eps DC (the C' of the next nonlocal factor), in place; column norms s are unchanged.
// with_norm: also the next factor's n_s (as launch_nlnorm) in the same kernel (nfac is overwritten).
// W != nullptr (exactly unitary factor; D == 1 and n == 1 passed): X <- W C_new, no norm.
cudaError_t launch_nlcarry(int ndom, int nproj, int norb, double eps, const double2* G, const double* D,
                           double2* DC, double2* X, const double* s, double* nfac, bool with_norm,
                           const double2* W, cudaStream_t st);

// GEMM-2 in place: psi[dom][r][n] <- nfac[dom][n] * psi[dom][r][n] + sum_m B[dom][r][m] Cp[dom][m][n]
// (Cp = C'' = C' diag(n), scaled by the norm / merge / carry kernels)
struct Gemm2Args {
  double2* psi;
  double2* psi_out = nullptr;  // nullptr: in place; else the result goes here (psi is only read)
  const double2* B;
  const double2* Cp;
  const double* nfac;
  int ndom, nproj, norb;
  long long ng;
  int num_sms;
  // int8-digit tensor-core path (nl_i8.cu): B's digit tiles and row scales from launch_bslice_i8, or nullptr
  const int8_t* bsl = nullptr;
  const double* bsig = nullptr;
  int sp = 0;  // the SP variant: Psi, B complex64, 4 digits per operand
};
cudaError_t launch_gemm2(const Gemm2Args& a, cudaStream_t st);
// GEMM-2 with FP64 accuracy on the tcgen05 int8 tensor cores (nl_i8.cu): nproj <= 64, norb <= 64.
bool gemm2_i8_supported(int nproj, int norb);
size_t gemm2_i8_bytes(int ndom, long long ng, int S);  // B digit tiles (S digits: 6 FP64, 4 SP)
size_t gemm2_i8_sig_bytes(int ndom, long long ng);  // B row scales
cudaError_t launch_bslice_i8(const void* B, bool sp, int ndom, int nproj, long long ng, int8_t* out, double* sig,
                             cudaStream_t st);
cudaError_t launch_gemm2_i8(const Gemm2Args& a, cudaStream_t st);
cudaError_t gemm_i8_set_attributes();
// GEMM-1 with FP64 accuracy on the int8 tensor cores (nl_i8.cu): split partials (same layout as launch_gemm1)
// of C = B^H Psi and the column norms; needs colE[dom][norb] from the K_y K_z pass that wrote Psi.
struct Gemm1I8Args {
  const double2* psi;
  const int8_t* bsl1;   // B digit blocks (launch_bslice1_i8)
  const int* bexp;      // [dom][nproj] B column exponents
  int* colE;            // [dom][norb] Psi orbital exponents (cleared by the last CTA)
  int* counter;         // [dom] CTA completion counters (zero between calls)
  const int* colsum;    // [dom][nsplit][S][nproj] column sums of B's digits per split (launch_bslice1_i8)
  double2* part;        // [dom][nsplit][nproj][norb]
  double* norms;        // [dom][nsplit][norb]
  int ndom, nproj, norb, nsplit;
  long long ng, rps;
  int sp = 0;  // the SP variant (complex64 Psi, 3 digits; colE from the SP z pass)
};
// The first nonlocal factor's GEMM-2 fused with the x pass of the local propagator (nl_fx.cu):
//   Psi[x][yz] <- K_x (Phi . (n Psi + B C''))  along every x-line (y, z), int8-digit tcgen05 products.
// B's digits and row scales in x-line order are made once at lfd_init (launch_bslicex_i8).
struct FxMaps;  // TMA descriptors (digits, Psi, Phi) -- host-owned, built at lfd_init
bool gemm2x_supported(const Geometry& g);
size_t gemm2x_digit_bytes(const Geometry& g);
size_t gemm2x_sig_bytes(const Geometry& g);
cudaError_t launch_bslicex_i8(const Geometry& g, const void* B, int8_t* dig, double* sig, cudaStream_t st);
FxMaps* gemm2x_maps_create(const Geometry& g, const int8_t* dig, void* psi, const void* phi);
void gemm2x_maps_destroy(FxMaps* m);
cudaError_t launch_gemm2x_i8(const Geometry& g, const FxMaps* m, void* psi, const DomCoef* coef, const double* nfac,
                             const double2* Cp, const double* sig, bool scaled, int num_sms, cudaStream_t st);
cudaError_t gemm2x_set_attributes();

size_t gemm1_i8_bytes(int ndom, long long ng, bool sp);
size_t gemm1_i8_colsum_bytes(int ndom, int nsplit, int nproj, bool sp);
long long gemm1_i8_rows_per_split(long long ng, int ndom, int num_sms);
cudaError_t launch_bslice1_i8(const void* B, bool sp, int ndom, int nproj, long long ng, long long rps, int nsplit,
                              int* bexp, int8_t* out, int* colsum, cudaStream_t st);
cudaError_t launch_gemm1_i8(const Gemm1I8Args& a, cudaStream_t st);
cudaError_t gemm_set_attributes();

// Density / current (a7). Output addressing: out index = base[dom] + x*sx + y*sy + z,
// j component d at + d*jstride.
struct DensArgs {
  const double2* psi;
  const float2* psi_sp = nullptr;  // SP variant: complex64 Psi (then psi is unused)
  const DomCoef* coef;
  const double* occ;
  double* rho;
  double* j;            // may be nullptr
  double* jline;        // [dom][density_blocks][3] per-CTA partial sums of j (for J)
  const long long* base;   // [dom] device array: rho offset of the domain's (0,0,0)
  const long long* jbase;  // [dom] device array: j offset of the domain's (0,0,0), component 0
  long long sx, sy, jstride;
  const double* v;      // v_loc copy [dom][ng] when energy partials are wanted, else nullptr
  double* epart;        // [dom][density_blocks][2] per-CTA sums of (kinetic, local) energy densities
  double* Jmac = nullptr;  // [dom][3]: the y-marching kernel's last CTA reduces jline into J (else k_jreduce)
  int* dcount = nullptr;   // [dom] CTA completion counters for that reduction (zero between launches)
};
struct DensMaps;  // TMA descriptors of Psi for the y-marching density kernel (dens.cu)
bool density_reduces_J(const DensMaps* m);  // launch_density writes J itself (no k_jreduce)
// nact: active orbitals (1 + last index with f != 0); f = 0 orbitals add exactly zero to rho, j, E
DensMaps* density_maps_create(const Geometry& g, const double2* psi, int nact);  // nullptr: generic kernel
cudaError_t density_maps_set_active(DensMaps* m, const Geometry& g, const double2* psi, int nact);
void density_maps_destroy(DensMaps* m);
cudaError_t launch_density(const Geometry& g, const DensArgs& a, const DensMaps* maps, cudaStream_t st);
int density_blocks(const Geometry& g);  // workspace bound on the CTAs per domain
int density_blocks_used(const Geometry& g, const DensMaps* m);  // CTAs per domain of launch_density
cudaError_t density_set_attributes();
cudaError_t launch_jreduce(const Geometry& g, const double* jline, int blocks, double* Jmac, cudaStream_t st);

// calc_energy / remap_occ reductions (energy.cu)
cudaError_t launch_energy_final(const Geometry& g, const double* epart, int blocks, const double2* C,
                                const double* D, const double* occ, double* E, cudaStream_t st);
cudaError_t launch_remap(const Geometry& g, int nref, const double2* C, const double* occ, double* out,
                         cudaStream_t st);

// SP variant projector GEMMs (nl_sp.cu; 3xTF32 on the warp-level tensor path). GEMM-1 takes the geometry
// of a Gemm1Args (part / norms / sizes / strides) with complex64 operands A, X; GEMM-2 rounds C'' to
// complex64 into X32 [ndom][nproj][norb] and updates psi in place.
cudaError_t launch_gemm1_sp(const Gemm1Args& a, const float2* A, const float2* X, cudaStream_t st);
cudaError_t launch_gemm2_sp(float2* psi, const float2* B, const double2* Cp, float2* X32, const double* nfac,
                            int ndom, int nproj, int norb, long long ng, cudaStream_t st, float2* psi_out = nullptr);
cudaError_t gemm_sp_set_attributes();

// Self-consistent step kernels (sc.cu, readings R23-R28).
cudaError_t launch_sc_maxwell_begin(double* st, const double* a_mid, const double* a_end, double dt, bool maxwell,
                                    const Geometry& g, DomCoef* coef_mid, DomCoef* coef_end, cudaStream_t s);
cudaError_t launch_sc_maxwell_end(double* st, const double* jbar, double dt, bool maxwell, cudaStream_t s);
cudaError_t launch_sc_jbar(const double* Jmac, int ndom, double w, double* out, cudaStream_t s);
cudaError_t launch_sc_vmid(const Geometry& g, const double* vion, const double* va, const double* vb, double wa,
                           double wb, const int* off, int GY, int GZ, double* vout, cudaStream_t s);
cudaError_t launch_sc_poisson(double2* spec, const int* gdims, const Geometry& g, cudaStream_t s);
cudaError_t launch_sc_vhxc(const double* rho, double* v, long long n, bool hartree, bool xc, cudaStream_t s);

}  // namespace lfd
