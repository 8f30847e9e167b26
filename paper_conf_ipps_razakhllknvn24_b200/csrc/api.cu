// api.cu -- the C ABI of include/lfd.h: validation, workspace layout, step sequencing, profiling.
// Every numerical step runs in the sm_100a kernels of kin.cu / nl.cu / dens.cu; this file only
// orders them on the context stream. There is no CPU fallback.
#include <cuda_runtime.h>
#include <cufft.h>
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <complex>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <set>
#include <string>
#include <vector>

#include "../../include/lfd.h"
#include "herm_eig.h"
#include "lfd_internal.h"

using lfd::DomCoef;
using lfd::Geometry;

namespace {

constexpr size_t kAlign = 256;
constexpr int kGraphChunk = 32;  // steps per captured CUDA graph (lfd_step_graph)
constexpr int kKC1 = 32;  // GEMM-1 rows per chunk (nl.cu)

size_t up(size_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

struct Layout {
  size_t phi, coef, G, D, occ, part, normp, dc, cprime, s, nfac, jline, base, vstage, rhostage, Jstage, hv[2], hrho[2], hJ[2], cref,
      epart, W, ones, x32, aseq, jseq, bsl, bsig, bsl1, bexp, colE, g1cnt, g1cs, btil, qmat, zero, bslx, sigx, dcount;
  int nref_cap;
  bool i8;  // GEMM-2 on the int8 tensor cores (nl_i8.cu): B digit tiles + row scales in the workspace
  bool fx;  // the first factor's GEMM-2 fused with the x pass (nl_fx.cu)
  int nsplit_i8;           // GEMM-1 on the int8 tensor cores: splits of rows_per_split_i8 rows
  long long rows_per_split_i8;
  size_t total;
  int nsplit;
  long long rows_per_split;
  int nsplit_g;              // split count of the one-time G = dV B^H B (partials of nproj^2 each)
  long long rows_per_split_g;
};

thread_local std::string g_tls_error = "no error";
std::mutex g_live_mu;
std::set<const void*> g_live;

bool is_live(const void* p) {
  std::lock_guard<std::mutex> lk(g_live_mu);
  return g_live.count(p) != 0;
}

lfd_status validate(const lfd_config* c, std::string& why) {
  if (!c) { why = "config is NULL"; return LFD_EINVAL; }
  if (c->abi_version != LFD_ABI_VERSION) { why = "abi_version mismatch"; return LFD_EINVAL; }
  if (c->ndomains < 1 || c->ndomains > LFD_MAX_DOMAINS) { why = "ndomains out of range"; return LFD_EINVAL; }
  if (c->nx < 2 || c->ny < 2 || c->nz < 2) { why = "each of nx, ny, nz must be >= 2"; return LFD_EINVAL; }
  if (c->bc != LFD_BC_PERIODIC && c->bc != LFD_BC_ZERO) { why = "bad bc"; return LFD_EINVAL; }
  if (c->bc == LFD_BC_PERIODIC && ((c->nx | c->ny | c->nz) & 1)) {
    why = "periodic boundary needs even nx, ny, nz (pair splitting, reading R8)";
    return LFD_EINVAL;
  }
  if (!(c->hx > 0) || !(c->hy > 0) || !(c->hz > 0) || !std::isfinite(c->hx * c->hy * c->hz)) {
    why = "spacings must be finite and > 0";
    return LFD_EINVAL;
  }
  if (c->norb < 1) { why = "norb must be >= 1"; return LFD_EINVAL; }
  if (c->nproj < 0 || c->nproj > 2048) { why = "nproj must be in [0, 2048]"; return LFD_EINVAL; }
  if (!(c->dt != 0.0) || !std::isfinite(c->dt)) { why = "dt must be finite and nonzero"; return LFD_EINVAL; }
  if (c->flags & ~(LFD_FLAG_NO_CARRY | LFD_FLAG_EXACT_NL | LFD_FLAG_SP | LFD_FLAG_NL_DMMA | LFD_FLAG_NL_I8 |
                   LFD_FLAG_DENSE_D | LFD_FLAG_NO_PDL)) {
    why = "unknown flags";
    return LFD_EINVAL;
  }
  if ((c->flags & LFD_FLAG_DENSE_D) && c->nproj > 512) {
    why = "LFD_FLAG_DENSE_D supports nproj <= 512";
    return LFD_EINVAL;
  }
  if (c->nref_max < 0 || c->nref_max > 2048) { why = "nref_max must be in [0, 2048]"; return LFD_EINVAL; }
  const long long ng = (long long)c->nx * c->ny * c->nz;
  if (ng * (long long)std::max(c->norb, std::max(c->nproj, 1)) >= (1LL << 31)) {
    why = "ng * max(norb, nproj) must be < 2^31 per domain";
    return LFD_EINVAL;
  }
  return LFD_OK;
}

// The projector GEMMs on the tcgen05 int8 tensor cores (nl_i8.cu): the default for FP64 contexts with
// nproj, norb <= 64 and >= 64K points per domain; LFD_FLAG_NL_DMMA selects the FP64 DMMA kernels.
// Small grids (< 64K points per domain, e.g. C1 / C3) stay on DMMA by default: there the int8 kernels' per-CTA
// set-up (C'' digits, TMEM allocation, the exponent handshake) is not amortised (C1: 0.084 vs 0.058 ms/step);
// LFD_FLAG_NL_I8 forces the int8 path wherever it is supported.
bool use_i8(const lfd_config* c) {
  const bool on = (c->flags & LFD_FLAG_NL_DMMA) == 0;  // (SP contexts: 4-digit int8 GEMMs, else 3xTF32 mma.sync)
  const long long ng = (long long)c->nx * c->ny * c->nz;
  const bool want = ng >= 65536 || (c->flags & LFD_FLAG_NL_I8);
  return on && want && lfd::gemm2_i8_supported(c->nproj, c->norb);
}

Geometry geometry(const lfd_config* c) {
  Geometry g;
  g.ndom = c->ndomains; g.nx = c->nx; g.ny = c->ny; g.nz = c->nz;
  g.norb = c->norb; g.nproj = c->nproj; g.bc = c->bc;
  g.hx = c->hx; g.hy = c->hy; g.hz = c->hz; g.dt = c->dt; g.dV = c->hx * c->hy * c->hz;
  g.ng = (long long)c->nx * c->ny * c->nz;
  g.sp = (c->flags & LFD_FLAG_SP) ? 1 : 0;
  g.i8 = use_i8(c) ? 1 : 0;
  return g;
}

Layout layout(const Geometry& g, int num_sms, int nref_max, bool dense = false) {
  Layout L{};
  L.i8 = g.i8 != 0;
  L.nref_cap = nref_max > 0 ? nref_max : std::max(g.norb, g.nproj);
  const int np = g.nproj, no = g.norb, nd = g.ndom;
  // split-K of GEMM-1: about one CTA per SM in total, each split a multiple of the chunk height
  int tiles = 0;
  if (np > 0) {
    const int t1 = ((np + 63) / 64) * ((no + 63) / 64);
    const int t2 = ((np + 63) / 64) * ((np + 63) / 64);
    tiles = std::min(t1, t2) * nd;
  }
  // pick the split count with the best wave efficiency (CTAs / (waves * SMs)), preferring fewer
  // splits unless more splits are clearly better; each split keeps >= 8 chunks of rows
  int nsplit = 1;
  if (tiles > 0) {
    double best = 0.0;
    const long long max_s = std::max<long long>(1, std::min<long long>(2LL * num_sms, g.ng / (2 * kKC1)));
    for (long long s = 1; s <= max_s; ++s) {
      const long long ctas = (long long)tiles * s;
      const long long waves = (ctas + num_sms - 1) / num_sms;
      const double eff = (double)ctas / (double)(waves * num_sms);
      if (eff > best + 0.02) {
        best = eff;
        nsplit = (int)s;
      }
    }
  }
  long long rps = (g.ng + nsplit - 1) / nsplit;
  rps = std::max<long long>(kKC1, (rps + kKC1 - 1) / kKC1 * kKC1);
  nsplit = (int)((g.ng + rps - 1) / rps);
  L.nsplit = nsplit;
  L.rows_per_split = rps;
  const size_t c16 = 16, d8 = 8;
  const size_t mn = (size_t)std::max(np * no, L.nref_cap * no);
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t at = o; o += up(std::max<size_t>(bytes, 1)); return at; };
  L.phi = take((size_t)nd * g.ng * c16);
  L.coef = take((size_t)nd * sizeof(DomCoef));
  L.G = take((size_t)nd * np * np * c16);
  L.D = take((size_t)nd * np * d8);
  L.occ = take((size_t)nd * no * d8);
  if (L.i8) {
    L.rows_per_split_i8 = lfd::gemm1_i8_rows_per_split(g.ng, nd, num_sms);
    L.nsplit_i8 = (int)((g.ng + L.rows_per_split_i8 - 1) / L.rows_per_split_i8);
  }
  const int nsplit_cap = std::max(nsplit, L.i8 ? L.nsplit_i8 : 0);
  // G needs nproj^2 per split: it takes as many splits as fit the per-step partial buffer (at least one), so
  // the workspace is sized by the per-step GEMM-1, not by the once-only Gram matrix
  {
    const long long gsz = std::max<long long>(1, (long long)np * np);
    long long sg = std::max<long long>(1, std::min<long long>(nsplit, (long long)nsplit_cap * (long long)mn / gsz));
    long long rg = (g.ng + sg - 1) / sg;
    rg = std::max<long long>(kKC1, (rg + kKC1 - 1) / kKC1 * kKC1);
    L.nsplit_g = (int)((g.ng + rg - 1) / rg);
    L.rows_per_split_g = rg;
  }
  L.part = take((size_t)nd * std::max((size_t)nsplit_cap * mn, (size_t)L.nsplit_g * np * np) * c16);
  L.normp = take((size_t)nd * nsplit_cap * no * d8);
  L.dc = take((size_t)nd * np * no * c16);
  L.cprime = take((size_t)nd * np * no * c16);
  L.s = take((size_t)nd * no * d8);
  L.nfac = take((size_t)nd * no * d8);
  L.jline = take((size_t)nd * lfd::density_blocks(g) * 3 * d8);
  L.dcount = take((size_t)nd * sizeof(int));  // density CTA completion counters (zero between launches)
  L.base = take((size_t)4 * nd * sizeof(long long));
  L.vstage = take((size_t)nd * g.ng * d8);
  L.rhostage = take((size_t)nd * g.ng * d8);
  L.Jstage = take((size_t)nd * 3 * d8);
  for (int k = 0; k < 2; ++k) {  // double-buffered staging of the host-buffer calls (copies on side streams)
    L.hv[k] = take((size_t)nd * g.ng * d8);
    L.hrho[k] = take((size_t)nd * g.ng * d8);
    L.hJ[k] = take((size_t)nd * 3 * d8);
  }
  L.cref = take((size_t)nd * std::max(L.nref_cap, np) * no * c16);
  L.epart = take((size_t)nd * lfd::density_blocks(g) * 2 * d8);
  L.W = take((size_t)2 * nd * np * c16);
  L.ones = take((size_t)nd * std::max(np, no) * d8);
  L.x32 = g.sp ? take((size_t)nd * np * std::max(no, dense ? np : 0) * 8) : 0;  // SP: GEMM-2 coefficient (c64)
  L.aseq = take((size_t)kGraphChunk * nd * 3 * d8);   // lfd_step_graph: A of the chunk's steps
  L.jseq = take((size_t)kGraphChunk * nd * 3 * d8);   // lfd_step_graph: J of the chunk's steps
  const int S = g.sp ? 4 : 6;  // int8 digits per operand
  L.bsl = L.i8 ? take(lfd::gemm2_i8_bytes(nd, g.ng, S)) : 0;
  L.bsig = L.i8 ? take(lfd::gemm2_i8_sig_bytes(nd, g.ng)) : 0;
  L.bsl1 = L.i8 ? take(lfd::gemm1_i8_bytes(nd, g.ng, g.sp)) : 0;
  L.g1cs = L.i8 ? take(lfd::gemm1_i8_colsum_bytes(nd, L.nsplit_i8, np, g.sp)) : 0;
  L.bexp = L.i8 ? take((size_t)nd * np * sizeof(int)) : 0;
  L.colE = L.i8 ? take((size_t)nd * no * sizeof(int)) : 0;
  L.g1cnt = L.i8 ? take((size_t)nd * sizeof(int)) : 0;
  // dense D (LFD_FLAG_DENSE_D): the rotated projectors B Q, the eigenvectors Q and a zero vector (GEMM-2's n)
  L.btil = dense ? take((size_t)nd * g.ng * np * (g.sp ? 8 : c16)) : 0;
  L.qmat = dense ? take((size_t)nd * np * np * c16) : 0;
  L.zero = dense ? take((size_t)nd * np * d8) : 0;
  // the first nonlocal factor's GEMM-2 fused with the x pass (nl_fx.cu): B's digits and scales in x-line order
  L.fx = lfd::gemm2x_supported(g);
  L.bslx = L.fx ? take(lfd::gemm2x_digit_bytes(g)) : 0;
  L.sigx = L.fx ? take(lfd::gemm2x_sig_bytes(g)) : 0;
  L.total = o;
  return L;
}

int query_sms(int device) {
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) return 0;
  return sms;
}

struct ProfSlot {
  int kid;
  cudaEvent_t a, b;
};

// ---- self-consistent step state (lfd_sc_*; sc.cu) ----------------------------------------------------
// Minimal NCCL declarations (the library is loaded with dlopen at lfd_sc_comm_init; no link dependency).
typedef struct {
  char internal[128];
} nccl_unique_id;
typedef void* nccl_comm;
typedef int (*nccl_get_unique_id_fn)(nccl_unique_id*);
typedef int (*nccl_comm_init_rank_fn)(nccl_comm*, int, nccl_unique_id, int);
typedef int (*nccl_all_reduce_fn)(const void*, void*, size_t, int, int, nccl_comm, cudaStream_t);
typedef int (*nccl_comm_destroy_fn)(nccl_comm);
typedef const char* (*nccl_error_string_fn)(int);
constexpr int kNcclFloat64 = 8, kNcclSum = 0;

struct Nccl {
  void* h = nullptr;
  nccl_get_unique_id_fn get_unique_id = nullptr;
  nccl_comm_init_rank_fn comm_init_rank = nullptr;
  nccl_all_reduce_fn all_reduce = nullptr;
  nccl_comm_destroy_fn comm_destroy = nullptr;
  nccl_error_string_fn error_string = nullptr;
};

const Nccl* nccl_load(std::string& why) {
  static Nccl n;
  static bool tried = false;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (!tried) {
    tried = true;
    n.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (n.h) {
      n.get_unique_id = (nccl_get_unique_id_fn)dlsym(n.h, "ncclGetUniqueId");
      n.comm_init_rank = (nccl_comm_init_rank_fn)dlsym(n.h, "ncclCommInitRank");
      n.all_reduce = (nccl_all_reduce_fn)dlsym(n.h, "ncclAllReduce");
      n.comm_destroy = (nccl_comm_destroy_fn)dlsym(n.h, "ncclCommDestroy");
      n.error_string = (nccl_error_string_fn)dlsym(n.h, "ncclGetErrorString");
    }
  }
  if (!n.h || !n.get_unique_id || !n.comm_init_rank || !n.all_reduce || !n.comm_destroy) {
    why = std::string("NCCL (libnccl.so.2) could not be loaded: ") + (n.h ? "missing symbols" : dlerror() ? dlerror() : "dlopen failed");
    return nullptr;
  }
  return &n;
}

struct ScLayout {
  size_t pack, vh0, vh1, vh2, spec, state, coef_end, gbase, off, jtmp, fftwork, psi_save, total;
  size_t fft_bytes;
};

struct ScState {
  bool ready = false;
  int flags = 0, n_corr = 0, nranks = 1, rank = 0;
  int gd[3] = {0, 0, 0};
  long long GN = 0;
  ScLayout L{};
  char* ws = nullptr;
  const double* vion = nullptr;
  int vi[3] = {0, 1, 2};  // rotation of the three global v_Hxc buffers: [t_n, t_n-1, new]
  cufftHandle plan_f = 0, plan_b = 0;
  bool plans = false;
  nccl_comm comm = nullptr;
  int comm_nranks = 1, comm_rank = 0;
  template <class T>
  T* at(size_t off) const { return reinterpret_cast<T*>(ws + off); }
  double* vh(int k) const { return at<double>(k == 0 ? L.vh0 : k == 1 ? L.vh1 : L.vh2); }
};

}  // namespace

struct lfd_ctx {
  lfd_config cfg;
  Geometry g;
  Layout L;
  double2* psi;
  const double2* proj;
  char* ws;
  size_t ws_bytes;
  cudaStream_t stream;
  int device;
  int num_sms;
  uint64_t launches = 0;
  // Projection carry: true while the workspace's DC / C' / s / n describe the GEMM-2 that produced the
  // current Psi, so the next nonlocal factor can take C from the exact identity C_new = (C + G X) n
  // instead of GEMM-1 (cleared by the local propagator, lfd_psi_modified and LFD_FLAG_NO_CARRY).
  bool c_valid = false;
  bool carry = true;
  // lfd_step_prologue: the first nonlocal factor of the next step has been applied already (Psi = N(Psi(t_n)));
  // the next lfd_step / lfd_step_sequence starts with the local factor. Observers of Psi are refused meanwhile.
  bool nl_pending = false;
  // int8-digit GEMM-1: the orbital exponents in the workspace describe the current Psi (set by the K_y K_z
  // pass that wrote it, consumed -- and cleared on the device -- by GEMM-1)
  bool colE_valid = false;
  bool no_pdl = false;    // LFD_FLAG_NO_PDL: plain stream order for every launch
  bool exact = false;     // LFD_FLAG_EXACT_NL: exactly unitary nonlocal factor (orthonormal B)
  bool kin_fused = true;  // Phi.K_y K_z in one pass (else separate y and z passes: lines too long for the ring)
  CUtensorMap psi_tmap;   // TMA descriptor of Psi for the fused pass
  lfd::DensMaps* dmaps = nullptr;  // TMA descriptors of Psi for the density kernel
  lfd::FxMaps* fxm = nullptr;      // TMA descriptors of the fused GEMM-2 + x pass (nullptr: not used)
  bool scaled = true;     // scaled pair form of the stencil (else the general 2x2 form: some cos(tau t) < 1/2)
  // lfd_set_vector_potential (ndom <= kCoefFuse) only records A; the coefficient tables are written by the next
  // phase kernel (lfd_set_potential) or, before any other kernel, by k_coef (launch())
  bool a_pending = false;
  double a_pend[3 * lfd::kCoefFuse];
  std::string err = "no error";
  // density-current global layout cache
  std::vector<long long> gbase_host;
  // profiling
  bool prof = false;
  std::vector<ProfSlot> slots;
  size_t nslot = 0;
  double prof_ms[LFD_K_COUNT] = {0};
  int64_t prof_n[LFD_K_COUNT] = {0};
  ScState sc;  // self-consistent step (lfd_sc_*)
  // lfd_step_graph: captured CUDA graphs of K steps (+ density), keyed by what changes the launch sequence
  struct Graph {
    cudaGraphExec_t exec = nullptr;
    int K = 0;
    bool cv0 = false, cv1 = false;  // projection carry valid before / after the chunk
    double* rho = nullptr;
    bool dens = false;
    uint64_t nlaunch = 0;  // kernels per replay
  };
  std::vector<Graph> graphs;
  cudaStream_t cap_stream = nullptr;  // private stream for capture only (the legacy stream cannot capture)
  // host-buffer calls: H2D / D2H on two side streams, double-buffered staging, created on first use
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t ev_vcopy[2] = {}, ev_vfree[2] = {}, ev_dens[2] = {}, ev_d2h[2] = {};
  long long nvh = 0, ndh = 0;  // host-buffer calls so far (slot = count % 2)

  template <class T>
  T* at(size_t off) const { return reinterpret_cast<T*>(ws + off); }
  DomCoef* coef() const { return at<DomCoef>(L.coef); }
  double2* phi() const { return at<double2>(L.phi); }
  // SP variant views (complex64 Psi, B, Phi)
  float2* psi32() const { return reinterpret_cast<float2*>(psi); }
  const float2* proj32() const { return reinterpret_cast<const float2*>(proj); }
  float2* phi32() const { return at<float2>(L.phi); }
  size_t celem() const { return g.sp ? 8 : 16; }
};

namespace {

lfd_status fail(lfd_ctx* c, lfd_status st, const std::string& msg) {
  if (c) c->err = msg; else g_tls_error = msg;
  return st;
}

lfd_status cuda_fail(lfd_ctx* c, cudaError_t e, const char* what) {
  std::string m = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
  return fail(c, LFD_ECUDA, m);
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

void prof_flush(lfd_ctx* c) {
  if (c->nslot == 0) return;
  cudaStreamSynchronize(c->stream);
  for (size_t i = 0; i < c->nslot; ++i) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, c->slots[i].a, c->slots[i].b) == cudaSuccess) {
      c->prof_ms[c->slots[i].kid] += ms;
      c->prof_n[c->slots[i].kid] += 1;
    }
  }
  c->nslot = 0;
}

lfd_status flush_A(lfd_ctx* c);
template <class F>
lfd_status launch(lfd_ctx* c, int kid, const char* name, F&& f) {
  if (c->a_pending && kid != LFD_K_PHASE) {  // every other kernel may read the coefficients
    const lfd_status fs = flush_A(c);
    if (fs != LFD_OK) return fs;
  }
  ProfSlot* s = nullptr;
  if (c->prof) {
    if (c->nslot == c->slots.size()) {
      if (c->slots.size() < 8192) {
        ProfSlot ns{};
        if (cudaEventCreate(&ns.a) != cudaSuccess || cudaEventCreate(&ns.b) != cudaSuccess)
          return fail(c, LFD_ECUDA, "cudaEventCreate failed");
        c->slots.push_back(ns);
      } else {
        prof_flush(c);
      }
    }
    s = &c->slots[c->nslot++];
    s->kid = kid;
    cudaEventRecord(s->a, c->stream);
  }
  cudaError_t e;
  if ((c->g.sp && !c->L.i8) || c->no_pdl) {  // the 3xTF32 SP contexts launch without PDL (C2 SP step 0.98 ms without, 1.12 ms
                             // with: the early-resident CTAs of the next kernel slow the SP GEMMs' cp.async rings)
    const bool prev = lfd::pdl_suspended();
    lfd::pdl_suspend(true);
    e = f();
    lfd::pdl_suspend(prev);
  } else {
    e = f();
  }
  if (s) cudaEventRecord(s->b, c->stream);
  c->launches++;
  if (e != cudaSuccess) return cuda_fail(c, e, name);
  return LFD_OK;
}

#define LFD_TRY(x)                 \
  do {                             \
    lfd_status st_ = (x);          \
    if (st_ != LFD_OK) return st_; \
  } while (0)

// 1 + the last orbital index with a nonzero occupation in any domain (at least 1): the density kernel
// reads only these (f = 0 orbitals add exactly zero to rho, j and the energies).
int active_orbitals(const Geometry& g, const double* occ) {
  int n = 1;
  for (int d = 0; d < g.ndom; ++d)
    for (int s = g.norb - 1; s >= n; --s)
      if (occ[(long long)d * g.norb + s] != 0.0) {
        n = s + 1;
        break;
      }
  return n;
}

lfd_status check_ctx(const lfd_ctx* c) {
  if (!c) { g_tls_error = "context is NULL"; return LFD_EINVAL; }
  if (!is_live(c)) { g_tls_error = "context is not live (destroyed or never created)"; return LFD_ESTATE; }
  return LFD_OK;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// GEMM-1 launch in the context's precision (the SP variant reads complex64 A and X).
cudaError_t gemm1_any(lfd_ctx* c, const lfd::Gemm1Args& a) {
  if (c->g.sp)
    return lfd::launch_gemm1_sp(a, reinterpret_cast<const float2*>(a.A), reinterpret_cast<const float2*>(a.X),
                                c->stream);
  return lfd::launch_gemm1(a, c->stream);
}

// Phi from v in the context's precision (vcopy as lfd::launch_phase).
cudaError_t phase_any(lfd_ctx* c, const double* v, double* vcopy) {
  lfd::CoefFuse cf{};
  if (c->a_pending) {  // the pending coefficient tables in the same launch
    for (int i = 0; i < 3 * c->g.ndom; ++i) cf.A[i / 3][i % 3] = c->a_pend[i];
    cf.count = c->g.ndom;
    cf.coef = c->coef();
    c->a_pending = false;
  }
  if (c->g.sp) return lfd::launch_phase_sp(c->g, v, c->phi32(), vcopy, c->scaled, c->stream, &cf);
  return lfd::launch_phase(c->g, v, c->phi(), vcopy, c->scaled, c->stream, &cf);
}

// GEMM-2 of a nonlocal factor: Psi <- (Psi + B C') diag(n), C' and n from the workspace; with out != nullptr
// the result goes to `out` (same layout) and Psi is only read.
lfd_status gemm2(lfd_ctx* c, double2* out = nullptr) {
  const Geometry& g = c->g;
  lfd::Gemm2Args a2;
  a2.psi = c->psi; a2.B = c->proj; a2.Cp = c->at<double2>(c->L.cprime); a2.nfac = c->at<double>(c->L.nfac);
  a2.ndom = g.ndom; a2.nproj = g.nproj; a2.norb = g.norb; a2.ng = g.ng; a2.num_sms = c->num_sms;
  a2.psi_out = out;
  if (c->L.i8) {
    a2.bsl = c->at<int8_t>(c->L.bsl);
    a2.bsig = c->at<double>(c->L.bsig);
    a2.sp = g.sp;
  }
  c->c_valid = false;
  if (g.sp && !c->L.i8)
    LFD_TRY(launch(c, LFD_K_NL_BACK, "k_gemm2_sp", [&] {
      return lfd::launch_gemm2_sp(c->psi32(), c->proj32(), a2.Cp, c->at<float2>(c->L.x32), a2.nfac, g.ndom, g.nproj,
                                  g.norb, g.ng, c->stream, reinterpret_cast<float2*>(out));
    }));
  else
    LFD_TRY(launch(c, LFD_K_NL_BACK, "k_gemm2", [&] { return lfd::launch_gemm2(a2, c->stream); }));
  c->c_valid = c->carry;
  return LFD_OK;
}

// Exact-factor coefficients: W1 = e^{-i (Delta/2) D} - 1 (one factor), W2 = e^{-i Delta D} - 1 (two merged).
const double2* exact_w(lfd_ctx* c, bool merged) {
  return c->at<double2>(c->L.W) + (merged ? (size_t)c->g.ndom * c->g.nproj : 0);
}

// GEMM-2 of a factor that the local propagator's x pass follows, fused with it (nl_fx.cu): Psi <- K_x(Phi .
// (n Psi + B C'')); afterwards the local propagator runs without its x pass.
lfd_status gemm2x(lfd_ctx* c) {
  c->c_valid = false;
  return launch(c, LFD_K_NL_BACKX, "k_gemm2x_i8", [&] {
    return lfd::launch_gemm2x_i8(c->g, c->fxm, c->g.sp ? (void*)c->psi32() : (void*)c->psi, c->coef(),
                                 c->at<double>(c->L.nfac),
                                 c->at<double2>(c->L.cprime), c->at<double>(c->L.sigx), c->scaled, c->num_sms,
                                 c->stream);
  });
}

// Eq. 6 nonlocal factor N on every domain (kernels a3, a4, a5); merged = N o N in one pass; fused = the GEMM-2
// also applies the next local factor's Phi . K_x (gemm2x; only when c->fxm).
lfd_status nl_half(lfd_ctx* c, bool merged = false, double2* out = nullptr, bool fused = false) {
  const Geometry& g = c->g;
  auto finish = [&]() { return fused ? gemm2x(c) : gemm2(c, out); };
  if (c->c_valid) {  // C of the current Psi from the previous factor (no GEMM-1, no reduction)
    double* D = c->at<double>(c->L.D);
    double2* DC = c->at<double2>(c->L.dc);
    double2* X = c->at<double2>(c->L.cprime);
    double* s = c->at<double>(c->L.s);
    double* nfac = c->at<double>(c->L.nfac);
    if (c->exact) {  // exactly unitary factor: C_new = C + G X, X = W C_new (n stays 1)
      LFD_TRY(launch(c, LFD_K_NL_CARRY, "k_nlcarry", [&] {
        return lfd::launch_nlcarry(g.ndom, g.nproj, g.norb, 0.5 * g.dt, c->at<double2>(c->L.G),
                                   c->at<double>(c->L.ones), DC, X, s, nfac, false, exact_w(c, merged), c->stream);
      }));
      return finish();
    }
    LFD_TRY(launch(c, LFD_K_NL_CARRY, "k_nlcarry", [&] {
      return lfd::launch_nlcarry(g.ndom, g.nproj, g.norb, 0.5 * g.dt, c->at<double2>(c->L.G), D, DC, X, s, nfac,
                                 !merged, nullptr, c->stream);
    }));
    if (merged)
      LFD_TRY(launch(c, LFD_K_NL_NORM, "k_nlmerge", [&] {
        return lfd::launch_nlmerge(g.ndom, g.nproj, g.norb, 0.5 * g.dt, c->at<double2>(c->L.G), D, DC, s, X, nfac,
                                   c->stream);
      }));
    return finish();
  }
  lfd::Gemm1Args a1;
  a1.A = c->proj;
  a1.X = c->psi;
  a1.part = c->at<double2>(c->L.part);
  a1.norms = c->at<double>(c->L.normp);
  a1.ndom = g.ndom; a1.mrows = g.nproj; a1.ncols = g.norb; a1.nsplit = c->L.nsplit;
  a1.ng = g.ng; a1.rows_per_split = c->L.rows_per_split;
  a1.a_dom_stride = g.ng * g.nproj; a1.x_dom_stride = g.ng * g.norb;
  int nsplit = c->L.nsplit;
  if (c->L.i8 && c->colE_valid) {  // int8-digit tensor-core GEMM-1 (Psi's orbital exponents from the K_y K_z pass)
    lfd::Gemm1I8Args ai;
    ai.psi = c->psi; ai.bsl1 = c->at<int8_t>(c->L.bsl1); ai.bexp = c->at<int>(c->L.bexp);
    ai.colE = c->at<int>(c->L.colE); ai.counter = c->at<int>(c->L.g1cnt); ai.colsum = c->at<int>(c->L.g1cs);
    ai.part = a1.part; ai.norms = a1.norms;
    ai.ndom = g.ndom; ai.nproj = g.nproj; ai.norb = g.norb; ai.nsplit = c->L.nsplit_i8;
    ai.ng = g.ng; ai.rps = c->L.rows_per_split_i8; ai.sp = g.sp;
    LFD_TRY(launch(c, LFD_K_NL_PROJ, "k_gemm1_i8", [&] { return lfd::launch_gemm1_i8(ai, c->stream); }));
    c->colE_valid = false;
    nsplit = c->L.nsplit_i8;
  } else {
    LFD_TRY(launch(c, LFD_K_NL_PROJ, "k_gemm1", [&] { return gemm1_any(c, a1); }));
  }
  lfd::ReduceArgs r;
  r.part = a1.part; r.normp = a1.norms;
  r.D = c->at<double>(c->L.D);
  r.out = c->at<double2>(c->L.dc);
  r.cprime = c->at<double2>(c->L.cprime);
  r.s = c->at<double>(c->L.s);
  r.ndom = g.ndom; r.mrows = g.nproj; r.ncols = g.norb; r.nsplit = nsplit;
  r.scale = g.dV; r.eps = 0.5 * g.dt;
  if (c->exact) {  // C (undecorated) and C'' = W C; n == 1 (set at init)
    r.D = nullptr;
    r.W = exact_w(c, merged);
    LFD_TRY(launch(c, LFD_K_NL_REDUCE, "k_reduce", [&] { return lfd::launch_reduce(r, c->stream); }));
    return finish();
  }
  LFD_TRY(launch(c, LFD_K_NL_REDUCE, "k_reduce", [&] { return lfd::launch_reduce(r, c->stream); }));
  if (merged)
    LFD_TRY(launch(c, LFD_K_NL_NORM, "k_nlmerge", [&] {
      return lfd::launch_nlmerge(g.ndom, g.nproj, g.norb, 0.5 * g.dt, c->at<double2>(c->L.G), r.D, r.out, r.s,
                                 r.cprime, c->at<double>(c->L.nfac), c->stream);
    }));
  else
    LFD_TRY(launch(c, LFD_K_NL_NORM, "k_nlnorm", [&] {
      return lfd::launch_nlnorm(g.ndom, g.nproj, g.norb, 0.5 * g.dt, c->at<double2>(c->L.G), r.out, r.s,
                                c->at<double>(c->L.nfac), r.cprime, c->stream);
    }));
  return finish();
}

// Local factor exp(-i Delta h_loc) of Eq. 6: Psi <- Phi . K_z K_y K_x (Phi . Psi) (kernels a6).
// src != nullptr: the first pass reads src (same layout) and writes Psi (out of place).
lfd_status local_prop(lfd_ctx* c, const double2* src = nullptr, bool skip_x = false) {
  c->c_valid = false;
  if (c->g.sp && c->kin_fused) {  // SP variant: Phi.K_x (unless fused into the GEMM-2), then Phi.K_y K_z fused
    if (!skip_x)
      LFD_TRY(launch(c, LFD_K_KIN_X, "k_kin_sp(x)", [&] {
        return lfd::launch_kin_sp(c->g, c->psi32(), c->coef(), c->phi32(), 0, 1, c->scaled, c->stream,
                                  reinterpret_cast<const float2*>(src));
      }));
    int* colE = c->L.i8 ? c->at<int>(c->L.colE) : nullptr;  // exponents for the int8-digit GEMM-1
    LFD_TRY(launch(c, LFD_K_KIN_YZ, "k_kin_yz_sp", [&] {
      return lfd::launch_kin_yz_sp(c->g, &c->psi_tmap, c->psi32(), c->coef(), c->phi32(), c->scaled, c->stream, colE);
    }));
    c->colE_valid = colE != nullptr;
    return LFD_OK;
  }
  if (c->g.sp) {  // SP variant: three FP32 line passes Phi.K_x, K_y, K_z.Phi (complex64 Psi)
    if (!skip_x)
      LFD_TRY(launch(c, LFD_K_KIN_X, "k_kin_sp(x)", [&] {
        return lfd::launch_kin_sp(c->g, c->psi32(), c->coef(), c->phi32(), 0, 1, c->scaled, c->stream,
                                  reinterpret_cast<const float2*>(src));
      }));
    LFD_TRY(launch(c, LFD_K_KIN_Y, "k_kin_sp(y)", [&] {
      return lfd::launch_kin_sp(c->g, c->psi32(), c->coef(), c->phi32(), 1, 0, c->scaled, c->stream);
    }));
    int* colE = c->L.i8 ? c->at<int>(c->L.colE) : nullptr;  // exponents for the int8-digit GEMM-1
    LFD_TRY(launch(c, LFD_K_KIN_Z, "k_kin_sp(z)", [&] {
      return lfd::launch_kin_sp(c->g, c->psi32(), c->coef(), c->phi32(), 2, 2, c->scaled, c->stream, nullptr, colE);
    }));
    c->colE_valid = colE != nullptr;
    return LFD_OK;
  }
  if (!skip_x)
    LFD_TRY(launch(c, LFD_K_KIN_X, "k_kin(x)",
                   [&] { return lfd::launch_kin(c->g, c->psi, c->coef(), c->phi(), 0, 1, c->scaled, c->stream, src); }));
  if (c->kin_fused) {
    int* colE = c->L.i8 ? c->at<int>(c->L.colE) : nullptr;
    LFD_TRY(launch(c, LFD_K_KIN_YZ, "k_kin_yz", [&] {
      return lfd::launch_kin_yz(c->g, &c->psi_tmap, c->psi, c->coef(), c->phi(), c->scaled, c->stream, colE);
    }));
    c->colE_valid = colE != nullptr;
    return LFD_OK;
  }
  LFD_TRY(launch(c, LFD_K_KIN_Y, "k_kin(y)",
                 [&] { return lfd::launch_kin(c->g, c->psi, c->coef(), c->phi(), 1, 0, c->scaled, c->stream); }));
  return launch(c, LFD_K_KIN_Z, "k_kin(z)",
                [&] { return lfd::launch_kin(c->g, c->psi, c->coef(), c->phi(), 2, 2, c->scaled, c->stream); });
}

// C[dom][m][n] = dV sum_r conj(A[r][m]) Psi[r][n] into out (GEMM-1 + fixed-order reduction).
lfd_status project(lfd_ctx* c, const double2* A, int mrows, double2* out) {
  const Geometry& g = c->g;
  lfd::Gemm1Args a1;
  a1.A = A; a1.X = c->psi; a1.part = c->at<double2>(c->L.part); a1.norms = nullptr;
  a1.ndom = g.ndom; a1.mrows = mrows; a1.ncols = g.norb; a1.nsplit = c->L.nsplit;
  a1.ng = g.ng; a1.rows_per_split = c->L.rows_per_split;
  a1.a_dom_stride = g.ng * mrows; a1.x_dom_stride = g.ng * g.norb;
  LFD_TRY(launch(c, LFD_K_NL_PROJ, "k_gemm1", [&] { return gemm1_any(c, a1); }));
  lfd::ReduceArgs r{};
  r.part = a1.part; r.normp = nullptr; r.D = nullptr; r.out = out; r.cprime = nullptr; r.s = nullptr;
  r.ndom = g.ndom; r.mrows = mrows; r.ncols = g.norb; r.nsplit = c->L.nsplit; r.scale = g.dV; r.eps = 0;
  return launch(c, LFD_K_NL_REDUCE, "k_reduce", [&] { return lfd::launch_reduce(r, c->stream); });
}

lfd_status set_A(lfd_ctx* c, const double* A) {
  c->a_pending = false;
  thread_local lfd::CoefParams tp;  // 12 KB kernel-parameter block (A captured by value)
  for (int d0 = 0; d0 < c->g.ndom; d0 += lfd::kCoefMaxPerLaunch) {
    const int cnt = std::min(lfd::kCoefMaxPerLaunch, c->g.ndom - d0);
    for (int i = 0; i < cnt; ++i)
      for (int d = 0; d < 3; ++d) tp.A[i][d] = A ? A[3 * (d0 + i) + d] : 0.0;
    LFD_TRY(launch(c, LFD_K_COEF, "k_coef",
                   [&] { return lfd::launch_coef(c->g, tp, d0, cnt, c->coef(), c->stream); }));
  }
  return LFD_OK;
}

lfd_status flush_A(lfd_ctx* c) {
  c->a_pending = false;
  return set_A(c, c->a_pend);
}

lfd_status density_into(lfd_ctx* c, double* rho, double* j, double* Jmac, const long long* base_dev, long long sx,
                        long long sy, long long jstride, bool energy = false, const DomCoef* coef = nullptr) {
  lfd::DensArgs a;
  a.psi = c->psi; a.coef = coef ? coef : c->coef(); a.occ = c->at<double>(c->L.occ);
  a.psi_sp = c->g.sp ? c->psi32() : nullptr;
  a.rho = rho; a.j = j; a.jline = c->at<double>(c->L.jline);
  a.base = base_dev; a.jbase = base_dev + c->g.ndom; a.sx = sx; a.sy = sy; a.jstride = jstride;
  a.v = energy ? c->at<double>(c->L.vstage) : nullptr;
  a.epart = energy ? c->at<double>(c->L.epart) : nullptr;
  a.Jmac = Jmac;
  a.dcount = c->at<int>(c->L.dcount);
  LFD_TRY(launch(c, LFD_K_DENSITY, "k_density", [&] { return lfd::launch_density(c->g, a, c->dmaps, c->stream); }));
  if (Jmac && !lfd::density_reduces_J(c->dmaps))
    LFD_TRY(launch(c, LFD_K_JREDUCE, "k_jreduce",
                   [&] { return lfd::launch_jreduce(c->g, a.jline, lfd::density_blocks_used(c->g, c->dmaps), Jmac, c->stream); }));
  return LFD_OK;
}


// ---- self-consistent step helpers --------------------------------------------------------------------
lfd_status sc_validate(const lfd_ctx* c, const lfd_sc_config* sc, std::string& why) {
  if (!sc) { why = "sc config is NULL"; return LFD_EINVAL; }
  if (sc->flags & ~(LFD_SC_HARTREE | LFD_SC_XC | LFD_SC_MAXWELL)) { why = "unknown SC flags"; return LFD_EINVAL; }
  if (sc->n_corr < 0 || sc->n_corr > 16) { why = "n_corr must be in [0, 16]"; return LFD_EINVAL; }
  for (int i = 0; i < 3; ++i)
    if (sc->gdims[i] < 1) { why = "gdims must be >= 1"; return LFD_EINVAL; }
  if (sc->nranks < 1 || sc->rank < 0 || sc->rank >= sc->nranks) { why = "bad nranks / rank"; return LFD_EINVAL; }
  if (!sc->dom_offset) { why = "dom_offset is NULL"; return LFD_EINVAL; }
  const Geometry& g = c->g;
  const long long GN = (long long)sc->gdims[0] * sc->gdims[1] * sc->gdims[2];
  if (GN >= (1LL << 31)) { why = "global grid too large"; return LFD_EINVAL; }
  const int nd[3] = {g.nx, g.ny, g.nz};
  for (int d = 0; d < g.ndom; ++d)
    for (int i = 0; i < 3; ++i)
      if (sc->dom_offset[3 * d + i] < 0 || sc->dom_offset[3 * d + i] + nd[i] > sc->gdims[i]) {
        why = "domain core outside the global grid";
        return LFD_EINVAL;
      }
  for (int a = 0; a < g.ndom; ++a)  // own cores must not overlap (boxes of equal shape)
    for (int b = a + 1; b < g.ndom; ++b) {
      bool sep = false;
      for (int i = 0; i < 3; ++i)
        sep = sep || std::abs(sc->dom_offset[3 * a + i] - sc->dom_offset[3 * b + i]) >= nd[i];
      if (!sep) { why = "domain cores overlap"; return LFD_EINVAL; }
    }
  if (sc->nranks == 1 && (long long)g.ndom * g.ng != GN) {
    why = "with nranks == 1 the domain cores must tile gdims exactly";
    return LFD_EINVAL;
  }
  return LFD_OK;
}

cudaError_t fft_work_bytes(const int* gd, size_t* bytes) {
  size_t wf = 0, wb = 0;
  cufftHandle pf, pb;
  if (cufftCreate(&pf) != CUFFT_SUCCESS) return cudaErrorUnknown;
  if (cufftCreate(&pb) != CUFFT_SUCCESS) { cufftDestroy(pf); return cudaErrorUnknown; }
  cufftSetAutoAllocation(pf, 0);
  cufftSetAutoAllocation(pb, 0);
  cufftResult r1 = cufftMakePlan3d(pf, gd[0], gd[1], gd[2], CUFFT_D2Z, &wf);
  cufftResult r2 = cufftMakePlan3d(pb, gd[0], gd[1], gd[2], CUFFT_Z2D, &wb);
  cufftDestroy(pf);
  cufftDestroy(pb);
  if (r1 != CUFFT_SUCCESS || r2 != CUFFT_SUCCESS) return cudaErrorUnknown;
  *bytes = std::max(wf, wb);
  return cudaSuccess;
}

ScLayout sc_layout(const Geometry& g, const lfd_sc_config* sc, size_t fft_bytes) {
  ScLayout L{};
  const long long GN = (long long)sc->gdims[0] * sc->gdims[1] * sc->gdims[2];
  const long long GH = (long long)sc->gdims[0] * sc->gdims[1] * (sc->gdims[2] / 2 + 1);
  const size_t d8 = 8, c16 = 16;
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t at = o; o += up(std::max<size_t>(bytes, 1)); return at; };
  L.pack = take((size_t)(GN + 3) * d8);
  L.vh0 = take((size_t)GN * d8);
  L.vh1 = take((size_t)GN * d8);
  L.vh2 = take((size_t)GN * d8);
  L.spec = take((size_t)GH * c16);
  L.state = take(32 * d8);
  L.coef_end = take((size_t)g.ndom * sizeof(DomCoef));
  L.gbase = take((size_t)2 * g.ndom * sizeof(long long));
  L.off = take((size_t)3 * g.ndom * sizeof(int));
  L.jtmp = take((size_t)3 * g.ndom * d8);
  L.fft_bytes = fft_bytes;
  L.fftwork = take(fft_bytes);
  L.psi_save = take((size_t)g.ndom * g.ng * g.norb * (g.sp ? 8 : c16));  // S = N(Psi(t_n)) (lfd_sc_step)
  L.total = o;
  return L;
}

// Eq.-6 step of every domain with the context's current Phi and coefficients.
lfd_status one_step(lfd_ctx* c) {
  const bool fx = c->fxm != nullptr && c->g.nproj > 0 && !c->nl_pending;
  if (c->g.nproj > 0 && !c->nl_pending) LFD_TRY(nl_half(c, false, nullptr, fx));
  c->nl_pending = false;
  LFD_TRY(local_prop(c, nullptr, fx));
  if (c->g.nproj > 0) LFD_TRY(nl_half(c));
  return LFD_OK;
}

// rho (global layout) and this rank's Jbar share into the pack buffer; SUM all-reduce over ranks.
lfd_status sc_density(lfd_ctx* c) {
  ScState& S = c->sc;
  const Geometry& g = c->g;
  double* pack = S.at<double>(S.L.pack);
  if (S.comm) {
    cudaError_t e = cudaMemsetAsync(pack, 0, sizeof(double) * (S.GN + 3), c->stream);
    if (e != cudaSuccess) return cuda_fail(c, e, "memset rho_g");
  }
  LFD_TRY(density_into(c, pack, nullptr, S.at<double>(S.L.jtmp), S.at<long long>(S.L.gbase),
                       (long long)S.gd[1] * S.gd[2], S.gd[2], S.GN, false, S.at<DomCoef>(S.L.coef_end)));
  LFD_TRY(launch(c, LFD_K_SC, "k_sc_jbar", [&] {
    return lfd::launch_sc_jbar(S.at<double>(S.L.jtmp), g.ndom, (double)g.ng / (double)S.GN, pack + S.GN, c->stream);
  }));
  if (S.comm) {  // the communicator of lfd_sc_comm_init (also used with nranks == 1 when set)
    std::string why;
    const Nccl* n = nccl_load(why);
    if (!n) return fail(c, LFD_EUNSUPPORTED, why);
    int r = n->all_reduce(pack, pack, (size_t)(S.GN + 3), kNcclFloat64, kNcclSum, S.comm, c->stream);
    if (r != 0) return fail(c, LFD_ECUDA, std::string("ncclAllReduce: ") + (n->error_string ? n->error_string(r) : "error"));
  }
  return LFD_OK;
}

// v_Hxc[rho_g] into the global buffer `out` (R23 Hartree by cuFFT, R24 exchange).
lfd_status sc_vhxc(lfd_ctx* c, double* out) {
  ScState& S = c->sc;
  const double* rho = S.at<double>(S.L.pack);
  const bool H = S.flags & LFD_SC_HARTREE, X = S.flags & LFD_SC_XC;
  if (H) {
    double2* spec = S.at<double2>(S.L.spec);
    cufftSetStream(S.plan_f, c->stream);
    cufftSetStream(S.plan_b, c->stream);
    LFD_TRY(launch(c, LFD_K_FFT, "cufftExecD2Z", [&] {
      return cufftExecD2Z(S.plan_f, const_cast<double*>(rho), reinterpret_cast<cufftDoubleComplex*>(spec)) == CUFFT_SUCCESS
                 ? cudaGetLastError() : cudaErrorUnknown;
    }));
    LFD_TRY(launch(c, LFD_K_SC, "k_sc_poisson", [&] { return lfd::launch_sc_poisson(spec, S.gd, c->g, c->stream); }));
    LFD_TRY(launch(c, LFD_K_FFT, "cufftExecZ2D", [&] {
      return cufftExecZ2D(S.plan_b, reinterpret_cast<cufftDoubleComplex*>(spec), out) == CUFFT_SUCCESS
                 ? cudaGetLastError() : cudaErrorUnknown;
    }));
  }
  return launch(c, LFD_K_SC, "k_sc_vhxc", [&] { return lfd::launch_sc_vhxc(rho, out, S.GN, H, X, c->stream); });
}

// v_loc = v_ion + wa va + wb vb (global buffers gathered per domain point), then Phi.
lfd_status sc_set_v(lfd_ctx* c, const double* va, double wa, const double* vb, double wb) {
  ScState& S = c->sc;
  double* vst = c->at<double>(c->L.vstage);
  LFD_TRY(launch(c, LFD_K_SC, "k_sc_vmid", [&] {
    return lfd::launch_sc_vmid(c->g, S.vion, va, vb, wa, wb, S.at<int>(S.L.off), S.gd[1], S.gd[2], vst, c->stream);
  }));
  return launch(c, LFD_K_PHASE, "k_phase",
                [&] { return phase_any(c, vst, vst); });
}

void sc_release(ScState& S) {
  if (S.plans) {
    cufftDestroy(S.plan_f);
    cufftDestroy(S.plan_b);
    S.plans = false;
  }
  S.ready = false;
}


// ---- lfd_step_graph: K steps (+ density) as one CUDA graph ---------------------------------------------
// The body every replay runs: per step k, the coefficient table from A in the workspace (aseq[k]), the
// Eq.-6 step, and (if requested) the density into rho and J into jseq[k].
lfd_status graph_body(lfd_ctx* c, int K, double* rho, bool dens) {
  const Geometry& g = c->g;
  for (int k = 0; k < K; ++k) {
    LFD_TRY(launch(c, LFD_K_COEF, "k_coef_dev", [&] {
      return lfd::launch_coef_dev(g, c->at<double>(c->L.aseq) + (size_t)k * g.ndom * 3, c->coef(), c->stream);
    }));
    LFD_TRY(one_step(c));
    if (dens)
      LFD_TRY(density_into(c, rho ? rho : c->at<double>(c->L.rhostage), nullptr,
                           c->at<double>(c->L.jseq) + (size_t)k * g.ndom * 3, c->at<long long>(c->L.base),
                           (long long)g.ny * g.nz, g.nz, g.ng));
  }
  return LFD_OK;
}

// The cached graph for (K, carry state, outputs), captured on first use.
lfd_status get_graph(lfd_ctx* c, int K, double* rho, bool dens, lfd_ctx::Graph** out) {
  for (auto& gr : c->graphs)
    if (gr.K == K && gr.cv0 == c->c_valid && gr.rho == rho && gr.dens == dens) {
      *out = &gr;
      return LFD_OK;
    }
  if (!c->cap_stream) {
    cudaError_t e = cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) return cuda_fail(c, e, "cudaStreamCreate (graph capture)");
  }
  if (c->a_pending) LFD_TRY(flush_A(c));  // (not into the captured graph)
  lfd_ctx::Graph gr;
  gr.K = K; gr.cv0 = c->c_valid; gr.rho = rho; gr.dens = dens;
  cudaStream_t orig = c->stream;
  const uint64_t l0 = c->launches;
  c->stream = c->cap_stream;
  cudaError_t e = cudaStreamBeginCapture(c->cap_stream, cudaStreamCaptureModeThreadLocal);
  if (e != cudaSuccess) { c->stream = orig; return cuda_fail(c, e, "cudaStreamBeginCapture"); }
  lfd::pdl_suspend(true);
  lfd_status st = graph_body(c, K, rho, dens);
  lfd::pdl_suspend(false);
  cudaGraph_t graph = nullptr;
  e = cudaStreamEndCapture(c->cap_stream, &graph);
  c->stream = orig;
  if (st != LFD_OK) { if (graph) cudaGraphDestroy(graph); c->c_valid = gr.cv0; return st; }
  if (e != cudaSuccess) { c->c_valid = gr.cv0; return cuda_fail(c, e, "cudaStreamEndCapture"); }
  e = cudaGraphInstantiate(&gr.exec, graph, 0);
  cudaGraphDestroy(graph);
  if (e != cudaSuccess) { c->c_valid = gr.cv0; return cuda_fail(c, e, "cudaGraphInstantiate"); }
  gr.cv1 = c->c_valid;  // the host-side carry logic ran during capture
  c->c_valid = gr.cv0;
  gr.nlaunch = c->launches - l0;
  c->launches = l0;
  c->graphs.push_back(gr);
  *out = &c->graphs.back();
  return LFD_OK;
}

void release_graphs(lfd_ctx* c) {
  for (auto& gr : c->graphs)
    if (gr.exec) cudaGraphExecDestroy(gr.exec);
  c->graphs.clear();
  if (c->cap_stream) cudaStreamDestroy(c->cap_stream);
  c->cap_stream = nullptr;
}

}  // namespace

extern "C" {

lfd_status lfd_workspace_size(const lfd_config* cfg, size_t* bytes) {
  std::string why;
  lfd_status st = validate(cfg, why);
  if (st != LFD_OK) return fail(nullptr, st, why);
  if (!bytes) return fail(nullptr, LFD_EINVAL, "bytes is NULL");
  const int sms = query_sms(cfg->device);
  if (sms <= 0) return fail(nullptr, LFD_ECUDA, "no CUDA device (the LFD library has no CPU fallback)");
  *bytes = layout(geometry(cfg), sms, cfg->nref_max, (cfg->flags & LFD_FLAG_DENSE_D) != 0).total;
  return LFD_OK;
}

lfd_status lfd_init(const lfd_config* cfg, void* psi, const void* proj, const double* dnl, const double* occ,
                    void* workspace, size_t ws_bytes, void* stream, lfd_ctx** out) {
  std::string why;
  lfd_status st = validate(cfg, why);
  if (st != LFD_OK) return fail(nullptr, st, why);
  if (!out) return fail(nullptr, LFD_EINVAL, "out is NULL");
  if (!psi || !workspace || !occ) return fail(nullptr, LFD_EINVAL, "psi, workspace and occ must be non-NULL");
  if ((cfg->nproj > 0) != (proj != nullptr)) return fail(nullptr, LFD_EINVAL, "proj must be non-NULL iff nproj > 0");
  if (cfg->nproj > 0 && !dnl) return fail(nullptr, LFD_EINVAL, "dnl must be non-NULL when nproj > 0");
  const uintptr_t amask = (cfg->flags & LFD_FLAG_SP) ? 7 : 15;
  if ((reinterpret_cast<uintptr_t>(psi) | reinterpret_cast<uintptr_t>(proj)) & amask)
    return fail(nullptr, LFD_EINVAL, "psi / proj must be aligned to their complex element (16 B, or 8 B with LFD_FLAG_SP)");
  if (reinterpret_cast<uintptr_t>(workspace) & (kAlign - 1))
    return fail(nullptr, LFD_EINVAL, "workspace must be 256-byte aligned");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || cfg->device < 0 || cfg->device >= ndev) {
    cudaGetLastError();
    return fail(nullptr, LFD_ECUDA, "no such CUDA device (the LFD library has no CPU fallback)");
  }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, cfg->device) != cudaSuccess) return fail(nullptr, LFD_ECUDA, "cudaGetDeviceProperties failed");
  if (prop.major != 10) return fail(nullptr, LFD_ECUDA, "this build targets sm_100a (B200) only");
  DeviceGuard dg(cfg->device);
  if (!is_device_ptr(psi) || !is_device_ptr(workspace) || (proj && !is_device_ptr(proj)))
    return fail(nullptr, LFD_EINVAL, "psi, proj and workspace must be device memory");
  const Geometry g = geometry(cfg);
  const bool dense = (cfg->flags & LFD_FLAG_DENSE_D) != 0;
  const Layout L = layout(g, prop.multiProcessorCount, cfg->nref_max, dense);
  // the real couplings the kernels use: D_u, or the eigenvalues w of a dense Hermitian D = Q diag(w) Q^H
  std::vector<double> dvals((size_t)g.ndom * g.nproj);
  std::vector<double2> qhost;
  if (g.nproj > 0 && !dense) std::copy(dnl, dnl + dvals.size(), dvals.begin());
  if (g.nproj > 0 && dense) {
    const int np = g.nproj;
    qhost.resize((size_t)g.ndom * np * np);
    std::vector<std::complex<double>> Dm((size_t)np * np), Q((size_t)np * np);
    for (int d = 0; d < g.ndom; ++d) {
      const double* src = dnl + (size_t)d * np * np * 2;
      double mx = 0.0, asym = 0.0;
      for (int u = 0; u < np; ++u)
        for (int v = 0; v < np; ++v) {
          Dm[(size_t)u * np + v] = {src[2 * ((size_t)u * np + v)], src[2 * ((size_t)u * np + v) + 1]};
          mx = std::max(mx, std::abs(Dm[(size_t)u * np + v]));
        }
      for (int u = 0; u < np; ++u)
        for (int v = 0; v < np; ++v)
          asym = std::max(asym, std::abs(Dm[(size_t)u * np + v] - std::conj(Dm[(size_t)v * np + u])));
      if (!std::isfinite(mx) || asym > 1e-12 * mx)
        return fail(nullptr, LFD_EINVAL, "LFD_FLAG_DENSE_D: dnl must be finite Hermitian matrices");
      if (lfd::herm_eig(np, Dm.data(), dvals.data() + (size_t)d * np, Q.data()) < 0)
        return fail(nullptr, LFD_EINVAL, "LFD_FLAG_DENSE_D: the eigensolver did not converge");
      for (size_t k = 0; k < (size_t)np * np; ++k)
        qhost[(size_t)d * np * np + k] = make_double2(Q[k].real(), Q[k].imag());
    }
  }
  if (ws_bytes < L.total) return fail(nullptr, LFD_ENOMEM, "workspace smaller than lfd_workspace_size()");
  cudaError_t e = lfd::gemm_set_attributes();
  if (e == cudaSuccess) e = lfd::density_set_attributes();
  if (e == cudaSuccess) e = lfd::kin_yz_set_attributes();
  if (e == cudaSuccess) e = lfd::gemm_sp_set_attributes();
  if (e == cudaSuccess) e = lfd::gemm_i8_set_attributes();
  if (e == cudaSuccess) e = lfd::gemm2x_set_attributes();
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaFuncSetAttribute");

  lfd_ctx* c = new (std::nothrow) lfd_ctx();
  if (!c) return fail(nullptr, LFD_ENOMEM, "host allocation failed");
  c->cfg = *cfg; c->g = g; c->L = L;
  c->psi = static_cast<double2*>(psi);
  c->proj = static_cast<const double2*>(proj);
  c->ws = static_cast<char*>(workspace);
  c->ws_bytes = ws_bytes;
  c->stream = static_cast<cudaStream_t>(stream);
  c->device = cfg->device;
  c->num_sms = prop.multiProcessorCount;
  c->carry = (cfg->flags & LFD_FLAG_NO_CARRY) == 0;
  c->no_pdl = (cfg->flags & LFD_FLAG_NO_PDL) != 0;
  c->scaled = c->scaled && lfd::kin_scaled_ok(g);
  c->kin_fused = c->kin_fused && lfd::kin_yz_supported(g);
  c->dmaps = lfd::density_maps_create(g, c->psi, active_orbitals(g, occ));
  if (c->kin_fused && lfd::kin_yz_tensor_map(g, c->psi, &c->psi_tmap) != cudaSuccess) {
    cudaGetLastError();
    c->kin_fused = false;  // descriptor not encodable (e.g. alignment): the separate y and z passes
  }
  {
    std::lock_guard<std::mutex> lk(g_live_mu);
    g_live.insert(c);
  }
  auto bail = [&](lfd_status s) {
    std::string m = c->err;
    lfd_destroy(c);
    return fail(nullptr, s, m);
  };
  // copies of the small host arrays (pageable H2D copies are staged before the call returns)
  if (g.nproj > 0) {
    e = cudaMemcpyAsync(c->at<double>(L.D), dvals.data(), sizeof(double) * g.ndom * g.nproj, cudaMemcpyHostToDevice,
                        c->stream);
    if (e != cudaSuccess) { cuda_fail(c, e, "copy dnl"); return bail(LFD_ECUDA); }
  }
  e = cudaMemcpyAsync(c->at<double>(L.occ), occ, sizeof(double) * g.ndom * g.norb, cudaMemcpyHostToDevice, c->stream);
  if (e != cudaSuccess) { cuda_fail(c, e, "copy occ"); return bail(LFD_ECUDA); }
  // local-layout output bases for the density kernel: rho [dom][ng], j [dom][3][ng]
  std::vector<long long> base(2 * g.ndom);
  for (int d = 0; d < g.ndom; ++d) {
    base[d] = (long long)d * g.ng;
    base[g.ndom + d] = (long long)d * 3 * g.ng;
  }
  e = cudaMemcpyAsync(c->at<long long>(L.base), base.data(), sizeof(long long) * base.size(), cudaMemcpyHostToDevice,
                      c->stream);
  if (e != cudaSuccess) { cuda_fail(c, e, "copy base"); return bail(LFD_ECUDA); }
  // initial state: v = 0 (Phi = 1), A = 0; density completion counters 0
  e = cudaMemsetAsync(c->at<double>(L.vstage), 0, sizeof(double) * g.ndom * g.ng, c->stream);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->at<int>(L.dcount), 0, sizeof(int) * g.ndom, c->stream);
  if (e != cudaSuccess) { cuda_fail(c, e, "memset"); return bail(LFD_ECUDA); }
  lfd_status s2 = launch(c, LFD_K_PHASE, "k_phase",
                         [&] { return phase_any(c, c->at<double>(L.vstage), c->at<double>(L.vstage)); });
  if (s2 != LFD_OK) return bail(s2);
  s2 = set_A(c, nullptr);
  if (s2 != LFD_OK) return bail(s2);
  if (dense && g.nproj > 0) {
    // B Q: the projectors rotated into D's eigenbasis (B D B^H = (B Q) diag(w) (B Q)^H), by the FP64 GEMM-2
    // out of place (Psi := B read-only, n = 0, C'' = Q); from here on the context's projectors are B Q
    e = cudaMemcpyAsync(c->at<double2>(L.qmat), qhost.data(), sizeof(double2) * qhost.size(), cudaMemcpyHostToDevice,
                        c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->at<double>(L.zero), 0, sizeof(double) * g.ndom * g.nproj, c->stream);
    if (e != cudaSuccess) { cuda_fail(c, e, "copy Q"); return bail(LFD_ECUDA); }
    if (g.sp) {
      s2 = launch(c, LFD_K_NL_BACK, "k_gemm2_sp(BQ)", [&] {
        return lfd::launch_gemm2_sp(const_cast<float2*>(c->proj32()), c->proj32(), c->at<double2>(L.qmat),
                                    c->at<float2>(L.x32), c->at<double>(L.zero), g.ndom, g.nproj, g.nproj, g.ng,
                                    c->stream, c->at<float2>(L.btil));
      });
    } else {
      lfd::Gemm2Args a2;
      a2.psi = const_cast<double2*>(c->proj); a2.B = c->proj; a2.Cp = c->at<double2>(L.qmat);
      a2.nfac = c->at<double>(L.zero); a2.ndom = g.ndom; a2.nproj = g.nproj; a2.norb = g.nproj; a2.ng = g.ng;
      a2.num_sms = c->num_sms; a2.psi_out = c->at<double2>(L.btil);
      s2 = launch(c, LFD_K_NL_BACK, "k_gemm2(BQ)", [&] { return lfd::launch_gemm2(a2, c->stream); });
    }
    if (s2 != LFD_OK) return bail(s2);
    e = cudaStreamSynchronize(c->stream);  // qhost (host staging) goes out of scope
    if (e != cudaSuccess) { cuda_fail(c, e, "B Q"); return bail(LFD_ECUDA); }
    c->proj = c->at<double2>(L.btil);
  }
  // Gram matrix G = dV B^H B (GEMM-1 with X = B, fixed-order reduction)
  if (g.nproj > 0) {
    lfd::Gemm1Args a1;
    a1.A = c->proj; a1.X = c->proj; a1.part = c->at<double2>(L.part); a1.norms = nullptr;
    a1.ndom = g.ndom; a1.mrows = g.nproj; a1.ncols = g.nproj; a1.nsplit = L.nsplit_g;
    a1.ng = g.ng; a1.rows_per_split = L.rows_per_split_g;
    a1.a_dom_stride = g.ng * g.nproj; a1.x_dom_stride = g.ng * g.nproj;
    s2 = launch(c, LFD_K_NL_PROJ, "k_gemm1(G)", [&] { return gemm1_any(c, a1); });
    if (s2 != LFD_OK) return bail(s2);
    lfd::ReduceArgs r{};
    r.part = a1.part; r.normp = nullptr; r.D = nullptr; r.out = c->at<double2>(L.G); r.cprime = nullptr; r.s = nullptr;
    r.ndom = g.ndom; r.mrows = g.nproj; r.ncols = g.nproj; r.nsplit = L.nsplit_g; r.scale = g.dV; r.eps = 0;
    s2 = launch(c, LFD_K_NL_REDUCE, "k_reduce(G)", [&] { return lfd::launch_reduce(r, c->stream); });
    if (s2 != LFD_OK) return bail(s2);
  }
  if (L.i8) {  // int8 digit tiles of B for the tensor-core GEMM-2 and GEMM-1 (B is constant, like G)
    s2 = launch(c, LFD_K_NL_BACK, "k_bslice_i8", [&] {
      return lfd::launch_bslice_i8(c->proj, g.sp, g.ndom, g.nproj, g.ng, c->at<int8_t>(L.bsl), c->at<double>(L.bsig),
                                   c->stream);
    });
    if (s2 != LFD_OK) return bail(s2);
    s2 = launch(c, LFD_K_NL_PROJ, "k_bslice1_i8", [&] {
      return lfd::launch_bslice1_i8(c->proj, g.sp, g.ndom, g.nproj, g.ng, L.rows_per_split_i8, L.nsplit_i8,
                                    c->at<int>(L.bexp), c->at<int8_t>(L.bsl1), c->at<int>(L.g1cs), c->stream);
    });
    if (s2 != LFD_OK) return bail(s2);
    e = cudaMemsetAsync(c->at<int>(L.colE), 0, sizeof(int) * g.ndom * g.norb, c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->at<int>(L.g1cnt), 0, sizeof(int) * g.ndom, c->stream);
    if (e != cudaSuccess) { cuda_fail(c, e, "memset"); return bail(LFD_ECUDA); }
  }
  if (L.fx) {  // B's digits in x-line order for the fused first factor
    s2 = launch(c, LFD_K_NL_BACKX, "k_bslicex_i8", [&] {
      return lfd::launch_bslicex_i8(g, g.sp ? (const void*)c->proj32() : (const void*)c->proj, c->at<int8_t>(L.bslx),
                                    c->at<double>(L.sigx), c->stream);
    });
    if (s2 != LFD_OK) return bail(s2);
    c->fxm = g.sp ? lfd::gemm2x_maps_create(g, c->at<int8_t>(L.bslx), c->psi32(), c->phi32())
                  : lfd::gemm2x_maps_create(g, c->at<int8_t>(L.bslx), c->psi, c->phi());
    // (no descriptors: the unfused GEMM-2 + x pass run instead)
  }
  if (cfg->flags & LFD_FLAG_EXACT_NL) {
    // exactly unitary nonlocal factor: needs dV B^H B = I (checked on G), then
    // exp(-i (Delta/2) B D B^H dV) = 1 + B diag(e^{-i (Delta/2) D} - 1) B^H dV with n = 1
    c->exact = true;
    if (g.nproj > 0) {
      std::vector<double2> Gh((size_t)g.ndom * g.nproj * g.nproj);
      e = cudaMemcpyAsync(Gh.data(), c->at<double2>(L.G), Gh.size() * sizeof(double2), cudaMemcpyDeviceToHost,
                          c->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
      if (e != cudaSuccess) { cuda_fail(c, e, "copy G"); return bail(LFD_ECUDA); }
      double dev = 0.0;
      for (int d = 0; d < g.ndom; ++d)
        for (int u = 0; u < g.nproj; ++u)
          for (int v = 0; v < g.nproj; ++v) {
            const double2 x = Gh[((size_t)d * g.nproj + u) * g.nproj + v];
            dev = std::max(dev, std::hypot(x.x - (u == v ? 1.0 : 0.0), x.y));
          }
      if (dev > (g.sp ? 1e-5 : 1e-9)) {  // SP: B is orthonormal to FP32 rounding only
        c->err = "LFD_FLAG_EXACT_NL needs dV-orthonormal projector columns (max |dV B^H B - I| = " +
                 std::to_string(dev) + ")";
        return bail(LFD_EINVAL);
      }
      std::vector<double2> Wh((size_t)2 * g.ndom * g.nproj);
      for (size_t i = 0; i < (size_t)g.ndom * g.nproj; ++i)
        for (int k = 0; k < 2; ++k) {  // k = 0: one factor (tau = Delta/2), 1: two merged (tau = Delta)
          const double ph = -(k + 1) * 0.5 * g.dt * dvals[i];
          Wh[k * (size_t)g.ndom * g.nproj + i] = make_double2(std::cos(ph) - 1.0, std::sin(ph));
        }
      e = cudaMemcpyAsync(c->at<double2>(L.W), Wh.data(), Wh.size() * sizeof(double2), cudaMemcpyHostToDevice,
                          c->stream);
      std::vector<double> ones((size_t)g.ndom * std::max(g.nproj, g.norb), 1.0);
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(c->at<double>(L.ones), ones.data(), ones.size() * sizeof(double), cudaMemcpyHostToDevice,
                            c->stream);
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(c->at<double>(L.nfac), ones.data(), sizeof(double) * g.ndom * g.norb,
                            cudaMemcpyHostToDevice, c->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);  // host staging vectors go out of scope
      if (e != cudaSuccess) { cuda_fail(c, e, "copy exact-factor coefficients"); return bail(LFD_ECUDA); }
    }
  }
  *out = c;
  return LFD_OK;
}

lfd_status lfd_set_potential(lfd_ctx* c, const double* vloc) {
  LFD_TRY(check_ctx(c));
  if (!vloc) return fail(c, LFD_EINVAL, "vloc is NULL");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(vloc)) return fail(c, LFD_EINVAL, "vloc must be device memory (use lfd_set_potential_host)");
  return launch(c, LFD_K_PHASE, "k_phase", [&] {
    return phase_any(c, vloc, c->at<double>(c->L.vstage));
  });
}

// The side streams and events of the host-buffer calls (created once; the copies then overlap the kernels
// of the context stream: the H2D of step n+1's v_loc runs during step n, the D2H of step n's rho / J during
// step n+1).
static lfd_status host_copy_init(lfd_ctx* c) {
  if (c->h2d) return LFD_OK;
  cudaError_t e = cudaStreamCreateWithFlags(&c->h2d, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->d2h, cudaStreamNonBlocking);
  for (int k = 0; k < 2 && e == cudaSuccess; ++k) {
    e = cudaEventCreateWithFlags(&c->ev_vcopy[k], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_vfree[k], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_dens[k], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_d2h[k], cudaEventDisableTiming);
  }
  if (e != cudaSuccess) return cuda_fail(c, e, "host copy streams");
  return LFD_OK;
}

lfd_status lfd_set_potential_host(lfd_ctx* c, const double* vloc_host) {
  LFD_TRY(check_ctx(c));
  if (!vloc_host) return fail(c, LFD_EINVAL, "vloc_host is NULL");
  DeviceGuard dg(c->device);
  LFD_TRY(host_copy_init(c));
  const int k = (int)(c->nvh & 1);
  double* stage = c->at<double>(c->L.hv[k]);
  // the H2D into slot k waits for the k_phase that read slot k two calls ago; k_phase waits for the H2D
  cudaError_t e = c->nvh >= 2 ? cudaStreamWaitEvent(c->h2d, c->ev_vfree[k], 0) : cudaSuccess;
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(stage, vloc_host, sizeof(double) * c->g.ndom * c->g.ng, cudaMemcpyHostToDevice, c->h2d);
  if (e == cudaSuccess) e = cudaEventRecord(c->ev_vcopy[k], c->h2d);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(c->stream, c->ev_vcopy[k], 0);
  if (e != cudaSuccess) return cuda_fail(c, e, "H2D vloc");
  LFD_TRY(launch(c, LFD_K_PHASE, "k_phase", [&] { return phase_any(c, stage, c->at<double>(c->L.vstage)); }));
  e = cudaEventRecord(c->ev_vfree[k], c->stream);
  if (e != cudaSuccess) return cuda_fail(c, e, "event");
  ++c->nvh;
  return LFD_OK;
}

lfd_status lfd_set_vector_potential(lfd_ctx* c, const double* A) {
  LFD_TRY(check_ctx(c));
  if (!A) return fail(c, LFD_EINVAL, "A is NULL");
  for (int i = 0; i < 3 * c->g.ndom; ++i)
    if (!std::isfinite(A[i])) return fail(c, LFD_EINVAL, "A must be finite");
  DeviceGuard dg(c->device);
  if (c->g.ndom <= lfd::kCoefFuse) {  // recorded now (by value), applied by the next kernel launch
    std::copy(A, A + 3 * c->g.ndom, c->a_pend);
    c->a_pending = true;
    return LFD_OK;
  }
  return set_A(c, A);
}


lfd_status lfd_step(lfd_ctx* c, int32_t nsteps) {
  LFD_TRY(check_ctx(c));
  if (nsteps < 0) return fail(c, LFD_EINVAL, "nsteps must be >= 0");
  DeviceGuard dg(c->device);
  for (int it = 0; it < nsteps; ++it) LFD_TRY(one_step(c));
  return LFD_OK;
}

lfd_status lfd_step_prologue(lfd_ctx* c) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "a step prologue is already pending");
  DeviceGuard dg(c->device);
  if (c->g.nproj > 0) LFD_TRY(nl_half(c));
  c->nl_pending = true;
  return LFD_OK;
}

lfd_status lfd_step_sequence(lfd_ctx* c, int32_t nsteps, const double* A_seq) {
  LFD_TRY(check_ctx(c));
  if (nsteps < 0) return fail(c, LFD_EINVAL, "nsteps must be >= 0");
  if (nsteps > 0 && !A_seq) return fail(c, LFD_EINVAL, "A_seq is NULL");
  for (long long i = 0; i < 3LL * c->g.ndom * nsteps; ++i)
    if (!std::isfinite(A_seq[i])) return fail(c, LFD_EINVAL, "A_seq must be finite");
  DeviceGuard dg(c->device);
  const bool nl = c->g.nproj > 0;
  const bool fx = c->fxm != nullptr && nl;
  bool x_done = false;  // the x pass of step n already ran inside the preceding factor's GEMM-2
  for (int n = 0; n < nsteps; ++n) {
    if (n == 0) LFD_TRY(set_A(c, A_seq));
    if (nl && n == 0 && !c->nl_pending) {  // first factor of the sequence
      LFD_TRY(nl_half(c, false, nullptr, fx));
      x_done = fx;
    }
    c->nl_pending = false;
    LFD_TRY(local_prop(c, nullptr, x_done));
    x_done = false;
    if (n + 1 < nsteps) LFD_TRY(set_A(c, A_seq + 3LL * c->g.ndom * (n + 1)));  // before a fused x pass reads it
    if (nl) {  // N of step n merged with N of step n+1 (and fused with step n+1's x pass)
      LFD_TRY(nl_half(c, n + 1 < nsteps, nullptr, fx && n + 1 < nsteps));
      x_done = fx && n + 1 < nsteps;
    }
  }
  return LFD_OK;
}

lfd_status lfd_step_graph(lfd_ctx* c, int32_t nsteps, const double* A_seq, double* rho, double* Jmac_seq) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  if (nsteps < 0) return fail(c, LFD_EINVAL, "nsteps must be >= 0");
  if (nsteps > 0 && !A_seq) return fail(c, LFD_EINVAL, "A_seq is NULL");
  for (long long i = 0; i < 3LL * c->g.ndom * nsteps; ++i)
    if (!std::isfinite(A_seq[i])) return fail(c, LFD_EINVAL, "A_seq must be finite");
  DeviceGuard dg(c->device);
  if ((rho && !is_device_ptr(rho)) || (Jmac_seq && !is_device_ptr(Jmac_seq)))
    return fail(c, LFD_EINVAL, "rho / Jmac_seq must be device memory");
  const Geometry& g = c->g;
  const bool dens = rho || Jmac_seq;
  const size_t ab = (size_t)g.ndom * 3 * sizeof(double);
  for (int s0 = 0; s0 < nsteps; s0 += kGraphChunk) {
    const int K = std::min(kGraphChunk, nsteps - s0);
    cudaError_t e = cudaMemcpyAsync(c->at<double>(c->L.aseq), A_seq + (size_t)s0 * g.ndom * 3, ab * K,
                                    cudaMemcpyHostToDevice, c->stream);
    if (e != cudaSuccess) return cuda_fail(c, e, "H2D A_seq");
    if (c->prof) {  // per-kernel timing needs events around every launch: run the same body eagerly
      LFD_TRY(graph_body(c, K, rho, dens));
    } else {
      lfd_ctx::Graph* gr = nullptr;
      LFD_TRY(get_graph(c, K, rho, dens, &gr));
      e = cudaGraphLaunch(gr->exec, c->stream);
      if (e != cudaSuccess) return cuda_fail(c, e, "cudaGraphLaunch");
      c->launches += gr->nlaunch;
      c->c_valid = gr->cv1;
    }
    if (Jmac_seq) {
      e = cudaMemcpyAsync(Jmac_seq + (size_t)s0 * g.ndom * 3, c->at<double>(c->L.jseq), ab * K,
                          cudaMemcpyDeviceToDevice, c->stream);
      if (e != cudaSuccess) return cuda_fail(c, e, "copy J");
    }
  }
  return LFD_OK;  // the coefficient table (the context's A) now holds A_seq[nsteps-1]
}

lfd_status lfd_density_current(lfd_ctx* c, double* rho, double* j, double* Jmac) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  if (!rho) return fail(c, LFD_EINVAL, "rho is NULL");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(rho) || (j && !is_device_ptr(j)) || (Jmac && !is_device_ptr(Jmac)))
    return fail(c, LFD_EINVAL, "rho / j / Jmac must be device memory");
  const Geometry& g = c->g;
  const long long* base = c->at<long long>(c->L.base);  // [rho bases | j bases]
  return density_into(c, rho, j, Jmac, base, (long long)g.ny * g.nz, g.nz, g.ng);
}

lfd_status lfd_density_current_global(lfd_ctx* c, double* rho_g, double* j_g, double* Jmac, const int32_t* off,
                                      const int32_t* gdims) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  if (!rho_g || !off || !gdims) return fail(c, LFD_EINVAL, "rho_g, dom_offset and gdims must be non-NULL");
  const Geometry& g = c->g;
  for (int i = 0; i < 3; ++i)
    if (gdims[i] < 1) return fail(c, LFD_EINVAL, "gdims must be >= 1");
  const int nd[3] = {g.nx, g.ny, g.nz};
  for (int d = 0; d < g.ndom; ++d)
    for (int i = 0; i < 3; ++i)
      if (off[3 * d + i] < 0 || off[3 * d + i] + nd[i] > gdims[i])
        return fail(c, LFD_EINVAL, "domain core outside the global grid");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(rho_g) || (j_g && !is_device_ptr(j_g)) || (Jmac && !is_device_ptr(Jmac)))
    return fail(c, LFD_EINVAL, "rho_g / j_g / Jmac must be device memory");
  const long long GY = gdims[1], GZ = gdims[2];
  const long long GN = (long long)gdims[0] * GY * GZ;
  std::vector<long long> base(2 * g.ndom);
  for (int d = 0; d < g.ndom; ++d) {
    base[d] = ((long long)off[3 * d] * GY + off[3 * d + 1]) * GZ + off[3 * d + 2];
    base[g.ndom + d] = base[d];
  }
  long long* bdev = c->at<long long>(c->L.base) + 2 * g.ndom;
  if (base != c->gbase_host) {
    cudaError_t e = cudaMemcpyAsync(bdev, base.data(), sizeof(long long) * base.size(), cudaMemcpyHostToDevice, c->stream);
    if (e != cudaSuccess) return cuda_fail(c, e, "copy global bases");
    c->gbase_host = base;
  }
  return density_into(c, rho_g, j_g, Jmac, bdev, GY * GZ, GZ, GN);
}

lfd_status lfd_density_current_host(lfd_ctx* c, double* rho_host, double* Jmac_host) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  DeviceGuard dg(c->device);
  const Geometry& g = c->g;
  LFD_TRY(host_copy_init(c));
  const int k = (int)(c->ndh & 1);
  double* rs = c->at<double>(c->L.hrho[k]);
  double* Js = c->at<double>(c->L.hJ[k]);
  // staging slot k is rewritten only after its D2H of two calls ago; the D2H waits for this density
  cudaError_t e = c->ndh >= 2 ? cudaStreamWaitEvent(c->stream, c->ev_d2h[k], 0) : cudaSuccess;
  if (e != cudaSuccess) return cuda_fail(c, e, "event wait");
  LFD_TRY(density_into(c, rs, nullptr, Js, c->at<long long>(c->L.base), (long long)g.ny * g.nz, g.nz, g.ng));
  e = cudaEventRecord(c->ev_dens[k], c->stream);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(c->d2h, c->ev_dens[k], 0);
  if (e == cudaSuccess && rho_host)
    e = cudaMemcpyAsync(rho_host, rs, sizeof(double) * g.ndom * g.ng, cudaMemcpyDeviceToHost, c->d2h);
  if (e == cudaSuccess && Jmac_host)
    e = cudaMemcpyAsync(Jmac_host, Js, sizeof(double) * g.ndom * 3, cudaMemcpyDeviceToHost, c->d2h);
  if (e == cudaSuccess) e = cudaEventRecord(c->ev_d2h[k], c->d2h);
  if (e != cudaSuccess) return cuda_fail(c, e, "D2H rho / J");
  ++c->ndh;
  return LFD_OK;
}

lfd_status lfd_wait_host_outputs(lfd_ctx* c, int32_t lag) {
  LFD_TRY(check_ctx(c));
  if (lag < 0 || lag > 1) return fail(c, LFD_EINVAL, "lag must be 0 or 1");
  if (c->ndh <= lag) return fail(c, LFD_ESTATE, "no such lfd_density_current_host call");
  DeviceGuard dg(c->device);
  cudaError_t e = cudaEventSynchronize(c->ev_d2h[(int)((c->ndh - 1 - lag) & 1)]);
  if (e != cudaSuccess) return cuda_fail(c, e, "asynchronous CUDA error");
  return LFD_OK;
}

lfd_status lfd_energy(lfd_ctx* c, double* E) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  if (!E) return fail(c, LFD_EINVAL, "E is NULL");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(E)) return fail(c, LFD_EINVAL, "E must be device memory");
  const Geometry& g = c->g;
  double2* C = nullptr;
  if (g.nproj > 0) {
    C = c->at<double2>(c->L.cref);
    LFD_TRY(project(c, c->proj, g.nproj, C));
  }
  LFD_TRY(density_into(c, c->at<double>(c->L.rhostage), nullptr, nullptr, c->at<long long>(c->L.base),
                       (long long)g.ny * g.nz, g.nz, g.ng, true));
  return launch(c, LFD_K_ENERGY, "k_energy_final", [&] {
    return lfd::launch_energy_final(g, c->at<double>(c->L.epart), lfd::density_blocks_used(g, c->dmaps), C,
                                    c->at<double>(c->L.D), c->at<double>(c->L.occ), E, c->stream);
  });
}

lfd_status lfd_remap_occ(lfd_ctx* c, const void* ref, int32_t nref, double* occ_out) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  if (!ref || !occ_out) return fail(c, LFD_EINVAL, "ref and occ_out must be non-NULL");
  if (nref < 1 || nref > c->L.nref_cap) return fail(c, LFD_EINVAL, "nref must be in [1, nref_max]");
  if (reinterpret_cast<uintptr_t>(ref) & (c->celem() - 1))
    return fail(c, LFD_EINVAL, "ref must be aligned to its complex element (16 B; 8 B with LFD_FLAG_SP)");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(ref) || !is_device_ptr(occ_out)) return fail(c, LFD_EINVAL, "ref / occ_out must be device memory");
  double2* C = c->at<double2>(c->L.cref);
  LFD_TRY(project(c, static_cast<const double2*>(ref), nref, C));
  return launch(c, LFD_K_ENERGY, "k_remap", [&] {
    return lfd::launch_remap(c->g, nref, C, c->at<double>(c->L.occ), occ_out, c->stream);
  });
}

lfd_status lfd_set_occupations(lfd_ctx* c, const double* occ) {
  LFD_TRY(check_ctx(c));
  if (!occ) return fail(c, LFD_EINVAL, "occ is NULL");
  DeviceGuard dg(c->device);
  cudaError_t e = cudaMemcpyAsync(c->at<double>(c->L.occ), occ, sizeof(double) * c->g.ndom * c->g.norb,
                                  cudaMemcpyHostToDevice, c->stream);
  if (e != cudaSuccess) return cuda_fail(c, e, "copy occ");
  e = lfd::density_maps_set_active(c->dmaps, c->g, c->psi, active_orbitals(c->g, occ));
  if (e == cudaErrorNotSupported) {  // more active orbitals than the y-marching kernel takes: the generic kernel
    lfd::density_maps_destroy(c->dmaps);
    c->dmaps = nullptr;
    e = cudaSuccess;
  }
  if (e != cudaSuccess) return cuda_fail(c, e, "density tensor map");
  release_graphs(c);  // captured graphs hold the density kernel's tensor maps by value
  return LFD_OK;
}

lfd_status lfd_sc_workspace_size(const lfd_ctx* c, const lfd_sc_config* sc, size_t* bytes) {
  LFD_TRY(check_ctx(c));
  std::string why;
  lfd_status st = sc_validate(c, sc, why);
  if (st != LFD_OK) return fail(const_cast<lfd_ctx*>(c), st, why);
  if (!bytes) return fail(const_cast<lfd_ctx*>(c), LFD_EINVAL, "bytes is NULL");
  DeviceGuard dg(c->device);
  size_t fb = 0;
  if (fft_work_bytes(sc->gdims, &fb) != cudaSuccess) return fail(const_cast<lfd_ctx*>(c), LFD_ECUDA, "cuFFT plan failed");
  *bytes = sc_layout(c->g, sc, fb).total;
  return LFD_OK;
}

lfd_status lfd_sc_init(lfd_ctx* c, const lfd_sc_config* sc, const double* vion, void* ws, size_t ws_bytes,
                       const double* Aext0, const double* A_ind0, const double* Adot0) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  std::string why;
  lfd_status st = sc_validate(c, sc, why);
  if (st != LFD_OK) return fail(c, st, why);
  if (!ws || !Aext0) return fail(c, LFD_EINVAL, "ws and Aext0 must be non-NULL");
  if (reinterpret_cast<uintptr_t>(ws) & (kAlign - 1)) return fail(c, LFD_EINVAL, "ws must be 256-byte aligned");
  for (int i = 0; i < 3; ++i)
    if (!std::isfinite(Aext0[i]) || (A_ind0 && !std::isfinite(A_ind0[i])) || (Adot0 && !std::isfinite(Adot0[i])))
      return fail(c, LFD_EINVAL, "Aext0 / A_ind0 / Adot0 must be finite");
  if ((sc->nranks > 1 || c->sc.comm) &&
      (!c->sc.comm || c->sc.comm_nranks != sc->nranks || c->sc.comm_rank != sc->rank))
    return fail(c, LFD_ESTATE, "nranks > 1 needs lfd_sc_comm_init with the same nranks / rank first");
  DeviceGuard dg(c->device);
  if (!is_device_ptr(ws) || (vion && !is_device_ptr(vion))) return fail(c, LFD_EINVAL, "ws / vion must be device memory");
  size_t fb = 0;
  if (fft_work_bytes(sc->gdims, &fb) != cudaSuccess) return fail(c, LFD_ECUDA, "cuFFT plan failed");
  const ScLayout L = sc_layout(c->g, sc, fb);
  if (ws_bytes < L.total) return fail(c, LFD_ENOMEM, "SC workspace smaller than lfd_sc_workspace_size()");
  ScState& S = c->sc;
  sc_release(S);
  S.flags = sc->flags; S.n_corr = sc->n_corr; S.nranks = sc->nranks; S.rank = sc->rank;
  for (int i = 0; i < 3; ++i) S.gd[i] = sc->gdims[i];
  S.GN = (long long)S.gd[0] * S.gd[1] * S.gd[2];
  S.L = L; S.ws = static_cast<char*>(ws); S.vion = vion;
  S.vi[0] = 0; S.vi[1] = 1; S.vi[2] = 2;
  // cuFFT plans on the caller's workspace (the library allocates nothing)
  size_t w1 = 0, w2 = 0;
  if (cufftCreate(&S.plan_f) != CUFFT_SUCCESS) return fail(c, LFD_ECUDA, "cufftCreate");
  if (cufftCreate(&S.plan_b) != CUFFT_SUCCESS) { cufftDestroy(S.plan_f); return fail(c, LFD_ECUDA, "cufftCreate"); }
  S.plans = true;
  cufftSetAutoAllocation(S.plan_f, 0);
  cufftSetAutoAllocation(S.plan_b, 0);
  if (cufftMakePlan3d(S.plan_f, S.gd[0], S.gd[1], S.gd[2], CUFFT_D2Z, &w1) != CUFFT_SUCCESS ||
      cufftMakePlan3d(S.plan_b, S.gd[0], S.gd[1], S.gd[2], CUFFT_Z2D, &w2) != CUFFT_SUCCESS ||
      cufftSetWorkArea(S.plan_f, S.at<void>(L.fftwork)) != CUFFT_SUCCESS ||
      cufftSetWorkArea(S.plan_b, S.at<void>(L.fftwork)) != CUFFT_SUCCESS) {
    sc_release(S);
    return fail(c, LFD_ECUDA, "cuFFT plan setup failed");
  }
  // host-side tables: global output bases of the domain cores and their offsets
  const Geometry& g = c->g;
  std::vector<long long> base(2 * g.ndom);
  std::vector<int> off(3 * g.ndom);
  for (int d = 0; d < g.ndom; ++d) {
    for (int i = 0; i < 3; ++i) off[3 * d + i] = sc->dom_offset[3 * d + i];
    base[d] = ((long long)off[3 * d] * S.gd[1] + off[3 * d + 1]) * S.gd[2] + off[3 * d + 2];
    base[g.ndom + d] = base[d];
  }
  double st0[32] = {0};
  for (int i = 0; i < 3; ++i) {
    st0[i] = A_ind0 ? A_ind0[i] : 0.0;
    st0[3 + i] = Adot0 ? Adot0[i] : 0.0;
  }
  cudaError_t e = cudaMemcpyAsync(S.at<long long>(L.gbase), base.data(), sizeof(long long) * base.size(),
                                  cudaMemcpyHostToDevice, c->stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(S.at<int>(L.off), off.data(), sizeof(int) * off.size(), cudaMemcpyHostToDevice, c->stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(S.at<double>(L.state), st0, sizeof(st0), cudaMemcpyHostToDevice, c->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);  // host staging goes out of scope
  if (e != cudaSuccess) { sc_release(S); return cuda_fail(c, e, "SC init copies"); }
  // state at t_0: coefficients of A(t_0) = A_ext(t_0) + A_ind(t_0), rho, Jbar, v_Hxc(t_0) = v_Hxc(t_-1)
  const double A0[3] = {Aext0[0] + st0[0], Aext0[1] + st0[1], Aext0[2] + st0[2]};
  double* state = S.at<double>(L.state);
  lfd_status r = launch(c, LFD_K_SC, "k_sc_maxwell_begin", [&] {
    return lfd::launch_sc_maxwell_begin(state, A0, A0, g.dt, false, g, c->coef(), S.at<DomCoef>(L.coef_end), c->stream);
  });
  if (r == LFD_OK) r = sc_density(c);
  if (r == LFD_OK) r = sc_vhxc(c, S.vh(S.vi[0]));
  if (r == LFD_OK) {
    e = cudaMemcpyAsync(S.vh(S.vi[1]), S.vh(S.vi[0]), sizeof(double) * S.GN, cudaMemcpyDeviceToDevice, c->stream);
    if (e != cudaSuccess) r = cuda_fail(c, e, "copy v_Hxc");
  }
  if (r == LFD_OK)
    r = launch(c, LFD_K_SC, "k_sc_maxwell_end", [&] {
      return lfd::launch_sc_maxwell_end(state, S.at<double>(L.pack) + S.GN, g.dt, false, c->stream);
    });
  if (r != LFD_OK) { sc_release(S); return r; }
  S.ready = true;
  return LFD_OK;
}

lfd_status lfd_sc_step(lfd_ctx* c, int32_t nsteps, const double* Aext) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  ScState& S = c->sc;
  if (!S.ready) return fail(c, LFD_ESTATE, "lfd_sc_init has not been called");
  if (nsteps < 0) return fail(c, LFD_EINVAL, "nsteps must be >= 0");
  if (nsteps == 0) return LFD_OK;
  if (!Aext) return fail(c, LFD_EINVAL, "Aext is NULL");
  for (long long i = 0; i < 3LL * (2LL * nsteps + 1); ++i)
    if (!std::isfinite(Aext[i])) return fail(c, LFD_EINVAL, "Aext must be finite");
  DeviceGuard dg(c->device);
  const Geometry& g = c->g;
  const bool maxwell = S.flags & LFD_SC_MAXWELL;
  double* state = S.at<double>(S.L.state);
  const size_t psi_bytes = (size_t)g.ndom * g.ng * g.norb * c->celem();
  auto cpy = [&](void* dst, const void* src, size_t n) -> lfd_status {
    cudaError_t e = cudaMemcpyAsync(dst, src, n, cudaMemcpyDeviceToDevice, c->stream);
    return e == cudaSuccess ? LFD_OK : cuda_fail(c, e, "SC device copy");
  };
  // Psi(t_n) lives in the caller's buffer P. The first nonlocal factor of Eq. 6 depends on Psi(t_n), B and
  // D only (not on v or A), so it is applied ONCE per step, out of place into the SC buffer S = N(Psi(t_n));
  // every sweep then runs the local factor from S into P (the first stencil pass reads S, writes P) and the
  // second nonlocal factor in place on P. S is never overwritten, so the corrector needs no copies, and the
  // last sweep leaves Psi(t_n+1) in P with the projection carry of its second factor for the next step.
  double2* Sbuf = S.at<double2>(S.L.psi_save);
  for (int n = 0; n < nsteps; ++n) {
    const double* a_mid = Aext + 3 * (2 * n + 1);
    const double* a_end = Aext + 3 * (2 * n + 2);
    LFD_TRY(launch(c, LFD_K_SC, "k_sc_maxwell_begin", [&] {
      return lfd::launch_sc_maxwell_begin(state, a_mid, a_end, g.dt, maxwell, g, c->coef(), S.at<DomCoef>(S.L.coef_end),
                                          c->stream);
    }));
    double* vn = S.vh(S.vi[0]);
    double* vp = S.vh(S.vi[1]);
    double* vnew = S.vh(S.vi[2]);
    LFD_TRY(sc_set_v(c, vn, 1.5, vp, -0.5));  // predictor (R27)
    if (g.nproj > 0) {
      LFD_TRY(nl_half(c, false, Sbuf));  // S = N(Psi(t_n))
    } else {
      cudaError_t e = cudaMemcpyAsync(Sbuf, c->psi, psi_bytes, cudaMemcpyDeviceToDevice, c->stream);
      if (e != cudaSuccess) return cuda_fail(c, e, "SC device copy");
    }
    for (int k = 0; k <= S.n_corr; ++k) {
      LFD_TRY(local_prop(c, Sbuf));
      if (g.nproj > 0) LFD_TRY(nl_half(c));
      LFD_TRY(sc_density(c));
      LFD_TRY(sc_vhxc(c, vnew));
      if (k < S.n_corr) LFD_TRY(sc_set_v(c, vn, 0.5, vnew, 0.5));  // corrector (R27)
    }
    LFD_TRY(launch(c, LFD_K_SC, "k_sc_maxwell_end", [&] {
      return lfd::launch_sc_maxwell_end(state, S.at<double>(S.L.pack) + S.GN, g.dt, maxwell, c->stream);
    }));
    const int old_prev = S.vi[1];
    S.vi[1] = S.vi[0];
    S.vi[0] = S.vi[2];
    S.vi[2] = old_prev;
  }
  // the context's A is now A(t_end): the density / energy calls use its coefficients
  return cpy(c->coef(), S.at<void>(S.L.coef_end), sizeof(DomCoef) * g.ndom);
}

lfd_status lfd_sc_read(lfd_ctx* c, double* state, double* rho_g, double* vhxc) {
  LFD_TRY(check_ctx(c));
  ScState& S = c->sc;
  if (!S.ready) return fail(c, LFD_ESTATE, "lfd_sc_init has not been called");
  DeviceGuard dg(c->device);
  if ((state && !is_device_ptr(state)) || (rho_g && !is_device_ptr(rho_g)) || (vhxc && !is_device_ptr(vhxc)))
    return fail(c, LFD_EINVAL, "state / rho_g / vhxc must be device memory");
  cudaError_t e = cudaSuccess;
  if (state) e = cudaMemcpyAsync(state, S.at<double>(S.L.state), 9 * sizeof(double), cudaMemcpyDeviceToDevice, c->stream);
  if (e == cudaSuccess && rho_g)
    e = cudaMemcpyAsync(rho_g, S.at<double>(S.L.pack), S.GN * sizeof(double), cudaMemcpyDeviceToDevice, c->stream);
  if (e == cudaSuccess && vhxc)
    e = cudaMemcpyAsync(vhxc, S.vh(S.vi[0]), S.GN * sizeof(double), cudaMemcpyDeviceToDevice, c->stream);
  if (e != cudaSuccess) return cuda_fail(c, e, "SC read");
  return LFD_OK;
}

lfd_status lfd_comm_unique_id(void* id128) {
  if (!id128) { g_tls_error = "id128 is NULL"; return LFD_EINVAL; }
  std::string why;
  const Nccl* n = nccl_load(why);
  if (!n) { g_tls_error = why; return LFD_EUNSUPPORTED; }
  nccl_unique_id id;
  int r = n->get_unique_id(&id);
  if (r != 0) { g_tls_error = "ncclGetUniqueId failed"; return LFD_ECUDA; }
  std::memcpy(id128, id.internal, sizeof(id.internal));
  return LFD_OK;
}

lfd_status lfd_sc_comm_init(lfd_ctx* c, int32_t nranks, int32_t rank, const void* id128) {
  LFD_TRY(check_ctx(c));
  if (nranks < 1 || rank < 0 || rank >= nranks || !id128) return fail(c, LFD_EINVAL, "bad nranks / rank / id");
  std::string why;
  const Nccl* n = nccl_load(why);
  if (!n) return fail(c, LFD_EUNSUPPORTED, why);
  DeviceGuard dg(c->device);
  if (c->sc.comm) {
    n->comm_destroy(c->sc.comm);
    c->sc.comm = nullptr;
  }
  nccl_unique_id id;
  std::memcpy(id.internal, id128, sizeof(id.internal));
  int r = n->comm_init_rank(&c->sc.comm, nranks, id, rank);
  if (r != 0) {
    c->sc.comm = nullptr;
    return fail(c, LFD_ECUDA, std::string("ncclCommInitRank: ") + (n->error_string ? n->error_string(r) : "error"));
  }
  c->sc.comm_nranks = nranks;
  c->sc.comm_rank = rank;
  return LFD_OK;
}

lfd_status lfd_psi_modified(lfd_ctx* c) {
  LFD_TRY(check_ctx(c));
  if (c->nl_pending) return fail(c, LFD_ESTATE, "Psi is between lfd_step_prologue and its step");
  c->c_valid = false;
  if (c->colE_valid) {  // orbital exponents of a Psi that no longer exists: clear them (stream order)
    DeviceGuard dg(c->device);
    cudaError_t e = cudaMemsetAsync(c->at<int>(c->L.colE), 0, sizeof(int) * c->g.ndom * c->g.norb, c->stream);
    if (e != cudaSuccess) return cuda_fail(c, e, "memset");
    c->colE_valid = false;
  }
  return LFD_OK;
}

lfd_status lfd_set_stream(lfd_ctx* c, void* stream) {
  LFD_TRY(check_ctx(c));
  c->stream = static_cast<cudaStream_t>(stream);
  return LFD_OK;
}

lfd_status lfd_sync(lfd_ctx* c) {
  LFD_TRY(check_ctx(c));
  DeviceGuard dg(c->device);
  cudaError_t e = cudaStreamSynchronize(c->stream);
  if (e == cudaSuccess && c->h2d) e = cudaStreamSynchronize(c->h2d);
  if (e == cudaSuccess && c->d2h) e = cudaStreamSynchronize(c->d2h);
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "asynchronous CUDA error");
  return LFD_OK;
}

lfd_status lfd_nl_path(const lfd_ctx* c, int32_t* path) {
  LFD_TRY(check_ctx(c));
  if (!path) return LFD_EINVAL;
  *path = c->g.nproj == 0 ? -1 : c->g.sp ? (c->L.i8 ? 3 : 2) : c->L.i8 ? 1 : 0;
  return LFD_OK;
}

lfd_status lfd_launch_count(const lfd_ctx* c, uint64_t* count) {
  LFD_TRY(check_ctx(c));
  if (!count) return LFD_EINVAL;
  *count = c->launches;
  return LFD_OK;
}

lfd_status lfd_profile_enable(lfd_ctx* c, int32_t enable) {
  LFD_TRY(check_ctx(c));
  c->prof = enable != 0;
  return LFD_OK;
}

lfd_status lfd_profile_read(lfd_ctx* c, double* ms, int64_t* launches) {
  LFD_TRY(check_ctx(c));
  DeviceGuard dg(c->device);
  prof_flush(c);
  for (int k = 0; k < LFD_K_COUNT; ++k) {
    if (ms) ms[k] = c->prof_ms[k];
    if (launches) launches[k] = c->prof_n[k];
    c->prof_ms[k] = 0;
    c->prof_n[k] = 0;
  }
  return LFD_OK;
}

const char* lfd_last_error(const lfd_ctx* c) {
  if (c && is_live(c)) return c->err.c_str();
  return g_tls_error.c_str();
}

lfd_status lfd_destroy(lfd_ctx* c) {
  if (!c) return LFD_OK;
  {
    std::lock_guard<std::mutex> lk(g_live_mu);
    if (!g_live.count(c)) {
      g_tls_error = "lfd_destroy: context is not live";
      return LFD_ESTATE;
    }
    g_live.erase(c);
  }
  {
    DeviceGuard dg(c->device);
    cudaStreamSynchronize(c->stream);
    if (c->h2d) {
      cudaStreamSynchronize(c->h2d);
      cudaStreamSynchronize(c->d2h);
      for (int k = 0; k < 2; ++k) {
        cudaEventDestroy(c->ev_vcopy[k]);
        cudaEventDestroy(c->ev_vfree[k]);
        cudaEventDestroy(c->ev_dens[k]);
        cudaEventDestroy(c->ev_d2h[k]);
      }
      cudaStreamDestroy(c->h2d);
      cudaStreamDestroy(c->d2h);
    }
    for (auto& s : c->slots) {
      cudaEventDestroy(s.a);
      cudaEventDestroy(s.b);
    }
  }
  lfd::density_maps_destroy(c->dmaps);
  lfd::gemm2x_maps_destroy(c->fxm);
  sc_release(c->sc);
  release_graphs(c);
  if (c->sc.comm) {
    std::string why;
    if (const Nccl* n = nccl_load(why)) n->comm_destroy(c->sc.comm);
  }
  delete c;
  return LFD_OK;
}

}  // extern "C"
