"""Thin ctypes binding of the C ABI in include/lfd.h (argument marshalling only).

Every entry point keeps the C name (``lfd_init``, ``lfd_step``, ...). Device buffers are torch CUDA
tensors; their data pointers are passed straight to the library and the current torch stream is used
as the context stream. There is no CPU fallback: if ``liblfd.so`` is missing or no sm_100 device is
present, the calls raise.

``Context`` is a convenience owner that allocates the workspace and keeps the borrowed tensors alive.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liblfd.so")

LFD_ABI_VERSION = 4
LFD_FLAG_NO_CARRY = 1
LFD_FLAG_EXACT_NL = 2
LFD_FLAG_SP = 4
LFD_FLAG_NL_DMMA = 8
LFD_FLAG_NL_I8 = 16
LFD_FLAG_DENSE_D = 32
LFD_FLAG_NO_PDL = 64
LFD_BC_PERIODIC = 0
LFD_BC_ZERO = 1
STATUS = {0: "LFD_OK", -1: "LFD_EINVAL", -2: "LFD_ENOMEM", -3: "LFD_ECUDA", -4: "LFD_ESTATE",
          -5: "LFD_EUNSUPPORTED"}
KERNELS = ("coef", "phase", "kin_x", "kin_y", "kin_z", "nl_proj", "nl_reduce", "nl_norm", "nl_back",
           "density", "jreduce", "energy", "nl_carry", "kin_yz", "sc", "fft", "nl_back_x")
LFD_SC_HARTREE = 1
LFD_SC_XC = 2
LFD_SC_MAXWELL = 4
EXPORTS = ("lfd_workspace_size", "lfd_init", "lfd_set_potential", "lfd_set_potential_host",
           "lfd_set_vector_potential", "lfd_step", "lfd_step_prologue", "lfd_step_sequence", "lfd_density_current", "lfd_density_current_global",
           "lfd_density_current_host", "lfd_wait_host_outputs", "lfd_energy", "lfd_remap_occ", "lfd_psi_modified", "lfd_set_occupations", "lfd_set_stream", "lfd_sync",
           "lfd_launch_count", "lfd_nl_path", "lfd_profile_enable", "lfd_profile_read", "lfd_last_error", "lfd_destroy",
           "lfd_sc_workspace_size", "lfd_sc_init", "lfd_sc_step", "lfd_sc_read", "lfd_comm_unique_id",
           "lfd_sc_comm_init", "lfd_step_graph")


class lfd_config(C.Structure):
    _fields_ = [("abi_version", C.c_int32), ("ndomains", C.c_int32), ("nx", C.c_int32), ("ny", C.c_int32),
                ("nz", C.c_int32), ("hx", C.c_double), ("hy", C.c_double), ("hz", C.c_double),
                ("bc", C.c_int32), ("norb", C.c_int32), ("nproj", C.c_int32), ("nref_max", C.c_int32),
                ("dt", C.c_double), ("device", C.c_int32), ("flags", C.c_int32)]


class lfd_sc_config(C.Structure):
    _fields_ = [("flags", C.c_int32), ("n_corr", C.c_int32), ("gdims", C.c_int32 * 3), ("nranks", C.c_int32),
                ("rank", C.c_int32), ("dom_offset", C.c_void_p)]


class LFDError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None


def load():
    """Load liblfd.so (raises if it was not built -- there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = C.CDLL(LIB_PATH)
    P, I32, D = C.c_void_p, C.c_int32, C.POINTER(C.c_double)
    cfgp = C.POINTER(lfd_config)
    sig = {
        "lfd_workspace_size": [cfgp, C.POINTER(C.c_size_t)],
        "lfd_init": [cfgp, P, P, P, P, P, C.c_size_t, P, C.POINTER(P)],
        "lfd_set_potential": [P, P],
        "lfd_set_potential_host": [P, P],
        "lfd_set_vector_potential": [P, P],
        "lfd_step": [P, I32],
        "lfd_step_prologue": [P],
        "lfd_step_sequence": [P, I32, P],
        "lfd_density_current": [P, P, P, P],
        "lfd_density_current_global": [P, P, P, P, P, P],
        "lfd_density_current_host": [P, P, P],
        "lfd_wait_host_outputs": [P, I32],
        "lfd_energy": [P, P],
        "lfd_remap_occ": [P, P, I32, P],
        "lfd_set_occupations": [P, P],
        "lfd_psi_modified": [P],
        "lfd_set_stream": [P, P],
        "lfd_sync": [P],
        "lfd_launch_count": [P, C.POINTER(C.c_uint64)],
        "lfd_nl_path": [P, C.POINTER(C.c_int32)],
        "lfd_profile_enable": [P, I32],
        "lfd_profile_read": [P, D, C.POINTER(C.c_int64)],
        "lfd_destroy": [P],
        "lfd_sc_workspace_size": [P, C.POINTER(lfd_sc_config), C.POINTER(C.c_size_t)],
        "lfd_sc_init": [P, C.POINTER(lfd_sc_config), P, P, C.c_size_t, P, P, P],
        "lfd_sc_step": [P, I32, P],
        "lfd_sc_read": [P, P, P, P],
        "lfd_comm_unique_id": [P],
        "lfd_sc_comm_init": [P, I32, I32, P],
        "lfd_step_graph": [P, I32, P, P, P],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = C.c_int
    lib.lfd_last_error.argtypes = [P]
    lib.lfd_last_error.restype = C.c_char_p
    _lib = lib
    return lib


def _check(rc: int, ctx=None):
    if rc != 0:
        msg = load().lfd_last_error(ctx).decode()
        raise LFDError(rc, msg)


def _dptr(t) -> C.c_void_p | None:
    if t is None:
        return None
    if not getattr(t, "is_cuda", False):
        raise TypeError("expected a CUDA tensor")
    if not t.is_contiguous():
        raise TypeError("expected a contiguous tensor")
    return C.c_void_p(t.data_ptr())


def _hptr(a, dtype=np.float64):
    """Host pointer of a numpy array or CPU tensor; returns (pointer, keepalive)."""
    if a is None:
        return None, None
    if hasattr(a, "data_ptr") and not getattr(a, "is_cuda", False):
        if not a.is_contiguous():
            raise TypeError("expected a contiguous host tensor")
        return C.c_void_p(a.data_ptr()), a
    arr = np.ascontiguousarray(a, dtype=dtype)
    return C.c_void_p(arr.ctypes.data), arr


def _hptr_async(a):
    """Host pointer for an ASYNC copy (lfd_set_potential_host / lfd_density_current_host): the buffer itself must
    be contiguous float64 (a converted temporary would be freed before the copy runs)."""
    if a is None:
        return None
    if hasattr(a, "data_ptr") and not getattr(a, "is_cuda", False):
        import torch
        if not a.is_contiguous() or a.dtype != torch.float64:
            raise TypeError("expected a contiguous float64 host tensor")
        return C.c_void_p(a.data_ptr())
    if not isinstance(a, np.ndarray) or a.dtype != np.float64 or not a.flags["C_CONTIGUOUS"]:
        raise TypeError("expected a C-contiguous float64 numpy array")
    return C.c_void_p(a.ctypes.data)


def _stream_ptr(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def make_config(ndomains, nx, ny, nz, hx, hy, hz, bc, norb, nproj, dt, device=0, nref_max=0,
                flags=0) -> lfd_config:
    return lfd_config(LFD_ABI_VERSION, ndomains, nx, ny, nz, hx, hy, hz, bc, norb, nproj, nref_max, dt, device,
                      flags)


# ---- 1:1 wrappers of the C entry points --------------------------------------------------------

def lfd_workspace_size(cfg: lfd_config) -> int:
    n = C.c_size_t(0)
    _check(load().lfd_workspace_size(C.byref(cfg), C.byref(n)))
    return n.value


def lfd_init(cfg, psi, proj, dnl, occ, workspace, stream=None) -> C.c_void_p:
    # dnl: real [ndom][nproj], or with LFD_FLAG_DENSE_D the complex Hermitian matrices [ndom][nproj][nproj]
    pd, _k1 = _hptr(dnl, np.complex128 if cfg.flags & LFD_FLAG_DENSE_D else np.float64)
    po, _k2 = _hptr(occ)
    ctx = C.c_void_p()
    _check(load().lfd_init(C.byref(cfg), _dptr(psi), _dptr(proj), pd, po, _dptr(workspace),
                           workspace.numel() * workspace.element_size(), _stream_ptr(stream), C.byref(ctx)))
    return ctx


def lfd_set_potential(ctx, vloc):
    _check(load().lfd_set_potential(ctx, _dptr(vloc)), ctx)


def lfd_set_potential_host(ctx, vloc_host):
    """vloc_host: contiguous float64 host buffer (pinned recommended), copied asynchronously: keep it unchanged
    until lfd_sync (or double-buffer it)."""
    _check(load().lfd_set_potential_host(ctx, _hptr_async(vloc_host)), ctx)


def lfd_set_vector_potential(ctx, A):
    p, _k = _hptr(A)
    _check(load().lfd_set_vector_potential(ctx, p), ctx)


def lfd_step(ctx, nsteps: int = 1):
    _check(load().lfd_step(ctx, int(nsteps)), ctx)


def lfd_step_prologue(ctx):
    _check(load().lfd_step_prologue(ctx), ctx)


def lfd_step_sequence(ctx, A_seq):
    """A_seq: host [nsteps, ndom, 3]; nsteps steps with merged adjacent nonlocal factors."""
    arr = np.ascontiguousarray(A_seq, dtype=np.float64)
    p, _k = _hptr(arr)
    _check(load().lfd_step_sequence(ctx, int(arr.shape[0]), p), ctx)


def lfd_step_graph(ctx, A_seq, rho=None, Jmac_seq=None):
    """A_seq: host [nsteps, ndom, 3]; the steps as captured CUDA graphs (chunks of 32), optional density / J."""
    arr = np.ascontiguousarray(A_seq, dtype=np.float64)
    p, _k = _hptr(arr)
    _check(load().lfd_step_graph(ctx, int(arr.shape[0]), p, _dptr(rho), _dptr(Jmac_seq)), ctx)


def lfd_density_current(ctx, rho, j=None, Jmac=None):
    _check(load().lfd_density_current(ctx, _dptr(rho), _dptr(j), _dptr(Jmac)), ctx)


def lfd_density_current_global(ctx, rho_g, j_g, Jmac, dom_offset, gdims):
    po, _k1 = _hptr(dom_offset, np.int32)
    pg, _k2 = _hptr(gdims, np.int32)
    _check(load().lfd_density_current_global(ctx, _dptr(rho_g), _dptr(j_g), _dptr(Jmac), po, pg), ctx)


def lfd_density_current_host(ctx, rho_host=None, Jmac_host=None):
    """rho_host / Jmac_host: contiguous float64 host buffers (pinned recommended), written asynchronously: read
    them after lfd_sync or lfd_wait_host_outputs."""
    _check(load().lfd_density_current_host(ctx, _hptr_async(rho_host), _hptr_async(Jmac_host)), ctx)


def lfd_wait_host_outputs(ctx, lag=0):
    _check(load().lfd_wait_host_outputs(ctx, lag), ctx)


def lfd_energy(ctx, E):
    """E: CUDA float64 [ndom, 4] (kinetic, local, nonlocal, total)."""
    _check(load().lfd_energy(ctx, _dptr(E)), ctx)


def lfd_remap_occ(ctx, ref, occ_out):
    """ref: CUDA complex128 [ndom, nx, ny, nz, nref]; occ_out: CUDA float64 [ndom, nref]."""
    _check(load().lfd_remap_occ(ctx, _dptr(ref), int(ref.shape[-1]), _dptr(occ_out)), ctx)


def lfd_psi_modified(ctx):
    _check(load().lfd_psi_modified(ctx), ctx)


def lfd_set_occupations(ctx, occ):
    p, _k = _hptr(occ)
    _check(load().lfd_set_occupations(ctx, p), ctx)


def lfd_set_stream(ctx, stream=None):
    _check(load().lfd_set_stream(ctx, _stream_ptr(stream)), ctx)


def lfd_sync(ctx):
    _check(load().lfd_sync(ctx), ctx)


def lfd_launch_count(ctx) -> int:
    n = C.c_uint64(0)
    _check(load().lfd_launch_count(ctx, C.byref(n)), ctx)
    return n.value


def lfd_nl_path(ctx) -> int:
    """0 FP64 DMMA, 1 int8-digit tcgen05 (FP64 accuracy), 2 SP 3xTF32, -1 no nonlocal factor."""
    n = C.c_int32(0)
    _check(load().lfd_nl_path(ctx, C.byref(n)), ctx)
    return n.value


def lfd_profile_enable(ctx, enable: bool = True):
    _check(load().lfd_profile_enable(ctx, 1 if enable else 0), ctx)


def lfd_profile_read(ctx) -> dict:
    ms = (C.c_double * len(KERNELS))()
    n = (C.c_int64 * len(KERNELS))()
    _check(load().lfd_profile_read(ctx, ms, n), ctx)
    return {k: (ms[i], n[i]) for i, k in enumerate(KERNELS)}


def lfd_last_error(ctx=None) -> str:
    return load().lfd_last_error(ctx).decode()


def lfd_destroy(ctx):
    _check(load().lfd_destroy(ctx))


def make_sc_config(flags, n_corr, gdims, dom_offset, nranks=1, rank=0):
    """Returns (config, keepalive): dom_offset host int32 [ndom, 3]."""
    off = np.ascontiguousarray(dom_offset, dtype=np.int32)
    cfg = lfd_sc_config(int(flags), int(n_corr), (C.c_int32 * 3)(*[int(g) for g in gdims]), int(nranks), int(rank),
                        C.c_void_p(off.ctypes.data))
    return cfg, off


def lfd_sc_workspace_size(ctx, sccfg) -> int:
    n = C.c_size_t(0)
    _check(load().lfd_sc_workspace_size(ctx, C.byref(sccfg), C.byref(n)), ctx)
    return n.value


def lfd_sc_init(ctx, sccfg, vion, ws, Aext0, A_ind0=None, Adot0=None):
    pa, _k1 = _hptr(Aext0)
    pi, _k2 = _hptr(A_ind0)
    pd, _k3 = _hptr(Adot0)
    _check(load().lfd_sc_init(ctx, C.byref(sccfg), _dptr(vion), _dptr(ws), ws.numel() * ws.element_size(), pa, pi,
                              pd), ctx)


def lfd_sc_step(ctx, Aext):
    """Aext: host [2*nsteps+1, 3] (A_ext at t_n, t_n + dt/2, t_n+1, ...)."""
    arr = np.ascontiguousarray(Aext, dtype=np.float64).reshape(-1, 3)
    if arr.shape[0] % 2 != 1:
        raise ValueError("Aext needs 2*nsteps+1 rows")
    p, _k = _hptr(arr)
    _check(load().lfd_sc_step(ctx, int((arr.shape[0] - 1) // 2), p), ctx)


def lfd_sc_read(ctx, state=None, rho_g=None, vhxc=None):
    _check(load().lfd_sc_read(ctx, _dptr(state), _dptr(rho_g), _dptr(vhxc)), ctx)


def lfd_comm_unique_id() -> bytes:
    buf = (C.c_char * 128)()
    _check(load().lfd_comm_unique_id(buf))
    return bytes(buf)


def lfd_sc_comm_init(ctx, nranks: int, rank: int, uid: bytes):
    buf = (C.c_char * 128).from_buffer_copy(uid)
    _check(load().lfd_sc_comm_init(ctx, int(nranks), int(rank), buf), ctx)


# ---- convenience owner ---------------------------------------------------------------------------

class Context:
    """Owns the workspace and keeps psi / proj alive for the context's lifetime.

    psi: CUDA complex128 tensor [ndom, nx, ny, nz, norb] (propagated in place);
    proj: CUDA complex128 tensor [ndom, nx, ny, nz, nproj] or None; dnl [ndom, nproj]; occ [ndom, norb]
    (host arrays). h = (hx, hy, hz).
    """

    def __init__(self, psi, proj, dnl, occ, h, dt, bc=LFD_BC_PERIODIC, stream=None, nref_max=0, flags=0):
        import torch
        if psi.dtype not in (torch.complex128, torch.complex64) or psi.dim() != 5:
            raise TypeError("psi must be complex128 (or complex64: the SP variant) [ndom, nx, ny, nz, norb]")
        if proj is not None and proj.dtype != psi.dtype:
            raise TypeError("proj must have psi's dtype")
        if psi.dtype == torch.complex64:
            flags |= LFD_FLAG_SP
        ndom, nx, ny, nz, norb = psi.shape
        nproj = 0 if proj is None else proj.shape[-1]
        self.cfg = make_config(ndom, nx, ny, nz, h[0], h[1], h[2], bc, norb, nproj, dt,
                               device=psi.device.index or 0, nref_max=nref_max, flags=flags)
        self.psi, self.proj = psi, proj
        ws = lfd_workspace_size(self.cfg)
        self.workspace = torch.empty(max(ws, 1), dtype=torch.uint8, device=psi.device)
        self.ctx = lfd_init(self.cfg, psi, proj, None if nproj == 0 else dnl, occ, self.workspace, stream)
        self.shape = (ndom, nx, ny, nz)

    def set_potential(self, vloc):
        if getattr(vloc, "is_cuda", False):
            lfd_set_potential(self.ctx, vloc)
        else:
            lfd_set_potential_host(self.ctx, vloc)

    def set_vector_potential(self, A):
        lfd_set_vector_potential(self.ctx, A)

    def step(self, n: int = 1):
        lfd_step(self.ctx, n)

    def step_sequence(self, A_seq):
        lfd_step_sequence(self.ctx, A_seq)

    def density_current(self, want_j: bool = True):
        import torch
        nd, nx, ny, nz = self.shape
        dev = self.psi.device
        rho = torch.empty((nd, nx, ny, nz), dtype=torch.float64, device=dev)
        j = torch.empty((nd, 3, nx, ny, nz), dtype=torch.float64, device=dev) if want_j else None
        J = torch.empty((nd, 3), dtype=torch.float64, device=dev)
        lfd_density_current(self.ctx, rho, j, J)
        return rho, j, J

    def energy(self):
        import torch
        E = torch.empty((self.shape[0], 4), dtype=torch.float64, device=self.psi.device)
        lfd_energy(self.ctx, E)
        return E

    def remap_occ(self, ref):
        import torch
        out = torch.empty((self.shape[0], ref.shape[-1]), dtype=torch.float64, device=self.psi.device)
        lfd_remap_occ(self.ctx, ref, out)
        return out

    def sc_init(self, gdims, dom_offset, vion=None, flags=LFD_SC_HARTREE | LFD_SC_XC | LFD_SC_MAXWELL, n_corr=1,
                Aext0=(0.0, 0.0, 0.0), A_ind0=None, Adot0=None, nranks=1, rank=0, comm_id=None):
        """Self-consistent step state (lfd_sc_*). vion: CUDA float64 [ndom, nx, ny, nz] or None.
        With nranks > 1, comm_id = the 128 bytes of lfd_comm_unique_id() from one rank."""
        import torch
        if nranks > 1:
            lfd_sc_comm_init(self.ctx, nranks, rank, comm_id)
        self.sc_cfg, self._sc_off = make_sc_config(flags, n_corr, gdims, dom_offset, nranks, rank)
        n = lfd_sc_workspace_size(self.ctx, self.sc_cfg)
        self.sc_ws = torch.empty(max(n, 1), dtype=torch.uint8, device=self.psi.device)
        self.vion = vion
        lfd_sc_init(self.ctx, self.sc_cfg, vion, self.sc_ws, Aext0, A_ind0, Adot0)
        self.gdims = tuple(int(g) for g in gdims)

    def sc_step(self, Aext):
        lfd_sc_step(self.ctx, Aext)

    def sc_read(self):
        """(state [9] = A_ind, dA_ind/dt, Jbar; rho_g [GX,GY,GZ]; v_Hxc [GX,GY,GZ]) as CUDA tensors."""
        import torch
        dev = self.psi.device
        st = torch.empty(9, dtype=torch.float64, device=dev)
        rho = torch.empty(self.gdims, dtype=torch.float64, device=dev)
        v = torch.empty(self.gdims, dtype=torch.float64, device=dev)
        lfd_sc_read(self.ctx, st, rho, v)
        return st, rho, v

    def psi_modified(self):
        lfd_psi_modified(self.ctx)

    def set_occupations(self, occ):
        lfd_set_occupations(self.ctx, occ)

    def sync(self):
        lfd_sync(self.ctx)

    def close(self):
        if self.ctx is not None:
            lfd_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
