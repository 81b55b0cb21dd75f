"""Python binding of libdgr (include/dgr.h): argument marshalling only.

Every step of the hot path runs in libdgr's CUDA kernels; this module only
converts torch tensors to pointers, picks torch's current CUDA stream, and
raises DgrError on failure.  There is no CPU fallback: if libdgr.so is
missing, importing the binding's device entry points raises.

Names follow the C ABI: octree_build, Mesh (dgr_mesh_create ... destroy),
Mesh.unzip, Mesh.rhs, Mesh.rhs_patches, Mesh.rk4_stage, Mesh.rk4_step,
Mesh.constraints, Mesh.ghost_exchange.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DGR_LIB") or os.path.join(HERE, "lib", "libdgr.so")

NF = 24
NPT = 343
NPATCH = 2197

MAP_OCTANTS, MAP_O2N, MAP_HANGING, MAP_PAD_SRC, MAP_PAD_KIND, MAP_ZIP = 0, 1, 2, 3, 4, 5
MAP_DOF_GID, MAP_DOF_XYZ, MAP_SEND, MAP_SEND_COUNTS, MAP_RECV_COUNTS = 6, 7, 8, 9, 10
MAP_LOCAL_OCTS, MAP_O2N_LOCAL, MAP_RHS_ORDER, MAP_SENDBUF = 11, 12, 13, 14
OPT_FUSED_UNZIP, OPT_PHASES, OPT_PREPASS, OPT_ZIP_STORE, OPT_GRAPH = 1, 2, 3, 4, 5
OPT_FUSE_RK4 = 7


class DgrError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"libdgr status {status}: {msg}")
        self.status = status


class _Octant(C.Structure):
    _fields_ = [("x", C.c_uint32), ("y", C.c_uint32), ("z", C.c_uint32), ("level", C.c_uint32)]


class _Puncture(C.Structure):
    _fields_ = [("x", C.c_double), ("y", C.c_double), ("z", C.c_double), ("m", C.c_double),
                ("level", C.c_int32), ("pad", C.c_int32)]


class _RefineDesc(C.Structure):
    _fields_ = [("xmin", C.c_double * 3), ("width", C.c_double), ("max_depth", C.c_int32),
                ("periodic", C.c_int32), ("level_min", C.c_int32), ("n_punct", C.c_int32),
                ("punct", C.POINTER(_Puncture)), ("rho", C.c_double)]


class _MeshDesc(C.Structure):
    _fields_ = [("xmin", C.c_double * 3), ("width", C.c_double), ("max_depth", C.c_int32),
                ("periodic", C.c_int32), ("rank", C.c_int32), ("nranks", C.c_int32),
                ("device", C.c_int32), ("pad", C.c_int32), ("nccl_id", C.c_void_p)]


class _Params(C.Structure):
    _fields_ = [("ko_sigma", C.c_double), ("eta", C.c_double), ("lambda_f0", C.c_double),
                ("lambda_f1", C.c_double), ("chi_floor", C.c_double),
                ("sommerfeld", C.c_int32), ("upwind", C.c_int32)]


class _Info(C.Structure):
    _fields_ = [("n_oct_global", C.c_int64), ("n_oct_local", C.c_int64),
                ("n_oct_ghost", C.c_int64), ("oct_begin", C.c_int64),
                ("n_dof_global", C.c_int64), ("n_dof_owned", C.c_int64),
                ("n_dof_ghost", C.c_int64), ("dof_stride", C.c_int64),
                ("patch_pitch", C.c_int64), ("n_hanging", C.c_int64), ("h_min", C.c_double),
                ("level_min", C.c_int32), ("level_max", C.c_int32),
                ("n_interp_slots", C.c_int64), ("n_interp_elems", C.c_int64),
                ("n_oct_interior", C.c_int64)]


_lib = None
EXPORTED = ["dgr_status_string", "dgr_last_error", "dgr_version", "dgr_octree_build",
            "dgr_mesh_create", "dgr_mesh_info_get", "dgr_mesh_export_maps", "dgr_mesh_destroy",
            "dgr_dof_coords", "dgr_unzip", "dgr_ghost_exchange", "dgr_rhs_patches", "dgr_rhs",
            "dgr_rk4_stage", "dgr_rk4_step", "dgr_rk4_step_host", "dgr_constraints",
            "dgr_last_launch_count",
            "dgr_profile_enable", "dgr_profile_read", "dgr_bench_dfma", "dgr_set_option",
            "dgr_group_create", "dgr_group_ghost_exchange", "dgr_group_rk4_step",
            "dgr_group_destroy", "dgr_rhs_inputs", "dgr_rhs_algebra", "dgr_regrid_indicator",
            "dgr_regrid_octree", "dgr_regrid_transfer", "dgr_psi4", "dgr_psi4_sphere",
            "dgr_psi4_modes"]
PROF_CLASSES = ["elements", "hanging", "unzip", "rhs", "zip_rk4", "exchange", "constraints",
                "interp"]


def lib():
    """Load libdgr.so (built by build.py / __graft_entry__.build()); raise if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libdgr.so not built ({LIB_PATH}); run "
                              "python -m paper_conf_sc_fernandonhzsgb22_b200.build")
        L = C.CDLL(LIB_PATH)
        vp, i64, i32, dp = C.c_void_p, C.c_int64, C.c_int, C.c_double
        L.dgr_status_string.restype = C.c_char_p
        L.dgr_status_string.argtypes = [i32]
        L.dgr_last_error.restype = C.c_char_p
        L.dgr_version.restype = C.c_char_p
        L.dgr_octree_build.argtypes = [C.POINTER(_RefineDesc), vp, C.POINTER(i64)]
        L.dgr_mesh_create.argtypes = [C.POINTER(_MeshDesc), vp, i64, vp, C.POINTER(vp)]
        L.dgr_mesh_info_get.argtypes = [vp, C.POINTER(_Info)]
        L.dgr_mesh_export_maps.argtypes = [vp, i32, vp, C.POINTER(C.c_size_t)]
        L.dgr_mesh_destroy.argtypes = [vp]
        L.dgr_dof_coords.argtypes = [vp, vp, vp]
        L.dgr_unzip.argtypes = [vp, vp, vp, i32, vp]
        L.dgr_ghost_exchange.argtypes = [vp, vp, vp]
        L.dgr_rhs_patches.argtypes = [vp, vp, vp, C.POINTER(_Params), vp]
        L.dgr_rhs.argtypes = [vp, vp, vp, C.POINTER(_Params), vp]
        L.dgr_rk4_stage.argtypes = [vp, i32, dp, vp, vp, vp, C.POINTER(_Params), vp]
        L.dgr_rk4_step.argtypes = [vp, dp, vp, C.POINTER(_Params), vp]
        L.dgr_rk4_step_host.argtypes = [vp, dp, i64, C.POINTER(vp), C.POINTER(vp),
                                        C.POINTER(_Params), vp]
        L.dgr_constraints.argtypes = [vp, vp, vp, vp, C.POINTER(_Params), vp]
        L.dgr_last_launch_count.restype = i64
        L.dgr_last_launch_count.argtypes = [vp]
        L.dgr_profile_enable.argtypes = [vp, i32]
        L.dgr_profile_read.argtypes = [vp, vp, vp, i32]
        L.dgr_bench_dfma.argtypes = [i32, i32, vp, C.POINTER(dp), C.POINTER(dp)]
        L.dgr_set_option.argtypes = [vp, i32, i64]
        L.dgr_group_create.argtypes = [C.POINTER(vp), i32, C.POINTER(vp)]
        L.dgr_group_ghost_exchange.argtypes = [vp, C.POINTER(vp), C.POINTER(vp)]
        L.dgr_group_rk4_step.argtypes = [vp, dp, C.POINTER(vp), C.POINTER(_Params), C.POINTER(vp)]
        L.dgr_group_destroy.argtypes = [vp]
        L.dgr_rhs_inputs.argtypes = [vp, vp, vp, i64, C.POINTER(_Params), vp]
        L.dgr_rhs_algebra.argtypes = [i32, i32, vp, vp, i64, i64, C.POINTER(_Params), vp]
        L.dgr_regrid_indicator.argtypes = [vp, vp, C.c_uint32, vp, vp]
        L.dgr_regrid_octree.argtypes = [vp, vp, dp, dp, i32, i32, vp, C.POINTER(i64)]
        L.dgr_regrid_transfer.argtypes = [vp, vp, vp, vp, vp]
        L.dgr_psi4.argtypes = [vp, vp, vp, vp, C.POINTER(_Params), vp]
        L.dgr_psi4_sphere.argtypes = [vp, vp, i64, vp, vp, vp]
        L.dgr_psi4_modes.argtypes = [vp, vp, vp, dp, i32, i32, i32, vp, vp, C.POINTER(_Params), vp]
        for f in ["dgr_octree_build", "dgr_mesh_create", "dgr_mesh_info_get",
                  "dgr_mesh_export_maps", "dgr_mesh_destroy", "dgr_dof_coords", "dgr_unzip",
                  "dgr_ghost_exchange", "dgr_rhs_patches", "dgr_rhs", "dgr_rk4_stage",
                  "dgr_rk4_step", "dgr_rk4_step_host", "dgr_constraints", "dgr_profile_enable", "dgr_profile_read", "dgr_set_option",
                  "dgr_bench_dfma", "dgr_group_create", "dgr_group_ghost_exchange",
                  "dgr_group_rk4_step", "dgr_group_destroy", "dgr_rhs_inputs",
                  "dgr_rhs_algebra", "dgr_regrid_indicator", "dgr_regrid_octree",
                  "dgr_regrid_transfer", "dgr_psi4", "dgr_psi4_sphere", "dgr_psi4_modes"]:
            getattr(L, f).restype = i32
        _lib = L
    return _lib


def _check(st):
    if st != 0:
        L = lib()
        raise DgrError(st, L.dgr_last_error().decode())


@dataclass
class Params:
    """RHS parameters (readings R6, R8, R13)."""
    ko_sigma: float = 0.4
    eta: float = 2.0
    lambda_f0: float = 1.0
    lambda_f1: float = 0.0
    chi_floor: float = 1e-4
    sommerfeld: int = 0   # 1: radiative outer boundary (reading R29)
    upwind: int = 0       # 1: lopsided advective derivatives (reading R9u)

    def _c(self):
        return _Params(self.ko_sigma, self.eta, self.lambda_f0, self.lambda_f1, self.chi_floor,
                       int(self.sommerfeld), int(self.upwind))


def octree_build(cfg) -> np.ndarray:
    """dgr_octree_build for a synth.configs.MeshConfig -> uint32 [n, 4] (x, y, z, level)."""
    L = lib()
    P = (_Puncture * max(1, len(cfg.punctures)))()
    for i, p in enumerate(cfg.punctures):
        P[i] = _Puncture(p.x, p.y, p.z, p.m, p.level, 0)
    d = _RefineDesc((C.c_double * 3)(*cfg.xmin), cfg.width, cfg.max_depth, int(cfg.periodic),
                    cfg.level_min, len(cfg.punctures), P, cfg.rho)
    n = C.c_int64(0)
    _check(L.dgr_octree_build(C.byref(d), None, C.byref(n)))
    out = np.zeros((n.value, 4), dtype=np.uint32)
    _check(L.dgr_octree_build(C.byref(d), out.ctypes.data, C.byref(n)))
    return out


def _ptr(t):
    return C.c_void_p(t.data_ptr())


def _dev(t, shape, what):
    """Validate a device tensor handed to libdgr (the kernels trust their sizes):
    CUDA, float64, contiguous, and at least `shape` (leading dims exact)."""
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{what}: expected a torch tensor")
    if t.device.type != "cuda" or t.dtype != torch.float64 or not t.is_contiguous():
        raise ValueError(f"{what}: must be a contiguous float64 CUDA tensor "
                         f"(got {t.dtype} on {t.device}, contiguous={t.is_contiguous()})")
    if t.dim() != len(shape) or any(a != b for a, b in zip(t.shape, shape)):
        raise ValueError(f"{what}: shape {tuple(t.shape)}, expected {tuple(shape)}")
    return _ptr(t)


def _stream():
    import torch
    if not torch.cuda.is_available():   # (host-only meshes: the library refuses device calls)
        return C.c_void_p(None)
    return C.c_void_p(torch.cuda.current_stream().cuda_stream)


class Mesh:
    """A dgr_mesh handle.  device=False builds host maps only (map export works
    without a GPU); device=True uploads maps and allocates workspace."""

    def __init__(self, cfg, octants=None, device=True, rank=0, nranks=1, nccl_id=None):
        L = lib()
        if octants is None:
            octants = octree_build(cfg)
        self.octants = np.ascontiguousarray(octants, dtype=np.uint32)
        self.cfg = cfg
        idbuf = None
        if nccl_id is not None:
            idbuf = C.create_string_buffer(bytes(nccl_id), 128)
        d = _MeshDesc((C.c_double * 3)(*cfg.xmin), cfg.width, cfg.max_depth, int(cfg.periodic),
                      rank, nranks, int(device), 0,
                      C.cast(idbuf, C.c_void_p) if idbuf is not None else None)
        h = C.c_void_p()
        stream = _stream() if device else None
        _check(L.dgr_mesh_create(C.byref(d), self.octants.ctypes.data, len(self.octants), stream,
                                 C.byref(h)))
        self._h = h
        self.device = device
        info = _Info()
        _check(L.dgr_mesh_info_get(h, C.byref(info)))
        self.info = {k: getattr(info, k) for k, _ in _Info._fields_}

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.dgr_mesh_destroy(h)
            self._h = None

    close = __del__

    # ------------------------------------------------------------ host maps
    def export(self, which, dtype):
        L = lib()
        n = C.c_size_t(0)
        _check(L.dgr_mesh_export_maps(self._h, which, None, C.byref(n)))
        out = np.empty(n.value // np.dtype(dtype).itemsize, dtype=dtype)
        if n.value:
            _check(L.dgr_mesh_export_maps(self._h, which, out.ctypes.data, C.byref(n)))
        return out

    def maps(self):
        no = self.info["n_oct_local"]
        return dict(
            octants=self.export(MAP_OCTANTS, np.int32).reshape(-1, 4),
            o2n=self.export(MAP_O2N, np.int32).reshape(no, NPT),
            hanging=self.export(MAP_HANGING, np.int32).reshape(-1, 3),
            pad_src=self.export(MAP_PAD_SRC, np.int32).reshape(no, NPATCH),
            pad_kind=self.export(MAP_PAD_KIND, np.uint8).reshape(no, NPATCH),
            zip=self.export(MAP_ZIP, np.int32).reshape(-1, 2),
            dof_gid=self.export(MAP_DOF_GID, np.int64),
        )

    def dof_xyz_host(self):
        return self.export(MAP_DOF_XYZ, np.float64).reshape(3, -1)

    @property
    def dof_stride(self):
        return self.info["dof_stride"]

    @property
    def n_dof(self):
        return self.info["n_dof_owned"] + self.info["n_dof_ghost"]

    # -------------------------------------------------------- device calls
    def _state(self, t, what):
        return _dev(t, (NF, self.dof_stride), what)

    def new_state(self, dtype=None):
        import torch
        return torch.zeros((NF, self.dof_stride), dtype=torch.float64, device="cuda")

    def dof_coords(self):
        import torch
        xyz = torch.empty((3, self.dof_stride), dtype=torch.float64, device="cuda")
        _check(lib().dgr_dof_coords(self._h, _dev(xyz, (3, self.dof_stride), "xyz"), _stream()))
        return xyz

    def unzip(self, u, nfields=NF, patches=None):
        import torch
        if patches is None:
            patches = torch.empty((nfields, self.info["n_oct_local"], self.info["patch_pitch"]),
                                  dtype=torch.float64, device="cuda")
        _check(lib().dgr_unzip(self._h, self._state(u, "u"),
                               _dev(patches, (nfields, self.info["n_oct_local"],
                                              self.info["patch_pitch"]), "patches"),
                               nfields, _stream()))
        return patches

    def rhs_patches(self, patches, prm=None, out=None):
        import torch
        if out is None:
            out = torch.empty((NF, self.info["n_oct_local"], NPT), dtype=torch.float64,
                              device="cuda")
        p = (prm or Params())._c()
        no, pp = self.info["n_oct_local"], self.info["patch_pitch"]
        _check(lib().dgr_rhs_patches(self._h, _dev(patches, (NF, no, pp), "patches"),
                                     _dev(out, (NF, no, NPT), "out"), C.byref(p), _stream()))
        return out

    def ghost_exchange(self, u):
        _check(lib().dgr_ghost_exchange(self._h, self._state(u, "u"), _stream()))

    def rhs(self, u, prm=None, out=None):
        import torch
        if out is None:
            out = torch.zeros_like(u)
        p = (prm or Params())._c()
        _check(lib().dgr_rhs(self._h, self._state(u, "u"), self._state(out, "out"), C.byref(p),
                             _stream()))
        return out

    def rk4_stage(self, s, dt, u_n, u_s, acc, prm=None):
        p = (prm or Params())._c()
        _check(lib().dgr_rk4_stage(self._h, s, float(dt), self._state(u_n, "u_n"),
                                   self._state(u_s, "u_s"), self._state(acc, "acc"),
                                   C.byref(p), _stream()))

    def rk4_step(self, u, dt, prm=None):
        p = (prm or Params())._c()
        _check(lib().dgr_rk4_step(self._h, float(dt), self._state(u, "u"), C.byref(p), _stream()))
        return u

    def rk4_step_host(self, u_in, u_out, dt, prm=None):
        """One RK4 step of each host state: u_out[j] = step(u_in[j]) (dgr_rk4_step_host).
        u_in / u_out: lists of contiguous fp64 CPU tensors [24, dof_stride], pinned
        for copy/compute overlap.  Enqueued on the current stream; the tensors must
        stay alive until it completes."""
        import torch
        if len(u_in) != len(u_out):
            raise ValueError("u_in and u_out differ in length")
        for t in list(u_in) + list(u_out):
            if (t.device.type != "cpu" or not t.is_contiguous() or t.dtype != torch.float64
                    or tuple(t.shape) != (24, self.dof_stride)):
                raise ValueError("host states must be contiguous fp64 CPU [24, dof_stride]")
        n = len(u_in)
        ins = (C.c_void_p * max(n, 1))(*[t.data_ptr() for t in u_in])
        outs = (C.c_void_p * max(n, 1))(*[t.data_ptr() for t in u_out])
        p = (prm or Params())._c()
        _check(lib().dgr_rk4_step_host(self._h, float(dt), n, ins, outs, C.byref(p), _stream()))
        return u_out

    def constraints(self, u, prm=None, out=None):
        import torch
        if out is None:
            out = torch.zeros((7, self.dof_stride), dtype=torch.float64, device="cuda")
        norms = np.zeros(14)
        p = (prm or Params())._c()
        _check(lib().dgr_constraints(self._h, self._state(u, "u"),
                                     _dev(out, (7, self.dof_stride), "out"), norms.ctypes.data,
                                     C.byref(p), _stream()))
        return out, norms.reshape(7, 2)

    def rhs_inputs(self, u, prm=None, out=None):
        """dgr_rhs_inputs: the 234 inputs of the RHS algebra at every interior point
        of the owned octants, [234, n_oct_local * 343] (codegen/bssn_sym.py order)."""
        import torch
        n = self.info["n_oct_local"] * NPT
        if out is None:
            out = torch.empty((N_ALG_IN, n), dtype=torch.float64, device="cuda")
        _dev(out, (N_ALG_IN, out.shape[1]), "out")
        p = (prm or Params())._c()
        _check(lib().dgr_rhs_inputs(self._h, self._state(u, "u"), _ptr(out), out.shape[1],
                                    C.byref(p), _stream()))
        return out

    # ------------------------------------------------------------ regrid
    def regrid_indicator(self, u, field_mask=0xFFFFFF, out=None):
        """dgr_regrid_indicator: wavelet indicator per owned octant (device tensor)."""
        import torch
        n = self.info["n_oct_local"]
        if out is None:
            out = torch.empty(n, dtype=torch.float64, device="cuda")
        _check(lib().dgr_regrid_indicator(self._h, self._state(u, "u"), int(field_mask),
                                          _dev(out, (n,), "out"), _stream()))
        return out

    def regrid_octree(self, w, eps_refine, eps_coarsen, level_min, level_max):
        """dgr_regrid_octree (host): the regridded leaves, uint32 [n, 4]."""
        w = np.ascontiguousarray(np.asarray(w, dtype=np.float64))
        if w.shape != (self.info["n_oct_global"],):
            raise ValueError("w: one value per global octant")
        n = C.c_int64(0)
        args = (float(eps_refine), float(eps_coarsen), int(level_min), int(level_max))
        _check(lib().dgr_regrid_octree(self._h, w.ctypes.data, *args, None, C.byref(n)))
        out = np.zeros((n.value, 4), dtype=np.uint32)
        _check(lib().dgr_regrid_octree(self._h, w.ctypes.data, *args, out.ctypes.data,
                                       C.byref(n)))
        return out

    def regrid_transfer(self, u, new_mesh, out=None):
        """dgr_regrid_transfer: the state on new_mesh interpolated from u on this mesh."""
        if out is None:
            out = new_mesh.new_state()
        _check(lib().dgr_regrid_transfer(self._h, self._state(u, "u"), new_mesh._h,
                                         new_mesh._state(out, "out"), _stream()))
        return out

    # ------------------------------------------------- gravitational waves
    def psi4(self, u, center=(0.0, 0.0, 0.0), prm=None, out=None):
        """dgr_psi4: Psi_4 (Re, Im) at every node of every owned octant,
        [2, n_oct_local * 343] device tensor (column e * 343 + node)."""
        import torch
        n = self.info["n_oct_local"] * NPT
        if out is None:
            out = torch.empty((2, n), dtype=torch.float64, device="cuda")
        c = (C.c_double * 3)(*center)
        p = (prm or Params())._c()
        _check(lib().dgr_psi4(self._h, self._state(u, "u"), c, _dev(out, (2, n), "out"),
                              C.byref(p), _stream()))
        return out

    def psi4_sphere(self, psi, xyz):
        """dgr_psi4_sphere: psi (from psi4()) at host points xyz [3, n] -> [2, n]."""
        xyz = np.ascontiguousarray(np.asarray(xyz, dtype=np.float64))
        n = xyz.shape[1]
        out = np.zeros((2, n))
        _check(lib().dgr_psi4_sphere(self._h, _dev(psi, (2, psi.shape[1]), "psi"), n,
                                     xyz.ctypes.data, out.ctypes.data, _stream()))
        return out

    def psi4_modes(self, u, center=(0.0, 0.0, 0.0), radius=50.0, n_theta=16, n_phi=32,
                   l_max=4, prm=None):
        """dgr_psi4_modes: {(l, m): C_lm} on a sphere (and the sphere values [2, n])."""
        nm = sum(2 * l + 1 for l in range(2, l_max + 1))
        modes = np.zeros(2 * nm)
        sph = np.zeros((2, n_theta * n_phi))
        c = (C.c_double * 3)(*center)
        p = (prm or Params())._c()
        _check(lib().dgr_psi4_modes(self._h, self._state(u, "u"), c, float(radius), int(n_theta),
                                    int(n_phi), int(l_max), modes.ctypes.data, sph.ctypes.data,
                                    C.byref(p), _stream()))
        out, q = {}, 0
        for l in range(2, l_max + 1):
            for m in range(-l, l + 1):
                out[(l, m)] = complex(modes[2 * q], modes[2 * q + 1])
                q += 1
        return out, sph

    def last_launch_count(self):
        return int(lib().dgr_last_launch_count(self._h))

    def set_fused(self, on=True):
        """DGR_OPT_FUSED_UNZIP: gather patches inside the RHS kernel (1) or unzip into
        the patch buffer first (0); bit-identical results."""
        _check(lib().dgr_set_option(self._h, OPT_FUSED_UNZIP, int(bool(on))))

    def set_prepass(self, on=True):
        """DGR_OPT_PREPASS: gt_ij stages in the metric pre-pass kernel (1) or in the
        RHS kernel (0); bit-identical results."""
        _check(lib().dgr_set_option(self._h, OPT_PREPASS, int(bool(on))))

    def set_zip_store(self, on=True):
        """DGR_OPT_ZIP_STORE: zip in the RHS kernel's store and stream the RK4 update
        (1) or write the RHS per octant point and zip-gather it (0); bit-identical."""
        _check(lib().dgr_set_option(self._h, OPT_ZIP_STORE, int(bool(on))))

    def set_graph(self, on=True):
        """DGR_OPT_GRAPH: rk4_step replays a CUDA graph of its four stages (captured
        at the second call with the same arguments); bit-identical to eager."""
        _check(lib().dgr_set_option(self._h, OPT_GRAPH, int(bool(on))))

    def set_fuse_rk4(self, on=True):
        """DGR_OPT_FUSE_RK4: rk4_step / rk4_step_host apply the RK4 stage update in the
        RHS kernel's epilogue (1) or in a separate streaming kernel (0); bit-identical."""
        _check(lib().dgr_set_option(self._h, OPT_FUSE_RK4, int(bool(on))))

    def set_phases(self, mode=0):
        """DGR_OPT_PHASES: 0 = overlap interior octants with the ghost exchange when
        there is a communicator; 1 = interior octants first, then the rest;
        2 = interior octants only (test hook)."""
        _check(lib().dgr_set_option(self._h, OPT_PHASES, int(mode)))

    def rhs_order(self):
        """Owned octants (local ids) in RHS order; the first info['n_oct_interior']
        need no ghost value."""
        return self.export(MAP_RHS_ORDER, np.int32)

    def profile_enable(self, on=True):
        _check(lib().dgr_profile_enable(self._h, int(on)))

    def profile_read(self, reset=True):
        """{class: (ms, launches)} of libdgr kernels since the last reset (CUDA events)."""
        ms = np.zeros(8)
        n = np.zeros(8, dtype=np.int64)
        _check(lib().dgr_profile_read(self._h, ms.ctypes.data, n.ctypes.data, int(reset)))
        return {PROF_CLASSES[i]: (float(ms[i]), int(n[i])) for i in range(8) if n[i]}


N_ALG_IN = 234
ALG_VARIANTS = ["sympygr_cse", "binary_reduce", "staged_cse"]


def rhs_algebra(variant, inp, prm=None, occ=False, out=None):
    """dgr_rhs_algebra: the generated A kernel `variant` (name or 0..2) on
    inp [234, n] -> [24, n] (algebra + KO)."""
    import torch
    v = ALG_VARIANTS.index(variant) if isinstance(variant, str) else int(variant)
    n = inp.shape[1]
    _dev(inp, (N_ALG_IN, n), "inp")
    if out is None:
        out = torch.empty((NF, n), dtype=torch.float64, device="cuda")
    _dev(out, (NF, n), "out")
    p = (prm or Params())._c()
    _check(lib().dgr_rhs_algebra(v, int(bool(occ)), _ptr(inp), _ptr(out), n, n, C.byref(p),
                                 _stream()))
    return out


class Group:
    """dgr_group: rank-meshes [rank 0 .. n-1] of one octree driven by this process
    (external-exchange meshes, nccl_id=None); libdgr does their ghost exchange
    (pack kernel, peer copies, unpack kernel).  Destroy (close) before the meshes."""

    def __init__(self, meshes):
        L = lib()
        self.meshes = list(meshes)
        hs = (C.c_void_p * len(self.meshes))(*[m._h.value for m in self.meshes])
        g = C.c_void_p()
        _check(L.dgr_group_create(hs, len(self.meshes), C.byref(g)))
        self._g = g

    def _lists(self, states, streams):
        n = len(self.meshes)
        if len(states) != n:
            raise ValueError("one state per rank")
        us = (C.c_void_p * n)(*[m._state(u, f"u[{r}]").value
                                for r, (m, u) in enumerate(zip(self.meshes, states))])
        if streams is None:
            streams = [_stream().value] * n
        ss = (C.c_void_p * n)(*streams)
        return us, ss

    def ghost_exchange(self, states, streams=None):
        us, ss = self._lists(states, streams)
        _check(lib().dgr_group_ghost_exchange(self._g, us, ss))

    def rk4_step(self, states, dt, prm=None, streams=None):
        us, ss = self._lists(states, streams)
        p = (prm or Params())._c()
        _check(lib().dgr_group_rk4_step(self._g, float(dt), us, C.byref(p), ss))
        return states

    def close(self):
        g = getattr(self, "_g", None)
        if g is not None and g.value and _lib is not None:
            _lib.dgr_group_destroy(g)
            self._g = None

    __del__ = close


def bench_dfma(blocks=148 * 8, iters=200000):
    """(ms, flops) of the fp64 FMA microbenchmark on the current device."""
    ms, fl = C.c_double(), C.c_double()
    _check(lib().dgr_bench_dfma(blocks, iters, _stream(), C.byref(ms), C.byref(fl)))
    return ms.value, fl.value
