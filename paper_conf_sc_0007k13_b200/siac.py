"""Thin Python binding of libsiac_b200.so (include/siac.h) -- argument marshalling only.

Every step of the path runs in the CUDA library; there is no CPU fallback.  If the shared
library is missing or fails to load, importing this module's functions raises.

    ctx = siac.create(V, T, C, k=3, h=0.01)          # siac_create
    vals = ctx.eval(points)                           # siac_eval (host buffers)
    ctx.eval_async(d_points, d_out, stream)           # siac_eval_async (device pointers / tensors)
    ctx.set_counting(True); ctx.stats()               # siac_set_counting / siac_stats
    ctx.destroy()                                     # siac_destroy
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsiac_b200.so")
# experiments only: SIAC_LIB_VARIANT=name loads libsiac_b200.<name>.so (built by tools/build_variant.py)
if os.environ.get("SIAC_LIB_VARIANT"):
    LIB_PATH = os.path.join(_HERE, f"libsiac_b200.{os.environ['SIAC_LIB_VARIANT']}.so")
SOURCES = [os.path.join(_HERE, "csrc", f) for f in (
    "siac.cu", "siac_eval_k.cu", "siac_internal.h", "siac_device.cuh", "siac_tile.cuh", "siac_ws.cuh",
    "siac_clipfast.cuh", "siac_jump.cuh", "siac_math.cpp", "siac_math.h", "siac_quadrature.h", "siac_io.cu",
    "siac3d.cu")]
SOURCES.append(os.path.join(os.path.dirname(_HERE), "include", "siac.h"))

NVCC_FLAGS = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
              "-Xcompiler", "-fPIC"]

SIAC_PERIODIC_X = 1
SIAC_PERIODIC_Y = 2
SIAC_BASIS_DUBINER_ORTHONORMAL = 0
SIAC_BASIS_MONOMIAL_REF = 1
SIAC_BOUNDARY_ZERO = 0
SIAC_BOUNDARY_ONESIDED = 1


def build(force: bool = False, verbose: bool = False, extra_flags=(), out_path: str | None = None) -> str:
    """Compile the CUDA library for sm_100a into paper_conf_sc_0007k13_b200/libsiac_b200.so.

    Translation units: csrc/siac.cu (C ABI, create/eval orchestration, small kernels),
    csrc/siac_eval_k.cu once per degree k = 1..4 and schedule part p = 0..3 (-DSIAC_K=k
    -DSIAC_PART=p; the evaluation kernels), and csrc/siac_math.cpp (host exact constants, g++).
    Objects live in csrc/build/<lib name>/ and are rebuilt only when their sources (or the
    flags) change; the compiles run in parallel on the available cores."""
    lib_path = out_path or LIB_PATH
    nvcc = os.environ.get("NVCC", "nvcc")
    tag = os.path.basename(lib_path).replace(".so", "")
    objdir = os.path.join(_HERE, "csrc", "build", tag)
    os.makedirs(objdir, exist_ok=True)
    flags = NVCC_FLAGS + list(extra_flags) + (["-Xptxas", "-v"] if verbose else [])
    cs = lambda *f: [os.path.join(_HERE, "csrc", x) for x in f]
    common = cs("siac_internal.h", "siac_device.cuh", "siac_quadrature.h") + [SOURCES[-1]]
    part_deps = {0: cs("siac_jump.cuh"), 1: [], 2: cs("siac_tile.cuh", "siac_clipfast.cuh"), 3: cs("siac_ws.cuh")}
    jobs = [(["g++", "-O2", "-std=c++17", "-fPIC", "-c", "-o", os.path.join(objdir, "siac_math.o")] + cs("siac_math.cpp"),
             os.path.join(objdir, "siac_math.o"), cs("siac_math.cpp", "siac_math.h"))]
    jobs.append(([nvcc] + flags + ["-c", "-o", os.path.join(objdir, "siac_io.o")] + cs("siac_io.cu"),
                 os.path.join(objdir, "siac_io.o"), cs("siac_io.cu", "siac_internal.h", "siac_math.h") + [SOURCES[-1]]))
    jobs.append(([nvcc] + flags + ["-c", "-o", os.path.join(objdir, "siac3d.o")] + cs("siac3d.cu"),
                 os.path.join(objdir, "siac3d.o"), cs("siac3d.cu", "siac_internal.h", "siac_math.h") + [SOURCES[-1]]))
    jobs.append(([nvcc] + flags + ["-c", "-o", os.path.join(objdir, "siac.o")] + cs("siac.cu"),
                 os.path.join(objdir, "siac.o"), cs("siac.cu", "siac_jump.cuh", "siac_math.h") + common))
    for k in (1, 2, 3, 4):
        for part in (0, 1, 2, 3):
            o = os.path.join(objdir, f"siac_eval_k{k}_p{part}.o")
            jobs.append(([nvcc] + flags + [f"-DSIAC_K={k}", f"-DSIAC_PART={part}", "-c", "-o", o] + cs("siac_eval_k.cu"),
                         o, cs("siac_eval_k.cu") + common + part_deps[part]))
    flag_file = os.path.join(objdir, "flags.txt")
    same_flags = os.path.exists(flag_file) and open(flag_file).read() == " ".join(flags)

    def stale(o, deps):
        return force or not same_flags or not os.path.exists(o) or any(
            os.path.getmtime(o) < os.path.getmtime(d) for d in deps)
    todo = [(cmd, o) for cmd, o, deps in jobs if stale(o, deps)]
    if not todo and os.path.exists(lib_path) and all(os.path.getmtime(lib_path) >= os.path.getmtime(o) for _, o, _ in jobs):
        return lib_path
    running, failed = [], []
    ncpu = max(1, len(os.sched_getaffinity(0)))

    def reap(p, c):
        out, _ = p.communicate()
        if p.returncode:
            failed.append((c, out))
        elif verbose and out:
            print(out)
    for cmd, o in todo:
        while len(running) >= ncpu:
            reap(*running.pop(0))
        running.append((subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True), cmd))
    for p, c in running:
        reap(p, c)
    if failed:
        raise RuntimeError("build failed:\n" + "\n".join(" ".join(c) + "\n" + o for c, o in failed))
    with open(flag_file, "w") as f:
        f.write(" ".join(flags))
    subprocess.check_call([nvcc, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", lib_path + ".tmp"]
                          + [o for _, o, _ in jobs])
    os.replace(lib_path + ".tmp", lib_path)
    return lib_path


class SiacError(RuntimeError):
    pass


class _Params(ctypes.Structure):
    _fields_ = [("k", ctypes.c_int32), ("h", ctypes.c_double), ("periodic", ctypes.c_int32),
                ("domain", ctypes.c_double * 4), ("device", ctypes.c_int32), ("cell_factor", ctypes.c_double),
                ("basis", ctypes.c_int32), ("boundary", ctypes.c_int32)]


class _CreateInfo(ctypes.Structure):
    _fields_ = [("total_ms", ctypes.c_double), ("host_ms", ctypes.c_double), ("h2d_ms", ctypes.c_double),
                ("index_ms", ctypes.c_double), ("jump_ms", ctypes.c_double), ("cross_ms", ctypes.c_double),
                ("device_bytes", ctypes.c_int64), ("bytes_per_triangle", ctypes.c_int64)]


class _Params3(ctypes.Structure):
    _fields_ = [("k", ctypes.c_int32), ("h", ctypes.c_double), ("periodic", ctypes.c_int32),
                ("domain", ctypes.c_double * 6), ("device", ctypes.c_int32)]


class _Counters(ctypes.Structure):
    _fields_ = [("n_points", ctypes.c_int64), ("candidates", ctypes.c_int64), ("pairs", ctypes.c_int64),
                ("pieces", ctypes.c_int64), ("subtris", ctypes.c_int64), ("corner_terms", ctypes.c_int64),
                ("cross_terms", ctypes.c_int64), ("cross_subtris", ctypes.c_int64), ("cross_polys", ctypes.c_int64)]


_lib = None


def lib():
    """Load libsiac_b200.so (raises if it is missing: no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        vp, D, I64, I32 = ctypes.c_void_p, ctypes.POINTER(ctypes.c_double), ctypes.c_int64, ctypes.c_int32
        L.siac_create.restype = ctypes.c_int
        L.siac_create.argtypes = [ctypes.POINTER(vp), D, I64, ctypes.POINTER(ctypes.c_int32), I64, D,
                                  ctypes.POINTER(_Params)]
        L.siac_eval.restype = ctypes.c_int
        L.siac_eval.argtypes = [vp, D, I64, D]
        L.siac_eval_async.restype = ctypes.c_int
        L.siac_eval_async.argtypes = [vp, vp, I64, vp, vp]
        L.siac_set_counting.restype = ctypes.c_int
        L.siac_set_counting.argtypes = [vp, I32]
        L.siac_stats.restype = ctypes.c_int
        L.siac_stats.argtypes = [vp, ctypes.POINTER(_Counters)]
        L.siac_get_create_info.restype = ctypes.c_int
        L.siac_get_create_info.argtypes = [vp, ctypes.POINTER(_CreateInfo)]
        L.siac_set_schedule.restype = ctypes.c_int
        L.siac_set_schedule.argtypes = [vp, I32]
        L.siac_set_graphs.restype = ctypes.c_int
        L.siac_set_graphs.argtypes = [vp, I32]
        L.siac_set_timing.restype = ctypes.c_int
        L.siac_set_timing.argtypes = [vp, I32]
        L.siac_timing.restype = ctypes.c_int
        L.siac_timing.argtypes = [vp, D, ctypes.POINTER(I64)]
        L.siac_probe_fp64.restype = ctypes.c_int
        L.siac_probe_fp64.argtypes = [I32, D]
        L.siac_info.restype = ctypes.c_int
        L.siac_info.argtypes = [vp, ctypes.POINTER(I64), ctypes.POINTER(I32), ctypes.POINTER(I32),
                                D, D]
        L.siac_host_tables.restype = ctypes.c_int
        L.siac_host_tables.argtypes = [I32, D, D]
        L.siac_debug_records.restype = ctypes.c_int
        L.siac_debug_records.argtypes = [vp, I32, I64, D, ctypes.POINTER(I32)]
        L.siac_destroy.restype = None
        L.siac_destroy.argtypes = [vp]
        L.siac_last_error.restype = ctypes.c_char_p
        L.siac_last_error.argtypes = [vp]
        L.siac_version.restype = ctypes.c_char_p
        L.siac_version.argtypes = []
        L.siac_projection_rule.restype = ctypes.c_int
        L.siac_projection_rule.argtypes = [I32, D, D]
        L.siac_map_points_async.restype = ctypes.c_int
        L.siac_map_points_async.argtypes = [vp, vp, I64, vp, I32, vp, vp]
        L.siac_project_async.restype = ctypes.c_int
        L.siac_project_async.argtypes = [I32, I32, vp, I64, vp, vp]
        L.siac_error_norms_async.restype = ctypes.c_int
        L.siac_error_norms_async.argtypes = [vp, vp, vp, I64, vp, vp]
        L.siac3_create.restype = ctypes.c_int
        L.siac3_create.argtypes = [ctypes.POINTER(vp), D, I64, ctypes.POINTER(ctypes.c_int32), I64, D,
                                   ctypes.POINTER(_Params3)]
        L.siac3_eval.restype = ctypes.c_int
        L.siac3_eval.argtypes = [vp, D, I64, D]
        L.siac3_eval_async.restype = ctypes.c_int
        L.siac3_eval_async.argtypes = [vp, vp, I64, vp, vp]
        L.siac3_set_schedule.restype = ctypes.c_int
        L.siac3_set_schedule.argtypes = [vp, I32]
        L.siac3_set_counting.restype = ctypes.c_int
        L.siac3_set_counting.argtypes = [vp, I32]
        L.siac3_stats.restype = ctypes.c_int
        L.siac3_stats.argtypes = [vp, ctypes.POINTER(I64), ctypes.POINTER(I64)]
        L.siac3_tet_rule.restype = ctypes.c_int
        L.siac3_tet_rule.argtypes = [I32, D]
        L.siac3_destroy.restype = None
        L.siac3_destroy.argtypes = [vp]
        L.siac3_last_error.restype = ctypes.c_char_p
        L.siac3_last_error.argtypes = [vp]
        _lib = L
    return _lib


EXPORTED = ["siac_create", "siac_eval", "siac_eval_async", "siac_set_counting", "siac_stats", "siac_get_create_info",
            "siac_set_schedule", "siac_set_graphs", "siac_set_timing", "siac_timing", "siac_probe_fp64",
            "siac_info", "siac_host_tables", "siac_debug_records",
            "siac_destroy", "siac_last_error", "siac_version",
            "siac_projection_rule", "siac_map_points_async", "siac_project_async", "siac_error_norms_async",
            "siac3_create", "siac3_eval", "siac3_eval_async", "siac3_set_schedule", "siac3_set_counting", "siac3_stats", "siac3_tet_rule",
            "siac3_destroy", "siac3_last_error"]


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _check(rc, ctx_ptr=None):
    if rc != 0:
        msg = lib().siac_last_error(ctx_ptr).decode()
        raise SiacError(f"siac error {rc}: {msg}")


class Context:
    """A siac_ctx: device-resident mesh + spatial index."""

    def __init__(self, V, T, C, k: int, h: float, periodic: int = 3, domain=(0.0, 0.0, 1.0, 1.0),
                 device: int = 0, cell_factor: float = 0.0, basis: int = 0, boundary: int = 0):
        L = lib()
        self._V = np.ascontiguousarray(V, dtype=np.float64).reshape(-1, 2)
        self._T = np.ascontiguousarray(T, dtype=np.int32).reshape(-1, 3)
        self._C = np.ascontiguousarray(C, dtype=np.float64)
        if 1 <= k <= 4 and self._C.size != len(self._T) * (k + 1) * (k + 2) // 2:   # (k itself: checked in C)
            raise ValueError(f"coeffs must have (k+1)(k+2)/2 = {(k + 1) * (k + 2) // 2} columns")
        p = _Params(int(k), float(h), int(periodic), (ctypes.c_double * 4)(*domain), int(device), float(cell_factor),
                    int(basis), int(boundary))
        ptr = ctypes.c_void_p()
        rc = L.siac_create(ctypes.byref(ptr), _dp(self._V), len(self._V),
                           self._T.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), len(self._T),
                           _dp(self._C), ctypes.byref(p))
        _check(rc, None)
        self._ptr = ptr
        self.k, self.h, self.periodic, self.domain, self.device = int(k), float(h), int(periodic), tuple(domain), device
        del self._V, self._T, self._C     # siac_create deep-copied them

    def eval(self, points) -> np.ndarray:
        """siac_eval: host points (n,2) -> host values (n,), H2D/D2H inside."""
        P = np.ascontiguousarray(points, dtype=np.float64).reshape(-1, 2)
        out = np.empty(len(P), dtype=np.float64)
        _check(lib().siac_eval(self._ptr, _dp(P), len(P), _dp(out)), self._ptr)
        return out

    def eval_into(self, points: np.ndarray, out: np.ndarray) -> None:
        """siac_eval into caller-owned host arrays (e.g. pinned torch tensors' numpy views).
        points: float64, C-contiguous, shape (n, 2); out: float64, C-contiguous, >= n values."""
        if not (isinstance(points, np.ndarray) and points.dtype == np.float64 and points.flags.c_contiguous
                and points.ndim == 2 and points.shape[1] == 2):
            raise ValueError("points must be a C-contiguous float64 array of shape (n, 2)")
        if not (isinstance(out, np.ndarray) and out.dtype == np.float64 and out.flags.c_contiguous
                and out.size >= len(points)):
            raise ValueError("out must be a C-contiguous float64 array with at least n values")
        _check(lib().siac_eval(self._ptr, _dp(points), len(points), _dp(out)), self._ptr)

    def eval_async(self, d_points, d_out, stream=None) -> None:
        """siac_eval_async on device memory: d_points / d_out are CUDA tensors (float64) or raw
        device pointers (ints); stream is a torch.cuda.Stream, a raw cudaStream_t int, or None
        (the current torch stream when tensors are given)."""
        n = None
        if hasattr(d_points, "data_ptr"):
            assert d_points.dtype.is_floating_point and d_points.element_size() == 8 and d_points.is_contiguous()
            assert d_out.element_size() == 8 and d_out.is_contiguous()
            n = d_points.numel() // 2
            assert d_out.numel() >= n
            pp, po = d_points.data_ptr(), d_out.data_ptr()
            if stream is None:
                import torch
                stream = torch.cuda.current_stream(d_points.device)
        else:
            raise TypeError("pass CUDA tensors (use eval_ptr for raw pointers)")
        sh = stream.cuda_stream if hasattr(stream, "cuda_stream") else (stream or 0)
        _check(lib().siac_eval_async(self._ptr, ctypes.c_void_p(pp), n, ctypes.c_void_p(po), ctypes.c_void_p(sh)),
               self._ptr)

    def eval_ptr(self, d_points: int, n: int, d_out: int, stream: int = 0) -> None:
        _check(lib().siac_eval_async(self._ptr, ctypes.c_void_p(d_points), int(n), ctypes.c_void_p(d_out),
                                     ctypes.c_void_p(stream)), self._ptr)

    def set_counting(self, on: bool = True) -> None:
        _check(lib().siac_set_counting(self._ptr, 1 if on else 0), self._ptr)

    def stats(self) -> dict:
        c = _Counters()
        _check(lib().siac_stats(self._ptr, ctypes.byref(c)), self._ptr)
        return {f: getattr(c, f) for f, _ in _Counters._fields_}

    def create_info(self) -> dict:
        """siac_get_create_info: siac_create's cost (ms per stage) and resident device bytes."""
        c = _CreateInfo()
        _check(lib().siac_get_create_info(self._ptr, ctypes.byref(c)), self._ptr)
        return {f: getattr(c, f) for f, _ in _CreateInfo._fields_}

    def set_schedule(self, schedule: int) -> None:
        """0 = default (fastest = 5), 1 = thread-per-point, 2 = warp-per-tile, 3 = warp-specialized, 4 = jump,
        5 = jump with closed-form cross terms, 6 = per-element (the paper's Alg. 3 mapping, scatter-add)."""
        _check(lib().siac_set_schedule(self._ptr, int(schedule)), self._ptr)

    def set_graphs(self, on: bool = True) -> None:
        """Replay CUDA graphs of repeated eval_async calls on the same buffers (siac_set_graphs)."""
        _check(lib().siac_set_graphs(self._ptr, 1 if on else 0), self._ptr)

    def set_timing(self, on: bool = True) -> None:
        _check(lib().siac_set_timing(self._ptr, 1 if on else 0), self._ptr)

    def timing(self) -> tuple[float, int]:
        """(sum of main-kernel ms, number of timed launches) since the last call."""
        ms, n = ctypes.c_double(), ctypes.c_int64()
        _check(lib().siac_timing(self._ptr, ctypes.byref(ms), ctypes.byref(n)), self._ptr)
        return ms.value, n.value

    def info(self) -> dict:
        nt, gx, gy = ctypes.c_int64(), ctypes.c_int32(), ctypes.c_int32()
        cw, ch = ctypes.c_double(), ctypes.c_double()
        _check(lib().siac_info(self._ptr, ctypes.byref(nt), ctypes.byref(gx), ctypes.byref(gy),
                               ctypes.byref(cw), ctypes.byref(ch)), self._ptr)
        return dict(n_triangles=nt.value, grid_nx=gx.value, grid_ny=gy.value, cell_w=cw.value, cell_h=ch.value)

    def debug_records(self, n: int, which: int = 0) -> np.ndarray:
        """First n device records in binning order: which = 0 mesh (Rec), 1 jump (JRec), 2 cross (XRec)."""
        rd = ctypes.c_int32()
        _check(lib().siac_debug_records(self._ptr, int(which), 0, None, ctypes.byref(rd)), self._ptr)
        out = np.empty((n, rd.value))
        _check(lib().siac_debug_records(self._ptr, int(which), n, _dp(out), ctypes.byref(rd)), self._ptr)
        return out

    def destroy(self) -> None:
        if getattr(self, "_ptr", None):
            lib().siac_destroy(self._ptr)
            self._ptr = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.destroy()


def create(V, T, C, k, h, periodic=3, domain=(0.0, 0.0, 1.0, 1.0), device=0, cell_factor=0.0, basis=0,
           boundary=0) -> Context:
    return Context(V, T, C, k, h, periodic, domain, device, cell_factor, basis, boundary)


def host_tables(k: int):
    """(cell_table (3k+1, k+1), basis_matrix (nb, nb)) computed by the library's host code."""
    nb = (k + 1) * (k + 2) // 2
    t = np.empty((3 * k + 1, k + 1))
    R = np.empty((nb, nb))
    _check(lib().siac_host_tables(int(k), _dp(t), _dp(R)), None)
    return t, R


def probe_fp64(device: int = 0) -> float:
    """Measured FP64 FMA throughput (TFLOP/s) of `device` (siac_probe_fp64)."""
    t = ctypes.c_double()
    _check(lib().siac_probe_fp64(int(device), ctypes.byref(t)), None)
    return t.value


def version() -> str:
    return lib().siac_version().decode()


# ---------------------------------------------------------------- steps either side of the path
# (SURVEY §8(f) NEXT-3): argument marshalling only; every step runs in csrc/siac_io.cu.

def _ptr(t):
    return ctypes.c_void_p(t.data_ptr())


def _stream_ptr(stream):
    return ctypes.c_void_p(0 if stream is None else stream.cuda_stream)


def projection_rule(n_quad: int):
    """(rs (n_quad^2, 2) unit-triangle nodes, w (n_quad^2,) reference-triangle weights)."""
    rs = np.empty((n_quad * n_quad, 2))
    w = np.empty(n_quad * n_quad)
    _check(lib().siac_projection_rule(int(n_quad), _dp(rs), _dp(w)), None)
    return rs, w


def map_points_async(d_V, d_T, d_rs, d_out, stream=None) -> None:
    """d_out[(t, q)] = v0 + r_q (v1 - v0) + s_q (v2 - v0); torch CUDA tensors (f64 / int32)."""
    _check(lib().siac_map_points_async(_ptr(d_V), _ptr(d_T), int(d_T.shape[0]), _ptr(d_rs), int(d_rs.shape[0]),
                                       _ptr(d_out), _stream_ptr(stream)), None)


def project_async(k: int, n_quad: int, d_f, d_coeffs, stream=None) -> None:
    """Orthonormal Dubiner modes (n_triangles, nb) of f sampled at the projection rule nodes."""
    _check(lib().siac_project_async(int(k), int(n_quad), _ptr(d_f), int(d_coeffs.shape[0]), _ptr(d_coeffs),
                                    _stream_ptr(stream)), None)


def error_norms_async(d_u, d_ref, d_w, d_out, stream=None) -> None:
    """d_out[0:3] = sqrt(sum w e^2), max |e|, sum w for e = u - ref (d_w may be None)."""
    _check(lib().siac_error_norms_async(_ptr(d_u), _ptr(d_ref), None if d_w is None else _ptr(d_w),
                                        int(d_u.shape[0]), _ptr(d_out), _stream_ptr(stream)), None)


# ---------------------------------------------------------------- tetrahedral meshes (NEXT-4)

def _check3(rc, ctx_ptr=None):
    if rc != 0:
        raise SiacError(f"siac3 error {rc}: {lib().siac3_last_error(ctx_ptr).decode()}")


class Context3:
    """A siac3_ctx (include/siac.h, tetrahedral meshes): coefficients of the reference-tetrahedron
    monomials r^a s^b t^c (modes by a+b+c, then c, then b)."""

    def __init__(self, V, T, C, k: int, h: float, periodic: int = 7, domain=(0.0, 0.0, 0.0, 1.0, 1.0, 1.0),
                 device: int = 0):
        L = lib()
        V = np.ascontiguousarray(V, dtype=np.float64).reshape(-1, 3)
        T = np.ascontiguousarray(T, dtype=np.int32).reshape(-1, 4)
        C = np.ascontiguousarray(C, dtype=np.float64)
        if 1 <= k <= 3 and C.size != len(T) * (k + 1) * (k + 2) * (k + 3) // 6:
            raise ValueError("coeffs must have (k+1)(k+2)(k+3)/6 columns")
        p = _Params3(int(k), float(h), int(periodic), (ctypes.c_double * 6)(*domain), int(device))
        ptr = ctypes.c_void_p()
        _check3(L.siac3_create(ctypes.byref(ptr), _dp(V), len(V), T.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                               len(T), _dp(C), ctypes.byref(p)), None)
        self._ptr = ptr
        self.k = int(k)

    def eval(self, points) -> np.ndarray:
        P = np.ascontiguousarray(points, dtype=np.float64).reshape(-1, 3)
        out = np.empty(len(P), dtype=np.float64)
        _check3(lib().siac3_eval(self._ptr, _dp(P), len(P), _dp(out)), self._ptr)
        return out

    def eval_async(self, d_points, d_out, stream=None) -> None:
        assert d_points.dtype.is_floating_point and d_points.element_size() == 8 and d_points.is_contiguous()
        assert d_out.element_size() == 8 and d_out.is_contiguous()
        n = d_points.numel() // 3
        assert d_out.numel() >= n
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(d_points.device)
        sh = stream.cuda_stream if hasattr(stream, "cuda_stream") else (stream or 0)
        _check3(lib().siac3_eval_async(self._ptr, ctypes.c_void_p(d_points.data_ptr()), n,
                                       ctypes.c_void_p(d_out.data_ptr()), ctypes.c_void_p(sh)), self._ptr)

    def set_schedule(self, schedule: int) -> None:
        """0: warp per point tile (default), 1: thread per point."""
        _check3(lib().siac3_set_schedule(self._ptr, int(schedule)), self._ptr)

    def set_counting(self, on: bool = True) -> None:
        _check3(lib().siac3_set_counting(self._ptr, 1 if on else 0), self._ptr)

    def stats(self) -> dict:
        a, b = ctypes.c_int64(), ctypes.c_int64()
        _check3(lib().siac3_stats(self._ptr, ctypes.byref(a), ctypes.byref(b)), self._ptr)
        return {"pairs": a.value, "pieces": b.value}

    def destroy(self) -> None:
        if getattr(self, "_ptr", None):
            lib().siac3_destroy(self._ptr)
            self._ptr = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def create3(V, T, C, k, h, periodic=7, domain=(0.0, 0.0, 0.0, 1.0, 1.0, 1.0), device=0) -> Context3:
    return Context3(V, T, C, k, h, periodic, domain, device)


def tet_rule(n: int) -> np.ndarray:
    """(n^3, 4): (r, s, t, weight) of the library's collapsed rule on the unit tetrahedron."""
    out = np.empty((n ** 3, 4))
    _check3(lib().siac3_tet_rule(int(n), _dp(out)), None)
    return out
