"""Thin Python binding of the C ABI in include/capgpu.h (ctypes; marshalling only).

Every step of the CapGPU path runs in the CUDA kernels of libcapgpu.so; this
module only allocates torch device tensors, fills the ABI structs and calls the
library.  There is no CPU fallback: if the library is missing the import of
`lib()` raises.

Names follow the ABI: capgpu_create / capgpu_identify / capgpu_assign_weights /
capgpu_control_step / capgpu_simulate (module functions), wrapped by the
`CapGPU` class for convenience.
"""
from __future__ import annotations

import ctypes as C
import os

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libcapgpu.so")

MAX_KNOBS, MAX_M, MAX_P, MAX_LEVELS = 16, 4, 64, 32
OK, E_INVALID, E_NOMEM, E_CUDA, E_NCCL, E_ORDER, E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
ST_CAP_INFEASIBLE, ST_SLO_INFEASIBLE, ST_SOLVER_CAP, ST_NONFINITE = 1, 2, 4, 8


_VP = C.c_void_p


class Horizons(C.Structure):
    _fields_ = [("P", C.c_int32), ("M", C.c_int32)]


class KnobBounds(C.Structure):
    _fields_ = [("f_min", C.c_double), ("f_max", C.c_double), ("n_levels", C.c_int32),
                ("sweep_base", C.c_int32), ("f_lo", C.c_double), ("r0", C.c_double)]


class Params(C.Structure):
    _fields_ = [("q", C.c_double), ("r0", C.c_double), ("theta_min", C.c_double), ("lam", C.c_double),
                ("rho", C.c_double), ("a_lo", C.c_double), ("a_hi", C.c_double), ("a_floor", C.c_double),
                ("gamma", C.c_double), ("noise_std", C.c_double), ("substeps", C.c_int32),
                ("caps_per_server", C.c_int32), ("seed", C.c_uint64), ("wmove", C.c_double),
                ("ref_alpha", C.c_double)]


class Shard(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("srv_begin", C.c_int64),
                ("n_servers_global", C.c_int64), ("use_nccl", C.c_int32), ("nccl_id", C.c_uint8 * 128)]


class Workload(C.Structure):
    _fields_ = [("demand_kind", C.c_int32), ("demand_frac", C.c_double), ("cap_frac0", C.c_double),
                ("cap_frac_rand", C.c_double), ("cap_frac_step", C.c_double), ("cap_period", C.c_int64),
                ("cap_lo", C.c_int64), ("cap_hi", C.c_int64), ("cap_mult", C.c_double),
                ("hierarchical", C.c_int32), ("rack", C.c_int32), ("block", C.c_int32),
                ("cluster_frac", C.c_double), ("rack_frac", C.c_double), ("cap_base_d", _VP),
                ("gain_dlo", C.c_double), ("gain_step", C.c_double),
                ("slo_period", C.c_int64), ("slo_lo", C.c_int64), ("slo_hi", C.c_int64),
                ("slo_a", C.c_double * MAX_KNOBS), ("slo_b", C.c_double * MAX_KNOBS),
                ("controller", C.c_int32), ("fs_levels", C.c_int32), ("safe_margin", C.c_double),
                ("p_pole", C.c_double), ("gpu_share", C.c_double)]


_VP = C.c_void_p


class Trace(C.Structure):
    _fields_ = [("sum_p_d", _VP), ("sumsq_p_d", _VP), ("max_p_d", _VP), ("sum_theta_d", _VP),
                ("n_viol_d", _VP), ("n_window_d", _VP), ("act_count_d", _VP), ("final_p_d", _VP), ("n_miss_d", _VP),
                ("n_trace", C.c_int32), ("trace_inst_d", _VP), ("p_d", _VP), ("cap_d", _VP), ("u_d", _VP),
                ("ahat_d", _VP), ("theta_d", _VP), ("active_d", _VP), ("rank_d", _VP), ("levels_d", _VP),
                ("status_d", _VP), ("agg_W_d", _VP), ("agg_P_d", _VP)]


SYMBOLS = ["capgpu_version", "capgpu_status_string", "capgpu_last_error", "capgpu_default_params",
           "capgpu_create", "capgpu_destroy", "capgpu_state_bytes", "capgpu_identify", "capgpu_set_prior",
           "capgpu_model_reset", "capgpu_assign_weights", "capgpu_control_step", "capgpu_simulate",
           "capgpu_sim_reset", "capgpu_sim_state", "capgpu_sim_caps", "capgpu_nccl_unique_id", "capgpu_shard_range",
           "capgpu_debug_gen", "capgpu_fp64_peak", "capgpu_simulate_group", "capgpu_tree_sum_host",
           "capgpu_debug_phase_counters", "capgpu_set_state", "capgpu_checkpoint_bytes", "capgpu_checkpoint_save",
           "capgpu_checkpoint_load", "capgpu_explicit_build", "capgpu_explicit_step"]

_lib = None


def lib():
    """Load libcapgpu.so (built in-tree by build.py).  Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    path = LIB_PATH
    var = os.environ.get("CAPGPU_LIB_VARIANT")
    if var:  # experiment / profiling builds (build.py VARIANTS), e.g. "timing" for tools/phase_timing.py
        path = os.path.join(_PKG, f"libcapgpu_{var}.so")
    if not os.path.exists(path):
        raise RuntimeError(f"{path} missing: run `python -m paper_conf_icpp_masw25_b200.build` "
                           "(there is no CPU fallback)")
    L = C.CDLL(path)
    L.capgpu_version.restype = C.c_char_p
    L.capgpu_status_string.restype = C.c_char_p
    L.capgpu_status_string.argtypes = [C.c_int]
    L.capgpu_last_error.restype = C.c_char_p
    L.capgpu_last_error.argtypes = [_VP]
    L.capgpu_default_params.argtypes = [C.POINTER(Params)]
    L.capgpu_create.argtypes = [C.POINTER(_VP), C.c_int64, C.c_int32, Horizons, C.POINTER(KnobBounds),
                                C.POINTER(Params), C.POINTER(Shard)]
    L.capgpu_destroy.argtypes = [_VP]
    L.capgpu_state_bytes.argtypes = [_VP]
    L.capgpu_state_bytes.restype = C.c_int64
    L.capgpu_identify.argtypes = [_VP, _VP, _VP, C.c_int32, _VP, _VP, _VP, _VP]
    L.capgpu_set_prior.argtypes = [_VP, _VP, _VP]
    L.capgpu_model_reset.argtypes = [_VP, _VP]
    L.capgpu_assign_weights.argtypes = [_VP, _VP, _VP, _VP, _VP, _VP, _VP]
    L.capgpu_control_step.argtypes = [_VP] + [_VP] * 10 + [_VP]
    L.capgpu_simulate.argtypes = [_VP, C.c_int64, C.POINTER(Workload), C.POINTER(Trace), _VP]
    L.capgpu_sim_reset.argtypes = [_VP]
    L.capgpu_sim_state.argtypes = [_VP, _VP, _VP, _VP, _VP, _VP]
    L.capgpu_sim_caps.argtypes = [_VP, _VP, _VP]
    L.capgpu_set_state.argtypes = [_VP, _VP, _VP, _VP, _VP, _VP]
    L.capgpu_explicit_build.argtypes = [_VP, _VP, _VP, _VP]
    L.capgpu_explicit_step.argtypes = [_VP, _VP, _VP, _VP, _VP, _VP, _VP, _VP]
    L.capgpu_checkpoint_bytes.argtypes = [_VP]
    L.capgpu_checkpoint_bytes.restype = C.c_int64
    L.capgpu_checkpoint_save.argtypes = [_VP, _VP, _VP]
    L.capgpu_checkpoint_load.argtypes = [_VP, _VP, _VP]
    L.capgpu_nccl_unique_id.argtypes = [C.POINTER(C.c_uint8 * 128)]
    L.capgpu_shard_range.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.c_int64, C.POINTER(C.c_int64)]
    L.capgpu_shard_range.restype = C.c_int64
    L.capgpu_debug_gen.argtypes = [_VP, C.c_int64, C.c_int32, C.c_double, _VP, _VP, _VP, _VP, _VP, _VP]
    L.capgpu_fp64_peak.argtypes = [C.POINTER(C.c_double), _VP]
    L.capgpu_simulate_group.argtypes = [C.POINTER(_VP), C.c_int32, C.c_int64, C.POINTER(Workload),
                                        C.POINTER(C.POINTER(Trace)), _VP]
    L.capgpu_tree_sum_host.argtypes = [C.POINTER(C.c_double), C.c_int64, C.POINTER(C.c_double)]
    L.capgpu_debug_phase_counters.argtypes = [_VP, _VP]
    _lib = L
    return L


class CapGPUError(RuntimeError):
    pass


def _check(rc: int, ctx=None):
    if rc != OK:
        L = lib()
        msg = L.capgpu_last_error(ctx).decode()
        raise CapGPUError(f"{L.capgpu_status_string(rc).decode()} ({rc}): {msg}")


def _ptr(t):
    return None if t is None else _VP(t.data_ptr())


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return _VP(s.cuda_stream)


def default_params() -> Params:
    p = Params()
    lib().capgpu_default_params(C.byref(p))
    return p


def shard_range(n_global: int, world: int, rank: int, granule: int = 1024):
    b = C.c_int64(0)
    n = lib().capgpu_shard_range(n_global, world, rank, granule, C.byref(b))
    if n < 0:
        raise CapGPUError("bad shard request")
    return int(b.value), int(n)


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(lib().capgpu_nccl_unique_id(C.byref(buf)))
    return bytes(buf)


def simulate_group(ctxs, periods: int, workload, trace_insts=None, summaries: bool = True):
    """capgpu_simulate_group: several shards of the hierarchical budget on one
    GPU stepping together with a loopback all-reduce.  Returns one output dict
    per context (like CapGPU.simulate)."""
    n = len(ctxs)
    trs, outs = [], []
    for q, g in enumerate(ctxs):
        tr, out = g._trace(periods, workload, None if trace_insts is None else trace_insts[q], summaries)
        trs.append(tr)
        outs.append(out)
    arr = (_VP * n)(*[g._ctx for g in ctxs])
    tptr = (C.POINTER(Trace) * n)(*[C.pointer(t) for t in trs])
    rc = lib().capgpu_simulate_group(arr, n, periods, C.byref(workload), tptr, _stream())
    _check(rc, ctxs[0]._ctx)
    return outs


def tree_sum_host(v) -> float:
    """The library's fixed-order pairwise tree (host copy of the device tree)."""
    import numpy as np
    a = np.ascontiguousarray(np.asarray(v, dtype=np.float64))
    out = C.c_double(0)
    _check(lib().capgpu_tree_sum_host(a.ctypes.data_as(C.POINTER(C.c_double)), a.size, C.byref(out)))
    return float(out.value)


def fp64_peak_tflops() -> float:
    out = C.c_double(0)
    _check(lib().capgpu_fp64_peak(C.byref(out), _stream()))
    return float(out.value)


def workload_from(desc: dict) -> Workload:
    wl = desc["workload"]
    w = Workload()
    w.demand_kind, w.demand_frac = wl["demand_kind"], wl["demand_frac"]
    w.cap_frac0, w.cap_frac_rand, w.cap_frac_step = wl["cap_frac0"], wl["cap_frac_rand"], wl["cap_frac_step"]
    w.cap_period, w.cap_lo, w.cap_hi, w.cap_mult = wl["cap_period"], wl["cap_lo"], wl["cap_hi"], wl["cap_mult"]
    w.hierarchical = int(wl.get("hierarchical", False))
    w.rack, w.block = wl.get("rack", 16), wl.get("block", 1024)
    w.cluster_frac, w.rack_frac = wl.get("cluster_frac", 0.55), wl.get("rack_frac", 0.9)
    w.gain_dlo, w.gain_step = wl.get("gain_dlo", 0.0), wl.get("gain_step", 0.0)
    w.slo_period, w.slo_lo, w.slo_hi = wl.get("slo_period", 0), wl.get("slo_lo", 0), wl.get("slo_hi", 0)
    for j, r in enumerate(wl.get("slo_a") or []):
        w.slo_a[j] = r
    for j, r in enumerate(wl.get("slo_b") or []):
        w.slo_b[j] = r
    w.controller, w.fs_levels = wl.get("controller", 0), wl.get("fs_levels", 1)
    w.safe_margin, w.p_pole = wl.get("safe_margin", 0.0), wl.get("p_pole", 0.5)
    w.gpu_share = wl.get("gpu_share", 0.5)
    return w


class CapGPU:
    """One context = one shard of servers on the current CUDA device."""

    def __init__(self, n_servers: int, n_gpus: int, P: int, M: int, knobs: list[dict], controller: dict,
                 seed: int = 1, caps_per_server: int = 1, srv_begin: int = 0, world: int = 1, rank: int = 0,
                 n_servers_global: int | None = None, nccl_id: bytes | None = None, device=None):
        self.L = lib()
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.n_srv, self.N, self.P, self.M = n_servers, 1 + n_gpus, P, M
        self.caps = caps_per_server
        self.n_inst = n_servers * caps_per_server
        self.S = controller.get("substeps", 4)
        kb = (KnobBounds * self.N)()
        for j, k in enumerate(knobs):
            kb[j].f_min, kb[j].f_max = k["f_min"], k["f_max"]
            kb[j].n_levels, kb[j].sweep_base = k["n_levels"], k["sweep_base"]
            kb[j].f_lo = k.get("f_lo", 0.0)
            kb[j].r0 = k.get("r0", 0.0)
        p = default_params()
        p.q, p.r0, p.theta_min, p.lam = controller["q"], controller["r0"], controller["theta_min"], controller["lam"]
        p.rho, p.a_lo, p.a_hi, p.a_floor = controller["rho"], controller["a_lo"], controller["a_hi"], controller["a_floor"]
        p.gamma, p.noise_std, p.substeps = controller["gamma"], controller["noise_std"], controller["substeps"]
        p.caps_per_server, p.seed = caps_per_server, seed
        p.wmove = controller.get("wmove", 0.0)
        p.ref_alpha = controller.get("ref_alpha", 0.0)
        sh = Shard()
        sh.rank, sh.world, sh.srv_begin = rank, world, srv_begin
        sh.n_servers_global = n_servers_global if n_servers_global is not None else srv_begin + n_servers
        if nccl_id is not None:
            sh.use_nccl = 1
            for i, b in enumerate(nccl_id):
                sh.nccl_id[i] = b
        self._ctx = _VP()
        with torch.cuda.device(self.device):
            _check(self.L.capgpu_create(C.byref(self._ctx), n_servers, n_gpus, Horizons(P, M), kb, C.byref(p),
                                        C.byref(sh)))

    @classmethod
    def from_config(cls, desc: dict, n_servers: int | None = None, **kw):
        return cls(n_servers if n_servers is not None else desc["n_servers"], desc["n_gpus"], desc["P"], desc["M"],
                   desc["knobs"], desc["controller"], seed=desc["seed"],
                   caps_per_server=desc["workload"]["n_caps"], **kw)

    def close(self):
        if self._ctx:
            self.L.capgpu_destroy(self._ctx)
            self._ctx = _VP()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _z(self, *shape, dtype=torch.float64):
        return torch.zeros(*shape, dtype=dtype, device=self.device)

    @property
    def state_bytes(self) -> int:
        return int(self.L.capgpu_state_bytes(self._ctx))

    # ---- S0
    def identify(self, F=None, p=None):
        n = self.n_srv
        A, Cc, r2 = self._z(self.N, n), self._z(n), self._z(n)
        rows = 0 if F is None else F.shape[0]
        _check(self.L.capgpu_identify(self._ctx, _ptr(F), _ptr(p), rows, _ptr(A), _ptr(Cc), _ptr(r2), _stream()),
               self._ctx)
        return A, Cc, r2

    def set_prior(self, A0):
        _check(self.L.capgpu_set_prior(self._ctx, _ptr(A0.contiguous()), _stream()), self._ctx)

    def model_reset(self):
        _check(self.L.capgpu_model_reset(self._ctx, _stream()), self._ctx)

    # ---- S2
    def assign_weights(self, thr, thr_max):
        th, R = self._z(self.N, self.n_srv), self._z(self.N, self.n_srv)
        rk = self._z(self.N, self.n_srv, dtype=torch.int8)
        _check(self.L.capgpu_assign_weights(self._ctx, _ptr(thr), _ptr(thr_max), _ptr(th), _ptr(R), _ptr(rk),
                                            _stream()), self._ctx)
        return th, R, rk

    # ---- S1-S3 on user measurements
    def control_step_buffers(self, ranks: bool = True, ahat: bool = True):
        """Output buffers of control_step (written entirely by the kernel; reusable)."""
        n = self.n_srv
        return dict(u=self._z(self.M, self.N, n), active=self._z(self.M, n, dtype=torch.int32),
                    rank=self._z(self.N, n, dtype=torch.int8) if ranks else None,
                    ahat=self._z(self.N, n) if ahat else None, status=self._z(n, dtype=torch.int32))

    def control_step(self, p_meas, f_applied, thr, thr_max, cap, out=None):
        o = out if out is not None else self.control_step_buffers()
        opt = lambda t: _ptr(t) if t is not None else None  # noqa: E731
        _check(self.L.capgpu_control_step(self._ctx, _ptr(p_meas), _ptr(f_applied), _ptr(thr), _ptr(thr_max),
                                          _ptr(cap), _ptr(o["u"]), _ptr(o["active"]), opt(o["rank"]),
                                          opt(o["ahat"]), _ptr(o["status"]), _stream()),
               self._ctx)
        return o

    # ---- closed loop
    def summary_buffers(self):
        """Per-instance summary outputs (written entirely by the kernel; reusable)."""
        ni, M = self.n_inst, self.M
        e = lambda *s, dtype=torch.float64: torch.empty(*s, dtype=dtype, device=self.device)  # noqa: E731
        return dict(sum_p=e(ni), sumsq_p=e(ni), max_p=e(ni), sum_theta=e(ni), n_viol=e(ni, dtype=torch.int32),
                    n_window=e(ni, dtype=torch.int32), act_count=e(M, ni, dtype=torch.int32), final_p=e(ni),
                    n_miss=e(ni, dtype=torch.int32))

    def simulate(self, periods: int, workload: Workload, trace_inst=None, summaries: bool = True,
                 traces=("p", "cap", "u", "ahat", "theta", "active", "rank", "levels", "status"), out=None):
        tr, out = self._trace(periods, workload, trace_inst, summaries, traces, out)
        _check(self.L.capgpu_simulate(self._ctx, periods, C.byref(workload), C.byref(tr), _stream()), self._ctx)
        return out

    def _trace(self, periods, workload, trace_inst=None, summaries=True,
               traces=("p", "cap", "u", "ahat", "theta", "active", "rank", "levels", "status"), out=None):
        ni, N, M, S = self.n_inst, self.N, self.M, self.S
        tr = Trace()
        if out is None:
            out = self.summary_buffers() if summaries else {}
        if summaries:
            for k in ("sum_p", "sumsq_p", "max_p", "sum_theta", "n_viol", "n_window", "act_count", "final_p",
                      "n_miss"):
                setattr(tr, k + "_d", _ptr(out[k]).value)
        if trace_inst is not None:
            ti = torch.as_tensor(trace_inst, dtype=torch.int64, device=self.device)
            nt = ti.numel()
            out["trace_inst"] = ti
            tr.n_trace = nt
            tr.trace_inst_d = _ptr(ti).value
            K = periods
            shapes = dict(p=((K, nt), torch.float64), cap=((K, nt), torch.float64),
                          u=((K, M, N, nt), torch.float64), ahat=((K, N, nt), torch.float64),
                          theta=((K, N, nt), torch.float64), active=((K, M, nt), torch.int32),
                          rank=((K, N, nt), torch.int8), levels=((K, S, N, nt), torch.uint8),
                          status=((K, nt), torch.int32))
            for k in traces:
                shp, dt = shapes[k]
                out["tr_" + k] = self._z(*shp, dtype=dt)
                setattr(tr, k + "_d", _ptr(out["tr_" + k]).value)
        if workload.hierarchical:
            out["agg_W"], out["agg_P"] = self._z(periods), self._z(periods)
            tr.agg_W_d, tr.agg_P_d = _ptr(out["agg_W"]).value, _ptr(out["agg_P"]).value
        return tr, out

    def sim_reset(self):
        _check(self.L.capgpu_sim_reset(self._ctx), self._ctx)

    def sim_state(self):
        ni, N = self.n_inst, self.N
        f, a, t, p = self._z(N, ni), self._z(N, ni), self._z(N, ni), self._z(ni)
        _check(self.L.capgpu_sim_state(self._ctx, _ptr(f), _ptr(a), _ptr(t), _ptr(p), _stream()), self._ctx)
        return dict(fbar=f, acc=a, thr=t, p=p)

    def explicit_build(self, thr, thr_max):
        """NEXT-3 explicit MPC, offline part: tabulate each server's piecewise-affine law."""
        _check(self.L.capgpu_explicit_build(self._ctx, _ptr(thr), _ptr(thr_max), _stream()), self._ctx)

    def explicit_step(self, p_meas, f_applied, cap):
        """NEXT-3 explicit MPC, online part: u_0 = law(beta) by table lookup."""
        n = self.n_srv
        u = self._z(self.N, n)
        act = self._z(n, dtype=torch.int32)
        st = self._z(n, dtype=torch.int32)
        _check(self.L.capgpu_explicit_step(self._ctx, _ptr(p_meas), _ptr(f_applied), _ptr(cap), _ptr(u), _ptr(act),
                                           _ptr(st), _stream()), self._ctx)
        return dict(u=u, active=act, status=st)

    def set_state(self, fbar=None, acc=None, thr=None, p=None):
        _check(self.L.capgpu_set_state(self._ctx, _ptr(fbar), _ptr(acc), _ptr(thr), _ptr(p), _stream()), self._ctx)

    def checkpoint(self):
        """Device blob (torch uint8) holding the whole context state (checkpoint / resume)."""
        buf = torch.empty(int(self.L.capgpu_checkpoint_bytes(self._ctx)), dtype=torch.uint8, device="cuda")
        _check(self.L.capgpu_checkpoint_save(self._ctx, _ptr(buf), _stream()), self._ctx)
        return buf

    def restore(self, blob):
        blob = blob.to("cuda")
        _check(self.L.capgpu_checkpoint_load(self._ctx, _ptr(blob), _stream()), self._ctx)

    def sim_caps(self):
        out = self._z(self.n_inst)
        _check(self.L.capgpu_sim_caps(self._ctx, _ptr(out), _stream()), self._ctx)
        return out

    def debug_gen(self, k: int, demand_kind: int = 1, demand_frac: float = 0.7):
        n, N = self.n_srv, self.N
        a, tm, c, dem, nz = self._z(N, n), self._z(N, n), self._z(n), self._z(N, n), self._z(n)
        _check(self.L.capgpu_debug_gen(self._ctx, k, demand_kind, demand_frac, _ptr(a), _ptr(tm), _ptr(c),
                                       _ptr(dem), _ptr(nz), _stream()), self._ctx)
        return dict(a_true=a, thr_max=tm, c_true=c, dem=dem, noise=nz)
