"""ctypes front-end of the CPU oracle (oracle/capgpu_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs.  The product package
(paper_conf_icpp_masw25_b200) never imports this module.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import sys

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_HERE)
if _ROOT not in sys.path:
    sys.path.insert(0, _ROOT)

from gen import configs  # noqa: E402

LIB_PATH = os.path.join(_HERE, "libcapgpu_oracle.so")
# tools/oracle_mutations.py points the tests at a deliberately mutated copy
_LIB_OVERRIDE = os.environ.get("CAPGPU_ORACLE_LIB")
SRC = [os.path.join(_HERE, "capgpu_oracle.c"), os.path.join(_HERE, "capgpu_oracle.h"),
       os.path.join(_ROOT, "gen", "capgpu_gen.h")]
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-std=c11", "-Wall", "-shared", "-fPIC"]

MAXN, MAXM, MAXL, MAXS = 16, 8, 32, 8
ST_CAP_INFEASIBLE, ST_SLO_INFEASIBLE, ST_SOLVER_CAP, ST_NONFINITE = 1, 2, 4, 8


def build(force: bool = False) -> str:
    """Compile the oracle shared library (gcc, no fast-math, no FP contraction)."""
    stale = force or not os.path.exists(LIB_PATH) or any(
        os.path.getmtime(s) > os.path.getmtime(LIB_PATH) for s in SRC)
    if stale:
        cmd = ["gcc", *CFLAGS, "-o", LIB_PATH, SRC[0], "-lm"]
        subprocess.run(cmd, check=True)
    return LIB_PATH


class OraCfg(C.Structure):
    _fields_ = [("n", C.c_int32), ("P", C.c_int32), ("M", C.c_int32), ("substeps", C.c_int32),
                ("n_levels", C.c_int32 * MAXN), ("sweep_base", C.c_int32 * MAXN),
                ("f_min", C.c_double * MAXN), ("f_max", C.c_double * MAXN),
                ("f_lo", C.c_double * MAXN), ("r0", C.c_double * MAXN),
                ("q", C.c_double), ("theta_min", C.c_double), ("lam", C.c_double),
                ("rho", C.c_double), ("a_lo", C.c_double), ("a_hi", C.c_double),
                ("a_floor", C.c_double), ("gamma", C.c_double), ("noise_std", C.c_double),
                ("seed", C.c_uint64), ("wmove", C.c_double), ("ref_alpha", C.c_double)]


class OraWorkload(C.Structure):
    _fields_ = [("periods", C.c_int32), ("n_caps", C.c_int32), ("demand_kind", C.c_int32),
                ("demand_frac", C.c_double), ("cap_frac0", C.c_double),
                ("cap_frac_rand", C.c_double), ("cap_frac_step", C.c_double),
                ("cap_period", C.c_int64), ("cap_lo", C.c_int64), ("cap_hi", C.c_int64),
                ("cap_mult", C.c_double), ("gain_dlo", C.c_double), ("gain_step", C.c_double),
                ("slo_period", C.c_int64), ("slo_lo", C.c_int64), ("slo_hi", C.c_int64),
                ("slo_a", C.c_double * MAXN), ("slo_b", C.c_double * MAXN),
                ("controller", C.c_int32), ("fs_levels", C.c_int32), ("safe_margin", C.c_double),
                ("p_pole", C.c_double), ("gpu_share", C.c_double)]


class OraSummary(C.Structure):
    _fields_ = [("sum_p", C.c_double), ("sumsq_p", C.c_double), ("max_p", C.c_double),
                ("sum_theta", C.c_double), ("n_window", C.c_int32), ("n_viol", C.c_int32),
                ("act_count", C.c_int32 * MAXM), ("n_miss", C.c_int32)]


class OraModel(C.Structure):
    _fields_ = [("w", C.c_double), ("mu_f", C.c_double * MAXN), ("mu_p", C.c_double),
                ("S_ff", (C.c_double * MAXN) * MAXN), ("S_fp", C.c_double * MAXN)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if _LIB_OVERRIDE:
            L = C.CDLL(_LIB_OVERRIDE)
        else:
            build()
            L = C.CDLL(LIB_PATH)
        dp, ip = C.POINTER(C.c_double), C.POINTER(C.c_int32)
        cp = C.POINTER(OraCfg)
        L.ora_levels.argtypes = [cp, C.c_int, dp, dp, dp]
        L.ora_slo_level.argtypes = [cp, C.c_int, C.c_double, dp]
        L.ora_slo_bounds.argtypes = [cp, C.POINTER(OraWorkload), C.c_int64, dp, ip]
        L.ora_slo_bounds.restype = C.c_uint32
        L.ora_identify_ls.argtypes = [C.c_int, C.c_int, dp, dp, dp, dp, dp]
        L.ora_sweep_rows.argtypes = [cp, C.c_uint64, C.c_int, dp, dp]
        L.ora_sweep_nrows.argtypes = [cp]
        L.ora_identify_server.argtypes = [cp, C.c_uint64, dp, dp, dp]
        L.ora_model_reset.argtypes = [C.POINTER(OraModel)]
        L.ora_model_push.argtypes = [cp, C.POINTER(OraModel), dp, C.c_double]
        L.ora_model_solve.argtypes = [cp, C.POINTER(OraModel), dp, dp]
        L.ora_model_definition.argtypes = [cp, C.c_int, dp, dp, dp, dp]
        L.ora_weights.argtypes = [cp, dp, dp, dp, dp, C.POINTER(C.c_int8)]
        L.ora_block_weights.argtypes = [cp, dp]
        u32p = C.POINTER(C.c_uint32)
        L.ora_mpc_stacked.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp, dp, u32p, u32p, ip]
        L.ora_mpc_bruteforce.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp, dp]
        L.ora_mpc_move.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp, dp, dp, u32p, u32p, ip]
        L.ora_mpc_move_bruteforce.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp, dp, dp]
        L.ora_mpc_move_cost.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp]
        L.ora_mpc_move_cost.restype = C.c_double
        L.ora_mpc_cost.argtypes = [cp, dp, dp, C.c_double, dp, dp]
        L.ora_mpc_cost.restype = C.c_double
        L.ora_mpc_classify.argtypes = [cp, dp, dp, C.c_double, dp, dp, dp, dp, u32p, u32p]
        # NEXT-3 reference trajectory (Q37): the same with the offset dref = P_s - p(k)
        L.ora_ref_pow.argtypes = [cp, C.c_int]
        L.ora_ref_pow.restype = C.c_double
        L.ora_mpc_stacked_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp, dp, dp, u32p, u32p, ip]
        L.ora_mpc_move_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp, dp, dp, dp, u32p, u32p, ip]
        L.ora_mpc_bruteforce_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp, dp, dp, dp]
        L.ora_mpc_cost_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp]
        L.ora_mpc_cost_ref.restype = C.c_double
        L.ora_mpc_move_cost_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp, dp]
        L.ora_mpc_move_cost_ref.restype = C.c_double
        L.ora_mpc_classify_ref.argtypes = [cp, dp, dp, C.c_double, C.c_double, dp, dp, dp, dp, u32p, u32p]
        L.ora_plant_step.argtypes = [cp, dp, C.c_double, dp, dp, C.c_double, dp, dp, dp, dp, dp,
                                     C.POINTER(C.c_uint8)]
        L.ora_gen_server.argtypes = [cp, C.c_uint64, dp, dp, dp, dp, dp]
        L.ora_gen_mix64.argtypes = [C.c_uint64]
        L.ora_gen_mix64.restype = C.c_uint64
        L.ora_gen_noise.argtypes = [cp, C.c_uint64, C.c_int64]
        L.ora_gen_noise.restype = C.c_double
        wp = C.POINTER(OraWorkload)
        L.ora_gen_demand.argtypes = [cp, wp, C.c_uint64, C.c_int64, dp]
        L.ora_gen_cap_base.argtypes = [cp, wp, C.c_uint64, C.c_int]
        L.ora_gen_cap_base.restype = C.c_double
        L.ora_simulate.argtypes = [cp, wp, C.c_int, C.POINTER(C.c_int64), dp, dp, dp, dp, u32p,
                                   u32p, C.POINTER(C.c_int8), C.POINTER(C.c_uint8), dp, dp, u32p,
                                   dp, C.POINTER(OraSummary), dp, C.c_int]
        L.ora_budget_caps.argtypes = [C.c_int, C.c_int, dp, dp, C.c_double, C.c_double,
                                      C.c_double, dp, dp]
        L.ora_simulate_baseline.argtypes = [cp, wp, C.c_int, C.POINTER(C.c_int64), dp, dp, dp,
                                            C.POINTER(C.c_uint8), dp, dp, C.POINTER(OraSummary)]
        L.ora_simulate_hier.argtypes = [cp, wp, C.c_int, C.c_int, C.c_double, C.c_double, dp, C.c_double,
                                        C.c_int, C.c_int, C.POINTER(C.c_int64), dp, dp, dp, u32p, u32p,
                                        C.POINTER(C.c_uint8), dp, dp, dp, dp]
        _lib = L
    return _lib


def _dp(a):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _arr(x, n=None):
    a = np.ascontiguousarray(np.asarray(x, dtype=np.float64))
    return a


def make_cfg(desc: dict) -> OraCfg:
    """Build an OraCfg from a gen.configs description (gen.configs.get(...))."""
    c = OraCfg()
    ks = desc["knobs"]
    ctl = desc["controller"]
    c.n = len(ks)
    c.P, c.M, c.substeps = desc["P"], desc["M"], ctl["substeps"]
    for j, k in enumerate(ks):
        c.n_levels[j] = k["n_levels"]
        c.sweep_base[j] = k["sweep_base"]
        c.f_min[j], c.f_max[j] = k["f_min"], k["f_max"]
        c.f_lo[j] = k.get("f_lo", k["f_min"])
        c.r0[j] = k.get("r0", ctl["r0"])
    c.q, c.theta_min, c.lam, c.rho = ctl["q"], ctl["theta_min"], ctl["lam"], ctl["rho"]
    c.a_lo, c.a_hi, c.a_floor = ctl["a_lo"], ctl["a_hi"], ctl["a_floor"]
    c.gamma, c.noise_std = ctl["gamma"], ctl["noise_std"]
    c.seed = desc["seed"]
    c.wmove = ctl.get("wmove", 0.0)
    c.ref_alpha = ctl.get("ref_alpha", 0.0)
    return c


def make_workload(desc: dict, periods: int | None = None) -> OraWorkload:
    w = OraWorkload()
    wl = desc["workload"]
    w.periods = desc["periods"] if periods is None else periods
    w.n_caps = wl["n_caps"]
    w.demand_kind, w.demand_frac = wl["demand_kind"], wl["demand_frac"]
    w.cap_frac0, w.cap_frac_rand, w.cap_frac_step = wl["cap_frac0"], wl["cap_frac_rand"], wl["cap_frac_step"]
    w.cap_period, w.cap_lo, w.cap_hi, w.cap_mult = wl["cap_period"], wl["cap_lo"], wl["cap_hi"], wl["cap_mult"]
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


class Oracle:
    """Convenience wrapper around one config."""

    def __init__(self, desc: dict):
        self.desc = desc
        self.cfg = make_cfg(desc)
        self.n = self.cfg.n
        self.M = self.cfg.M
        self.S = self.cfg.substeps
        self.L = lib()

    # ---- grid
    def levels(self, j):
        L = self.cfg.n_levels[j]
        lv, mid, g = np.zeros(L), np.zeros(max(L - 1, 1)), np.zeros(L)
        self.L.ora_levels(C.byref(self.cfg), j, _dp(lv), _dp(mid), _dp(g))
        return lv, mid[: L - 1], g

    # ---- SLO (NEXT-1)
    def slo_level(self, j, ratio):
        fr = np.zeros(1)
        q = self.L.ora_slo_level(C.byref(self.cfg), j, float(ratio), _dp(fr))
        return int(q), float(fr[0])

    def slo_bounds(self, k, periods=None):
        w = make_workload(self.desc, periods)
        lo = np.zeros(self.n); q = np.zeros(self.n, dtype=np.int32)
        st = self.L.ora_slo_bounds(C.byref(self.cfg), C.byref(w), int(k), _dp(lo),
                                   q.ctypes.data_as(C.POINTER(C.c_int32)))
        return lo, q, int(st)

    # ---- S0
    def identify_ls(self, F, p):
        F = _arr(F); p = _arr(p)
        rows, n = F.shape
        A = np.zeros(n); Cc = np.zeros(1); r2 = np.zeros(1)
        rc = self.L.ora_identify_ls(n, rows, _dp(F), _dp(p), _dp(A), _dp(Cc), _dp(r2))
        if rc != 0:
            raise RuntimeError(f"ora_identify_ls rc={rc}")
        return A, float(Cc[0]), float(r2[0])

    def sweep_rows(self, server, noisy=True):
        rows = self.L.ora_sweep_nrows(C.byref(self.cfg))
        F = np.zeros((rows, self.n)); p = np.zeros(rows)
        self.L.ora_sweep_rows(C.byref(self.cfg), server, int(noisy), _dp(F), _dp(p))
        return F, p

    def identify_server(self, server):
        A = np.zeros(self.n); Cc = np.zeros(1); r2 = np.zeros(1)
        self.L.ora_identify_server(C.byref(self.cfg), server, _dp(A), _dp(Cc), _dp(r2))
        return A, float(Cc[0]), float(r2[0])

    # ---- S1
    def model_new(self):
        m = OraModel()
        self.L.ora_model_reset(C.byref(m))
        return m

    def model_push(self, m, f, p):
        f = _arr(f)
        self.L.ora_model_push(C.byref(self.cfg), C.byref(m), _dp(f), float(p))

    def model_solve(self, m, A0):
        A0 = _arr(A0); out = np.zeros(self.n)
        self.L.ora_model_solve(C.byref(self.cfg), C.byref(m), _dp(A0), _dp(out))
        return out

    def model_definition(self, F_hist, p_hist, A0):
        F_hist = _arr(F_hist); p_hist = _arr(p_hist); A0 = _arr(A0); out = np.zeros(self.n)
        self.L.ora_model_definition(C.byref(self.cfg), len(p_hist), _dp(F_hist), _dp(p_hist),
                                    _dp(A0), _dp(out))
        return out

    # ---- S2
    def weights(self, thr, thr_max):
        thr = _arr(thr); thr_max = _arr(thr_max)
        th, R = np.zeros(self.n), np.zeros(self.n)
        rk = np.zeros(self.n, dtype=np.int8)
        self.L.ora_weights(C.byref(self.cfg), _dp(thr), _dp(thr_max), _dp(th), _dp(R),
                           rk.ctypes.data_as(C.POINTER(C.c_int8)))
        return th, R, rk

    # ---- S3
    def block_weights(self):
        ct = np.zeros(self.M)
        self.L.ora_block_weights(C.byref(self.cfg), _dp(ct))
        return ct

    def mpc(self, Ahat, R, beta, lo, hi, m, dref=0.0):
        """Eq. 9-10a as one dense stacked QP; dref = P_s - p(k) feeds the
        reference trajectory when cfg ref_alpha > 0 (NEXT-3, Q37)."""
        Ahat, R, lo, hi, m = map(_arr, (Ahat, R, lo, hi, m))
        u = np.zeros((self.M, self.n))
        act = np.zeros(self.M, dtype=np.uint32); tie = np.zeros(self.M, dtype=np.uint32)
        it = np.zeros(1, dtype=np.int32)
        st = self.L.ora_mpc_stacked_ref(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), float(dref), _dp(lo),
                                        _dp(hi), _dp(m), _dp(u),
                                    act.ctypes.data_as(C.POINTER(C.c_uint32)),
                                    tie.ctypes.data_as(C.POINTER(C.c_uint32)),
                                    it.ctypes.data_as(C.POINTER(C.c_int32)))
        return u, act, tie, int(st), int(it[0])

    def mpc_move(self, Ahat, R, beta, fbar, lo, hi, m, dref=0.0):
        """NEXT-3: Eq. 9 + move suppression (cfg wmove), dense generic active set."""
        Ahat, R, fbar, lo, hi, m = map(_arr, (Ahat, R, fbar, lo, hi, m))
        u = np.zeros((self.M, self.n))
        act = np.zeros(self.M, dtype=np.uint32); tie = np.zeros(self.M, dtype=np.uint32)
        it = np.zeros(1, dtype=np.int32)
        st = self.L.ora_mpc_move_ref(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), float(dref), _dp(fbar),
                                     _dp(lo), _dp(hi),
                                 _dp(m), _dp(u), act.ctypes.data_as(C.POINTER(C.c_uint32)),
                                 tie.ctypes.data_as(C.POINTER(C.c_uint32)), it.ctypes.data_as(C.POINTER(C.c_int32)))
        return u, act, tie, int(st), int(it[0])

    def mpc_move_bruteforce(self, Ahat, R, beta, fbar, lo, hi, m):
        Ahat, R, fbar, lo, hi, m = map(_arr, (Ahat, R, fbar, lo, hi, m))
        u = np.zeros((self.M, self.n))
        rc = self.L.ora_mpc_move_bruteforce(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), _dp(fbar), _dp(lo),
                                            _dp(hi), _dp(m), _dp(u))
        if rc != 0:
            raise ValueError("bruteforce needs M*N <= 10")
        return u

    def mpc_move_cost(self, Ahat, R, beta, fbar, m, u):
        Ahat, R, fbar, m, u = map(_arr, (Ahat, R, fbar, m, u))
        return self.L.ora_mpc_move_cost(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), _dp(fbar), _dp(m), _dp(u))

    def mpc_bruteforce(self, Ahat, R, beta, lo, hi, m, dref=0.0, fbar=None):
        Ahat, R, lo, hi, m = map(_arr, (Ahat, R, lo, hi, m))
        u = np.zeros((self.M, self.n))
        fb = _dp(_arr(fbar)) if fbar is not None else None
        rc = self.L.ora_mpc_bruteforce_ref(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), float(dref), fb,
                                           _dp(lo), _dp(hi), _dp(m), _dp(u))
        if rc != 0:
            raise ValueError("bruteforce needs M*N <= 10")
        return u

    def mpc_cost(self, Ahat, R, beta, m, u, dref=0.0):
        Ahat, R, m, u = map(_arr, (Ahat, R, m, u))
        return self.L.ora_mpc_cost_ref(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), float(dref), _dp(m),
                                       _dp(u))

    def ref_pow(self, i):
        return self.L.ora_ref_pow(C.byref(self.cfg), int(i))

    def classify(self, Ahat, R, beta, lo, hi, m, u, dref=0.0):
        Ahat, R, lo, hi, m, u = map(_arr, (Ahat, R, lo, hi, m, u))
        act = np.zeros(self.M, dtype=np.uint32); tie = np.zeros(self.M, dtype=np.uint32)
        self.L.ora_mpc_classify_ref(C.byref(self.cfg), _dp(Ahat), _dp(R), float(beta), float(dref), _dp(lo),
                                _dp(hi), _dp(m), _dp(u),
                                act.ctypes.data_as(C.POINTER(C.c_uint32)),
                                tie.ctypes.data_as(C.POINTER(C.c_uint32)))
        return act, tie

    # ---- S4
    def plant_step(self, a_true, c_true, thr_max, dem, noise, u0, acc):
        a_true, thr_max, dem, u0 = map(_arr, (a_true, thr_max, dem, u0))
        acc = _arr(acc).copy()
        fbar, thr = np.zeros(self.n), np.zeros(self.n)
        p = np.zeros(1)
        lv = np.zeros((self.S, self.n), dtype=np.uint8)
        self.L.ora_plant_step(C.byref(self.cfg), _dp(a_true), float(c_true), _dp(thr_max),
                              _dp(dem), float(noise), _dp(u0), _dp(acc), _dp(fbar), _dp(p),
                              _dp(thr), lv.ctypes.data_as(C.POINTER(C.c_uint8)))
        return fbar, float(p[0]), thr, acc, lv

    # ---- generator
    def gen_server(self, server):
        n = self.n
        a, thr_max, base, amp = np.zeros(n), np.zeros(n), np.zeros(n), np.zeros(n)
        ct = np.zeros(1)
        self.L.ora_gen_server(C.byref(self.cfg), server, _dp(a), _dp(ct), _dp(thr_max), _dp(base), _dp(amp))
        return dict(a_true=a, c_true=float(ct[0]), thr_max=thr_max, base=base, amp=amp)

    def gen_noise(self, server, k):
        return self.L.ora_gen_noise(C.byref(self.cfg), server, k)

    def gen_demand(self, server, k, periods=None):
        w = make_workload(self.desc, periods)
        dem = np.zeros(self.n)
        self.L.ora_gen_demand(C.byref(self.cfg), C.byref(w), server, k, _dp(dem))
        return dem

    def gen_cap_base(self, server, cap_idx=0):
        w = make_workload(self.desc)
        return self.L.ora_gen_cap_base(C.byref(self.cfg), C.byref(w), server, cap_idx)

    # ---- closed loop
    def simulate(self, inst, periods=None, caps_override=None, definition_mode=False, traces=True):
        inst = np.ascontiguousarray(np.asarray(inst, dtype=np.int64))
        ni = len(inst)
        w = make_workload(self.desc, periods)
        K, n, M, S = w.periods, self.n, self.M, self.S
        out = {}
        if traces:
            out = dict(p=np.zeros((K, ni)), cap=np.zeros((K, ni)), u=np.zeros((K, ni, M, n)),
                       active=np.zeros((K, ni, M), dtype=np.uint32),
                       tie=np.zeros((K, ni, M), dtype=np.uint32),
                       rank=np.zeros((K, ni, n), dtype=np.int8),
                       levels=np.zeros((K, ni, S, n), dtype=np.uint8),
                       ahat=np.zeros((K, ni, n)), theta=np.zeros((K, ni, n)),
                       status=np.zeros((K, ni), dtype=np.uint32))
        final_p = np.zeros(ni)
        summ = (OraSummary * ni)()
        A0 = np.zeros((ni, n))
        co = None
        if caps_override is not None:
            co = np.ascontiguousarray(np.asarray(caps_override, dtype=np.float64))
            assert co.shape == (K, ni)

        def P(name, ct=C.c_double):
            return out[name].ctypes.data_as(C.POINTER(ct)) if traces else None

        rc = self.L.ora_simulate(C.byref(self.cfg), C.byref(w), ni,
                                 inst.ctypes.data_as(C.POINTER(C.c_int64)),
                                 _dp(co) if co is not None else None,
                                 P("p"), P("cap"), P("u"), P("active", C.c_uint32),
                                 P("tie", C.c_uint32), P("rank", C.c_int8), P("levels", C.c_uint8),
                                 P("ahat"), P("theta"), P("status", C.c_uint32), _dp(final_p),
                                 summ, _dp(A0), int(definition_mode))
        if rc != 0:
            raise RuntimeError(f"ora_simulate rc={rc}")
        out["final_p"] = final_p
        out["A0"] = A0
        out["summary"] = summaries_to_numpy(summ, M)
        return out

    def simulate_baseline(self, inst, periods=None, traces=True):
        """NEXT-2 baseline controller of the workload (controller 1..5) on the same plant."""
        inst = np.ascontiguousarray(np.asarray(inst, dtype=np.int64))
        ni = len(inst)
        w = make_workload(self.desc, periods)
        K, n, S = w.periods, self.n, self.S
        out = {}
        if traces:
            out = dict(p=np.zeros((K, ni)), cap=np.zeros((K, ni)), u=np.zeros((K, ni, n)),
                       levels=np.zeros((K, ni, S, n), dtype=np.uint8), theta=np.zeros((K, ni, n)))
        final_p = np.zeros(ni)
        summ = (OraSummary * ni)()

        def P(name, ct=C.c_double):
            return out[name].ctypes.data_as(C.POINTER(ct)) if traces else None

        rc = self.L.ora_simulate_baseline(C.byref(self.cfg), C.byref(w), ni, inst.ctypes.data_as(C.POINTER(C.c_int64)),
                                          P("p"), P("cap"), P("u"), P("levels", C.c_uint8), P("theta"),
                                          _dp(final_p), summ)
        if rc != 0:
            raise RuntimeError(f"ora_simulate_baseline rc={rc}")
        out["final_p"] = final_p
        out["summary"] = summaries_to_numpy(summ, self.M)
        return out

    def simulate_hier(self, n_servers, tr_srv, periods=None, W_replay=None, W0_replay=0.0, n_total=None):
        """cfg 4 hierarchical budget, every server stepping together (Q16).
        Replay mode (W_replay given): simulate only servers [0, n_servers) of an
        n_total-server cluster, taking the cluster sums W(k) from W_replay."""
        wl = self.desc["workload"]
        w = make_workload(self.desc, periods)
        K, n, M, S = w.periods, self.n, self.M, self.S
        tr_srv = np.ascontiguousarray(np.asarray(tr_srv, dtype=np.int64))
        nt = len(tr_srv)
        out = dict(p=np.zeros((K, nt)), cap=np.zeros((K, nt)), u=np.zeros((K, nt, M, n)),
                   active=np.zeros((K, nt, M), dtype=np.uint32), tie=np.zeros((K, nt, M), dtype=np.uint32),
                   levels=np.zeros((K, nt, S, n), dtype=np.uint8), theta=np.zeros((K, nt, n)),
                   agg_W=np.zeros(K), agg_P=np.zeros(K), final_p=np.zeros(n_servers))
        wr = None if W_replay is None else np.ascontiguousarray(np.asarray(W_replay, dtype=np.float64))
        u32 = C.POINTER(C.c_uint32)
        rc = self.L.ora_simulate_hier(C.byref(self.cfg), C.byref(w), n_servers, wl.get("rack", 16),
                                      wl.get("cluster_frac", 0.55), wl.get("rack_frac", 0.9),
                                      _dp(wr) if wr is not None else None, float(W0_replay),
                                      int(n_total if n_total is not None else n_servers), nt,
                                      tr_srv.ctypes.data_as(C.POINTER(C.c_int64)), _dp(out["p"]), _dp(out["cap"]),
                                      _dp(out["u"]), out["active"].ctypes.data_as(u32),
                                      out["tie"].ctypes.data_as(u32),
                                      out["levels"].ctypes.data_as(C.POINTER(C.c_uint8)), _dp(out["theta"]),
                                      _dp(out["agg_W"]),
                                      _dp(out["agg_P"]), _dp(out["final_p"]))
        if rc != 0:
            raise RuntimeError(f"ora_simulate_hier rc={rc}")
        return out

    def budget_caps(self, pmin, w, W, B_c, pmin_tot, B_rack_max, rack):
        pmin, w, B_rack_max = map(_arr, (pmin, w, B_rack_max))
        cap = np.zeros(len(pmin))
        self.L.ora_budget_caps(len(pmin), rack, _dp(pmin), _dp(w), float(W), float(B_c),
                               float(pmin_tot), _dp(B_rack_max), _dp(cap))
        return cap


def summaries_to_numpy(summ, M):
    ni = len(summ)
    d = dict(sum_p=np.zeros(ni), sumsq_p=np.zeros(ni), max_p=np.zeros(ni), sum_theta=np.zeros(ni),
             n_window=np.zeros(ni, dtype=np.int32), n_viol=np.zeros(ni, dtype=np.int32),
             act_count=np.zeros((ni, M), dtype=np.int32), n_miss=np.zeros(ni, dtype=np.int32))
    for i, s in enumerate(summ):
        d["sum_p"][i], d["sumsq_p"][i], d["max_p"][i] = s.sum_p, s.sumsq_p, s.max_p
        d["sum_theta"][i], d["n_window"][i], d["n_viol"][i] = s.sum_theta, s.n_window, s.n_viol
        d["act_count"][i] = list(s.act_count)[:M]
        d["n_miss"][i] = s.n_miss
    return d


def oracle_for(cfg: int, **overrides) -> Oracle:
    return Oracle(configs.get(cfg, **overrides))
