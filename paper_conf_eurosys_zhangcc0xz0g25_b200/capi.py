"""ctypes binding of the C ABI in include/bless/bless.h (same names).

Argument marshalling only: every step of the hot path runs in the native
library ``lib/libbless.so`` (scheduler, launches, kernels).  Loading fails
loudly if the library is missing -- there is no Python or CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libbless.so")

BL_MAX_TENANTS = 16
BL_MAX_SQUAD = 128
BL_DEVICE_NONE = -1

# bl_status
BL_OK, BL_PENDING = 0, 1
BL_E_INVALID, BL_E_QUOTA, BL_E_STATE, BL_E_CUDA, BL_E_OOM, BL_E_FULL, BL_E_NOTFOUND, BL_E_TIMEOUT = \
    -1, -2, -3, -4, -5, -6, -7, -8
STATUS_NAMES = {0: "BL_OK", 1: "BL_PENDING", -1: "BL_E_INVALID", -2: "BL_E_QUOTA", -3: "BL_E_STATE",
                -4: "BL_E_CUDA", -5: "BL_E_OOM", -6: "BL_E_FULL", -7: "BL_E_NOTFOUND", -8: "BL_E_TIMEOUT"}
# bl_policy / bl_clock
BL_POLICY_BLESS, BL_POLICY_ISO, BL_POLICY_STATIC, BL_POLICY_TEMPORAL, BL_POLICY_UNBOUND = 0, 1, 2, 3, 4
POLICIES = {"BLESS": 0, "ISO": 1, "STATIC": 2, "TEMPORAL": 3, "UNBOUND": 4}
BL_CLOCK_WALL, BL_CLOCK_VIRTUAL = 0, 1
# ops
BL_OP_GEMM, BL_OP_CONV, BL_OP_POOL, BL_OP_ELTWISE, BL_OP_IM2COL, BL_OP_VIRTUAL = 0, 1, 2, 3, 4, 15
BL_OP_LAYERNORM, BL_OP_ATTENTION, BL_OP_EMBED, BL_OP_DWCONV = 5, 6, 7, 8
BL_F32, BL_BF16 = 0, 1
BL_ACT_NONE, BL_ACT_RELU, BL_ACT_RELU6, BL_ACT_GELU = 0, 1, 2, 3
ACTS = {"none": 0, "relu": 1, "relu6": 2, "gelu": 3}
BL_POOL_MAX, BL_POOL_AVG, BL_POOL_GLOBAL_AVG = 0, 1, 2


class bl_params(C.Structure):
    _fields_ = [("sm_unit", C.c_int32), ("squad_max", C.c_int32), ("split_pct", C.c_int32),
                ("seed_all", C.c_int32), ("policy", C.c_int32), ("clock", C.c_int32),
                ("squad_overhead_ns", C.c_int64), ("temporal_period_ns", C.c_int64),
                ("temporal_work_conserving", C.c_int32), ("max_inflight_squads", C.c_int32),
                ("lookahead_ns", C.c_int64), ("max_requests", C.c_int64),
                ("ablate", C.c_int32), ("sm_limit", C.c_int32),
                ("squad_max_solo", C.c_int32), ("barrier", C.c_int32)]


class bl_op(C.Structure):
    _fields_ = [("kind", C.c_int32), ("dtype", C.c_int32), ("act", C.c_int32), ("flags", C.c_int32),
                ("dims", C.c_int64 * 12), ("ptr", C.c_void_p * 8), ("fparam", C.c_float * 4)]


class bl_req_info(C.Structure):
    _fields_ = [("req", C.c_uint64), ("tenant", C.c_int32), ("status", C.c_int32),
                ("arrival_ns", C.c_int64), ("start_ns", C.c_int64), ("finish_ns", C.c_int64)]


class bl_decision(C.Structure):
    _fields_ = [("now", C.c_int64), ("t_hat", C.c_int64), ("t_nsp", C.c_int64),
                ("n_active", C.c_int32), ("n_part", C.c_int32), ("config_sp", C.c_int32), ("n_picks", C.c_int32),
                ("act_tenant", C.c_int32 * BL_MAX_TENANTS), ("act_next", C.c_int32 * BL_MAX_TENANTS),
                ("act_arrival", C.c_int64 * BL_MAX_TENANTS),
                ("part_tenant", C.c_int32 * BL_MAX_TENANTS), ("part_p", C.c_int32 * BL_MAX_TENANTS),
                ("pick_tenant", C.c_int32 * BL_MAX_SQUAD), ("pick_kernel", C.c_int32 * BL_MAX_SQUAD),
                ("pick_lo", C.c_int16 * BL_MAX_SQUAD), ("pick_hi", C.c_int16 * BL_MAX_SQUAD)]


class bl_launch_rec(C.Structure):
    _fields_ = [("seq", C.c_uint64), ("tenant", C.c_int32), ("kernel", C.c_int32),
                ("lo", C.c_int16), ("hi", C.c_int16), ("nsm", C.c_int32), ("fallback", C.c_int32),
                ("start_ns", C.c_int64), ("end_ns", C.c_int64), ("req", C.c_uint64),
                ("sm_mask", C.c_uint32 * 8)]


class bl_temporal_rec(C.Structure):
    _fields_ = [("t", C.c_int64), ("gpu_free", C.c_int64), ("slice_end", C.c_int64), ("dur", C.c_int64),
                ("sid", C.c_int64), ("last_sid", C.c_int64), ("turn_end", C.c_int64), ("turn", C.c_int32),
                ("work_mask", C.c_int32), ("tenant", C.c_int32), ("kernel", C.c_int32),
                ("work_conserving", C.c_int32), ("reserved", C.c_int32)]


class bl_dispatch_entry(C.Structure):
    _fields_ = [("ctx", C.c_int32), ("tenant", C.c_int32), ("arrival_ns", C.c_int64)]


class bl_kernel_info(C.Structure):
    _fields_ = [("family", C.c_char * 32), ("tiles", C.c_int32), ("grid", C.c_int32), ("block", C.c_int32),
                ("smem", C.c_int32), ("flops", C.c_double), ("bytes", C.c_double)]


class bl_device_info(C.Structure):
    _fields_ = [("device", C.c_int32), ("sm_count", C.c_int32), ("max_smid", C.c_int32),
                ("cc_major", C.c_int32), ("cc_minor", C.c_int32), ("tpc_pairs_found", C.c_int32),
                ("globaltimer_res_ns", C.c_int64), ("clock_offset_ns", C.c_int64),
                ("l2_bytes", C.c_int64), ("smem_per_block_optin", C.c_int64),
                ("smid_to_lid", C.c_uint8 * 256)]


class BlessError(RuntimeError):
    def __init__(self, fn, status, msg):
        super().__init__(f"{fn} -> {STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


_P = C.POINTER
_SIGS = {
    "bl_params_default": (None, [_P(bl_params)]),
    "bl_create": (C.c_int, [C.c_int, _P(bl_params), C.c_void_p, C.c_size_t, _P(C.c_void_p)]),
    "bl_destroy": (C.c_int, [C.c_void_p]),
    "bl_device_info_get": (C.c_int, [C.c_void_p, _P(bl_device_info)]),
    "bl_register_tenant": (C.c_int, [C.c_void_p, C.c_double, C.c_char_p, _P(C.c_int)]),
    "bl_set_stream": (C.c_int, [C.c_void_p, C.c_int, C.c_void_p]),
    "bl_set_tenant_slo": (C.c_int, [C.c_void_p, C.c_int, C.c_int64]),
    "bl_append_kernel": (C.c_int, [C.c_void_p, C.c_int, _P(bl_op), _P(C.c_int)]),
    "bl_run_kernel": (C.c_int, [C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int]),
    "bl_set_tenant_io": (C.c_int, [C.c_void_p, C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p,
                                   C.c_void_p, C.c_size_t]),
    "bl_kernel_info_get": (C.c_int, [C.c_void_p, C.c_int, C.c_int, _P(bl_kernel_info)]),
    "bl_profile_kernel": (C.c_int, [C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int, _P(C.c_int64), _P(C.c_int)]),
    "bl_profile_tenant": (C.c_int, [C.c_void_p, C.c_int, C.c_int]),
    "bl_set_profile_row": (C.c_int, [C.c_void_p, C.c_int, C.c_int, _P(C.c_int64), C.c_int]),
    "bl_get_profile_row": (C.c_int, [C.c_void_p, C.c_int, C.c_int, _P(C.c_int64), _P(C.c_int)]),
    "bl_save_profile": (C.c_int, [C.c_void_p, C.c_char_p]),
    "bl_load_profile": (C.c_int, [C.c_void_p, C.c_char_p]),
    "bl_tenant_info": (C.c_int, [C.c_void_p, C.c_int, _P(C.c_int), _P(C.c_int), _P(C.c_int64)]),
    "bl_start": (C.c_int, [C.c_void_p]),
    "bl_submit": (C.c_int, [C.c_void_p, C.c_int, C.c_int64, _P(C.c_uint64)]),
    "bl_poll": (C.c_int, [C.c_void_p, C.c_uint64, _P(bl_req_info)]),
    "bl_drain": (C.c_int, [C.c_void_p, C.c_int64]),
    "bl_stop": (C.c_int, [C.c_void_p]),
    "bl_decisions": (C.c_int, [C.c_void_p, C.c_size_t, _P(bl_decision), C.c_size_t, _P(C.c_size_t)]),
    "bl_launches": (C.c_int, [C.c_void_p, C.c_size_t, _P(bl_launch_rec), C.c_size_t, _P(C.c_size_t)]),
    "bl_reset": (C.c_int, [C.c_void_p, _P(bl_params)]),
    "bl_decide": (C.c_int, [C.c_void_p, C.c_int64, C.c_int, _P(C.c_int32), _P(C.c_int64), _P(C.c_int32),
                            _P(bl_decision)]),
    "bl_temporal_log": (C.c_int, [C.c_void_p, C.c_size_t, _P(bl_temporal_rec), C.c_size_t, _P(C.c_size_t)]),
    "bl_time_decide": (C.c_int, [C.c_void_p, _P(bl_decision), C.c_size_t, C.c_int, _P(C.c_int64), _P(C.c_int64)]),
    "bl_dispatch": (C.c_int, [_P(C.c_void_p), C.c_int, _P(bl_dispatch_entry), C.c_size_t, C.c_int64,
                              _P(C.c_uint64)]),
    "bl_predict": (C.c_int, [C.c_void_p, C.c_int, _P(C.c_int32), _P(C.c_int32), _P(C.c_int32), _P(C.c_int64)]),
    "bl_run_squad": (C.c_int, [C.c_void_p, C.c_int, _P(C.c_int32), _P(C.c_int32), _P(C.c_int16), _P(C.c_int16),
                               C.c_int, _P(C.c_int64), _P(C.c_int64)]),
    "bl_deployment_check": (C.c_int, [C.c_void_p, _P(C.c_int64), C.c_int64, C.c_int32, _P(C.c_int32),
                                      _P(C.c_int32)]),
    "bl_place": (C.c_int, [C.c_int, _P(C.c_int64), _P(C.c_int64), C.c_int, _P(C.c_int64), C.c_int32,
                           _P(C.c_int32)]),
    "bl_debug_overhead": (C.c_int, [C.c_void_p, C.c_int, C.c_int, _P(C.c_int64)]),
    "bl_debug_chain": (C.c_int, [C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, _P(C.c_int64),
                                 _P(C.c_int64)]),
    "bl_now_ns": (C.c_int64, []),
    "bl_last_error": (C.c_char_p, []),
    "bl_version": (C.c_char_p, []),
}

_lib = None


def lib():
    """Load libbless.so (raises if it was not built -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"native library missing: {LIB_PATH} (run __graft_entry__.build())")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def exported_symbols():
    return list(_SIGS)


def check(fn: str, status: int, allow=(BL_OK,)):
    if status not in allow:
        raise BlessError(fn, status, (lib().bl_last_error() or b"").decode())
    return status


def default_params(**kw) -> bl_params:
    p = bl_params()
    lib().bl_params_default(C.byref(p))
    for k, v in kw.items():
        if k == "policy" and isinstance(v, str):
            v = POLICIES[v]
        setattr(p, k, int(v))
    return p


class Ctx:
    """One bl_ctx (one GPU, or BL_DEVICE_NONE).  Thin RAII wrapper."""

    def __init__(self, device: int = 0, params: bl_params | None = None, **kw):
        self.params = params or default_params(**kw)
        h = C.c_void_p()
        check("bl_create", lib().bl_create(device, C.byref(self.params), None, 0, C.byref(h)))
        self.h = h
        self.device = device

    def close(self):
        if getattr(self, "h", None):
            lib().bl_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # setup -------------------------------------------------------------
    def device_info(self) -> bl_device_info:
        out = bl_device_info()
        check("bl_device_info_get", lib().bl_device_info_get(self.h, C.byref(out)))
        return out

    def register_tenant(self, quota: float, name: str) -> int:
        t = C.c_int()
        check("bl_register_tenant", lib().bl_register_tenant(self.h, float(quota), name.encode(), C.byref(t)))
        return t.value

    def set_slo(self, tenant: int, slo_ns: int):
        check("bl_set_tenant_slo", lib().bl_set_tenant_slo(self.h, tenant, int(slo_ns)))

    def set_stream(self, tenant: int, stream_ptr: int):
        check("bl_set_stream", lib().bl_set_stream(self.h, tenant, C.c_void_p(stream_ptr)))

    def append_kernel(self, tenant: int, op: bl_op) -> int:
        k = C.c_int()
        check("bl_append_kernel", lib().bl_append_kernel(self.h, tenant, C.byref(op), C.byref(k)))
        return k.value

    def run_kernel(self, tenant: int, k: int, lo: int = 0, hi: int = 1 << 15):
        check("bl_run_kernel", lib().bl_run_kernel(self.h, tenant, k, lo, hi))

    def set_tenant_io(self, tenant: int, host_in: int, dev_in: int, in_bytes: int, dev_out: int, host_out: int,
                      out_bytes: int):
        check("bl_set_tenant_io", lib().bl_set_tenant_io(self.h, tenant, C.c_void_p(host_in), C.c_void_p(dev_in),
                                                         in_bytes, C.c_void_p(dev_out), C.c_void_p(host_out),
                                                         out_bytes))

    def debug_overhead(self, variant: int, reps: int = 200) -> int:
        ns = C.c_int64()
        check("bl_debug_overhead", lib().bl_debug_overhead(self.h, variant, reps, C.byref(ns)))
        return ns.value

    def debug_chain(self, tenant: int, lo: int, hi: int, graph: int, reps: int = 5):
        dv, hv = C.c_int64(), C.c_int64()
        check("bl_debug_chain", lib().bl_debug_chain(self.h, tenant, lo, hi, graph, reps, C.byref(dv), C.byref(hv)))
        return dv.value, hv.value

    def kernel_info(self, tenant: int, k: int) -> bl_kernel_info:
        out = bl_kernel_info()
        check("bl_kernel_info_get", lib().bl_kernel_info_get(self.h, tenant, k, C.byref(out)))
        return out

    def profile_kernel(self, tenant: int, k: int, sm_count: int, reps: int = 10):
        ns, d = C.c_int64(), C.c_int()
        check("bl_profile_kernel", lib().bl_profile_kernel(self.h, tenant, k, sm_count, reps, C.byref(ns), C.byref(d)))
        return ns.value, d.value

    def profile_tenant(self, tenant: int, reps: int = 10):
        check("bl_profile_tenant", lib().bl_profile_tenant(self.h, tenant, reps))

    def set_profile_row(self, tenant: int, k: int, t_ns, d: int):
        arr = (C.c_int64 * len(t_ns))(*[int(v) for v in t_ns])
        check("bl_set_profile_row", lib().bl_set_profile_row(self.h, tenant, k, arr, int(d)))

    def get_profile_row(self, tenant: int, k: int, S: int):
        arr = (C.c_int64 * S)()
        d = C.c_int()
        check("bl_get_profile_row", lib().bl_get_profile_row(self.h, tenant, k, arr, C.byref(d)))
        return list(arr), d.value

    def save_profile(self, path: str):
        check("bl_save_profile", lib().bl_save_profile(self.h, path.encode()))

    def load_profile(self, path: str):
        check("bl_load_profile", lib().bl_load_profile(self.h, path.encode()))

    def tenant_info(self, tenant: int):
        q, m, T = C.c_int(), C.c_int(), C.c_int64()
        check("bl_tenant_info", lib().bl_tenant_info(self.h, tenant, C.byref(q), C.byref(m), C.byref(T)))
        return q.value, m.value, T.value

    # runtime -----------------------------------------------------------
    def start(self):
        check("bl_start", lib().bl_start(self.h))

    def submit(self, tenant: int, arrival_ns: int) -> int:
        r = C.c_uint64()
        check("bl_submit", lib().bl_submit(self.h, tenant, int(arrival_ns), C.byref(r)))
        return r.value

    def poll(self, req: int):
        info = bl_req_info()
        st = lib().bl_poll(self.h, req, C.byref(info))
        check("bl_poll", st, allow=(BL_OK, BL_PENDING))
        return st, info

    def drain(self, timeout_ns: int = -1):
        check("bl_drain", lib().bl_drain(self.h, int(timeout_ns)))

    def stop(self):
        check("bl_stop", lib().bl_stop(self.h))

    def reset(self, params: bl_params | None = None):
        if params is not None:
            self.params = params
        check("bl_reset", lib().bl_reset(self.h, C.byref(self.params) if params is not None else None))

    def decisions(self):
        n = C.c_size_t()
        lib().bl_decisions(self.h, 0, None, 0, C.byref(n))
        buf = (bl_decision * max(1, n.value))()
        got = C.c_size_t()
        lib().bl_decisions(self.h, 0, buf, n.value, C.byref(got))
        return [buf[i] for i in range(got.value)]

    def launches(self):
        n = C.c_size_t()
        lib().bl_launches(self.h, 0, None, 0, C.byref(n))
        buf = (bl_launch_rec * max(1, n.value))()
        got = C.c_size_t()
        lib().bl_launches(self.h, 0, buf, n.value, C.byref(got))
        return [buf[i] for i in range(got.value)]

    def temporal_log(self):
        n = C.c_size_t()
        lib().bl_temporal_log(self.h, 0, None, 0, C.byref(n))
        buf = (bl_temporal_rec * max(1, n.value))()
        got = C.c_size_t()
        lib().bl_temporal_log(self.h, 0, buf, n.value, C.byref(got))
        return [buf[i] for i in range(got.value)]

    def time_decide(self, recs, reps: int = 1):
        """Native timing of decide() on logged records: (total_ns, total_picks)."""
        arr = (bl_decision * max(1, len(recs)))(*recs)
        ns, picks = C.c_int64(), C.c_int64()
        check("bl_time_decide", lib().bl_time_decide(self.h, arr, len(recs), int(reps), C.byref(ns), C.byref(picks)))
        return ns.value, picks.value

    def predict(self, picks, p=None) -> int:
        """Eq. 2 (p None, NSP) or Eq. 1 for split p of a squad [(tenant, kernel)]."""
        n = len(picks)
        t = (C.c_int32 * n)(*[x[0] for x in picks])
        k = (C.c_int32 * n)(*[x[1] for x in picks])
        pp = (C.c_int32 * len(p))(*p) if p is not None else None
        out = C.c_int64()
        check("bl_predict", lib().bl_predict(self.h, n, t, k, pp, C.byref(out)))
        return out.value

    def run_squad(self, picks, reps: int = 3):
        """Execute a squad [(tenant, kernel, lo, hi)]: (median makespan ns, per-pick ns)."""
        n = len(picks)
        t = (C.c_int32 * n)(*[x[0] for x in picks])
        k = (C.c_int32 * n)(*[x[1] for x in picks])
        lo = (C.c_int16 * n)(*[x[2] for x in picks])
        hi = (C.c_int16 * n)(*[x[3] for x in picks])
        ms = C.c_int64()
        kn = (C.c_int64 * n)()
        check("bl_run_squad", lib().bl_run_squad(self.h, n, t, k, lo, hi, int(reps), C.byref(ms), kn))
        return ms.value, list(kn)

    def deployment_check(self, mem_bytes, free_bytes: int = 0, span_x: int = 30):
        """(admissible, reason): reason 0 ok, 1 kernel-duration span, 2 memory (R33)."""
        m = (C.c_int64 * len(mem_bytes))(*[int(x) for x in mem_bytes])
        ok, why = C.c_int32(), C.c_int32()
        check("bl_deployment_check", lib().bl_deployment_check(self.h, m, int(free_bytes), int(span_x),
                                                               C.byref(ok), C.byref(why)))
        return bool(ok.value), why.value

    def decide(self, now: int, active):
        """active: list of (tenant, arrival, next_kernel)."""
        n = len(active)
        t = (C.c_int32 * n)(*[a[0] for a in active])
        a = (C.c_int64 * n)(*[a[1] for a in active])
        k = (C.c_int32 * n)(*[a[2] for a in active])
        out = bl_decision()
        check("bl_decide", lib().bl_decide(self.h, int(now), n, t, a, k, C.byref(out)))
        return out


def now_ns() -> int:
    return lib().bl_now_ns()


def place(mem_bytes, avg_kernel_ns, gpu_free_bytes, span_x: int = 30):
    """Tenant -> GPU placement (bl_place, L171, R33): list of GPU indices (-1 = none)."""
    n, G = len(mem_bytes), len(gpu_free_bytes)
    out = (C.c_int32 * max(1, n))()
    check("bl_place", lib().bl_place(n, (C.c_int64 * max(1, n))(*[int(x) for x in mem_bytes]),
                                     (C.c_int64 * max(1, n))(*[int(x) for x in avg_kernel_ns]), G,
                                     (C.c_int64 * max(1, G))(*[int(x) for x in gpu_free_bytes]), int(span_x), out))
    return [out[i] for i in range(n)]


def dispatch(ctxs, entries, base_ns: int = 0):
    """Box-wide trace dispatcher (bl_dispatch): entries = [(ctx_index, tenant,
    arrival_ns)] sorted by arrival; returns the request ids.  Blocks (busy-waits
    in native code, GIL released) until every entry is submitted."""
    hs = (C.c_void_p * len(ctxs))(*[c.h.value for c in ctxs])
    ent = (bl_dispatch_entry * max(1, len(entries)))(*[bl_dispatch_entry(int(c), int(t), int(a))
                                                        for c, t, a in entries])
    out = (C.c_uint64 * max(1, len(entries)))()
    check("bl_dispatch", lib().bl_dispatch(hs, len(ctxs), ent, len(entries), int(base_ns), out))
    return [out[i] for i in range(len(entries))]


def decision_to_tuple(d: bl_decision):
    """Flatten a record to comparable plain values."""
    picks = [(d.pick_tenant[i], d.pick_kernel[i], d.pick_lo[i], d.pick_hi[i]) for i in range(d.n_picks)]
    parts = [d.part_tenant[i] for i in range(d.n_part)]
    cfg = tuple(d.part_p[i] for i in range(d.n_part)) if d.config_sp else None
    active = [(d.act_tenant[i], d.act_arrival[i], d.act_next[i]) for i in range(d.n_active)]
    return {"now": d.now, "active": active, "picks": picks, "parts": parts, "config": cfg,
            "t_hat": d.t_hat, "t_nsp": d.t_nsp}
