"""Thin ctypes binding of libtsplit.so (include/ts.h).  Argument marshalling only:
every step of the hot path runs inside the library.  Fails loudly when the
library is missing — there is no CPU fallback."""

from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# (TSPLIT_LIB: another in-tree build of the same library, for same-box A/B timing runs)
LIB_PATH = os.environ.get("TSPLIT_LIB") or os.path.join(_PKG, "libtsplit.so")

OPS = {"linear": 0, "relu": 1, "gelu": 2, "tanh": 3, "layernorm": 4, "add": 5, "dropout": 6,
       "softmax": 7, "attn_qk": 8, "attn_pv": 9, "embed": 10, "cls": 11, "xent": 12,
       "conv2d": 13, "batchnorm": 14, "maxpool": 15, "avgpool": 16, "flatten": 17, "attention": 18}
DTYPES = {"f32": 0, "bf16": 1, "i32": 2}
KINDS = {"param": 0, "input": 1, "label": 2, "act": 3}
RESIDE, SWAP, RECOMPUTE = 0, 1, 2
STATUS = ["OK", "ERR_ARG", "ERR_GRAPH", "ERR_INFEASIBLE", "ERR_BUDGET", "ERR_HOST_MEM",
          "ERR_CUDA", "ERR_NCCL", "ERR_STATE", "ERR_NO_GPU"]


class TensorDesc(C.Structure):
    _fields_ = [("dtype", C.c_int32), ("kind", C.c_int32), ("ndim", C.c_int32), ("shape", C.c_int64 * 6)]


class OpDesc(C.Structure):
    _fields_ = [("kind", C.c_int32), ("n_in", C.c_int32), ("n_out", C.c_int32),
                ("inp", C.POINTER(C.c_int32)), ("out", C.POINTER(C.c_int32)),
                ("n_iattr", C.c_int32), ("iattr", C.POINTER(C.c_int64)),
                ("n_fattr", C.c_int32), ("fattr", C.POINTER(C.c_double))]


class TensorCfg(C.Structure):
    _fields_ = [("tensor_id", C.c_int32), ("opt", C.c_int32), ("p_num", C.c_int32), ("dim", C.c_int32),
                ("prefetch_lead", C.c_int32), ("release_lag", C.c_int32)]


class PlanStats(C.Structure):
    _fields_ = [("static_bytes", C.c_uint64), ("peak_live", C.c_uint64), ("peak_extent", C.c_uint64),
                ("d2h_bytes", C.c_uint64), ("h2d_bytes", C.c_uint64), ("n_items", C.c_int64),
                ("n_compute", C.c_int64), ("n_replay", C.c_int64), ("predicted_s", C.c_double),
                ("compute_flop", C.c_double), ("n_split_tensors", C.c_int64), ("n_swap_tensors", C.c_int64),
                ("n_recompute_tensors", C.c_int64), ("recompute_cache_bytes", C.c_uint64)]


class AllocEvent(C.Structure):
    _fields_ = [("seq", C.c_int64), ("item", C.c_int32), ("kind", C.c_int32), ("key", C.c_int32),
                ("piece", C.c_int32), ("offset", C.c_uint64), ("bytes", C.c_uint64)]


class Hw(C.Structure):
    _fields_ = [("tensor_flops", C.c_double), ("simt_flops", C.c_double), ("hbm_bw", C.c_double),
                ("d2h_bw", C.c_double), ("h2d_bw", C.c_double), ("launch_s", C.c_double)]


class SessionCfg(C.Structure):
    _fields_ = [("device", C.c_int32), ("slab", C.c_void_p), ("slab_bytes", C.c_uint64),
                ("stream_compute", C.c_void_p), ("stream_d2h", C.c_void_p), ("stream_h2d", C.c_void_p),
                ("nccl_comm", C.c_void_p), ("world_size", C.c_int32), ("use_cuda_graph", C.c_int32),
                ("lr", C.c_float), ("step0", C.c_uint32), ("sample_offset", C.c_int64),
                ("host_numa_node", C.c_int32), ("grad_allreduce_bf16", C.c_int32)]


class TsError(RuntimeError):
    def __init__(self, status, msg):
        self.status = STATUS[status] if 0 <= status < len(STATUS) else str(status)
        super().__init__(f"{self.status}: {msg}")


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_icde_niemyc22_b200.build` "
                              "(no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        vp, u64, i32, i64 = C.c_void_p, C.c_uint64, C.c_int32, C.c_int64
        P = C.POINTER
        sig = {
            "ts_last_error": (C.c_char_p, []),
            "ts_version": (C.c_char_p, []),
            "ts_graph_define": (i32, [P(TensorDesc), i32, P(OpDesc), i32, i32, i32, P(vp)]),
            "ts_graph_destroy": (None, [vp]),
            "ts_graph_schedule": (i32, [vp, P(i32), i32, P(i32)]),
            "ts_graph_static_bytes": (i32, [vp, P(u64)]),
            "ts_profile_analytic": (i32, [vp, P(Hw), P(vp)]),
            "ts_profile_set": (i32, [vp, i32, i32, C.c_double, C.c_double]),
            "ts_profile_set_pcie": (i32, [vp, C.c_double, C.c_double]),
            "ts_profile_destroy": (None, [vp]),
            "ts_plan_default": (i32, [vp, P(vp)]),
            "ts_plan": (i32, [vp, u64, vp, P(vp)]),
            "ts_plan_ex": (i32, [vp, C.c_uint64, vp, C.c_uint32, P(vp)]),
            "ts_plan_get": (i32, [vp, i32, P(TensorCfg)]),
            "ts_plan_set": (i32, [vp, P(TensorCfg)]),
            "ts_plan_set_many": (i32, [vp, P(TensorCfg), i32]),
            "ts_plan_stats": (i32, [vp, P(PlanStats)]),
            "ts_plan_set_recompute_cache": (i32, [vp, C.c_uint64]),
            "ts_plan_trace": (i32, [vp, P(AllocEvent), u64, P(u64)]),
            "ts_plan_items": (i32, [vp, P(i32), u64, P(u64)]),
            "ts_plan_grad_buckets": (i32, [vp, u64, P(i64), u64, P(u64)]),
            "ts_plan_serialize": (i32, [vp, vp, u64, P(u64)]),
            "ts_plan_roofline": (i32, [vp, C.c_double, C.c_double, P(C.c_double), P(C.c_double), P(C.c_double)]),
            "ts_plan_deserialize": (i32, [vp, vp, u64, P(vp)]),
            "ts_plan_destroy": (None, [vp]),
        }
        optional = {
            "ts_session_create": (i32, [vp, vp, P(SessionCfg), P(vp)]),
            "ts_session_destroy": (None, [vp]),
            "ts_set_param": (i32, [vp, i32, vp]),
            "ts_get_param": (i32, [vp, i32, vp]),
            "ts_get_grad": (i32, [vp, i32, vp]),
            "ts_param_ptr": (i32, [vp, i32, P(vp)]),
            "ts_grad_ptr": (i32, [vp, i32, P(vp)]),
            "ts_step": (i32, [vp, P(vp), i32, P(C.c_float)]),
            "ts_step_async": (i32, [vp, P(vp), i32]),
            "ts_session_trace": (i32, [vp, P(AllocEvent), u64, P(u64)]),
            "ts_session_launches": (i32, [vp, P(i64)]),
            "ts_session_host_pool": (i32, [vp, P(u64), P(i32)]),
            "ts_session_profile_items": (i32, [vp, i32]),
            "ts_session_item_times": (i32, [vp, P(C.c_float), u64, P(u64)]),
            "ts_session_gemm_times": (i32, [vp, P(C.c_double), P(C.c_float), P(i32), u64, P(u64)]),
            "ts_session_gemm_kinds": (i32, [vp, P(i32), P(i32), u64, P(u64)]),
            "ts_session_gemm_shapes": (i32, [vp, P(i32), u64, P(u64)]),
            "ts_profile_measure": (i32, [vp, vp, u64, P(vp), i32, i32, P(vp)]),
            "ts_profile_get": (i32, [vp, i32, i32, P(C.c_double), P(C.c_double)]),
            "ts_profile_pcie": (i32, [vp, P(C.c_double), P(C.c_double)]),
            "ts_nccl_unique_id": (i32, [vp]),
            "ts_nccl_comm_init": (i32, [vp, i32, i32, P(vp)]),
            "ts_nccl_comm_destroy": (i32, [vp]),
            "ts_gemm_bf16": (i32, [i32, i32, i32, i32, vp, i64, i64, i32, vp, i64, i64, i32,
                                   vp, i64, i64, i32, C.c_float, C.c_float, vp, vp]),
            "ts_gemm_bf16_grouped": (i32, [i32, i32, i32, i32, i32, P(vp), i64, i32, P(vp), i64, i32, P(vp), i64,
                                           i32, C.c_float, C.c_float, P(vp), vp]),
            "ts_gemm_bf16_epi": (i32, [i32, i32, i32, i32, vp, i64, i32, vp, i64, i32, vp, i64, C.c_float, vp, vp,
                                       i64, vp]),
            "ts_gemm_set_mode": (i32, [i32]),
            "ts_gemm_last_config": (i32, [P(i32)]),
            "ts_gemm_f32": (i32, [i32, i32, i32, vp, i64, i32, vp, i64, i32, vp, i64, C.c_float, C.c_float,
                                  vp, vp]),
            "ts_conv2d": (i32, [i32, i32, P(i32), vp, vp, vp, vp, vp, i32, vp, P(i32)]),
            "ts_row_op": (i32, [i32, i32, vp, vp, vp, i64, i32, vp, u64, i32, vp]),
            "ts_attention": (i32, [i32, i32, P(i32), P(C.c_float), vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, i32, vp,
                                   vp, P(i32)]),
        }
        for name, (res, args) in list(sig.items()) + list(optional.items()):
            if not hasattr(L, name):
                if name in sig:
                    raise ImportError(f"libtsplit.so lacks {name}")
                continue
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status):
    if status != 0:
        raise TsError(status, lib().ts_last_error().decode())


def exported_symbols():
    """Names of the ts_* functions include/ts.h declares."""
    import re
    hdr = open(os.path.join(os.path.dirname(_PKG), "include", "ts.h")).read()
    return sorted(set(re.findall(r"^\s*(?:ts_status|void|const char\*)\s+(ts_\w+)\s*\(", hdr, re.M)))


# --------------------------------------------------------------------------- graph
class Graph:
    def __init__(self, spec: dict):
        self.spec = spec
        ts, ops = spec["tensors"], spec["ops"]
        self.n = len(ts)
        td = (TensorDesc * len(ts))()
        for i, t in enumerate(ts):
            td[i].dtype = DTYPES[t["dtype"]]
            td[i].kind = KINDS[t["kind"]]
            td[i].ndim = len(t["shape"])
            for d, s in enumerate(t["shape"]):
                td[i].shape[d] = s
        od = (OpDesc * len(ops))()
        self._keep = []
        for i, o in enumerate(ops):
            ins = (C.c_int32 * len(o["inputs"]))(*o["inputs"])
            outs = (C.c_int32 * len(o["outputs"]))(*o["outputs"])
            ia = (C.c_int64 * max(1, len(o["iattrs"])))(*o["iattrs"])
            fa = (C.c_double * max(1, len(o["fattrs"])))(*o["fattrs"])
            self._keep += [ins, outs, ia, fa]
            od[i].kind = OPS[o["kind"]]
            od[i].n_in, od[i].n_out = len(o["inputs"]), len(o["outputs"])
            od[i].inp, od[i].out = ins, outs
            od[i].n_iattr, od[i].iattr = len(o["iattrs"]), ia
            od[i].n_fattr, od[i].fattr = len(o["fattrs"]), fa
        h = C.c_void_p()
        check(lib().ts_graph_define(td, len(ts), od, len(ops), spec["samples"], DTYPES[spec["dtype"]], C.byref(h)))
        self.h = h
        self.names = {t["name"]: t["id"] for t in ts}

    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().ts_graph_destroy(self.h)
        except Exception:  # interpreter teardown: the library may already be gone
            pass

    def schedule(self):
        n = C.c_int32()
        buf = (C.c_int32 * len(self.spec["ops"]))()
        check(lib().ts_graph_schedule(self.h, buf, len(buf), C.byref(n)))
        return list(buf[:n.value])

    def static_bytes(self):
        v = C.c_uint64()
        check(lib().ts_graph_static_bytes(self.h, C.byref(v)))
        return v.value


class Profile:
    def __init__(self, graph: Graph, hw: dict | None = None, _handle=None):
        self.graph = graph
        if _handle is not None:
            self.h = _handle
            return
        h = C.c_void_p()
        hwp = None
        if hw:
            hwp = C.byref(Hw(**hw))
        check(lib().ts_profile_analytic(graph.h, hwp, C.byref(h)))
        self.h = h

    @classmethod
    def measure(cls, graph: Graph, inputs: dict, max_p: int = 16, device: int = 0):
        """Measured profile (ts_profile_measure) on a scratch slab of the unsplit peak."""
        import torch
        peak = Plan.default(graph).stats()["peak_extent"]
        slab = torch.empty(peak, dtype=torch.uint8, device=f"cuda:{device}")
        ids = [t["id"] for t in graph.spec["tensors"] if t["kind"] in ("input", "label")]
        arr = (C.c_void_p * len(ids))()
        for i, tid in enumerate(ids):
            arr[i] = inputs[graph.spec["tensors"][tid]["name"]].data_ptr()
        h = C.c_void_p()
        check(lib().ts_profile_measure(graph.h, slab.data_ptr(), peak, arr, 0, max_p, C.byref(h)))
        del slab
        torch.cuda.empty_cache()
        return cls(graph, _handle=h)

    def get(self, op, p_num):
        f, b = C.c_double(), C.c_double()
        check(lib().ts_profile_get(self.h, op, p_num, C.byref(f), C.byref(b)))
        return f.value, b.value

    def pcie(self):
        d, h = C.c_double(), C.c_double()
        check(lib().ts_profile_pcie(self.h, C.byref(d), C.byref(h)))
        return d.value, h.value

    def set(self, op, p_num, fwd_s, bwd_s):
        check(lib().ts_profile_set(self.h, op, p_num, fwd_s, bwd_s))

    def set_pcie(self, d2h, h2d):
        check(lib().ts_profile_set_pcie(self.h, d2h, h2d))

    def to_dict(self) -> dict:
        """Every (op, p_num) entry and the PCIe bandwidths (to replay a measured profile)."""
        ops = {}
        for o in range(len(self.graph.spec["ops"])):
            ops[o] = {p: self.get(o, p) for p in (1, 2, 4, 8, 16)}
        return {"ops": ops, "pcie": self.pcie()}

    @classmethod
    def from_dict(cls, graph, d: dict):
        pr = cls(graph)
        for o, row in d["ops"].items():
            for p, (f, b) in row.items():
                pr.set(int(o), int(p), f, b)
        pr.set_pcie(*d["pcie"])
        return pr

    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().ts_profile_destroy(self.h)
        except Exception:  # interpreter teardown: the library may already be gone
            pass


class Plan:
    def __init__(self, graph: Graph, h):
        self.graph, self.h = graph, h

    @classmethod
    def default(cls, graph):
        h = C.c_void_p()
        check(lib().ts_plan_default(graph.h, C.byref(h)))
        return cls(graph, h)

    @classmethod
    def plan(cls, graph, budget_bytes, profile: Profile | None = None, no_split=False, memory_centric=False):
        """ts_plan / ts_plan_ex: no_split = the "TSPLIT w/o Split" ablation,
        memory_centric = no LRU recompute cache (Fig. 11 strategy only)."""
        h = C.c_void_p()
        flags = (1 if no_split else 0) | (2 if memory_centric else 0)
        check(lib().ts_plan_ex(graph.h, int(budget_bytes), profile.h if profile else None, flags, C.byref(h)))
        return cls(graph, h)

    @classmethod
    def deserialize(cls, graph, blob: bytes):
        h = C.c_void_p()
        buf = C.create_string_buffer(blob, len(blob))
        check(lib().ts_plan_deserialize(graph.h, buf, len(blob), C.byref(h)))
        return cls(graph, h)

    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().ts_plan_destroy(self.h)
        except Exception:  # interpreter teardown: the library may already be gone
            pass

    def get(self, tid):
        c = TensorCfg()
        check(lib().ts_plan_get(self.h, tid, C.byref(c)))
        return (c.opt, c.p_num, c.prefetch_lead)

    def set(self, tid, opt=RESIDE, p_num=1, prefetch_lead=1, dim=0, release_lag=0):
        c = TensorCfg(tid, opt, p_num, dim, prefetch_lead, release_lag)
        check(lib().ts_plan_set(self.h, C.byref(c)))

    def get_dim(self, tid) -> int:
        c = TensorCfg()
        check(lib().ts_plan_get(self.h, tid, C.byref(c)))
        return c.dim

    def get_lag(self, tid) -> int:
        """Release lag of a swapped tensor (reading D-LAG)."""
        c = TensorCfg()
        check(lib().ts_plan_get(self.h, tid, C.byref(c)))
        return c.release_lag

    def oracle_cfg(self) -> dict:
        """{tensor id: (opt, p_num, lead, dim, lag)} — the plan in the oracle simulator's form."""
        out = {}
        for t in range(self.graph.n):
            c = TensorCfg()
            check(lib().ts_plan_get(self.h, t, C.byref(c)))
            out[t] = (c.opt, c.p_num, c.prefetch_lead, c.dim, c.release_lag)
        return out

    def set_many(self, cfgs: dict):
        """{tensor id: (opt, p_num, prefetch_lead[, dim[, release_lag]])} applied and validated together
        (a channel-split chain is legal only as a whole, reading D-CH)."""
        arr = (TensorCfg * len(cfgs))()
        for i, (t, c) in enumerate(cfgs.items()):
            arr[i] = TensorCfg(t, c[0], c[1], c[3] if len(c) > 3 else 0, c[2], c[4] if len(c) > 4 else 0)
        check(lib().ts_plan_set_many(self.h, arr, len(cfgs)))

    def set_recompute_cache(self, cache_bytes: int):
        """D-LRU recompute cache limit in bytes (0 = memory-centric; 2**64-1 = unbounded)."""
        check(lib().ts_plan_set_recompute_cache(self.h, C.c_uint64(cache_bytes)))

    def stats(self):
        s = PlanStats()
        check(lib().ts_plan_stats(self.h, C.byref(s)))
        return {f: getattr(s, f) for f, _ in PlanStats._fields_}

    def trace(self):
        n = C.c_uint64()
        check(lib().ts_plan_trace(self.h, None, 0, C.byref(n)))
        buf = (AllocEvent * n.value)()
        check(lib().ts_plan_trace(self.h, buf, n.value, C.byref(n)))
        return [(e.seq, e.item, "A" if e.kind == 0 else "F", e.key, e.piece, e.offset, e.bytes) for e in buf]

    def items(self):
        n = C.c_uint64()
        check(lib().ts_plan_items(self.h, None, 0, C.byref(n)))
        buf = (C.c_int32 * (4 * n.value))()
        check(lib().ts_plan_items(self.h, buf, len(buf), C.byref(n)))
        kinds = ["F", "B", "R", "SO", "SI"]
        return [(kinds[buf[4 * i]], buf[4 * i + 1], buf[4 * i + 2], buf[4 * i + 3]) for i in range(n.value)]

    def grad_buckets(self, bucket_bytes: int = 32 << 20):
        """[(after_item, grad offset, bytes)] spans of the data-parallel allreduce buckets."""
        n = C.c_uint64()
        check(lib().ts_plan_grad_buckets(self.h, bucket_bytes, None, 0, C.byref(n)))
        buf = (C.c_int64 * (3 * n.value))()
        check(lib().ts_plan_grad_buckets(self.h, bucket_bytes, buf, len(buf), C.byref(n)))
        return [(buf[3 * i], buf[3 * i + 1], buf[3 * i + 2]) for i in range(n.value)]

    def roofline(self, tensor_flops: float, hbm_bw: float):
        """(seconds, flop, bytes): sum over the plan's micro-ops of max(F / peak, bytes / bw)."""
        s, f, b = C.c_double(), C.c_double(), C.c_double()
        check(lib().ts_plan_roofline(self.h, tensor_flops, hbm_bw, C.byref(s), C.byref(f), C.byref(b)))
        return s.value, f.value, b.value

    def serialize(self) -> bytes:
        n = C.c_uint64()
        check(lib().ts_plan_serialize(self.h, None, 0, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        check(lib().ts_plan_serialize(self.h, buf, n.value, C.byref(n)))
        return buf.raw

    def cfg_dict(self):
        return {t: self.get(t) for t in range(self.graph.n)}


# --------------------------------------------------------------------------- session
class Session:
    """A device session: the plan's pool is one torch-allocated slab (torch is the
    device-memory plumbing; all work runs in libtsplit)."""

    def __init__(self, graph: Graph, plan: Plan, device: int = 0, slab_bytes: int | None = None,
                 lr: float = 0.0, use_cuda_graph: bool = True, nccl_comm: int | None = None,
                 world_size: int = 1, step0: int = 0, streams=None, sample_offset: int = 0,
                 host_numa_node: int = -1, grad_allreduce_bf16: bool = False):
        import torch
        if not torch.cuda.is_available():
            raise TsError(9, "no CUDA device: the TSPLIT runtime has no CPU fallback")
        self.graph, self.plan = graph, plan
        st = plan.stats()
        self.slab_bytes = int(slab_bytes or st["peak_extent"])
        self.slab = torch.empty(self.slab_bytes, dtype=torch.uint8, device=f"cuda:{device}")
        cfg = SessionCfg()
        cfg.device = device
        cfg.slab = self.slab.data_ptr()
        cfg.slab_bytes = self.slab_bytes
        cfg.nccl_comm = nccl_comm
        if streams is not None:  # (compute, d2h, h2d) torch.cuda.Stream objects
            self.streams = streams
            cfg.stream_compute, cfg.stream_d2h, cfg.stream_h2d = [s.cuda_stream for s in streams]
        cfg.world_size = world_size
        cfg.use_cuda_graph = 1 if use_cuda_graph else 0
        cfg.lr = lr
        cfg.step0 = step0
        cfg.sample_offset = sample_offset
        cfg.host_numa_node = host_numa_node
        cfg.grad_allreduce_bf16 = 1 if grad_allreduce_bf16 else 0
        h = C.c_void_p()
        check(lib().ts_session_create(graph.h, plan.h, C.byref(cfg), C.byref(h)))
        self.h = h
        spec = graph.spec
        self.input_ids = [t["id"] for t in spec["tensors"] if t["kind"] in ("input", "label")]

    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().ts_session_destroy(self.h)
        except Exception:  # interpreter teardown: the library may already be gone
            pass

    def set_params(self, params: dict):
        for t in self.graph.spec["tensors"]:
            if t["kind"] == "param":
                a = np.ascontiguousarray(params[t["name"]], dtype=np.float32)
                check(lib().ts_set_param(self.h, t["id"], a.ctypes.data))

    def _ptrs(self, inputs):
        arr = (C.c_void_p * len(self.input_ids))()
        for i, tid in enumerate(self.input_ids):
            x = inputs[self.graph.spec["tensors"][tid]["name"]]
            arr[i] = x.data_ptr() if hasattr(x, "data_ptr") else x.ctypes.data
        return arr

    def step(self, inputs: dict, on_host: bool | None = None) -> float:
        """inputs: name -> torch tensor (device or pinned host) or numpy array (host)."""
        if on_host is None:
            x0 = inputs[self.graph.spec["tensors"][self.input_ids[0]]["name"]]
            on_host = not (hasattr(x0, "is_cuda") and x0.is_cuda)
        loss = C.c_float()
        check(lib().ts_step(self.h, self._ptrs(inputs), 1 if on_host else 0, C.byref(loss)))
        return loss.value

    def host_pool(self):
        """(bytes, NUMA node or -1) of the pinned swap pool."""
        b, n = C.c_uint64(), C.c_int32()
        check(lib().ts_session_host_pool(self.h, C.byref(b), C.byref(n)))
        return b.value, n.value

    def step_async(self, inputs: dict, on_host: bool = False):
        check(lib().ts_step_async(self.h, self._ptrs(inputs), 1 if on_host else 0))

    def grads(self) -> dict:
        out = {}
        for t in self.graph.spec["tensors"]:
            if t["kind"] == "param":
                a = np.empty(t["shape"], np.float32)
                check(lib().ts_get_grad(self.h, t["id"], a.ctypes.data))
                out[t["name"]] = a
        return out

    def param(self, name) -> np.ndarray:
        t = self.graph.spec["tensors"][self.graph.names[name]]
        a = np.empty(t["shape"], np.float32)
        check(lib().ts_get_param(self.h, t["id"], a.ctypes.data))
        return a

    def trace(self):
        n = C.c_uint64()
        check(lib().ts_session_trace(self.h, None, 0, C.byref(n)))
        buf = (AllocEvent * n.value)()
        check(lib().ts_session_trace(self.h, buf, n.value, C.byref(n)))
        return [(e.seq, e.item, "A" if e.kind == 0 else "F", e.key, e.piece, e.offset, e.bytes) for e in buf]

    def profile_items(self, enable=True):
        check(lib().ts_session_profile_items(self.h, 1 if enable else 0))

    def item_times(self):
        n = C.c_uint64()
        check(lib().ts_session_item_times(self.h, None, 0, C.byref(n)))
        buf = (C.c_float * n.value)()
        check(lib().ts_session_item_times(self.h, buf, n.value, C.byref(n)))
        return list(buf)

    def gemm_times(self):
        """[(flop, ms, batch)] of every GEMM launch of the last profiled step."""
        n = C.c_uint64()
        check(lib().ts_session_gemm_times(self.h, None, None, None, 0, C.byref(n)))
        f = (C.c_double * n.value)()
        m = (C.c_float * n.value)()
        b = (C.c_int32 * n.value)()
        check(lib().ts_session_gemm_times(self.h, f, m, b, n.value, C.byref(n)))
        return list(zip(f, m, b))

    def gemm_kinds(self):
        """[(kind, tc)] per record of gemm_times: kind 0 GEMM, 1/2/3 conv fprop/dgrad/wgrad."""
        n = C.c_uint64()
        check(lib().ts_session_gemm_kinds(self.h, None, None, 0, C.byref(n)))
        k = (C.c_int32 * n.value)()
        t = (C.c_int32 * n.value)()
        check(lib().ts_session_gemm_kinds(self.h, k, t, n.value, C.byref(n)))
        return list(zip(k, t))

    def gemm_shapes(self):
        """[(M, N, K, flags)] per record of gemm_times."""
        n = C.c_uint64()
        check(lib().ts_session_gemm_shapes(self.h, None, 0, C.byref(n)))
        b = (C.c_int32 * (4 * n.value))()
        check(lib().ts_session_gemm_shapes(self.h, b, len(b), C.byref(n)))
        return [tuple(b[4 * i:4 * i + 4]) for i in range(n.value)]

    def launches(self) -> int:
        n = C.c_int64()
        check(lib().ts_session_launches(self.h, C.byref(n)))
        return n.value


def inputs_to_device(graph: Graph, arrays: dict, device="cuda:0", pinned_host=False):
    import torch
    out = {}
    for t in graph.spec["tensors"]:
        if t["kind"] in ("input", "label"):
            a = arrays[t["name"]]
            if t["dtype"] == "i32":
                x = torch.from_numpy(np.ascontiguousarray(a, np.int32))
            elif t["dtype"] == "bf16":
                x = torch.from_numpy(np.ascontiguousarray(a, np.float32)).to(torch.bfloat16)
            else:
                x = torch.from_numpy(np.ascontiguousarray(a, np.float32))
            out[t["name"]] = x.pin_memory() if pinned_host else x.to(device)
    return out


def nccl_comm(rank: int, world: int, broadcast):
    """Create a NCCL communicator; `broadcast(bytes) -> bytes` ships rank 0's id."""
    buf = C.create_string_buffer(128)
    if rank == 0:
        check(lib().ts_nccl_unique_id(buf))
    raw = broadcast(buf.raw if rank == 0 else None)
    idb = C.create_string_buffer(raw, 128)
    comm = C.c_void_p()
    check(lib().ts_nccl_comm_init(idb, world, rank, C.byref(comm)))
    return comm.value


def conv2d(mode: int, geom, x, w, dy, out, bias=None, acc: int = 0, stream=None) -> bool:
    """Run one conv micro-op kernel through the C ABI (`ts_conv2d`, include/ts.h) on
    torch device tensors (argument marshalling only).  mode 1 fprop -> out = y,
    2 dgrad -> out = dx, 3 wgrad -> out = dw (fp32).  Returns True when the tcgen05
    implicit-GEMM path ran."""
    import torch
    dt = DTYPES["bf16"] if w.dtype == torch.bfloat16 else DTYPES["f32"]
    g = (C.c_int32 * 9)(*[int(v) for v in geom])
    ptr = (lambda t: C.c_void_p(t.data_ptr()) if t is not None else None)
    used = C.c_int32(0)
    st = C.c_void_p(stream if stream is not None else torch.cuda.current_stream().cuda_stream)
    check(lib().ts_conv2d(mode, dt, g, ptr(x), ptr(w), ptr(dy), ptr(out), ptr(bias), acc, st, C.byref(used)))
    return bool(used.value)


def attention(mode: int, geom, alpha: float, p: float, q, k, v, c=None, lse=None, dc=None, dq=None, dk=None,
              dv=None, acc: int = 0, ws=None, stream=None, mask=None) -> int:
    """One fused-attention kernel call through the C ABI (`ts_attention`) on torch device
    tensors (marshalling only).  geom = (nb, heads, seq, d, seed, b0, step).  Returns the
    path: 0 CUDA cores, 1 mma.sync, 2 tcgen05 (forward)."""
    import torch
    dt = DTYPES["bf16"] if q.dtype == torch.bfloat16 else DTYPES["f32"]
    g = (C.c_int32 * 7)(*[int(x) for x in geom])
    fa = (C.c_float * 2)(alpha, p)
    ptr = (lambda t: C.c_void_p(t.data_ptr()) if t is not None else None)
    used = C.c_int32(0)
    st = C.c_void_p(stream if stream is not None else torch.cuda.current_stream().cuda_stream)
    lse_p = C.cast(C.c_void_p(lse.data_ptr()), C.POINTER(C.c_float)) if lse is not None else None
    ws_p = C.c_void_p(ws.data_ptr()) if ws is not None else None
    check(lib().ts_attention(mode, dt, g, fa, ptr(q), ptr(k), ptr(v), ptr(c), lse_p, ptr(mask), ptr(dc), ptr(dq),
                             ptr(dk), ptr(dv), acc, ws_p, st, C.byref(used)))
    return used.value


def column_sum(x, out, ws, acc: int = 0, stream=None):
    """out (+)= x.sum(0) through ts_row_op (x: [rows, n] bf16 / fp32 torch device tensor,
    out: fp32 [n], ws: fp32 workspace whose last 4 KB start zeroed)."""
    import torch
    dt = DTYPES["bf16"] if x.dtype == torch.bfloat16 else DTYPES["f32"]
    st = C.c_void_p(stream if stream is not None else torch.cuda.current_stream().cuda_stream)
    check(lib().ts_row_op(0, dt, C.c_void_p(x.data_ptr()), None, C.c_void_p(out.data_ptr()), x.shape[0], x.shape[1],
                          C.c_void_p(ws.data_ptr()), ws.numel() * 4, acc, st))
