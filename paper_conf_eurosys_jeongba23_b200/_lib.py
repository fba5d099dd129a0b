"""ctypes marshalling for include/deepplan.h (no computation here)."""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# DP_LIB: another build of the same library (A/B timing tools); the in-tree build by default
_LIB_PATH = os.environ.get("DP_LIB") or os.path.join(_HERE, "libdeepplan.so")

LOAD, DHA = 0, 1
MODES = {"BASELINE": 0, "PIPESWITCH": 1, "GREEDY": 2, "DHA": 3, "PT": 4, "PT_DHA": 5, "DHA_LINK": 6,
         "PT_DHA_LINK": 7, "PT_DHA_BAL": 8, "PT_DHA_LINK_BAL": 9, "PT_DHA_STRIPE": 10, "PT_DHA_LINK_STRIPE": 11}
UNIT_KINDS = {0: "emb", 1: "ln", 2: "linear"}
FAMILIES = {"bert": 0, "roberta": 1, "gpt2": 2}
DTYPES = {"fp16": 0, "bf16": 1, "fp32": 2}
ACTS = {"none": 0, "gelu_erf": 1, "gelu_tanh": 2, "tanh": 3}
PT_TRANSPORTS = {"dma": 0, "sm": 1, "ce": 2}  # dp_engine_opts.pt_transport: DP_PT_DMA / _SM / _CE
DP_MAX_DEVICES = 8


class DeepPlanError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"deepplan error {code}: {msg}")
        self.code = code


if not os.path.exists(_LIB_PATH):
    raise ImportError(
        f"{_LIB_PATH} is missing: build it with `python paper_conf_eurosys_jeongba23_b200/build.py` "
        "(there is no CPU fallback)")

lib = C.CDLL(_LIB_PATH)

i8p = C.POINTER(C.c_int8)
i32p = C.POINTER(C.c_int32)
i64p = C.POINTER(C.c_int64)


class CostTable(C.Structure):
    _fields_ = [("n", C.c_int32), ("bytes", i64p), ("load_ns", i64p), ("fwd_ns", i64p),
                ("exe_mem_ns", i64p), ("exe_dha_ns", i64p), ("dha_link_ns", i64p)]


class Plan(C.Structure):
    _fields_ = [("n", C.c_int32), ("mode", C.c_int32), ("k", C.c_int32), ("serial", C.c_int32),
                ("method", i8p), ("slot", i8p)]


class EngineOpts(C.Structure):
    _fields_ = [("chunk_bytes", C.c_int64), ("n_h2d_streams", C.c_int32), ("use_graph", C.c_int32),
                ("gemm_bn", C.c_int32), ("debug_delay_us", C.c_int32), ("debug_poison", C.c_int32),
                ("use_pdl", C.c_int32), ("fuse_ln", C.c_int32), ("tail_bytes", C.c_int64),
                ("persistent", C.c_int32), ("pt_transport", C.c_int32), ("profile_chain", C.c_int32),
                ("trace_units", C.c_int32), ("attention_tc", C.c_int32), ("reserved", C.c_int32 * 1)]


class ModelConfig(C.Structure):
    _fields_ = [("family", C.c_int32), ("vocab", C.c_int32), ("max_pos", C.c_int32),
                ("type_vocab", C.c_int32), ("hidden", C.c_int32), ("heads", C.c_int32),
                ("ffn", C.c_int32), ("layers", C.c_int32), ("dtype", C.c_int32),
                ("pad_idx", C.c_int32), ("ln_eps", C.c_double)]


class UnitInfo(C.Structure):
    _fields_ = [("kind", C.c_int32), ("nparams", C.c_int32), ("first_param", C.c_int32),
                ("reserved", C.c_int32), ("bytes", C.c_int64), ("arena_offset", C.c_int64),
                ("name", C.c_char * 32)]


class ParamInfo(C.Structure):
    _fields_ = [("hf_name", C.c_char * 96), ("ndim", C.c_int32), ("unit", C.c_int32),
                ("shape", C.c_int64 * 2), ("bytes", C.c_int64)]


class RunStats(C.Structure):
    _fields_ = [("h2d_bytes", C.c_int64 * DP_MAX_DEVICES), ("nvlink_bytes", C.c_int64 * DP_MAX_DEVICES),
                ("dha_weight_bytes", C.c_int64), ("n_copies", C.c_int32), ("n_events", C.c_int32),
                ("n_kernels", C.c_int32), ("n_units", C.c_int32), ("wall_enqueue_us", C.c_float),
                ("reserved", C.c_float * 3)]


class TraceEvent(C.Structure):
    _fields_ = [("arrival_ns", C.c_int64), ("instance", C.c_int32), ("reserved", C.c_int32)]


class ServeOpts(C.Structure):
    _fields_ = [("plan_mode", C.c_int32), ("k_max", C.c_int32), ("ngpu", C.c_int32), ("dry_run", C.c_int32),
                ("per_gpu_budget_bytes", C.c_int64), ("slo_ns", C.c_int64), ("nmodels", C.c_int32),
                ("no_prewarm", C.c_int32), ("cold_ns", i64p), ("warm_ns", i64p), ("resident_bytes", i64p),
                ("model_of_instance", i32p), ("ninstances", C.c_int32), ("batch", C.c_int32),
                ("seq", C.c_int32), ("reserved1", C.c_int32), ("plans", C.POINTER(C.POINTER(Plan))),
                ("seq_of_model", i32p)]


class ServeResult(C.Structure):
    _fields_ = [("start_ns", C.c_int64), ("finish_ns", C.c_int64), ("gpu", C.c_int32), ("cold", C.c_int32),
                ("nevicted", C.c_int32), ("sec_mask", C.c_int32), ("decide_ns", C.c_int64)]


def _sig(name, args, res=C.c_int32):
    f = getattr(lib, name)
    f.argtypes = args
    f.restype = res
    return f


vp = C.c_void_p
_sig("dp_last_error", [], C.c_char_p)
_sig("dp_abi_version", [])
_sig("dp_plan_generate", [C.POINTER(CostTable), C.c_int32, C.c_int32, C.POINTER(Plan)])
_sig("dp_plan_simulate", [C.POINTER(CostTable), C.POINTER(Plan), i64p, i64p, i64p])
_sig("dp_plan_partition", [i64p, C.c_int32, C.c_int32, i8p])
_sig("dp_plan_exhaustive", [C.POINTER(CostTable), C.POINTER(Plan), i32p, C.c_int32, C.POINTER(Plan), i64p])
_sig("dp_context_create", [i32p, C.c_int32, C.POINTER(vp)])
_sig("dp_context_destroy", [vp])
_sig("dp_context_set_opts", [vp, C.POINTER(EngineOpts)])
_sig("dp_context_get_opts", [vp, C.POINTER(EngineOpts)])
_sig("dp_peer_unique_id", [vp])
_sig("dp_peer_init", [vp, vp, C.c_int32, C.c_int32])
_sig("dp_peer_init_ipc", [vp, C.c_int32, C.c_int32])
_sig("dp_peer_set_slot_ranks", [vp, C.c_int32, i32p, C.c_int32])
_sig("dp_device_numa_node", [C.c_int32])
_sig("dp_host_numa_node", [vp])
_sig("dp_host_alloc_node", [C.c_int64, C.c_int32, C.POINTER(vp)])
_sig("dp_measure_h2d_concurrent", [i32p, C.c_int32, C.c_int64, C.c_int32, C.POINTER(C.c_double)])
_sig("dp_select_secondaries", [C.POINTER(C.c_double), C.POINTER(C.c_double), i32p, C.c_int32, C.c_int32,
                               C.c_int32, i32p])
_sig("dp_peer_ipc_export", [vp, vp, vp])
_sig("dp_peer_ipc_import", [vp, vp, vp])
_sig("dp_pt_forward", [vp, vp, C.c_int64, vp])
_sig("dp_config_params", [C.POINTER(ModelConfig), C.POINTER(ParamInfo), C.c_int32, i32p])
_sig("dp_model_create", [vp, C.POINTER(ModelConfig), C.POINTER(vp), C.c_int32, C.POINTER(vp)])
_sig("dp_model_destroy", [vp, vp])
_sig("dp_model_clone", [vp, vp, C.POINTER(vp)])
_sig("dp_model_num_units", [vp])
_sig("dp_model_unit_info", [vp, C.c_int32, C.POINTER(UnitInfo)])
_sig("dp_model_bytes", [vp], C.c_int64)
_sig("dp_model_arena", [vp, C.POINTER(vp), i64p])
_sig("dp_transfer_schedule", [C.POINTER(ModelConfig), C.POINTER(Plan), C.c_int32, C.c_int64, C.c_int64, i64p, i64p,
                              i32p, i32p, C.c_int32, i32p])
_sig("dp_measure_h2d", [C.c_int32, C.c_int64, C.c_int32, C.POINTER(C.c_double)])
_sig("dp_profile",[vp, vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.POINTER(CostTable)])
_sig("dp_infer_cold", [vp, vp, C.POINTER(Plan), C.c_int32, i32p, C.c_int32, vp, C.c_int32, C.c_int32, vp, vp, vp,
                       C.POINTER(RunStats)])
_sig("dp_run_timeline", [vp, vp, C.c_int32, C.c_int32, i64p, i64p, i64p, i64p])
_sig("dp_infer_warm", [vp, vp, C.c_int32, vp, C.c_int32, C.c_int32, vp, vp, vp, C.POINTER(RunStats)])
_sig("dp_model_evict", [vp, vp, C.c_int32])
_sig("dp_lm_head", [vp, vp, C.c_int32, vp, C.c_int32, C.c_int32, vp, vp])
_sig("dp_model_is_resident", [vp, C.c_int32])
_sig("dp_model_resident_bytes", [vp, C.c_int32], C.c_int64)
_sig("dp_pool_stats", [vp, C.c_int32, i64p, i64p])
_sig("dp_pool_trim", [vp, C.c_int32, i64p])
_sig("dp_plan_resident_bytes", [vp, C.POINTER(Plan)], C.c_int64)
_sig("dp_host_alloc", [C.c_int64, C.POINTER(vp)])
_sig("dp_host_free", [vp])
_sig("dp_embed", [vp, C.c_int32, C.c_int32, C.c_int32, vp, vp, vp, vp, vp, C.c_int32, C.c_double, C.c_int32,
                  C.c_int32, vp, vp])
_sig("dp_linear", [vp, C.c_int32, vp, vp, vp, C.c_int32, vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                   C.c_int32, C.c_int32, C.c_int32, C.c_int32, vp])
_sig("dp_gemm_tc", [vp, C.c_int32, vp, vp, vp, C.c_int32, vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                    C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32, vp])
_sig("dp_layernorm", [vp, vp, vp, vp, vp, C.c_int32, C.c_int32, C.c_double, C.c_int32, C.c_int32, vp])
_sig("dp_attention", [vp, C.c_int32, vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32, vp])
_sig("dp_attention_tc", [vp, C.c_int32, vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32, vp])
_sig("dp_serve_run", [vp, C.POINTER(vp), C.c_int32, C.POINTER(TraceEvent), C.c_int32, C.POINTER(ServeOpts),
                      C.POINTER(ServeResult)])


def _check(st: int):
    if st != 0:
        raise DeepPlanError(st, lib.dp_last_error().decode(errors="replace"))


def _i64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int64))


def _ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t)


# --------------------------------------------------------------------------------------
# Planner
# --------------------------------------------------------------------------------------

_COST_KEYS = ("bytes", "load_ns", "fwd_ns", "exe_mem_ns", "exe_dha_ns")


def _cost(cost: dict):
    arrs = [_i64(cost[k]) for k in _COST_KEYS]
    n = len(arrs[0])
    if cost.get("dha_link_ns") is not None:
        arrs.append(_i64(cost["dha_link_ns"]))
    for a in arrs:
        if len(a) != n:
            raise ValueError("cost table arrays differ in length")
    ptrs = [_ptr(a, i64p) for a in arrs] + ([None] if len(arrs) == 5 else [])
    ct = CostTable(n, *ptrs)
    return ct, arrs


def _mode(mode) -> int:
    return MODES[mode] if isinstance(mode, str) else int(mode)


class PlanArrays:
    """Owns the int8 method/slot arrays behind a Plan struct."""

    def __init__(self, n: int, method=None, slot=None, mode: int = 1, k: int = 1, serial: int = 0):
        self.method = np.zeros(n, dtype=np.int8) if method is None else np.ascontiguousarray(method, dtype=np.int8)
        self.slot = np.zeros(n, dtype=np.int8) if slot is None else np.ascontiguousarray(slot, dtype=np.int8)
        self.s = Plan(n, mode, k, serial, _ptr(self.method, i8p), _ptr(self.slot, i8p))

    @property
    def k(self):
        return self.s.k

    @property
    def serial(self):
        return self.s.serial

    @property
    def mode(self):
        return self.s.mode


def plan_generate(cost: dict, mode, k: int = 1) -> PlanArrays:
    ct, keep = _cost(cost)
    p = PlanArrays(ct.n)
    _check(lib.dp_plan_generate(C.byref(ct), _mode(mode), int(k), C.byref(p.s)))
    return p


def plan_simulate(cost: dict, plan: PlanArrays):
    ct, keep = _cost(cost)
    lat = C.c_int64()
    stall = np.zeros(ct.n, dtype=np.int64)
    link = np.zeros(max(1, plan.k), dtype=np.int64)
    _check(lib.dp_plan_simulate(C.byref(ct), C.byref(plan.s), C.byref(lat), _ptr(stall, i64p), _ptr(link, i64p)))
    return int(lat.value), stall, link


def plan_partition(nbytes, k: int) -> np.ndarray:
    b = _i64(nbytes)
    part = np.zeros(len(b), dtype=np.int8)
    _check(lib.dp_plan_partition(_ptr(b, i64p), len(b), int(k), _ptr(part, i8p)))
    return part


def plan_exhaustive(cost: dict, base: PlanArrays, free_idx):
    ct, keep = _cost(cost)
    fr = np.ascontiguousarray(free_idx, dtype=np.int32)
    out = PlanArrays(ct.n)
    lat = C.c_int64()
    _check(lib.dp_plan_exhaustive(C.byref(ct), C.byref(base.s), _ptr(fr, i32p), len(fr), C.byref(out.s),
                                  C.byref(lat)))
    return int(lat.value), out


# --------------------------------------------------------------------------------------
# Context / model
# --------------------------------------------------------------------------------------

def _stream_ptr(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _dptr(t) -> int:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def peer_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib.dp_peer_unique_id(C.cast(buf, vp)))
    return buf.raw


class Context:
    def __init__(self, devs=(0,)):
        arr = np.ascontiguousarray(devs, dtype=np.int32)
        h = vp()
        _check(lib.dp_context_create(_ptr(arr, i32p), len(arr), C.byref(h)))
        self.h = h
        self.devs = list(devs)

    def set_opts(self, chunk_bytes=None, n_h2d_streams=None, use_graph=None, gemm_bn=None, debug_delay_us=None,
                 debug_poison=None, use_pdl=None, tail_bytes=None, fuse_ln=None, persistent=None,
                 pt_transport=None, profile_chain=None, trace_units=None, attention_tc=None):
        o = EngineOpts()
        _check(lib.dp_context_get_opts(self.h, C.byref(o)))
        if chunk_bytes is not None:
            o.chunk_bytes = int(chunk_bytes)
        if n_h2d_streams is not None:
            o.n_h2d_streams = int(n_h2d_streams)
        if use_graph is not None:
            o.use_graph = int(use_graph)
        if gemm_bn is not None:
            o.gemm_bn = int(gemm_bn)
        if debug_delay_us is not None:
            o.debug_delay_us = int(debug_delay_us)
        if debug_poison is not None:
            o.debug_poison = int(debug_poison)
        if use_pdl is not None:
            o.use_pdl = int(use_pdl)
        if tail_bytes is not None:
            o.tail_bytes = int(tail_bytes)
        if fuse_ln is not None:
            o.fuse_ln = 1 if fuse_ln else 0
        if persistent is not None:
            o.persistent = 1 if persistent else 0
        if profile_chain is not None:
            o.profile_chain = 1 if profile_chain else 0
        if trace_units is not None:
            o.trace_units = 1 if trace_units else 0
        if attention_tc is not None:  # 0 by sequence length, 1 always K5t, 2 never (True / False: 1 / 2)
            o.attention_tc = (1 if attention_tc else 2) if isinstance(attention_tc, bool) else int(attention_tc)
        if pt_transport is not None:
            o.pt_transport = PT_TRANSPORTS[pt_transport] if isinstance(pt_transport, str) else int(pt_transport)
        _check(lib.dp_context_set_opts(self.h, C.byref(o)))

    def pool_stats(self, dev: int = 0):
        """(reserved, in_use) bytes of the device's HBM slot pool."""
        r, u = C.c_int64(), C.c_int64()
        _check(lib.dp_pool_stats(self.h, int(dev), C.byref(r), C.byref(u)))
        return int(r.value), int(u.value)

    def pool_trim(self, dev: int = 0) -> int:
        f = C.c_int64()
        _check(lib.dp_pool_trim(self.h, int(dev), C.byref(f)))
        return int(f.value)

    def peer_init(self, uid: bytes, rank: int, nranks: int):
        buf = C.create_string_buffer(uid, 128)
        _check(lib.dp_peer_init(self.h, C.cast(buf, vp), int(rank), int(nranks)))

    def peer_init_ipc(self, rank: int, nranks: int):
        """Multi-process PT without NCCL (SM forwarder over CUDA IPC)."""
        _check(lib.dp_peer_init_ipc(self.h, int(rank), int(nranks)))

    def set_slot_ranks(self, primary: int, ranks):
        """PT slot s (1..k-1) of `primary`'s cold starts is carried by ranks[s-1]."""
        arr = np.ascontiguousarray(list(ranks) or [0], dtype=np.int32)
        _check(lib.dp_peer_set_slot_ranks(self.h, int(primary), _ptr(arr, i32p), len(ranks) + 1))

    def close(self):
        if self.h:
            _check(lib.dp_context_destroy(self.h))
            self.h = None


def model_config(shape, dtype: str = "fp16") -> ModelConfig:
    """Build a dp_model_config from any object with the HF shape fields (e.g. synth.ModelShape)."""
    return ModelConfig(FAMILIES[shape.family], shape.vocab, shape.max_pos, shape.type_vocab, shape.hidden,
                       shape.heads, shape.ffn, shape.layers, DTYPES[dtype], getattr(shape, "pad_idx", 0),
                       float(shape.ln_eps))


def config_params(shape, dtype: str = "fp16"):
    cfg = model_config(shape, dtype)
    cnt = C.c_int32()
    _check(lib.dp_config_params(C.byref(cfg), None, 0, C.byref(cnt)))
    infos = (ParamInfo * cnt.value)()
    _check(lib.dp_config_params(C.byref(cfg), infos, cnt.value, C.byref(cnt)))
    return [dict(name=p.hf_name.decode(), ndim=p.ndim, unit=p.unit, shape=tuple(p.shape[:p.ndim]), bytes=p.bytes)
            for p in infos]


def transfer_schedule(shape, plan: "PlanArrays", slot: int, chunk_bytes: int, tail_bytes: int = 2 << 20,
                      dtype: str = "fp16"):
    """Pieces (offset, bytes, first_unit, last_unit) carried by one plan slot's link."""
    cfg = model_config(shape, dtype)
    cnt = C.c_int32()
    _check(lib.dp_transfer_schedule(C.byref(cfg), C.byref(plan.s), int(slot), int(chunk_bytes), int(tail_bytes),
                                    None, None, None, None, 0, C.byref(cnt)))
    n = cnt.value
    off, nb = np.zeros(n, np.int64), np.zeros(n, np.int64)
    fu, lu = np.zeros(n, np.int32), np.zeros(n, np.int32)
    _check(lib.dp_transfer_schedule(C.byref(cfg), C.byref(plan.s), int(slot), int(chunk_bytes), int(tail_bytes),
                                    _ptr(off, i64p), _ptr(nb, i64p), _ptr(fu, i32p), _ptr(lu, i32p), n,
                                    C.byref(cnt)))
    return off, nb, fu, lu


def config_units(shape, dtype: str = "fp16"):
    """Unit names / byte counts of a config without registering a model (host-only)."""
    ps = config_params(shape, dtype)
    nunits = max(p["unit"] for p in ps) + 1
    nb = np.zeros(nunits, np.int64)
    for p in ps:
        nb[p["unit"]] += p["bytes"]
    return nb


class Model:
    """A model registered in the library's pinned arena.  ``weights`` maps HF state-dict
    names to host arrays in the storage dtype (fp16 / bf16 bit patterns)."""

    def __init__(self, ctx: Context, shape, weights, dtype: str = "fp16"):
        self.ctx = ctx
        self.shape = shape
        self.dtype = dtype
        self.cfg = model_config(shape, dtype)
        params = config_params(shape, dtype)
        keep = []
        ptrs = (vp * len(params))()
        for i, p in enumerate(params):
            a = np.ascontiguousarray(weights[p["name"]])
            if tuple(a.shape) != p["shape"] or a.nbytes != p["bytes"]:
                raise ValueError(f"{p['name']}: expected shape {p['shape']} ({p['bytes']} B), got {a.shape}")
            keep.append(a)
            ptrs[i] = a.ctypes.data
        h = vp()
        _check(lib.dp_model_create(ctx.h, C.byref(self.cfg), ptrs, len(params), C.byref(h)))
        self.h = h
        self.n = lib.dp_model_num_units(h)

    def clone(self) -> "Model":
        m = Model.__new__(Model)
        m.ctx, m.shape, m.dtype, m.cfg, m.n = self.ctx, self.shape, self.dtype, self.cfg, self.n
        h = vp()
        _check(lib.dp_model_clone(self.ctx.h, self.h, C.byref(h)))
        m.h = h
        return m

    def units(self):
        out = []
        for i in range(self.n):
            u = UnitInfo()
            _check(lib.dp_model_unit_info(self.h, i, C.byref(u)))
            out.append(dict(name=u.name.decode(), kind=UNIT_KINDS[u.kind], bytes=u.bytes, offset=u.arena_offset,
                            nparams=u.nparams, first_param=u.first_param))
        return out

    def unit_bytes(self) -> np.ndarray:
        return np.array([u["bytes"] for u in self.units()], dtype=np.int64)

    @property
    def nbytes(self) -> int:
        return int(lib.dp_model_bytes(self.h))

    def arena(self) -> np.ndarray:
        p = vp()
        n = C.c_int64()
        _check(lib.dp_model_arena(self.h, C.byref(p), C.byref(n)))
        return np.ctypeslib.as_array(C.cast(p, C.POINTER(C.c_uint8)), shape=(n.value,))

    def profile(self, dev: int, batch: int, seq: int, iters: int = 10) -> dict:
        arrs = {k: np.zeros(self.n, dtype=np.int64) for k in _COST_KEYS + ("dha_link_ns",)}
        ct = CostTable(self.n, *[_ptr(arrs[k], i64p) for k in _COST_KEYS + ("dha_link_ns",)])
        _check(lib.dp_profile(self.ctx.h, self.h, int(dev), int(batch), int(seq), int(iters), C.byref(ct)))
        return arrs

    def infer_cold(self, plan: PlanArrays, primary: int, ids, out, pooled=None, secondaries=(), stream=None) -> dict:
        sec = np.ascontiguousarray(list(secondaries) or [0], dtype=np.int32)
        st = RunStats()
        B, S = ids.shape
        _check(lib.dp_infer_cold(self.ctx.h, self.h, C.byref(plan.s), int(primary), _ptr(sec, i32p),
                                 len(secondaries), _dptr(ids), B, S, _dptr(out), _dptr(pooled),
                                 _stream_ptr(stream), C.byref(st)))
        return _stats(st)

    def infer_cold_raw(self, plan: PlanArrays, primary: int, ids_ptr, batch, seq, out_ptr, pooled_ptr, stream_ptr,
                       secondaries=()):
        """Pointer-level variant (secondary ranks pass NULL buffers)."""
        sec = np.ascontiguousarray(list(secondaries) or [0], dtype=np.int32)
        st = RunStats()
        _check(lib.dp_infer_cold(self.ctx.h, self.h, C.byref(plan.s), int(primary), _ptr(sec, i32p),
                                 len(secondaries), ids_ptr, batch, seq, out_ptr, pooled_ptr, stream_ptr,
                                 C.byref(st)))
        return _stats(st)

    def timeline(self, dev: int) -> dict:
        """Per-unit ready / start / end / stall ns of the last traced cold start (opts.trace_units)."""
        arrs = {k: np.zeros(self.n, dtype=np.int64) for k in ("ready_ns", "start_ns", "end_ns", "stall_ns")}
        _check(lib.dp_run_timeline(self.ctx.h, self.h, int(dev), self.n, *[_ptr(arrs[k], i64p) for k in
                                                                           ("ready_ns", "start_ns", "end_ns",
                                                                            "stall_ns")]))
        return arrs

    def infer_warm(self, dev: int, ids, out, pooled=None, stream=None) -> dict:
        st = RunStats()
        B, S = ids.shape
        _check(lib.dp_infer_warm(self.ctx.h, self.h, int(dev), _dptr(ids), B, S, _dptr(out), _dptr(pooled),
                                 _stream_ptr(stream), C.byref(st)))
        return _stats(st)

    def lm_head(self, dev: int, hidden, logits, rows: int | None = None, ld_hidden: int | None = None,
                stream=None):
        """GPT-2 tied LM head (dp_lm_head): logits[r] = hidden_row_r . wte^T (fp32).  `hidden` is a
        device tensor whose first element is row 0; rows are ld_hidden elements apart."""
        rows = rows if rows is not None else logits.shape[0]
        ld = ld_hidden if ld_hidden is not None else self.shape.hidden
        _check(lib.dp_lm_head(self.ctx.h, self.h, int(dev), _dptr(hidden), int(ld), int(rows), _dptr(logits),
                              _stream_ptr(stream)))

    def ipc_export(self) -> bytes:
        """This rank's DP_IPC_HANDLE_BYTES block (HBM slots + mailbox) for the SM forwarder."""
        buf = C.create_string_buffer(128)
        _check(lib.dp_peer_ipc_export(self.ctx.h, self.h, C.cast(buf, vp)))
        return buf.raw

    def ipc_import(self, blocks):
        """Open the other ranks' blocks (a list of bytes in rank order)."""
        data = b"".join(bytes(b) for b in blocks)
        buf = C.create_string_buffer(data, len(data))
        _check(lib.dp_peer_ipc_import(self.ctx.h, self.h, C.cast(buf, vp)))

    def evict(self, dev: int):
        _check(lib.dp_model_evict(self.ctx.h, self.h, int(dev)))

    def is_resident(self, dev: int) -> bool:
        return bool(lib.dp_model_is_resident(self.h, int(dev)))

    def resident_bytes(self, dev: int) -> int:
        """HBM bytes held while resident (loaded units only; DHA units stay in host memory)."""
        return int(lib.dp_model_resident_bytes(self.h, int(dev)))

    def close(self):
        if self.h:
            _check(lib.dp_model_destroy(self.ctx.h, self.h))
            self.h = None


def _stats(st: RunStats) -> dict:
    return dict(h2d_bytes=list(st.h2d_bytes), nvlink_bytes=list(st.nvlink_bytes),
                dha_weight_bytes=st.dha_weight_bytes, n_copies=st.n_copies, n_events=st.n_events,
                n_kernels=st.n_kernels, n_units=st.n_units, wall_enqueue_us=st.wall_enqueue_us)


# --------------------------------------------------------------------------------------
# Pinned host memory and kernel hooks
# --------------------------------------------------------------------------------------

def measure_h2d(dev: int, nbytes: int = 256 << 20, reps: int = 5) -> float:
    """Pinned H2D GB/s of device `dev` (the link roofline denominator)."""
    g = C.c_double()
    _check(lib.dp_measure_h2d(int(dev), int(nbytes), int(reps), C.byref(g)))
    return float(g.value)


def device_numa_node(dev: int) -> int:
    return int(lib.dp_device_numa_node(int(dev)))


def host_numa_node(p) -> int:
    return int(lib.dp_host_numa_node(_dptr(p)))


def host_alloc_node(nbytes: int, node: int) -> int:
    p = vp()
    _check(lib.dp_host_alloc_node(int(nbytes), int(node), C.byref(p)))
    return p.value


def measure_h2d_concurrent(devs, nbytes: int = 256 << 20, reps: int = 5) -> list:
    """Per-device GB/s when all `devs` copy host -> device at the same time."""
    d = np.ascontiguousarray(devs, dtype=np.int32)
    out = (C.c_double * len(d))()
    _check(lib.dp_measure_h2d_concurrent(_ptr(d, i32p), len(d), int(nbytes), int(reps), out))
    return [float(x) for x in out]


def select_secondaries(solo_gbs, pair_gbs, primary: int, k: int, numa=None) -> list:
    """dp_select_secondaries: k-1 secondaries for `primary` from measured link rates."""
    solo = np.ascontiguousarray(solo_gbs, dtype=np.float64)
    pair = np.ascontiguousarray(pair_gbs, dtype=np.float64)
    n = len(solo)
    nm = None if numa is None else np.ascontiguousarray(numa, dtype=np.int32)
    out = np.zeros(max(1, k - 1), dtype=np.int32)
    _check(lib.dp_select_secondaries(solo.ctypes.data_as(C.POINTER(C.c_double)),
                                     pair.ctypes.data_as(C.POINTER(C.c_double)),
                                     None if nm is None else _ptr(nm, i32p), n, int(primary), int(k),
                                     _ptr(out, i32p)))
    return [int(x) for x in out[:k - 1]]


def pt_forward(src, dst, nbytes: int, stream=None):
    """SM-driven PT forwarder kernel (host-mapped src -> local or peer HBM dst)."""
    _check(lib.dp_pt_forward(_dptr(src), _dptr(dst), int(nbytes), _stream_ptr(stream)))


def host_alloc(nbytes: int) -> int:
    p = vp()
    _check(lib.dp_host_alloc(int(nbytes), C.byref(p)))
    return p.value


def host_free(p: int):
    _check(lib.dp_host_free(p))


def embed(ids, seq, word, pos, type_, ln_g, ln_b, hidden, eps, out, dtype="fp16", pos_offset=0, out_f32=False,
          stream=None):
    ntok = ids.numel() if hasattr(ids, "numel") else int(np.prod(ids.shape))
    _check(lib.dp_embed(_dptr(ids), ntok, int(seq), int(pos_offset), _dptr(word), _dptr(pos), _dptr(type_),
                        _dptr(ln_g), _dptr(ln_b), int(hidden), float(eps), DTYPES[dtype], int(bool(out_f32)),
                        _dptr(out), _stream_ptr(stream)))


def linear(x, ldx, w, b, residual, ldr, y, ldy, M, N, K, act="none", path=0, dtype="fp16", io=0, stream=None):
    _check(lib.dp_linear(_dptr(x), int(ldx), _dptr(w), _dptr(b), _dptr(residual), int(ldr), _dptr(y), int(ldy),
                         int(M), int(N), int(K), ACTS[act] if isinstance(act, str) else int(act), int(path),
                         DTYPES[dtype], int(io), _stream_ptr(stream)))


def gemm_tc(x, ldx, w, b, residual, ldr, y, ldy, M, N, K, act="none", bn=0, split=0, dtype="fp16", io=0,
            stream=None):
    """The resident tcgen05 GEMM with its tile forced: bn 0 = the cost model's choice, > 0 one CTA
    per 128 x bn tile, < 0 a CTA pair per 256 x |bn| tile (K2p); split > 0 forces the K split."""
    _check(lib.dp_gemm_tc(_dptr(x), int(ldx), _dptr(w), _dptr(b), _dptr(residual), int(ldr), _dptr(y), int(ldy),
                          int(M), int(N), int(K), ACTS[act] if isinstance(act, str) else int(act), DTYPES[dtype],
                          int(io), int(bn), int(split), _stream_ptr(stream)))


def layernorm(x, r, g, b, y, rows, n, eps, dtype="fp16", x_f32=False, stream=None):
    _check(lib.dp_layernorm(_dptr(x), _dptr(r), _dptr(g), _dptr(b), _dptr(y), int(rows), int(n), float(eps),
                            DTYPES[dtype], int(bool(x_f32)), _stream_ptr(stream)))


def attention(qkv, ldqkv, ctx_out, batch, seq, hidden, heads, causal, dtype="fp16", stream=None):
    _check(lib.dp_attention(_dptr(qkv), int(ldqkv), _dptr(ctx_out), int(batch), int(seq), int(hidden), int(heads),
                            int(bool(causal)), DTYPES[dtype], _stream_ptr(stream)))


def attention_tc(qkv, ldqkv, ctx_out, batch, seq, hidden, heads, causal, dtype="fp16", stream=None):
    """The tcgen05 attention core (K5t; the engine uses it from 384 tokens, opts.attention_tc)."""
    _check(lib.dp_attention_tc(_dptr(qkv), int(ldqkv), _dptr(ctx_out), int(batch), int(seq), int(hidden), int(heads),
                               int(bool(causal)), DTYPES[dtype], _stream_ptr(stream)))


# --------------------------------------------------------------------------------------
# Serving harness
# --------------------------------------------------------------------------------------

def plan_resident_bytes(model: "Model", plan: "PlanArrays") -> int:
    """HBM bytes the model holds when resident under `plan` (loaded units only)."""
    return int(lib.dp_plan_resident_bytes(model.h, C.byref(plan.s)))


def serve_run(arrival_ns, instance, *, ngpu, per_gpu_budget_bytes, cold_ns, warm_ns, resident_bytes,
              model_of_instance, slo_ns=100_000_000, dry_run=True, ctx: Context | None = None, models=None,
              plans=None, batch=1, seq=128, plan_mode="DHA", k_max=1, seq_of_model=None, prewarm=True):
    arrival_ns = _i64(arrival_ns)
    instance = np.ascontiguousarray(instance, dtype=np.int32)
    n = len(arrival_ns)
    trace = (TraceEvent * max(n, 1))()
    for i in range(n):
        trace[i].arrival_ns = int(arrival_ns[i])
        trace[i].instance = int(instance[i])
    cold = _i64(cold_ns)
    warm = _i64(warm_ns)
    rb = _i64(resident_bytes)
    moi = np.ascontiguousarray(model_of_instance, dtype=np.int32)
    o = ServeOpts()
    o.plan_mode = _mode(plan_mode)
    o.k_max = int(k_max)
    o.ngpu = int(ngpu)
    o.dry_run = int(bool(dry_run))
    o.no_prewarm = 0 if prewarm else 1
    o.per_gpu_budget_bytes = int(per_gpu_budget_bytes)
    o.slo_ns = int(slo_ns)
    o.nmodels = len(cold)
    o.cold_ns = _ptr(cold, i64p)
    o.warm_ns = _ptr(warm, i64p)
    o.resident_bytes = _ptr(rb, i64p)
    o.model_of_instance = _ptr(moi, i32p)
    o.ninstances = len(moi)
    o.batch = int(batch)
    o.seq = int(seq)
    som = None
    if seq_of_model is not None:
        som = np.ascontiguousarray(seq_of_model, dtype=np.int32)
        o.seq_of_model = _ptr(som, i32p)
    mh = None
    if not dry_run:
        pp = (C.POINTER(Plan) * len(plans))(*[C.pointer(p.s) for p in plans])
        o.plans = C.cast(pp, C.POINTER(C.POINTER(Plan)))
        mh = (vp * len(models))(*[m.h.value for m in models])
    res = (ServeResult * max(n, 1))()
    _check(lib.dp_serve_run(ctx.h if ctx else None, mh, len(models) if models else 0, trace, n, C.byref(o), res))
    out = {k: np.array([getattr(res[i], k) for i in range(n)], dtype=np.int64)
           for k in ("start_ns", "finish_ns", "gpu", "cold", "nevicted", "sec_mask", "decide_ns")}
    return out
