"""Thin Python layer over the C ABI: torch tensors in, C pointers out.

PyTorch provides device memory and streams only; every step of the path
runs in libe3.so.  Names follow the C ABI (include/e3.h):

    DeviceModel      weights of an EE model resident in HBM (bf16)
    split_desc       e3_split_desc for layers [begin, end) of a model
    Split            e3_split_create / e3_split_run
    Queue            e3_queue_* and e3_rebatch
    Comm             e3_comm_* (NCCL world communicator, or an in-process loopback set)
    Pipeline         e3_pipeline_create / e3_pipeline_run / e3_pipeline_trace
    ExitBuffers      device arrays of exit records indexed by input id
    ops              kernel-level entry points (e3_ops.h)
"""
from __future__ import annotations

import ctypes as C
from typing import List, Optional, Sequence

import numpy as np
import torch

from . import _lib
from ._lib import check, lib

_LAYER_KEYS = ("w_qkv", "b_qkv", "w_o", "b_o", "ln1_g", "ln1_b", "w_1", "b_1", "w_2", "b_2", "w_3",
               "ln2_g", "ln2_b")
_RAMP_KEYS = ("w_p", "b_p", "w_c", "b_c", "ln_g", "ln_b")


def _ptr(t: Optional[torch.Tensor]):
    return None if t is None else C.c_void_p(t.data_ptr())


def _stream(stream) -> C.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


def to_bf16(a, device) -> torch.Tensor:
    """float32 array holding bf16-representable values -> bf16 tensor (exact)."""
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32))
    return t.to(device=device, dtype=torch.bfloat16)


class DeviceModel:
    """EE-model weights uploaded once to HBM; builds the e3_weights struct.

    llama: layer tensors w_gate / w_up / w_down travel as w_1 / w_3 / w_2; the
    ramps share one LM head (uploaded once); `kv` is the KVCache the decode
    step reads and appends to."""

    _LLAMA_NAMES = {"w_gate": "w_1", "w_up": "w_3", "w_down": "w_2"}

    def __init__(self, cfg, weights, device="cuda:0", kv=None):
        self.cfg = cfg
        self.device = torch.device(device)
        ren = self._LLAMA_NAMES if cfg.arch == "llama" else {}
        self.layers = [{ren.get(k, k): to_bf16(v, self.device) for k, v in w.items()} for w in weights["layers"]]
        uploaded = {}
        self.ramps = []
        for w in weights["ramps"]:
            if id(w) not in uploaded:
                uploaded[id(w)] = {k: to_bf16(v, self.device) for k, v in w.items()}
            self.ramps.append(uploaded[id(w)])
        n_l, n_r = len(self.layers), len(self.ramps)
        self._lw = (_lib.LayerWeights * max(n_l, 1))()
        for i, w in enumerate(self.layers):
            for k in _LAYER_KEYS:
                setattr(self._lw[i], k, w[k].data_ptr() if k in w else None)
        self._rw = (_lib.RampWeights * max(n_r, 1))()
        for i, w in enumerate(self.ramps):
            for k in _RAMP_KEYS:
                setattr(self._rw[i], k, w[k].data_ptr() if k in w else None)
        self.kv = kv
        self.c_weights = _lib.Weights(n_l, self._lw, n_r, self._rw, C.pointer(kv.c) if kv is not None else None)

    def ramp_struct(self, r):
        return self._rw[r]


class KVCache:
    """Caller-owned KV cache of the llama decode step (e3_kv_cache): per layer
    K and V [n_slots, kv_heads, max_ctx, head_dim] bf16, the slot of every
    token id and the cached length of every slot."""

    def __init__(self, cfg, n_slots, max_ctx, id_capacity, device="cuda:0", dtype="bf16"):
        """dtype: element type of the cache, that of the splits reading it
        ("bf16" for E3_DTYPE_BF16 splits, "fp32" for E3_DTYPE_FP32)."""
        dev = torch.device(device)
        kvh, d = cfg.kv_heads or cfg.heads, cfg.head_dim
        shape = (n_slots, kvh, max_ctx, d)
        tdt = {"bf16": torch.bfloat16, "fp32": torch.float32}[dtype]
        self.k = [torch.zeros(shape, dtype=tdt, device=dev) for _ in range(cfg.layers)]
        self.v = [torch.zeros(shape, dtype=tdt, device=dev) for _ in range(cfg.layers)]
        self.slot_of_id = torch.zeros(id_capacity, dtype=torch.int32, device=dev)
        self.pos_of_slot = torch.full((n_slots,), cfg.ctx, dtype=torch.int32, device=dev)
        self._kp = (C.c_void_p * cfg.layers)(*[t.data_ptr() for t in self.k])
        self._vp = (C.c_void_p * cfg.layers)(*[t.data_ptr() for t in self.v])
        self.c = _lib.KVCache(cfg.layers, self._kp, self._vp, n_slots, max_ctx, self.slot_of_id.data_ptr(),
                              id_capacity, self.pos_of_slot.data_ptr())


def split_desc(cfg, begin: int, end: int, tau, batch: Optional[int] = None,
               inner: str = "exact", dtype: str = "bf16") -> _lib.SplitDesc:
    """e3_split_desc for layers [begin, end) of cfg (must end in a ramp).
    dtype: "bf16" (bf16 activations) or "fp32" (fp32 activations, E3_DTYPE_FP32)."""
    d = _lib.SplitDesc()
    d.arch = _lib.ARCH[cfg.arch]
    d.dtype = _lib.DTYPE[dtype]
    d.hidden, d.heads, d.kv_heads, d.ffn = cfg.hidden, cfg.heads, cfg.kv_heads, cfg.ffn
    d.seq_len, d.num_labels, d.ctx_len = cfg.seq, cfg.classes, cfg.ctx
    d.norm_eps = cfg.norm_eps
    d.layer_begin, d.layer_end = begin, end
    rs = [(r, l) for r, l in enumerate(cfg.ramp_layers) if begin <= l < end]
    d.n_ramps = len(rs)
    for j, (r, l) in enumerate(rs):
        d.ramp_layer[j] = l
        d.ramp_index[j] = r
        d.tau[j] = float(tau[r])
    d.test = _lib.TEST[cfg.test]
    d.final_ramp = int(bool(rs) and rs[-1][0] == cfg.n_ramps - 1)
    d.inner = _lib.INNER[inner]
    d.batch = cfg.batch if batch is None else batch
    d.rope_theta = float(getattr(cfg, "rope_theta", 10000.0))
    return d


class ExitBuffers:
    """Exit records indexed by input id (e3_exits)."""

    def __init__(self, capacity: int, classes: int, n_ramps: int, device, logits=True, hidden=0,
                 hidden_dtype=torch.bfloat16, ramp_metrics=False):
        """hidden > 0: also record each token's exit hidden row ([capacity,
        hidden], the activation dtype) -- needed by Pipeline.decode.
        ramp_metrics: also record the exit metric of every ramp a row is
        evaluated at ([capacity, n_ramps], NaN where not evaluated)."""
        dev = torch.device(device)
        self.capacity = capacity
        self.exit_layer = torch.full((capacity,), -1, dtype=torch.int32, device=dev)
        self.label = torch.full((capacity,), -1, dtype=torch.int32, device=dev)
        self.conf = torch.full((capacity,), float("nan"), dtype=torch.float32, device=dev)
        self.logits = torch.zeros((capacity, classes), dtype=torch.float32, device=dev) if logits else None
        self.n_exit = torch.zeros((1,), dtype=torch.int32, device=dev)
        self.ramp_count = torch.zeros((max(n_ramps, 1),), dtype=torch.int32, device=dev)
        # dependent exits (E3_TEST_PATIENCE): per-input counter state, zero per job
        self.state = torch.zeros((capacity,), dtype=torch.int32, device=dev)
        self.hidden = torch.zeros((capacity, hidden), dtype=hidden_dtype, device=dev) if hidden else None
        self.ramp_metric = torch.full((capacity, max(n_ramps, 1)), float("nan"), dtype=torch.float32,
                                      device=dev) if ramp_metrics else None
        self.c = _lib.Exits(self.exit_layer.data_ptr(), self.label.data_ptr(), self.conf.data_ptr(),
                            None if self.logits is None else self.logits.data_ptr(), capacity,
                            self.n_exit.data_ptr(), self.ramp_count.data_ptr(), self.state.data_ptr(),
                            None if self.hidden is None else self.hidden.data_ptr(),
                            None if self.ramp_metric is None else self.ramp_metric.data_ptr(), max(n_ramps, 1))

    def reset(self):
        self.exit_layer.fill_(-1)
        self.label.fill_(-1)
        self.conf.fill_(float("nan"))
        if self.logits is not None:
            self.logits.zero_()
        self.n_exit.zero_()
        self.ramp_count.zero_()
        self.state.zero_()
        if self.ramp_metric is not None:
            self.ramp_metric.fill_(float("nan"))


class Split:
    """One split on one constant-size batch (e3_split_create / e3_split_run)."""

    def __init__(self, model: DeviceModel, desc: _lib.SplitDesc):
        self.model, self.desc = model, desc
        h = C.c_void_p()
        check(lib.e3_split_create(C.byref(desc), C.byref(model.c_weights), model.device.index or 0,
                                  C.byref(h)), "e3_split_create")
        self.h = h

    def run(self, x, ids, x_out, id_out, n_surv, exits: Optional[ExitBuffers] = None,
            n_valid: Optional[torch.Tensor] = None, stream=None):
        check(lib.e3_split_run(self.h, _stream(stream), _ptr(x), _ptr(ids), _ptr(n_valid), _ptr(x_out),
                               _ptr(id_out), _ptr(n_surv), C.byref(exits.c) if exits else None),
              "e3_split_run")

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None and _lib.lib is not None:
            _lib.lib.e3_split_destroy(self.h)
            self.h = None


class Queue:
    """Device FIFO of survivor rows (e3_queue_*), with e3_rebatch top-up."""

    def __init__(self, device, row_bytes: int, cap_rows: int):
        h = C.c_void_p()
        check(lib.e3_queue_create(torch.device(device).index or 0, row_bytes, cap_rows, C.byref(h)),
              "e3_queue_create")
        self.h = h

    def push(self, rows, ids, n_dev, max_rows, stream=None):
        check(lib.e3_queue_push(self.h, _stream(stream), _ptr(rows), _ptr(ids), _ptr(n_dev), max_rows),
              "e3_queue_push")

    def count(self) -> int:
        c = C.c_int32()
        check(lib.e3_queue_count(self.h, C.byref(c)), "e3_queue_count")
        return c.value

    def rebatch(self, B, flush, x_out, id_out, n_valid_dev, stream=None) -> bool:
        e = C.c_int32()
        check(lib.e3_rebatch(self.h, _stream(stream), B, int(flush), _ptr(x_out), _ptr(id_out),
                             _ptr(n_valid_dev), C.byref(e)), "e3_rebatch")
        return bool(e.value)

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None and _lib.lib is not None:
            _lib.lib.e3_queue_destroy(self.h)
            self.h = None


def make_plan(cfg, bounds: Sequence[int], tau, batch=None, inner="exact", lag=1,
              queue_cap_batches=4, trace=False, dtype="bf16", placement=None, transport="nccl",
              deterministic=False) -> _lib.Plan:
    """Plan with split s covering layers [bounds[s], bounds[s+1]).

    placement: None (every split on the calling rank) or, per split, the list
    of communicator ranks hosting its replicas (e3_plan.replicas/device_of)."""
    p = _lib.Plan()
    p.n_splits = len(bounds) - 1
    for s in range(p.n_splits):
        p.split[s] = split_desc(cfg, bounds[s], bounds[s + 1], tau, batch, inner, dtype)
    p.lag = lag
    p.queue_cap_batches = queue_cap_batches
    p.trace = int(trace)
    if placement is not None:
        assert len(placement) == p.n_splits
        off = 0
        for s, ranks in enumerate(placement):
            p.replicas[s] = len(ranks)
            for j, r in enumerate(ranks):
                p.device_of[off + j] = int(r)
            off += len(ranks)
    p.transport = _lib.TRANSPORT[transport]
    p.deterministic = int(deterministic)
    return p


class Comm:
    """e3_comm: the library-owned communicator of one rank.

    Comm.unique_id() on one rank, broadcast the bytes (torch.distributed), then
    Comm.nccl(uid, rank, world, device) on every rank; or Comm.loopback(world,
    device) for every rank of a plan inside this process (one device)."""

    def __init__(self, handle):
        self.h = handle

    @staticmethod
    def unique_id() -> bytes:
        buf = C.create_string_buffer(_lib.E3_COMM_ID_BYTES)
        check(lib.e3_comm_unique_id(buf), "e3_comm_unique_id")
        return buf.raw

    @classmethod
    def nccl(cls, uid: bytes, rank: int, world: int, device: int) -> "Comm":
        h = C.c_void_p()
        check(lib.e3_comm_init(C.create_string_buffer(uid, _lib.E3_COMM_ID_BYTES), rank, world, device,
                               C.byref(h)), "e3_comm_init")
        return cls(h)

    @classmethod
    def loopback(cls, world: int, device: int = 0) -> List["Comm"]:
        hs = (C.c_void_p * world)()
        check(lib.e3_comm_init_loopback(world, device, hs), "e3_comm_init_loopback")
        return [cls(C.c_void_p(hs[i])) for i in range(world)]

    def rank_world(self):
        r, w = C.c_int32(), C.c_int32()
        check(lib.e3_comm_rank(self.h, C.byref(r), C.byref(w)), "e3_comm_rank")
        return r.value, w.value

    def close(self):
        if getattr(self, "h", None) and _lib is not None and _lib.lib is not None:
            _lib.lib.e3_comm_destroy(self.h)
            self.h = None


class Pipeline:
    """The splits of a plan this rank hosts (e3_pipeline_*): all of them on one
    GPU, or this rank's stage of a multi-rank plan (comm given)."""

    def __init__(self, model: DeviceModel, plan: _lib.Plan, comm: Optional[Comm] = None):
        self.model, self.plan, self.comm = model, plan, comm
        h = C.c_void_p()
        check(lib.e3_pipeline_create(C.byref(plan), C.byref(model.c_weights), model.device.index or 0,
                                     comm.h if comm is not None else None, C.byref(h)), "e3_pipeline_create")
        self.h = h
        self.B = plan.split[0].batch

    def run(self, x, ids, exits: ExitBuffers, stream=None) -> _lib.Stats:
        """x [n,S,H] and ids [n] int64, both on the device or both on the host
        (x None / ids None: no inputs on this rank)."""
        st = _lib.Stats()
        n = int(ids.shape[0]) if ids is not None else 0
        check(lib.e3_pipeline_run(self.h, _stream(stream), _ptr(x) if n else None,
                                  _ptr(ids) if n else None, n, C.byref(exits.c), C.byref(st)),
              "e3_pipeline_run")
        return st

    def run_out(self, x, ids, exits: ExitBuffers, x_out, id_out, stream=None):
        """Stage of a stage pipeline: survivors of the (non-final) last split are
        appended to x_out / id_out; returns (stats, number of survivors)."""
        st = _lib.Stats()
        n_out = C.c_int64()
        n = int(ids.shape[0])
        check(lib.e3_pipeline_run_out(self.h, _stream(stream), _ptr(x) if n else None, _ptr(ids) if n else None,
                                      n, C.byref(exits.c), C.byref(st), _ptr(x_out), _ptr(id_out),
                                      int(id_out.shape[0]), C.byref(n_out)), "e3_pipeline_run_out")
        return st, n_out.value

    def decode(self, x, ids, steps: int, embed, exits: ExitBuffers, stream=None):
        """Multi-step greedy early-exit decode (e3_decode_run): x [n, H] the
        first inputs (overwritten with the next inputs), ids [n], embed [V, H]
        on the device; returns (tokens [steps, n] int32, stats)."""
        n = int(ids.shape[0])
        tokens = torch.empty((steps, n), dtype=torch.int32, device=ids.device)
        st = _lib.Stats()
        check(lib.e3_decode_run(self.h, _stream(stream), _ptr(x), _ptr(ids), n, steps, _ptr(embed), _ptr(tokens),
                                C.byref(exits.c), C.byref(st)), "e3_decode_run")
        return tokens, st

    def trace(self):
        n = C.c_int64()
        check(lib.e3_pipeline_trace(self.h, None, None, None, 0, C.byref(n)), "e3_pipeline_trace")
        k = n.value
        split = (C.c_int32 * max(k, 1))()
        nv = (C.c_int32 * max(k, 1))()
        ids = np.zeros(max(k, 1) * self.B, dtype=np.int64)
        check(lib.e3_pipeline_trace(self.h, split, nv, ids.ctypes.data_as(C.c_void_p), k, C.byref(n)),
              "e3_pipeline_trace")
        ids = ids[:k * self.B].reshape(k, self.B)
        return [(split[i], nv[i], tuple(int(v) for v in ids[i, :nv[i]])) for i in range(k)]

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None and _lib.lib is not None:
            _lib.lib.e3_pipeline_destroy(self.h)
            self.h = None


class ops:
    """Kernel-level entry points (include/e3_ops.h)."""

    @staticmethod
    def dec_gemm(X, W, epilogue="store", W2=None, resid=None, out=None, stream=None):
        """Decode GEMM (swap-AB tcgen05, stream-K): X [T,K] bf16, W [N,K]."""
        T, K = X.shape
        N = W.shape[0]
        out = torch.empty((T, N), dtype=torch.bfloat16, device=X.device) if out is None else out
        epi = {"store": 0, "resid": 1, "swiglu": 2}[epilogue]
        check(lib.e3_op_dec_gemm(_stream(stream), _ptr(X), T, _ptr(W), _ptr(W2), N, K, epi, _ptr(resid), _ptr(out)),
              "e3_op_dec_gemm")
        return out

    @staticmethod
    def gemm_ln(A, W, bias, resid, g, b, eps, pre=None, out=None, stream=None):
        """out = LN(A W^T + bias + resid) (fused O projection + LayerNorm); pre
        receives the pre-LN rows when given."""
        M, K = A.shape
        N = W.shape[0]
        out = torch.empty((M, N), dtype=torch.bfloat16, device=A.device) if out is None else out
        check(lib.e3_op_gemm_ln(_stream(stream), _ptr(A), _ptr(W), _ptr(bias), _ptr(resid), _ptr(g), _ptr(b),
                                float(eps), _ptr(pre), _ptr(out), M, N, K), "e3_op_gemm_ln")
        return out

    @staticmethod
    def gemm(A, W, bias, epilogue="bias", resid=None, out=None, stream=None):
        M, K = A.shape
        N = W.shape[0]
        out = torch.empty((M, N), dtype=torch.bfloat16, device=A.device) if out is None else out
        check(lib.e3_op_gemm(_stream(stream), _ptr(A), A.stride(0), _ptr(W), _ptr(bias), _ptr(resid),
                             _ptr(out), M, N, K, _lib.EPI[epilogue]), "e3_op_gemm")
        return out

    @staticmethod
    def attention(qkv, B, S, H, heads, out=None, stream=None):
        out = torch.empty((B * S, H), dtype=torch.bfloat16, device=qkv.device) if out is None else out
        check(lib.e3_op_attention(_stream(stream), _ptr(qkv), _ptr(out), B, S, H, heads), "e3_op_attention")
        return out

    @staticmethod
    def layernorm(x, g, b, eps, out=None, stream=None):
        rows, H = x.shape
        out = torch.empty_like(x) if out is None else out
        check(lib.e3_op_layernorm(_stream(stream), _ptr(x), _ptr(g), _ptr(b), _ptr(out), rows, H, eps),
              "e3_op_layernorm")
        return out

    @staticmethod
    def ramp(cfg, model: DeviceModel, r, x, ids, tau, alive, exits: ExitBuffers, final=False,
             layer=None, init_alive=True, n_valid=None, stream=None):
        B, S, H = x.shape
        layer = cfg.ramp_layers[r] if layer is None else layer
        rw = model.ramp_struct(r)
        check(lib.e3_op_ramp(_stream(stream), _lib.ARCH[cfg.arch], _ptr(x), _ptr(ids), B, S, H, cfg.classes,
                             C.byref(rw), _lib.TEST[cfg.test], float(tau), int(final), layer, r,
                             cfg.norm_eps, _ptr(alive), int(init_alive), _ptr(n_valid), C.byref(exits.c)),
              "e3_op_ramp")

    @staticmethod
    def compact(x, ids, alive, x_out, id_out, n_surv, stream=None):
        B = x.shape[0]
        row_bytes = x[0].numel() * x.element_size()
        check(lib.e3_op_compact(_stream(stream), _ptr(x), _ptr(ids), _ptr(alive), B, row_bytes, _ptr(x_out),
                                _ptr(id_out), _ptr(n_surv)), "e3_op_compact")
