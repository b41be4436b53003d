"""ctypes binding of libe3.so (include/e3.h, include/e3_ops.h).

Argument marshalling only: every step of the path runs in the CUDA library.
There is no fallback: if libe3.so is missing or fails to load, importing
this module raises (build it with ``python -m paper_conf_sosp_iyergdpgn24_b200.build``).
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("E3_LIB_PATH") or os.path.join(HERE, "libe3.so")   # override: diagnostics only

E3_MAX_RAMPS = 64
E3_MAX_SPLITS = 64
E3_MAX_REPLICA_SLOTS = 256
E3_COMM_ID_BYTES = 128

STATUS = {0: "E3_OK", 1: "E3_EINVAL", 2: "E3_EUNSUPPORTED", 3: "E3_ECUDA", 4: "E3_ENCCL",
          5: "E3_ECAPACITY", 6: "E3_ESTATE"}

ARCH = {"bert": 0, "vit": 1, "llama": 2}
TEST = {"maxprob": 0, "entropy": 1, "patience": 2}
INNER = {"exact": 0, "disabled": 1}
DTYPE = {"bf16": 0, "fp32": 1}
EPI = {"bias": 0, "bias_gelu": 1, "bias_resid": 2}
TRANSPORT = {"nccl": 0, "p2p": 1, "loopback": 2}

P = C.c_void_p
I32 = C.c_int32
I64 = C.c_int64


class E3Error(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = lib.e3_last_error().decode(errors="replace") if lib is not None else ""
        super().__init__(f"{where}: {STATUS.get(status, status)}: {msg}")


class SplitDesc(C.Structure):
    _fields_ = [("arch", I32), ("dtype", I32), ("hidden", I32), ("heads", I32), ("kv_heads", I32),
                ("ffn", I32), ("seq_len", I32), ("num_labels", I32), ("ctx_len", I32),
                ("norm_eps", C.c_float), ("layer_begin", I32), ("layer_end", I32), ("n_ramps", I32),
                ("ramp_layer", I32 * E3_MAX_RAMPS), ("ramp_index", I32 * E3_MAX_RAMPS),
                ("tau", C.c_float * E3_MAX_RAMPS), ("test", I32), ("final_ramp", I32),
                ("inner", I32), ("batch", I32), ("rope_theta", C.c_float)]


class LayerWeights(C.Structure):
    _fields_ = [(n, P) for n in ("w_qkv", "b_qkv", "w_o", "b_o", "ln1_g", "ln1_b", "w_1", "b_1",
                                 "w_2", "b_2", "ln2_g", "ln2_b", "w_3")]


class RampWeights(C.Structure):
    _fields_ = [(n, P) for n in ("w_p", "b_p", "w_c", "b_c", "ln_g", "ln_b")]


class KVCache(C.Structure):
    _fields_ = [("n_layers", I32), ("k", C.POINTER(P)), ("v", C.POINTER(P)), ("n_slots", I32),
                ("max_ctx", I32), ("slot_of_id", P), ("id_capacity", I64), ("pos_of_slot", P)]


class Weights(C.Structure):
    _fields_ = [("n_layers", I32), ("layer", C.POINTER(LayerWeights)), ("n_ramps", I32),
                ("ramp", C.POINTER(RampWeights)), ("kv", C.POINTER(KVCache))]


class Exits(C.Structure):
    _fields_ = [("exit_layer", P), ("label", P), ("conf", P), ("logits", P), ("capacity", I64),
                ("n_exit", P), ("ramp_count", P), ("state", P), ("hidden", P), ("ramp_metric", P),
                ("ramp_metric_stride", I32)]


class Plan(C.Structure):
    _fields_ = [("n_splits", I32), ("split", SplitDesc * E3_MAX_SPLITS), ("lag", I32),
                ("queue_cap_batches", I32), ("trace", I32), ("replicas", I32 * E3_MAX_SPLITS),
                ("device_of", I32 * E3_MAX_REPLICA_SLOTS), ("transport", I32), ("deterministic", I32)]


class Stats(C.Structure):
    _fields_ = [("runs", I64), ("batches", I64 * E3_MAX_SPLITS), ("valid_rows", I64 * E3_MAX_SPLITS),
                ("padded_rows", I64 * E3_MAX_SPLITS), ("rows_out", I64 * E3_MAX_SPLITS),
                ("host_waits", I64), ("host_launch_ms", C.c_double), ("host_sync_ms", C.c_double),
                ("msgs_sent", I64), ("msgs_recv", I64), ("flushes", I64 * E3_MAX_SPLITS)]


# name -> (restype, argtypes); every symbol include/*.h declares
SIGNATURES = {
    "e3_last_error": (C.c_char_p, []),
    "e3_version": (C.c_char_p, []),
    "e3_split_create": (I32, [C.POINTER(SplitDesc), C.POINTER(Weights), C.c_int, C.POINTER(P)]),
    "e3_split_destroy": (I32, [P]),
    "e3_split_run": (I32, [P, P, P, P, P, P, P, P, C.POINTER(Exits)]),
    "e3_queue_create": (I32, [C.c_int, I64, I32, C.POINTER(P)]),
    "e3_queue_destroy": (I32, [P]),
    "e3_queue_push": (I32, [P, P, P, P, P, I32]),
    "e3_queue_count": (I32, [P, C.POINTER(I32)]),
    "e3_rebatch": (I32, [P, P, I32, I32, P, P, P, C.POINTER(I32)]),
    "e3_comm_unique_id": (I32, [C.c_char_p]),
    "e3_comm_init": (I32, [C.c_char_p, C.c_int, C.c_int, C.c_int, C.POINTER(P)]),
    "e3_comm_init_loopback": (I32, [C.c_int, C.c_int, C.POINTER(P)]),
    "e3_comm_rank": (I32, [P, C.POINTER(I32), C.POINTER(I32)]),
    "e3_comm_destroy": (I32, [P]),
    "e3_pipeline_create": (I32, [C.POINTER(Plan), C.POINTER(Weights), C.c_int, P, C.POINTER(P)]),
    "e3_pipeline_destroy": (I32, [P]),
    "e3_pipeline_run": (I32, [P, P, P, P, I64, C.POINTER(Exits), C.POINTER(Stats)]),
    "e3_pipeline_run_out": (I32, [P, P, P, P, I64, C.POINTER(Exits), C.POINTER(Stats), P, P, I64,
                                  C.POINTER(I64)]),
    "e3_pipeline_trace": (I32, [P, P, P, P, I64, C.POINTER(I64)]),
    "e3_decode_run": (I32, [P, P, P, P, I64, I32, P, P, C.POINTER(Exits), C.POINTER(Stats)]),
    "e3_op_gemm": (I32, [P, P, I64, P, P, P, P, I32, I32, I32, I32]),
    "e3_op_dec_gemm": (I32, [P, P, I32, P, P, I32, I32, I32, P, P]),
    "e3_op_gemm_ln": (I32, [P, P, P, P, P, P, P, C.c_float, P, P, I32, I32, I32]),
    "e3_op_attention": (I32, [P, P, P, I32, I32, I32, I32]),
    "e3_op_layernorm": (I32, [P, P, P, P, P, I32, I32, C.c_float]),
    "e3_op_ramp": (I32, [P, I32, P, P, I32, I32, I32, I32, C.POINTER(RampWeights), I32, C.c_float, I32,
                         I32, I32, C.c_float, P, I32, P, C.POINTER(Exits)]),
    "e3_op_compact": (I32, [P, P, P, P, I32, I64, P, P, P]),
    "e3_kernel_launches": (C.c_longlong, []),
    "e3_profile_enable": (I32, [I32]),
    "e3_debug_gemm_trace": (I32, [P]),
    "e3_debug_timeline": (I32, [P]),
    "e3_profile_reset": (I32, []),
    "e3_profile_read": (I32, [I32, C.POINTER(C.c_double), C.POINTER(C.c_double), C.POINTER(C.c_double),
                              C.POINTER(C.c_longlong), C.POINTER(C.c_char_p)]),
}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built; run python -m paper_conf_sosp_iyergdpgn24_b200.build")
    L = C.CDLL(LIB_PATH)
    for name, (res, args) in SIGNATURES.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = None
lib = _load()


def check(status, where):
    if status != 0:
        raise E3Error(status, where)
