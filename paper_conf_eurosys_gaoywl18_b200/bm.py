"""Thin ctypes binding of the C-ABI in include/bm.h (libbm.so): argument marshalling only.

Every step of the hot path runs inside libbm.so (C++ scheduler + sm_100a kernels). There is
no Python or CPU fallback: if libbm.so is missing this module raises at import, and on a
machine without an sm_100 GPU bm_create fails with BM_E_NODEV (except the BM_CLOCK_DRY
scheduler-only mode, which never touches a device).
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbm.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with "
                      "`python -m paper_conf_eurosys_gaoywl18_b200.build` (no CPU fallback exists)")
lib = C.CDLL(LIB_PATH)

# ---------------------------------------------------------------- constants (bm.h)
OK, E_INVAL, E_NOMEM, E_FULL, E_AGAIN, E_CUDA, E_STATE, E_NODEV = 0, -1, -2, -3, -4, -5, -6, -7
PREC_BF16, PREC_FP32 = 0, 1
CLOCK_WALL, CLOCK_VIRTUAL, CLOCK_DRY = 0, 1, 2
CELL_LSTM, CELL_LSTM_PROJ, CELL_TREE_LEAF, CELL_TREE_INTERNAL = 0, 1, 2, 3
REQ_CHAIN, REQ_SEQ2SEQ, REQ_TREE = 0, 1, 2
POLICY_CELLULAR, POLICY_GRAPH = 0, 1
ROW_FIRST, ROW_LAST, ROW_PARITY = 1, 2, 4


class Config(C.Structure):
    _fields_ = [(n, C.c_int) for n in (
        "device", "precision", "clock", "hidden", "pool_layers", "max_slots", "max_requests",
        "max_tasks_to_submit", "min_followon_batch", "schedule_when_outstanding_leq",
        "max_decode_len", "keep_results", "record_logits", "time_kernels", "record_log",
        "persistent", "policy", "bucket_width", "workers", "devices")] + [
        ("roof_hbm_gbs", C.c_double), ("roof_tc_tflops", C.c_double)]


class CellDesc(C.Structure):
    _fields_ = [(n, C.c_int) for n in ("kind", "hidden", "layers", "vocab", "max_batch", "priority")]


class Weights(C.Structure):
    _fields_ = [("W", C.POINTER(C.POINTER(C.c_float))), ("b", C.POINTER(C.POINTER(C.c_float))),
                ("E", C.POINTER(C.c_float)), ("W_out", C.POINTER(C.c_float)),
                ("b_out", C.POINTER(C.c_float))]


class Request(C.Structure):
    _fields_ = [("kind", C.c_int), ("cell0", C.c_int), ("cell1", C.c_int), ("n", C.c_int),
                ("tokens", C.POINTER(C.c_int32)), ("decode_len", C.c_int),
                ("left", C.POINTER(C.c_int32)), ("right", C.POINTER(C.c_int32)),
                ("arrival", C.c_double), ("user_tag", C.c_uint64),
                ("eos_stop", C.c_int), ("eos_id", C.c_int32), ("dry_eos_step", C.c_int)]


class Completion(C.Structure):
    _fields_ = [("req_id", C.c_uint64), ("user_tag", C.c_uint64), ("t_arrival", C.c_double),
                ("t_first", C.c_double), ("t_done", C.c_double)]


class Result(C.Structure):
    _fields_ = [("h", C.POINTER(C.c_float)), ("c", C.POINTER(C.c_float)),
                ("tokens", C.POINTER(C.c_int32)), ("logits", C.POINTER(C.c_float))]


class TaskRecord(C.Structure):
    _fields_ = [("task", C.c_int), ("cell", C.c_int), ("tick", C.c_double),
                ("first_row", C.c_int), ("n_rows", C.c_int), ("worker", C.c_int)]


class RowRecord(C.Structure):
    _fields_ = [("req_id", C.c_uint64), ("node", C.c_int), ("slot", C.c_int)]


class StepRow(C.Structure):
    _fields_ = [("a", C.c_int32), ("b", C.c_int32), ("slot", C.c_int32), ("flags", C.c_int32)]


K_LSTM_PAIR, K_LSTM, K_LEAF, K_INTERNAL, K_PROJ, K_SIMT, K_PERSISTENT, K_CLASSES = 0, 1, 2, 3, 4, 5, 6, 8
K_NAMES = {K_LSTM_PAIR: "cell_pair_kernel (LSTM, cta_group::2)", K_LSTM: "cell_step_sm100_kernel<EPI_LSTM>",
           K_LEAF: "cell_step_sm100_kernel<EPI_LEAF>", K_INTERNAL: "cell_step_sm100_kernel<EPI_INTERNAL>",
           K_PROJ: "cell_step_sm100_kernel<EPI_PROJ> (projection + argmax)", K_SIMT: "fp32 SIMT cell kernels",
           K_PERSISTENT: "lstm_persistent_kernel (per task)"}


class Stats(C.Structure):
    _fields_ = [("tasks", C.c_uint64), ("rows", C.c_uint64), ("kernel_launches", C.c_uint64),
                ("sched_ns", C.c_double), ("schedule_calls", C.c_uint64),
                ("launch_ns", C.c_double), ("retire_ns", C.c_double),
                ("k_launches", C.c_uint64 * K_CLASSES), ("k_span_launches", C.c_uint64 * K_CLASSES)] + [
        (n, C.c_double * K_CLASSES) for n in ("k_span_ms", "k_rows", "k_bytes", "k_flops", "k_roof_hbm_ms",
                                              "k_roof_tc_ms", "k_roof_ms")] + [
        ("migrations", C.c_uint64), ("migration_bytes", C.c_double)]


class LaunchRecord(C.Structure):
    _fields_ = [("kclass", C.c_int), ("b", C.c_int), ("span_ns", C.c_uint64)]


# exported symbols (tests/test_abi.py checks them against include/bm.h)
_P = C.c_void_p
_SIGS = {
    "bm_config_default": (None, [C.POINTER(Config)]),
    "bm_create": (C.c_int, [C.POINTER(Config), C.POINTER(_P)]),
    "bm_destroy": (None, [_P]),
    "bm_strerror": (C.c_char_p, [C.c_int]),
    "bm_abi_version": (C.c_int, []),
    "bm_load_cell": (C.c_int, [_P, C.POINTER(CellDesc), C.POINTER(Weights), C.POINTER(C.c_int)]),
    "bm_submit": (C.c_int, [_P, C.POINTER(Request), C.POINTER(C.c_uint64)]),
    "bm_submit_many": (C.c_int, [_P, C.POINTER(Request), C.c_int, C.POINTER(C.c_uint64),
                                 C.POINTER(C.c_int)]),
    "bm_schedule_step": (C.c_int, [_P, C.POINTER(C.c_int)]),
    "bm_poll": (C.c_int, [_P, C.POINTER(Completion), C.c_int, C.POINTER(C.c_int)]),
    "bm_run": (C.c_int, [_P, C.POINTER(C.c_int)]),
    "bm_read_result": (C.c_int, [_P, C.c_uint64, C.POINTER(Result)]),
    "bm_release": (C.c_int, [_P, C.c_uint64]),
    "bm_read_results_many": (C.c_int, [_P, C.c_uint64, C.c_int, C.POINTER(C.c_float),
                                       C.POINTER(C.c_float), C.POINTER(C.c_int32), C.c_int]),
    "bm_read_log": (C.c_int, [_P, C.POINTER(TaskRecord), C.c_int, C.POINTER(C.c_int)]),
    "bm_read_log_rows": (C.c_int, [_P, C.POINTER(RowRecord), C.c_int, C.POINTER(C.c_int)]),
    "bm_cell_step": (C.c_int, [_P, C.c_int, C.POINTER(StepRow), C.c_int, C.c_int]),
    "bm_pool_write": (C.c_int, [_P, C.c_int, C.c_int, C.POINTER(C.c_int32), C.c_int,
                                C.POINTER(C.c_float), C.POINTER(C.c_float)]),
    "bm_pool_read": (C.c_int, [_P, C.c_int, C.c_int, C.POINTER(C.c_int32), C.c_int,
                               C.POINTER(C.c_float), C.POINTER(C.c_float)]),
    "bm_result_rows": (C.c_int, [_P, C.POINTER(C.c_int32), C.c_int, C.POINTER(C.c_float),
                                 C.POINTER(C.c_float)]),
    "bm_tokens": (C.c_int, [_P, C.POINTER(C.c_int32), C.c_int, C.POINTER(C.c_int32), C.c_int]),
    "bm_get_stats": (C.c_int, [_P, C.POINTER(Stats)]),
    "bm_reset_stats": (C.c_int, [_P]),
    "bm_read_launch_log": (C.c_int, [_P, C.POINTER(LaunchRecord), C.c_int, C.POINTER(C.c_int)]),
    "bm_stream": (C.c_void_p, [_P]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args


class _Prepared:
    def __init__(self, arr, toks, lr):
        self.arr, self.toks, self.lr = arr, toks, lr
        # numpy view of the arrival field of every bm_request (no per-request Python objects)
        self.arrival = np.ndarray((len(arr),), np.float64, buffer=arr, offset=Request.arrival.offset,
                                  strides=(C.sizeof(Request),))
        self.base_arrival = self.arrival.copy()

    def set_time_scale(self, scale: float):
        """arrival_i = base arrival_i * scale (a unit-rate Poisson trace becomes rate 1/scale)."""
        self.arrival[:] = self.base_arrival * scale


class BMError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {lib.bm_strerror(status).decode()} ({status})")


def _ck(status: int, where: str) -> int:
    if status != OK:
        raise BMError(status, where)
    return status


def _f32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32)


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.int32)


def _fp(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(C.POINTER(C.c_float))


def _ip(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(C.POINTER(C.c_int32))


def default_config(**kw) -> Config:
    cfg = Config()
    lib.bm_config_default(C.byref(cfg))
    for k, v in kw.items():
        setattr(cfg, k, float(v) if k.startswith("roof_") else int(v))
    return cfg


class Engine:
    """One engine per GPU (include/bm.h). Methods mirror the C entry points one to one."""

    def __init__(self, **cfg):
        self.cfg = default_config(**cfg)
        h = C.c_void_p()
        _ck(lib.bm_create(C.byref(self.cfg), C.byref(h)), "bm_create")
        self.h = h
        self._keep = []

    def close(self):
        if getattr(self, "h", None):
            lib.bm_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---------------------------------------------------------------- cells
    def load_cell(self, kind: int, layers: int, vocab: int, max_batch: int, priority: int,
                  W: Sequence[np.ndarray], b: Sequence[np.ndarray], E: Optional[np.ndarray] = None,
                  W_out: Optional[np.ndarray] = None, b_out: Optional[np.ndarray] = None) -> int:
        """Arrays are numpy (host, copied up) or fp32 CUDA tensors on the engine's device
        (anything with data_ptr(): adopted in place, e.g. after an NCCL broadcast)."""
        d = CellDesc(kind, self.cfg.hidden, layers, vocab, max_batch, priority)
        keep = []

        def ptr(x):
            if x is None:
                return None
            if hasattr(x, "data_ptr"):
                keep.append(x)
                return C.cast(C.c_void_p(x.data_ptr()), C.POINTER(C.c_float))
            a = _f32(x)
            keep.append(a)
            return _fp(a)
        Wa = (C.POINTER(C.c_float) * len(W))(*[ptr(x) for x in W])
        ba = (C.POINTER(C.c_float) * len(b))(*[ptr(x) for x in b])
        w = Weights(Wa, ba, ptr(E), ptr(W_out), ptr(b_out))
        cid = C.c_int()
        _ck(lib.bm_load_cell(self.h, C.byref(d), C.byref(w), C.byref(cid)), "bm_load_cell")
        return cid.value

    # ---------------------------------------------------------------- requests
    def submit(self, kind: int, cell0: int, cell1: int, tokens, arrival: float = 0.0,
               decode_len: int = 0, left=None, right=None, tag: int = 0,
               eos_id: Optional[int] = None, dry_eos_step: int = -1) -> int:
        """eos_id (SEQ2SEQ): stop decoding at <eos> = eos_id, decode_len is then the maximum
        length (bm_request.eos_stop); dry_eos_step: BM_CLOCK_DRY scheduler tests only."""
        t = _i32(tokens)
        l = _i32(left) if left is not None else None
        r = _i32(right) if right is not None else None
        q = Request(kind, cell0, cell1, len(t), _ip(t), decode_len, _ip(l), _ip(r),
                    float(arrival), tag, 1 if eos_id is not None else 0,
                    eos_id if eos_id is not None else -1, dry_eos_step)
        rid = C.c_uint64()
        _ck(lib.bm_submit(self.h, C.byref(q), C.byref(rid)), "bm_submit")
        return rid.value

    def prepare_requests(self, reqs, cells_for_kind, time_scale: float = 1.0):
        """Marshal a list of workloads.gen.Request into a bm_request array (kept alive on the
        returned object) for submit_many. cells_for_kind: {kind: (cell0, cell1)}."""
        toks = np.ascontiguousarray(np.concatenate([q.tokens for q in reqs]).astype(np.int32))
        trees = [q for q in reqs if q.left is not None]
        lr = np.ascontiguousarray(np.concatenate([np.concatenate([q.left, q.right]) for q in trees])
                                  .astype(np.int32)) if trees else np.zeros(1, np.int32)
        arr = (Request * len(reqs))()
        base = toks.ctypes.data
        lbase = lr.ctypes.data
        off = loff = 0
        ip = C.POINTER(C.c_int32)
        for i, q in enumerate(reqs):
            c0, c1 = cells_for_kind[q.kind]
            n = len(q.tokens)
            a = arr[i]
            a.kind, a.cell0, a.cell1, a.n = q.kind, c0, c1, n
            a.tokens = C.cast(base + 4 * off, ip)
            a.decode_len = q.decode_len
            if q.left is not None:
                a.left = C.cast(lbase + 4 * loff, ip)
                a.right = C.cast(lbase + 4 * (loff + n), ip)
                loff += 2 * n
            a.arrival = q.arrival * time_scale
            a.user_tag = i
            off += n
        return _Prepared(arr, toks, lr)

    def submit_many(self, prepared) -> int:
        first = C.c_uint64()
        n = C.c_int()
        _ck(lib.bm_submit_many(self.h, prepared.arr, len(prepared.arr), C.byref(first), C.byref(n)),
            "bm_submit_many")
        return first.value

    def read_results_many(self, first_id: int, n: int, h: Optional[np.ndarray] = None,
                          tokens: Optional[np.ndarray] = None, release: bool = True,
                          c: Optional[np.ndarray] = None):
        _ck(lib.bm_read_results_many(self.h, first_id, n, _fp(h), _fp(c), _ip(tokens), 1 if release else 0),
            "bm_read_results_many")

    def schedule_step(self) -> int:
        n = C.c_int()
        s = lib.bm_schedule_step(self.h, C.byref(n))
        if s == E_AGAIN:
            return -1
        _ck(s, "bm_schedule_step")
        return n.value

    _COMP_DT = np.dtype([("req_id", "<u8"), ("user_tag", "<u8"), ("t_arrival", "<f8"),
                         ("t_first", "<f8"), ("t_done", "<f8")])

    def poll_array(self, cap: int = 1 << 16) -> np.ndarray:
        """bm_poll into a numpy structured array (fields as bm_completion): no per-record
        Python objects, for drivers that retire tens of thousands of requests per call."""
        out = np.empty(cap, dtype=self._COMP_DT)
        n = C.c_int()
        _ck(lib.bm_poll(self.h, out.ctypes.data_as(C.POINTER(Completion)), cap, C.byref(n)), "bm_poll")
        return out[:n.value]

    def poll(self, cap: int = 1 << 16) -> List[Completion]:
        buf = (Completion * cap)()
        n = C.c_int()
        _ck(lib.bm_poll(self.h, buf, cap, C.byref(n)), "bm_poll")
        return [buf[i] for i in range(n.value)]

    def run(self) -> int:
        n = C.c_int()
        _ck(lib.bm_run(self.h, C.byref(n)), "bm_run")
        return n.value

    def read_result(self, rid: int, layers: int, decode_len: int = 0, vocab: int = 0):
        H = self.cfg.hidden
        h = np.zeros((layers, H), np.float32)
        c = np.zeros((layers, H), np.float32)
        L = self.cfg.pool_layers
        hh = np.zeros((L, H), np.float32)
        cc = np.zeros((L, H), np.float32)
        toks = np.zeros(max(decode_len, 1), np.int32)
        lg = np.zeros((max(decode_len, 1), vocab), np.float32) if vocab else None
        res = Result(_fp(hh), _fp(cc), _ip(toks), _fp(lg))
        _ck(lib.bm_read_result(self.h, rid, C.byref(res)), "bm_read_result")
        h[:] = hh[:layers]
        c[:] = cc[:layers]
        return {"h": h, "c": c, "tokens": toks[:decode_len], "logits": lg}

    def release(self, rid: int):
        _ck(lib.bm_release(self.h, rid), "bm_release")

    def read_log(self):
        n = C.c_int()
        _ck(lib.bm_read_log(self.h, None, 0, C.byref(n)), "bm_read_log")
        tasks = (TaskRecord * max(n.value, 1))()
        _ck(lib.bm_read_log(self.h, tasks, n.value, C.byref(n)), "bm_read_log")
        m = C.c_int()
        _ck(lib.bm_read_log_rows(self.h, None, 0, C.byref(m)), "bm_read_log_rows")
        rows = (RowRecord * max(m.value, 1))()
        _ck(lib.bm_read_log_rows(self.h, rows, m.value, C.byref(m)), "bm_read_log_rows")
        out = []
        for i in range(n.value):
            t = tasks[i]
            rr = [(int(rows[j].req_id), rows[j].node, rows[j].slot)
                  for j in range(t.first_row, t.first_row + t.n_rows)]
            out.append({"task": t.task, "cell": t.cell, "tick": t.tick, "rows": rr, "worker": t.worker})
        return out

    # ---------------------------------------------------------------- direct cell access
    def cell_step(self, cell: int, rows, sync: bool = True):
        """rows: int32 array [b, 4] = (a, b, slot, flags) per bm_step_row."""
        r = _i32(rows).reshape(-1, 4)
        arr = (StepRow * len(r)).from_buffer_copy(r.tobytes())
        _ck(lib.bm_cell_step(self.h, cell, arr, len(r), 0 if sync else 1), "bm_cell_step")

    def pool_write(self, layer: int, parity: int, slots, h=None, c=None):
        s = _i32(slots)
        hh = _f32(h) if h is not None else None
        cc = _f32(c) if c is not None else None
        _ck(lib.bm_pool_write(self.h, layer, parity, _ip(s), len(s), _fp(hh), _fp(cc)), "bm_pool_write")

    def pool_read(self, layer: int, parity: int, slots):
        s = _i32(slots)
        H = self.cfg.hidden
        h = np.zeros((len(s), H), np.float32)
        c = np.zeros((len(s), H), np.float32)
        _ck(lib.bm_pool_read(self.h, layer, parity, _ip(s), len(s), _fp(h), _fp(c)), "bm_pool_read")
        return h, c

    def result_rows(self, idx):
        i = _i32(idx)
        LH = self.cfg.hidden * self.cfg.pool_layers
        h = np.zeros((len(i), self.cfg.pool_layers, self.cfg.hidden), np.float32)
        c = np.zeros_like(h)
        _ck(lib.bm_result_rows(self.h, _ip(i), len(i), _fp(h), _fp(c)), "bm_result_rows")
        return h, c

    def tokens(self, slots, values=None):
        s = _i32(slots)
        v = _i32(values) if values is not None else np.zeros(len(s), np.int32)
        _ck(lib.bm_tokens(self.h, _ip(s), len(s), _ip(v), 1 if values is not None else 0), "bm_tokens")
        return v

    def stats(self) -> dict:
        st = Stats()
        _ck(lib.bm_get_stats(self.h, C.byref(st)), "bm_get_stats")
        out = {}
        for k, _ in Stats._fields_:
            v = getattr(st, k)
            out[k] = list(v) if k.startswith("k_") else v
        return out

    def reset_stats(self):
        _ck(lib.bm_reset_stats(self.h), "bm_reset_stats")

    _LAUNCH_DT = np.dtype([("kclass", "<i4"), ("b", "<i4"), ("span_ns", "<u8")])

    def launch_log(self, cap: int = 1 << 16) -> np.ndarray:
        """bm_read_launch_log: (kernel class, rows, device span ns) of the last launches."""
        out = np.zeros(cap, dtype=self._LAUNCH_DT)
        n = C.c_int()
        _ck(lib.bm_read_launch_log(self.h, out.ctypes.data_as(C.POINTER(LaunchRecord)), cap, C.byref(n)),
            "bm_read_launch_log")
        return out[:n.value]

    def stream(self) -> int:
        return int(lib.bm_stream(self.h) or 0)
