"""Thin ctypes binding over libmimose.so (include/mimose.h).  Argument
marshalling only: every step of the hot path runs in the library's kernels.
PyTorch supplies device memory (the arena slab), the CUDA stream and, for
data parallelism, the process group that broadcasts the ncclUniqueId.

The library must be built in-tree (``python -m
paper_conf_ipps_liaolysshfyctzlq23_b200.build``); importing this module fails
loudly if it is missing — there is no fallback path.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Dict, List, Optional

import numpy as np

from . import workload as wl

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libmimose.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} missing: build it with `python -m paper_conf_ipps_liaolysshfyctzlq23_b200.build`")
_lib = C.CDLL(LIB_PATH)

OK, E_INVALID, E_STATE, E_NOT_READY, E_INFEASIBLE, E_BUDGET, E_CUDA, E_NCCL, E_NODEVICE = range(9)
PHASE_SHELTERED, PHASE_RESPONSIVE = 0, 1


class MimoseError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"[{status}] {msg}")
        self.status = status


class Config(C.Structure):
    _fields_ = [("arch", C.c_int32), ("head", C.c_int32), ("dtype", C.c_int32),
                ("n_layers", C.c_int32), ("hidden", C.c_int32), ("heads", C.c_int32),
                ("ffn", C.c_int32), ("vocab", C.c_int32), ("max_pos", C.c_int32),
                ("type_vocab", C.c_int32), ("pos_offset", C.c_int32), ("n_choices", C.c_int32),
                ("n_labels", C.c_int32), ("p_drop", C.c_float), ("ln_eps", C.c_float),
                ("seed", C.c_uint64), ("budget_bytes", C.c_int64), ("reserve_bytes", C.c_int64),
                ("enforce_budget", C.c_int32), ("collect_iters", C.c_int32),
                ("bucket_num", C.c_int32), ("bucket_den", C.c_int32), ("degree", C.c_int32),
                ("max_seqs", C.c_int32), ("max_seq_len", C.c_int32),
                ("arena_base", C.c_void_p), ("arena_bytes", C.c_int64), ("stream", C.c_void_p),
                ("rank", C.c_int32), ("world", C.c_int32), ("nccl_id", C.c_void_p),
                ("use_tc", C.c_int32), ("pad_id", C.c_int32), ("granularity", C.c_int32),
                ("comm_force", C.c_int32), ("nccl_max_ctas", C.c_int32), ("check_plans", C.c_int32),
                ("zero1", C.c_int32), ("n_dec_layers", C.c_int32), ("ffn_layers", C.c_void_p)]


class BatchS(C.Structure):
    _fields_ = [("input_ids", C.c_void_p), ("token_type", C.c_void_p), ("lengths", C.c_void_p),
                ("labels", C.c_void_p), ("n_seqs", C.c_int32), ("seq_len", C.c_int32),
                ("on_host", C.c_int32), ("dec_ids", C.c_void_p), ("dec_lengths", C.c_void_p),
                ("dec_len", C.c_int32), ("pad_", C.c_int32)]


class Plan(C.Structure):
    _fields_ = [("drop_mask", C.c_uint64), ("n_dropped", C.c_int32), ("from_cache", C.c_int32),
                ("input_size", C.c_int64), ("predicted_peak", C.c_int64), ("budget", C.c_int64),
                ("status", C.c_int32), ("pad_", C.c_int32)]

    @property
    def dropped(self) -> List[int]:
        return [l for l in range(64) if (self.drop_mask >> l) & 1]


class SampleS(C.Structure):
    _fields_ = [("x", C.c_int64), ("C", C.c_int64), ("E", C.c_int64), ("Hd", C.c_int64),
                ("Th", C.c_int64), ("Tb", C.c_int64), ("Te", C.c_int64),
                ("a", C.c_int64 * 64), ("y", C.c_int64 * 64), ("t_ms", C.c_float * 64), ("xt", C.c_int64)]


class Stats(C.Structure):
    _fields_ = [("live_bytes", C.c_int64), ("peak_bytes", C.c_int64), ("max_peak_bytes", C.c_int64),
                ("persistent_bytes", C.c_int64), ("budget_bytes", C.c_int64), ("violations", C.c_int64),
                ("steps", C.c_int64), ("collect_steps", C.c_int64), ("shuttled_steps", C.c_int64),
                ("plan_calls", C.c_int64), ("plan_cache_hits", C.c_int64), ("plan_cache_misses", C.c_int64),
                ("n_samples", C.c_int64), ("phase", C.c_int32), ("last_n_dropped", C.c_int32),
                ("last_drop_mask", C.c_uint64), ("last_predicted_peak", C.c_int64),
                ("planner_us_total", C.c_double), ("collector_ms_total", C.c_double),
                ("kernel_launches", C.c_int64), ("allreduce_calls", C.c_int64),
                ("allreduce_bytes", C.c_int64), ("plan_checks", C.c_int64),
                ("comm_nranks", C.c_int32), ("pad_", C.c_int32)]

    def asdict(self) -> Dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class Series(C.Structure):
    _fields_ = [("C", C.c_int64), ("E", C.c_int64), ("Hd", C.c_int64), ("Th", C.c_int64),
                ("Tb", C.c_int64), ("Te", C.c_int64), ("a", C.POINTER(C.c_int64)),
                ("y", C.POINTER(C.c_int64)), ("n_layers", C.c_int32)]


_P = C.c_void_p
_lib.mimose_default_config.argtypes = [C.POINTER(Config)]
_lib.mimose_init.argtypes = [C.POINTER(Config), C.POINTER(_P)]
_lib.mimose_destroy.argtypes = [_P]
_lib.mimose_last_error.argtypes = [_P]
_lib.mimose_last_error.restype = C.c_char_p
_lib.mimose_num_params.argtypes = [_P, C.POINTER(C.c_int64)]
for _n in ("mimose_set_params", "mimose_get_params", "mimose_get_grads", "mimose_get_master"):
    getattr(_lib, _n).argtypes = [_P, _P, C.c_int64]
_lib.mimose_collect.argtypes = [_P, C.POINTER(BatchS), C.POINTER(C.c_float)]
_lib.mimose_plan.argtypes = [_P, C.c_int64, C.POINTER(Plan)]
_lib.mimose_forward.argtypes = [_P, C.POINTER(BatchS), C.POINTER(Plan), C.POINTER(C.c_float)]
_lib.mimose_backward.argtypes = [_P]
_lib.mimose_step.argtypes = [_P, C.c_float, C.c_float, C.c_float, C.c_float, C.c_float]
_lib.mimose_get_stats.argtypes = [_P, C.POINTER(Stats)]
_lib.mimose_phase.argtypes = [_P, C.POINTER(C.c_int32)]
_lib.mimose_get_sample.argtypes = [_P, C.c_int32, C.POINTER(SampleS)]
_lib.mimose_dry_run.argtypes = [_P, C.c_int32, C.c_int32, C.c_uint64, C.POINTER(C.c_int64)]
_lib.mimose_dry_collect.argtypes = [_P, C.c_int32, C.c_int32, C.POINTER(SampleS)]
_lib.mimose_dry_run2.argtypes = [_P, C.c_int32, C.c_int32, C.c_int32, C.c_uint64, C.POINTER(C.c_int64)]
_lib.mimose_dry_collect2.argtypes = [_P, C.c_int32, C.c_int32, C.c_int32, C.POINTER(SampleS)]
_lib.mimose_plan2.argtypes = [_P, C.c_int64, C.c_int64, C.POINTER(Plan)]
_lib.mimose_predicted_peak.argtypes = [C.POINTER(Series), C.c_uint64]
_lib.mimose_predicted_peak.restype = C.c_int64
_lib.mimose_plan_series.argtypes = [C.POINTER(Series), C.c_int64, C.c_int64, C.c_int32, C.c_int32,
                                    C.POINTER(C.c_uint64), C.POINTER(C.c_int64)]
_lib.mimose_fit_predict.argtypes = [C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.c_int32, C.c_int32,
                                    C.POINTER(C.c_int64), C.c_int32, C.POINTER(C.c_int64)]

_lib.mimose_nccl_unique_id.argtypes = [_P]
_lib.mimose_set_optimizer.argtypes = [_P, C.c_float, C.c_float, C.c_float, C.c_float, C.c_float, C.c_int32]
_lib.mimose_probe.argtypes = [_P, C.c_int32]
_lib.mimose_probe_read.argtypes = [_P, C.POINTER(C.c_double), C.POINTER(C.c_double), C.POINTER(C.c_int64)]
_lib.mimose_set_planner.argtypes = [_P, C.c_int32]

EXPORTED = ["mimose_default_config", "mimose_init", "mimose_destroy", "mimose_last_error",
            "mimose_status_str", "mimose_num_params", "mimose_set_params", "mimose_get_params",
            "mimose_get_grads", "mimose_collect", "mimose_plan", "mimose_forward", "mimose_backward",
            "mimose_step", "mimose_get_stats", "mimose_phase", "mimose_get_sample", "mimose_dry_run",
            "mimose_dry_collect", "mimose_predicted_peak", "mimose_plan_series", "mimose_fit_predict",
            "mimose_nccl_unique_id", "mimose_probe", "mimose_probe_read", "mimose_set_optimizer",
            "mimose_set_planner", "mimose_get_master", "mimose_plan2", "mimose_dry_run2",
            "mimose_dry_collect2"]


_lib.mimose_tc_available.restype = C.c_int32
EXPORTED.append("mimose_tc_available")


_lib.mimose_debug_gemm.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.c_int32, _P, C.c_int64, C.c_int64,
                                   _P, C.c_int64, C.c_int64, _P, C.c_int64, _P, C.c_int32, C.c_int32, _P]
EXPORTED.append("mimose_debug_gemm")


def debug_gemm(epi, M, N, K, A, a_sm, a_sk, B, b_sn, b_sk, Cm, ldc, bias=None, split=1, use_tc=True, stream=0):
    """Test hook over one library GEMM (torch tensors in, device pointers out)."""
    st = _lib.mimose_debug_gemm(epi, M, N, K, A.data_ptr(), a_sm, a_sk, B.data_ptr(), b_sn, b_sk, Cm.data_ptr(),
                                ldc, bias.data_ptr() if bias is not None else None, split, 1 if use_tc else 0,
                                stream)
    if st != OK:
        raise MimoseError(st, "debug_gemm")


_lib.mimose_debug_gemm_grouped.argtypes = ([C.c_int32, C.c_int32, C.c_int32, _P, C.c_int64, C.c_int64, _P,
                                             C.c_int64, C.c_int64, _P] * 2 + [_P])
EXPORTED.append("mimose_debug_gemm_grouped")


def debug_gemm_grouped(op1, C1, op2, C2, stream=0):
    """Test hook: two fp32 GEMMs (M, N, K, A, a_sm, a_sk, B, b_sn, b_sk) in one grouped launch."""
    args = []
    for (M, N, K, A, a_sm, a_sk, B, b_sn, b_sk), Cm in ((op1, C1), (op2, C2)):
        args += [M, N, K, A.data_ptr(), a_sm, a_sk, B.data_ptr(), b_sn, b_sk, Cm.data_ptr()]
    st = _lib.mimose_debug_gemm_grouped(*args, stream)
    if st != OK:
        raise MimoseError(st, "debug_gemm_grouped")


_lib.mimose_debug_gemm_ex.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.c_int32, _P, C.c_int64, C.c_int64,
                                      _P, C.c_int64, C.c_int64, _P, C.c_int64, _P, _P, _P, C.c_int64, _P, C.c_int64,
                                      C.c_int32, C.c_int32, _P]
EXPORTED.append("mimose_debug_gemm_ex")


def debug_gemm_ex(epi, M, N, K, A, a_sm, a_sk, B, b_sn, b_sk, Cm, ldc, C2=None, bias=None, res=None, ldr=0,
                  aux=None, ldx=0, split=1, use_tc=True, stream=0):
    """Test hook over one library GEMM with any epilogue (torch tensors in)."""
    ptr = lambda t: t.data_ptr() if t is not None else None
    st = _lib.mimose_debug_gemm_ex(epi, M, N, K, ptr(A), a_sm, a_sk, ptr(B), b_sn, b_sk, ptr(Cm), ldc, ptr(C2),
                                   ptr(bias), ptr(res), ldr, ptr(aux), ldx, split, 1 if use_tc else 0, stream)
    if st != OK:
        raise MimoseError(st, "debug_gemm_ex")


_lib.mimose_debug_options.argtypes = [C.c_int32, C.c_int32]
_lib.mimose_debug_options.restype = None
EXPORTED.append("mimose_debug_options")


def debug_options(gemm_mode: int = -1, attn_tc: int = -1):
    _lib.mimose_debug_options(gemm_mode, attn_tc)


def tc_gemm_available() -> bool:
    return bool(_lib.mimose_tc_available())


def nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    st = _lib.mimose_nccl_unique_id(buf)
    if st != OK:
        raise MimoseError(st, "ncclGetUniqueId failed")
    return buf.raw


def make_config(cfg: wl.ModelConfig, **kw) -> Config:
    c = Config()
    _lib.mimose_default_config(C.byref(c))
    c.arch = cfg.arch
    c.head = cfg.head
    c.dtype = 0 if cfg.dtype == "fp32" else 1
    c.n_layers, c.hidden, c.heads, c.ffn = cfg.n_layers, cfg.hidden, cfg.heads, cfg.ffn
    c.vocab, c.max_pos, c.type_vocab, c.pos_offset = cfg.vocab, cfg.max_pos, cfg.type_vocab, cfg.pos_offset
    c.n_choices, c.n_labels = cfg.n_choices, cfg.n_labels
    c.p_drop, c.ln_eps = cfg.p_drop, cfg.ln_eps
    c.seed = wl.dropout_seed(cfg)
    c.max_seqs, c.max_seq_len = cfg.n_seqs, cfg.max_seq
    c.pad_id = cfg.pad_id
    c.n_dec_layers = cfg.n_dec_layers
    if cfg.ffn_layers:                       # heterogeneous stages: per-layer FFN widths
        arr = (C.c_int32 * cfg.n_layers)(*cfg.ffn_layers)
        c._ffn_keep = arr                    # alive until mimose_init has copied it
        c.ffn_layers = C.cast(arr, C.c_void_p)
    for k, v in kw.items():
        setattr(c, k, v)
    return c


class Mimose:
    """One library context.  ``slab`` = a CUDA uint8 torch tensor (the arena) or
    None for a host-only context (collector / estimator / planner accounting)."""

    def __init__(self, cfg: wl.ModelConfig, budget: int = 0, slab=None, stream=None,
                 rank: int = 0, world: int = 1, nccl_id: Optional[bytes] = None, **kw):
        self.cfg = cfg
        c = make_config(cfg, **kw)
        c.budget_bytes = int(budget)
        c.rank, c.world = rank, world
        self._nccl = None
        if nccl_id is not None:
            self._nccl = C.create_string_buffer(bytes(nccl_id), 128)
            c.nccl_id = C.cast(self._nccl, C.c_void_p)
        if slab is not None:
            c.arena_base = slab.data_ptr()
            c.arena_bytes = slab.numel()
            c.stream = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream or 0)
        self._slab = slab
        self._cfg = c
        h = _P()
        st = _lib.mimose_init(C.byref(c), C.byref(h))
        self.h = h
        if st != OK:
            msg = _lib.mimose_last_error(h).decode() if h.value else "init failed"
            if h.value:
                _lib.mimose_destroy(h)
            self.h = _P()
            raise MimoseError(st, msg)
        n = C.c_int64()
        _lib.mimose_num_params(self.h, C.byref(n))
        self.n_params = n.value
        # checkpoint units: layers, or 2L attention / FFN blocks (granularity=1);
        # encoder-decoder: encoder then decoder layers
        self.n_units = cfg.n_layers * (2 if c.granularity == 1 else 1) + cfg.n_dec_layers

    # -- lifecycle --
    def close(self):
        if self.h and self.h.value:
            _lib.mimose_destroy(self.h)
            self.h = _P()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _chk(self, st: int, allow=()):
        if st != OK and st not in allow:
            raise MimoseError(st, _lib.mimose_last_error(self.h).decode())
        return st

    # -- parameters --
    def set_params(self, blob: np.ndarray):
        b = np.ascontiguousarray(blob, np.float32)
        self._chk(_lib.mimose_set_params(self.h, b.ctypes.data, b.size))

    def get_params(self) -> np.ndarray:
        b = np.empty(self.n_params, np.float32)
        self._chk(_lib.mimose_get_params(self.h, b.ctypes.data, b.size))
        return b

    def get_master(self) -> np.ndarray:
        b = np.empty(self.n_params, np.float32)
        self._chk(_lib.mimose_get_master(self.h, b.ctypes.data, b.size))
        return b

    def get_grads(self) -> np.ndarray:
        b = np.empty(self.n_params, np.float32)
        self._chk(_lib.mimose_get_grads(self.h, b.ctypes.data, b.size))
        return b

    # -- batches --
    @staticmethod
    def batch_struct(ids, tt, lens, labels, n_seqs, seq_len, on_host, dec_ids=None, dec_lens=None,
                     dec_len=0) -> BatchS:
        def ptr(a):
            if a is None:
                return None
            return a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data
        return BatchS(ptr(ids), ptr(tt), ptr(lens), ptr(labels), n_seqs, seq_len, 1 if on_host else 0,
                      ptr(dec_ids), ptr(dec_lens), dec_len, 0)

    def host_batch(self, b: wl.Batch) -> BatchS:
        self._keep = [np.ascontiguousarray(x, np.int32) for x in (b.input_ids, b.token_type, b.lengths, b.labels)]
        if b.dec_ids is not None:
            self._keep += [np.ascontiguousarray(b.dec_ids, np.int32), np.ascontiguousarray(b.dec_lengths, np.int32)]
            return self.batch_struct(*self._keep[:4], b.n_seqs, b.seq_len, True, self._keep[4], self._keep[5],
                                     b.dec_len)
        return self.batch_struct(*self._keep, b.n_seqs, b.seq_len, True)

    # -- the method --
    def collect(self, batch: BatchS, want_loss: bool = True) -> Optional[float]:
        loss = C.c_float()
        self._chk(_lib.mimose_collect(self.h, C.byref(batch), C.byref(loss) if want_loss else None))
        return loss.value if want_loss else None

    def plan(self, x: int, xt: Optional[int] = None) -> Plan:
        """The plan for input size x (or the 2-D key (x, xt) of an encoder-decoder)."""
        p = Plan()
        if xt is None:
            self._chk(_lib.mimose_plan(self.h, int(x), C.byref(p)), allow=(E_INFEASIBLE,))
        else:
            self._chk(_lib.mimose_plan2(self.h, int(x), int(xt), C.byref(p)), allow=(E_INFEASIBLE,))
        return p

    def set_planner(self, kind: int):
        """0 = Algorithm 1 greedy (default), 1 = exact fewest-recompute planner."""
        self._chk(_lib.mimose_set_planner(self.h, int(kind)))

    def forward(self, batch: BatchS, plan: Optional[Plan] = None, want_loss: bool = True) -> Optional[float]:
        loss = C.c_float()
        self._chk(_lib.mimose_forward(self.h, C.byref(batch), C.byref(plan) if plan is not None else None,
                                      C.byref(loss) if want_loss else None))
        return loss.value if want_loss else None

    def backward(self):
        self._chk(_lib.mimose_backward(self.h))

    def set_optimizer(self, lr=1e-4, beta1=0.9, beta2=0.999, eps=1e-8, wd=0.0, fused=True):
        self._chk(_lib.mimose_set_optimizer(self.h, lr, beta1, beta2, eps, wd, 1 if fused else 0))

    def step(self, lr=1e-4, beta1=0.9, beta2=0.999, eps=1e-8, wd=0.0):
        self._chk(_lib.mimose_step(self.h, lr, beta1, beta2, eps, wd))

    # -- introspection --
    def stats(self) -> Dict:
        s = Stats()
        self._chk(_lib.mimose_get_stats(self.h, C.byref(s)))
        return s.asdict()

    @property
    def phase(self) -> int:
        p = C.c_int32()
        self._chk(_lib.mimose_phase(self.h, C.byref(p)))
        return p.value

    def sample(self, i: int) -> Dict:
        s = SampleS()
        self._chk(_lib.mimose_get_sample(self.h, i, C.byref(s)))
        return _sample_dict(s, self.n_units)

    def dry_run(self, n_seqs: int, seq_len: int, dropped=(), dec_len: Optional[int] = None) -> int:
        mask = 0
        for l in dropped:
            mask |= 1 << int(l)
        pk = C.c_int64()
        if dec_len is None:
            self._chk(_lib.mimose_dry_run(self.h, n_seqs, seq_len, C.c_uint64(mask), C.byref(pk)))
        else:
            self._chk(_lib.mimose_dry_run2(self.h, n_seqs, seq_len, dec_len, C.c_uint64(mask), C.byref(pk)))
        return pk.value

    def probe(self, kind: int = 1):
        self._chk(_lib.mimose_probe(self.h, kind))

    def probe_read(self):
        ms, fl, n = C.c_double(), C.c_double(), C.c_int64()
        self._chk(_lib.mimose_probe_read(self.h, C.byref(ms), C.byref(fl), C.byref(n)))
        return ms.value, fl.value, n.value

    def dry_collect(self, n_seqs: int, seq_len: int, dec_len: Optional[int] = None) -> Dict:
        s = SampleS()
        if dec_len is None:
            self._chk(_lib.mimose_dry_collect(self.h, n_seqs, seq_len, C.byref(s)))
        else:
            self._chk(_lib.mimose_dry_collect2(self.h, n_seqs, seq_len, dec_len, C.byref(s)))
        return _sample_dict(s, self.n_units)


def _sample_dict(s: SampleS, L: int) -> Dict:
    return dict(x=s.x, xt=s.xt, C=s.C, E=s.E, Hd=s.Hd, Th=s.Th, Tb=s.Tb, Te=s.Te,
                a=list(s.a[:L]), y=list(s.y[:L]), t_ms=list(s.t_ms[:L]))


def _series(p: Dict):
    L = len(p["a"])
    a = (C.c_int64 * L)(*p["a"])
    y = (C.c_int64 * L)(*p["y"])
    return Series(p["C"], p["E"], p["Hd"], p["Th"], p["Tb"], p["Te"], a, y, L), (a, y)


def predicted_peak(p: Dict, dropped=()) -> int:
    s, keep = _series(p)
    mask = sum(1 << int(l) for l in dropped)
    return _lib.mimose_predicted_peak(C.byref(s), C.c_uint64(mask))


PLANNER_GREEDY, PLANNER_EXACT, PLANNER_EXACT_TIME = 0, 1, 2


def plan_series(p: Dict, budget: int, reserve: int = 0, num: int = 9, den: int = 10, planner: int = PLANNER_GREEDY):
    """The library's planner on explicit per-series sizes (test hook)."""
    if planner == PLANNER_EXACT:
        num = 0
    s, keep = _series(p)
    mask = C.c_uint64()
    pk = C.c_int64()
    st = _lib.mimose_plan_series(C.byref(s), budget, reserve, num, den, C.byref(mask), C.byref(pk))
    return st, [l for l in range(64) if (mask.value >> l) & 1], pk.value


_lib.mimose_plan_series_cost.argtypes = [C.POINTER(Series), C.POINTER(C.c_int64), C.c_int64, C.c_int64,
                                         C.POINTER(C.c_uint64), C.POINTER(C.c_int64)]
EXPORTED.append("mimose_plan_series_cost")


def plan_series_cost(p: Dict, cost, budget: int, reserve: int = 0):
    """The library's time-weighted exact planner on explicit series and costs (test hook)."""
    s, keep = _series(p)
    L = len(p["a"])
    cst = (C.c_int64 * L)(*[int(v) for v in cost])
    mask = C.c_uint64()
    pk = C.c_int64()
    st = _lib.mimose_plan_series_cost(C.byref(s), cst, budget, reserve, C.byref(mask), C.byref(pk))
    return st, [l for l in range(64) if (mask.value >> l) & 1], pk.value


def fit_predict(xs, ys, x_eval, degree: int = 2) -> List[int]:
    n = len(xs)
    X = (C.c_int64 * n)(*[int(v) for v in xs])
    Y = (C.c_int64 * n)(*[int(v) for v in ys])
    m = len(x_eval)
    XE = (C.c_int64 * m)(*[int(v) for v in x_eval])
    out = (C.c_int64 * m)()
    st = _lib.mimose_fit_predict(X, Y, n, degree, XE, m, out)
    if st != OK:
        raise MimoseError(st, "fit_predict")
    return list(out)
