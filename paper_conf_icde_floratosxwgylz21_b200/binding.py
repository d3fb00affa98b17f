"""Thin ctypes binding of include/nestgpu.h (argument marshalling only).

Every step of the hot path runs in libnestgpu.so's CUDA kernels; this module
only converts Python objects to the C structs and back.  There is no CPU
fallback: if the shared library is missing or no CUDA device is present the
calls raise.

PyTorch is used for plumbing only: the device arena is a torch uint8 tensor
and the stream is torch's current stream (so NCCL collectives issued through
torch.distributed order correctly with the engine's kernels).
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("NESTGPU_LIB") or os.path.join(_HERE, "libnestgpu.so")

OK, ERR_INVALID, ERR_OOM, ERR_TYPE, ERR_UNSUPPORTED, ERR_OVERFLOW, ERR_CUDA, ERR_BUFFER = 0, -1, -2, -3, -4, -5, -6, -7
DT = {"int32": 0, "int64": 1, "decimal": 2, "date": 3, "decimal32": 4}
CMP = {"=": 0, "!=": 1, "<": 2, "<=": 3, ">": 4, ">=": 5}
AGG = {"min": 0, "max": 1, "sum": 2, "count": 3, "avg": 4, "exists": 5, "not_exists": 6}
N_STAGES = 6
STAGES = ("outer_filter", "inner_filter", "sort", "subquery", "finalize", "total")

# The exported C symbols (tests check that the library exports all of them).
SYMBOLS = ("nestgpu_create", "nestgpu_destroy", "nestgpu_last_error", "nestgpu_launch_count",
           "nestgpu_set_stream", "nestgpu_mark", "nestgpu_release", "nestgpu_arena_usage",
           "nestgpu_load_column", "nestgpu_alloc_column", "nestgpu_column_info", "nestgpu_gather_column",
           "nestgpu_build_index", "nestgpu_drop_index", "nestgpu_index_info",
           "nestgpu_index_create_empty", "nestgpu_exec_correlated", "nestgpu_result_to_host",
           "nestgpu_exec_collect", "nestgpu_collection_in", "nestgpu_column_from_device",
           "nestgpu_set_option", "nestgpu_set_profiling", "nestgpu_last_profile",
           "nestgpu_cost_calibrate", "nestgpu_cost_estimate_plan",
           "nestgpu_window_create", "nestgpu_window_open", "nestgpu_window_close", "nestgpu_window_free",
           "nestgpu_result_put")
STRATEGIES = ("nested_loop", "index", "nested_loop_cached", "index_cached")
OPT_MALLOC_SCRATCH = 1
OPT_BNL_SHAPE = 2
OPT_GRAPHS = 3
OPT_SORT = 4   # 0 / 1 LSD onesweep (default), 2 MSD bucket sort experiment
OPT_TINY = 5   # 1 (default): one-launch path for tiny nested-loop queries; 0: the regular sequence


class NestGPUError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("nestgpu error %d: %s" % (code, msg))
        self.code = code


class Pred(ctypes.Structure):
    _fields_ = [("col", ctypes.c_int32), ("op", ctypes.c_int32), ("literal", ctypes.c_int64),
                ("rhs_col", ctypes.c_int32)]


class ColumnDesc(ctypes.Structure):
    _fields_ = [("dtype", ctypes.c_int32), ("scale", ctypes.c_int32), ("n", ctypes.c_int64),
                ("d_values", ctypes.c_void_p), ("d_valid", ctypes.c_void_p)]


class IndexDesc(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("key_bytes", ctypes.c_int32), ("payload_bytes", ctypes.c_int32),
                ("d_keys", ctypes.c_void_p), ("d_payload", ctypes.c_void_p)]


class Plan(ctypes.Structure):
    _fields_ = [("outer_preds", ctypes.c_void_p), ("n_outer_preds", ctypes.c_int32),
                ("outer_key_cols", ctypes.c_int32 * 2), ("inner_key_cols", ctypes.c_int32 * 2),
                ("n_key_cols", ctypes.c_int32), ("corr_op", ctypes.c_int32),
                ("inner_preds", ctypes.c_void_p), ("n_inner_preds", ctypes.c_int32),
                ("agg", ctypes.c_int32), ("agg_col", ctypes.c_int32),
                ("outer_cmp_col", ctypes.c_int32), ("outer_op", ctypes.c_int32),
                ("lhs_mult", ctypes.c_int64), ("rhs_mult", ctypes.c_int64),
                ("index", ctypes.c_int32), ("row_id_base", ctypes.c_int64),
                ("emit_all", ctypes.c_int32), ("dedup", ctypes.c_int32)]


class Result(ctypes.Structure):
    _fields_ = [("n_rows", ctypes.c_int64), ("n_evaluated", ctypes.c_int64),
                ("d_row_ids", ctypes.c_void_p), ("d_values", ctypes.c_void_p),
                ("d_valid", ctypes.c_void_p), ("d_passed", ctypes.c_void_p),
                ("d_avg_sum", ctypes.c_void_p), ("d_avg_cnt", ctypes.c_void_p)]


class Collection(ctypes.Structure):
    _fields_ = [("n_outer", ctypes.c_int64), ("n_values", ctypes.c_int64),
                ("d_row_ids", ctypes.c_void_p), ("d_offsets", ctypes.c_void_p),
                ("d_values", ctypes.c_void_p), ("d_owner", ctypes.c_void_p)]


class IpcHandle(ctypes.Structure):
    _fields_ = [("bytes", ctypes.c_ubyte * 64)]


class CostParams(ctypes.Structure):
    _fields_ = [("launch_ms", ctypes.c_double), ("filter_ms_per_row", ctypes.c_double),
                ("hist_ms_per_key_digit", ctypes.c_double), ("sort_ms_per_key", ctypes.c_double),
                ("sort_ms_per_byte", ctypes.c_double),
                ("probe_ms_per_step", ctypes.c_double), ("range_ms_per_elem", ctypes.c_double),
                ("aux_ms_per_elem", ctypes.c_double), ("bnl_ms_per_pair", (ctypes.c_double * 4) * 2),
                ("final_ms_per_row", ctypes.c_double), ("materialize_ms_per_byte", ctypes.c_double),
                ("group_ms_per_key", ctypes.c_double), ("sync_ms", ctypes.c_double),
                ("exec_overhead_ms", ctypes.c_double), ("build_overhead_ms", ctypes.c_double),
                ("dedup_overhead_ms", ctypes.c_double)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_ if k != "bnl_ms_per_pair"}
        d["bnl_ms_per_pair"] = [list(row) for row in self.bnl_ms_per_pair]
        return d


class CostInput(ctypes.Structure):
    _fields_ = [("n_r", ctypes.c_int64), ("n_s", ctypes.c_int64), ("n_rp", ctypes.c_int64),
                ("n_sp", ctypes.c_int64), ("n_distinct", ctypes.c_int64), ("sum_k", ctypes.c_int64),
                ("survivors", ctypes.c_int64), ("key_bytes", ctypes.c_int32), ("payload_bytes", ctypes.c_int32),
                ("sort_passes", ctypes.c_int32), ("dedup_passes", ctypes.c_int32),
                ("narrow_keys", ctypes.c_int32), ("corr_op", ctypes.c_int32), ("agg", ctypes.c_int32)]


class CostEstimate(ctypes.Structure):
    _fields_ = [("ms", ctypes.c_double * 4), ("index_build_ms", ctypes.c_double), ("outer_ms", ctypes.c_double),
                ("nested_ms", ctypes.c_double * 4), ("best", ctypes.c_int32)]


class Prepared:
    """A plan marshalled once (Engine.prepare): the C struct and the
    predicate arrays it points to, kept alive together."""

    def __init__(self, plan_struct, keep):
        self.plan = plan_struct
        self._keep = keep
        self.ref = ctypes.byref(plan_struct)


_lib = None


def cost_estimate(params, n_r, n_s, n_rp, n_sp, n_distinct, sum_k, survivors, key_bytes, payload_bytes,
                  sort_passes, dedup_passes, corr_op, agg, narrow_keys=0):
    """Eqs. (1)-(9) of the paper's cost model for one plan shape
    (nestgpu_cost_estimate_plan; host arithmetic, no device).  params: a
    CostParams (from Engine.cost_calibrate) or its as_dict().  Returns
    {strategy: predicted ms, "best": strategy, "index_build_ms", "outer_ms"}."""
    lib = load_library()
    if isinstance(params, dict):
        p = CostParams()
        for k, v in params.items():
            if k == "bnl_ms_per_pair":
                for w, row in enumerate(v):
                    for i, x in enumerate(row):
                        p.bnl_ms_per_pair[w][i] = x
            else:
                setattr(p, k, v)
        params = p
    ci = CostInput(int(n_r), int(n_s), int(n_rp), int(n_sp), int(n_distinct), int(sum_k), int(survivors),
                   int(key_bytes), int(payload_bytes), int(sort_passes), int(dedup_passes), int(narrow_keys),
                   CMP[corr_op], AGG[agg])
    e = CostEstimate()
    st = lib.nestgpu_cost_estimate_plan(ctypes.byref(params), ctypes.byref(ci), ctypes.byref(e))
    if st != OK:
        raise NestGPUError(st, "cost_estimate_plan rejected its input")
    out = {name: e.ms[i] for i, name in enumerate(STRATEGIES)}
    out["nested"] = {name: e.nested_ms[i] for i, name in enumerate(STRATEGIES)}
    out["best"] = STRATEGIES[e.best]
    out["index_build_ms"] = e.index_build_ms
    out["outer_ms"] = e.outer_ms
    return out


def load_library(path=LIB_PATH):
    """Load libnestgpu.so (raises if it was not built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError("libnestgpu.so not built (%s); run __graft_entry__.build() -- "
                          "there is no CPU fallback" % path)
    lib = ctypes.CDLL(path)
    vp, i32, i64, sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
    P = ctypes.POINTER
    sig = {
        "nestgpu_create": (i32, [ctypes.c_int, vp, sz, vp, P(vp)]),
        "nestgpu_destroy": (i32, [vp]),
        "nestgpu_last_error": (ctypes.c_char_p, [vp]),
        "nestgpu_launch_count": (i64, [vp]),
        "nestgpu_set_stream": (i32, [vp, vp]),
        "nestgpu_mark": (i32, [vp, P(ctypes.c_uint64)]),
        "nestgpu_release": (i32, [vp, ctypes.c_uint64]),
        "nestgpu_arena_usage": (i32, [vp, P(sz), P(sz)]),
        "nestgpu_load_column": (i32, [vp, i32, i32, vp, vp, i64, P(i32)]),
        "nestgpu_alloc_column": (i32, [vp, i32, i32, i64, i32, P(i32)]),
        "nestgpu_column_info": (i32, [vp, i32, P(ColumnDesc)]),
        "nestgpu_gather_column": (i32, [vp, i32, vp, i64, i64, P(i32)]),
        "nestgpu_build_index": (i32, [vp, P(i32), i32, i32, vp, i32, P(i32)]),
        "nestgpu_drop_index": (i32, [vp, i32]),
        "nestgpu_index_info": (i32, [vp, i32, P(IndexDesc)]),
        "nestgpu_index_create_empty": (i32, [vp, i64, i32, i32, P(i32), i32, i32, vp, i32, P(IndexDesc), P(i32)]),
        "nestgpu_exec_correlated": (i32, [vp, P(Plan), P(Result)]),
        "nestgpu_result_to_host": (i32, [vp, P(Result), vp, vp, vp, vp, vp, vp, i64]),
        "nestgpu_exec_collect": (i32, [vp, P(Plan), P(Collection)]),
        "nestgpu_collection_in": (i32, [vp, P(Collection), i32, i64, i32, P(Result)]),
        "nestgpu_column_from_device": (i32, [vp, i32, i32, vp, vp, i64, P(i32)]),
        "nestgpu_set_option": (i32, [vp, i32, i64]),
        "nestgpu_cost_calibrate": (i32, [vp, i64, P(CostParams)]),
        "nestgpu_cost_estimate_plan": (i32, [P(CostParams), P(CostInput), P(CostEstimate)]),
        "nestgpu_set_profiling": (i32, [vp, i32]),
        "nestgpu_window_create": (i32, [vp, i64, P(vp), P(IpcHandle)]),
        "nestgpu_window_open": (i32, [vp, P(IpcHandle), P(vp)]),
        "nestgpu_window_close": (i32, [vp, vp]),
        "nestgpu_window_free": (i32, [vp, vp]),
        "nestgpu_result_put": (i32, [vp, P(Result), vp, i64, i64]),
        "nestgpu_last_profile": (i32, [vp, P(ctypes.c_float), i32]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def _device_view(ptr, n, device):
    """int64 torch tensor aliasing n values of device memory at ptr (memory
    the library owns, e.g. a window; no copy).  Built on a __cuda_array_interface__
    shim, so torch keeps no ownership."""
    import torch

    class _Shim:
        __cuda_array_interface__ = {"shape": (int(n),), "typestr": "<i8", "data": (int(ptr), False), "version": 2,
                                    "strides": None}

    return torch.as_tensor(_Shim(), device=device)


def _np_ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def _host_array(values):
    """numpy view of host data (numpy array or CPU torch tensor, pinned or not)."""
    if isinstance(values, np.ndarray):
        return np.ascontiguousarray(values)
    try:
        import torch
        if isinstance(values, torch.Tensor):
            if values.is_cuda:
                raise TypeError("load_column takes host data; device data goes through alloc_column")
            return values.contiguous().numpy()
    except ImportError:
        pass
    return np.ascontiguousarray(values)


class Engine:
    """One nestgpu context on one GPU.

    arena_bytes: size of the device memory pool (a torch uint8 tensor owned by
    this object); stream: a torch.cuda.Stream (default: current stream).
    """

    def __init__(self, device=0, arena_bytes=1 << 30, stream=None):
        import torch
        self._torch = torch
        self.lib = load_library()
        if not torch.cuda.is_available():
            raise RuntimeError("nestgpu needs a CUDA device (no CPU fallback)")
        self.device = torch.device("cuda", device)
        self.arena = torch.empty(int(arena_bytes), dtype=torch.uint8, device=self.device)
        self.stream = stream or torch.cuda.current_stream(self.device)
        h = ctypes.c_void_p()
        self._check(self.lib.nestgpu_create(device, ctypes.c_void_p(self.arena.data_ptr()), int(arena_bytes),
                                            ctypes.c_void_p(self.stream.cuda_stream), ctypes.byref(h)), ctx=None)
        self.ctx = h

    # ------------------------------------------------------------ basics
    def _check(self, st, ctx="self"):
        if st != OK:
            msg = b""
            c = self.ctx if ctx == "self" else None
            if c is not None:
                msg = self.lib.nestgpu_last_error(c) or b""
            raise NestGPUError(st, msg.decode(errors="replace"))

    def close(self):
        if getattr(self, "ctx", None):
            self.lib.nestgpu_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def launch_count(self):
        return int(self.lib.nestgpu_launch_count(self.ctx))

    def mark(self):
        m = ctypes.c_uint64()
        self._check(self.lib.nestgpu_mark(self.ctx, ctypes.byref(m)))
        return m.value

    def release(self, mark):
        self._check(self.lib.nestgpu_release(self.ctx, int(mark)))

    def arena_usage(self):
        a, b = ctypes.c_size_t(), ctypes.c_size_t()
        self._check(self.lib.nestgpu_arena_usage(self.ctx, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def cost_calibrate(self, n_rows=0):
        """Measure the cost model's K_i on this GPU (nestgpu_cost_calibrate)."""
        p = CostParams()
        self._check(self.lib.nestgpu_cost_calibrate(self.ctx, int(n_rows), ctypes.byref(p)))
        return p

    def set_option(self, option, value):
        """Ablation knobs (nestgpu_set_option), e.g. OPT_MALLOC_SCRATCH."""
        self._check(self.lib.nestgpu_set_option(self.ctx, int(option), int(value)))

    def set_profiling(self, on=True):
        self._check(self.lib.nestgpu_set_profiling(self.ctx, 1 if on else 0))

    def last_profile(self):
        arr = (ctypes.c_float * N_STAGES)()
        self._check(self.lib.nestgpu_last_profile(self.ctx, arr, N_STAGES))
        return dict(zip(STAGES, list(arr)))

    # ------------------------------------------------------------ columns
    def load_column(self, values, valid=None, dtype=None, scale=0):
        v = _host_array(values)
        if dtype is None:
            dtype = "int32" if v.dtype.itemsize == 4 else "int64"
        want = np.int32 if DT[dtype] in (0, 3, 4) else np.int64
        if v.dtype != want:
            v = v.astype(want)
        m = None
        if valid is not None:
            m = _host_array(valid).astype(np.uint8, copy=False)
            if len(m) != len(v):
                raise ValueError("validity length")
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_load_column(self.ctx, DT[dtype], int(scale), _np_ptr(v), _np_ptr(m),
                                                 len(v), ctypes.byref(out)))
        return out.value

    def load_table(self, cols, valid=None, dtypes=None):
        valid = valid or {}
        dtypes = dtypes or {}
        return {name: self.load_column(arr, valid.get(name), dtypes.get(name)) for name, arr in cols.items()}

    def alloc_column(self, n, dtype="int32", with_valid=False, scale=0):
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_alloc_column(self.ctx, DT[dtype], int(scale), int(n), int(bool(with_valid)),
                                                  ctypes.byref(out)))
        return out.value

    def column_info(self, col):
        d = ColumnDesc()
        self._check(self.lib.nestgpu_column_info(self.ctx, int(col), ctypes.byref(d)))
        return {"dtype": d.dtype, "scale": d.scale, "n": d.n, "d_values": d.d_values, "d_valid": d.d_valid}

    def gather_column(self, src_col, res, row_id_base=0):
        """New column = src_col at a result's row ids (multi-level nesting,
        P:229: one level's survivors feed the block above).  `res` is a Result
        or a (device int64 pointer, n) pair, e.g. a collection's d_owner."""
        ptr, n = (res.d_row_ids, res.n_rows) if isinstance(res, Result) else res
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_gather_column(self.ctx, int(src_col), ctypes.c_void_p(ptr), int(n),
                                                   int(row_id_base), ctypes.byref(out)))
        return out.value

    def arena_view(self, ptr, nbytes):
        """torch uint8 view of arena bytes [ptr, ptr+nbytes) (for NCCL)."""
        off = int(ptr) - self.arena.data_ptr()
        if off < 0 or off + nbytes > self.arena.numel():
            raise ValueError("pointer outside the arena")
        return self.arena[off:off + int(nbytes)]

    # ------------------------------------------------------------ plans
    @staticmethod
    def _preds(preds, names):
        arr = (Pred * max(1, len(preds)))()
        for i, p in enumerate(preds):
            arr[i].col = names[p["col"]]
            arr[i].op = CMP[p["op"]]
            if p.get("rhs") is not None:
                arr[i].rhs_col = names[p["rhs"]]
                arr[i].literal = 0
            else:
                arr[i].rhs_col = -1
                arr[i].literal = int(p["lit"])
        return arr, len(preds)

    def build_index(self, S, key, payload=None, inner_preds=()):
        """S: {name: col id}; key: list of 1-2 names; payload: name or None."""
        keys = (ctypes.c_int32 * 2)(*[S[k] for k in key] + [0] * (2 - len(key)))
        parr, np_ = self._preds(list(inner_preds), S)
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_build_index(self.ctx, keys, len(key), S[payload] if payload else -1,
                                                 ctypes.cast(parr, ctypes.c_void_p), np_, ctypes.byref(out)))
        return out.value

    def index_for_plan(self, plan, S):
        return self.build_index(S, plan["inner_key"],
                                plan["agg_col"] if plan["agg"] in ("min", "max", "sum", "avg") else None,
                                plan["inner_preds"])

    def drop_index(self, idx):
        self._check(self.lib.nestgpu_drop_index(self.ctx, int(idx)))

    def index_info(self, idx):
        d = IndexDesc()
        self._check(self.lib.nestgpu_index_info(self.ctx, int(idx), ctypes.byref(d)))
        return {"n": d.n, "key_bytes": d.key_bytes, "payload_bytes": d.payload_bytes,
                "d_keys": d.d_keys, "d_payload": d.d_payload}

    def index_create_empty(self, S, key, payload, inner_preds, n, key_bytes, payload_bytes):
        keys = (ctypes.c_int32 * 2)(*[S[k] for k in key] + [0] * (2 - len(key)))
        parr, np_ = self._preds(list(inner_preds), S)
        d = IndexDesc()
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_index_create_empty(
            self.ctx, int(n), int(key_bytes), int(payload_bytes), keys, len(key), S[payload] if payload else -1,
            ctypes.cast(parr, ctypes.c_void_p), np_, ctypes.byref(d), ctypes.byref(out)))
        return out.value, {"n": d.n, "key_bytes": d.key_bytes, "payload_bytes": d.payload_bytes,
                           "d_keys": d.d_keys, "d_payload": d.d_payload}

    def _plan(self, plan, R, S, index, emit_all, row_id_base, dedup):
        p = Plan()
        opa, p.n_outer_preds = self._preds(plan["outer_preds"], R)
        ipa, p.n_inner_preds = self._preds(plan["inner_preds"], S)
        p.outer_preds = ctypes.cast(opa, ctypes.c_void_p)
        p.inner_preds = ctypes.cast(ipa, ctypes.c_void_p)
        nk = len(plan["outer_key"])
        p.n_key_cols = nk
        for i in range(nk):
            p.outer_key_cols[i] = R[plan["outer_key"][i]]
            p.inner_key_cols[i] = S[plan["inner_key"][i]]
        p.corr_op = CMP[plan["corr_op"]]
        p.agg = AGG[plan["agg"]]
        p.agg_col = S[plan["agg_col"]] if plan.get("agg_col") else -1
        p.outer_cmp_col = R[plan["outer_cmp_col"]] if plan.get("outer_cmp_col") else -1
        p.outer_op = CMP[plan["outer_op"]]
        p.lhs_mult = int(plan["lhs_mult"])
        p.rhs_mult = int(plan["rhs_mult"])
        p.index = int(index)
        p.row_id_base = int(row_id_base)
        p.emit_all = 1 if emit_all else 0
        p.dedup = 1 if dedup else 0
        self._keep = (opa, ipa)
        return p

    def prepare(self, plan, R, S, index=-1, emit_all=False, row_id_base=0, dedup=False):
        """Marshal a plan into its C struct once (Prepared); exec(prepared)
        then skips the per-call Python marshalling -- the repeated-query
        path of small, latency-bound queries."""
        p = self._plan(plan, R, S, index, emit_all, row_id_base, dedup)
        return Prepared(p, self._keep)

    def exec(self, plan, R=None, S=None, index=-1, emit_all=False, row_id_base=0, dedup=False):
        """Run one plan (datagen.plans dict, or a Prepared from prepare()).
        R / S map column names to ids.  dedup: evaluate each distinct
        correlated value once (P:331 caching)."""
        if isinstance(plan, Prepared):
            res = Result()
            self._check(self.lib.nestgpu_exec_correlated(self.ctx, plan.ref, ctypes.byref(res)))
            return res
        p = self._plan(plan, R, S, index, emit_all, row_id_base, dedup)
        res = Result()
        self._check(self.lib.nestgpu_exec_correlated(self.ctx, ctypes.byref(p), ctypes.byref(res)))
        return res

    # ------------------------------------------------------------ type-J
    def exec_collect(self, plan, R, S, index, row_id_base=0):
        """Type-J subquery results as two-level arrays (nestgpu_collection);
        plan["agg_col"] is the selected column, `index` must carry it."""
        p = self._plan(plan, R, S, index, False, row_id_base, False)
        coll = Collection()
        self._check(self.lib.nestgpu_exec_collect(self.ctx, ctypes.byref(p), ctypes.byref(coll)))
        return coll

    def collection_to_numpy(self, coll):
        torch = self._torch
        n, m = coll.n_outer, coll.n_values

        def dev(ptr, k):
            if k == 0 or not ptr:
                return np.zeros(0, np.int64)
            return self.arena_view(ptr, k * 8).view(torch.int64).cpu().numpy()

        return {"row": dev(coll.d_row_ids, n), "offsets": dev(coll.d_offsets, n + 1) if n else np.zeros(1, np.int64),
                "values": dev(coll.d_values, m), "owner": dev(coll.d_owner, m)}

    def collection_in(self, coll, x_col, row_id_base=0, emit_all=False):
        """R.x IN (type-J list) for every level-1 entry (nestgpu_collection_in)."""
        res = Result()
        self._check(self.lib.nestgpu_collection_in(self.ctx, ctypes.byref(coll), int(x_col), int(row_id_base),
                                                   1 if emit_all else 0, ctypes.byref(res)))
        return res

    def column_from_device(self, d_src, n, dtype="int64", d_valid=None, scale=0):
        """Materialise a column from device int64 values (a result's / a
        collection's arrays): Res[i] = Materialize(...) of Fig. 4."""
        out = ctypes.c_int32()
        self._check(self.lib.nestgpu_column_from_device(self.ctx, DT[dtype], int(scale), ctypes.c_void_p(d_src),
                                                        ctypes.c_void_p(d_valid) if d_valid else None, int(n),
                                                        ctypes.byref(out)))
        return out.value

    def result_to_numpy(self, res, avg=None, out=None):
        """Copy a result to host arrays.  out: optional dict of preallocated
        host arrays ("row", "value" int64; "valid", "passed" uint8; "sum",
        "cnt" int64 for AVG) with room for the rows -- e.g. views of pinned
        memory reused across calls, so the copy runs at full PCIe speed;
        the returned arrays are then views of them."""
        n = res.n_rows
        if out is None:
            out = {"row": np.empty(n, np.int64), "value": np.empty(n, np.int64),
                   "valid": np.empty(n, np.uint8), "passed": np.empty(n, np.uint8)}
            if res.d_avg_sum:
                out["sum"] = np.empty(n, np.int64)
                out["cnt"] = np.empty(n, np.int64)
        else:
            keys = ("row", "value", "valid", "passed") + (("sum", "cnt") if res.d_avg_sum else ())
            if min(len(out[k]) for k in keys) < n:
                raise ValueError("result_to_numpy: %d rows do not fit the given buffers" % n)
            out = {k: out[k][:n] for k in keys}
        s, c = (out["sum"], out["cnt"]) if res.d_avg_sum else (None, None)
        self._check(self.lib.nestgpu_result_to_host(self.ctx, ctypes.byref(res), _np_ptr(out["row"]),
                                                    _np_ptr(out["value"]), _np_ptr(out["valid"]),
                                                    _np_ptr(out["passed"]), _np_ptr(s), _np_ptr(c), n))
        return out

    # ------------------------------------------------------------ peer windows (multi-GPU gather)
    def window_create(self, cap):
        """A device window of cap (row id, value) rows other processes can map;
        returns (device pointer, 64 IPC handle bytes)."""
        p, h = ctypes.c_void_p(), IpcHandle()
        self._check(self.lib.nestgpu_window_create(self.ctx, int(cap), ctypes.byref(p), ctypes.byref(h)))
        return p.value, bytes(h.bytes)

    def window_open(self, handle_bytes):
        h = IpcHandle()
        ctypes.memmove(h.bytes, bytes(handle_bytes), 64)
        p = ctypes.c_void_p()
        self._check(self.lib.nestgpu_window_open(self.ctx, ctypes.byref(h), ctypes.byref(p)))
        return p.value

    def window_close(self, ptr):
        self._check(self.lib.nestgpu_window_close(self.ctx, ctypes.c_void_p(ptr)))

    def window_free(self, ptr):
        self._check(self.lib.nestgpu_window_free(self.ctx, ctypes.c_void_p(ptr)))

    def result_put(self, res, window_ptr, cap, offset):
        """Store res's (row id, value) rows into window rows [offset, offset+n)."""
        self._check(self.lib.nestgpu_result_put(self.ctx, ctypes.byref(res), ctypes.c_void_p(window_ptr), int(cap),
                                                int(offset)))

    def window_tensors(self, ptr, cap, n):
        """torch views (row ids, values) of the first n rows of an OWN window."""
        torch = self._torch
        if n == 0:
            e = torch.empty(0, dtype=torch.int64, device=self.device)
            return e, e
        return (_device_view(ptr, n, self.device), _device_view(ptr + 8 * int(cap), n, self.device))

    def result_tensors(self, res):
        """torch views of the device result (valid until the next exec)."""
        torch = self._torch
        n = res.n_rows

        def view(ptr, dt, w):
            if not ptr or n == 0:
                return torch.empty(0, dtype=dt, device=self.device)
            return self.arena_view(ptr, n * w).view(dt)

        return {"row": view(res.d_row_ids, torch.int64, 8), "value": view(res.d_values, torch.int64, 8),
                "valid": view(res.d_valid, torch.uint8, 1), "passed": view(res.d_passed, torch.uint8, 1)}
