"""xreduce -- B200-native (sm_100a) parallel reductions over 1-3 level loop nests.

Thin ctypes binding over ``libxreduce.so`` (include/xreduce.h).  Argument
marshalling only: every step of the reduction runs in the library's CUDA
kernels.  PyTorch is used for device memory, streams and process groups.
There is NO CPU fallback: if the shared library is missing this import fails
loudly (build it with ``python tools/build_native.py`` or
``__graft_entry__.build()``).

Paper: Xu, Tian, Yan, Chandrasekaran, Chapman, "Reduction Operations in
Parallel Loops for GPGPUs", PMAM'14; see DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# XR_LIB_PATH: load another build of the same library (tools/ A/B variants only)
LIB_PATH = os.environ.get("XR_LIB_PATH") or os.path.join(_HERE, "libxreduce.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"xreduce: {LIB_PATH} is missing -- build the CUDA library first "
        "(python tools/build_native.py); there is no CPU fallback")
_lib = ctypes.CDLL(LIB_PATH)

# ---- codes (include/xreduce.h)
OP_ADD, OP_MUL, OP_MAX, OP_MIN, OP_BAND, OP_BOR, OP_BXOR, OP_LAND, OP_LOR = range(9)
INT32, INT64, FP32, FP64 = range(4)
GANG, WORKER, VECTOR, INIT_FROM_OUT = 0x1, 0x2, 0x4, 0x100
OK, ERR_INVALID, ERR_UNSUPPORTED, ERR_CUDA, ERR_NCCL, ERR_NOMEM = range(6)
SHAPES = {0: "none", 1: "fill", 2: "ident", 3: "R", 4: "KR", 5: "RK", 6: "KRK", 7: "RKR"}
KERNELS = {0: "none", 1: "fill", 2: "ident", 3: "seg", 4: "col", 5: "stream", 6: "coltma", 7: "rows", 8: "colflat", 9: "rkr",
           10: "colsmall", 11: "rcluster", 12: "shortrow", 13: "thincol"}
COLL_NONE, COLL_ALLREDUCE, COLL_ALLGATHER_COMBINE, COLL_ALLGATHER = range(4)

OPS = {"+": OP_ADD, "*": OP_MUL, "max": OP_MAX, "min": OP_MIN, "&": OP_BAND, "|": OP_BOR,
       "^": OP_BXOR, "&&": OP_LAND, "||": OP_LOR}
DTYPES = {"int32": INT32, "int64": INT64, "fp32": FP32, "fp64": FP64}


class XReduceError(RuntimeError):
    def __init__(self, status: int, where: str = ""):
        msg = _lib.xr_strerror(status).decode()
        super().__init__(f"{where}: {msg}" if where else msg)
        self.status = status


class PlanInfo(ctypes.Structure):
    _fields_ = [("shape", ctypes.c_int), ("kernel", ctypes.c_int),
                ("cdims", ctypes.c_int64 * 3), ("out_count", ctypes.c_int64),
                ("group", ctypes.c_int), ("vec", ctypes.c_int), ("splits", ctypes.c_int64),
                ("units", ctypes.c_int64), ("grid", ctypes.c_int64), ("block", ctypes.c_int),
                ("ws_bytes", ctypes.c_int64), ("tickets", ctypes.c_int64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["cdims"] = list(self.cdims)
        d["shape"] = SHAPES[self.shape]
        d["kernel"] = KERNELS[self.kernel]
        return d


class Var(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int), ("dtype", ctypes.c_int), ("in_", ctypes.c_void_p),
                ("out", ctypes.c_void_p)]


class VarAt(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int), ("dtype", ctypes.c_int), ("level_mask", ctypes.c_uint),
                ("in_", ctypes.c_void_p), ("out", ctypes.c_void_p)]


class ShardInfo(ctypes.Structure):
    _fields_ = [("collective", ctypes.c_int), ("nccl_op", ctypes.c_int),
                ("merge_init", ctypes.c_int), ("local_init_from_out", ctypes.c_int),
                ("local_count", ctypes.c_int64), ("global_count", ctypes.c_int64),
                ("out_offset", ctypes.c_int64), ("gang_offset", ctypes.c_int64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_i64p = ctypes.POINTER(ctypes.c_int64)
_vp = ctypes.c_void_p
_c = ctypes.c_int
_u = ctypes.c_uint

_SIGS = {
    "xr_reduce": (_c, [_c, _c, _i64p, _u, _vp, _vp, _vp]),
    "xr_out_count": (_c, [_i64p, _u, _i64p]),
    "xr_strerror": (ctypes.c_char_p, [_c]),
    "xr_reduce_host": (_c, [_c, _c, _i64p, _u, _vp, _vp, _vp]),
    "xr_host_chunks": (_c, [_i64p, _u, _c, ctypes.c_int64, ctypes.c_int64, _i64p, _i64p]),
    "xr_plan_describe": (_c, [_c, _c, _i64p, _u, ctypes.c_uint64, _c, ctypes.POINTER(PlanInfo)]),
    "xr_reserve": (_c, [_c, _c, _i64p, _u, _vp]),
    "xr_shutdown": (_c, []),
    "xr_launch_count": (ctypes.c_int64, []),
    "xr_debug_timeline": (_c, [_vp, ctypes.c_int64]),
    "xr_heat_step": (_c, [ctypes.c_int64, ctypes.c_int64, _vp, _vp, _vp, _vp]),
    "xr_heat_run": (_c, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, _vp, _vp, _vp, _vp]),
    "xr_shard_plan": (_c, [_c, _c, _i64p, _u, _c, _c, ctypes.POINTER(ShardInfo)]),
    "xr_comm_get_unique_id": (_c, [_vp]),
    "xr_comm_init": (_c, [ctypes.POINTER(_vp), _c, _c, _vp, _c]),
    "xr_comm_destroy": (_c, [_vp]),
    "xr_reduce_sharded": (_c, [_c, _c, _i64p, _u, _vp, _vp, _vp, _vp]),
    "xr_reduce_sharded_host": (_c, [_c, _c, _i64p, _u, _vp, _vp, _vp, _vp]),
    "xr_reduce_sharded_sim": (_c, [_c, _c, _i64p, _u, ctypes.POINTER(_vp), _c, _vp, _vp]),
    "xr_reduce_fused_sim": (_c, [_c, _c, _i64p, _u, ctypes.POINTER(_vp), _c, ctypes.POINTER(_vp)]),
    "xr_comm_set_fused": (_c, [_vp, _c]),
    "xr_comm_query": (_c, [_vp, ctypes.POINTER(_c), ctypes.POINTER(_c)]),
    "xr_transform_reduce": (_c, [_c, _c, _i64p, _u, _vp, _vp, _vp, _vp]),
    "xr_reduce_paper": (_c, [_c, _c, _i64p, _u, _vp, _vp, _c, _c, _c, _vp]),
    "xr_reduce_multi": (_c, [_c, ctypes.POINTER(Var), _i64p, _u, _vp]),
    "xr_reduce_multi_at": (_c, [_c, ctypes.POINTER(VarAt), _i64p, _vp]),
    "xr_heat_step_sharded": (_c, [ctypes.c_int64, ctypes.c_int64, _vp, _vp, _vp, _vp, _vp]),
    "xr_heat_run_sharded": (_c, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, _vp, _vp, _vp, _vp, _vp]),
    "xr_heat_run_sharded_sim": (_c, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, _c, ctypes.POINTER(_vp),
                                     ctypes.POINTER(_vp), _vp, _vp]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_SIGS)


def _dims(d):
    return (ctypes.c_int64 * 3)(*[int(v) for v in d])


def _check(st: int, where: str):
    if st != OK:
        raise XReduceError(st, where)


def mask_of(levels) -> int:
    """'gwv'-style string (or an int) -> level mask."""
    if isinstance(levels, int):
        return levels
    m = 0
    for ch in levels.lower():
        m |= {"g": GANG, "w": WORKER, "v": VECTOR}[ch]
    return m


def _op(op):
    return OPS[op] if isinstance(op, str) else int(op)


def _dt(dt):
    return DTYPES[dt] if isinstance(dt, str) else int(dt)


# ---------------------------------------------------------------- raw C ABI
def xr_reduce(op, dtype, nest_dims, level_mask, in_ptr: int, out_ptr: int, stream: int = 0) -> int:
    return _lib.xr_reduce(_op(op), _dt(dtype), _dims(nest_dims), mask_of(level_mask),
                          in_ptr or None, out_ptr or None, stream or None)


def xr_out_count(nest_dims, level_mask) -> int:
    c = ctypes.c_int64(0)
    _check(_lib.xr_out_count(_dims(nest_dims), mask_of(level_mask), ctypes.byref(c)), "xr_out_count")
    return int(c.value)


def xr_strerror(status: int) -> str:
    return _lib.xr_strerror(status).decode()


def xr_plan_describe(op, dtype, nest_dims, level_mask, in_addr: int = 0, num_sms: int = 148) -> dict:
    info = PlanInfo()
    _check(_lib.xr_plan_describe(_op(op), _dt(dtype), _dims(nest_dims), mask_of(level_mask),
                                 in_addr, num_sms, ctypes.byref(info)), "xr_plan_describe")
    return info.as_dict()


def xr_shard_plan(op, dtype, local_dims, level_mask, nranks: int, rank: int) -> dict:
    info = ShardInfo()
    _check(_lib.xr_shard_plan(_op(op), _dt(dtype), _dims(local_dims), mask_of(level_mask),
                              nranks, rank, ctypes.byref(info)), "xr_shard_plan")
    return info.as_dict()


def xr_reduce_host(op, dtype, nest_dims, level_mask, in_host_ptr: int, out_host_ptr: int,
                   stream: int = 0) -> int:
    return _lib.xr_reduce_host(_op(op), _dt(dtype), _dims(nest_dims), mask_of(level_mask),
                               in_host_ptr or None, out_host_ptr or None, stream or None)


def xr_host_chunks(nest_dims, level_mask, dtype, cap_bytes: int) -> list:
    """The chunk schedule of xr_reduce_host (host only): a list of
    (dims, in_off, out_off, first) tuples."""
    n = ctypes.c_int64(0)
    _check(_lib.xr_host_chunks(_dims(nest_dims), mask_of(level_mask), _dt(dtype), cap_bytes, 0, None,
                               ctypes.byref(n)), "xr_host_chunks")
    buf = (ctypes.c_int64 * (6 * max(n.value, 1)))()
    _check(_lib.xr_host_chunks(_dims(nest_dims), mask_of(level_mask), _dt(dtype), cap_bytes, n.value,
                               ctypes.cast(buf, _i64p), ctypes.byref(n)), "xr_host_chunks")
    return [((buf[6 * k], buf[6 * k + 1], buf[6 * k + 2]), buf[6 * k + 3], buf[6 * k + 4], bool(buf[6 * k + 5]))
            for k in range(n.value)]


def xr_reserve(op, dtype, nest_dims, level_mask, stream: int = 0) -> int:
    return _lib.xr_reserve(_op(op), _dt(dtype), _dims(nest_dims), mask_of(level_mask), stream or None)


def xr_shutdown() -> int:
    return _lib.xr_shutdown()


def xr_launch_count() -> int:
    return int(_lib.xr_launch_count())


def xr_reduce_fused_sim(op, dtype, local_dims, level_mask, shard_ptrs, out_ptrs) -> int:
    a = (_vp * len(shard_ptrs))(*shard_ptrs)
    o = (_vp * len(out_ptrs))(*out_ptrs)
    return _lib.xr_reduce_fused_sim(_op(op), _dt(dtype), _dims(local_dims), mask_of(level_mask), a,
                                    len(shard_ptrs), o)


def xr_heat_step(nj, ni, t1_ptr, t2_ptr, residual_ptr, stream: int = 0) -> int:
    return _lib.xr_heat_step(nj, ni, t1_ptr, t2_ptr, residual_ptr, stream or None)


def xr_heat_run(nj, ni, iters, t1_ptr, t2_ptr, residuals_ptr, stream: int = 0) -> int:
    return _lib.xr_heat_run(nj, ni, iters, t1_ptr, t2_ptr, residuals_ptr, stream or None)


def xr_reduce_sharded_sim(op, dtype, local_dims, level_mask, shard_ptrs, out_ptr, stream: int = 0) -> int:
    arr = (_vp * len(shard_ptrs))(*shard_ptrs)
    return _lib.xr_reduce_sharded_sim(_op(op), _dt(dtype), _dims(local_dims), mask_of(level_mask),
                                      arr, len(shard_ptrs), out_ptr, stream or None)


XFORMS = {"disk": 1, "dot": 2}


def xr_reduce_multi(variables, nest_dims, level_mask, stream: int = 0) -> int:
    """variables: iterable of (op, dtype, in_ptr, out_ptr)."""
    vs = list(variables)
    arr = (Var * len(vs))(*[Var(_op(o), _dt(d), i or None, p or None) for o, d, i, p in vs])
    return _lib.xr_reduce_multi(len(vs), arr, _dims(nest_dims), mask_of(level_mask), stream or None)


def xr_reduce_multi_at(variables, nest_dims, stream: int = 0) -> int:
    """variables: iterable of (op, dtype, level_mask, in_ptr, out_ptr) -- each
    variable reduced at its own levels, one launch (include/xreduce.h)."""
    vs = list(variables)
    arr = (VarAt * len(vs))(*[VarAt(_op(o), _dt(d), mask_of(m), i or None, p or None) for o, d, m, i, p in vs])
    return _lib.xr_reduce_multi_at(len(vs), arr, _dims(nest_dims), stream or None)


def xr_reduce_paper(op, dtype, nest_dims, level_mask, in_ptr: int, out_ptr: int, num_gangs: int = 0,
                    num_workers: int = 0, vector_length: int = 0, stream: int = 0) -> int:
    """The paper's own scheme (A/B baseline, include/xreduce.h)."""
    return _lib.xr_reduce_paper(_op(op), _dt(dtype), _dims(nest_dims), mask_of(level_mask), in_ptr or None,
                                out_ptr or None, num_gangs, num_workers, vector_length, stream or None)


def xr_transform_reduce(xform, dtype, nest_dims, level_mask, x_ptr: int, y_ptr: int, out_ptr: int,
                        stream: int = 0) -> int:
    return _lib.xr_transform_reduce(XFORMS[xform] if isinstance(xform, str) else int(xform), _dt(dtype),
                                    _dims(nest_dims), mask_of(level_mask), x_ptr or None, y_ptr or None,
                                    out_ptr or None, stream or None)


def xr_heat_run_sharded_sim(n_local, ni, iters, t1_ptrs, t2_ptrs, residuals_ptr, stream: int = 0) -> int:
    a = (_vp * len(t1_ptrs))(*t1_ptrs)
    b = (_vp * len(t2_ptrs))(*t2_ptrs)
    return _lib.xr_heat_run_sharded_sim(n_local, ni, iters, len(t1_ptrs), a, b, residuals_ptr, stream or None)


def xr_heat_run_sharded(n_local, ni, iters, t1_ptr, t2_ptr, residuals_ptr, comm, stream: int = 0) -> int:
    return _lib.xr_heat_run_sharded(n_local, ni, iters, t1_ptr, t2_ptr, residuals_ptr, comm.handle,
                                    stream or None)


# ---------------------------------------------------------------- torch-facing helpers
_TORCH_DT = None


def _torch_dtypes():
    global _TORCH_DT
    if _TORCH_DT is None:
        import torch
        _TORCH_DT = {torch.int32: INT32, torch.int64: INT64, torch.float32: FP32, torch.float64: FP64}
    return _TORCH_DT


def _stream_handle(stream=None, device=None) -> int:
    import torch
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return int(s.cuda_stream)


def _nest_of(x, nest):
    """The (n0, n1, n2) view of tensor ``x``: ``nest`` if given (its product
    must equal x.numel()), else x.shape with leading dimensions beyond the
    last two flattened into n0 (and missing ones padded with 1 on the left)."""
    if nest is None:
        shp = [int(v) for v in x.shape]
        if len(shp) > 3:
            lead = 1
            for v in shp[:-2]:
                lead *= v
            shp = [lead] + shp[-2:]
        nest = [1] * (3 - len(shp)) + shp
    nest = [int(v) for v in nest]
    if len(nest) != 3 or any(v < 0 for v in nest):
        raise ValueError(f"nest must be 3 non-negative extents, got {nest}")
    if nest[0] * nest[1] * nest[2] != x.numel():
        raise ValueError(f"nest {tuple(nest)} has {nest[0] * nest[1] * nest[2]} elements but the tensor has "
                         f"{x.numel()}")
    return nest


def _check_out(out, x, count: int):
    if out.dtype != x.dtype:
        raise ValueError(f"out dtype {out.dtype} differs from the input's {x.dtype}")
    if out.device != x.device:
        raise ValueError(f"out is on {out.device}, the input on {x.device}")
    if out.numel() < count or not out.is_contiguous():
        raise ValueError(f"out must be contiguous with at least {count} elements (has {out.numel()})")


def reduce(x, op="+", levels="gwv", nest=None, out=None, init=None, stream=None):
    """Reduce CUDA tensor ``x`` (viewed as nest ``(n0, n1, n2)``; default:
    x.shape, leading dims beyond 3 flattened into n0) over ``levels``;
    returns the compact output tensor (shape = the kept extents).  Runs on
    x's device, on ``stream`` or that device's current stream."""
    import torch
    if not x.is_cuda:
        raise ValueError("xreduce.reduce needs a CUDA tensor (no CPU fallback)")
    if x.dtype not in _torch_dtypes():
        raise ValueError(f"unsupported dtype {x.dtype} (int32, int64, float32, float64)")
    x = x.contiguous()
    nest = _nest_of(x, nest)
    mask = mask_of(levels)
    dt = _torch_dtypes()[x.dtype]
    kept = [nest[d] for d in range(3) if not (mask >> d) & 1]
    count = xr_out_count(nest, mask)
    with torch.cuda.device(x.device):
        if out is None:
            out = torch.empty(kept if kept else [1], dtype=x.dtype, device=x.device)
        _check_out(out, x, count)
        if init is not None:
            out.copy_(torch.as_tensor(init, dtype=x.dtype, device=x.device).reshape(out.shape))
            mask |= INIT_FROM_OUT
        _check(xr_reduce(_op(op), dt, nest, mask, x.data_ptr(), out.data_ptr(), _stream_handle(stream, x.device)),
               "xr_reduce")
    return out


class Comm:
    """An xreduce NCCL communicator built over a torch.distributed process group
    (the 128-byte NCCL unique id is broadcast with torch.distributed)."""

    def __init__(self, group=None, device: int | None = None):
        import torch
        import torch.distributed as dist
        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        self.device = torch.cuda.current_device() if device is None else device
        uid = (ctypes.c_char * 128)()
        if self.rank == 0:
            _check(_lib.xr_comm_get_unique_id(ctypes.cast(uid, _vp)), "xr_comm_get_unique_id")
        obj = [bytes(uid) if self.rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        uid = (ctypes.c_char * 128).from_buffer_copy(obj[0])
        self._h = _vp()
        _check(_lib.xr_comm_init(ctypes.byref(self._h), self.nranks, self.rank,
                                 ctypes.cast(uid, _vp), self.device), "xr_comm_init")

    @property
    def handle(self):
        return self._h

    def set_fused(self, enable: bool) -> int:
        return _lib.xr_comm_set_fused(self._h, 1 if enable else 0)

    def query(self):
        f, st = ctypes.c_int(0), ctypes.c_int(0)
        _check(_lib.xr_comm_query(self._h, ctypes.byref(f), ctypes.byref(st)), "xr_comm_query")
        return {"fused": bool(f.value), "status": st.value}

    def close(self):
        if self._h:
            _check(_lib.xr_comm_destroy(self._h), "xr_comm_destroy")
            self._h = _vp()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def reduce_sharded(x_local, comm: Comm, op="+", levels="gwv", nest_local=None, out=None, init=None,
                   stream=None):
    """Gang-sharded reduction: every rank passes its contiguous gang slice;
    returns the GLOBAL result on every rank (include/xreduce.h)."""
    import torch
    if not x_local.is_cuda:
        raise ValueError("xreduce.reduce_sharded needs a CUDA tensor (no CPU fallback)")
    if x_local.dtype not in _torch_dtypes():
        raise ValueError(f"unsupported dtype {x_local.dtype} (int32, int64, float32, float64)")
    x_local = x_local.contiguous()
    nest_local = _nest_of(x_local, nest_local)
    mask = mask_of(levels)
    info = xr_shard_plan(op, _torch_dtypes()[x_local.dtype], nest_local, mask, comm.nranks, comm.rank)
    with torch.cuda.device(x_local.device):
        if out is None:
            out = torch.empty(max(info["global_count"], 1), dtype=x_local.dtype, device=x_local.device)
        _check_out(out, x_local, info["global_count"])
        if init is not None:
            out.copy_(torch.as_tensor(init, dtype=x_local.dtype, device=out.device).reshape(out.shape))
            mask |= INIT_FROM_OUT
        _check(_lib.xr_reduce_sharded(_op(op), _torch_dtypes()[x_local.dtype], _dims(nest_local), mask,
                                      x_local.data_ptr(), out.data_ptr(), comm.handle,
                                      _stream_handle(stream, x_local.device)), "xr_reduce_sharded")
    return out
