"""Python binding of libll.so — the B200-native linear-layout conversion library.

Argument marshalling only: every step of the hot path runs in libll.so (host
planner in C++, sm_100a kernels specialised with NVRTC).  PyTorch is used for
device memory and streams.  There is no CPU fallback: if libll.so is missing the
import fails; on a machine without a GPU the device calls raise LLError(LL_ERR_CUDA).

Names follow the C ABI of include/ll.h (ll_layout_create, ll_compose, ll_invert,
ll_plan_convert, ll_convert, ll_plan_gather, ll_gather, ll_plan_reduce, ll_reduce).
"""
from __future__ import annotations

import ctypes as C
import json
import os
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libll.so")

# NCCL for DEVICE plans is dlopen'ed by libll.so on first use.  Point it at the same
# libnccl.so.2 torch links (the venv's nvidia-nccl wheel), so that a later `import
# torch` does not meet an older system libnccl.so.2 already loaded under that soname.
if not os.environ.get("LL_NCCL_LIB"):
    try:
        import importlib.util as _ilu
        _spec = _ilu.find_spec("nvidia.nccl")
        for _d in (list(_spec.submodule_search_locations) if _spec and _spec.submodule_search_locations else []):
            _cand = os.path.join(_d, "lib", "libnccl.so.2")
            if os.path.exists(_cand):
                os.environ["LL_NCCL_LIB"] = _cand
                break
    except Exception:
        pass

if not os.path.exists(_LIB_PATH):
    # a fresh checkout: compile the library in-tree (nvcc for sm_100a, no GPU needed);
    # without nvcc the import fails loudly — there is no fallback implementation
    try:
        import importlib.util as _ilu2
        _bspec = _ilu2.spec_from_file_location("ll_build_lib", os.path.join(_HERE, "build_lib.py"))
        _bmod = _ilu2.module_from_spec(_bspec)
        _bspec.loader.exec_module(_bmod)
        _bmod.build()
    except Exception as _e:  # noqa: BLE001 - reported as the import error
        raise ImportError(f"{_LIB_PATH} is missing and could not be built ({_e}); build it with "
                          f"`python -c 'import __graft_entry__ as g; g.build()'`") from None
_lib = C.CDLL(_LIB_PATH)

STATUS = ["OK", "INVALID_ARG", "DIM_MISMATCH", "NOT_SURJECTIVE", "NOT_INVERTIBLE", "NOT_DIVISIBLE",
          "UNSUPPORTED", "ALIAS", "MISALIGNED", "CUDA", "NVRTC", "NCCL", "OOM"]
CLASSES = ["NOOP", "REGPERM", "SHUFFLE", "SMEM", "CTA", "DEVICE"]


class LLError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"LL_ERR_{STATUS[status] if status < len(STATUS) else status}: {msg}")
        self.status = status


class _Dim(C.Structure):
    _fields_ = [("name", C.c_char_p), ("log2_size", C.c_int)]


class _Opts(C.Structure):
    _fields_ = [("force_class", C.c_int), ("max_vec_bytes", C.c_int), ("sigma", C.c_int),
                ("tile_bytes", C.c_int), ("thread_bytes", C.c_int), ("generic", C.c_int),
                ("comm", C.c_void_p), ("exchange", C.c_int), ("smem_instr", C.c_int), ("reduce_op", C.c_int),
                ("pipe", C.c_int), ("min_blocks", C.c_int)]


_P = C.c_void_p
_PP = C.POINTER(C.c_void_p)
_sig = {
    "ll_layout_create": [C.POINTER(_Dim), C.c_int, C.POINTER(_Dim), C.c_int, C.POINTER(C.c_int64), _PP],
    "ll_layout_info": [_P, C.POINTER(C.c_int)] * 1 + [C.POINTER(C.c_int)] * 3,
    "ll_layout_dim": [_P, C.c_int, C.c_int, C.POINTER(C.c_char_p), C.POINTER(C.c_int)],
    "ll_layout_bases": [_P, C.POINTER(C.c_int64)],
    "ll_layout_apply": [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int64)],
    "ll_layout_props": [_P] + [C.POINTER(C.c_int)] * 4,
    "ll_compose": [_P, _P, _PP],
    "ll_invert": [_P, _PP],
    "ll_product": [_P, _P, _PP],
    "ll_left_divide": [_P, _P, _PP],
    "ll_kernel_basis": [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int)],
    "ll_plan_convert": [_P, _P, C.c_int, C.POINTER(_Opts), _PP],
    "ll_plan_class": [_P, C.POINTER(C.c_int)],
    "ll_plan_workspace_bytes": [_P, C.POINTER(C.c_size_t)],
    "ll_plan_buffer_bytes": [_P] + [C.POINTER(C.c_size_t)] * 3,
    "ll_plan_describe": [_P, C.c_char_p, C.c_size_t],
    "ll_plan_source": [_P, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)],
    "ll_plan_prepare": [_P],
    "ll_jit_precompile": [_P],
    "ll_convert": [_P, _P, _P, _P, _P],
    "ll_plan_gather": [_P, C.c_int, C.c_int, C.POINTER(_Opts), _PP],
    "ll_gather": [_P, _P, _P, _P, _P],
    "ll_plan_reduce": [_P, C.c_int, C.POINTER(_Opts), _PP],
    "ll_plan_reduce_out_elems": [_P, C.POINTER(C.c_size_t)],
    "ll_reduce": [_P, _P, _P, _P],
    "ll_plan_scan": [_P, C.c_int, C.POINTER(_Opts), _PP],
    "ll_scan": [_P, _P, _P, _P],
    "ll_plan_simulate": [_P, _P, _P],
    "ll_comm_create": [_P, C.c_int, C.c_int, _PP],
    "ll_comm_get_unique_id": [_P],
    "ll_comm_create_loopback": [C.c_int, _PP],
    "ll_comm_check": [_P],
    "ll_plan_device_stages": [_P, _PP, _PP, C.POINTER(C.c_size_t), C.POINTER(C.c_int)],
    "ll_plan_device_peers": [_P, C.c_int, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_int)],
    "ll_comm_create_peers": [C.c_int, C.c_int, _PP, _PP, C.c_size_t, _PP],
    "ll_plan_autotune": [_P, _P, C.c_int, C.POINTER(_Opts), _P, _P, _P, C.c_int, _PP],
    "ll_ipc_export": [_P, _P],
    "ll_ipc_import": [_P, _PP],
    "ll_ipc_close": [_P],
    "ll_layout_blocked": [C.c_int] + [C.POINTER(C.c_int)] * 5 + [_PP],
    "ll_layout_mma_acc": [C.c_int, C.c_int, C.c_int, C.c_int, _PP],
    "ll_layout_mma_swizzle": [C.c_int] * 5 + [_PP],
    "ll_layout_slice": [_P, C.c_int, _PP],
    "ll_layout_contiguity": [_P, C.c_int, C.c_int, C.POINTER(C.c_int)],
    "ll_layout_mma_operand": [C.c_int] * 6 + [_PP],
    "ll_layout_tmem_32x32b": [C.c_int, C.c_int, _PP],
    "ll_layout_tmem": [C.c_char_p, C.c_int, C.c_int, _PP],
    "ll_convert_host": [_P, _P, _P, C.c_size_t, _P, C.c_int, C.POINTER(C.c_void_p)],
}
for _name, _args in _sig.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = C.c_int
_lib.ll_layout_destroy.argtypes = [_P]
_lib.ll_layout_destroy.restype = None
_lib.ll_plan_destroy.argtypes = [_P]
_lib.ll_plan_destroy.restype = None
_lib.ll_comm_destroy.argtypes = [_P]
_lib.ll_comm_destroy.restype = None
_lib.ll_last_error.restype = C.c_char_p
_lib.ll_version.restype = C.c_char_p
_lib.ll_plan_opts_default.argtypes = [C.POINTER(_Opts)]
_lib.ll_plan_opts_default.restype = None

_lib.ll_comm_create_loopback.restype = C.c_int
EXPORTED = sorted(list(_sig) + ["ll_layout_destroy", "ll_plan_destroy", "ll_comm_destroy", "ll_last_error",
                                "ll_version", "ll_plan_opts_default"])


def _check(st: int):
    if st != 0:
        raise LLError(st, _lib.ll_last_error().decode(errors="replace"))


def library_path() -> str:
    return _LIB_PATH


def version() -> str:
    return _lib.ll_version().decode()


EXCHANGES = ("auto", "collective", "peer")
# ll_plan_opts.smem_instr: auto (Thm 5.1 selection), vectorised ld/st.shared only, or
# prefer stmatrix / ldmatrix wherever their tile divides
SMEM_INSTRS = ["auto", "vec", "matrix"]
# ll_plan_opts.reduce_op (ll_plan_reduce)
REDUCE_OPS = ["sum", "max", "min"]
PEER_FLAG_BYTES = 512
IPC_HANDLE_BYTES = 72


def _opts(force_class=None, max_vec_bytes=16, sigma=0, tile_bytes=0, thread_bytes=0, generic=False, comm=None,
          exchange="auto", smem_instr="auto", reduce_op="sum", pipe="auto", min_blocks=0):
    o = _Opts()
    _lib.ll_plan_opts_default(C.byref(o))
    if force_class is not None:
        o.force_class = CLASSES.index(force_class) if isinstance(force_class, str) else int(force_class)
    o.max_vec_bytes = max_vec_bytes
    o.sigma = {"coalesced": 0, "faithful": 1}.get(sigma, sigma) if isinstance(sigma, str) else int(sigma)
    o.tile_bytes = tile_bytes
    o.thread_bytes = thread_bytes
    o.generic = int(bool(generic))
    o.comm = comm.handle if comm is not None else None
    o.exchange = EXCHANGES.index(exchange) if isinstance(exchange, str) else int(exchange)
    o.smem_instr = SMEM_INSTRS.index(smem_instr) if isinstance(smem_instr, str) else int(smem_instr)
    o.reduce_op = REDUCE_OPS.index(reduce_op) if isinstance(reduce_op, str) else int(reduce_op)
    o.pipe = {"auto": 0, "off": 1, "on": 2, "staged": 3, "bulk": 4, "bulkst": 5}[pipe] if isinstance(pipe, str) else int(pipe)
    o.min_blocks = int(min_blocks)
    return o


class Layout:
    """ll_layout: a linear layout between labelled F2 spaces (Def 4.1)."""

    def __init__(self, in_dims: Sequence[Tuple[str, int]], out_dims: Sequence[Tuple[str, int]],
                 bases: Dict[str, Sequence[Sequence[int]]] = None, _handle=None):
        if _handle is not None:
            self.handle = _handle
            return
        ins = (_Dim * max(1, len(in_dims)))(*[_Dim(n.encode(), b) for n, b in in_dims])
        outs = (_Dim * max(1, len(out_dims)))(*[_Dim(n.encode(), b) for n, b in out_dims])
        rows = []
        for n, b in in_dims:
            vecs = list((bases or {}).get(n, []))
            if len(vecs) != b:
                raise ValueError(f"dim {n}: {len(vecs)} basis vectors for {b} bits")
            rows += [list(v) for v in vecs]
        arr = (C.c_int64 * max(1, len(rows) * len(out_dims)))(*[c for r in rows for c in r])
        h = C.c_void_p()
        _check(_lib.ll_layout_create(ins, len(in_dims), outs, len(out_dims), arr, C.byref(h)))
        self.handle = h

    @classmethod
    def from_spec(cls, spec) -> "Layout":
        """From a literal spec {"out": [(name, bits)], "in": [(dim, [logical bit names])]}."""
        from workloads.configs import spec_to_bases
        in_dims, out_dims, bases = spec_to_bases(spec)
        return cls(in_dims, out_dims, bases)

    def __del__(self):
        h = getattr(self, "handle", None)
        if h and _lib is not None:
            _lib.ll_layout_destroy(h)
        self.handle = None

    def _info(self):
        a, b, c, d = C.c_int(), C.c_int(), C.c_int(), C.c_int()
        _check(_lib.ll_layout_info(self.handle, C.byref(a), C.byref(b), C.byref(c), C.byref(d)))
        return a.value, b.value, c.value, d.value

    def dims(self, out: bool):
        n_in, n_out, _, _ = self._info()
        res = []
        for i in range(n_out if out else n_in):
            nm, sz = C.c_char_p(), C.c_int()
            _check(_lib.ll_layout_dim(self.handle, int(out), i, C.byref(nm), C.byref(sz)))
            res.append((nm.value.decode(), sz.value))
        return res

    @property
    def in_dims(self):
        return self.dims(False)

    @property
    def out_dims(self):
        return self.dims(True)

    @property
    def d_in(self):
        return self._info()[2]

    @property
    def d_out(self):
        return self._info()[3]

    def bases(self) -> List[Tuple[int, ...]]:
        _, n_out, d_in, _ = self._info()
        arr = (C.c_int64 * max(1, d_in * n_out))()
        _check(_lib.ll_layout_bases(self.handle, arr))
        return [tuple(arr[k * n_out:(k + 1) * n_out]) for k in range(d_in)]

    def cols(self) -> List[int]:
        """Logical flat index (row-major, last dim fastest) per input bit."""
        out = self.out_dims
        res = []
        for v in self.bases():
            f = 0
            for (n, b), c in zip(out, v):
                f = (f << b) | c
            res.append(f)
        return res

    def apply(self, in_coords: Sequence[int]) -> Tuple[int, ...]:
        n_in, n_out, _, _ = self._info()
        a = (C.c_int64 * max(1, n_in))(*in_coords)
        b = (C.c_int64 * max(1, n_out))()
        _check(_lib.ll_layout_apply(self.handle, a, b))
        return tuple(b[:n_out])

    def props(self) -> Dict[str, bool]:
        v = [C.c_int() for _ in range(4)]
        _check(_lib.ll_layout_props(self.handle, *[C.byref(x) for x in v]))
        return dict(zip(["surjective", "injective", "distributed", "memory"], [bool(x.value) for x in v]))

    def compose(self, inner: "Layout") -> "Layout":
        """self ∘ inner (Def 4.2)."""
        h = C.c_void_p()
        _check(_lib.ll_compose(self.handle, inner.handle, C.byref(h)))
        return Layout(None, None, _handle=h)

    def invert(self) -> "Layout":
        h = C.c_void_p()
        _check(_lib.ll_invert(self.handle, C.byref(h)))
        return Layout(None, None, _handle=h)

    def product(self, other: "Layout") -> "Layout":
        h = C.c_void_p()
        _check(_lib.ll_product(self.handle, other.handle, C.byref(h)))
        return Layout(None, None, _handle=h)

    def left_divide(self, M1: "Layout") -> "Layout":
        h = C.c_void_p()
        _check(_lib.ll_left_divide(self.handle, M1.handle, C.byref(h)))
        return Layout(None, None, _handle=h)

    def contiguity(self, elem_bytes: int, max_vec_bytes: int = 16) -> int:
        """Contiguous elements per thread, capped at max_vec_bytes."""
        e = C.c_int()
        _check(_lib.ll_layout_contiguity(self.handle, int(elem_bytes), int(max_vec_bytes), C.byref(e)))
        return e.value

    def kernel_basis(self) -> List[int]:
        arr = (C.c_int64 * 64)()
        n = C.c_int()
        _check(_lib.ll_kernel_basis(self.handle, arr, C.byref(n)))
        return list(arr[:n.value])


def _ints(v):
    return (C.c_int * len(v))(*[int(x) for x in v])


def ll_layout_blocked(shape, size_per_thread, threads_per_warp, warps_per_cta, order) -> Layout:
    """Blocked layout (Prop 9.1); see include/ll.h."""
    h = C.c_void_p()
    _check(_lib.ll_layout_blocked(len(shape), _ints(shape), _ints(size_per_thread), _ints(threads_per_warp),
                                  _ints(warps_per_cta), _ints(order), C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_mma_acc(M, N, warps_m, warps_n=1) -> Layout:
    h = C.c_void_p()
    _check(_lib.ll_layout_mma_acc(M, N, warps_m, warps_n, C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_mma_swizzle(log2_rows, log2_cols, vec, per_phase, max_phase) -> Layout:
    h = C.c_void_p()
    _check(_lib.ll_layout_mma_swizzle(log2_rows, log2_cols, vec, per_phase, max_phase, C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_mma_operand(is_rhs, rows, cols, bitwidth, warps_m=1, warps_n=1) -> Layout:
    h = C.c_void_p()
    _check(_lib.ll_layout_mma_operand(int(is_rhs), rows, cols, bitwidth, warps_m, warps_n, C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_tmem_32x32b(M, N) -> Layout:
    h = C.c_void_p()
    _check(_lib.ll_layout_tmem_32x32b(M, N, C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_tmem(shape: str, M: int, N: int) -> Layout:
    """tcgen05.ld.<shape> fragment of a 128 x N fp32 TMEM accumulator (ll.h)."""
    h = C.c_void_p()
    _check(_lib.ll_layout_tmem(shape.encode(), M, N, C.byref(h)))
    return Layout(None, None, _handle=h)


def ll_layout_slice(L: Layout, dim: int) -> Layout:
    h = C.c_void_p()
    _check(_lib.ll_layout_slice(L.handle, dim, C.byref(h)))
    return Layout(None, None, _handle=h)


# ---- ABI-named functions -------------------------------------------------------------
def ll_layout_create(in_dims, out_dims, bases) -> Layout:
    return Layout(in_dims, out_dims, bases)


def ll_compose(outer: Layout, inner: Layout) -> Layout:
    return outer.compose(inner)


def ll_invert(L: Layout) -> Layout:
    return L.invert()


def _stream_ptr(stream):
    if stream is None:
        import torch
        return C.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


def _ptr(t):
    if t is None:
        return None
    if hasattr(t, "data_ptr"):
        if not t.is_cuda:
            raise LLError(1, "device entry points take CUDA tensors")
        return C.c_void_p(t.data_ptr())
    return C.c_void_p(int(t))


class Plan:
    """ll_plan: a conversion (ll_plan_convert), gather or reduce plan."""

    def __init__(self, handle, kind: str):
        self.handle = handle
        self.kind = kind

    def __del__(self):
        h = getattr(self, "handle", None)
        if h and _lib is not None:
            _lib.ll_plan_destroy(h)
        self.handle = None

    @property
    def cls(self) -> str:
        c = C.c_int()
        _check(_lib.ll_plan_class(self.handle, C.byref(c)))
        return CLASSES[c.value]

    def describe(self) -> dict:
        buf = C.create_string_buffer(1 << 20)
        _check(_lib.ll_plan_describe(self.handle, buf, len(buf)))
        return json.loads(buf.value.decode())

    def source(self) -> str:
        n = C.c_size_t()
        _check(_lib.ll_plan_source(self.handle, None, 0, C.byref(n)))
        buf = C.create_string_buffer(n.value + 1)
        _check(_lib.ll_plan_source(self.handle, buf, len(buf), C.byref(n)))
        return buf.value.decode()

    def buffer_bytes(self):
        """(src, dst, idx) bytes the execution call touches (ll_plan_buffer_bytes)."""
        a, b, c = C.c_size_t(), C.c_size_t(), C.c_size_t()
        _check(_lib.ll_plan_buffer_bytes(self.handle, C.byref(a), C.byref(b), C.byref(c)))
        return a.value, b.value, c.value

    def check_buffers(self, src=None, dst=None, idx=None, workspace=None):
        """Raise LLError when a torch tensor is smaller than the plan's buffer (raw
        pointers cannot be checked and pass through).  Plans are immutable, so the
        sizes are queried once and cached (keeps small launches off the host path)."""
        need = self.__dict__.get("_need")
        if need is None:
            need = dict(zip(("src", "dst", "idx"), self.buffer_bytes()))
            need["workspace"] = self.workspace_bytes() if self.kind == "convert" else 0
            self._need = need
        for name, t in (("src", src), ("dst", dst), ("idx", idx), ("workspace", workspace)):
            if t is None or isinstance(t, int) or not hasattr(t, "numel"):
                if name == "workspace" and t is None and need[name] > 0:
                    raise LLError(1, f"{name}: the plan needs {need[name]} bytes of workspace")
                continue
            have = t.numel() * t.element_size()
            if have < need[name]:
                raise LLError(1, f"{name}: {have} bytes < the plan's {need[name]} bytes")
            if not t.is_contiguous():
                raise LLError(1, f"{name}: tensor must be contiguous")

    def workspace_bytes(self) -> int:
        n = C.c_size_t()
        _check(_lib.ll_plan_workspace_bytes(self.handle, C.byref(n)))
        return n.value

    def prepare(self):
        _check(_lib.ll_plan_prepare(self.handle))
        return self

    def precompile(self):
        _check(_lib.ll_jit_precompile(self.handle))
        return self

    def out_elems(self) -> int:
        n = C.c_size_t()
        _check(_lib.ll_plan_reduce_out_elems(self.handle, C.byref(n)))
        return n.value

    def device_peers(self, rank: int):
        """(send_peers, recv_peers) of a collective DEVICE plan for `rank`: send chunk j
        goes to send_peers[j], recv chunk i comes from recv_peers[i] (ll.h)."""
        n = C.c_int()
        sp, rp = (C.c_int * 64)(), (C.c_int * 64)()
        _check(_lib.ll_plan_device_peers(self.handle, int(rank), sp, rp, C.byref(n)))
        return list(sp[:n.value]), list(rp[:n.value])

    def device_stages(self):
        """(pack, unpack, chunk_elems, nranks) of a DEVICE plan; stages are None when
        they are the identity.  Stage plans are views owned by this plan."""
        pk, up = C.c_void_p(), C.c_void_p()
        ch, nr = C.c_size_t(), C.c_int()
        _check(_lib.ll_plan_device_stages(self.handle, C.byref(pk), C.byref(up), C.byref(ch), C.byref(nr)))
        wrap = lambda h: _Stage(h, self) if h.value else None
        return wrap(pk), wrap(up), ch.value, nr.value

    def simulate(self, src: np.ndarray, dst_elems: int) -> np.ndarray:
        """Host emulation of the plan's kernel schedule (test hook, no GPU)."""
        src = np.ascontiguousarray(src)
        dst = np.zeros(dst_elems, dtype=src.dtype)
        _check(_lib.ll_plan_simulate(self.handle, src.ctypes.data_as(C.c_void_p), dst.ctypes.data_as(C.c_void_p)))
        return dst


class _Stage(Plan):
    """A borrowed stage view of a DEVICE plan (kept alive by its parent)."""

    def __init__(self, handle, parent):
        super().__init__(handle, "convert")
        self.parent = parent

    def __del__(self):
        self.handle = None


class Comm:
    """ll_comm: NCCL communicator (one per rank) or a single-process loopback."""

    def __init__(self, handle, nranks):
        self.handle, self.nranks = handle, nranks

    def check(self):
        """ll_comm_check: raise LLError(NCCL) if the communicator recorded an
        asynchronous NCCL error (failure detection)."""
        _check(_lib.ll_comm_check(self.handle))

    @classmethod
    def loopback(cls, nranks: int) -> "Comm":
        h = C.c_void_p()
        _check(_lib.ll_comm_create_loopback(int(nranks), C.byref(h)))
        return cls(h, nranks)

    @classmethod
    def from_process_group(cls, group=None) -> "Comm":
        """Bootstrap NCCL: rank 0's ncclUniqueId is broadcast over the torch group."""
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        uid = (C.c_char * 128)()
        if rank == 0:
            _check(_lib.ll_comm_get_unique_id(uid))
        obj = [bytes(uid)]
        dist.broadcast_object_list(obj, src=0, group=group)
        uid = (C.c_char * 128).from_buffer_copy(obj[0])
        h = C.c_void_p()
        _check(_lib.ll_comm_create(uid, world, rank, C.byref(h)))
        return cls(h, world)

    @classmethod
    def peers(cls, dst_window, flags, group=None) -> "Comm":
        """Peer-window communicator (LL_EXCHANGE_PEER, §8(f) N4).  dst_window: this
        rank's dst buffer (CUDA tensor, the `dst` of every ll_convert on it); flags:
        a zeroed CUDA tensor of >= PEER_FLAG_BYTES.  The other ranks' buffers are
        mapped with CUDA IPC; the handles travel over the torch process group."""
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        if flags.numel() * flags.element_size() < PEER_FLAG_BYTES:
            raise ValueError("flags must hold at least PEER_FLAG_BYTES")
        hd, hf = ipc_export(dst_window), ipc_export(flags)
        allh = [None] * world
        dist.all_gather_object(allh, (hd, hf), group=group)
        opened, dptr, fptr = [], [], []
        for q in range(world):
            if q == rank:
                dptr.append(dst_window.data_ptr())
                fptr.append(flags.data_ptr())
            else:
                d, f = ipc_import(allh[q][0]), ipc_import(allh[q][1])
                opened += [d, f]
                dptr.append(d)
                fptr.append(f)
        da = (C.c_void_p * world)(*dptr)
        fa = (C.c_void_p * world)(*fptr)
        h = C.c_void_p()
        _check(_lib.ll_comm_create_peers(world, rank, da, fa, dst_window.numel() * dst_window.element_size(),
                                         C.byref(h)))
        c = cls(h, world)
        c._opened, c._keep = opened, (dst_window, flags)
        return c

    def __del__(self):
        h = getattr(self, "handle", None)
        if h and _lib is not None:
            _lib.ll_comm_destroy(h)
        self.handle = None
        for ptr in getattr(self, "_opened", []):
            if _lib is not None:
                _lib.ll_ipc_close(C.c_void_p(ptr))
        self._opened = []


def ipc_export(t) -> bytes:
    """CUDA IPC handle (IPC_HANDLE_BYTES) of a CUDA tensor's memory."""
    buf = (C.c_char * IPC_HANDLE_BYTES)()
    _check(_lib.ll_ipc_export(C.c_void_p(t.data_ptr()), buf))
    return bytes(buf)


def ipc_import(handle: bytes) -> int:
    """Map another process's exported buffer; returns its device address here."""
    buf = (C.c_char * IPC_HANDLE_BYTES).from_buffer_copy(handle)
    p = C.c_void_p()
    _check(_lib.ll_ipc_import(buf, C.byref(p)))
    return p.value


def ll_plan_convert(A: Layout, B: Layout, elem_bytes: int, **opts) -> Plan:
    h = C.c_void_p()
    o = _opts(**opts)
    _check(_lib.ll_plan_convert(A.handle, B.handle, int(elem_bytes), C.byref(o), C.byref(h)))
    p = Plan(h, "convert")
    p.comm = opts.get("comm")   # keep the communicator alive as long as the plan
    return p


def ll_plan_autotune(A: Layout, B: Layout, elem_bytes: int, src, dst, stream=None, iters: int = 10, **opts) -> Plan:
    """Fastest plan among the candidate kernel decompositions, timed on src/dst."""
    h = C.c_void_p()
    o = _opts(**opts)
    _check(_lib.ll_plan_autotune(A.handle, B.handle, int(elem_bytes), C.byref(o), _ptr(src), _ptr(dst),
                                 _stream_ptr(stream), int(iters), C.byref(h)))
    p = Plan(h, "convert")
    p.comm = opts.get("comm")
    return p


def ll_convert(src, dst, plan: Plan, stream=None, workspace=None):
    """dst <- convert(src) on `stream` (torch CUDA tensors or raw device pointers)."""
    plan.check_buffers(src, dst, workspace=workspace)
    _check(_lib.ll_convert(_ptr(src), _ptr(dst), _ptr(workspace), plan.handle, _stream_ptr(stream)))


def ll_convert_host(src_host, dst_host, dev_buf, plan: Plan, streams):
    """End-to-end conversion from pinned HOST tensors through the device (chunked H2D ->
    kernel -> D2H pipeline over `streams`); dev_buf is a CUDA tensor used as scratch."""
    arr = (C.c_void_p * len(streams))(*[s.cuda_stream for s in streams])
    _check(_lib.ll_convert_host(C.c_void_p(src_host.data_ptr()), C.c_void_p(dst_host.data_ptr()),
                                C.c_void_p(dev_buf.data_ptr()), dev_buf.numel() * dev_buf.element_size(),
                                plan.handle, len(streams), arr))


def ll_plan_gather(L: Layout, axis: int, elem_bytes: int, **opts) -> Plan:
    h = C.c_void_p()
    o = _opts(**opts)
    _check(_lib.ll_plan_gather(L.handle, int(axis), int(elem_bytes), C.byref(o), C.byref(h)))
    return Plan(h, "gather")


def ll_gather(src, idx, dst, plan: Plan, stream=None):
    plan.check_buffers(src, dst, idx)
    _check(_lib.ll_gather(_ptr(src), _ptr(idx), _ptr(dst), plan.handle, _stream_ptr(stream)))


def ll_plan_reduce(L: Layout, axis: int, **opts) -> Plan:
    h = C.c_void_p()
    o = _opts(**opts)
    _check(_lib.ll_plan_reduce(L.handle, int(axis), C.byref(o), C.byref(h)))
    return Plan(h, "reduce")


def ll_plan_scan(L: Layout, axis: int, **opts) -> Plan:
    h = C.c_void_p()
    o = _opts(**opts)
    _check(_lib.ll_plan_scan(L.handle, int(axis), C.byref(o), C.byref(h)))
    return Plan(h, "scan")


def ll_scan(src, dst, plan: Plan, stream=None):
    plan.check_buffers(src, dst)
    _check(_lib.ll_scan(_ptr(src), _ptr(dst), plan.handle, _stream_ptr(stream)))


def ll_reduce(src, dst, plan: Plan, stream=None):
    plan.check_buffers(src, dst)
    _check(_lib.ll_reduce(_ptr(src), _ptr(dst), plan.handle, _stream_ptr(stream)))
