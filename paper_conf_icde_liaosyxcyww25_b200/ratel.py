"""Thin ctypes binding of libratel.so -- same names as include/ratel.h.

Argument marshalling only: every step of the optimizer path runs in the CUDA
library.  There is no fallback: if libratel.so is missing or fails to load,
importing this module raises ImportError.

Errors: a non-zero status becomes ``RatelError(code, message)`` carrying the
C code (RATEL_EINVAL, RATEL_ESTATE, ...) and ratel_last_error()'s text.
Pointers are passed as integers (``tensor.data_ptr()``); CUDA streams as
integers (``torch.cuda.Stream.cuda_stream``) or None.
"""
from __future__ import annotations

import ctypes
import os

_LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libratel.so")

RATEL_OK = 0
RATEL_EINVAL = -1
RATEL_ESTATE = -2
RATEL_ECUDA = -3
RATEL_ENCCL = -4
RATEL_ENOMEM = -5
RATEL_ENONFINITE = -6
RATEL_EIO = -7

RATEL_DEVICE = 0
RATEL_PINNED_HOST = 1
RATEL_HOST_COMPUTE = 2
RATEL_SSD = 3
RATEL_SSD_HOST_COMPUTE = 4
RATEL_ADAMW = 0
RATEL_ADAM_L2 = 1
RATEL_STAGING_PIPELINED = 0
RATEL_STAGING_SERIALIZED = 1
RATEL_STAGING_ZERO_COPY = 2
RATEL_COMM_AUTO = 0
RATEL_COMM_NONE = 1
RATEL_COMM_NCCL = 2
RATEL_UPDATE_TMA = 0
RATEL_UPDATE_LDG = 1
RATEL_UPDATE_LDG_LITE = 2
RATEL_SSD_DUPLEX = 0
RATEL_SSD_SIMPLEX = 1
RATEL_SSD_IO_PREAD = 0
RATEL_SSD_IO_URING = 1
RATEL_MAX_BLOCKS = 4096
RATEL_MAX_RANGES_PER_BLOCK = 32

_NAMES = {0: "RATEL_OK", -1: "RATEL_EINVAL", -2: "RATEL_ESTATE", -3: "RATEL_ECUDA",
          -4: "RATEL_ENCCL", -5: "RATEL_ENOMEM", -6: "RATEL_ENONFINITE",
          -7: "RATEL_EIO"}


class RatelError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_NAMES.get(code, code)}: {msg}")
        self.code = code


class ratel_config(ctypes.Structure):
    _fields_ = [
        ("mode", ctypes.c_int),
        ("max_grad_norm", ctypes.c_double),
        ("pipeline_depth", ctypes.c_int),
        ("staging", ctypes.c_int),
        ("tile_elems", ctypes.c_uint64),
        ("max_ctas", ctypes.c_int),
        ("timing", ctypes.c_int),
        ("comm", ctypes.c_int),
        ("host_threads", ctypes.c_int),
        ("update_streams", ctypes.c_int),
        ("cta_tiles", ctypes.c_int),
        ("k1_kernel", ctypes.c_int),
        ("ssd_schedule", ctypes.c_int),
        ("ssd_io", ctypes.c_int),
    ]


class ratel_range(ctypes.Structure):
    _fields_ = [
        ("param_bf16", ctypes.c_void_p),
        ("grad_bf16", ctypes.c_void_p),
        ("grad_is_rank_slice", ctypes.c_int),
        ("master", ctypes.c_void_p),
        ("exp_avg", ctypes.c_void_p),
        ("exp_avg_sq", ctypes.c_void_p),
        ("numel", ctypes.c_uint64),
        ("apply_weight_decay", ctypes.c_int),
    ]


class ratel_swap_model(ctypes.Structure):
    """include/ratel_plan.h: Table I quantities."""
    _fields_ = [(f, ctypes.c_double) for f in
                ("thp_g", "bw_g", "bw_s2m", "bw_m2s", "mem_m_avail", "params", "flop_f")]


class ratel_swap_layer(ctypes.Structure):
    _fields_ = [("act_bytes", ctypes.c_double), ("recompute_flop", ctypes.c_double)]


class ratel_swap_plan(ctypes.Structure):
    _fields_ = [("n_swap", ctypes.c_int)] + [(f, ctypes.c_double) for f in
                                              ("a_g2m", "flop_r", "t_f", "t_b", "t_iter", "t_min")]


def load_library(path: str = _LIB_PATH, strict: bool = True):
    """Load a libratel.so build and declare its signatures (tools load
    build-variant copies through this; the package uses the in-tree one)."""
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: build it with "
                          "`python -c 'import __graft_entry__ as g; g.build()'` (no CPU fallback exists)")
    lib = ctypes.CDLL(path)
    P, I, U64, D = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64, ctypes.c_double
    sig = {
        "ratel_default_config": (None, [ctypes.POINTER(ratel_config)]),
        "ratel_get_nccl_unique_id": (I, [P]),
        "ratel_init": (I, [I, I, I, P, ctypes.POINTER(ratel_config)]),
        "ratel_register_block": (I, [I, ctypes.POINTER(ratel_range), I, I]),
        "ratel_adam_step": (I, [D, D, D, D, D, ctypes.c_int64]),
        "ratel_offload_grad_chunk": (I, [I, P]),
        "ratel_sync": (I, [P]),
        "ratel_block_wait": (I, [I, P]),
        "ratel_refresh_params": (I, [I, P]),
        "ratel_register_peer_params": (I, [I, I, ctypes.POINTER(P), I]),
        "ratel_register_peer_grads": (I, [I, I, ctypes.POINTER(P), I, D]),
        "ratel_register_ssd": (I, [I, I, I, U64]),
        "ratel_ssd_range_bytes": (U64, [U64, I, I]),
        "ratel_finalize": (I, []),
        "ratel_last_error": (ctypes.c_char_p, []),
        "ratel_padded_numel": (U64, [U64, I]),
        "ratel_rank_slice": (I, [U64, I, I, ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "ratel_optimizer_stream": (P, []),
        "ratel_get_grad_sumsq": (I, [ctypes.POINTER(D)]),
        "ratel_kernel_timing": (I, [ctypes.POINTER(D), ctypes.POINTER(ctypes.c_int64), I]),
        "ratel_launch_count": (ctypes.c_int64, []),
        "ratel_alloc_pinned": (I, [U64, ctypes.POINTER(P)]),
        "ratel_free_pinned": (I, [P]),
        "ratel_gen_stream_key": (U64, [U64, U64, U64, U64]),
        "ratel_gen_theta0": (I, [P, U64, U64, U64, P]),
        "ratel_gen_grad16": (I, [P, U64, U64, U64, P]),
        "ratel_test_bf16_rne": (I, [P, P, U64, P]),
        "ratel_test_fill_f32": (I, [P, U64, ctypes.c_float, P]),
        "ratel_swap_iter_time": (I, [ctypes.POINTER(ratel_swap_model), D, D, ctypes.POINTER(D),
                                     ctypes.POINTER(D)]),
        "ratel_swap_recompute_flop": (I, [ctypes.POINTER(ratel_swap_layer), I, D, D, ctypes.POINTER(D)]),
        "ratel_plan_activation_swap": (I, [ctypes.POINTER(ratel_swap_layer), I, ctypes.POINTER(ratel_swap_model),
                                           D, ctypes.POINTER(I), ctypes.POINTER(ratel_swap_plan)]),
    }
    for name, (res, args) in sig.items():
        if not strict and not hasattr(lib, name):
            continue   # an older build variant (tools/ only)
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


# RATEL_LIB lets tools load a build variant (tools/k1_sweep.py builds them);
# it must name an existing libratel build -- there is no fallback either way.
LIB_PATH = os.environ.get("RATEL_LIB", _LIB_PATH)
_lib = load_library(LIB_PATH)


def lib():
    return _lib


def _check(rc: int) -> None:
    if rc != RATEL_OK:
        raise RatelError(rc, (_lib.ratel_last_error() or b"").decode(errors="replace"))


CUDA_STREAM_LEGACY = 0x1   # cudaStreamLegacy


def _stream(s):
    """None -> NULL (ratel_sync: block the host); a torch stream -> its
    handle, torch's legacy default stream (handle 0) -> cudaStreamLegacy so
    that ratel_sync(torch.cuda.current_stream()) stays stream-ordered there
    too instead of turning into the host-blocking NULL form."""
    if s is None:
        return None
    if hasattr(s, "cuda_stream"):
        h = s.cuda_stream
        return h if h != 0 else CUDA_STREAM_LEGACY
    return int(s)


# --------------------------------------------------------------------- ABI
def ratel_default_config() -> ratel_config:
    c = ratel_config()
    _lib.ratel_default_config(ctypes.byref(c))
    return c


def ratel_get_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.ratel_get_nccl_unique_id(buf))
    return buf.raw


def ratel_init(device: int, rank: int = 0, world_size: int = 1, nccl_unique_id: bytes | None = None,
               cfg: ratel_config | None = None) -> None:
    uid = None
    if nccl_unique_id is not None:
        assert len(nccl_unique_id) == 128
        uid = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
    _check(_lib.ratel_init(device, rank, world_size, uid, ctypes.byref(cfg) if cfg is not None else None))


def ratel_register_block(block_id: int, ranges, residency: int = RATEL_DEVICE) -> None:
    arr = (ratel_range * len(ranges))(*ranges)
    _check(_lib.ratel_register_block(block_id, arr, len(ranges), residency))


def ratel_register_peer_params(block_id: int, range_idx: int, peer_params) -> None:
    """peer_params: one pointer (int, tensor or None) per rank."""
    ptrs = [(p.data_ptr() if hasattr(p, "data_ptr") else (int(p) if p else None)) for p in peer_params]
    arr = (ctypes.c_void_p * len(ptrs))(*ptrs)
    _check(_lib.ratel_register_peer_params(block_id, range_idx, arr, len(ptrs)))


def ratel_register_peer_grads(block_id: int, range_idx: int, rank_grads, grad_scale: float) -> None:
    """rank_grads: every rank's full-range G16 of the range (int, tensor or
    None for this rank), rank order; grad_scale 1/N = data-parallel mean."""
    ptrs = [(p.data_ptr() if hasattr(p, "data_ptr") else (int(p) if p else None)) for p in rank_grads]
    arr = (ctypes.c_void_p * len(ptrs))(*ptrs)
    _check(_lib.ratel_register_peer_grads(block_id, range_idx, arr, len(ptrs), grad_scale))


def ratel_register_ssd(block_id: int, range_idx: int, fd: int, offset: int) -> None:
    """RATEL_SSD block: the range's theta/m/v live in file `fd` at `offset`
    (layout: ratel_ssd_range_bytes)."""
    _check(_lib.ratel_register_ssd(block_id, range_idx, fd, offset))


def ratel_ssd_range_bytes(numel: int, world_size: int = 1, rank: int = 0) -> int:
    return int(_lib.ratel_ssd_range_bytes(numel, world_size, rank))


# ---------------------------------------------------------------- swap planner
# include/ratel_plan.h (§IV-D, Eq. 1-8, Algorithm 1): host-only.
def _swap_layers(layers):
    """layers: iterable of (act_bytes, recompute_flop) pairs."""
    layers = list(layers)
    arr = (ratel_swap_layer * max(len(layers), 1))()
    for i, (a, f) in enumerate(layers):
        arr[i].act_bytes, arr[i].recompute_flop = float(a), float(f)
    return arr, len(layers)


def ratel_swap_iter_time(model: ratel_swap_model, a_g2m: float, flop_r: float):
    """Eq. 4 / Eq. 5 -> (T_f, T_b) in seconds."""
    tf, tb = ctypes.c_double(), ctypes.c_double()
    _check(_lib.ratel_swap_iter_time(ctypes.byref(model), a_g2m, flop_r, ctypes.byref(tf), ctypes.byref(tb)))
    return tf.value, tb.value


def ratel_swap_recompute_flop(layers, flop_f: float, a_g2m: float) -> float:
    """Eq. 7: FLOP_r after swapping a_g2m bytes along the OB order."""
    arr, n = _swap_layers(layers)
    out = ctypes.c_double()
    _check(_lib.ratel_swap_recompute_flop(arr, n, flop_f, a_g2m, ctypes.byref(out)))
    return out.value


def ratel_plan_activation_swap(layers, model: ratel_swap_model, a_inter_block: float):
    """Algorithm 1 -> (swapped layer indices in OB order, full OB order, plan)."""
    arr, n = _swap_layers(layers)
    order = (ctypes.c_int * max(n, 1))()
    plan = ratel_swap_plan()
    _check(_lib.ratel_plan_activation_swap(arr, n, ctypes.byref(model), a_inter_block, order, ctypes.byref(plan)))
    full = list(order)[:n]
    return full[:plan.n_swap], full, plan


def ratel_adam_step(lr: float, beta1: float, beta2: float, eps: float, weight_decay: float, step: int) -> None:
    _check(_lib.ratel_adam_step(lr, beta1, beta2, eps, weight_decay, step))


def ratel_offload_grad_chunk(block_id: int, stream=None) -> None:
    _check(_lib.ratel_offload_grad_chunk(block_id, _stream(stream)))


def ratel_block_wait(block_id: int, stream=None) -> None:
    _check(_lib.ratel_block_wait(block_id, _stream(stream)))


def ratel_sync(stream=None) -> None:
    _check(_lib.ratel_sync(_stream(stream)))


def ratel_refresh_params(block_id: int, stream=None) -> None:
    _check(_lib.ratel_refresh_params(block_id, _stream(stream)))


def ratel_finalize() -> None:
    _check(_lib.ratel_finalize())


def ratel_last_error() -> str:
    return (_lib.ratel_last_error() or b"").decode(errors="replace")


def ratel_padded_numel(numel: int, world_size: int) -> int:
    return int(_lib.ratel_padded_numel(numel, world_size))


def ratel_rank_slice(numel: int, world_size: int, rank: int) -> tuple[int, int]:
    b, e = ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib.ratel_rank_slice(numel, world_size, rank, ctypes.byref(b), ctypes.byref(e)))
    return int(b.value), int(e.value)


def ratel_optimizer_stream() -> int | None:
    return _lib.ratel_optimizer_stream()


def ratel_get_grad_sumsq() -> float:
    out = ctypes.c_double()
    _check(_lib.ratel_get_grad_sumsq(ctypes.byref(out)))
    return out.value


def ratel_kernel_timing(reset: bool = False) -> tuple[float, int]:
    ms, n = ctypes.c_double(), ctypes.c_int64()
    _check(_lib.ratel_kernel_timing(ctypes.byref(ms), ctypes.byref(n), int(reset)))
    return ms.value, n.value


def ratel_launch_count() -> int:
    return int(_lib.ratel_launch_count())


def ratel_alloc_pinned(nbytes: int) -> int:
    out = ctypes.c_void_p()
    _check(_lib.ratel_alloc_pinned(nbytes, ctypes.byref(out)))
    return int(out.value)


def ratel_free_pinned(ptr: int) -> None:
    _check(_lib.ratel_free_pinned(ptr))


def pinned_tensor(nfloats: int):
    """An fp32 CPU tensor over exact-size page-locked memory from
    ratel_alloc_pinned (freed when the returned owner is collected)."""
    import numpy as np
    import torch

    class _Owner:
        def __init__(self, n):
            self.ptr = ratel_alloc_pinned(n * 4)
            buf = (ctypes.c_float * n).from_address(self.ptr)
            self.tensor = torch.from_numpy(np.ctypeslib.as_array(buf))

        def __del__(self):
            if getattr(self, "ptr", 0):
                ratel_free_pinned(self.ptr)
                self.ptr = 0
    return _Owner(nfloats)


# -------------------------------------------------- include/ratel_gen.h
def ratel_gen_stream_key(seed: int, tag: int, step: int, block: int) -> int:
    return int(_lib.ratel_gen_stream_key(seed, tag, step, block))


def ratel_gen_theta0(dst_ptr: int, n: int, start: int, key: int, stream=None) -> None:
    _check(_lib.ratel_gen_theta0(dst_ptr, n, start, key, _stream(stream)))


def ratel_gen_grad16(dst_ptr: int, n: int, start: int, key: int, stream=None) -> None:
    _check(_lib.ratel_gen_grad16(dst_ptr, n, start, key, _stream(stream)))


def ratel_test_bf16_rne(in_ptr: int, out_ptr: int, n: int, stream=None) -> None:
    _check(_lib.ratel_test_bf16_rne(in_ptr, out_ptr, n, _stream(stream)))


def ratel_test_fill_f32(dst_ptr: int, n: int, value: float, stream=None) -> None:
    _check(_lib.ratel_test_fill_f32(dst_ptr, n, value, _stream(stream)))


def make_range(param, grad, master, exp_avg, exp_avg_sq, numel: int, apply_weight_decay: int = 1,
               grad_is_rank_slice: int = 0) -> ratel_range:
    """Build a ratel_range from tensors (or raw integer pointers)."""
    def p(x):
        if x is None:
            return None
        return x.data_ptr() if hasattr(x, "data_ptr") else int(x)
    return ratel_range(p(param), p(grad), grad_is_rank_slice, p(master), p(exp_avg), p(exp_avg_sq),
                       numel, apply_weight_decay)
