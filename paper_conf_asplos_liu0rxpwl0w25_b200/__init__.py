"""comet-b200: the W4Ax hot path of COMET (ASPLOS'25) on B200 (sm_100a).

Thin ctypes binding over ``lib/libcomet.so`` (C ABI in ``include/comet.h``).  Every step of
the path runs in the library's CUDA kernels; this module only marshals torch tensors
(device memory, streams) into the C calls and raises on error.  There is no CPU fallback:
if the library is missing, importing the binding raises.

Names follow the C ABI:  quantize_act, pack_weight, Plan (comet_plan_create),
w4ax_gemm, w4ax_linear_host.
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "lib", "libcomet.so")
HEADER_PATH = os.path.join(os.path.dirname(_PKG), "include", "comet.h")

COMET_F16, COMET_BF16, COMET_F32 = 0, 1, 2
BLOCK_K = 128
TILE_W = 128
SCALE_PAD = 16


class CometError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {0: "COMET_OK", 1: "COMET_ERR_INVALID_ARG", 2: "COMET_ERR_UNSUPPORTED_SHAPE",
           3: "COMET_ERR_MISALIGNED", 4: "COMET_ERR_NOT_SM100A", 5: "COMET_ERR_WORKSPACE_TOO_SMALL",
           6: "COMET_ERR_CUDA"}


class ActLayout(ctypes.Structure):
    _fields_ = [("codes_off", ctypes.c_size_t), ("qsum_off", ctypes.c_size_t),
                ("corr_off", ctypes.c_size_t), ("total_bytes", ctypes.c_size_t),
                ("Mp", ctypes.c_int64), ("nb", ctypes.c_int64)]


class SchedConfig(ctypes.Structure):
    _fields_ = [("tile_n", ctypes.c_int), ("num_sms", ctypes.c_int), ("split_mode", ctypes.c_int),
                ("cost_int4", ctypes.c_float), ("cost_int8", ctypes.c_float),
                ("stages", ctypes.c_int), ("device_plan", ctypes.c_int),
                ("orientation", ctypes.c_int), ("tile_w", ctypes.c_int),
                ("reserved", ctypes.c_int * 4)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int64), ("N", ctypes.c_int64), ("K", ctypes.c_int64),
                ("tile_n", ctypes.c_int), ("num_ctas", ctypes.c_int), ("split_mode", ctypes.c_int),
                ("stages", ctypes.c_int), ("orientation", ctypes.c_int), ("tile_w", ctypes.c_int),
                ("n_tiles", ctypes.c_int64), ("n_items", ctypes.c_int64),
                ("n_split_tiles", ctypes.c_int64), ("max_cta_cost", ctypes.c_double),
                ("mean_cta_cost", ctypes.c_double)]


_lib = None


def lib():
    """Load libcomet.so (built in-tree by build.build()).  Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_asplos_liu0rxpwl0w25_b200.build`"
                          " (there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, I64, I32, SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
    sig = {
        "comet_act_layout": (I32, [I64, I64, ctypes.POINTER(ActLayout)]),
        "comet_act_packed_bytes": (SZ, [I64, I64]),
        "comet_act_scales_count": (SZ, [I64, I64]),
        "comet_quantize_act": (I32, [P, I32, I64, I64, I64, P, P, P, P, P]),
        "comet_weight_packed_bytes": (SZ, [I64, I64]),
        "comet_pack_weight": (I32, [P, I64, I64, P, P]),
        "comet_pack_weight_perm": (I32, [P, I64, I64, P, P, P]),
        "comet_channel_amax": (I32, [P, I32, I64, I64, I64, P, P]),
        "comet_calibrate_perm": (I32, [P, I64, ctypes.c_double, P, P, ctypes.POINTER(I64)]),
        "comet_kv4_quantize": (I32, [P, I32, I64, I64, I64, I32, P, P, P, P]),
        "comet_kv4_dequantize": (I32, [P, P, P, I64, I64, I32, P, I32, I64, P]),
        "comet_sched_config_default": (None, [ctypes.POINTER(SchedConfig)]),
        "comet_plan_create": (I32, [I64, I64, I64, P, ctypes.POINTER(SchedConfig), ctypes.POINTER(P),
                                    ctypes.POINTER(SZ)]),
        "comet_plan_destroy": (I32, [P]),
        "comet_plan_info": (I32, [P, ctypes.POINTER(PlanInfo)]),
        "comet_plan_describe": (I32, [P, P, I64, ctypes.POINTER(I64)]),
        "comet_w4ax_gemm": (I32, [P, P, P, P, P, P, I32, I64, P, P, P, SZ, P]),
        "comet_w4ax_gemm_grouped": (I32, [P, P, P, P, P, P, I32, I64, P, P, SZ, P]),
        "comet_w4ax_linear": (I32, [P, P, I32, I64, P, P, P, I32, I64, P, SZ, P]),
        "comet_linear_scratch_bytes": (SZ, [P, I32, I32]),
        "comet_w4ax_linear_host": (I32, [P, P, I32, P, P, P, I32, P, SZ, P, SZ, P]),
        "comet_w4ax_linear_host_async": (I32, [P, P, I32, P, P, P, I32, P, SZ, P, SZ, P]),
        "comet_linear_host_wait": (I32, [P]),
        "comet_debug_widen": (I32, [ctypes.c_uint64, I64, I32, P, P]),
        "comet_rs_recv_bytes": (SZ, [I64, I64, I32]),
        "comet_w4ax_gemm_rs": (I32, [P, P, P, P, P, P, I32, I32, P, SZ, P]),
        "comet_rs_reduce": (I32, [P, I32, I32, I64, I64, P, I32, I64, P]),
        "comet_status_string": (ctypes.c_char_p, [I32]),
        "comet_last_error": (ctypes.c_char_p, []),
        "comet_version": (ctypes.c_char_p, []),
        "comet_last_launch_count": (I32, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def declared_symbols() -> list[str]:
    """Function names declared in include/comet.h."""
    with open(HEADER_PATH) as f:
        txt = f.read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(comet_[a-z0-9_]+)\s*\(", txt)))


def _check(st: int):
    if st != 0:
        raise CometError(st, lib().comet_last_error().decode())


def _stream(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dt(t) -> int:
    import torch
    return {torch.float16: COMET_F16, torch.bfloat16: COMET_BF16, torch.float32: COMET_F32}[t]


def _tags_np(tags) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(tags, dtype=np.uint8))


def act_layout(M: int, K: int) -> dict:
    L = ActLayout()
    _check(lib().comet_act_layout(M, K, ctypes.byref(L)))
    return {f: getattr(L, f) for f, _ in ActLayout._fields_}


def last_launch_count() -> int:
    return int(lib().comet_last_launch_count())


def _perm_ptr(perm, K):
    import torch
    if perm is None:
        return None
    assert perm.is_cuda and perm.dtype == torch.int32 and perm.is_contiguous() and perm.numel() == K
    return ctypes.c_void_p(perm.data_ptr())


def quantize_act(x, tags, *, perm=None, out=None, stream=None):
    """FMPQ quantisation (comet_quantize_act).  x: [M, K] float16/bfloat16 CUDA tensor;
    perm: optional [K] int32 CUDA tensor, the fused channel permutation (x'[:, k] = x[:, perm[k]]).
    Returns (act_packed uint8 tensor, act_scales float32 tensor [nb*Mp])."""
    import torch
    assert x.is_cuda and x.dim() == 2 and x.stride(1) == 1
    M, K = x.shape
    t = _tags_np(tags)
    lay = act_layout(M, K)
    if out is None:
        act = torch.empty(lay["total_bytes"], dtype=torch.uint8, device=x.device)
        sc = torch.empty(lay["nb"] * lay["Mp"], dtype=torch.float32, device=x.device)
    else:
        act, sc = out
    _check(lib().comet_quantize_act(ctypes.c_void_p(x.data_ptr()), _dt(x.dtype), M, K, x.stride(0),
                                    t.ctypes.data_as(ctypes.c_void_p), _perm_ptr(perm, K),
                                    ctypes.c_void_p(act.data_ptr()), ctypes.c_void_p(sc.data_ptr()),
                                    _stream(stream)))
    return act, sc


def pack_weight(w_codes, *, perm=None, out=None, stream=None):
    """comet_pack_weight(_perm): [N, K] int8 codes in [-8, 7] -> [N, K/2] packed uint8; with
    perm ([K] int32 CUDA tensor) the columns are permuted first, W'[:, k] = W[:, perm[k]]."""
    import torch
    assert w_codes.is_cuda and w_codes.dtype == torch.int8 and w_codes.is_contiguous()
    N, K = w_codes.shape
    wp = out if out is not None else torch.empty((N, K // 2), dtype=torch.uint8, device=w_codes.device)
    if perm is None:
        _check(lib().comet_pack_weight(ctypes.c_void_p(w_codes.data_ptr()), N, K,
                                       ctypes.c_void_p(wp.data_ptr()), _stream(stream)))
    else:
        _check(lib().comet_pack_weight_perm(ctypes.c_void_p(w_codes.data_ptr()), N, K, _perm_ptr(perm, K),
                                            ctypes.c_void_p(wp.data_ptr()), _stream(stream)))
    return wp


def channel_amax(x, *, out=None, stream=None):
    """comet_channel_amax: per-channel max |x| over the rows of a calibration sample.
    x: [M, K] float16/bfloat16 CUDA tensor -> [K] float32 CUDA tensor."""
    import torch
    assert x.is_cuda and x.dim() == 2 and x.stride(1) == 1
    M, K = x.shape
    a = out if out is not None else torch.empty(K, dtype=torch.float32, device=x.device)
    _check(lib().comet_channel_amax(ctypes.c_void_p(x.data_ptr()), _dt(x.dtype), M, K, x.stride(0),
                                    ctypes.c_void_p(a.data_ptr()), _stream(stream)))
    return a


def calibrate_perm(amax, ratio: float = 10.0):
    """comet_calibrate_perm (host): outlier channels (amax > ratio * median) first.
    amax: [K] float32 (numpy or tensor).  Returns (perm int32 [K], tags uint8 [K/128], n_outliers)."""
    a = np.ascontiguousarray(np.asarray(amax.cpu() if hasattr(amax, "cpu") else amax, dtype=np.float32))
    K = a.shape[0]
    perm = np.empty(K, dtype=np.int32)
    tags = np.empty(max(K // BLOCK_K, 1), dtype=np.uint8)
    n = ctypes.c_int64(0)
    _check(lib().comet_calibrate_perm(a.ctypes.data_as(ctypes.c_void_p), K, float(ratio),
                                      perm.ctypes.data_as(ctypes.c_void_p),
                                      tags.ctypes.data_as(ctypes.c_void_p), ctypes.byref(n)))
    return perm, tags, int(n.value)


def kv4_quantize(kv, group: int = 128, *, out=None, stream=None):
    """comet_kv4_quantize: [T, C] float16/bfloat16 CUDA tensor -> (codes uint8 [T, C/2],
    scales float32 [ceil(T/group), C], mins float32 [ceil(T/group), C])."""
    import torch
    assert kv.is_cuda and kv.dim() == 2 and kv.stride(1) == 1
    T, C = kv.shape
    ng = (T + group - 1) // group
    if out is None:
        out = (torch.empty((T, C // 2), dtype=torch.uint8, device=kv.device),
               torch.empty((ng, C), dtype=torch.float32, device=kv.device),
               torch.empty((ng, C), dtype=torch.float32, device=kv.device))
    codes, scales, mins = out
    _check(lib().comet_kv4_quantize(ctypes.c_void_p(kv.data_ptr()), _dt(kv.dtype), T, C, kv.stride(0), group,
                                    ctypes.c_void_p(codes.data_ptr()), ctypes.c_void_p(scales.data_ptr()),
                                    ctypes.c_void_p(mins.data_ptr()), _stream(stream)))
    return codes, scales, mins


def kv4_dequantize(codes, scales, mins, group: int = 128, *, out=None, out_dtype=None, stream=None):
    """comet_kv4_dequantize: -> [T, C] float16 (default) / bfloat16 CUDA tensor."""
    import torch
    T, C = codes.shape[0], codes.shape[1] * 2
    if out is None:
        out = torch.empty((T, C), dtype=out_dtype or torch.float16, device=codes.device)
    _check(lib().comet_kv4_dequantize(ctypes.c_void_p(codes.data_ptr()), ctypes.c_void_p(scales.data_ptr()),
                                      ctypes.c_void_p(mins.data_ptr()), T, C, group,
                                      ctypes.c_void_p(out.data_ptr()), _dt(out.dtype), out.stride(0),
                                      _stream(stream)))
    return out


class Plan:
    """comet_plan_create: the persistent-CTA tile schedule for one GEMM shape and tag set."""

    def __init__(self, M: int, N: int, K: int, tags, *, tile_n: int = 0, num_sms: int = 0,
                 split_mode: int = -1, cost_int4: float = 1.0, cost_int8: float = 1.0,
                 device_plan: bool = True, orientation: int = 0, tile_w: int = 0):
        L = lib()
        cfg = SchedConfig()
        L.comet_sched_config_default(ctypes.byref(cfg))
        cfg.tile_n, cfg.num_sms, cfg.split_mode = tile_n, num_sms, split_mode
        cfg.cost_int4, cfg.cost_int8 = cost_int4, cost_int8
        cfg.device_plan = 1 if device_plan else 0
        cfg.orientation = orientation
        cfg.tile_w = tile_w
        self.tags = _tags_np(tags)
        h = ctypes.c_void_p()
        ws = ctypes.c_size_t()
        _check(L.comet_plan_create(M, N, K, self.tags.ctypes.data_as(ctypes.c_void_p), ctypes.byref(cfg),
                                   ctypes.byref(h), ctypes.byref(ws)))
        self._h = h
        self.M, self.N, self.K = M, N, K
        self.workspace_bytes = int(ws.value)
        self._ws = None

    @property
    def handle(self):
        return self._h

    def info(self) -> dict:
        i = PlanInfo()
        _check(lib().comet_plan_info(self._h, ctypes.byref(i)))
        return {f: getattr(i, f) for f, _ in PlanInfo._fields_}

    def describe(self) -> np.ndarray:
        """[n_items, 4] int32 rows (cta, tile, kb_begin, kb_end) in execution order."""
        n = ctypes.c_int64()
        _check(lib().comet_plan_describe(self._h, None, 0, ctypes.byref(n)))
        buf = np.zeros((max(1, n.value), 4), dtype=np.int32)
        _check(lib().comet_plan_describe(self._h, buf.ctypes.data_as(ctypes.c_void_p), n.value,
                                         ctypes.byref(n)))
        return buf[: n.value]

    def workspace(self, device="cuda"):
        """Zero-initialised workspace tensor (kept with the plan; one per plan)."""
        import torch
        if self._ws is None:
            self._ws = torch.zeros(max(256, self.workspace_bytes), dtype=torch.uint8, device=device)
        return self._ws

    def close(self):
        if self._h:
            lib().comet_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def w4ax_gemm(plan: Plan, act_packed, act_scales, w_packed, w_scales, *, out=None,
              out_dtype=None, debug: bool = False, debug_blocks: bool = False, stream=None):
    """comet_w4ax_gemm.  Returns y [M, N] (and debug int32 accumulators when requested)."""
    import torch
    dev = act_packed.device
    if out is None:
        out = torch.empty((plan.M, plan.N), dtype=out_dtype or torch.float16, device=dev)
    dacc = torch.empty((plan.M, plan.N), dtype=torch.int32, device=dev) if (debug or debug_blocks) else None
    dblk = (torch.empty((plan.K // BLOCK_K, plan.M, plan.N), dtype=torch.int32, device=dev)
            if debug_blocks else None)
    ws = plan.workspace(dev)
    _check(lib().comet_w4ax_gemm(plan.handle, ctypes.c_void_p(act_packed.data_ptr()),
                                 ctypes.c_void_p(act_scales.data_ptr()),
                                 ctypes.c_void_p(w_packed.data_ptr()),
                                 ctypes.c_void_p(w_scales.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                 _dt(out.dtype), out.stride(0),
                                 ctypes.c_void_p(dacc.data_ptr()) if dacc is not None else None,
                                 ctypes.c_void_p(dblk.data_ptr()) if dblk is not None else None,
                                 ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(stream)))
    if debug_blocks:
        return out, dacc, dblk
    if debug:
        return out, dacc
    return out


def w4ax_linear_fused(plan: Plan, x, w_packed, w_scales, *, out=None, out_dtype=None, stream=None):
    """comet_w4ax_linear: the decode layer with kernel 1 fused into the GEMM, M <= 8, for plans
    with orientation 4 (the warp-level decode kernel; the reduction is a second launch) or
    orientation 1 with 16-token tiles.  x: [M, K] float16 / bfloat16 on the device."""
    import torch
    dev = x.device
    if out is None:
        out = torch.empty((plan.M, plan.N), dtype=out_dtype or torch.float16, device=dev)
    ws = plan.workspace(dev)
    _check(lib().comet_w4ax_linear(plan.handle, ctypes.c_void_p(x.data_ptr()), _dt(x.dtype), x.stride(0),
                                   ctypes.c_void_p(w_packed.data_ptr()), ctypes.c_void_p(w_scales.data_ptr()),
                                   ctypes.c_void_p(out.data_ptr()), _dt(out.dtype), out.stride(0),
                                   ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(stream)))
    return out


def w4ax_gemm_grouped(plan: Plan, act_packed, act_scales, w_packed, w_scales_grouped, *, out=None,
                      out_dtype=None, debug: bool = False, stream=None):
    """comet_w4ax_gemm_grouped (NEXT-3): group-wise weight scales w_scales_grouped [K/128, N]
    float32.  The plan must have orientation 1.  Returns y (and the exact int32 accumulators)."""
    import torch
    dev = act_packed.device
    if out is None:
        out = torch.empty((plan.M, plan.N), dtype=out_dtype or torch.float16, device=dev)
    dacc = torch.empty((plan.M, plan.N), dtype=torch.int32, device=dev) if debug else None
    ws = plan.workspace(dev)
    assert w_scales_grouped.dtype == torch.float32 and w_scales_grouped.is_contiguous()
    _check(lib().comet_w4ax_gemm_grouped(plan.handle, ctypes.c_void_p(act_packed.data_ptr()),
                                         ctypes.c_void_p(act_scales.data_ptr()),
                                         ctypes.c_void_p(w_packed.data_ptr()),
                                         ctypes.c_void_p(w_scales_grouped.data_ptr()),
                                         ctypes.c_void_p(out.data_ptr()), _dt(out.dtype), out.stride(0),
                                         ctypes.c_void_p(dacc.data_ptr()) if dacc is not None else None,
                                         ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(stream)))
    return (out, dacc) if debug else out


def w4ax_linear(plan: Plan, x, w_packed, w_scales, *, perm=None, out=None, out_dtype=None, stream=None):
    """The whole hot path for one linear layer on device tensors: one fused launch
    (comet_w4ax_linear) for decode plans with 16-token tiles, else quantize_act (with the fused
    channel permutation when perm is given; w_packed then packed with the same perm) +
    w4ax_gemm."""
    info = plan.info()
    aligned = x.data_ptr() % 16 == 0 and (x.stride(0) * x.element_size()) % 16 == 0
    if perm is None and info["orientation"] == 4 and aligned:
        # the warp-level decode kernel quantises its own K range: no kernel-1 launch
        return w4ax_linear_fused(plan, x, w_packed, w_scales, out=out, out_dtype=out_dtype, stream=stream)
    if (perm is None and aligned and info["orientation"] == 1 and info["tile_n"] == 16 and plan.M <= 4
            and info["n_tiles"] * -(-plan.K // 512) <= 12 * info["num_ctas"]):
        # the fused launch wins while the CTAs' quantiser warps keep up with the weight stream:
        # small layers (<= 12 pipeline stages per CTA; LLaMA-3-70B qkv at M <= 4: 18.5 ->
        # 16.3-17.0 us per layer step) -- DESIGN.md §7.4
        return w4ax_linear_fused(plan, x, w_packed, w_scales, out=out, out_dtype=out_dtype, stream=stream)
    act, sc = quantize_act(x, plan.tags, perm=perm, stream=stream)
    return w4ax_gemm(plan, act, sc, w_packed, w_scales, out=out, out_dtype=out_dtype, stream=stream)


def debug_widen(first_word: int, n: int, int8_block: bool = False, *, out=None, stream=None):
    """comet_debug_widen: the GEMM kernels' widening of the packed words first_word ..
    first_word + n - 1 (mod 2^32) -> [n, 2] int32 CUDA tensor (lo / hi byte words)."""
    import torch
    if out is None:
        out = torch.empty((n, 2), dtype=torch.int32, device="cuda")
    _check(lib().comet_debug_widen(first_word, n, 1 if int8_block else 0, ctypes.c_void_p(out.data_ptr()),
                                   _stream(stream)))
    return out


def rs_recv_bytes(M: int, N: int, world: int) -> int:
    return int(lib().comet_rs_recv_bytes(M, N, world))


def w4ax_gemm_rs(plan: Plan, act_packed, act_scales, w_packed, w_scales, recv_ptrs, rank: int, *, stream=None):
    """comet_w4ax_gemm_rs (NEXT-2): this rank's row-parallel GEMM with the reduce-scatter fused
    into the epilogue.  recv_ptrs: [world] device addresses (ints) of every rank's receive buffer
    as mapped in this process (comet_rs_recv_bytes bytes each)."""
    world = len(recv_ptrs)
    arr = (ctypes.c_void_p * world)(*[ctypes.c_void_p(int(p)) for p in recv_ptrs])
    ws = plan.workspace(act_packed.device)
    _check(lib().comet_w4ax_gemm_rs(plan.handle, ctypes.c_void_p(act_packed.data_ptr()),
                                    ctypes.c_void_p(act_scales.data_ptr()), ctypes.c_void_p(w_packed.data_ptr()),
                                    ctypes.c_void_p(w_scales.data_ptr()), arr, world, rank,
                                    ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(stream)))


def rs_reduce(recv_local, world: int, rank: int, M: int, N: int, *, out=None, out_dtype=None, stream=None):
    """comet_rs_reduce (NEXT-2): the owner's sum of the world slots of its receive buffer ->
    its rows of Y ([min(ms, M - rank*ms), N], ms = ceil(M / world))."""
    import torch
    ms = -(-M // world)
    rows = max(0, min(ms, M - rank * ms))
    if out is None:
        out = torch.empty((rows, N), dtype=out_dtype or torch.float16, device=recv_local.device)
    _check(lib().comet_rs_reduce(ctypes.c_void_p(recv_local.data_ptr()), world, rank, M, N,
                                 ctypes.c_void_p(out.data_ptr()), _dt(out.dtype), out.stride(0), _stream(stream)))
    return out


def linear_scratch_bytes(plan: Plan, xdt: int, ydt: int) -> int:
    return int(lib().comet_linear_scratch_bytes(plan.handle, xdt, ydt))


def w4ax_linear_host(plan: Plan, x_host, w_packed, w_scales, y_host, scratch, *, stream=None,
                     blocking: bool = True):
    """comet_w4ax_linear_host(_async): host (pinned) x in, host y out; H2D, quantise, GEMM, D2H
    (chunk-pipelined over three streams for M >= 2048).  blocking=False returns at once: y_host
    is complete after linear_host_wait(plan) (or a device synchronize)."""
    ws = plan.workspace(w_packed.device)
    fn = lib().comet_w4ax_linear_host if blocking else lib().comet_w4ax_linear_host_async
    _check(fn(plan.handle, ctypes.c_void_p(x_host.data_ptr()), _dt(x_host.dtype),
              ctypes.c_void_p(w_packed.data_ptr()), ctypes.c_void_p(w_scales.data_ptr()),
              ctypes.c_void_p(y_host.data_ptr()), _dt(y_host.dtype),
              ctypes.c_void_p(scratch.data_ptr()), scratch.numel(),
              ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(stream)))
    return y_host


def linear_host_wait(plan: Plan):
    """comet_linear_host_wait: block until the plan's last host-buffer call has landed in y_host."""
    _check(lib().comet_linear_host_wait(plan.handle))
