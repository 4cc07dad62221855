"""libsat: B200-native (sm_100a) summed-area tables -- Python binding.

Thin ctypes marshalling over ``libsat.so`` (C ABI in ``include/libsat.h``):
every step of the SAT runs in the library's CUDA kernels; torch is used only
for device memory, streams and process groups.  There is no CPU fallback: if
the extension is missing or the device is not a B200 the calls raise.

    S(i, j) = sum_{y <= i} sum_{x <= j} A(y, x)        (Eq. 1)

Type pairs: uint8 -> int32 (wrap mod 2^32), float32 -> float32,
float64 -> float64; also uint8 -> float32 (``out_dtype=torch.float32``, NPP's
8u32f) and int32 -> int32 (wrap mod 2^32).

Entry points: ``sat`` (single / batched), ``sat_exclusive`` (Eq. 2 and the
NPP (H+1) x (W+1) layout), ``sat_band`` (carry-in row), ``sat_host`` (host in,
host out), ``sat_dist`` / ``sat_dist_chained`` (row bands across ranks),
``sat_band_chained`` (one band of a chain), ``rect_sums`` / ``box_filter``
(SAT consumers).
"""
from __future__ import annotations

import ctypes
import os
import threading

__all__ = ["SatError", "Plan", "sat", "sat_host", "sat_exclusive", "sat_band", "SatComm", "sat_dist",
           "sat_dist_chained", "sat_band_chained", "new_chain_buffer", "chain_bytes", "ChainLink",
           "PeerLink", "SatChain", "rect_sums",
           "box_filter", "band_partition", "sat_sq", "integral_histogram", "sat_brlt",
           "PAIR_8U_32S", "PAIR_32F_32F", "PAIR_64F_64F", "PAIR_8U_32F", "PAIR_32S_32S", "lib",
           "LIB_PATH"]

PAIR_8U_32S, PAIR_32F_32F, PAIR_64F_64F, PAIR_8U_32F, PAIR_32S_32S = 0, 1, 2, 3, 4
PAIR_8U_SQ, PAIR_8U_HIST4 = 5, 6  # multi-channel: (S, S of squares) / 4 histogram bins
_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SAT_LIBRARY") or os.path.join(_HERE, "libsat.so")
COMM_ID_BYTES = 128

_lib = None
_lock = threading.Lock()


class SatError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__(f"{where}: {_status_name(status)}: {detail}")


def _status_name(s: int) -> str:
    return lib().sat_status_string(s).decode()


def lib():
    """ctypes handle of libsat.so; raises if the extension was not built."""
    global _lib
    if _lib is None:
        with _lock:
            if _lib is None:
                if not os.path.exists(LIB_PATH):
                    raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build()")
                L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
                i32, i64, vp, sz = ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_size_t
                sigs = {
                    "sat_version": ([], i32),
                    "sat_plan_create": ([ctypes.POINTER(vp), i32, i32, i64, i64, i64], i32),
                    "sat_plan_workspace_bytes": ([vp, ctypes.POINTER(sz)], i32),
                    "sat_plan_destroy": ([vp], i32),
                    "sat_plan_set_timeout": ([vp, ctypes.c_uint64], i32),
                    "sat_plan_status": ([vp, vp], i32),
                    "sat_plan_set_carry": ([vp, i32], i32),
                    "sat_compute": ([vp, vp, vp, i64, i64, i64, i64, i32, vp], i32),
                    "sat_compute_batched": ([vp, vp, vp, i64, i64, i64, i64, i64, i64, i64, i32, vp], i32),
                    "sat_compute_band": ([vp, vp, vp, i64, i64, i64, i64, vp, i32, vp], i32),
                    "sat_compute_host": ([vp, vp, vp, i64, i64, i64, i64, i32, vp], i32),
                    "sat_compute_exclusive": ([vp, vp, vp, i64, i64, i64, i64, i32, vp, i32, vp], i32),
                    "sat_compute_hist4": ([vp, vp, vp, i64, i64, i64, i64, i64, i64, i64, vp, i32, vp], i32),
                    "sat_compute_brlt": ([i32, vp, vp, vp, i64, i64, i64, i64, i64, vp], i32),
                    "sat_rect_sums": ([vp, vp, i64, i64, i64, vp, i64, vp, i32, vp], i32),
                    "sat_chain_bytes": ([i32, i64], sz),
                    "sat_compute_band_chained": ([vp, vp, vp, i64, i64, i64, i64, vp, vp, vp, ctypes.c_uint32, i32, vp], i32),
                    "sat_chain_link_create": ([i32, i32, i64, ctypes.POINTER(vp)], i32),
                    "sat_chain_link_destroy": ([vp], i32),
                    "sat_chain_ipc_handle": ([vp, vp], i32),
                    "sat_chain_open_peer": ([i32, vp, ctypes.POINTER(vp)], i32),
                    "sat_chain_close_peer": ([vp], i32),
                    "sat_compute_dist_chained": ([vp, vp, vp, vp, i64, i64, i64, i64, i32, vp], i32),
                    "sat_box_filter": ([vp, vp, vp, i64, i64, i64, i64, i64, i64, i32, vp], i32),
                    "sat_comm_unique_id": ([vp], i32),
                    "sat_comm_create": ([ctypes.POINTER(vp), vp, i32, i32, i32], i32),
                    "sat_comm_destroy": ([vp], i32),
                    "sat_compute_dist": ([vp, vp, vp, vp, i64, i64, i64, i64, i32, vp], i32),
                    "sat_dist_acc_bytes": ([i32], sz),
                    "sat_dist_colsum": ([vp, vp, i64, i64, i64, vp, vp], i32),
                    "sat_dist_carry": ([vp, vp, i32, i32, i64, vp, vp], i32),
                    "sat_band_partition": ([i64, i32, i32, ctypes.POINTER(i64), ctypes.POINTER(i64)], i32),
                    "sat_status_string": ([i32], ctypes.c_char_p),
                    "sat_last_error": ([], ctypes.c_char_p),
                }
                for name, (args, res) in sigs.items():
                    if not hasattr(L, name) and os.environ.get("SAT_LIBRARY"):
                        continue  # an explicitly chosen older build (same-box A/B tools)
                    f = getattr(L, name)
                    f.argtypes = args
                    f.restype = res
                _lib = L
    return _lib


def _check(status: int, where: str):
    if status != 0:
        raise SatError(status, where, lib().sat_last_error().decode())


def _torch():
    import torch
    return torch


def pair_of_dtype(dtype, out=None) -> int:
    """Type pair of an input dtype; uint8 with a float32 output is 8u->32f."""
    torch = _torch()
    m = {torch.uint8: PAIR_8U_32S, torch.float32: PAIR_32F_32F, torch.float64: PAIR_64F_64F,
         torch.int32: PAIR_32S_32S}
    if dtype not in m:
        raise TypeError(f"unsupported input dtype {dtype}; expected uint8, int32, float32 or float64")
    if dtype == torch.uint8 and out == torch.float32:
        return PAIR_8U_32F
    return m[dtype]


def out_dtype(pair: int):
    torch = _torch()
    return {PAIR_8U_32S: torch.int32, PAIR_32F_32F: torch.float32, PAIR_64F_64F: torch.float64,
            PAIR_8U_32F: torch.float32, PAIR_32S_32S: torch.int32, PAIR_8U_SQ: torch.int32,
            PAIR_8U_HIST4: torch.int32}[pair]


_out_dtype_of = out_dtype  # for functions whose `out_dtype` parameter shadows the helper


def _stream_ptr(stream, device):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return ctypes.c_void_p(s.cuda_stream)


class Plan:
    """A libsat plan: a pair, size limits and the look-back workspace."""

    def __init__(self, pair: int, max_h: int, max_w: int, max_batch: int = 1, device=None):
        torch = _torch()
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.device = dev
        self.pair, self.max_h, self.max_w, self.max_batch = pair, max_h, max_w, max_batch
        h = ctypes.c_void_p()
        _check(lib().sat_plan_create(ctypes.byref(h), dev.index, pair, max_h, max_w, max_batch),
               "sat_plan_create")
        self._h = h

    @property
    def handle(self):
        return self._h

    def workspace_bytes(self) -> int:
        n = ctypes.c_size_t()
        _check(lib().sat_plan_workspace_bytes(self._h, ctypes.byref(n)), "sat_plan_workspace_bytes")
        return n.value

    def set_timeout(self, ns: int):
        """Bound every cross-CTA / cross-GPU carry wait of later launches (ns)."""
        _check(lib().sat_plan_set_timeout(self._h, int(ns)), "sat_plan_set_timeout")

    def set_carry(self, mode: str):
        """Cross-cluster carry of later launches: "auto" (by shape), "lookback"
        or "tree" (integer pairs; see sat_plan_set_carry)."""
        m = {"auto": 0, "lookback": 1, "tree": 2}[mode]
        _check(lib().sat_plan_set_carry(self._h, m), "sat_plan_set_carry")

    def status(self, stream=None):
        """Synchronise `stream`; raise SatError(SAT_ERR_TIMEOUT) if a bounded
        carry wait of an earlier launch ran out (that output is wrong)."""
        _check(lib().sat_plan_status(self._h, _stream_ptr(stream, self.device)), "sat_plan_status")

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            lib().sat_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def fits(self, h, w, batch=1) -> bool:
        return h <= self.max_h and w <= self.max_w and batch <= self.max_batch

    # -- raw pointer calls (sizes in elements, pitches in bytes) ---------------
    def compute_ptr(self, inp: int, out: int, h: int, w: int, in_pitch: int, out_pitch: int,
                    stream=None):
        _check(lib().sat_compute(self._h, inp, out, h, w, in_pitch, out_pitch, self.pair,
                                 _stream_ptr(stream, self.device)), "sat_compute")

    def compute_batched_ptr(self, inp, out, h, w, in_pitch, out_pitch, in_is, out_is, batch,
                            stream=None):
        _check(lib().sat_compute_batched(self._h, inp, out, h, w, in_pitch, out_pitch, in_is,
                                         out_is, batch, self.pair, _stream_ptr(stream, self.device)),
               "sat_compute_batched")

    def compute_band_ptr(self, inp, out, h, w, in_pitch, out_pitch, carry_in, stream=None):
        _check(lib().sat_compute_band(self._h, inp, out, h, w, in_pitch, out_pitch, carry_in,
                                      self.pair, _stream_ptr(stream, self.device)),
               "sat_compute_band")

    def compute_host_ptr(self, inp, out, h, w, in_pitch, out_pitch, stream=None):
        _check(lib().sat_compute_host(self._h, inp, out, h, w, in_pitch, out_pitch, self.pair,
                                      _stream_ptr(stream, self.device)), "sat_compute_host")


_plans: dict = {}


_KNOBS = ("SAT_FORCE_GENERIC", "SAT_CLUSTER", "SAT_SHORT", "SAT_DEEP", "SAT_TREE", "SAT_MAX_CLUSTERS",
          "SAT_FORCE_CLUSTERS", "SAT_LOG")


def _plan_for(device, pair, h, w, batch) -> Plan:
    # libsat reads its tuning knobs once per plan: plans are cached per knob setting
    key = (device.index, pair, tuple(os.environ.get(k) for k in _KNOBS))
    p = _plans.get(key)
    if p is None or not p.fits(h, w, batch):
        if p is not None:
            _torch().cuda.synchronize(device)
            # grow within the same order of magnitude of workspace, else size to the request
            gh, gw, gb = max(h, p.max_h), max(w, p.max_w), max(batch, p.max_batch)
            if gh * gw * gb <= 2 * max(h * w * batch, p.max_h * p.max_w * p.max_batch):
                h, w, batch = gh, gw, gb
            p.close()
        p = Plan(pair, h, w, batch, device)
        _plans[key] = p
    return p


def _row_layout(t):
    if t.dim() not in (2, 3):
        raise ValueError("expected a [H, W] or [N, H, W] tensor")
    if t.stride(-1) != 1:
        raise ValueError("the last dimension must be contiguous (stride 1)")
    es = t.element_size()
    H, W = t.shape[-2], t.shape[-1]
    pitch = t.stride(-2) * es if H > 1 else max(W * es, t.stride(-2) * es)
    img = t.stride(0) * es if t.dim() == 3 else H * pitch
    return pitch, img


def sat(x, out=None, plan: Plan | None = None, stream=None, out_dtype=None):
    """Inclusive SAT of a CUDA tensor [H, W] or [N, H, W] (uint8/float32/float64).

    Returns ``out`` (allocated if None: int32 / float32 / float64).  A uint8
    input with out_dtype (or out) float32 selects the 8u->32f pair."""
    torch = _torch()
    if not x.is_cuda:
        raise ValueError("sat() needs a CUDA tensor (use sat_host for host arrays)")
    pair = pair_of_dtype(x.dtype, out.dtype if out is not None else out_dtype)
    if out is None:
        out = torch.empty(x.shape, dtype=_out_dtype_of(pair), device=x.device)
    elif out.dtype != _out_dtype_of(pair) or out.shape != x.shape or out.device != x.device:
        raise ValueError("out has the wrong dtype/shape/device")
    H, W = x.shape[-2], x.shape[-1]
    N = x.shape[0] if x.dim() == 3 else 1
    if H == 0 or W == 0 or N == 0:
        return out
    ip, iis = _row_layout(x)
    op, ois = _row_layout(out)
    p = plan if plan is not None else _plan_for(x.device, pair, H, W, N)
    if x.dim() == 3 and N > 1:
        p.compute_batched_ptr(x.data_ptr(), out.data_ptr(), H, W, ip, op, iis, ois, N, stream)
    else:
        p.compute_ptr(x.data_ptr(), out.data_ptr(), H, W, ip, op, stream)
    return out


def sat_exclusive(x, full: bool = True, nval=0, out=None, plan: Plan | None = None, stream=None,
                  out_dtype=None):
    """Exclusive SAT (Eq. 2) of a CUDA tensor [H, W] plus nVal on every
    element: full=True gives NPP's / OpenCV's (H+1) x (W+1) layout, full=False
    Eq. 2's H x W.  sat_compute_exclusive does all the work."""
    torch = _torch()
    if not x.is_cuda or x.dim() != 2:
        raise ValueError("sat_exclusive() needs a 2-D CUDA tensor")
    pair = pair_of_dtype(x.dtype, out.dtype if out is not None else out_dtype)
    H, W = x.shape
    shape = (H + 1, W + 1) if full else (H, W)
    if out is None:
        # rows padded to 16 bytes (a view), so the kernel's shifted stores stay vectorised
        per16 = 16 // torch.empty((), dtype=_out_dtype_of(pair)).element_size()
        cols = -(-max(shape[1], 1) // per16) * per16
        out = torch.empty((shape[0], cols), dtype=_out_dtype_of(pair), device=x.device)[:, :shape[1]]
    elif out.dtype != _out_dtype_of(pair) or tuple(out.shape) != shape or out.device != x.device:
        raise ValueError("out has the wrong dtype/shape/device")
    if out.numel() == 0:
        return out
    ctype = {0: ctypes.c_int32, 1: ctypes.c_float, 2: ctypes.c_double, 3: ctypes.c_float,
             4: ctypes.c_int32}[pair]
    nv = ctype(nval)
    ip = _row_layout(x)[0] if H > 0 and W > 0 else max(W, 1) * x.element_size()
    op = _row_layout(out)[0]
    p = plan if plan is not None else _plan_for(x.device, pair, max(H, 1), max(W, 1), 1)
    _check(lib().sat_compute_exclusive(p.handle, x.data_ptr() if x.numel() else None,
                                       out.data_ptr(), H, W, ip, op, 1 if full else 0,
                                       ctypes.byref(nv), pair, _stream_ptr(stream, x.device)),
           "sat_compute_exclusive")
    return out


def sat_sq(x, out=None, plan: Plan | None = None, stream=None):
    """SAT and SAT of squares of a uint8 CUDA image [H, W] or batch [N, H, W]
    in ONE pass (Viola-Jones variance normalisation, PAPER.md:18-24 [2]):
    returns int32 [..., H, W, 2] = (S, Q), both exact mod 2^32."""
    torch = _torch()
    if x.dtype != torch.uint8 or not x.is_cuda:
        raise ValueError("sat_sq() takes a uint8 CUDA tensor")
    if out is None:
        out = torch.empty((*x.shape, 2), dtype=torch.int32, device=x.device)
    if out.dtype != torch.int32 or tuple(out.shape) != (*x.shape, 2) or out.stride(-1) != 1 \
            or out.stride(-2) != 2:
        raise ValueError("out must be int32 [..., H, W, 2] with contiguous (S, Q) pairs")
    H, W = x.shape[-2], x.shape[-1]
    N = x.shape[0] if x.dim() == 3 else 1
    if H == 0 or W == 0 or N == 0:
        return out
    ip, iis = _row_layout(x)
    op, ois = out.stride(-3) * 4, (out.stride(0) * 4 if x.dim() == 3 else H * out.stride(-3) * 4)
    p = plan if plan is not None else _plan_for(x.device, PAIR_8U_SQ, H, W, N)
    p.compute_batched_ptr(x.data_ptr(), out.data_ptr(), H, W, ip, op, iis if N > 1 else H * ip,
                          ois, N, stream)
    return out


def integral_histogram(x, bins=16, bin_of=None, out=None, plan: Plan | None = None, stream=None):
    """Integral histogram of a uint8 CUDA image [H, W] ([34], [38]):
    K = `bins` bins, value v in bin bin_of[v] (default: K equal-width bins,
    bin_of[v] = v * K // 256).  Returns int32 [ceil(K/4), H, W, 4]: bin
    4 * g + c is out[g, ..., c] (interleaved 4-bin groups; one single-pass
    launch per group)."""
    import numpy as np
    torch = _torch()
    if x.dtype != torch.uint8 or not x.is_cuda or x.dim() != 2:
        raise ValueError("integral_histogram() takes a 2-D uint8 CUDA tensor")
    table = (np.arange(256) * bins // 256) if bin_of is None else np.asarray(bin_of)
    if table.shape != (256,) or table.min() < 0 or table.max() > 255:
        raise ValueError("bin_of must be 256 bin indices in [0, 255]")
    lut = (ctypes.c_uint8 * 256)(*[int(v) for v in table])
    ngroups = (bins + 3) // 4
    H, W = x.shape
    if out is None:
        out = torch.empty((ngroups, H, W, 4), dtype=torch.int32, device=x.device)
    if H == 0 or W == 0:
        return out
    ip = _row_layout(x)[0]
    p = plan if plan is not None else _plan_for(x.device, PAIR_8U_HIST4, H, W, 1)
    for g in range(ngroups):
        o = out[g]
        _check(lib().sat_compute_hist4(p.handle, x.data_ptr(), o.data_ptr(), H, W, ip,
                                       o.stride(0) * 4, H * ip, H * o.stride(0) * 4, 1, lut, 4 * g,
                                       _stream_ptr(stream, x.device)), "sat_compute_hist4")
    return out


def sat_brlt(x, out=None, tmp=None, stream=None):
    """ABLATION (not the product path): the paper's two-pass BRLT-ScanRow x 2
    (Sec. IV-B) for uint8 / float32 / float64 [H, W] CUDA tensors;
    tmp is the [W, H] intermediate (allocated if None)."""
    torch = _torch()
    pair = pair_of_dtype(x.dtype)
    H, W = x.shape
    if out is None:
        out = torch.empty((H, W), dtype=out_dtype(pair), device=x.device)
    if tmp is None:
        tmp = torch.empty((W, H), dtype=out_dtype(pair), device=x.device)
    _check(lib().sat_compute_brlt(pair, x.data_ptr(), out.data_ptr(), tmp.data_ptr(), H, W,
                                  _row_layout(x)[0], _row_layout(out)[0], _row_layout(tmp)[0],
                                  _stream_ptr(stream, x.device)), "sat_compute_brlt")
    return out


def rect_sums(S, rects, plan: Plan | None = None, stream=None):
    """Sums of A over half-open rectangles [y0, y1) x [x0, x1) from its inclusive
    SAT S (a CUDA tensor as returned by sat(), or by sat_sq() / one group of
    integral_histogram() -- [H, W, K] -> [n, K] results); rects: int32 CUDA
    tensor [n, 4] of (y0, x0, y1, x1), clamped to the image."""
    torch = _torch()
    if S.dim() == 3:  # multi-channel SAT [H, W, K]
        pair = {2: PAIR_8U_SQ, 4: PAIR_8U_HIST4}[S.shape[2]]
        H, W = S.shape[0], S.shape[1]
        oshape = lambda n: (n, S.shape[2])
    else:
        pair = {torch.int32: 0, torch.float32: 1, torch.float64: 2}[S.dtype]
        H, W = S.shape
        oshape = lambda n: (n,)
    rects = rects.to(device=S.device, dtype=torch.int32).contiguous()
    if rects.dim() != 2 or rects.shape[1] != 4:
        raise ValueError("rects must be [n, 4]")
    out = torch.empty(oshape(rects.shape[0]), dtype=S.dtype, device=S.device)
    if rects.shape[0] == 0:
        return out
    if S.dim() == 3:
        if S.stride(2) != 1 or S.stride(1) != S.shape[2]:
            raise ValueError("a multi-channel SAT must have contiguous [W, K] rows")
        sp = S.stride(0) * 4 if H > 0 and W > 0 else max(W, 1) * S.shape[2] * 4
    else:
        sp = _row_layout(S)[0] if H > 0 and W > 0 else max(W, 1) * S.element_size()
    p = plan if plan is not None else _plan_for(S.device, pair, max(H, 1), max(W, 1), 1)
    _check(lib().sat_rect_sums(p.handle, S.data_ptr() if S.numel() else None, H, W, sp,
                               rects.data_ptr(), rects.shape[0], out.data_ptr(), pair,
                               _stream_ptr(stream, S.device)), "sat_rect_sums")
    return out


def box_filter(S, ry: int, rx: int, out=None, plan: Plan | None = None, stream=None):
    """Box sums of radius (ry, rx), clipped at the borders, from the inclusive SAT S."""
    torch = _torch()
    pair = {torch.int32: 0, torch.float32: 1, torch.float64: 2}[S.dtype]
    H, W = S.shape
    if out is None:
        out = torch.empty((H, W), dtype=S.dtype, device=S.device)
    if H == 0 or W == 0:
        return out
    p = plan if plan is not None else _plan_for(S.device, pair, H, W, 1)
    _check(lib().sat_box_filter(p.handle, S.data_ptr(), out.data_ptr(), H, W, _row_layout(S)[0],
                                _row_layout(out)[0], ry, rx, pair, _stream_ptr(stream, S.device)),
           "sat_box_filter")
    return out


def sat_band(x, carry_in=None, out=None, plan: Plan | None = None, stream=None, out_dtype=None):
    """SAT of a row band given the SAT row above it (carry_in: [W] of the output dtype)."""
    torch = _torch()
    pair = pair_of_dtype(x.dtype, out.dtype if out is not None else out_dtype)
    if out is None:
        out = torch.empty(x.shape, dtype=_out_dtype_of(pair), device=x.device)
    H, W = x.shape
    if H == 0 or W == 0:
        return out
    ip, _ = _row_layout(x)
    op, _ = _row_layout(out)
    cptr = None
    if carry_in is not None:
        if carry_in.dtype != _out_dtype_of(pair) or carry_in.numel() < W or not carry_in.is_contiguous():
            raise ValueError("carry_in must be a contiguous [W] tensor of the output dtype")
        cptr = carry_in.data_ptr()
    p = plan if plan is not None else _plan_for(x.device, pair, H, W, 1)
    p.compute_band_ptr(x.data_ptr(), out.data_ptr(), H, W, ip, op, cptr, stream)
    return out


def sat_host(x, out=None, plan: Plan | None = None, device=None, stream=None):
    """End-to-end SAT of a HOST (CPU, ideally pinned) tensor into a host tensor.

    Streams row bands through the GPU (H2D, SAT with carry-in, D2H overlapped);
    returns after synchronising the stream."""
    torch = _torch()
    if x.is_cuda:
        raise ValueError("sat_host() takes a host tensor")
    pair = pair_of_dtype(x.dtype, out.dtype if out is not None else None)
    if out is None:
        out = torch.empty(x.shape, dtype=out_dtype(pair), pin_memory=x.is_pinned())
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    H, W = x.shape
    if H == 0 or W == 0:
        return out
    ip, _ = _row_layout(x)
    op, _ = _row_layout(out)
    p = plan if plan is not None else _plan_for(dev, pair, H, W, 1)
    s = stream if stream is not None else torch.cuda.current_stream(dev)
    p.compute_host_ptr(x.data_ptr(), out.data_ptr(), H, W, ip, op, s)
    s.synchronize()
    return out


# ---------------------------------------------------------------------------
# Multi-GPU

def band_partition(H: int, nranks: int, rank: int):
    """Rows [r0, r1) of rank `rank` (libsat's sat_band_partition, reading R14:
    the first H mod P ranks get one extra row)."""
    r0, r1 = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().sat_band_partition(H, nranks, rank, ctypes.byref(r0), ctypes.byref(r1)),
           "sat_band_partition")
    return r0.value, r1.value


class SatComm:
    """NCCL communicator for sat_dist, bootstrapped over a torch process group."""

    def __init__(self, group=None, device=None):
        torch = _torch()
        import torch.distributed as dist

        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.device = dev
        buf = (ctypes.c_uint8 * COMM_ID_BYTES)()
        if self.rank == 0:
            _check(lib().sat_comm_unique_id(buf), "sat_comm_unique_id")
        t = torch.tensor(list(bytes(buf)), dtype=torch.uint8)
        if dist.get_backend(group) == "nccl":
            t = t.to(dev)
        dist.broadcast(t, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
        raw = bytes(t.cpu().tolist())
        idbuf = (ctypes.c_uint8 * COMM_ID_BYTES).from_buffer_copy(raw)
        h = ctypes.c_void_p()
        _check(lib().sat_comm_create(ctypes.byref(h), idbuf, self.nranks, self.rank, dev.index),
               "sat_comm_create")
        self._h = h

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            lib().sat_comm_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def sat_dist(band, comm: SatComm, out=None, plan: Plan | None = None, stream=None):
    """Row-banded SAT: `band` holds this rank's rows of one image (ranks in order)."""
    torch = _torch()
    pair = pair_of_dtype(band.dtype, out.dtype if out is not None else None)
    if out is None:
        out = torch.empty(band.shape, dtype=out_dtype(pair), device=band.device)
    H, W = band.shape
    ip, _ = _row_layout(band) if H > 0 else (W * band.element_size(), 0)
    op, _ = _row_layout(out) if H > 0 else (W * out.element_size(), 0)
    p = plan if plan is not None else _plan_for(band.device, pair, max(H, 1), W, 1)
    _check(lib().sat_compute_dist(p.handle, comm._h, band.data_ptr() if H else None,
                                  out.data_ptr() if H else None, H, W, ip, op, pair,
                                  _stream_ptr(stream, band.device)), "sat_compute_dist")
    return out


def dist_colsum(band, plan: Plan | None = None, stream=None, pair=None):
    """Step 1 of sat_dist: the band's column totals (uint32 or float64 [W])."""
    torch = _torch()
    pair = pair_of_dtype(band.dtype) if pair is None else pair
    H, W = band.shape
    acc = torch.empty(W, dtype=torch.int32 if pair in (PAIR_8U_32S, PAIR_32S_32S) else torch.float64, device=band.device)
    ip = band.stride(0) * band.element_size() if H > 1 else W * band.element_size()
    p = plan if plan is not None else _plan_for(band.device, pair, max(H, 1), W, 1)
    _check(lib().sat_dist_colsum(p.handle, band.data_ptr() if H else None, H, W, ip,
                                 acc.data_ptr(), _stream_ptr(stream, band.device)), "sat_dist_colsum")
    return acc


def dist_carry(gathered, rank: int, pair: int, plan: Plan | None = None, stream=None):
    """Step 3 of sat_dist: carry row S(r0-1, .) for `rank` from the [P, W] gathered totals."""
    torch = _torch()
    P, W = gathered.shape
    carry = torch.empty(W, dtype=out_dtype(pair), device=gathered.device)
    p = plan if plan is not None else _plan_for(gathered.device, pair, 1, W, 1)
    _check(lib().sat_dist_carry(p.handle, gathered.contiguous().data_ptr(), P, rank, W,
                                carry.data_ptr(), _stream_ptr(stream, gathered.device)),
           "sat_dist_carry")
    return carry


# ---------------------------------------------------------------------------
# Chained row bands (single-pass multi-GPU path)

IPC_HANDLE_BYTES = 64


def chain_bytes(pair: int, w: int) -> int:
    """Bytes of one chain link (ack words + two receive slots) for width w."""
    return int(lib().sat_chain_bytes(pair, w))


def new_chain_buffer(pair: int, w: int, device=None):
    """A zero-filled chain link as a uint8 CUDA tensor (single-process chains;
    torch allocations are 512-byte aligned)."""
    torch = _torch()
    return torch.zeros(chain_bytes(pair, w), dtype=torch.uint8, device=device or "cuda")


class ChainLink:
    """A chain link allocated by libsat (cudaMalloc, zeroed): exportable over CUDA IPC."""

    def __init__(self, pair: int, w: int, device=None):
        torch = _torch()
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        h = ctypes.c_void_p()
        _check(lib().sat_chain_link_create(dev.index, pair, w, ctypes.byref(h)), "sat_chain_link_create")
        self.ptr, self.device = h.value, dev

    def ipc_handle(self) -> bytes:
        buf = (ctypes.c_uint8 * IPC_HANDLE_BYTES)()
        _check(lib().sat_chain_ipc_handle(self.ptr, buf), "sat_chain_ipc_handle")
        return bytes(buf)

    def close(self):
        if getattr(self, "ptr", None):
            lib().sat_chain_link_destroy(self.ptr)
            self.ptr = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class PeerLink:
    """Another process's chain link mapped into this one (CUDA IPC)."""

    def __init__(self, handle: bytes, device=None):
        torch = _torch()
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        buf = (ctypes.c_uint8 * IPC_HANDLE_BYTES).from_buffer_copy(handle)
        h = ctypes.c_void_p()
        _check(lib().sat_chain_open_peer(dev.index, buf, ctypes.byref(h)), "sat_chain_open_peer")
        self.ptr = h.value

    def close(self):
        if getattr(self, "ptr", None):
            lib().sat_chain_close_peer(self.ptr)
            self.ptr = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _link_ptr(link):
    if link is None:
        return None
    if isinstance(link, int):
        return link
    if hasattr(link, "data_ptr"):
        return link.data_ptr()
    return link.ptr


def sat_band_chained(x, link_self, link_above, link_below, epoch: int, out=None,
                     plan: Plan | None = None, stream=None):
    """SAT of one band of a chain: its carry-in row arrives (in the kernel)
    through link_self from the band above, its bottom row goes to link_below;
    links are tensors from new_chain_buffer, ChainLink / PeerLink objects or
    raw device pointers (None: no such neighbour)."""
    torch = _torch()
    pair = pair_of_dtype(x.dtype, out.dtype if out is not None else None)
    H, W = x.shape
    if out is None:
        out = torch.empty(x.shape, dtype=out_dtype(pair), device=x.device)
    p = plan if plan is not None else _plan_for(x.device, pair, H, W, 1)
    _check(lib().sat_compute_band_chained(
        p.handle, x.data_ptr(), out.data_ptr(), H, W, _row_layout(x)[0], _row_layout(out)[0],
        _link_ptr(link_self), _link_ptr(link_above), _link_ptr(link_below), epoch, pair,
        _stream_ptr(stream, x.device)), "sat_compute_band_chained")
    return out


class SatChain:
    """Chained row bands across the ranks of a torch process group (any
    backend): each rank owns a ChainLink; the links' CUDA IPC handles are
    exchanged once over the group; every call is then ONE kernel per rank with
    device-side flow control (no collective per call)."""

    def __init__(self, pair: int, w: int, group=None, device=None):
        import torch.distributed as dist

        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        self.pair, self.w = pair, w
        self.link = ChainLink(pair, w, device)
        self.device = self.link.device
        handles = [None] * self.nranks
        dist.all_gather_object(handles, self.link.ipc_handle(), group=group)
        self.above = PeerLink(handles[self.rank - 1], self.device) if self.rank > 0 else None
        self.below = PeerLink(handles[self.rank + 1], self.device) if self.rank + 1 < self.nranks else None
        self.epoch = 0

    def sat(self, band, out=None, plan: Plan | None = None, stream=None):
        """This rank's band of the chained SAT (rows in rank order)."""
        self.epoch += 1
        return sat_band_chained(band, self.link, self.above, self.below, self.epoch, out=out,
                                plan=plan, stream=stream)

    def close(self):
        for l in (self.above, self.below, self.link):
            if l is not None:
                l.close()


def sat_dist_chained(band, comm: SatComm, out=None, plan: Plan | None = None, stream=None):
    """Row-banded SAT across ranks with chained carries over peer memory (one
    kernel per rank, no column-sum pass); links bootstrapped over the NCCL comm."""
    torch = _torch()
    pair = pair_of_dtype(band.dtype, out.dtype if out is not None else None)
    if out is None:
        out = torch.empty(band.shape, dtype=out_dtype(pair), device=band.device)
    H, W = band.shape
    p = plan if plan is not None else _plan_for(band.device, pair, max(H, 1), W, 1)
    _check(lib().sat_compute_dist_chained(p.handle, comm._h, band.data_ptr(), out.data_ptr(), H, W,
                                          _row_layout(band)[0], _row_layout(out)[0], pair,
                                          _stream_ptr(stream, band.device)),
           "sat_compute_dist_chained")
    return out
