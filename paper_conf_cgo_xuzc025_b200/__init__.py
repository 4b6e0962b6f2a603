"""PolyHankel forward convolution on B200 (sm_100a) — Python binding.

A thin ctypes layer over the in-tree C-ABI library `_lib/libpolyconv.so`
(include/polyconv.h).  It only marshals arguments: every step of the hot path
(packing, coefficient MAC, extraction) runs in the library's CUDA kernels.
PyTorch supplies device memory and streams.  There is no CPU fallback: if the
library is missing the import of the binding fails loudly.

    from paper_conf_cgo_xuzc025_b200 import Plan
    plan = Plan((N, C, H, W), (K, C, R, S), stride=(1, 1), padding=(1, 1), math="bf16")
    y = plan.forward(x, w)          # x, w: CUDA tensors (fp32, or bf16 with math="bf16")
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("POLYCONV_LIB") or os.path.join(_PKG, "_lib", "libpolyconv.so")  # override: A/B runs

SUCCESS, BAD_PARAM, NOT_SUPPORTED, ALLOC_FAILED, EXECUTION_FAILED = range(5)
F32, BF16 = 0, 1
MATH = {"fp32": 0, "tf32": 1, "bf16": 2}
KERNEL = {"auto": 0, "tc": 1, "fp32": 2, "thin": 3, "tc_pertap": 4, "tc_fused": 5, "tc_pair": 6, "tc_1x1": 7, "tc_hankel": 8, "fft": 9}
KERNEL_NAME = {v: k for k, v in KERNEL.items()}
LAYOUT = {"planar": 0, "interleaved": 1}


class PolyconvError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(msg)
        self.status = status


class Info(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in "N C H W K R S sh sw ph pw P Q Hp Wp".split()] + [
        ("L_A", ctypes.c_longlong), ("L_U", ctypes.c_longlong), ("Cp", ctypes.c_int), ("Kp", ctypes.c_int),
        ("kernel", ctypes.c_int), ("tile_m", ctypes.c_int), ("tile_n", ctypes.c_int), ("stages", ctypes.c_int),
        ("launches", ctypes.c_int), ("workspace_bytes", ctypes.c_size_t)]

    def asdict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["kernel"] = KERNEL_NAME.get(d["kernel"], d["kernel"])
        return d


EXPORTS = ["polyconv_plan", "polyconv_plan_set_kernel", "polyconv_output_dims", "polyconv_plan_info",
           "polyconv_forward", "polyconv_forward_scatter", "polyconv_forward_host", "polyconv_plan_set_timing_events", "polyconv_pack_input", "polyconv_pack_filter", "polyconv_packed_bytes",
           "polyconv_extract", "polyconv_destroy", "polyconv_status_string", "polyconv_last_error",
           "polyconv_abi_version", "polyconv_flip_filter", "polyconv_swap_nc",
           "polyconv_dilate", "polyconv_wgrad"]

_lib = None


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load the C-ABI library (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError("polyconv CUDA library not built: %s missing (run `python -m "
                          "paper_conf_cgo_xuzc025_b200.build` or __graft_entry__.build())" % path)
    lib = ctypes.CDLL(path)
    vp, ip, i = ctypes.c_void_p, ctypes.POINTER(ctypes.c_int), ctypes.c_int
    P = ctypes.POINTER(ctypes.c_void_p)
    lib.polyconv_plan.argtypes = [P] + [i] * 11 + [i, i, i]
    lib.polyconv_plan_set_kernel.argtypes = [vp, i]
    lib.polyconv_output_dims.argtypes = [vp, ip, ip]
    lib.polyconv_plan_info.argtypes = [vp, ctypes.POINTER(Info)]
    lib.polyconv_forward.argtypes = [vp, vp, vp, vp, vp]
    lib.polyconv_forward_host.argtypes = [vp, vp, vp, vp, vp]
    lib.polyconv_forward_scatter.argtypes = [vp, vp, vp, ctypes.POINTER(vp), i, i, i, vp]
    lib.polyconv_plan_set_timing_events.argtypes = [vp, vp, vp]
    lib.polyconv_pack_input.argtypes = [vp, vp, vp, i, vp]
    lib.polyconv_pack_filter.argtypes = [vp, vp, vp, i, vp]
    lib.polyconv_packed_bytes.argtypes = [vp, i, i, ctypes.POINTER(ctypes.c_size_t)]
    lib.polyconv_extract.argtypes = [vp, vp, vp, vp]
    lib.polyconv_destroy.argtypes = [vp]
    lib.polyconv_status_string.argtypes = [i]
    lib.polyconv_status_string.restype = ctypes.c_char_p
    lib.polyconv_last_error.argtypes = [vp]
    lib.polyconv_last_error.restype = ctypes.c_char_p
    lib.polyconv_abi_version.argtypes = []
    lib.polyconv_flip_filter.argtypes = [vp, vp, i, i, i, i, i, vp]
    lib.polyconv_swap_nc.argtypes = [vp, vp, i, i, ctypes.c_longlong, i, vp]
    lib.polyconv_dilate.argtypes = [vp, vp] + [i] * 8 + [i, vp]
    lib.polyconv_wgrad.argtypes = [vp, vp, vp, vp] + [i] * 11 + [i, vp]
    for name in EXPORTS:
        if name not in ("polyconv_status_string", "polyconv_last_error"):
            getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def status_string(status: int) -> str:
    return load_library().polyconv_status_string(status).decode()


def _stream_ptr(stream, device=None):
    """cudaStream_t of `stream`, else torch's current stream of `device` (the tensors'
    device, not necessarily the current one)."""
    import torch
    if stream is None:
        stream = torch.cuda.current_stream(device)
    return ctypes.c_void_p(stream.cuda_stream)


def _on_device(t):
    """Context making t's device current for a library call (the layout entry points take no
    device argument and launch on the current device)."""
    import torch
    return torch.cuda.device(t.device)


class Plan:
    """One convolution problem (shapes, stride, padding, dtype, math) on one device.

    math: "fp32" (SIMT FFMA), "tf32" or "bf16" (tcgen05 tensor cores).
    io_dtype: "f32" or "bf16" (bf16 requires math="bf16").
    kernel: "auto" | "tc" | "fp32" | "thin" (force a MAC variant).
    """

    def __init__(self, x_shape, w_shape, stride=(1, 1), padding=(0, 0), math="bf16", io_dtype="f32",
                 device: int = 0, kernel: str = "auto"):
        self._lib = load_library()
        N, C, H, W = x_shape
        K, C2, R, S = w_shape
        if C != C2:
            raise PolyconvError(BAD_PARAM, "channel mismatch")
        self.x_shape, self.w_shape = tuple(x_shape), tuple(w_shape)
        self.stride, self.padding = tuple(stride), tuple(padding)
        self.math, self.io_dtype, self.device = math, io_dtype, device
        h = ctypes.c_void_p()
        st = self._lib.polyconv_plan(ctypes.byref(h), N, C, H, W, K, R, S, stride[0], stride[1], padding[0],
                                     padding[1], BF16 if io_dtype == "bf16" else F32, MATH[math], device)
        if st != SUCCESS:
            raise PolyconvError(st, "polyconv_plan: %s" % status_string(st))
        self._h = h
        if kernel != "auto":
            self._check(self._lib.polyconv_plan_set_kernel(self._h, KERNEL[kernel]), "set_kernel")
        P, Q = ctypes.c_int(), ctypes.c_int()
        self._check(self._lib.polyconv_output_dims(self._h, ctypes.byref(P), ctypes.byref(Q)), "output_dims")
        self.P, self.Q = P.value, Q.value

    # -- helpers ---------------------------------------------------------------
    def _check(self, st, what):
        if st != SUCCESS:
            detail = self._lib.polyconv_last_error(self._h).decode() if getattr(self, "_h", None) else ""
            raise PolyconvError(st, "polyconv_%s: %s %s" % (what, status_string(st), detail))

    @property
    def handle(self):
        return self._h

    @property
    def output_shape(self):
        return (self.x_shape[0], self.w_shape[0], self.P, self.Q)

    def info(self) -> dict:
        inf = Info()
        self._check(self._lib.polyconv_plan_info(self._h, ctypes.byref(inf)), "plan_info")
        return inf.asdict()

    def _io_torch_dtype(self):
        import torch
        return torch.bfloat16 if self.io_dtype == "bf16" else torch.float32

    def _check_tensor(self, t, shape, name):
        import torch
        if not isinstance(t, torch.Tensor) or not t.is_cuda:
            raise PolyconvError(BAD_PARAM, "%s must be a CUDA tensor" % name)
        if tuple(t.shape) != tuple(shape):
            raise PolyconvError(BAD_PARAM, "%s shape %s != %s" % (name, tuple(t.shape), tuple(shape)))
        if t.dtype != self._io_torch_dtype():
            raise PolyconvError(BAD_PARAM, "%s dtype %s != %s" % (name, t.dtype, self._io_torch_dtype()))
        if not t.is_contiguous():
            raise PolyconvError(BAD_PARAM, "%s must be contiguous" % name)

    # -- the hot path ------------------------------------------------------------
    def forward(self, x, w, y=None, stream=None):
        """y[N][K][P][Q] = conv(x, w) via pack -> coefficient MAC -> extraction."""
        import torch
        self._check_tensor(x, self.x_shape, "x")
        self._check_tensor(w, self.w_shape, "w")
        if y is None:
            y = torch.empty(self.output_shape, dtype=self._io_torch_dtype(), device=x.device)
        else:
            self._check_tensor(y, self.output_shape, "y")
        self._check(self._lib.polyconv_forward(self._h, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(w.data_ptr()),
                                               ctypes.c_void_p(y.data_ptr()), _stream_ptr(stream, self.device)), "forward")
        return y

    def forward_scatter(self, x, w, y_ptrs, k_total, k_offset, stream=None):
        """Output-channel shard with the all-gather fused into the epilogue (f4): this plan's
        K channels are stored at channel offset `k_offset` of every buffer in `y_ptrs`
        (device addresses of [N][k_total][P][Q] outputs: local, or peers' mapped over NVLink,
        e.g. torch symmetric memory's buffer_ptrs).  Only TC_HANKEL plans (NOT_SUPPORTED else)."""
        self._check_tensor(x, self.x_shape, "x")
        self._check_tensor(w, self.w_shape, "w")
        ptrs = (ctypes.c_void_p * len(y_ptrs))(*[int(v) for v in y_ptrs])
        self._check(self._lib.polyconv_forward_scatter(self._h, ctypes.c_void_p(x.data_ptr()),
                                                       ctypes.c_void_p(w.data_ptr()), ptrs, len(y_ptrs),
                                                       int(k_total), int(k_offset), _stream_ptr(stream, self.device)),
                    "forward_scatter")

    def forward_host(self, x, w, y, stream=None):
        """End-to-end call: x, w, y are (pinned) CPU tensors; the library copies
        them to/from its own device buffers on `stream` and runs the forward.
        Asynchronous: synchronise the stream before reading y."""
        for t, shp, nm in ((x, self.x_shape, "x"), (w, self.w_shape, "w"), (y, self.output_shape, "y")):
            if t.is_cuda or tuple(t.shape) != tuple(shp) or t.dtype != self._io_torch_dtype() or not t.is_contiguous():
                raise PolyconvError(BAD_PARAM, "%s must be a contiguous host tensor %s of %s" % (nm, shp, self.io_dtype))
        self._check(self._lib.polyconv_forward_host(self._h, ctypes.c_void_p(x.data_ptr()),
                                                    ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(y.data_ptr()),
                                                    _stream_ptr(stream, self.device)), "forward_host")
        return y

    def set_timing_events(self, start, stop):
        """Record torch.cuda.Event start/stop around the MAC kernel of every later
        forward (None, None clears)."""
        for ev in (start, stop):
            if ev is not None and not ev.cuda_event:
                ev.record()  # torch creates the underlying cudaEvent_t lazily
        sp = ctypes.c_void_p(start.cuda_event) if start is not None else None
        ep = ctypes.c_void_p(stop.cuda_event) if stop is not None else None
        self._check(self._lib.polyconv_plan_set_timing_events(self._h, sp, ep), "set_timing_events")

    def forward_ptr(self, x_ptr: int, w_ptr: int, y_ptr: int, stream_ptr: int = 0):
        """Raw-pointer forward (no checks beyond the library's)."""
        self._check(self._lib.polyconv_forward(self._h, ctypes.c_void_p(x_ptr), ctypes.c_void_p(w_ptr),
                                               ctypes.c_void_p(y_ptr), ctypes.c_void_p(stream_ptr)), "forward")

    # -- single steps (bit-exact tests) ------------------------------------------------
    def packed_bytes(self, which: str, layout: str) -> int:
        b = ctypes.c_size_t()
        self._check(self._lib.polyconv_packed_bytes(self._h, 0 if which == "input" else 1, LAYOUT[layout],
                                                    ctypes.byref(b)), "packed_bytes")
        return b.value

    def pack_input(self, x, layout="planar", stream=None):
        """a2: returns the packed A_{n,c}(t) words as a uint8 CUDA tensor."""
        import torch
        self._check_tensor(x, self.x_shape, "x")
        out = torch.empty(self.packed_bytes("input", layout), dtype=torch.uint8, device=x.device)
        self._check(self._lib.polyconv_pack_input(self._h, ctypes.c_void_p(x.data_ptr()),
                                                  ctypes.c_void_p(out.data_ptr()), LAYOUT[layout],
                                                  _stream_ptr(stream, self.device)), "pack_input")
        return out

    def pack_filter(self, w, layout="planar", stream=None):
        """a3: returns the packed U_{k,c}(t) words as a uint8 CUDA tensor."""
        import torch
        self._check_tensor(w, self.w_shape, "w")
        out = torch.empty(self.packed_bytes("filter", layout), dtype=torch.uint8, device=w.device)
        self._check(self._lib.polyconv_pack_filter(self._h, ctypes.c_void_p(w.data_ptr()),
                                                   ctypes.c_void_p(out.data_ptr()), LAYOUT[layout],
                                                   _stream_ptr(stream, self.device)), "pack_filter")
        return out

    def extract(self, coeffs, stream=None):
        """a5: y from the full fp32 product coefficients [N][K][L_A+L_U-1]."""
        import torch
        inf = self.info()
        Lp = inf["L_A"] + inf["L_U"] - 1
        if not coeffs.is_cuda or coeffs.dtype != torch.float32 or tuple(coeffs.shape) != (self.x_shape[0],
                                                                                           self.w_shape[0], Lp):
            raise PolyconvError(BAD_PARAM, "coeffs must be float32 CUDA [N][K][L_A+L_U-1]")
        y = torch.empty(self.output_shape, dtype=self._io_torch_dtype(), device=coeffs.device)
        self._check(self._lib.polyconv_extract(self._h, ctypes.c_void_p(coeffs.data_ptr()),
                                               ctypes.c_void_p(y.data_ptr()), _stream_ptr(stream, self.device)), "extract")
        return y

    def close(self):
        h = getattr(self, "_h", None)
        if h:
            self._lib.polyconv_destroy(h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _dtype_code(t):
    import torch
    if t.dtype == torch.bfloat16:
        return BF16
    if t.dtype == torch.float32:
        return F32
    raise PolyconvError(BAD_PARAM, "dtype %s (float32 or bfloat16)" % t.dtype)


def flip_filter(w, stream=None):
    """f4 layout step (include/polyconv.h): wt[c][k][R-1-i][S-1-j] = w[k][c][i][j]."""
    import torch
    if not w.is_cuda or not w.is_contiguous() or w.dim() != 4:
        raise PolyconvError(BAD_PARAM, "w must be a contiguous 4-D CUDA tensor")
    K, C, R, S = w.shape
    wt = torch.empty((C, K, R, S), dtype=w.dtype, device=w.device)
    with _on_device(w):
        st = load_library().polyconv_flip_filter(ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(wt.data_ptr()), K, C,
                                                R, S, _dtype_code(w), _stream_ptr(stream, w.device))
    if st != SUCCESS:
        raise PolyconvError(st, "polyconv_flip_filter: %s" % status_string(st))
    return wt


def swap_nc(x, stream=None):
    """f4 layout step (include/polyconv.h): xt[c][n][...] = x[n][c][...]."""
    import torch
    if not x.is_cuda or not x.is_contiguous() or x.dim() < 2:
        raise PolyconvError(BAD_PARAM, "x must be a contiguous CUDA tensor of rank >= 2")
    N, C = x.shape[:2]
    hw = x.numel() // (N * C) if x.numel() else 0
    xt = torch.empty((C, N) + tuple(x.shape[2:]), dtype=x.dtype, device=x.device)
    with _on_device(x):
        st = load_library().polyconv_swap_nc(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(xt.data_ptr()), N, C, hw,
                                            _dtype_code(x), _stream_ptr(stream, x.device))
    if st != SUCCESS:
        raise PolyconvError(st, "polyconv_swap_nc: %s" % status_string(st))
    return xt


def dilate(x, stride, extra=(0, 0), stream=None):
    """f4 layout step (include/polyconv.h): x on the stride lattice of a zero plane, plus
    `extra` zero rows / columns at the bottom / right."""
    import torch
    if not x.is_cuda or not x.is_contiguous() or x.dim() != 4:
        raise PolyconvError(BAD_PARAM, "x must be a contiguous 4-D CUDA tensor")
    N, C, H, W = x.shape
    (sh, sw), (eh, ew) = stride, extra
    xd = torch.empty((N, C, (H - 1) * sh + 1 + eh, (W - 1) * sw + 1 + ew), dtype=x.dtype, device=x.device)
    with _on_device(x):
        st = load_library().polyconv_dilate(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(xd.data_ptr()), N, C, H,
                                           W, sh, sw, eh, ew, _dtype_code(x), _stream_ptr(stream, x.device))
    if st != SUCCESS:
        raise PolyconvError(st, "polyconv_dilate: %s" % status_string(st))
    return xd


def wgrad(x, dy, w_shape, stride=(1, 1), padding=(0, 0), stream=None):
    """f4 (include/polyconv.h): dw[k][c][i][j] = sum dy[n][k][oh][ow] * xpad[n][c][sh*oh+i][sw*ow+j]."""
    import torch
    for t, nm in ((x, "x"), (dy, "dy")):
        if not t.is_cuda or not t.is_contiguous() or t.dim() != 4:
            raise PolyconvError(BAD_PARAM, "%s must be a contiguous 4-D CUDA tensor" % nm)
    if x.dtype != dy.dtype:
        raise PolyconvError(BAD_PARAM, "x and dy must share a dtype")
    if x.device != dy.device:
        raise PolyconvError(BAD_PARAM, "x and dy must be on one device")
    N, C, H, W = x.shape
    K, Cw, R, S = w_shape
    if Cw != C:
        raise PolyconvError(BAD_PARAM, "w_shape[1] = %d but x has %d channels" % (Cw, C))
    P = (H + 2 * padding[0] - R) // stride[0] + 1
    Q = (W + 2 * padding[1] - S) // stride[1] + 1
    if tuple(dy.shape) != (N, K, P, Q):
        raise PolyconvError(BAD_PARAM, "dy must be %s, got %s" % ((N, K, P, Q), tuple(dy.shape)))
    dw = torch.empty((K, C, R, S), dtype=x.dtype, device=x.device)
    ws = torch.empty(K * C * R * S, dtype=torch.float32, device=x.device)
    with _on_device(x):
        st = load_library().polyconv_wgrad(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(dy.data_ptr()),
                                          ctypes.c_void_p(dw.data_ptr()), ctypes.c_void_p(ws.data_ptr()), N, C, H, W,
                                          K, R, S, stride[0], stride[1], padding[0], padding[1], _dtype_code(x),
                                          _stream_ptr(stream, x.device))
    if st != SUCCESS:
        raise PolyconvError(st, "polyconv_wgrad: %s" % status_string(st))
    return dw


def conv2d(x, w, stride=(1, 1), padding=(0, 0), math="bf16", kernel="auto", out=None):
    """One-shot convenience: plan + forward (the plan is cached per shape); `out` (optional)
    receives y in place."""
    key = (tuple(x.shape), tuple(w.shape), tuple(stride), tuple(padding), math,
           "bf16" if str(x.dtype) == "torch.bfloat16" else "f32", x.device.index or 0, kernel)
    plan = _PLANS.get(key)
    if plan is None:
        plan = Plan(x.shape, w.shape, stride, padding, math, key[5], key[6], kernel)
        _PLANS[key] = plan
    return plan.forward(x, w, out)


_PLANS: dict = {}
