"""Time the hot-path pieces separately on the bench workload (debug tool).
usage: python tools/phase_time.py [bf16|tf32] [kernels...]
Prints median CUDA-event times (L2 flushed before each rep) of: the standalone
interleaved input pack, and full forwards with each requested MAC kernel."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_xuzc025_b200 as pc, synth

math = sys.argv[1] if len(sys.argv) > 1 else "bf16"
kernels = sys.argv[2:] or ["tc", "tc_fused"]
shape = synth.CONV3X
io = "bf16" if math == "bf16" else "f32"
dt = torch.bfloat16 if io == "bf16" else torch.float32
x, w = synth.make_inputs(shape, 1, "uniform")
x, w = torch.from_numpy(x).cuda().to(dt), torch.from_numpy(w).cuda().to(dt)
flush = torch.empty(64 << 20, device="cuda")
evict = torch.empty(64 << 20, device="cuda")
MODE = os.environ.get("FLUSH", "write+read")
REPS = 50


def timeit(fn, flush_l2=True):
    ts = []
    for it in range(REPS + 5):
        if flush_l2:
            flush.zero_()
            if MODE == "write+read":  # write back the dirty lines before the timed region
                evict.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record()
        torch.cuda.synchronize()
        if it >= 5:
            ts.append(a.elapsed_time(b) * 1e3)
    return statistics.median(ts), min(ts)


plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io)
lib = pc.load_library()
import ctypes
nb = ctypes.c_size_t()
lib.polyconv_packed_bytes(plan.handle, 0, 1, ctypes.byref(nb))
dst = torch.empty(nb.value // 2 + 16, dtype=torch.bfloat16, device="cuda")
st = torch.cuda.current_stream()
def pack():
    lib.polyconv_pack_input(plan.handle, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(dst.data_ptr()), 1,
                            ctypes.c_void_p(st.cuda_stream))
wdst = torch.empty(w.numel() * 4, dtype=torch.bfloat16, device="cuda")
def packf():
    lib.polyconv_pack_filter(plan.handle, ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(wdst.data_ptr()), 1,
                             ctypes.c_void_p(st.cuda_stream))
print("pack_filter tap-major: med %.2f us min %.2f us" % timeit(packf))
tiny = torch.zeros(4, device="cuda")
print("one tiny torch kernel: med %.2f us min %.2f us" % timeit(lambda: tiny.zero_()))
print("two tiny torch kernels: med %.2f us min %.2f us" % timeit(lambda: (tiny.zero_(), tiny.zero_())))
print("flush mode", MODE); print("pack_input interleaved: med %.2f us min %.2f us (%d bytes out)" % (*timeit(pack), nb.value))
for k in kernels:
    p = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io, kernel=k)
    y = p.forward(x, w)
    med, mn = timeit(lambda: p.forward(x, w, y))
    medw, mnw = timeit(lambda: p.forward(x, w, y), flush_l2=False)
    print("forward %-9s %s: cold med %.2f us min %.2f | warm med %.2f min %.2f | %s" % (
        k, math, med, mn, medw, mnw, p.info()))
import torch.nn.functional as Fn
torch.backends.cudnn.benchmark = True
xc, wc = x.contiguous(memory_format=torch.channels_last), w.contiguous(memory_format=torch.channels_last)
for _ in range(5):
    Fn.conv2d(xc, wc, padding=1)
print("cudnn channels_last: cold med %.2f min %.2f" % timeit(lambda: Fn.conv2d(xc, wc, padding=1)))
print("cudnn nchw: cold med %.2f min %.2f" % timeit(lambda: Fn.conv2d(x, w, padding=1)))
src = torch.empty(x.numel(), dtype=torch.bfloat16, device="cuda"); dd = torch.empty_like(src)
print("torch copy 6.4MB: cold med %.2f min %.2f" % timeit(lambda: dd.copy_(src)))
print("empty event pair: med %.2f min %.2f" % timeit(lambda: None))
