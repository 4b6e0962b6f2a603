"""H2D / D2H of one conv3x step's bytes (6.4 MB) from differently allocated pinned host buffers:
torch pin_memory (cudaHostAlloc default), cudaHostAlloc write-combined, cudaHostRegister'd
malloc; median of 30 (CUDA events), one and both directions."""
import ctypes, json, statistics, sys
import torch
cudart = ctypes.CDLL(torch.cuda.__file__.replace("__init__.py", "") + "../lib/libcudart.so.12") if False else None
import torch.cuda
nb = 6422528
dev = torch.empty(nb, dtype=torch.uint8, device="cuda")
dev2 = torch.empty(nb, dtype=torch.uint8, device="cuda")
lib = ctypes.CDLL("libcudart.so")  # torch's bundled runtime is already loaded
lib.cudaHostAlloc.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_size_t, ctypes.c_uint]
lib.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p]
def halloc(flags):
    p = ctypes.c_void_p()
    assert lib.cudaHostAlloc(ctypes.byref(p), nb, flags) == 0
    return p.value
bufs = {"torch_pin": (torch.empty(nb, dtype=torch.uint8).pin_memory().data_ptr(), torch.empty(nb, dtype=torch.uint8).pin_memory().data_ptr()),
        "hostalloc_default": (halloc(0), halloc(0)),
        "hostalloc_wc": (halloc(4), halloc(0)),
        "hostalloc_portable_mapped": (halloc(1 | 2), halloc(1 | 2))}
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
out = {}
for name, (hin, hout) in bufs.items():
    r = {}
    for mode in ("h2d", "d2h", "both"):
        ts = []
        for it in range(33):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if mode in ("h2d", "both"):
                lib.cudaMemcpyAsync(ctypes.c_void_p(dev.data_ptr()), ctypes.c_void_p(hin), nb, 1, ctypes.c_void_p(s1.cuda_stream))
            if mode in ("d2h", "both"):
                lib.cudaMemcpyAsync(ctypes.c_void_p(hout), ctypes.c_void_p(dev2.data_ptr()), nb, 2, ctypes.c_void_p(s2.cuda_stream))
            torch.cuda.synchronize()
            e1.record(); torch.cuda.synchronize()
            if it >= 3: ts.append(e0.elapsed_time(e1))
        r[mode] = round(statistics.median(ts) * 1e3, 1)
    out[name] = r
print(json.dumps(out))
