"""Per-CTA phase trace of the CTA-pair kernel (mac_pair.cu, POLYCONV_PAIR_DEBUG&8),
conv3_x bench shape, L2 flushed before each launch.  Debug tool."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_cgo_xuzc025_b200 as pc, synth

shape = synth.CONV3X
x, w = synth.make_inputs(shape, 1, "uniform")
x, w = torch.from_numpy(x).cuda().bfloat16(), torch.from_numpy(w).cuda().bfloat16()
plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16", kernel="tc_pair")
print(plan.info())
lib = pc.load_library()
buf = (ctypes.c_ulonglong * (160 * 16))()
flush = torch.empty(64 << 20, device="cuda")  # 256 MiB (float32), as bench.py
evict = torch.empty(64 << 20, device="cuda")  # 256 MiB: no dirty flush lines remain
os.environ["POLYCONV_PAIR_DEBUG"] = str(8 | (int(sys.argv[1]) if len(sys.argv) > 1 else 0))
for it in range(3):
    if os.environ.get("FLUSH", "1") == "1":
        flush.zero_()
        evict.sum()
    y = plan.forward(x, w)
    torch.cuda.synchronize()
os.environ["POLYCONV_PAIR_DEBUG"] = "0"
lib.polyconv_dbg_pair_trace(buf)
a = np.array(buf, dtype=np.float64).reshape(160, 16)
a = a[a[:, 0] > 0]
t0 = a[:, 0].min()
names = ["start", "pack_done", "counter_passed", "win0", "win1", "win2", "win3", "tile0_issued", "tile1_issued",
         "epi0_ready", "epi0_done", "epi1_ready", "filter_last", "end", "bands_ready0", "prod_last_tma"]
print("CTAs", len(a))
for k, nm in enumerate(names):
    col = a[:, k]
    col = col[col > 0]
    if len(col) == 0:
        continue
    rel = (col - t0) / 1e3
    print("  %-16s n=%3d min %7.2f  med %7.2f  max %7.2f us" % (nm, len(col), rel.min(), np.median(rel), rel.max()))

clk = (ctypes.c_ulonglong * (160 * 2))()
lib.polyconv_dbg_pair_clk(clk)
c = np.array(clk, dtype=np.float64).reshape(160, 2)[: len(a)]
raw = np.array(buf, dtype=np.float64).reshape(160, 16)[: len(a)]
mhz = (c[:, 1] - c[:, 0]) / (raw[:, 13] - raw[:, 0]) * 1e3
print("  SM clock during the kernel: med %.0f MHz (min %.0f, max %.0f)" % (np.median(mhz), mhz.min(), mhz.max()))

pk = (ctypes.c_ulonglong * (160 * 4))()
lib.polyconv_dbg_pair_pk(pk)
k = np.array(pk, dtype=np.float64).reshape(160, 4)[: len(a)]
for col, nm in enumerate(["pk_filter_done", "pk_band_staged", "pk_band_written", "pk_band_gathered"]):
    v = k[:, col]
    v = v[v > 0]
    if len(v):
        rel = (v - t0) / 1e3
        print("  %-16s n=%3d min %7.2f  med %7.2f  max %7.2f us" % (nm, len(v), rel.min(), np.median(rel), rel.max()))

iss = (ctypes.c_ulonglong * (160 * 4))()
lib.polyconv_dbg_pair_iss(iss)
k = np.array(iss, dtype=np.float64).reshape(160, 4)[: len(a)]
for col, nm in enumerate(["iss_c0_filter", "iss_c0_issued", "iss_c1_filter", "iss_c1_issued"]):
    v = k[:, col]
    v = v[v > 0]
    if len(v):
        rel = (v - t0) / 1e3
        print("  %-16s n=%3d min %7.2f  med %7.2f  max %7.2f us" % (nm, len(v), rel.min(), np.median(rel), rel.max()))
