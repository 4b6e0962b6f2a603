"""Per-CTA phase trace of the tensor-core MAC (globaltimer), conv3_x bench shape.
Debug tool: POLYCONV_TC_DEBUG bit 8 makes mac_tc2 record timestamps."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_cgo_xuzc025_b200 as pc, synth

shape = synth.CONV3X
math = sys.argv[1] if len(sys.argv) > 1 else "bf16"
modes = [int(m) for m in sys.argv[2:]] or [0]
io = "bf16" if math == "bf16" else "f32"
dt = torch.bfloat16 if io == "bf16" else torch.float32
x, w = synth.make_inputs(shape, 1, "uniform")
x, w = torch.from_numpy(x).cuda().to(dt), torch.from_numpy(w).cuda().to(dt)
plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io, kernel=os.environ.get("KERN", "auto"))
print(plan.info())
lib = pc.load_library()
buf = (ctypes.c_ulonglong * (160 * 8))()
flush = torch.empty(64 << 20, device="cuda")
evict = torch.empty(64 << 20, device="cuda")
names = ["setup", "first_B_full", "mma_issued", "epi_start", "epi_end", "packer_win0", "cta_end"]
for mode in modes:
    os.environ["POLYCONV_TC_DEBUG"] = str(8 | mode)
    for it in range(3):
        flush.zero_()
        evict.sum()  # write back the flush's dirty lines before the launch
        y = plan.forward(x, w)
        torch.cuda.synchronize()
    lib.polyconv_dbg_tc2_trace(buf)
    a = np.array(buf, dtype=np.float64).reshape(160, 8)[: plan.info()["tile_m"] and 148]
    a = a[a[:, 0] > 0]
    t0 = a[:, 0].min()
    rel = (a - t0) / 1e3

    print("mode", mode, "CTAs", len(a), "start spread %.2f us" % (rel[:, 0].max()))
    nm_list = names if not (mode & 64) else ["setup", "pk_waited", "pk_zeroed", "pk_barrier", "pk_scattered",
                                              "packer_win0", "cta_end"]
    if mode & 32:
        raw = np.array(buf, dtype=np.float64).reshape(160, 8)[:len(a)]
        cyc = raw[:, 3] - raw[:, 2]
        ns = None
        print("  MMA phase in SM cycles: min %d med %d max %d" % (cyc.min(), np.median(cyc), cyc.max()))
        continue
    if mode & 128:
        eb = (ctypes.c_ulonglong * (160 * 8))()
        lib.polyconv_dbg_tc2_epi(eb)
        e = np.array(eb, dtype=np.float64).reshape(160, 8)[:len(a)]
        for k, nm in enumerate(["tmem_ld", "stage_st", "bar1", "pos_table", "copy_out", "bar2"]):
            print("  epi %-10s cycles med %7d max %7d" % (nm, np.median(e[:, k]), e[:, k].max()))
    if mode & 16:
        pkb = (ctypes.c_ulonglong * (160 * 8))()
        lib.polyconv_dbg_tc2_pk(pkb)
        pk = np.array(pkb, dtype=np.float64).reshape(160, 8)[:len(a)]
        pkn = ["box0_landed", "box1_landed", "box2_landed", "box3_landed", "box4_landed", "box5_landed",
               "win0_packed_pw0", "xld_win0_issued"]
        print("  pk box0 transpose cycles: med %d max %d; window-1 box0: med %d max %d" % (
            np.median(pk[:, 5]), pk[:, 5].max(), np.median(pk[:, 4]), pk[:, 4].max()))
        for k, nm in enumerate(pkn):
            if k in (4, 5): continue
            col = (pk[:, k] - t0) / 1e3
            col = col[pk[:, k] > 0] if (pk[:, k] > 0).any() else col
            print("  pk %-16s min %7.2f  med %7.2f  max %7.2f us" % (nm, col.min(), np.median(col), col.max()))
    for k, nm in enumerate(nm_list, 1):
        col = rel[:, k]
        print("  %-14s min %7.2f  med %7.2f  max %7.2f us" % (nm, col.min(), np.median(col), col.max()))
os.environ["POLYCONV_TC_DEBUG"] = "0"

