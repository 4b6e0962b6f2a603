import os, sys
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch, synth, oracle
from synth import ConvShape
from helpers import gpu_forward, normwise
shapes = {"mx_s2": ConvShape("mx_s2", 2, 48, 20, 20, 64, 3, 3, 2, 2, 1, 1),
          "s2_c64": ConvShape("s2_c64", 2, 64, 20, 20, 64, 3, 3, 2, 2, 1, 1),
          "s1_c48": ConvShape("s1_c48", 2, 48, 20, 20, 64, 3, 3, 1, 1, 1, 1),
          "s1_c48_h16": ConvShape("s1_c48_h16", 2, 48, 16, 16, 64, 3, 3, 1, 1, 1, 1)}
sh = shapes[sys.argv[1]]
io = sys.argv[2] if len(sys.argv) > 2 else "bf16"
x, w = synth.make_inputs(sh, 5, "int")
y, plan = gpu_forward(sh, x, w, math="bf16", io=io, kernel="tc_pair")
ref = oracle.conv2d(x, w, sh.stride, sh.padding)
print(sys.argv[1:], "maxdiff", float(np.abs(y - ref).max()))
