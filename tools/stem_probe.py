import sys, torch
sys.path.insert(0, '.')
import paper_conf_cgo_xuzc025_b200 as pc
x = torch.randn(256, 3, 224, 224, device='cuda').bfloat16()
w = torch.randn(64, 3, 7, 7, device='cuda').bfloat16()
plan = pc.Plan(x.shape, w.shape, (2, 2), (3, 3), math="bf16", io_dtype="bf16")
print(plan.info())
y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device='cuda')
for _ in range(3):
    plan.forward(x, w, y)
torch.cuda.synchronize()
