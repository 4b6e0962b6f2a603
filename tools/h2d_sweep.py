import torch, json
def rate(fn, n, reps=20):
    fn(); torch.cuda.synchronize()
    a,b=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps): fn()
    b.record(); torch.cuda.synchronize()
    return round(n/(a.elapsed_time(b)/reps)/1e6,1)
out={}
for mb in (1,2,4,6.4,8,16,32,64):
    n=int(mb*2**20)
    h=torch.empty(n,dtype=torch.uint8).pin_memory(); d=torch.empty(n,dtype=torch.uint8,device="cuda")
    out[str(mb)]=rate(lambda: d.copy_(h,non_blocking=True),n)
big=torch.empty(128<<20,dtype=torch.uint8).pin_memory()
for mb in (2,6.4,16):
    n=int(mb*2**20); d=torch.empty(n,dtype=torch.uint8,device="cuda"); h=big[:n]
    out["slice_of_128MB_"+str(mb)]=rate(lambda: d.copy_(h,non_blocking=True),n)
print(json.dumps(out))
