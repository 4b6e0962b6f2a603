"""Host<->device copy rates on this box (pinned memory): H2D alone, D2H alone, and both directions
on two streams at once — the ceiling for bench.py's e2e leg (polyconv_forward_host)."""
import json
import torch


def rate(fn, nbytes, reps=20):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / reps
    return {"ms": ms, "GB_s": nbytes / ms / 1e6}


def main():
    out = {}
    for mb in (6.4, 64):
        n = int(mb * 2 ** 20)
        h_in = torch.empty(n, dtype=torch.uint8).pin_memory()
        h_out = torch.empty(n, dtype=torch.uint8).pin_memory()
        d_in = torch.empty(n, dtype=torch.uint8, device="cuda")
        d_out = torch.empty(n, dtype=torch.uint8, device="cuda")
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        cur = torch.cuda.current_stream()

        def both():
            s1.wait_stream(cur)
            s2.wait_stream(cur)
            with torch.cuda.stream(s1):
                d_in.copy_(h_in, non_blocking=True)
            with torch.cuda.stream(s2):
                h_out.copy_(d_out, non_blocking=True)
            cur.wait_stream(s1)
            cur.wait_stream(s2)

        out["%gMB" % mb] = {
            "h2d": rate(lambda: d_in.copy_(h_in, non_blocking=True), n),
            "d2h": rate(lambda: h_out.copy_(d_out, non_blocking=True), n),
            "both_2streams": rate(both, 2 * n),
        }
    print(json.dumps(out))




def bind_local_numa(dev=0):
    """Pin this process to the CPUs NVML reports as local to `dev` (so pinned host buffers are
    first-touched on the GPU's NUMA node). Returns the CPU count or 0."""
    import os
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(dev)
    words = pynvml.nvmlDeviceGetCpuAffinity(h, (os.cpu_count() + 63) // 64)
    cpus = {i * 64 + b for i, w in enumerate(words) for b in range(64) if (w >> b) & 1}
    cpus &= set(range(os.cpu_count()))
    if cpus:
        os.sched_setaffinity(0, cpus)
    return len(cpus)


if __name__ == "__main__":
    import sys
    if "--bind" in sys.argv:
        print("bound to", bind_local_numa(), "cpus")
    main()
