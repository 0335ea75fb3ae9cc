"""Host<->device copy bandwidth on the box (pinned memory, CUDA events):
H2D alone, D2H alone, and both directions at once on two streams — the
ceiling for bench.py's e2e (fop_run_host_many moves 1.007 GB in and 0.667 GB
out per step)."""
import torch

N = 512 << 20
h_in = torch.empty(N, dtype=torch.uint8).pin_memory()
h_out = torch.empty(N, dtype=torch.uint8).pin_memory()
d_a = torch.empty(N, dtype=torch.uint8, device="cuda")
d_b = torch.empty(N, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


def both():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur)
    s2.wait_stream(cur)
    with torch.cuda.stream(s1):
        d_a.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_b, non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


t = timed(lambda: d_a.copy_(h_in, non_blocking=True))
print(f"H2D alone   {N / t / 1e6:7.1f} GB/s")
t = timed(lambda: h_out.copy_(d_b, non_blocking=True))
print(f"D2H alone   {N / t / 1e6:7.1f} GB/s")
t = timed(both)
print(f"both at once {2 * N / t / 1e6:7.1f} GB/s total ({N / t / 1e6:.1f} each way)")
