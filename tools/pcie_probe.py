"""PCIe ceiling for bench.py's e2e leg: pinned H2D of one step's inputs, D2H of
its results, alone and concurrently on two streams (CUDA events, median of 20)."""
import statistics
import torch

dev = torch.device("cuda:0")
h_in = torch.empty(36_560_920 // 8, dtype=torch.int64).pin_memory()
h_out = torch.empty(25_881_616 // 8, dtype=torch.int64).pin_memory()
d_in = torch.empty_like(h_in, device=dev)
d_out = torch.empty_like(h_out, device=dev)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def t(fn, reps=20):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def both():
    cur = torch.cuda.current_stream()
    ev = torch.cuda.Event()
    ev.record(cur)
    s1.wait_event(ev)
    s2.wait_event(ev)
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


h2d = t(lambda: d_in.copy_(h_in, non_blocking=True))
d2h = t(lambda: h_out.copy_(d_out, non_blocking=True))
bb = t(both)
print(f"H2D {h2d:.3f} ms = {h_in.numel() * 8 / h2d / 1e6:.1f} GB/s; D2H {d2h:.3f} ms = {h_out.numel() * 8 / d2h / 1e6:.1f} GB/s; "
      f"both {bb:.3f} ms -> e2e ceiling {139364 / bb * 1e3 / 1e6:.0f} M nodes/s (ALL10 step)")
