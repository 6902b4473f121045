"""Where the pipelined e2e leg loses time against the PCIe ceiling: the bench's
copy pattern (9 input tensors up, 4 result tensors down, per step, two buffer
sets, three streams) with (a) no compute, (b) a 110 us device sleep as the
compute, (c) one concatenated input buffer instead of nine."""
import statistics
import sys

import torch

dev = torch.device("cuda:0")
IN = [24_766_640, 4_779_504, 1_114_920, 557_456, 557_456, 1_593_168, 1_593_168, 1_593_168, 2_640]  # bytes (ALL10)
OUT = [24_766_640, 1_114_912, 64, 16]


def run(n_steps, compute, concat):
    ins = [IN] if not concat else [[sum(IN)]]
    ins = ins[0]
    pinned = [torch.empty(b // 8, dtype=torch.int64).pin_memory() for b in ins]
    sets = []
    for _ in range(2):
        sets.append(dict(d_in=[torch.empty_like(p, device=dev) for p in pinned],
                         d_out=[torch.empty(b // 8, dtype=torch.int64, device=dev) for b in OUT],
                         h_out=[torch.empty(b // 8, dtype=torch.int64).pin_memory() for b in OUT],
                         ev_in=torch.cuda.Event(), ev_cp=torch.cuda.Event(), ev_out=torch.cuda.Event()))
    s_in, s_cp, s_out = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()

    def steps(n):
        for k in range(n):
            S = sets[k % 2]
            with torch.cuda.stream(s_in):
                if k >= 2:
                    s_in.wait_event(S["ev_cp"])
                for d, h in zip(S["d_in"], pinned):
                    d.copy_(h, non_blocking=True)
                S["ev_in"].record(s_in)
            with torch.cuda.stream(s_cp):
                s_cp.wait_event(S["ev_in"])
                if k >= 2:
                    s_cp.wait_event(S["ev_out"])
                if compute:
                    torch.cuda._sleep(int(110e-6 * 1.965e9))
                S["ev_cp"].record(s_cp)
            with torch.cuda.stream(s_out):
                s_out.wait_event(S["ev_cp"])
                for h, d in zip(S["h_out"], S["d_out"]):
                    h.copy_(d, non_blocking=True)
                S["ev_out"].record(s_out)

    steps(2)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s_in)
    steps(n_steps)
    for S in sets:
        s_out.wait_event(S["ev_out"])
    b.record(s_out)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n_steps


for compute in (False, True):
    for concat in (False, True):
        ms = statistics.median(run(50, compute, concat) for _ in range(3))
        print(f"compute={compute!s:5} concat_inputs={concat!s:5}: {ms:.3f} ms/step -> {139364 / ms / 1e3:.0f} M nodes/s",
              flush=True)
