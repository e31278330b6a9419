"""GPU-timeline cost of stream operations (run on the GPU box): N back-to-back event records
(timing / no-timing), empty kernels, and a cooperative vs plain launch, between two timing events."""
import torch

torch.cuda.init()
s = torch.cuda.current_stream()
N = 50


def timed(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        torch.cuda._sleep(200000)  # host head start: the GPU never waits for submission
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) * 1000.0)
    return best


base = timed(lambda: None)
evs_t = [torch.cuda.Event(enable_timing=True) for _ in range(N)]
evs_n = [torch.cuda.Event(enable_timing=False) for _ in range(N)]
t_t = timed(lambda: [e.record(s) for e in evs_t])
t_n = timed(lambda: [e.record(s) for e in evs_n])
x = torch.zeros(1, device="cuda")
t_k = timed(lambda: [x.add_(1) for _ in range(N)])
print(f"empty region {base:.2f} us; per record: timing {(t_t - base) / N:.2f} us, no-timing {(t_n - base) / N:.2f} us;"
      f" per tiny kernel {(t_k - base) / N:.2f} us")
