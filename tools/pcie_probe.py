"""Host<->device copy rates of pinned memory (the bound of the e2e leg, hgemm_host):
H2D alone, D2H alone, and both at once on two streams (experiments)."""
import torch

n_in, n_out = 256 << 20, 128 << 20
h_in = torch.empty(n_in, dtype=torch.uint8).pin_memory()
h_out = torch.empty(n_out, dtype=torch.uint8).pin_memory()
d_in = torch.empty(n_in, dtype=torch.uint8, device="cuda")
d_out = torch.empty(n_out, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def both():
    ev = torch.cuda.Event()
    ev.record()
    s1.wait_event(ev)
    s2.wait_event(ev)
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


t_in = timed(lambda: d_in.copy_(h_in, non_blocking=True))
t_out = timed(lambda: h_out.copy_(d_out, non_blocking=True))
t_both = timed(both)
print(f"H2D 256 MiB: {t_in:.3f} ms ({n_in / t_in / 1e6:.1f} GB/s); D2H 128 MiB: {t_out:.3f} ms "
      f"({n_out / t_out / 1e6:.1f} GB/s); both at once: {t_both:.3f} ms")
