"""Raw host<->device copy bandwidth of this box (pinned, one stream and two streams): the e2e leg's link bound."""
import torch

n = 192_000_000 // 4
h = torch.empty(n, dtype=torch.float32).pin_memory()
d = torch.empty(n, dtype=torch.float32, device="cuda")
ho = torch.empty(16_000_000, dtype=torch.float32).pin_memory()
do = torch.empty(16_000_000, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for _ in range(3):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()


def timed(fn, reps=10):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


t = timed(lambda: d.copy_(h, non_blocking=True))
print(f"H2D one copy of 192 MB: {t:.3f} ms = {192e6 / t / 1e6:.1f} GB/s")
chunk = n // 24


def chunks():
    for i in range(24):
        d[i * chunk:(i + 1) * chunk].copy_(h[i * chunk:(i + 1) * chunk], non_blocking=True)


t = timed(chunks)
print(f"H2D 24 chunks of 8 MB: {t:.3f} ms = {192e6 / t / 1e6:.1f} GB/s")


def two_streams():
    with torch.cuda.stream(s1):
        d[: n // 2].copy_(h[: n // 2], non_blocking=True)
    with torch.cuda.stream(s2):
        d[n // 2:].copy_(h[n // 2:], non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


t = timed(two_streams)
print(f"H2D two streams: {t:.3f} ms = {192e6 / t / 1e6:.1f} GB/s")
t = timed(lambda: ho.copy_(do, non_blocking=True))
print(f"D2H 64 MB: {t:.3f} ms = {64e6 / t / 1e6:.1f} GB/s")


def both():
    with torch.cuda.stream(s1):
        d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        ho.copy_(do, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


t = timed(both)
print(f"H2D 192 MB + concurrent D2H 64 MB: {t:.3f} ms (H2D alone 3.46 ms at 55.5 GB/s)")
