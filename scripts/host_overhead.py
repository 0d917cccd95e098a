"""Host enqueue cost of one bench step vs its device time (development tool)."""
import os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402

n = 4000
bufs = [torch.rand(n, n, device="cuda") for _ in range(3)]
gpu = E.gpu_params_query(0)
for engine, mode in ((4, 3), (2, 2)):
    def step():
        d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2)
        tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=mode)
        d.set_exec(split_pct=50, engine=engine, time_kernels=1)
        E.run(d, tiles, bufs)
        return d
    for _ in range(5):
        step()
    torch.cuda.synchronize()
    K = 100
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t = time.perf_counter(); s.record()
    for _ in range(K):
        step()
    host = (time.perf_counter() - t) / K * 1e3
    e.record(); torch.cuda.synchronize()
    print(f"engine {engine}: host enqueue {host:.3f} ms/step, device {s.elapsed_time(e) / K:.3f} ms/step")
    # host cost with the device idle (a sync per step)
    t = time.perf_counter()
    for _ in range(20):
        step(); torch.cuda.synchronize()
    print(f"engine {engine}: step with sync {(time.perf_counter() - t) / 20 * 1e3:.3f} ms")
# the same descriptor reused (no per-step model / plan): the device-side cost of the call alone
d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2)
tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=3)
for tk in (1, 0):
    d.set_exec(split_pct=50, engine=4, time_kernels=tk)
    for _ in range(5):
        E.run(d, tiles, bufs)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t = time.perf_counter(); s.record()
    for _ in range(100):
        E.run(d, tiles, bufs)
    host = (time.perf_counter() - t) / 100 * 1e3
    e.record(); torch.cuda.synchronize()
    print(f"reused descriptor, time_kernels={tk}: host {host:.3f} ms/call, device {s.elapsed_time(e) / 100:.3f} ms/call")
