"""conv-2d / mttkrp: host enqueue cost per eatss_run vs device time (is the bench's 10-call loop host-bound?)."""
import os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402

gpu = E.gpu_params_query(0)
for kind, dims in (("conv-2d", (8192, 5)), ("mttkrp", (512, 32, 512, 512))):
    d = E.desc_builtin(kind, dims)
    bufs = [torch.rand(d.buffer_elems(i), device="cuda") * 2 - 1 for i in range(d.num_buffers)]
    tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=1)
    d.set_exec(split_pct=50, engine=1)
    for iters in (10, 50, 10):
        E.run(d, tiles, bufs)
        torch.cuda.synchronize()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t = time.perf_counter(); s.record()
        for _ in range(iters):
            E.run(d, tiles, bufs)
        host = (time.perf_counter() - t) / iters * 1e3
        e.record(); torch.cuda.synchronize()
        print(f"{kind} iters {iters}: host {host:.3f} ms/call, device {s.elapsed_time(e) / iters:.3f} ms/call", flush=True)
    # device time of the kernel alone with the host out of the way: a graph-free burst after a sleep kernel
    torch.cuda._sleep(50_000_000)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(10):
        E.run(d, tiles, bufs)
    e.record(); torch.cuda.synchronize()
    print(f"{kind} queued behind a sleep: device {s.elapsed_time(e) / 10:.3f} ms/call", flush=True)
