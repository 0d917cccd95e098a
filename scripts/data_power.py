"""Device time / power of the tensor GEMM step for different input distributions (dev tool)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402
import synth  # noqa: E402

n = 4000
dev = torch.device("cuda", 0)
cases = {
    "torch.rand[0,1)": [torch.rand(n, n, device=dev) for _ in range(3)],
    "U[-1,1) numpy": [torch.from_numpy(synth.uniform((n, n), s)).to(dev) for s in (2, 0, 1)],
}
d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, 2)
tiles = (128, 256, 32)
for name, bufs in cases.items():
    r = E.sweep(d, [tiles], bufs, device=0, warmup=5, min_window_s=2.0)[0]
    print(f"{name:18s} {r.ms_per_run:.3f} ms  {r.tflops:.1f} TF  {r.avg_watts:.0f} W  {r.gflops_per_watt:.1f} GF/W  sm {r.sm_mhz_median:.0f} MHz")
d.set_scalars(1.5, 1.0)
for name, bufs in cases.items():
    r = E.sweep(d, [tiles], bufs, device=0, warmup=5, min_window_s=2.0)[0]
    print(f"beta=1 {name:11s} {r.ms_per_run:.3f} ms  {r.tflops:.1f} TF  {r.avg_watts:.0f} W  {r.gflops_per_watt:.1f} GF/W  sm {r.sm_mhz_median:.0f} MHz")
