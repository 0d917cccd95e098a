"""e2e (eatss_run_host, pinned host buffers) of gemm N=4000 at several row-block counts."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402
import synth  # noqa: E402

N = 4000
A = torch.from_numpy(synth.uniform((N, N), 0)).pin_memory()
B = torch.from_numpy(synth.uniform((N, N), 1)).pin_memory()
C = torch.from_numpy(synth.uniform((N, N), 2)).pin_memory()
d = E.desc_builtin("gemm", (N, N, N))
d.set_scalars(1.5, 1.2)
gpu = E.gpu_params_query(0)
tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=2)
d.set_exec(split_pct=50, engine=2)
s = torch.cuda.current_stream()
for rb in (1, 4, 8, 16, 32):
    for _ in range(2):
        E.run_host(d, tiles, [C, A, B], rb, s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(10):
        E.run_host(d, tiles, [C, A, B], rb, s)
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print(f"row_blocks {rb}: {ms:.3f} ms  {2 * N ** 3 / (ms * 1e-3) / 1e12:.2f} TFLOP/s  "
          f"H2D {192e6 / (ms * 1e-3) / 1e9:.1f} GB/s-equivalent", flush=True)
