"""Interleaved timing of ccsd_t_d1 dims-48 tensor/SIMT variants on one set of buffers (dev tool)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402

n = int(os.environ.get("N", "48"))
dims = (int(os.environ.get("H3", n)),) + (n,) * 6
d = E.desc_builtin("ccsd_t_d1", dims)
bufs = [torch.rand(d.buffer_elems(i), device="cuda") * 2 - 1 for i in range(3)]
flops = d.flops
variants = [(2, t) for t in [(1, 1, 1, 48, 2, 48, 48), (1, 2, 1, 48, 2, 48, 48), (1, 2, 2, 48, 1, 48, 48),
                             (1, 1, 2, 48, 1, 48, 48)]]
if os.environ.get("SIMT"):
    variants.append((1, (4, 4, 4, 4, 4, 32, 4)))
res = {}
for rep in range(3):
    for eng, t in variants:
        d.set_exec(50, eng, time_kernels=1)
        E.run(d, t, bufs)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for _ in range(3):
            E.run(d, t, bufs)
        e.record(); torch.cuda.synchronize()
        ms = s.elapsed_time(e) / 3
        k = E.last_kernel_ms(d)[0]
        res.setdefault((eng, t), []).append((ms, k))
for (eng, t), v in res.items():
    ms = min(x[0] for x in v); k = min(x[1] for x in v)
    gb = (2 * 4 * d.buffer_elems(0)) / 1e9
    print(f"engine {eng} tiles {t}: call {ms:.2f} ms  kernel {k:.2f} ms  {gb / k:.2f} TB/s  {flops / k / 1e9:.1f} TF  "
          f"all={[round(x[0], 2) for x in v]}")
