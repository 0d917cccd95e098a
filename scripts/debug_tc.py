"""Debug helper: tensor engine vs an fp64 torch matmul, error map per tile (dev only)."""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4000
tiles = tuple(int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "16,1024,16").split(","))
g = torch.Generator(device="cuda").manual_seed(0)
A = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
B = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
C0 = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
ref = 1.5 * (A.double() @ B.double()) + 1.2 * C0.double()
for eng in (1, 2):
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, eng)
    C = C0.clone()
    E.run(d, tiles, [C, A, B]); torch.cuda.synchronize()
    err = (C.double() - ref)
    rel = err.norm() / ref.norm()
    Ti, Tj = tiles[0], tiles[1]
    bad = (err.abs() > 1e-3 * ref.abs().max())
    print(f"engine {eng}: normwise {rel.item():.3e}, bad entries {bad.sum().item()}")
    if bad.any():
        idx = bad.nonzero()
        ti = (idx[:, 0] // Ti).unique(); tj = (idx[:, 1] // Tj).unique()
        print("  bad i-tiles", ti[:20].tolist(), "count", len(ti), " bad j-tiles", tj.tolist())
        print("  bad i-rows within tile", (idx[:, 0] % Ti).unique().tolist()[:20], " j within tile sample", (idx[:, 1] % Tj).unique()[:10].tolist())
