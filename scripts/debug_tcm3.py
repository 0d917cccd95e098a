import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E
np.set_printoptions(linewidth=220, suppress=True, precision=1)
M, N, K = 128, 32, 32
A = (np.arange(M)[:, None] * 1 + np.arange(K)[None, :] * 0).astype(np.float32) % 7   # A[i][k] = i%7
B = (np.arange(K)[:, None] * 0 + np.arange(N)[None, :]).astype(np.float32)           # B[k][j] = j
ref = A.astype(np.float64) @ B.astype(np.float64)
for dbg in [1, 1 | 2, 1 | 4, 1 | 8, 1 | 4 | 8, 1 | 2 | 4]:
    os.environ["EATSS_TCM_DEBUG"] = str(dbg)
    d = E.desc_builtin("gemm", (M, N, K)); d.set_scalars(1.0, 0.0); d.set_exec(50, 2)
    C = torch.zeros(M, N, device="cuda")
    E.run(d, (128, 32, 32), [C, torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()]); torch.cuda.synchronize()
    c = C.cpu().numpy()
    print("dbg", dbg, "rows16-18:", c[16:19, :8].tolist(), " ok?", np.allclose(c[16:], ref[16:]))
print("ref rows16-18", ref[16:19, :8].tolist())
