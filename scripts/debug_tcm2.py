import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["EATSS_TCM_DEBUG"] = "1"
import paper_conf_cgo_jayaweerakwk24_b200 as E
np.set_printoptions(linewidth=220, suppress=True)
M, N, K = 128, 32, 32
A = (np.arange(M)[:, None] * 1000 + np.arange(K)[None, :]).astype(np.float32)   # A[i][k] = 1000 i + k
B = (np.arange(K)[:, None] * 100 + np.arange(N)[None, :] + 0.5).astype(np.float32)  # B[k][j] = 100 k + j + .5
d = E.desc_builtin("gemm", (M, N, K)); d.set_scalars(1.0, 0.0); d.set_exec(50, 2)
C = torch.zeros(M, N, device="cuda")
E.run(d, (128, 32, 32), [C, torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()]); torch.cuda.synchronize()
c = C.cpu().numpy().ravel()
print("smem A words:", c[:48]); print("smem A words 32..: ", c[32:64])
print("smem B words:", c[256:256 + 48])
ref = A.astype(np.float64) @ B.astype(np.float64)
print("rows 16..19 of C:", C.cpu().numpy()[16:20, :6]); print("ref:", ref[16:20, :6])
