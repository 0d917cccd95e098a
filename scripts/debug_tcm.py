"""Debug the tcgen05 SS-GEMM with structured inputs (dev only)."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E
np.set_printoptions(linewidth=200, suppress=True)
def run(A, B, tiles):
    M, K = A.shape; N = B.shape[1]
    d = E.desc_builtin("gemm", (M, N, K)); d.set_scalars(1.0, 0.0); d.set_exec(50, 2)
    C = torch.zeros(M, N, device="cuda")
    E.run(d, tiles, [C, torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()]); torch.cuda.synchronize()
    return C.cpu().numpy()
M, N, K = 128, 32, 32
A = np.zeros((M, K), np.float32); A[np.arange(32), np.arange(32)] = 1
B = (np.arange(K)[:, None] * 100 + np.arange(N)[None, :]).astype(np.float32)
C = run(A, B, (128, 32, 32))
print("identity-A test: max err", np.abs(C[:32] - B).max(), " rows>=32 max", np.abs(C[32:]).max())
print(C[:6, :10]); print("expected"); print(B[:6, :10])
# one-hot in A column -> picks B row
A2 = np.zeros((M, K), np.float32); A2[:, 5] = 1
C2 = run(A2, B, (128, 32, 32)); print("A[:,5]=1 -> each row should be B[5]:", C2[0, :8], "vs", B[5, :8], " row 77:", C2[77, :8])
A3 = np.zeros((M, K), np.float32); A3[3, :] = 1
C3 = run(A3, B, (128, 32, 32)); print("A[3,:]=1 -> row 3 = colsum(B):", C3[3, :8], "vs", B.sum(0)[:8], " other rows max", np.abs(np.delete(C3, 3, 0)).max())
