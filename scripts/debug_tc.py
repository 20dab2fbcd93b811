"""Debug helper for the tcgen05 SGEMM: structured inputs -> print how C deviates."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402


def run(A, B, kernel="sgemm_tf32", impl=0):
    M, K = A.shape
    N = B.shape[1]
    ctx = svp.Context(num_gpus=1, sgemm_impl=impl)
    kid = ctx.register_kernel(kernel)
    tA, tB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    tC = torch.full((M, N), -7.0, device="cuda")
    ctx.submit(0, kid, svp.args_sgemm(M, N, K), [(tA.data_ptr(), A.nbytes, 1, 0), (tB.data_ptr(), B.nbytes, 1, 0),
                                                (tC.data_ptr(), tC.numel() * 4, 2, 0)])
    ctx.flush()
    C = tC.cpu().numpy()
    ctx.close()
    return C


def show(name, C, R):
    ok = np.isclose(C, R, rtol=1e-3, atol=1e-3)
    print(f"== {name}: exact-ish {ok.mean():.4f}  zeros {np.mean(C == 0):.4f}  untouched {np.mean(C == -7):.4f}")
    if not ok.all():
        bad = np.argwhere(~ok)
        print("   first bad:", [(int(i), int(j), float(C[i, j]), float(R[i, j])) for i, j in bad[:6]])
        print("   C[0,:40]", C[0, :40].round(2).tolist())
        print("   R[0,:40]", R[0, :40].round(2).tolist())
        print("   C[:20,0]", C[:20, 0].round(2).tolist())
        print("   R[:20,0]", R[:20, 0].round(2).tolist())


M, N, K = 128, 256, 32
ar = np.arange
for k0 in (0, 1, 7, 8, 31):
    A = np.zeros((M, K), np.float32); A[:, k0] = 1
    B = np.zeros((K, N), np.float32); B[k0, :] = ar(N)
    show(f"col-id k0={k0}", run(A, B), A @ B)
A = np.zeros((M, K), np.float32); A[:, 0] = ar(M)
B = np.zeros((K, N), np.float32); B[0, :] = 1
show("row-id", run(A, B), A @ B)
g = np.random.default_rng(0)
A = g.integers(-3, 4, (M, K)).astype(np.float32)
B = g.integers(-3, 4, (K, N)).astype(np.float32)
show("rand 128x256x32", run(A, B), A @ B)
A = g.integers(-3, 4, (256, 64)).astype(np.float32)
B = g.integers(-3, 4, (64, 512)).astype(np.float32)
show("rand 256x512x64", run(A, B), A @ B)
show("rand 256x512x64 3xtf32", run(A, B, "sgemm", 1), A @ B)
