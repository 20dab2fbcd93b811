"""Probe the TMEM layout of a kind::f16 A operand (scripts/tc_tmem_a.cu)."""
import ctypes
import os
import subprocess
import sys

import numpy as np
import torch

HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "libtcprobe_ta.so")
subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-shared", "-Xcompiler", "-fPIC",
                "-o", so, os.path.join(HERE, "tc_tmem_a.cu")], check=True)
L = ctypes.CDLL(so)
L.tc_probe_ta.argtypes = [ctypes.c_void_p] * 2 + [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32,
                                                  ctypes.c_int, ctypes.c_int]


def idesc(N=256, M=128, a_major=0, b_major=0):
    return (1 << 4) | (1 << 7) | (1 << 10) | (a_major << 15) | (b_major << 16) | ((N >> 3) << 17) | ((M >> 4) << 24)


def desc(off, lbo, sbo, layout=2):
    return ((off >> 4) & 0x3FFF) | (((lbo >> 4) & 0x3FFF) << 16) | (((sbo >> 4) & 0x3FFF) << 32) | (1 << 46) | (layout << 61)


def put_kmajor_sw128(img, base, X, esize):
    R, C = X.shape
    raw = X.view(np.uint8).reshape(R, C * esize)
    for r in range(R):
        for ch in range(8):
            dst = base + r * 128 + ((ch ^ (r % 8)) * 16)
            img[dst:dst + 16] = raw[r, ch * 16:(ch + 1) * 16]


g = np.random.default_rng(0)
K = 64
A = torch.from_numpy(g.integers(-3, 4, (128, K)).astype(np.float32)).to(torch.bfloat16)
B = torch.from_numpy(g.integers(-3, 4, (K, 256)).astype(np.float32)).to(torch.bfloat16)
Af, Bf = A.float().numpy(), B.float().numpy()
img = np.zeros(65536, np.uint8)
put_kmajor_sw128(img, 0, B.t().contiguous().view(torch.int16).numpy(), 2)  # 256 rows x 64 k = 32 KiB
a16 = A.view(torch.int16).numpy().view(np.uint16).astype(np.uint32)
layouts = {
    # column c of lane m = (k = 2c | k = 2c+1 << 16)
    "pairs_lo_even": (a16[:, 0::2] | (a16[:, 1::2] << 16)),
    "pairs_hi_even": (a16[:, 1::2] | (a16[:, 0::2] << 16)),
}
ok_any = False
for name, W in layouts.items():
    W = np.ascontiguousarray(W.astype(np.uint32))
    for nk in (1, 4):
        d = [desc(kk * 32, 16, 1024) for kk in range(nk)]
        td = torch.tensor(np.array(d, dtype=np.uint64).view(np.int64)).cuda()
        timg = torch.from_numpy(img).cuda()
        tA = torch.from_numpy(W.view(np.int32)).cuda()
        tD = torch.zeros(128, 256, device="cuda")
        rc = L.tc_probe_ta(timg.data_ptr(), tA.data_ptr(), W.shape[1], td.data_ptr(), tD.data_ptr(), idesc(), nk, 8)
        D = tD.cpu().numpy()
        R = Af[:, :16 * nk] @ Bf[:16 * nk]
        ok = np.isclose(D, R).mean()
        ok_any |= ok == 1.0
        print(f"{name} nk={nk}: rc={rc} ok={ok:.4f} nan={np.isnan(D).mean():.3f}")
        if ok < 1:
            print("   D[0,:6]", D[0, :6].tolist(), "R[0,:6]", R[0, :6].tolist())
        sys.stdout.flush()
print("ANY_OK", ok_any)
