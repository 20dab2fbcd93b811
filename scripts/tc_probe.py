"""Drive scripts/tc_micro.cu (scripts/libtcprobe.so): smem images + descriptors built here."""
import ctypes
import os
import sys

import numpy as np
import torch

L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libtcprobe.so"))
L.tc_probe.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_int, ctypes.c_int,
                       ctypes.c_void_p]


def idesc(kind="tf32", a_major=0, b_major=0, N=256, M=128):
    fmt = 2 if kind == "tf32" else 1  # TF32=2, BF16=1
    return (1 << 4) | (fmt << 7) | (fmt << 10) | (a_major << 15) | (b_major << 16) | ((N >> 3) << 17) | ((M >> 4) << 24)


def desc(off, lbo, sbo, layout=2, version=1):
    return ((off >> 4) & 0x3FFF) | (((lbo >> 4) & 0x3FFF) << 16) | (((sbo >> 4) & 0x3FFF) << 32) | (version << 46) | (layout << 61)


def put_kmajor_sw128(img, base, X, esize):
    """X: rows x (128/esize) elements, each row 128 B, 128-B swizzle within 8-row atoms."""
    R, C = X.shape
    per = 16 // esize
    raw = X.view(np.uint8).reshape(R, C * esize)
    for r in range(R):
        for ch in range(8):
            dst = base + r * 128 + ((ch ^ (r % 8)) * 16)
            img[dst:dst + 16] = raw[r, ch * 16:(ch + 1) * 16]


def put_mnmajor_sw128(img, base, B):
    """B: K x N fp32 (N contiguous): 32-col blocks of K rows x 128 B, swizzled."""
    K, N = B.shape
    raw = B.view(np.uint8).reshape(K, N * 4)
    for j in range(N // 32):
        for k in range(K):
            for ch in range(8):
                dst = base + j * (K * 128) + k * 128 + ((ch ^ (k % 8)) * 16)
                img[dst:dst + 16] = raw[k, j * 128 + ch * 16: j * 128 + (ch + 1) * 16]


def put_kmajor_interleave(img, base, X, esize):
    """SWIZZLE_NONE K-major: 8-row x 16-B core matrices; k-cores adjacent (LBO=128), m-groups at SBO."""
    R, C = X.shape
    raw = X.view(np.uint8).reshape(R, C * esize)
    kc = C * esize // 16
    for r in range(R):
        for c in range(kc):
            dst = base + (r // 8) * (kc * 128) + c * 128 + (r % 8) * 16
            img[dst:dst + 16] = raw[r, c * 16:(c + 1) * 16]
    return kc * 128  # SBO


def run(img, descs, idv, nk, kind):
    timg = torch.from_numpy(img).cuda()
    td = torch.tensor(np.array(descs, dtype=np.uint64).view(np.int64)).cuda()
    tD = torch.zeros(128, 256, device="cuda")
    dbg = torch.zeros(8, dtype=torch.int32, device="cuda")
    rc = L.tc_probe(timg.data_ptr(), td.data_ptr(), tD.data_ptr(), idv, nk, kind, dbg.data_ptr())
    return rc, tD.cpu().numpy()


def report(name, rc, D, R):
    ok = np.isclose(D, R)
    print(f"{name}: rc={rc} ok={ok.mean():.4f} nan={np.isnan(D).mean():.3f} zeros={np.mean(D == 0):.3f}")
    if not ok.all():
        print("   D[0,:8]", D[0, :8].tolist(), " R[0,:8]", R[0, :8].tolist())
        print("   D[:6,0]", D[:6, 0].tolist(), " R[:6,0]", R[:6, 0].tolist())
    sys.stdout.flush()


g = np.random.default_rng(0)
A = g.integers(-3, 4, (128, 32)).astype(np.float32)
B = g.integers(-3, 4, (32, 256)).astype(np.float32)
R1, R4 = A[:, :8] @ B[:8], A @ B

# E1: A K-major SW128, B MN-major SW128 (what libsvp does)
img = np.zeros(65536, np.uint8)
put_kmajor_sw128(img, 0, A, 4)
put_mnmajor_sw128(img, 16384, B)
for nk, R in ((1, R1), (4, R4)):
    d = []
    for kk in range(nk):
        d += [desc(kk * 32, 16, 1024), desc(16384 + kk * 1024, 4096, 1024)]
    report(f"E1 tf32 A-K B-MN nk={nk}", *run(img, d, idesc("tf32", 0, 1), nk, 0), R)

# E2: both K-major SW128 (B^T rows)
img = np.zeros(65536, np.uint8)
put_kmajor_sw128(img, 0, A, 4)
put_kmajor_sw128(img, 16384, np.ascontiguousarray(B.T), 4)
for ver in (1, 0):
    for nk, R in ((1, R1), (4, R4)):
        d = []
        for kk in range(nk):
            d += [desc(kk * 32, 16, 1024, version=ver), desc(16384 + kk * 32, 16, 1024, version=ver)]
        report(f"E2 tf32 both K-major SW128 ver={ver} nk={nk}", *run(img, d, idesc("tf32", 0, 0), nk, 0), R)

# E4: SWIZZLE_NONE K-major both
img = np.zeros(65536, np.uint8)
sboA = put_kmajor_interleave(img, 0, A, 4)
sboB = put_kmajor_interleave(img, 16384, np.ascontiguousarray(B.T), 4)
for nk, R in ((1, R1), (4, R4)):
    d = []
    for kk in range(nk):
        d += [desc(kk * 256, 128, sboA, layout=0), desc(16384 + kk * 256, 128, sboB, layout=0)]
    report(f"E4 tf32 K-major INTERLEAVE nk={nk}", *run(img, d, idesc("tf32", 0, 0), nk, 0), R)
    d = []
    for kk in range(nk):
        d += [desc(kk * 256, sboA, 128, layout=0), desc(16384 + kk * 256, sboB, 128, layout=0)]
    report(f"E4' (lbo/sbo swapped) nk={nk}", *run(img, d, idesc("tf32", 0, 0), nk, 0), R)

# E6: tf32 B MN-major with the 32-B-atom 128-B swizzle (LayoutType SWIZZLE_128B_BASE32B = 1)
def put_mnmajor_sw128_32b(img, base, B):
    K, N = B.shape
    raw = B.view(np.uint8).reshape(K, N * 4)
    for j in range(N // 32):
        for k in range(K):
            for g in range(4):
                dst = base + j * (K * 128) + k * 128 + ((g ^ (k % 4)) * 32)
                img[dst:dst + 32] = raw[k, j * 128 + g * 32: j * 128 + (g + 1) * 32]


img = np.zeros(65536, np.uint8)
put_kmajor_sw128(img, 0, A, 4)
put_mnmajor_sw128_32b(img, 16384, B)
for (lbo, sbo) in ((4096, 512), (512, 4096), (4096, 1024)):
    for nk, R in ((1, R1), (4, R4)):
        d = []
        for kk in range(nk):
            d += [desc(kk * 32, 16, 1024), desc(16384 + kk * 1024, lbo, sbo, layout=1)]
        report(f"E6 tf32 A-K B-MN SW128_BASE32B lbo={lbo} sbo={sbo} nk={nk}", *run(img, d, idesc("tf32", 0, 1), nk, 0), R)

# E5: bf16, both K-major SW128
Ab = torch.from_numpy(g.integers(-3, 4, (128, 64)).astype(np.float32)).to(torch.bfloat16)
Bb = torch.from_numpy(g.integers(-3, 4, (64, 256)).astype(np.float32)).to(torch.bfloat16)
img = np.zeros(65536, np.uint8)
put_kmajor_sw128(img, 0, Ab.view(torch.int16).numpy(), 2)
put_kmajor_sw128(img, 16384, Bb.t().contiguous().view(torch.int16).numpy(), 2)
Af, Bf = Ab.float().numpy(), Bb.float().numpy()
for nk in (1, 4):
    d = []
    for kk in range(nk):
        d += [desc(kk * 32, 16, 1024), desc(16384 + kk * 32, 16, 1024)]
    report(f"E5 bf16 both K-major SW128 nk={nk}", *run(img, d, idesc("bf16", 0, 0), nk, 1), Af[:, :16 * nk] @ Bf[:16 * nk])
