"""Roofline-ceiling microbenchmarks on the GPU box (tooling; results -> profiles/).

    python tools/ubench.py [--out profiles/r01/ubench.json]

Builds tools/libubench.so (nvcc, sm_100a) if needed, then measures with CUDA events:
HBM streaming copy, shared-memory atomic rate (hist256's access pattern), FP32 FFMA
rate, and pinned PCIe H2D / D2H / bidirectional bandwidth.
"""
import argparse
import ctypes
import json
import os
import subprocess

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
SRC, LIB = os.path.join(HERE, "ubench.cu"), os.path.join(HERE, "libubench.so")


def build():
    if not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", "-o", LIB, SRC])
    return ctypes.CDLL(LIB)


def timed(fn, reps=5):
    s = torch.cuda.current_stream()
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / 1e3)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    L = build()
    vp = ctypes.c_void_p
    L.ub_copy.argtypes = [vp, vp, ctypes.c_size_t, ctypes.c_int, ctypes.c_int, vp]
    L.ub_atoms.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
    L.ub_ffma.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
    L.ub_atoms16.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
    L.ub_ffma2.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
    L.ub_dfma.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
    props = torch.cuda.get_device_properties(0)
    sms = props.multi_processor_count
    st = torch.cuda.current_stream().cuda_stream
    res = {"gpu": props.name, "sms": sms}

    n = 2 << 30
    a = torch.empty(n, dtype=torch.uint8, device="cuda")
    b = torch.empty(n, dtype=torch.uint8, device="cuda")
    for grid_mult in (4, 8, 16):
        t = timed(lambda: L.ub_copy(a.data_ptr(), b.data_ptr(), n, sms * grid_mult, 256, st))
        res[f"copy_gbs_grid{grid_mult}x"] = 2 * n / t / 1e9
    del a, b

    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    iters = 4096
    for blocks_per_sm in (4, 6):
        grid = sms * blocks_per_sm
        t = timed(lambda: L.ub_atoms(out.data_ptr(), iters, grid, 256, st))
        lanes = grid * 256 * iters * 4
        res[f"smem_atomics_per_s_{blocks_per_sm}cta"] = lanes / t
        res[f"smem_atomic_lanes_per_clk_per_sm_{blocks_per_sm}cta"] = lanes / t / sms / (props.clock_rate * 1e3) \
            if hasattr(props, "clock_rate") else None
    res["hist256_ceiling_gbs_if_atomic_bound"] = res["smem_atomics_per_s_6cta"] / 1e9
    sweep = {}
    for fn, name in ((L.ub_atoms, "u32"), (L.ub_atoms16, "u16x2")):
        for block in (256, 512):
            for bps in (1, 2, 3, 4, 6, 8):
                if block * bps > 2048:
                    continue
                grid = sms * bps
                t = timed(lambda: fn(out.data_ptr(), iters, grid, block, st))
                sweep[f"{name}_b{block}_x{bps}"] = round(grid * block * iters * 4 / t / 1e12, 3)
    res["smem_atomics_Tlanes_per_s_sweep"] = sweep

    f = torch.zeros(1, device="cuda")
    fi = 2000
    t = timed(lambda: L.ub_ffma(f.data_ptr(), fi, sms * 8, 256, st))
    res["ffma_tflops"] = sms * 8 * 256 * fi * 64 * 2 / t / 1e12
    t = timed(lambda: L.ub_ffma2(f.data_ptr(), fi, sms * 8, 256, st))
    res["ffma2_tflops"] = sms * 8 * 256 * fi * 64 * 2 * 2 / t / 1e12
    fd = torch.zeros(1, dtype=torch.float64, device="cuda")
    t = timed(lambda: L.ub_dfma(fd.data_ptr(), fi // 4, sms * 8, 256, st))
    res["dfma_tflops"] = sms * 8 * 256 * (fi // 4) * 64 * 2 / t / 1e12

    nb = 512 << 20
    h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    h2 = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nb, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nb, dtype=torch.uint8, device="cuda")
    res["pcie_h2d_gbs"] = nb / timed(lambda: d.copy_(h, non_blocking=True)) / 1e9
    res["pcie_d2h_gbs"] = nb / timed(lambda: h.copy_(d, non_blocking=True)) / 1e9
    s2 = torch.cuda.Stream()

    def both():
        d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s2)

    res["pcie_bidir_gbs"] = 2 * nb / timed(both) / 1e9
    line = json.dumps(res, indent=1)
    print(line)
    if args.out:
        with open(args.out, "w") as fo:
            fo.write(line + "\n")


if __name__ == "__main__":
    main()
