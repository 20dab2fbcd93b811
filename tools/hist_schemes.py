"""Ceiling table of 256-bin histogram counting schemes on one B200.

    python tools/hist_schemes.py [--gib 1] [--out profiles/r02/hist_schemes.json]

Builds tools/hist_schemes.cu with nvcc into /tmp, streams --gib GiB of bytes (uniform
U{0..255} and 90 %-skewed, as the cfg5 hist256 VPs) through each scheme at its full
occupancy grid, checks the counts against torch.bincount and reports device-timed GB/s
(CUDA events, 10 launches after 2 warm-ups), the fraction of measured HBM, and bytes per
SM-clock at the max SM clock.
"""
import argparse
import ctypes
import json
import os
import subprocess
import sys

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SCHEMES = ["lane_replicated_atoms", "match_any_aggregated", "private_u16_lds_sts", "private_u8_lds_sts",
           "shared_atoms_one_table"]


def build():
    so = "/tmp/hist_schemes.so"
    src = os.path.join(HERE, "hist_schemes.cu")
    if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-shared", "-Xcompiler", "-fPIC", "-o", so, src])
    L = ctypes.CDLL(so)
    L.hs_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int,
                         ctypes.c_void_p]
    L.hs_blocks_per_sm.argtypes = [ctypes.c_int]
    return L


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gib", type=float, default=1.0)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02", "hist_schemes.json"))
    args = ap.parse_args()
    L = build()
    torch.cuda.set_device(0)
    props = torch.cuda.get_device_properties(0)
    sms = props.multi_processor_count
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}
    n = int(args.gib * (1 << 30)) // 16 * 16
    g = torch.Generator(device="cuda").manual_seed(5)
    data = {"uniform": torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda", generator=g)}
    sk = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda", generator=g)
    hot = torch.rand(n, device="cuda", generator=g) < 0.9
    sk[hot] = 77
    data["skewed90"] = sk
    del hot
    counts = torch.zeros(256, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()
    rows = []
    for si, name in enumerate(SCHEMES):
        bps = L.hs_blocks_per_sm(si)
        grid = max(1, bps) * sms
        for dname, d in data.items():
            want = torch.bincount(d, minlength=256).to(torch.int64)
            ok = True
            ts = []
            for it in range(12):
                counts.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                rc = L.hs_run(si, d.data_ptr(), n, counts.data_ptr(), grid, stream.cuda_stream)
                e1.record(stream)
                torch.cuda.synchronize()
                assert rc == 0, (name, rc)
                if it >= 2:
                    ts.append(e0.elapsed_time(e1) / 1e3)
                if it == 2:
                    ok = bool(torch.equal(counts.to(torch.int64), want))
            t = sorted(ts)[len(ts) // 2]
            gbs = n / t / 1e9
            row = {"scheme": name, "data": dname, "blocks_per_sm": bps, "grid": grid, "bytes": n,
                   "median_s": t, "gbs": gbs, "frac_of_measured_hbm": gbs / float(peaks["hbm_gbs"]),
                   "bytes_per_sm_clk_at_max": gbs * 1e9 / (sms * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6),
                   "counts_exact": ok}
            rows.append(row)
            print(json.dumps(row), flush=True)
    out = {"gpu": props.name, "sms": sms, "hbm_gbs_measured": peaks["hbm_gbs"], "target_gbs_70pct": 0.7 * float(
        peaks["hbm_gbs"]), "rows": rows}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    sys.exit(main())
