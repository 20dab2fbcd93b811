"""Per-kernel SASS instruction summary of libsvp.so (cuobjdump -sass), the evidence that the
hot kernels are Blackwell-native (B200_PROFILING.md: UTC*MMA = tcgen05.mma, LDTM / STTM =
tcgen05.ld / st, UTMALDG / UBLKCP = TMA / bulk copies).

    python tools/sass_summary.py [--lib paper_conf_dac_jungc15_b200/libsvp.so] [--out profiles/r02/sass_summary.md]
"""
import argparse
import collections
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["UTCHMMA", "UTCQMMA", "UTCBAR", "LDTM", "STTM", "UTMALDG", "UBLKCP", "SYNCS", "FFMA2", "FFMA", "DMMA", "DFMA",
        "ATOMS", "MATCH", "LDG", "STG", "LDS", "STS", "MUFU", "F2FP", "BAR"]


def demangle(names):
    try:
        out = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.split("\n")
        return out[:len(names)]
    except Exception:
        return names


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lib", default=os.path.join(ROOT, "paper_conf_dac_jungc15_b200", "libsvp.so"))
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02", "sass_summary.md"))
    args = ap.parse_args()
    sass = subprocess.run(["cuobjdump", "-sass", args.lib], capture_output=True, text=True, check=True).stdout
    funcs = collections.OrderedDict()
    cur = None
    for line in sass.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            funcs[cur] = collections.Counter()
            continue
        m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", line)
        if m and cur:
            op = m.group(2)
            base = op.split(".")[0]
            funcs[cur]["_total"] += 1
            for k in KEYS:
                if base == k or (k in ("UTCHMMA", "UTCQMMA") and base.startswith(k)):
                    funcs[cur][k] += 1
                    if op.startswith("UTCHMMA.2CTA") or op.startswith("UTCQMMA.2CTA"):
                        funcs[cur]["(2CTA)"] += 1
                    break
    names = demangle(list(funcs))
    rows = ["| kernel | instrs | " + " | ".join(KEYS + ["(2CTA)"]) + " |",
            "|---|---:|" + "---:|" * (len(KEYS) + 1)]
    for (mangled, cnt), name in zip(funcs.items(), names):
        short = re.sub(r"\(.*", "", name).replace("svp::", "")
        rows.append(f"| `{short}` | {cnt['_total']} | " + " | ".join(str(cnt[k]) if cnt[k] else "" for k in KEYS + ["(2CTA)"]) + " |")
    hdr = (f"# SASS instruction summary of `{os.path.relpath(args.lib, ROOT)}`\n\n"
           "Static counts per kernel (cuobjdump -sass; `tools/sass_summary.py`). UTCHMMA / UTCQMMA = "
           "tcgen05.mma (`(2CTA)`: cta_group::2), LDTM / STTM = tcgen05.ld / st, UTMALDG = TMA tensor "
           "loads, UBLKCP = bulk copies, SYNCS = mbarrier ops, FFMA2 = fma.rn.f32x2.\n\n")
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        f.write(hdr + "\n".join(rows) + "\n")
    print(args.out)


if __name__ == "__main__":
    main()
