"""Per-config results table from committed bench lines.

    python tools/baseline_table.py profiles/r02/bench/bench_cfg{1,2,3,4,5}.json
"""
import json
import sys


def fmt(x, nd=0):
    return "—" if x is None else (f"{x:,.{nd}f}")


def main(paths):
    rows = ["| config | jobs/s (device-resident) | ms/step | e2e jobs/s (host-resident) | e2e ms/step | "
            "vs B1 serial-sync | vs B2 serial-async | vs B3 serial-graph | dominant kernel: achieved / peak (frac) | "
            "memory-bound kernels, HBM frac | oracle on host cores (jobs/s, cores) | SM MHz |",
            "|---|---:|---:|---:|---:|---:|---:|---:|---|---:|---:|---:|"]
    for p in paths:
        d = json.load(open(p))
        r = d["roofline"]
        sp = d.get("speedup_vs_serial", {})
        cpu = d.get("cpu_baseline") or {}
        e2e = d.get("e2e") or {}
        rows.append(
            f"| {d['config']['workload'].split(':')[0]} | {fmt(d['value'])} | {d['ms_per_step']:.3f} | "
            f"{fmt(e2e.get('value'), 1)} | {fmt(e2e.get('ms_per_step'), 2)} | "
            f"{fmt(sp.get('B1_serial_sync'), 2)}× | {fmt(sp.get('B2_serial_async'), 2)}× | "
            f"{fmt(sp.get('B3_serial_graph'), 2)}× | {r['kernel'].split(' (')[0]}: {r['achieved']:.0f} / {r['peak']:.0f} "
            f"{r['unit']} ({r['frac']:.2f}) | "
            f"{fmt(d.get('hbm_frac_membound'), 3)} | {fmt(cpu.get('value'), 2)}, {cpu.get('cores', '—')} | "
            f"{(d.get('clocks') or {}).get('sm_mhz', '—')} |")
    print("\n".join(rows))


if __name__ == "__main__":
    main(sys.argv[1:])
