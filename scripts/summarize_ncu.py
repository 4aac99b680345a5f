#!/usr/bin/env python3
"""Summarise ncu captures into profiles/<round>/ (committed evidence).

  python scripts/summarize_ncu.py --round r01 --launches gpurun_out/r01/launches_road24m.csv \
      --full road24m=gpurun_out/r01/prof_road24m.ncu-rep --full rmat24=gpurun_out/r01/prof_rmat24.ncu-rep

Writes profiles/<round>/launch_shares_<wl>.json, profiles/<round>/ncu_<wl>.json/.md and updates
profiles/ncu_traffic.json (dram read+write bytes per launch of the persistent kernel, used by
bench.py's roofline.traffic).
"""
import argparse, csv, collections, io, json, os, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_read.sum",
    "lts__t_sectors_op_write.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    # atomic throughput (claims: atom.or; leaf claims: red.or; stack control: atom.cas)
    "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", "lts__t_requests_srcunit_tex_op_atom_dot_cas.sum",
    "lts__t_requests_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_atom_dot_alu.avg.per_cycle_elapsed",
    "lts__t_sectors_srcunit_tex_op_atom_dot_alu.avg.peak_sustained",
    "lts__t_sectors_srcunit_tex_op_atom_dot_alu_lookup_hit.sum",
]


def unit_scale(unit):
    return {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
            "msecond": 1e-3, "second": 1.0}.get(unit, 1.0)


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = {}
    for r in rows[2:]:
        for i, name in enumerate(h):
            if name in METRICS:
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                res[name] = {"value": v, "unit": units[i]}
        break
    return res


def stall_reasons(rep, top=12):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, r = rows[0], rows[2]
    st = {}
    for i, name in enumerate(h):
        if name.startswith("smsp__average_warp_latency_issue_stalled_") or name.startswith("smsp__pcsamp_warps_issue_stalled_"):
            if name.endswith(".ratio") or name.endswith(".sum") or "pcsamp" in name:
                try:
                    st[name] = float(r[i].replace(",", ""))
                except ValueError:
                    pass
    return dict(sorted(st.items(), key=lambda kv: -kv[1])[:top])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r01")
    ap.add_argument("--launches", action="append", default=[])
    ap.add_argument("--full", action="append", default=[])
    a = ap.parse_args()
    outdir = os.path.join(ROOT, "profiles", a.round)
    os.makedirs(outdir, exist_ok=True)
    for path in a.launches:
        rows = list(csv.reader(open(path)))
        hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[hi]
        ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
        agg = collections.OrderedDict()
        for r in rows[hi + 1:]:
            if len(r) <= vi:
                continue
            k = r[ki].split("(")[0]
            ns = float(r[vi].replace(",", "")) * (1e3 if r[ui] == "usecond" else 1e6 if r[ui] == "msecond" else 1)
            agg.setdefault(k, []).append(ns)
        tot = sum(sum(v) for v in agg.values())
        shares = {k: {"launches": len(v), "avg_us": round(sum(v) / len(v) / 1e3, 3),
                      "total_ms": round(sum(v) / 1e6, 3), "share": round(sum(v) / tot, 4)} for k, v in agg.items()}
        wl = os.path.basename(path).replace("launches_", "").replace(".csv", "")
        json.dump({"source": path, "note": "ncu --metrics gpu__time_duration.sum --clock-control none "
                   "(cold-cache, serialised: compare shares, not absolutes)", "kernels": shares},
                  open(os.path.join(outdir, f"launch_shares_{wl}.json"), "w"), indent=1)
        print(wl, json.dumps(shares, indent=1))
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for spec in a.full:
        wl, rep = spec.split("=", 1)
        m = raw(rep)
        b = m["dram__bytes_read.sum"]["value"] * unit_scale(m["dram__bytes_read.sum"]["unit"]) + \
            m["dram__bytes_write.sum"]["value"] * unit_scale(m["dram__bytes_write.sum"]["unit"])
        st = stall_reasons(rep)
        rec = {"workload": wl, "source": rep, "metrics": m, "dram_bytes_per_launch": b, "stalls": st}
        json.dump(rec, open(os.path.join(outdir, f"ncu_{wl}.json"), "w"), indent=1)
        traffic[wl] = round(b)
        with open(os.path.join(outdir, f"ncu_{wl}.md"), "w") as f:
            f.write(f"# ncu --set full: dfs_persistent_kernel, workload {wl}\n\n| metric | value | unit |\n|---|---|---|\n")
            for k, v in m.items():
                f.write(f"| {k} | {v['value']:.6g} | {v['unit']} |\n")
            f.write(f"\nDRAM bytes per launch (read+write): {b / 1e6:.1f} MB\n\nTop stall metrics:\n\n")
            for k, v in st.items():
                f.write(f"- {k}: {v:.4g}\n")
        print(wl, "dram MB", round(b / 1e6, 1))
    json.dump(traffic, open(traffic_path, "w"), indent=1)


if __name__ == "__main__":
    main()
