#!/usr/bin/env python3
"""One-page markdown summary of an `ncu --set full` capture (one kernel launch).

    python scripts/ncu_md.py <capture.ncu-rep | raw.csv> <out.md> --title "..." [--traffic-key road24m]

Reads the raw page (ncu -i ... --page raw --csv, or an already extracted CSV), writes the key
throughput / occupancy / traffic metrics and the top warp-stall reasons, and with --traffic-key
records dram__bytes_read.sum + dram__bytes_write.sum in profiles/ncu_traffic.json (bench.py's
roofline.traffic).
"""
import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic",
    "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", "lts__t_requests_srcunit_tex_op_atom_dot_cas.sum",
    "lts__t_requests_srcunit_tex_op_red.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def load(path):
    if path.endswith(".csv"):
        text = open(path).read()
    else:
        text = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(text)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}


def num(s):
    return float(s.replace(",", "")) if s not in ("", "n/a") else float("nan")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("src")
    ap.add_argument("out")
    ap.add_argument("--title", default="")
    ap.add_argument("--traffic-key")
    a = ap.parse_args()
    d = load(a.src)
    lines = [f"# ncu --set full: {a.title}", "", f"Source: `{os.path.basename(a.src)}`; kernel "
             f"`{d.get('Kernel Name', ('?', ''))[0][:120]}`", "", "| metric | value | unit |", "|---|---|---|"]
    for k in KEYS:
        if k in d:
            lines.append(f"| {k} | {d[k][0]} | {d[k][1]} |")
    rd, wr = d.get("dram__bytes_read.sum"), d.get("dram__bytes_write.sum")
    traffic = None
    if rd and wr:
        traffic = num(rd[0]) * UNIT_SCALE.get(rd[1], 1) + num(wr[0]) * UNIT_SCALE.get(wr[1], 1)
        lines += ["", f"DRAM bytes per launch (read + write): {traffic / 1e6:.1f} MB"]
    st = [(k, num(v[0])) for k, v in d.items() if "pcsamp_warps_issue_stalled" in k and not k.endswith("not_issued")]
    st.sort(key=lambda kv: -kv[1])
    tot = sum(v for _, v in st) or 1.0
    lines += ["", "Warp-stall samples (top 10, share of all stall samples):", ""]
    for k, v in st[:10]:
        lines.append(f"- {k.replace('smsp__pcsamp_warps_issue_stalled_', '')}: {v:.3g} ({100 * v / tot:.1f}%)")
    os.makedirs(os.path.dirname(os.path.abspath(a.out)), exist_ok=True)
    with open(a.out, "w") as f:
        f.write("\n".join(lines) + "\n")
    if a.traffic_key and traffic is not None:
        p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        t = json.load(open(p)) if os.path.exists(p) else {}
        t[a.traffic_key] = {"bytes": int(traffic), "source": os.path.relpath(os.path.abspath(a.out), ROOT)}
        with open(p, "w") as f:
            json.dump(t, f, indent=1)
    print(a.out, traffic)


if __name__ == "__main__":
    main()
