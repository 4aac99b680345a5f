"""Summarise an ncu source page (SASS) export: top stall instructions (optionally for lines executed
between --min and --max times) and the per-reason stall breakdown."""
import csv, subprocess, sys, argparse, collections
ap = argparse.ArgumentParser()
ap.add_argument("rep"); ap.add_argument("--top", type=int, default=40)
ap.add_argument("--min", type=int, default=0); ap.add_argument("--max", type=int, default=1 << 62)
a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
ia, isrc = h.index("Address"), h.index("Source")
iss = h.index("Warp Stall Sampling (All Samples)"); ie = h.index("Instructions Executed")
stall_cols = [k for k, n in enumerate(h) if n.startswith("stall_") or n.startswith("Stall")]
data = []
for r in rows[2:]:
    try:
        data.append((int(r[iss]), int(r[ie]), r[ia][-5:], r[isrc].strip(), r))
    except (ValueError, IndexError):
        pass
sel = [d for d in data if a.min <= d[1] <= a.max]
tot = sum(d[0] for d in sel) or 1
print("samples", tot, "insts", sum(d[1] for d in sel), "lines", len(sel))
for d in sorted(sel, reverse=True)[:a.top]:
    print(f"{d[0]:8d} {100*d[0]/tot:5.1f}% {d[1]:12d} {d[2]} {d[3][:100]}")
