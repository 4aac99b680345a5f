"""Per-instruction hot path of an ncu source (SASS) export: instructions executed at least
--min times, in address order, with their stall samples; plus the stall-reason totals."""
import argparse, csv, subprocess
ap = argparse.ArgumentParser()
ap.add_argument("rep"); ap.add_argument("--min", type=float, default=5e5)
ap.add_argument("--reasons", action="store_true")
a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
ie, iss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
ia, isrc = h.index("Address"), h.index("Source")
st = [k for k, n in enumerate(h) if n.startswith("stall_") and "Not Issued" not in n]
tot = {h[k]: 0 for k in st}
n_hot = samp_hot = samp_all = 0
for r in rows[2:]:
    try:
        e, s = int(r[ie]), int(r[iss])
    except (ValueError, IndexError):
        continue
    samp_all += s
    for k in st:
        try:
            tot[h[k]] += int(r[k])
        except ValueError:
            pass
    if e >= a.min:
        n_hot += 1; samp_hot += s
        if not a.reasons:
            top = max(st, key=lambda k: int(r[k]) if r[k].isdigit() else 0)
            print(f"{r[ia][-5:]} {e:10d} {s:7d} {h[top][6:]:>14s}  {r[isrc].strip()[:80]}")
print(f"# hot instructions {n_hot}, samples hot {samp_hot} / all {samp_all}")
for k, v in sorted(tot.items(), key=lambda x: -x[1])[:12]:
    print(f"# {k:24s} {v}")
