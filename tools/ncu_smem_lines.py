"""Per-source-line shared-memory wavefronts (and excess from bank conflicts) of one kernel in an .ncu-rep."""
import csv, subprocess, sys, collections
rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass",
                      "-k", "regex:" + kern], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = None
agg = collections.defaultdict(lambda: [0.0, 0.0, ""])
for r in rows:
    if len(r) > 4 and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr):
        continue
    try:
        line = int(r[0])
    except ValueError:
        continue
    w = float(r[hdr.index("L1 Wavefronts Shared")] or 0)
    x = float(r[hdr.index("L1 Wavefronts Shared Excessive")] or 0)
    agg[line][0] += w
    agg[line][1] += x
    agg[line][2] = r[1][:90]
tot = sum(v[0] for v in agg.values()) or 1
print(f"total smem wavefronts {tot:.4g}, excessive {sum(v[1] for v in agg.values()):.4g}")
for line, (w, x, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{line:5d} {100*w/tot:6.2f}% wf {w:12.4g} excess {x:12.4g}  {src}")
