"""Per-source-line warp-stall samples and instruction counts from an .ncu-rep."""
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
    s = float(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
    n = float(r[hdr.index("Instructions Executed")] or 0)
    agg[line][0] += s
    agg[line][1] += n
    agg[line][2] = r[1][:90]
tot = sum(v[0] for v in agg.values()) or 1
for line, (s, n, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{line:5d} {100*s/tot:6.2f}% stall-samples {n:14.0f} inst  {src}")
