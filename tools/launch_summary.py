"""Per-kernel totals of an ncu launch list (`ncu --metrics gpu__time_duration.sum --csv`):
python tools/launch_summary.py launches.csv [title] [--until NAME]
(--until: stop at the first launch whose kernel name contains NAME, e.g. the
bench's option-path runs after its timed regions: --until k_rhs_fi)"""
import collections, csv, sys
until = None
if "--until" in sys.argv:
    i = sys.argv.index("--until")
    until = sys.argv[i + 1]
    del sys.argv[i:i + 2]
rows = list(csv.reader(open(sys.argv[1])))
hdr, agg = None, collections.defaultdict(lambda: [0, 0.0])
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr) or r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
        continue
    if until and until in r[hdr.index("Kernel Name")]:
        break
    k = r[hdr.index("Kernel Name")].split("(")[0]
    v, u = float(r[hdr.index("Metric Value")].replace(",", "")), r[hdr.index("Metric Unit")]
    v = v / 1e6 if u == "ns" else (v / 1e3 if u == "us" else v)
    agg[k][0] += 1
    agg[k][1] += v
STEP = ("k_rhs", "k_gt_pre", "k_interp", "k_zip_rk4", "k_rk4", "k_pack")   # kernels of an RK4 stage
step = {k: v for k, v in agg.items() if any(s in k for s in STEP)}
tot = sum(v[1] for v in step.values())
print(sys.argv[2] if len(sys.argv) > 2 else "ncu launch list (cold-cache serialised per-launch times)")
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    sh = f"{100 * t / tot:5.1f}%" if k in step else "  -  "
    print(f"{k[:60]:60s} launches {n:4d}  total {t:9.3f} ms  mean {t / n:8.3f} ms  share {sh}")
