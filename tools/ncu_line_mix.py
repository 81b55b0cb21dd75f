"""Per-CUDA-line instruction mix (fp64 / shared-memory / other) of one kernel from
`ncu -i REP --page source --csv --print-source=cuda,sass -k KERNEL` output."""
import csv, re, collections, sys
rows = list(csv.reader(open(sys.argv[1])))
top_n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
hdr = next(r for r in rows if r and r[0] == "Line No")
I = hdr.index("Instructions Executed")
agg = collections.defaultdict(collections.Counter)
src, cur = {}, None
for r in rows[rows.index(hdr) + 1:]:
    if len(r) < len(hdr):
        continue
    if r[0].strip():
        try:
            cur = int(r[0])
        except ValueError:
            continue
        src[cur] = r[1].strip()[:80]
        continue
    m = re.match(r'(@!?U?P\w+\s+)?([A-Z0-9_]+)', r[3].strip())
    if not m or r[I] in ("", "-"):
        continue
    op = m.group(2)
    cls = "fp64" if op in ("DFMA", "DADD", "DMUL") else ("smem" if op in ("LDS", "STS", "LDSM") else "other")
    agg[cur][cls] += float(r[I])
tot = collections.Counter()
for c in agg.values():
    tot.update(c)
T = sum(tot.values())
print("warp instructions:", {k: f"{v:.3g} ({100 * v / T:.1f}%)" for k, v in tot.items()})
print("lines with the most non-fp64, non-smem instructions:")
for l, c in sorted(agg.items(), key=lambda x: -x[1]["other"])[:top_n]:
    print(f"{l:5d} other {c['other'] / 1e6:7.1f}M fp64 {c['fp64'] / 1e6:7.1f}M smem {c['smem'] / 1e6:6.1f}M  {src.get(l, '')}")
