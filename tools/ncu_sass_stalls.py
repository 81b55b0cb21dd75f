"""Stall reasons and per-opcode instruction/stall shares of one kernel from
`ncu -i REP --page source --csv --print-source=sass -k KERNEL` output (CSV file)."""
import csv, collections, re, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
S, I = ix["Warp Stall Sampling (All Samples)"], ix["Instructions Executed"]
tot_s = sum(float(r[S] or 0) for r in data)
tot_i = sum(float(r[I] or 0) for r in data)
reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
op_s, op_i, rs = collections.Counter(), collections.Counter(), collections.Counter()
for r in data:
    m = re.match(r'(@!?U?P\w+\s+)?([A-Z0-9_.]+)', r[1].strip())
    op = m.group(2).split('.')[0] if m else r[1].strip()
    op_s[op] += float(r[S] or 0)
    op_i[op] += float(r[I] or 0)
    for h in reasons:
        rs[h] += float(r[ix[h]] or 0)
print(f"stall samples {tot_s:.0f}, warp instructions {tot_i:.4g}")
print("stall reasons (share of samples):")
for h, v in rs.most_common():
    if v: print(f"  {h[6:]:20s} {100 * v / tot_s:6.2f}%")
print("opcodes (share of instructions / of stall samples):")
for op, v in op_i.most_common(30):
    print(f"  {op:10s} inst {100 * v / tot_i:6.2f}%  stalls {100 * op_s[op] / tot_s:6.2f}%")
print("top stalled instructions:")
for i in sorted(range(len(data)), key=lambda i: -float(data[i][S] or 0))[:15]:
    r = data[i]
    rr = sorted(((float(r[ix[h]] or 0), h[6:]) for h in reasons), reverse=True)[:2]
    print(f"  {100 * float(r[S]) / tot_s:5.2f}%  {r[1].strip()[:50]:50s} {rr}")
