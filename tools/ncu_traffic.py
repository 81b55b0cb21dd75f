"""Per-kernel DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum, bytes per
launch) from one `ncu --set full` capture, written as JSON for bench.py's
roofline "traffic" field:  python tools/ncu_traffic.py rep.ncu-rep path out.json"""
import csv, json, os, subprocess, sys
rep, path, outp = sys.argv[1], sys.argv[2], sys.argv[3]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, units = rows[0], rows[1]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
# (the bench's "rhs" class brackets the whole RHS launch: k_gt_pre + k_rhs)
names = {"k_gt_pre": "rhs", "k_rhs": "rhs", "k_unzip": "unzip", "k_interp": "interp",
         "k_zip_rk4": "zip_rk4", "k_rk4": "zip_rk4"}
res = json.load(open(outp)) if os.path.exists(outp) else {}
res[path] = {}
last = {}
for r in rows[2:]:
    kn = r[hdr.index("Kernel Name")]
    k = next((k for k in names if k in kn), None)
    if k is None:
        continue
    tot = 0.0
    for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        i = hdr.index(m)
        tot += float(r[i].replace(",", "")) * scale[units[i]]
    last[k] = tot   # (last launch of each kernel wins)
for k, v in last.items():
    res[path][names[k]] = res[path].get(names[k], 0.0) + v
res["source"] = "ncu --set full --clock-control none, C3 on 1 B200 (profiles/)"
json.dump(res, open(outp, "w"), indent=1)
print(json.dumps(res, indent=1))
