"""Executed fp64 FLOPs of a kernel from an ncu --set full report:
2*DFMA + DADD + DMUL thread instructions (per-cycle sums x elapsed cycles)."""
import csv, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
points = float(sys.argv[3]) if len(sys.argv) > 3 else None
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "-k", "regex:" + kern],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, units = rows[0], rows[1]
for r in rows[2:]:
    g = lambda k: float(r[hdr.index(k)].replace(",", ""))
    cyc = g("sm__cycles_elapsed.avg") if "sm__cycles_elapsed.avg" in hdr else None
    t_ms = g("gpu__time_duration.sum")
    fl = 0.0
    for op, w in (("dfma", 2), ("dadd", 1), ("dmul", 1)):
        fl += w * g(f"smsp__sass_thread_inst_executed_op_{op}_pred_on.sum.per_cycle_elapsed") * cyc
    print(f"{r[hdr.index('Kernel Name')][:40]}: time {t_ms:.3f} ms, cycles {cyc:.4g}, "
          f"fp64 flops {fl:.4g}, {fl / (t_ms * 1e-3) / 1e12:.2f} TFLOP/s" +
          (f", {fl / points:.0f} flop/point" if points else ""))
