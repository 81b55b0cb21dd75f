"""Fit the ringdown of an extracted Psi_4 mode (tools/evolve.py output):
A e^{-gamma t} cos(omega t + phi) on a window after the mode's peak, compared
with the fundamental l = 2 quasi-normal mode of a Schwarzschild black hole of
mass M (M omega = 0.37367, M gamma = 0.08896; Leaver 1985).

    python tools/ringdown_fit.py profiles/r2o_waveform_c3.txt [column=Re C22] [t0_offset] [width]
"""
import sys

import numpy as np
from scipy.optimize import curve_fit

path = sys.argv[1]
col = int(sys.argv[2]) if len(sys.argv) > 2 else 1   # 1: Re C22, 2: Im C22, 3: |C20|, 6: Re C20
off = float(sys.argv[3]) if len(sys.argv) > 3 else 3.0
width = float(sys.argv[4]) if len(sys.argv) > 4 else 35.0
rows = []
for line in open(path):
    parts = line.split()
    if len(parts) < 6 or line.startswith("#"):
        continue
    try:
        rows.append([float(x) for x in parts])
    except ValueError:
        continue
n = min(len(r) for r in rows)
d = np.array([r[:n] for r in rows])
t, y = d[:, 0], d[:, col]
ip = int(np.argmax(np.abs(y)))
sel = (t >= t[ip] + off) & (t <= t[ip] + off + width)
f = lambda tt, a, g, w, p: a * np.exp(-g * (tt - t[ip])) * np.cos(w * (tt - t[ip]) + p)
p0 = [abs(y[ip]), 0.09, 0.37, 0.0]
best = None
for ph in np.linspace(-np.pi, np.pi, 8, endpoint=False):
    try:
        popt, _ = curve_fit(f, t[sel], y[sel], p0=[p0[0], p0[1], p0[2], ph], maxfev=20000)
    except RuntimeError:
        continue
    res = np.sum((f(t[sel], *popt) - y[sel]) ** 2)
    if best is None or res < best[0]:
        best = (res, popt)
res, (a, g, w, p) = best
rel = np.sqrt(res / np.sum(y[sel] ** 2))
print(f"peak of column {col} at t = {t[ip]:.2f} M (|y| = {abs(y[ip]):.3e}); fit window "
      f"[{t[ip] + off:.1f}, {t[ip] + off + width:.1f}] M, {sel.sum()} samples, rel. residual {rel:.3f}")
print(f"M omega = {abs(w):.4f} (Schwarzschild l=2 n=0: 0.3737), M gamma = {g:.4f} (0.0890)")
