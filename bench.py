"""Benchmark: fp64 BSSN RK4 step on a Brill-Lindquist BBH octree (libdgr, B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl reference]
    python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N ...

Metric (BASELINE.json): "BSSN RHS fp64 GFLOP/s & RK4 step time (grid pts/s)".
`value` = unique grid points (DOFs) advanced by one full RK4 step per second,
summed over ranks (whole job), inputs resident in HBM.  Default workload:
configs[2], Brill-Lindquist q=1, levels 3..12, rho=2.5 (24,284 octants,
5.07M DOFs = 121.6M unknowns; the paper's 125M-unknown strong-scaling case,
P:L440) — the config the metric's "at 1/2/4/8 B200" is quoted on.  With N>1
the octree is partitioned along the Morton curve (strong scaling) and ghost
DOFs are exchanged with NCCL every RK stage.

One JSON line on rank 0 (the driver's contract).  L2 hygiene: every stage
streams the 10.2 GB patch buffer (>> 126 MB L2), so inputs are larger than L2.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "BSSN RHS fp64 GFLOP/s & RK4 step time (grid pts/s) at 1/2/4/8 B200"
UNIT = "grid-pts/s"

# Algorithmic work per unit:
UNZIP_BYTES_PER_OCT = 24 * (2197 + 216) * 8       # write every patch point, read every DOF once
ZIP_BYTES_PER_DOF_STAGE = 24 * 34                 # avg over the 4 stages of read k,u_n,acc / write acc,u_s
INTERP_BYTES_PER_SLOT = 24 * 8                     # write every slot once
INTERP_BYTES_PER_ELEM = 24 * 343 * 8 + 343 * 4    # read the element's nodal values once (+ o2s)
RHS_BYTES_PER_OCT = 24 * (2197 + 343) * 8         # patch read + rhs write (eq 21a denominator)
PAPER_FLOPS_PER_POINT = 5502 + 3998               # eq (21a) numerator per point, O_A from Q_L = 6.68
# executed fp64 FLOPs per interior point (2 DFMA + DADD + DMUL thread instructions from
# ncu sm__sass_thread_inst_executed_op_d{fma,add,mul}_pred_on, C3, 8,329,412 points;
# profiles/r3y_flops*.csv, round 2 final code): fused = k_gt_pre 976.5 + k_rhs
# 3,603.4 x 343/352 (k_rhs runs its 9 threads without a point through the same
# warp-wide code since the tensor-memory value store; their share is discounted;
# k_rhs now also applies the RK4 stage update, ~58 FLOP per point), two-pass =
# the single k_rhs 4,451.2 x 343/352.  (History: 4,411.4 / 4,356.0 before the
# round-2 session's TMEM / fused-update changes; round 1 5,358 / 5,265 before the
# Ricci / At^ij contraction-order and trace-free-once changes.)
RHS_EXEC_FLOPS_PER_POINT = {"fused": 976.5 + 3603.4 * 343 / 352, "two-pass": 4451.2 * 343 / 352}
# DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum) from one
# ncu --set full capture of the C3 workload on 1 GPU, per path
# (profiles/ncu_traffic_c3.json, written by tools/ncu_traffic.py)
_TRAFFIC_JSON = os.path.join(ROOT, "profiles", "ncu_traffic_c3.json")
NCU_TRAFFIC_C3 = json.load(open(_TRAFFIC_JSON)) if os.path.exists(_TRAFFIC_JSON) else {}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6650.0), d.get("sm_max_mhz", 1965.0), "measured"
    return 6650.0, 1965.0, "fallback"


class Clocks:
    """SM clock / event-reason sampling during the timed region (B200_PROFILING.md
    clocks line): NVML, else nvidia-smi."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.source = None
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

        def run_nvml(nv, h):
            # NVML directly: ~ms per query, so a sub-second timed region still
            # gets tens of samples (nvidia-smi takes ~0.3 s per call)
            names = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                     nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
            while not self._stop.is_set():
                try:
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    self.samples.append(
                        [str(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)),
                         str(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)),
                         str(nv.nvmlDeviceGetPowerUsage(h) / 1000.0), hex(r)]
                        + ["Active" if r & b else "Not Active" for b in names])
                except Exception:
                    pass
                self._stop.wait(0.02)

        def run():
            try:
                import pynvml as nv
                nv.nvmlInit()
                h = nv.nvmlDeviceGetHandleByIndex(int(self.index))
                self.source = "nvml"
                return run_nvml(nv, h)
            except Exception:
                self.source = "nvidia-smi"
            while not self._stop.is_set():
                try:
                    out = subprocess.run(["nvidia-smi", "-i", str(self.index),
                                          f"--query-gpu={q}", "--format=csv,noheader,nounits"],
                                         capture_output=True, text=True, timeout=5).stdout
                    f = [x.strip() for x in out.strip().split(",")]
                    if len(f) >= 8:
                        self.samples.append(f)
                except Exception:
                    pass
                self._stop.wait(0.2)

        self._t = threading.Thread(target=run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"],
                    "samples": 0}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if s[4 + i].lower().startswith("active")})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.samples), "source": self.source}


def _cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:  # noqa: BLE001
        pass
    return None


def cpu_baseline_oracle(cfg, n_sample=None, reps=1, one_core=True):
    """The oracle as it stands, on the host cores, on a bounded sample of the
    workload: element reconstruction (hanging points) for ALL octants, then
    octant-to-patch + RHS for a contiguous Morton range of octants spread over
    all cores (forked workers, 1 BLAS thread each, the oracle's own
    rk4._chunk_rhs); one RK4 step = 4 such stages over all octants,
    extrapolated linearly in the octant count.  Also a 1-core figure (one
    worker, a smaller sample)."""
    import multiprocessing as mp

    from oracle import bssn
    from oracle import rk4 as ork4
    from oracle import unzip as ouz
    from oracle.maps import OracleMesh
    from synth import initial
    cores = len(os.sched_getaffinity(0))
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords())
    ouz.padding_sources_cached(om, np.arange(1))           # maps: built once, not timed
    n_s = min(om.n_oct, n_sample or 24 * cores)
    start = int(np.random.default_rng(0).integers(0, om.n_oct - n_s + 1))

    def measure(n_s, workers, reps):
        bounds = np.linspace(start, start + n_s, 4 * workers + 1).astype(int)
        chunks = [(int(x), int(y)) for x, y in zip(bounds[:-1], bounds[1:]) if y > x]
        full, sample = [], []
        for _ in range(reps):
            t0 = time.perf_counter()
            E = ouz.elements(om, u)
            t1 = time.perf_counter()
            ork4._G.update(mesh=om, E=E, prm=bssn.Params())
            with mp.get_context("fork").Pool(workers) as pool:   # workers inherit _G by fork
                t2 = time.perf_counter()
                pool.map(ork4._chunk_rhs, chunks)
                t3 = time.perf_counter()
            ork4._G.clear()
            full.append(4.0 * ((t1 - t0) + (t3 - t2) * om.n_oct / n_s))
            sample.append(4.0 * ((t1 - t0) + (t3 - t2)))
        return float(np.median(full)), float(np.median(sample))

    step_s, sample_s = measure(n_s, cores, reps)
    res = {"value": om.n_dof / step_s, "unit": UNIT, "cores": cores, "kind": "oracle",
           "sample": (f"1 RK4 step = 4 x (hanging reconstruction for all {om.n_oct} octants + "
                      f"unzip+RHS of {n_s} Morton-contiguous octants on {cores} worker "
                      f"processes); timed {sample_s:.1f} s per step on the sample, "
                      f"scaled x{om.n_oct / n_s:.1f} in the RHS part to all {om.n_oct} octants"),
           "step_s": step_s, "sample_step_s": sample_s,
           "extrapolation_factor": om.n_oct / n_s, "sample_octants": n_s,
           "cpu_model": _cpu_model(),
           "numpy_threads": {k: os.environ.get(k) for k in
                             ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS")},
           "threads_per_worker": 1}
    if one_core:
        n1 = max(1, min(om.n_oct, 16))
        s1, _ = measure(n1, 1, 1)
        res["one_core"] = {"value": om.n_dof / s1, "unit": UNIT, "cores": 1,
                           "sample": f"{n1} octants on one worker, scaled to {om.n_oct}"}
    return res


def _nccl_summary(path):
    """Transport facts from NCCL_DEBUG=INFO (rank 0's log)."""
    if not path or not os.path.exists(path):
        return None
    txt = open(path, errors="replace").read()
    return {"log": path, "nvls": "NVLS" in txt and "NVLS multicast support is not available" not in txt,
            "p2p_nvlink": "via P2P" in txt, "lines": txt.count("\n")}


def run_reference(args, cfg):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cb = cpu_baseline_oracle(cfg, reps=args.warmup + args.steps, one_core=False)
    # ms_per_step is what one timed step took (the bounded sample); value is
    # the throughput that implies for the whole workload
    line = {"impl": "reference", "metric": METRIC, "value": cb["value"], "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": cb["sample_step_s"] * 1e3,
            "full_step_s_extrapolated": cb["step_s"],
            "extrapolation_factor": cb["extrapolation_factor"],
            "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic Brill-Lindquist",
            "config": {"workload": cfg.name + ": " + cfg.description},
            "cpu_baseline": {k: cb[k] for k in ("value", "unit", "cores", "kind", "sample",
                                                "cpu_model", "numpy_threads",
                                                "extrapolation_factor")},
            "e2e": {"value": cb["value"], "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c3")
    ap.add_argument("--impl", default="dgr", choices=["dgr", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-options", action="store_true",
                    help="skip the radiative-boundary / lopsided-advection step timings")
    ap.add_argument("--cpu-sample", type=int, default=None)
    ap.add_argument("--path", default="fused", choices=["fused", "two-pass"],
                    help="fused: patches gathered inside the RHS kernel; two-pass: unzip first")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    from synth import configs, initial
    cfg = configs.get(args.config)
    if args.impl == "reference":
        return run_reference(args, cfg)

    import torch
    import torch.distributed as dist

    import paper_conf_sc_fernandonhzsgb22_b200 as dgr

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    nccl_log = None
    if world > 1 and "NCCL_DEBUG" not in os.environ:
        # NCCL's transport choices (NVLink P2P, NVLS) for the JSON line; the log
        # goes to a file so rank 0's stdout stays one JSON line
        nccl_log = f"/tmp/dgr_nccl_{os.getpid()}.log"
        os.environ["NCCL_DEBUG"] = "INFO"
        os.environ["NCCL_DEBUG_FILE"] = nccl_log
    torch.cuda.set_device(local)
    nccl_id = None
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        obj = [bytes(torch.cuda.nccl.unique_id()) if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]

    octs = dgr.octree_build(cfg)
    mesh = dgr.Mesh(cfg, octs, rank=rank, nranks=world, nccl_id=nccl_id)
    mesh.set_fused(args.path == "fused")
    info = mesh.info
    xyz = mesh.dof_xyz_host()
    u = torch.zeros((24, mesh.dof_stride), dtype=torch.float64, device="cuda")
    u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz))
    dt = 0.25 * info["h_min"]
    prm = dgr.Params()

    # fp64 roofline denominator: DFMA microbenchmark on this device
    dfma_ms, dfma_fl = dgr.bench_dfma(148 * 8, 20000)
    dfma_tflops = dfma_fl / dfma_ms / 1e9

    def barrier():
        if world > 1:
            dist.barrier()

    for _ in range(args.warmup):
        mesh.rk4_step(u, dt, prm)
    torch.cuda.synchronize()
    launches_per_step = mesh.last_launch_count()   # libdgr kernels per step (graph or eager)

    # ---- timed region: device-resident state (one CUDA-graph launch per step
    # on one rank, DGR_OPT_GRAPH: captured during the warm-up)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    with Clocks(local) as clk:
        e0.record()
        for _ in range(args.steps):
            mesh.rk4_step(u, dt, prm)
        e1.record()
        torch.cuda.synchronize()
    barrier()
    ms = e0.elapsed_time(e1) / args.steps
    # ---- the same K steps again with CUDA events around every libdgr launch
    # (on its launching stream; eager launches): per-kernel times for the rooflines
    mesh.profile_read(reset=True)
    mesh.profile_enable(True)
    barrier()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(args.steps):
        mesh.rk4_step(u, dt, prm)
    e1.record()
    torch.cuda.synchronize()
    barrier()
    mesh.profile_enable(False)
    prof = mesh.profile_read(reset=True)
    ms_profiled = e0.elapsed_time(e1) / args.steps
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    n_dof = info["n_dof_global"]
    value = n_dof / (ms_max * 1e-3)
    finite = bool(torch.isfinite(u[:, :info["n_dof_owned"]]).all())

    # ---- a7: constraint diagnostics (not part of the RK4 step)
    cons = None
    if world == 1:
        # (a diagnostic: a failure here is reported in the line, not fatal to it)
        try:
            mesh.constraints(u)                               # allocates the patch buffer
            torch.cuda.synchronize()
            mesh.profile_read(reset=True)
            mesh.profile_enable(True)
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c0.record()
            for _ in range(3):
                _, norms = mesh.constraints(u)
            c1.record()
            torch.cuda.synchronize()
            mesh.profile_enable(False)
            cp = mesh.profile_read(reset=True)
            cons = {"ms_per_call": c0.elapsed_time(c1) / 3,
                    "kernels_ms_per_call": {k: v[0] / 3 for k, v in cp.items()},
                    "H_L2": float(norms[0, 0]), "H_max": float(norms[0, 1])}
        except Exception as ex:  # noqa: BLE001
            mesh.profile_enable(False)
            cons = {"error": str(ex)}

    # ---- end to end through the public API with host buffers.  Headline:
    # dgr_rk4_step_host over K host states (each step copies its input from
    # pinned host memory and its result back; the copies of neighbouring
    # steps overlap the current step on the copy engines).  Also reported: the
    # same copies serialised with the step (one dgr_rk4_step per state).
    host_in = torch.empty((24, mesh.dof_stride), dtype=torch.float64, pin_memory=True)
    host_in.copy_(u.cpu())
    host_out = [torch.empty_like(host_in).pin_memory() for _ in range(2)]
    mesh.rk4_step_host([host_in] * 3, [host_out[j % 2] for j in range(3)], dt, prm)
    torch.cuda.synchronize()
    barrier()
    e0.record()
    mesh.rk4_step_host([host_in] * args.steps, [host_out[j % 2] for j in range(args.steps)],
                       dt, prm)
    e1.record()
    torch.cuda.synchronize()
    barrier()
    ms_e2e = e0.elapsed_time(e1) / args.steps
    e2e_launches = mesh.last_launch_count()
    ud = torch.empty_like(u)
    ud.copy_(host_in, non_blocking=True)
    mesh.rk4_step(ud, dt, prm)
    host_out[0].copy_(ud, non_blocking=True)
    torch.cuda.synchronize()
    barrier()
    e0.record()
    for _ in range(args.steps):
        ud.copy_(host_in, non_blocking=True)
        mesh.rk4_step(ud, dt, prm)
        host_out[0].copy_(ud, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    barrier()
    ms_e2e_serial = e0.elapsed_time(e1) / args.steps
    t = torch.tensor([ms_e2e, ms_e2e_serial], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_e2e, ms_e2e_serial = float(t[0].item()), float(t[1].item())
    bytes_io = 24 * info["n_dof_owned"] * 8   # rows the library copies per state
    bytes_serial = host_in.numel() * 8

    # ---- the same step with the dgr_params options (radiative outer boundary
    # R29 — the one long evolutions use —, lopsided advection R9u): context for
    # the headline, which runs the default parameters (graph replay, 5 steps;
    # on a copy of the state, after the timed regions)
    opts = None
    if world == 1 and not args.no_options:
        try:
            opts = {}
            uo = u.clone()
            for name, op in (("sommerfeld", dgr.Params(sommerfeld=1)), ("upwind", dgr.Params(upwind=1))):
                for _ in range(3):
                    mesh.rk4_step(uo, dt, op)
                torch.cuda.synchronize()
                o0, o1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                o0.record()
                for _ in range(5):
                    mesh.rk4_step(uo, dt, op)
                o1.record()
                torch.cuda.synchronize()
                opts[name + "_ms_per_step"] = o0.elapsed_time(o1) / 5
            del uo
        except Exception as ex:  # noqa: BLE001
            opts = {"error": str(ex)}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    # ---- rooflines of the kernels, from the CUDA-event profile of the timed region
    hbm_peak, sm_max_mhz, peak_kind = _peaks()
    fp64_peak = 148 * 64 * 2 * sm_max_mhz * 1e6 / 1e12         # TFLOP/s, unit counts x max clock
    no, nl = info["n_oct_local"], info["n_oct_local"] + info["n_oct_ghost"]
    kern = {}
    for name, (tot_ms, n) in prof.items():
        avg = tot_ms / max(n, 1)
        kern[name] = {"ms_per_launch": avg, "launches": n, "ms_per_step": tot_ms / args.steps}
    def hbm(name, bytes_per_launch):
        k = kern.get(name)
        if not k:
            return None
        ach = bytes_per_launch / (k["ms_per_launch"] * 1e-3) / 1e9
        k.update({"bound": "hbm", "achieved": ach, "peak": hbm_peak, "unit": "GB/s",
                  "frac": ach / hbm_peak, "algorithmic_bytes_per_launch": bytes_per_launch})
    hbm("unzip", UNZIP_BYTES_PER_OCT * no)
    hbm("interp", INTERP_BYTES_PER_SLOT * info["n_interp_slots"] +
        INTERP_BYTES_PER_ELEM * info["n_interp_elems"])
    hbm("zip_rk4", ZIP_BYTES_PER_DOF_STAGE * info["n_dof_owned"])
    if "rhs" in kern:
        k = kern["rhs"]
        sec = k["ms_per_launch"] * 1e-3
        pts = no * 343
        nominal = pts * PAPER_FLOPS_PER_POINT / sec / 1e12
        k["paper_nominal_tflops"] = nominal
        k["hbm_GBps_algorithmic"] = RHS_BYTES_PER_OCT * no / sec / 1e9
        if RHS_EXEC_FLOPS_PER_POINT:
            ach = pts * RHS_EXEC_FLOPS_PER_POINT[args.path] / sec / 1e12
            k.update({"bound": "alu", "achieved": ach, "peak": fp64_peak, "unit": "TFLOP/s",
                      "frac": ach / fp64_peak, "peak_measured_dfma": dfma_tflops,
                      "flops": "executed (ncu DFMA x2 + DADD + DMUL per point)",
                      "frac_nominal": nominal / fp64_peak,
                      "frac_nominal_note": "paper-nominal eq 21a, 9,500 FLOP per point"})
        else:
            k.update({"bound": "alu", "achieved": nominal, "peak": fp64_peak, "unit": "TFLOP/s",
                      "frac": nominal / fp64_peak, "flops": "paper-nominal (eq 21a)",
                      "peak_measured_dfma": dfma_tflops})
    dom = max(kern, key=lambda n: kern[n]["ms_per_step"]) if kern else None
    roof = None
    if dom and "bound" in kern[dom]:
        k = kern[dom]
        roof = {"kernel": dom, "bound": k["bound"], "achieved": k["achieved"], "peak": k["peak"],
                "unit": k["unit"], "frac": k["frac"],
                "frac_nominal": k.get("frac_nominal"), "flops": k.get("flops"),
                "traffic": (NCU_TRAFFIC_C3.get(args.path, {}).get(dom)
                            if cfg.name == "c3" and world == 1 else None),
                "traffic_unit": "bytes per launch (ncu dram read+write)",
                "peak_source": (f"MEASURED_PEAKS.json ({peak_kind})" if k["bound"] == "hbm" else
                                "148 SM x 64 DFMA/clk x 2 x sm_max_mhz (derived)")}
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        try:
            cb = cpu_baseline_oracle(cfg, n_sample=args.cpu_sample)
            cpu = {k: cb[k] for k in ("value", "unit", "cores", "kind", "sample", "cpu_model",
                                      "numpy_threads", "extrapolation_factor", "one_core")}
        except Exception as ex:  # noqa: BLE001
            cpu = {"value": None, "unit": UNIT, "cores": 1, "kind": "oracle",
                   "sample": f"failed: {ex}"}
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic Brill-Lindquist puncture data (seeded, synth/initial.py)",
        "config": {"workload": f"{cfg.name}: {cfg.description}", "octants": info["n_oct_global"],
                   "dofs": n_dof, "unknowns": 24 * n_dof, "levels": [info["level_min"],
                                                                    info["level_max"]],
                   "dt": dt, "path": args.path,
                   "l2": ("inputs larger than L2 (state 0.97 GB + gather maps 0.2 GB + slots "
                          "streamed every stage"
                          + (", 10 GB patch buffer per stage)" if args.path == "two-pass" else ")")),
                   "parallelism": f"morton-partition x{world}"},
        "rhs_gflops": (kern.get("rhs", {}).get("achieved", 0) * 1e3) or None,
        "octant_points_per_s": info["n_oct_global"] * 343 / (ms_max * 1e-3),
        "roofline": roof,
        "kernels": kern,
        "kernel_timing": ("CUDA events around every libdgr launch on its stream, over a second "
                          f"pass of the same {args.steps} steps (eager launches): "
                          f"{ms_profiled:.3f} ms/step"),
        "fp64_dfma_tflops_measured": dfma_tflops,
        "cpu_baseline": cpu,
        "e2e": {"value": n_dof / (ms_e2e * 1e-3), "unit": UNIT, "h2d_bytes_per_step": bytes_io,
                "d2h_bytes_per_step": bytes_io, "ms_per_step": ms_e2e,
                "api": "dgr_rk4_step_host (pinned host states, copies overlapped with the "
                       "neighbouring steps)", "launches_per_step": e2e_launches / args.steps,
                "serial": {"value": n_dof / (ms_e2e_serial * 1e-3), "ms_per_step": ms_e2e_serial,
                           "h2d_bytes_per_step": bytes_serial, "d2h_bytes_per_step": bytes_serial,
                           "api": "copy_ -> dgr_rk4_step -> copy_ on one stream"}},
        "constraints": cons,
        "options": opts,
        "gpu_launches": launches_per_step * args.steps,
        "clocks": clk.summary(),
        "finite": finite,
        "nccl": _nccl_summary(nccl_log) if world > 1 else None,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
