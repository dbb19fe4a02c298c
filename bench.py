"""Benchmark of the B200 phase-field step (BASELINE.json metric: MLUP/s per
GPU, fp64, and % of roofline).

    python bench.py [--gpus N --steps K --warmup W] [--impl reference]
    torchrun --nproc-per-node N bench.py --gpus N ...

One "step" = one full time step of the hot path (Algorithm 1: phi-sweep,
phi ghosts, mu-sweep, mu ghosts, swap; plus the moving-window check every
window_check steps) over the whole domain.  Workload (config 2 of
BASELINE.json): 256^3 cells per GPU, ternary eutectic (4 phases, 2 mu),
frozen-temperature directional solidification with moving window, IC-L,
synthetic C.4 parameters.  For N > 1 the growth axis stays unsplit and the
blocks tile x-y (weak scaling, 256^3 per GPU).  Prints one JSON line on
rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MLUP/s per GPU (fp64) at 1/2/4/8 B200 and % of roofline"
UNIT = "MLUP/s"
# Table 1, P1, split accounting: algorithmic fp64 ops per cell
F_PHI = 66 + 124 + 202 + 282 + 9          # phi-split: adds + muls + divs = 683
F_MU = 256 + 389 + 75 + 90 + 17 + 21 + 18  # mu-split: adds + muls + divs + sqrts + rsqrts = 866
F_STEP = F_PHI + F_MU                      # 1549
Q_STEP = 96                                # bytes/cell: read phi, mu; write phi, mu (fp64)
# P2 (Table 1, P2 split columns): phi 364+368 adds, 792+557 muls, 18+14 divs;
# mu 142+26 adds, 248+46 muls, 6+9 divs, 3 sqrts, 12 rsqrts
F_STEP_P2 = (364 + 368 + 792 + 557 + 18 + 14) + (142 + 26 + 248 + 46 + 6 + 9 + 3 + 12)  # 2605
Q_STEP_P2 = 2 * (3 + 1) * 8                # read + write phi (3) and mu (1)
# fp64 peak derived from unit counts and clocks: 148 SMs x 64
# FP64 FMA lanes x 2 flop x 1.965 GHz (clocks.max.sm)
SMS, FP64_LANES, SM_MAX_GHZ = 148, 64, 1.965


def fp64_peak_tflops():
    return SMS * FP64_LANES * 2 * SM_MAX_GHZ / 1e3


def grid_for(n):
    return {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (4, 2, 1)}.get(n, (n, 1, 1))


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        return json.load(open(p))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self, first: int = 0):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines[max(first - 1, 0):]:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
                power.append(float(f[3]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm),
                "power_w_max": max(power) if power else None}


def ncu_summary(key, kernel="mu_sweep"):
    """A per-launch figure of the committed ncu --set full summary
    (profiles/ncu_summary.json; 256^3 launch), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        return json.load(open(p))[kernel][key]
    except Exception:
        return None


def traffic_per_launch():
    """dram read+write bytes per mu-sweep launch from the committed ncu summary, or None."""
    return ncu_summary("dram_bytes_per_launch")


def cpu_baseline(P, bc, seconds=12.0, shape=(64, 96, 96), strong=False):
    """The oracle, as it stands, on the host cores (bounded sample)."""
    from oracle import oracle as O
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    O.build()
    cores = os.cpu_count() or 1
    O.set_threads(cores)
    phi, mu = I.ic_voronoi(shape, seed=20191117) if strong else I.ic_lamellar(shape, seed=20191117)
    o = O.Oracle(shape, P, bc)
    o.init(phi, mu)
    n = 0
    t0 = time.perf_counter()
    while True:
        o.step(1)
        n += 1
        el = time.perf_counter() - t0
        if el >= seconds or n >= 200:
            break
    cells = shape[0] * shape[1] * shape[2]
    O.set_threads(0)
    return {"value": cells * n / el / 1e6, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{n} step(s) of the config-{4 if strong else 2} workload on a {shape[2]}x{shape[1]}x{shape[0]} "
                      f"(x*y*z) {'IC-V periodic' if strong else 'IC-L DS'} block, OpenMP over z on {cores} host "
                      f"threads, {el:.1f} s"}


def run_reference(args, rank, world):
    """--impl reference: the oracle on the host cores, each step a bounded
    sample (one oracle step on a 64x64x32 sub-block of the workload)."""
    if rank != 0:
        return
    from oracle import oracle as O
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    O.build()
    cores = os.cpu_count() or 1
    O.set_threads(cores)
    shape = (32, 64, 64)
    P = I.params_c4("ds")
    P["T0"] = I.ds_T0(8, P["G"])
    phi, mu = I.ic_lamellar(shape, seed=20191117, z_front=8)
    o = O.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    o.step(args.warmup)
    t0 = time.perf_counter()
    o.step(args.steps)
    el = time.perf_counter() - t0
    cells = shape[0] * shape[1] * shape[2]
    val = cells * args.steps / el / 1e6
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": "config 2 sample: 64x64x32 sub-block of the 256^3 DS moving-window run, IC-L, C.4",
                   "global": [64, 64, 32]},
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"{args.steps} oracle steps on 64x64x32, OpenMP on {cores} threads"},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=256, help="block edge per GPU")
    ap.add_argument("--config", default="weak", choices=["weak", "strong"],
                    help="weak: config 2/3 (n^3 DS block per GPU); strong: config 4 (fixed 512x512x1024 "
                         "periodic domain, z-slabs)")
    ap.add_argument("--variant", default="jit", choices=["jit", "tuned", "naive", "split"])
    ap.add_argument("--autotune", type=int, default=2, metavar="PASSES",
                    help="run pf_autotune (coordinate search over the JIT tuning knobs, timed on this block) with "
                         "this many passes before the warm-up; 0 = built-in defaults")
    ap.add_argument("--tuning", default=None, help="JSON dict of pf_tuning knobs set before the auto-tuning")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-stress", action="store_true", help="skip the stress-set (general-expression) line")
    ap.add_argument("--no-p2", action="store_true", help="skip the P2 (NEXT-4) line")
    args = ap.parse_args()
    assert args.warmup >= 3 or args.impl == "reference" or os.environ.get("PF_BENCH_ALLOW_SHORT"), "W >= 3"

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import numpy as np
    import torch
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf

    torch.cuda.set_device(local_rank)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    strong = args.config == "strong"
    n = args.n
    if strong:  # config 4: fixed 512 x 512 x 1024 periodic domain in z-slabs, IC-V
        procs = (1, 1, world)
        gshape = (1024, 512, 512)
        P = I.params_c4("periodic")
        bc = I.BC_PERIODIC
    else:  # configs 2/3: n^3 DS block per GPU, growth axis z unsplit
        procs = grid_for(world)
        gshape = (n, n * procs[1], n * procs[0])  # (nz, ny, nx)
        # growing front (inputs.DS_BENCH): it starts one plane above the
        # window threshold, so the first check shifts and the window keeps
        # following the front (one plane per ~260 steps at 256^3)
        z_front = n // 2 + 2
        P = I.params_ds_growth(z_front, window_check=10, window_frac=0.5, **I.DS_BENCH)
        bc = I.BC_DS
    uid = None
    if world > 1:
        t = torch.zeros(128, dtype=torch.uint8, device="cuda")
        if rank == 0:
            t.copy_(torch.tensor(list(pf.nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(t, 0)
        uid = bytes(t.cpu().tolist())
    g = pf.PhaseField(gshape, P, bc=bc, procs=procs, rank=rank, world=world, device=local_rank, nccl_uid=uid)
    g.set_variant(args.variant)
    lshape = g.local
    if strong:
        # IC-V on a 256^3 periodic tile (24 grains, S§8(d) density), tiled
        # periodically over the global domain; this rank's slab
        # (tiled on the device: the slab is up to 12.9 GB of fields)
        tphi, tmu = I.ic_voronoi((256, 256, 256), seed=20191117)
        dev = torch.device("cuda", local_rank)
        z0 = g.offset[0]
        iz = torch.tensor([(z0 + k) % 256 for k in range(lshape[0])], device=dev)
        iy = torch.arange(lshape[1], device=dev) % 256
        ix = torch.arange(lshape[2], device=dev) % 256
        phi_d = torch.from_numpy(tphi).to(dev)[:, iz][:, :, iy][:, :, :, ix].contiguous()
        mu_d = torch.from_numpy(tmu).to(dev)[:, iz][:, :, iy][:, :, :, ix].contiguous()
        del tphi, tmu
        g.init_fields(phi_d, mu_d)
        del phi_d, mu_d
        torch.cuda.empty_cache()
        args.no_e2e = True  # no host copy of the slab (e2e is measured on the weak-scaling workload)
    else:
        phi, mu = I.ic_lamellar(lshape, seed=20191117 + rank, z_front=z_front)
        phi_pin = torch.from_numpy(phi).pin_memory()
        mu_pin = torch.from_numpy(mu).pin_memory()
        g.init_fields(phi_pin, mu_pin)
    stream = g.stream
    cells_local = lshape[0] * lshape[1] * lshape[2]
    tune_rep = None
    if args.tuning and args.variant == "jit":
        g.set_tuning(json.loads(args.tuning))
    if args.autotune > 0 and args.variant == "jit":
        t_at = time.time()
        # collective: same choice on every rank; with the kernel-variant ablation
        # (full / split / fused, NEXT-2) on the single-GPU weak workload
        rep = g.autotune(passes=args.autotune, reps=5, variants=(world == 1 and not strong))
        tune_rep = {"passes": args.autotune, "seconds": round(time.time() - t_at, 1),
                    "phi": rep["phi"], "mu": rep["mu"], "step": rep.get("step"), "variants": rep.get("variants"),
                    "tried": len(rep["tried"])}

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---- warm-up (the clock sampler spins up meanwhile) ----
    # per-kernel timing (CUDA events around every sweep) is on from the
    # warm-up on; pf_step then launches every step directly (no graph runs)
    g.profile(True)
    clocks = ClockSampler(local_rank)
    clocks.start()
    g.step(args.warmup)
    barrier()
    t_wait = time.time()
    # step until the sampler has two clock lines; the decision is a max over
    # ranks, so every rank steps (and exchanges halos) the same number of times
    while max_over_ranks(1.0 if (len(clocks.lines) < 2 and time.time() - t_wait < 3.0) else 0.0) > 0:
        g.step(1)
        torch.cuda.synchronize()
    # realign with the window checks (pf_step runs graphs of window_check
    # steps, or 8 without a window, when they are used) so that no capture
    # would fall inside the timed region
    K = int(P.get("window_check", 0)) or 8
    g.step((K - g.state()["step"] % K) % K + 2 * K)
    barrier()
    # ---- timed region (device events on the library's stream) ----
    g.profile(True)
    zoff0 = g.state()["z_off"]
    n_clk0 = len(clocks.lines)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    barrier()
    e0.record(stream)
    g.step(args.steps)
    e1.record(stream)
    e1.synchronize()
    barrier()
    ms = e0.elapsed_time(e1)
    clk = clocks.stop(n_clk0)
    prof = g.profile_read()
    ms_max = max_over_ranks(ms)
    launches = sum(v[1] for v in prof.values())
    mon = g.monitor()
    st = g.state()
    window = None
    if not strong:
        # one window shift by one plane (front-height reduction excluded),
        # timed on its own after the timed region: the cost of each shift
        # (the state is re-initialised by the e2e leg)
        w0, w1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        w0.record(stream)
        g.shift_window(1)
        w1.record(stream)
        w1.synchronize()
        shift_ms = max_over_ranks(w0.elapsed_time(w1))
        window = {"check_every": int(P["window_check"]), "z_off_before": zoff0, "z_off_after": st["z_off"],
                  "shifts_in_timed_region": st["z_off"] - zoff0,
                  "check_and_shift_ms_total": prof["window"][0], "check_and_shift_ms_per_step":
                      prof["window"][0] / args.steps,
                  "shift_ms": shift_ms,
                  "pulling_speed_v": P["v"], "gradient_G": P["G"],
                  "note": "z_off counts planes shifted since init (warm-up included); a shift is an out-of-place "
                          "copy of both fields plus a ghost fill; the front advances ~1 plane per ~260 steps "
                          "(profiles/r02_ds_tune.jsonl)"}

    total_cells = cells_local * world
    value = total_cells * args.steps / (ms_max * 1e-3) / 1e6  # whole-job MLUP/s
    # ---- roofline of the dominant kernel (mu-sweep) ----
    mu_ms, mu_n = prof["mu_sweep"]
    phi_ms, phi_n = prof["phi_sweep"]
    peak_tf = fp64_peak_tflops()
    mu_tf = F_MU * cells_local / (mu_ms / mu_n * 1e-3) / 1e12 if mu_n else None
    phi_tf = F_PHI * cells_local / (phi_ms / phi_n * 1e-3) / 1e12 if phi_n else None
    peaks = measured_peaks()
    hbm = peaks.get("hbm_gbs", 6650.0)
    R = min(peak_tf * 1e12 / F_STEP, hbm * 1e9 / Q_STEP) / 1e6  # MLUP/s per GPU
    rec = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": "strong" if strong else "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": ("config 4: fixed 512x512x1024 periodic domain in z-slabs, ternary eutectic "
                                "N=4/K-1=2, IC-V (256^3 periodic tile), C.4 parameters") if strong else
                               (f"config 2: {n}^3 block per GPU, ternary eutectic N=4/K-1=2, frozen-T directional "
                                f"solidification (v={P['v']}, G={P['G']}), moving window (check every 10 steps), "
                                f"IC-L, C.4 parameters"),
                   "global_xyz": [gshape[2], gshape[1], gshape[0]], "procs_xyz": list(procs),
                   "parallelism": f"domain decomposition {procs[0]}x{procs[1]}x{procs[2]}",
                   "variant": args.variant, "tuning": g.tuning() if args.variant == "jit" else None,
                   "l2": f"inputs larger than L2 ({(6 * 2) * cells_local * 8 / 1e9:.2f} GB of fields per GPU)"},
        "per_gpu_mlups": value / world,
        "step_roofline": {"R_mlups": R, "F_flop_per_cell": F_STEP, "Q_bytes_per_cell": Q_STEP,
                          "frac": (value / world) / R, "peak_fp64_tflops": peak_tf, "hbm_gbs": hbm},
        "roofline": {"bound": "alu", "kernel": "mu_sweep", "achieved": mu_tf, "peak": peak_tf, "unit": "TFLOP/s",
                     "frac": (mu_tf / peak_tf) if mu_tf else None,
                     # the committed ncu capture is of the 256^3 block launch
                     "traffic": traffic_per_launch() if cells_local == 256 ** 3 else None,
                     "flop_per_cell": F_MU, "cells_per_launch": cells_local,
                     # context: the fp64 work the specialised kernel actually issues (ncu, DADD + DMUL
                     # + 2 DFMA per cell at 256^3) and the rate it sustains at this launch time
                     "hw_flop_per_cell": ncu_summary("hw_flop_per_cell"),
                     "hw_achieved": (ncu_summary("hw_flop_per_cell") * cells_local / (mu_ms / mu_n * 1e-3) / 1e12)
                     if (mu_n and ncu_summary("hw_flop_per_cell")) else None,
                     "hw_frac": ((ncu_summary("hw_flop_per_cell") * cells_local / (mu_ms / mu_n * 1e-3) / 1e12) / peak_tf)
                     if (mu_n and ncu_summary("hw_flop_per_cell")) else None,
                     "avg_launch_ms": mu_ms / mu_n if mu_n else None,
                     "peak_note": "derived: 148 SMs x 64 FP64 lanes x 2 x 1.965 GHz (DESIGN.md §6); measured DFMA "
                                  "36.8 TF/s at 1965 MHz (profiles/r02_fp64_micro.json)",
                     "frac_note": "frac: Table-1 algorithmic flops (866/cell); hw_frac: fp64 work the specialised "
                                  "kernel issues (DADD + DMUL + 2 DFMA per cell, ncu)"},
        "kernels": {"phi_sweep_ms": phi_ms / max(phi_n, 1), "mu_sweep_ms": mu_ms / max(mu_n, 1),
                    "phi_sweep_tflops": phi_tf, "share_mu": mu_ms / ms if ms else None,
                    "share_phi": phi_ms / ms if ms else None,
                    "ghost_ms_total": prof["ghost"][0], "window_ms_total": prof["window"][0]},
        "gpu_launches": launches,
        "autotune": tune_rep,
        "clocks": clk,
        "state": {"step": st["step"], "z_off": st["z_off"], "max_sum_err": mon[0], "min_phi": mon[1]},
        "window": window,
    }
    # ---- the same steps with the anti-trapping skip (tuning mu_atskip): the
    # mu-sweep skips eq. 10 in warps where it is exactly 0 (bulk phases);
    # same results, data-dependent time -- reported beside the headline, not
    # as it (the headline kernel does the full work everywhere)
    if args.variant == "jit" and not strong and world == 1:
        tsave = g.tuning()
        g.set_tuning(dict(tsave, mu_atskip=1))
        g.step(3)
        barrier()
        g.profile(True)
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        na = max(20, min(args.steps, 100))
        a0.record(stream)
        g.step(na)
        a1.record(stream)
        a1.synchronize()
        pa = g.profile_read()
        ams = a0.elapsed_time(a1)
        rec["atskip"] = {"value": cells_local * na / (ams * 1e-3) / 1e6, "unit": UNIT, "steps": na,
                         "ms_per_step": ams / na, "mu_sweep_ms": pa["mu_sweep"][0] / max(pa["mu_sweep"][1], 1),
                         "phi_sweep_ms": pa["phi_sweep"][0] / max(pa["phi_sweep"][1], 1),
                         "note": "same workload and state continuing after the timed region, tuning mu_atskip = 1 "
                                 "(bitwise-equal results, tests/test_gpu_autotune.py); data-dependent"}
        g.set_tuning(tsave)
    # ---- end-to-end through the public API with host buffers ----
    if not args.no_e2e:
        g.profile(False)
        out_phi = torch.empty_like(phi_pin).pin_memory()
        out_mu = torch.empty_like(mu_pin).pin_memory()
        barrier()
        t0 = time.perf_counter()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        g.init_fields(phi_pin, mu_pin)
        g.step(args.steps)
        g.download(out=(out_phi, out_mu))
        f1.record(stream)
        f1.synchronize()
        barrier()
        ems = max_over_ranks(max(f0.elapsed_time(f1), (time.perf_counter() - t0) * 1e3))
        bytes_state = (phi_pin.numel() + mu_pin.numel()) * 8
        rec["e2e"] = {"value": total_cells * args.steps / (ems * 1e-3) / 1e6, "unit": UNIT,
                      "h2d_bytes_per_step": bytes_state / args.steps, "d2h_bytes_per_step": bytes_state / args.steps,
                      "chunk_steps": args.steps,
                      "note": f"one chunk = pf_init_fields from pinned host memory, {args.steps} steps, pf_download to "
                              "pinned host memory, all inside the timed region (the copies amortise over the chunk: "
                              "the value depends on the chunk length)"}
    # ---- general-expression path: the stress parameter set S (unequal gamma,
    # A1 != 0, non-diagonal chi / D, mu_inf != 0: none of the specialised
    # simplifications apply), same block, boundaries and IC
    if world == 1 and not strong and not args.no_stress and args.variant == "jit":
        g.close()
        torch.cuda.empty_cache()
        Ps = I.params_stress(window_check=10, window_frac=0.5)
        gs = pf.PhaseField(gshape, Ps, bc=bc, device=local_rank)
        gs.init_fields(phi_pin, mu_pin)
        st_tune = None
        if args.autotune > 0:  # the specialised sweeps of this parameter set tuned on their own
            t_st = time.time()
            rs = gs.autotune(passes=1, reps=3)
            st_tune = {"passes": 1, "seconds": round(time.time() - t_st, 1), "phi": rs["phi"], "mu": rs["mu"],
                       "tuning": gs.tuning()}
        gs.profile(True)
        gs.step(max(args.warmup, 3) + 10)
        torch.cuda.synchronize()
        gs.profile(True)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        nst = max(20, min(args.steps, 100))
        s0.record(gs.stream)
        gs.step(nst)
        s1.record(gs.stream)
        s1.synchronize()
        sms = s0.elapsed_time(s1)
        sp = gs.profile_read()
        rec["stress_set"] = {
            "value": cells_local * nst / (sms * 1e-3) / 1e6, "unit": UNIT, "steps": nst, "ms_per_step": sms / nst,
            "mu_sweep_ms": sp["mu_sweep"][0] / max(sp["mu_sweep"][1], 1),
            "phi_sweep_ms": sp["phi_sweep"][0] / max(sp["phi_sweep"][1], 1),
            "frac_of_R": (cells_local * nst / (sms * 1e-3) / 1e6) / R,
            "autotune": st_tune,
            "note": "parameter set S of SURVEY C.4 (general expressions), same block / BCs / IC; the specialised "
                    "sweeps of S auto-tuned on their own (1 pass) unless --autotune 0"}
        gs.close()
    # ---- P2 parameterisation: 3 phases,
    # 1 mu, anisotropic phi (pf_p2.cu), n^3 periodic block, IC-V
    if world == 1 and not strong and not args.no_p2:
        torch.cuda.empty_cache()
        P2 = I.params_p2()
        g2 = pf.PhaseField((n, n, n), P2, device=local_rank)
        ph2, mu2 = I.ic_voronoi((n, n, n), seed=20191117, N=3, M=1)
        g2.init_fields(ph2, mu2)
        p2_tune = None
        if args.autotune > 0:  # the P2 kernel choices (p2_* knobs) timed on this block
            t_p2 = time.time()
            r2 = g2.autotune(reps=3)
            p2_tune = {"seconds": round(time.time() - t_p2, 1), "phi": r2["phi"], "mu": r2["mu"],
                       "best": {k: v for k, v in g2.tuning().items() if k.startswith("p2_")}}
        g2.profile(True)
        g2.step(3)
        torch.cuda.synchronize()
        g2.profile(True)
        n2 = max(10, min(args.steps, 40))
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(g2.stream)
        g2.step(n2)
        s1.record(g2.stream)
        s1.synchronize()
        ms2 = s0.elapsed_time(s1)
        pr2 = g2.profile_read()
        val2 = n ** 3 * n2 / (ms2 * 1e-3) / 1e6
        # the same kernel choices, generic build (variant tuned: run-time
        # parameters): what the run-time specialisation gains on P2
        gen2 = None
        if args.variant == "jit":
            g2.set_variant("tuned")
            g2.step(3)
            g2.profile(True)
            ng = max(5, n2 // 2)
            s0.record(g2.stream)
            g2.step(ng)
            s1.record(g2.stream)
            s1.synchronize()
            msg = s0.elapsed_time(s1)
            prg = g2.profile_read()
            gen2 = {"value": n ** 3 * ng / (msg * 1e-3) / 1e6, "ms_per_step": msg / ng,
                    "phi_sweep_ms": prg["phi_sweep"][0] / max(prg["phi_sweep"][1], 1),
                    "mu_sweep_ms": prg["mu_sweep"][0] / max(prg["mu_sweep"][1], 1),
                    "note": "variant tuned: the same kernels compiled ahead of time on run-time parameters"}
            g2.set_variant("jit")
        R2 = min(peak_tf * 1e12 / F_STEP_P2, hbm * 1e9 / Q_STEP_P2) / 1e6
        rec["p2"] = {"value": val2, "unit": UNIT, "steps": n2, "ms_per_step": ms2 / n2,
                     "phi_sweep_ms": pr2["phi_sweep"][0] / max(pr2["phi_sweep"][1], 1),
                     "mu_sweep_ms": pr2["mu_sweep"][0] / max(pr2["mu_sweep"][1], 1),
                     "R_mlups": R2, "frac_of_R": val2 / R2, "F_flop_per_cell": F_STEP_P2, "autotune": p2_tune,
                     "workload": f"P2: {n}^3 periodic block, 3 phases / 1 mu, anisotropic gamma (reading B6), IC-V",
                     "variant": args.variant, "generic": gen2,
                     "note": "P2 sweeps (pf_p2_dev.cuh side-staged bodies, run-time specialised on the P2 parameters "
                             "unless --variant tuned): z-marching tiles, each face flux once with both sides from "
                             "shared memory, L2 prefetch; kernel choices auto-tuned"}
        # P2 in directional solidification (NEXT-4 "dendritic DS"): the same
        # kernels (the tuning found above) on a grain / liquid front with DS
        # boundaries, frozen gradient and moving window
        p2tun = {k: v for k, v in g2.tuning().items() if k.startswith("p2_")}
        g2.close()
        torch.cuda.empty_cache()
        zf = n // 2 + 2
        P3 = I.params_p2_ds(zf)
        g3 = pf.PhaseField((n, n, n), P3, bc=I.BC_DS, device=local_rank)
        ph3, mu3 = I.ic_p2_front((n, n, n), seed=20191117, z_front=zf)
        g3.init_fields(ph3, mu3)
        del ph3, mu3
        g3.set_tuning(p2tun)
        g3.step(5)
        g3.profile(True)
        zo0 = g3.state()["z_off"]
        s0.record(g3.stream)
        g3.step(n2)
        s1.record(g3.stream)
        s1.synchronize()
        ms3 = s0.elapsed_time(s1)
        pr3 = g3.profile_read()
        val3 = n ** 3 * n2 / (ms3 * 1e-3) / 1e6
        rec["p2"]["ds"] = {"value": val3, "ms_per_step": ms3 / n2, "frac_of_R": val3 / R2,
                           "phi_sweep_ms": pr3["phi_sweep"][0] / max(pr3["phi_sweep"][1], 1),
                           "mu_sweep_ms": pr3["mu_sweep"][0] / max(pr3["mu_sweep"][1], 1),
                           "z_off_before": zo0, "z_off_after": g3.state()["z_off"],
                           "workload": f"P2 directional solidification: {n}^3 DS block (params_p2_ds: G = {P3['G']}, "
                                       f"v = {P3['v']}, moving window), two grains under liquid (ic_p2_front)",
                           "note": "data-dependent: the P2 kernels' exact-zero branches (zero pair gradient in the "
                                   "anisotropy, the anti-trapping guard of reading A11) skip work in the bulk "
                                   "grains and liquid, so frac_of_R (Table-1 credit) overstates the issued work"}
        g3.close()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rec["cpu_baseline"] = cpu_baseline(P, bc, strong=strong)
    if rank == 0:
        print(json.dumps(rec), flush=True)
    g.close()  # (idempotent)
    if dist is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
