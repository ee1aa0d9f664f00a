#!/usr/bin/env python
"""Benchmark of the B200 HPGMG-FV hot path (metric of BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl sf|reference]

Workload: BASELINE config 5 / config 4 at N=1 --
an HPGMG-shaped variable-coefficient Helmholtz problem (a = b = 1, tanh beta,
manufactured rhs) with 512^3 cells per GPU, z-slab decomposed over N GPUs
(global (512,512,512), (512,512,1024), (512,1024,1024), (1024,1024,1024) for
N = 1, 2, 4, 8: weak scaling).  One STEP = one full solve: an F-cycle, then
V-cycles (2+2 colour-fused GSRB pairs, P0, exact bottom) until
||f - Au||inf / ||f||inf < 1e-10.  value = DOF/s = (cells solved by all ranks)
/ time.  Inputs (10.7 GB per GPU) exceed the 126 MB L2 many times over, so
no L2 flush is needed between steps.

Also measured in the same run: the GSRB smoother of BASELINE config 3 (256^3,
one fused RB pair per call) in GStencil/s and algorithmic GB/s, the roofline
of the dominant kernel (the fused RB-pair kernel on the finest level), an
end-to-end number through the C ABI with host buffers, and the CPU oracle on
a bounded sample (rank 0, N = 1).
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

GSRB_BYTES_PER_CELL = 64      # PAPER.md:669-672 (x r+w, rhs, alpha, beta x3, lambda)
GSRB_KERNEL_BYTES_PER_CELL = 56   # lambda-form smoother never reads alpha
F_OVER_V = 8.0 / 7.0          # F-cycle cost in finest-level V-cycles (sum over levels)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="sf", choices=["sf", "reference"])
    p.add_argument("--side", type=int, default=512, help="cells per side per GPU (weak scaling)")
    p.add_argument("--gsrb-n", type=int, default=256)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--quick", action="store_true", help="skip the side measurements")
    p.add_argument("--comm", default="p2p", choices=["p2p", "nccl"],
                   help="N>1 transport: device-initiated peer-memory exchanges (p2p) or NCCL")
    return p.parse_args()


def dims_for(n, gpus):
    from paper_conf_ipps_zhangdmwbf17_b200.parallel import weak_dims
    return weak_dims(n, gpus)


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self.proc = index, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = sorted(float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit())
        mx = max(float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit())
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if len(r) > 3 + i and r[3 + i].lower().startswith("active")})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx,
                "reasons": reasons, "samples": len(self.rows)}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            p = json.load(fh)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy, burst)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic():
    """dram bytes read+write per launch of the fused pair kernel from the
    committed `ncu --set full` capture (profiles/), keyed by level size."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as fh:
            return json.load(fh)
    except Exception:
        return {}


# ------------------------------------------------------------------ oracle (cpu)
def oracle_threads():
    """Host cores this process may use (the oracle's OpenMP build runs on all)."""
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


class OracleSolver:
    """The CPU oracle solving the workload's problem exactly as a bench step
    does (F-cycle, then V-cycles with 2+2 GSRB pairs, P0, exact bottom, until
    ||f - Au||inf / ||f||inf < 1e-10), with its OpenMP build on all host cores
    (the plane loops of oracle.c; same arithmetic as the single-thread build,
    which the pins and parity tests use)."""

    def __init__(self, shape):
        from oracle import oracle as O
        from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I
        O.use_openmp(True)
        self.cores = O.lib().or_set_threads(oracle_threads())   # the threads it actually runs
        nx, ny, nz = shape
        self.shape = shape
        h = I.level_h(nx, ny, nz)
        coeffs = I.hpgmg_coeffs(nx, ny, nz, h)
        _, self.f = I.manufactured(nx, ny, nz, 1.0, 1.0, h)
        self.mg = O.MG(nx, ny, nz, h, 1.0, 1.0, *coeffs)
        del coeffs
        self.desc = (f"one complete oracle solve (F-cycle + V-cycles, 2+2 GSRB pairs, P0, exact "
                     f"bottom, to 1e-10) of the HPGMG VC Helmholtz problem at {nx}x{ny}x{nz}, "
                     f"OpenMP build on {self.cores} host cores")

    def solve_seconds(self):
        """(seconds, cycles, final relres) of one measured solve from u = 0."""
        t0 = time.perf_counter()
        _, hist = self.mg.solve(self.f, fcycle=True, rtol=1e-10)
        return time.perf_counter() - t0, len(hist), hist[-1] if hist else None


def host_memory_allows(shape):
    """The oracle hierarchy of `shape` needs ~40 doubles per cell of host RAM."""
    try:
        import psutil
        avail = psutil.virtual_memory().available
    except Exception:
        avail = 0
    return avail > shape[0] * shape[1] * shape[2] * 8 * 40


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


# The reference arm's step: one complete oracle solve of the workload's problem
# at 256^3 (1/8 of the 512^3 per-GPU DOFs): a few seconds on a many-core host,
# so --steps 20 --warmup 5 ends within minutes.  Multigrid work per DOF is
# size-independent (11-12 cycles at 256^3 and 512^3), so DOF/s of the sample
# is the CPU's rate on the workload; bench's default run also measures one
# 512^3 oracle solve (cpu_baseline) when the host has the memory.
REFERENCE_SAMPLE = (256, 256, 256)


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    nx, ny, nz = dims_for(args.side, 1)
    shp = REFERENCE_SAMPLE if nx * ny * nz > 256**3 else (nx, ny, nz)
    smp = OracleSolver(shp)
    cells = shp[0] * shp[1] * shp[2]
    steps, cyc, rr = [], None, None
    for s in range(args.warmup + args.steps):
        t, cyc, rr = smp.solve_seconds()
        if s >= args.warmup:
            steps.append(t)
    t_solve = sum(steps) / len(steps)
    val = cells / t_solve
    sample = (f"{smp.desc}: {cyc} cycles, final relres {rr:.2e}, {t_solve:.2f} s per solve "
              f"(mean of {len(steps)} measured solves); each step is one such solve -- a "
              f"{shp[0]}^3 sample of the {nx}x{ny}x{nz} per-GPU workload (same problem, solver "
              f"and tolerance; DOF/s of the sample)")
    line = {"impl": "reference", "metric": "HPGMG-FV DOF/s (F-cycle + V-cycles to 1e-10)",
            "value": val, "unit": "DOF/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_solve * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"C5 HPGMG-FV VC Helmholtz {nx}x{ny}x{nz} per GPU",
                       "global": [nx, ny, nz]},
            "cpu_baseline": {"value": val, "unit": "DOF/s", "cores": smp.cores, "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model(),
                             "sample_shape": list(shp), "cycles": cyc},
            "e2e": {"value": val, "unit": "DOF/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import sf

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # SF_BENCH_SHARED_GPU=1 (tests only): every rank on cuda:0, gloo process group
    shared = os.environ.get("SF_BENCH_SHARED_GPU") == "1"
    local = 0 if shared else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    host_group = None
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
            host_group = dist.group.WORLD
        else:
            dist.init_process_group("nccl", device_id=dev)
            host_group = dist.new_group(backend="gloo")   # IPC-handle exchange (p2p)
    sf.lib()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    from paper_conf_ipps_zhangdmwbf17_b200.parallel import max_over_ranks as _mor

    def max_over_ranks(x):
        return _mor(x, device=None if shared else dev)

    nx, ny, nz = dims_for(args.side, world)
    comm = None
    transport = args.comm if world > 1 else "none"
    h = 1.0 / max(nx, ny, nz)
    if world > 1 and args.comm == "p2p":
        # device-initiated transport over CUDA IPC; if any rank cannot map its
        # peers' buffers, every rank gets the same error (sf_ipc_register) and
        # all fall back to NCCL together
        comm = sf.Comm.p2p(host_group)
        try:
            L = sf.Level(nx, ny, nz, h, comm=comm)
        except sf.SfError as e:
            comm.close()
            print(f"bench: p2p transport unavailable ({e}); using NCCL", file=sys.stderr)
            comm = sf.Comm.nccl()
            sf.sf_comm_check(comm.h, torch.cuda.current_stream().cuda_stream)   # health check
            transport = "nccl (p2p unavailable)"
            L = sf.Level(nx, ny, nz, h, comm=comm)
    else:
        if world > 1:
            comm = sf.Comm.nccl()
            sf.sf_comm_check(comm.h, torch.cuda.current_stream().cuda_stream)   # health check
        L = sf.Level(nx, ny, nz, h, comm=comm)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)       # HPGMG problem + manufactured f
    M = sf.MG(L, 1.0, 1.0)
    stream = L.stream
    dof_local = nx * ny * (nz // world)

    def step():
        return sf.sf_solve(M.handle, True, 1e-10, 50)

    for _ in range(args.warmup):
        st, cyc, hist = step()
    sf.sf_launch_count(reset=True)
    # live duration of the dominant kernel inside the timed region: the fused
    # pair stamps %globaltimer per launch on the finest level (CUDA events cannot
    # bracket a kernel node of a graph)
    sf.sf_level_pair_timing(L.handle, 1)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    prof = os.environ.get("SF_PROFILE_TIMED") == "1"   # ncu --profile-from-start off
    with ClockSampler(local) as clk:
        if prof:
            torch.cuda.cudart().cudaProfilerStart()
        e0.record(stream)
        for _ in range(args.steps):
            st, cyc, hist = step()
        e1.record(stream)
        barrier()
        if prof:
            torch.cuda.cudart().cudaProfilerStop()
    launches = sf.sf_launch_count(reset=True)
    live_pair_ms, live_pairs = sf.sf_level_pair_timing(L.handle, 0)
    live_var = sf.sf_level_pair_timing_variants(L.handle)
    live_rrf = sf.sf_level_pair_timing_rrf(L.handle)
    t = max_over_ranks(e0.elapsed_time(e1) / 1e3)
    value = dof_local * world * args.steps / t
    ms_step = t / args.steps * 1e3

    # error vs the manufactured solution (O(h^2) pin)
    u = L.download(sf.SF_U)
    from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I
    err = None
    if world == 1 and nx * ny * nz <= 512**3:
        ue, _ = I.manufactured(nx, ny, nz, 1.0, 1.0, h)
        err = float(np.abs(u - ue).max())
        del ue
    del u

    side = {}
    if not args.quick:
        side = side_measurements(args, sf, torch, L, M, world, rank, barrier, max_over_ranks,
                                 dof_local, cyc, comm)

    if rank == 0:
        pk, pk_src = peaks()
        fine_pair = side.get("fine_pair_ms")
        roof = None
        if live_pairs:
            # a pair split around a halo exchange (interior + boundary launch) is
            # booked once with both launches' durations: mean = time per pair
            pair_ms = live_pair_ms
            alg = GSRB_BYTES_PER_CELL * dof_local
            ach = alg / (pair_ms / 1e3) / 1e9
            tr = ncu_traffic().get(f"{nx}x{ny}x{nz // world}")
            kb = GSRB_KERNEL_BYTES_PER_CELL * dof_local
            roof = {"bound": "hbm", "achieved": ach, "peak": pk, "unit": "GB/s",
                    "frac": ach / pk, "traffic": tr,
                    "kernel": "gsrb_pair_tma_kernel (colour-fused RB pair, finest level; all four "
                              "variants: plain, check-fused RESID/BRES, P0-fused INTERP)",
                    "algorithmic_bytes_per_launch": alg,
                    "algorithmic_basis": "64 B/cell per RB pair (PAPER.md:669-672, SURVEY 8d)",
                    "kernel_compulsory_bytes_per_launch": kb,
                    "frac_of_kernel_compulsory": kb / (pair_ms / 1e3) / 1e9 / pk,
                    "note": "lambda-form update reads 56 of the paper's 64 B/cell (alpha enters "
                            "only through lambda = 1/diag(A)); traffic = ncu DRAM bytes per launch "
                            "(plain variant)",
                    "launch_ms": pair_ms,
                    "launch_ms_how": "mean per RB pair over the finest level's fused-pair "
                                     "launches inside the timed region (in-kernel %globaltimer, "
                                     "first CTA start to last CTA end; sf_level_pair_timing)",
                    "launches_in_timed_region": live_pairs, "peak_source": pk_src,
                    "live_per_variant": {k: {"ms": v[0], "pairs": v[1],
                                             "frac": (alg / (v[0] / 1e3) / 1e9 / pk) if v[0] else None}
                                         for k, v in live_var.items()},
                    "live_pair_residual_restrict": {
                        "ms": live_rrf[0], "launches": live_rrf[1],
                        "what": "the last pre-smoothing pair fused with the delta-form "
                                "residual + restriction (gsrb_rr.cu), in-kernel timed like the "
                                "pairs; not in launch_ms (it replaces a pair AND the separate "
                                "residual_restrict pass)"},
                    "share_of_step": live_pairs * live_pair_ms / (t * 1e3),
                    "isolated_plain_pair_ms": fine_pair,
                    "isolated_plain_pair_frac": (alg / (fine_pair / 1e3) / 1e9 / pk
                                                 if fine_pair else None)}
        line = {
            "metric": "HPGMG-FV DOF/s (F-cycle + V-cycles to 1e-10)",
            "value": value, "unit": "DOF/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (HPGMG-shaped VC Helmholtz, manufactured rhs, on-device init)",
            "config": {"workload": f"C5 HPGMG-FV VC Helmholtz {nx}x{ny}x{nz // world} per GPU",
                       "global": [nx, ny, nz], "parallelism": f"z-slab x{world}",
                       "transport": transport,
                       "cycles_per_solve": cyc, "final_relres": hist[-1] if hist else None,
                       "max_err_vs_manufactured": err,
                       "smoother": "colour-fused GSRB, 2+2 pairs", "l2": "inputs >> L2, no flush"},
            "clocks": clk.summary(),
            "gpu_launches": launches,
            "roofline": roof,
        }
        line.update({k: v for k, v in side.items() if k in (
            "e2e", "gsrb_c3", "vcycle", "fcycle", "fcycle_strong", "read_bw", "cpu_baseline", "fig7_256",
            "gsrb_size_sweep", "dsl_256", "c1_16", "c2_64") or k.startswith("fig7_")})
        print(json.dumps(line), flush=True)
    M.close()
    L.close()
    if comm:
        comm.close()
    if world > 1:
        dist.destroy_process_group()


def side_measurements(args, sf, torch, L, M, world, rank, barrier, max_over_ranks, dof_local,
                      cyc, comm=None):
    out = {}
    stream = L.stream
    nx, ny, nz = L.gnx, L.gny, L.gnz

    def timed(fn, reps, warm=3):
        for _ in range(warm):
            fn()
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(reps):
            fn()
        b.record(stream)
        barrier()
        return max_over_ranks(a.elapsed_time(b) / reps)

    # dominant kernel: one fused RB pair on the finest level (1 launch per call at N=1)
    fine_pair = timed(lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1,
                                                sf.SF_SMOOTH_FUSED), 20)
    out["fine_pair_ms"] = fine_pair
    # V-cycle alone (finest level; the solve = 1 F + cyc-1 V)
    vms = timed(lambda: sf.sf_vcycle(M.handle, 0), 5, warm=2)
    out["vcycle"] = {"ms": vms, "dof_s": dof_local * world / (vms / 1e3)}
    # C4's figure of merit: one F-cycle (HPGMG FOM), same level and operator
    fms = timed(lambda: sf.sf_fcycle(M.handle), 3, warm=1)
    out["fcycle"] = {"ms": fms, "dof_s": dof_local * world / (fms / 1e3),
                     "note": "C4 / HPGMG FOM: one F-cycle (PL up, one V per level) on the workload"}
    # BASELINE C4: the side^3 problem itself split across the ranks -- strong
    # scaling of one F-cycle (at N = 1 this is the fcycle line above)
    if world > 1 and args.side % world == 0 and (args.side // world) % 2 == 0:
        n = args.side
        Ls = sf.Level(n, n, n, 1.0 / n, comm=comm)
        sf.sf_init_problem(Ls.handle, 1, 1.0, 1.0, 1)
        Ms = sf.MG(Ls, 1.0, 1.0)
        sms = timed(lambda: sf.sf_fcycle(Ms.handle), 3, warm=1)
        out["fcycle_strong"] = {"global": [n, n, n], "ms": sms, "dof_s": n**3 / (sms / 1e3),
                                "note": "C4: one F-cycle of the global problem in z-slabs over "
                                        "the ranks (strong scaling; max over ranks)"}
        Ms.close()
        Ls.close()
        torch.cuda.empty_cache()
    else:
        out["fcycle_strong"] = {"global": [nx, ny, nz], "ms": fms, "dof_s": dof_local * world / (fms / 1e3),
                                "note": "C4 at N = 1: the fcycle line"}
    # read-dominated bandwidth (PAPER.md:684-696's dot-product bound): L2 norm of u
    # (8 B/cell, read-only); each call ends with an 8-byte D2H and a host sync
    rms = timed(lambda: sf.sf_norm(L.handle, sf.SF_U, sf.SF_NORM_L2), 10, warm=2)
    out["read_bw"] = {"ms": rms, "gbs": 8 * dof_local / (rms / 1e3) / 1e9,
                      "kernel": "norm_pair_kernel (sum of squares, 8 B/cell read)",
                      "note": "includes per-call host sync; context for the copy peak"}
    # Fig 7's CC operators (NEXT-2) at the workload's finest level as well
    # (PAPER.md:698-784 quote them at 256^3 only; gsrb_c3 / fig7_256 below)
    if rank == 0 and world == 1:
        pk, _ = peaks()
        fig7b = {}
        for name, fn, bpc in (
                ("cc_7pt_laplacian", lambda: sf.sf_apply_laplacian(L.handle, sf.SF_R, sf.SF_U), 16),
                ("cc_jacobi_w2/3", lambda: sf.sf_jacobi(L.handle, sf.SF_R, sf.SF_U, sf.SF_F,
                                                         2.0 / 3.0), 24)):
            m_ = timed(fn, 20, warm=3)
            fig7b[name] = {"ms": m_, "gstencil_s": dof_local / (m_ / 1e3) / 1e9,
                           "alg_gbs": bpc * dof_local / (m_ / 1e3) / 1e9,
                           "frac_of_peak": bpc * dof_local / (m_ / 1e3) / 1e9 / pk,
                           "bytes_per_cell": bpc}
        out[f"fig7_{nx}"] = fig7b
    # pairs on the finest level per solve: F: (pre+post) ; each V: 4 pairs
    pairs_per_solve = 4 * cyc
    out["fine_pair_share"] = None

    # e2e: through the C ABI with host buffers (pinned): every step copies its
    # f host->device and its u device->host; sf_solve_stream overlaps the copies
    # of the neighbouring steps with each solve (the serving path)
    host_f = torch.empty(L.host_shape(sf.SF_F), dtype=torch.float64, pin_memory=True)
    host_u = [torch.empty(L.host_shape(sf.SF_U), dtype=torch.float64, pin_memory=True)
              for _ in range(2)]
    L.download(sf.SF_F, host_f.numpy())
    nb = host_f.numel() * 8
    # right-hand sides per streamed call: the timed region's K steps (fill and
    # drain -- the first upload, the last download -- amortised over them)
    reps = max(2, min(args.steps, 32))
    M.solve_stream([host_f] * 2, host_u)          # warm-up (staging allocation paths)
    barrier()
    t0 = time.perf_counter()
    M.solve_stream([host_f] * reps, [host_u[k % 2] for k in range(reps)])
    barrier()
    te = max_over_ranks((time.perf_counter() - t0) / reps)
    h2d_ms, solve_ms, d2h_ms, wall_ms = sf.sf_solve_stream_stats(M.handle)
    # the same, one step at a time with no overlap (upload, solve, download)
    def e2e_step():
        sf.sf_level_upload(L.handle, sf.SF_F, host_f.data_ptr())
        sf.sf_solve(M.handle, True, 1e-10, 50)
        sf.sf_level_download(L.handle, sf.SF_U, host_u[0].data_ptr())
    barrier()
    t1 = time.perf_counter()
    for _ in range(2):
        e2e_step()
    barrier()
    ts = max_over_ranks((time.perf_counter() - t1) / 2)
    out["e2e"] = {"value": dof_local * world / te, "unit": "DOF/s", "h2d_bytes_per_step": nb,
                  "d2h_bytes_per_step": nb, "ms_per_step": te * 1e3, "steps": reps,
                  "how": "sf_solve_stream over `steps` right-hand sides from pinned host memory: "
                         "H2D of f[k+1] and D2H of u[k-1] overlap solve k (wall clock, host "
                         "timer, incl. pipeline fill and drain)",
                  "serial_ms_per_step": ts * 1e3,
                  "serial_value": dof_local * world / ts,
                  "phases_ms": {"h2d_f": h2d_ms, "solve_incl_pack": solve_ms, "d2h_u": d2h_ms,
                                "wall_per_rhs": wall_ms,
                                "how": "CUDA events on the H2D, level and D2H streams inside "
                                       "sf_solve_stream (sf_solve_stream_stats), rank 0"}}

    # BASELINE config 3: 256^3 GSRB smoother throughput (rank 0's GPU only)
    if rank == 0:
        n3 = args.gsrb_n
        G = sf.Level(n3, n3, n3, 1.0 / n3)
        sf.sf_init_problem(G.handle, 1, 1.0, 1.0, 1)
        sf.sf_rebuild_operator(G.handle, 1.0, 1.0)
        s = G.stream

        def pair():
            sf.sf_smooth_gsrb(G.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
        for _ in range(10):
            pair()
        s.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        for _ in range(100):
            pair()
        b.record(s)
        s.synchronize()
        ms = a.elapsed_time(b) / 100
        cells = n3**3
        pk, _ = peaks()
        gbs = GSRB_BYTES_PER_CELL * cells / (ms / 1e3) / 1e9
        # colour (unfused) sweeps for comparison
        def pair_c():
            sf.sf_smooth_gsrb(G.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_COLOUR)
        for _ in range(3):
            pair_c()
        a.record(s)
        for _ in range(20):
            pair_c()
        b.record(s)
        s.synchronize()
        msc = a.elapsed_time(b) / 20
        # Fig 7 analogue: the paper's three operators at 256^3,
        # GPU algorithmic bytes (no write-allocate): CC 7pt 16 B, CC Jacobi 24 B,
        # VC GSRB 64 B per cell per RB pair (paper's write-allocate counts: 24/40/64)
        def per_call(fn, reps=50):
            for _ in range(5):
                fn()
            s.synchronize()
            a.record(s)
            for _ in range(reps):
                fn()
            b.record(s)
            s.synchronize()
            return a.elapsed_time(b) / reps
        fig7 = {}
        for name, fn, bpc in (
                ("cc_7pt_laplacian", lambda: sf.sf_apply_laplacian(G.handle, sf.SF_R, sf.SF_U), 16),
                ("cc_jacobi_w2/3", lambda: sf.sf_jacobi(G.handle, sf.SF_R, sf.SF_U, sf.SF_F,
                                                         2.0 / 3.0), 24)):
            m_ = per_call(fn)
            fig7[name] = {"ms": m_, "gstencil_s": cells / (m_ / 1e3) / 1e9,
                          "alg_gbs": bpc * cells / (m_ / 1e3) / 1e9,
                          "frac_of_peak": bpc * cells / (m_ / 1e3) / 1e9 / pk, "bytes_per_cell": bpc}
        fig7["vc_gsrb_pair"] = {"ms": ms, "gstencil_s": cells / (ms / 1e3) / 1e9, "alg_gbs": gbs,
                                "frac_of_peak": gbs / pk, "bytes_per_cell": 64}
        # NEXT-3 Chebyshev step (72 B/cell: x, x_prev, rhs, alpha, beta x3, Dinv, out)
        lam = sf.sf_lambda_max(G.handle, sf.SF_TMP, 1.0, 1.0, 10, True)
        mc = per_call(lambda: sf.sf_smooth_chebyshev(G.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1,
                                                     0.13 * lam, 1.05 * lam), 30)
        fig7["vc_chebyshev_step"] = {"ms": mc, "gstencil_s": cells / (mc / 1e3) / 1e9,
                                     "alg_gbs": 72 * cells / (mc / 1e3) / 1e9,
                                     "frac_of_peak": 72 * cells / (mc / 1e3) / 1e9 / pk,
                                     "bytes_per_cell": 72}
        out["fig7_256"] = fig7
        # Fig 8 analogue: fused RB pair throughput vs level size
        sweep = {}
        for n_ in (32, 64, 128):
            Gs = sf.Level(n_, n_, n_, 1.0 / n_, stream=s)
            sf.sf_init_problem(Gs.handle, 1, 1.0, 1.0, 1)
            sf.sf_rebuild_operator(Gs.handle, 1.0, 1.0)
            m_ = per_call(lambda: sf.sf_smooth_gsrb(Gs.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1,
                                                    sf.SF_SMOOTH_FUSED), 200)
            sweep[str(n_)] = {"ms": m_, "gstencil_s": n_**3 / (m_ / 1e3) / 1e9,
                              "alg_gbs": 64 * n_**3 / (m_ / 1e3) / 1e9}
            Gs.close()
        sweep[str(n3)] = {"ms": ms, "gstencil_s": cells / (ms / 1e3) / 1e9, "alg_gbs": gbs}
        out["gsrb_size_sweep"] = sweep
        # NEXT-4: the generic engine's JIT kernels for the same operators (the
        # paper's DSL path): Fig 4's RB pair and A3, rendered + NVRTC-compiled
        from paper_conf_ipps_zhangdmwbf17_b200 import stencil as SD
        hh = 1.0 / n3
        dpair = SD.hpgmg_gsrb_pair(1.0, 1.0, hh).compile()
        dop = SD.hpgmg_apply_op(1.0, 1.0, hh).compile()
        md = per_call(lambda: dpair(G), 20)
        mo = per_call(lambda: dop(G), 20)
        out["dsl_256"] = {
            "gsrb_pair_ms": md, "gsrb_pair_launches": dpair.phases,
            "gsrb_pair_alg_gbs": 2 * 64 * cells / (md / 1e3) / 1e9,
            "gsrb_pair_frac_of_peak": 2 * 64 * cells / (md / 1e3) / 1e9 / pk,
            "vs_handwritten_colour_sweeps": msc / md, "vs_fused_pair": ms / md,
            "apply_op_ms": mo, "apply_op_alg_gbs": 48 * cells / (mo / 1e3) / 1e9,
            "apply_op_frac_of_peak": 48 * cells / (mo / 1e3) / 1e9 / pk,
            "note": "JIT (NVRTC sm_100a) kernels of the generic stencil engine; basis 64 B/cell "
                    "per colour sweep (2 per pair) and 48 B/cell for A3"}
        dpair.close()
        dop.close()
        out["gsrb_c3"] = {"n": n3, "ms_per_rb_pair": ms,
                          "frac_of_kernel_compulsory": GSRB_KERNEL_BYTES_PER_CELL * cells / (ms / 1e3)
                          / 1e9 / pk,
                          "gstencil_s": 2 * cells / 2 / (ms / 1e3) / 1e9,
                          "point_updates_per_s": cells / (ms / 1e3),
                          "alg_gbs": gbs, "frac_of_peak": gbs / pk,
                          "colour_sweeps_ms_per_rb_pair": msc,
                          "note": "GStencil/s = point updates/s (each cell updated once per pair)"}
        G.close()
        # BASELINE configs 1 and 2 (parity configs; latency-bound, timed for context):
        # C1 16^3 CC Poisson, 2 RB pairs (4 sweeps) + residual; C2 64^3 VC Helmholtz,
        # V-cycle solve from u = 0 to 1e-10 (one graph launch, device-side loop)
        import numpy as np
        from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I
        G1 = sf.Level(16, 16, 16, 1.0 / 16, stream=s)
        G1.set_coeffs(*I.constant_coeffs(16, 16, 16))
        sf.sf_rebuild_operator(G1.handle, 0.0, 1.0)

        def c1():
            sf.sf_smooth_gsrb(G1.handle, sf.SF_U, sf.SF_F, 0.0, 1.0, 2)
            sf.sf_residual(G1.handle, sf.SF_R, sf.SF_U, sf.SF_F, 0.0, 1.0)
        m1 = per_call(c1, 200)
        G1.close()
        G2 = sf.Level(64, 64, 64, 1.0 / 64, stream=s)
        sf.sf_init_problem(G2.handle, 1, 1.0, 1.0, 1)
        M2 = sf.MG(G2, 1.0, 1.0)
        zeros = torch.zeros((64, 64, 64), dtype=torch.float64, pin_memory=True)

        def c2u():   # pinned u = 0: the upload is an async copy on the solve's stream
            G2.upload_async(sf.SF_U, zeros.data_ptr())
            return sf.sf_solve(M2.handle, False, 1e-10, 50)

        def c2():    # u = 0 set on the device (sf_level_zero), then the solve
            sf.sf_level_zero(G2.handle, sf.SF_U)
            return sf.sf_solve(M2.handle, False, 1e-10, 50)

        def wall(fn):
            fn()
            s.synchronize()
            t2 = time.perf_counter()
            for _ in range(20):
                r = fn()
            return (time.perf_counter() - t2) / 20 * 1e3, r
        m2u, _ = wall(c2u)
        m2, (_, cyc2, hist2) = wall(c2)
        ue2, _ = I.manufactured(64, 64, 64, 1.0, 1.0, 1.0 / 64)
        err2 = float(np.abs(G2.download(sf.SF_U) - ue2).max())
        rho = (hist2[-1] / hist2[0]) ** (1.0 / max(1, len(hist2) - 1)) if len(hist2) > 1 else None
        M2.close()
        G2.close()
        out["c1_16"] = {"ms": m1, "what": "2 RB pairs + residual, 16^3 CC Poisson (event-timed)"}
        out["c2_64"] = {"ms_per_solve": m2, "cycles": cyc2, "final_relres": hist2[-1],
                        "mean_rho": rho, "max_err_vs_manufactured": err2,
                        "what": "64^3 VC Helmholtz V-cycle solve from u = 0 to 1e-10 (wall clock: "
                                "sf_level_zero(U) + sf_solve incl. its host sync)",
                        "ms_per_solve_upload": m2u,
                        "what_upload": "the same with u = 0 uploaded from pinned host memory "
                                       "(2 MiB H2D) instead of zeroed on the device"}
        if world == 1 and not args.no_cpu_baseline:
            # one measured oracle solve of the workload itself (512^3: ~25 s on
            # 16 cores) when the host has the memory, else the 256^3 sample
            shp = (nx, ny, nz) if host_memory_allows((nx, ny, nz)) else REFERENCE_SAMPLE
            smp = OracleSolver(shp)
            t_s, cyc_o, rr_o = smp.solve_seconds()
            cells_o = shp[0] * shp[1] * shp[2]
            out["cpu_baseline"] = {
                "value": cells_o / t_s, "unit": "DOF/s", "cores": smp.cores, "kind": "oracle",
                "cpu_model": cpu_model(), "sample_shape": list(shp), "cycles": cyc_o,
                "seconds": t_s,
                "sample": f"{smp.desc}: {cyc_o} cycles, final relres {rr_o:.2e}, {t_s:.2f} s "
                          f"(measured, not extrapolated)"}
            del smp
    out["fine_pair_share"] = (4 * (cyc - 1) + 4 * 1) * fine_pair / (
        (out["vcycle"]["ms"]) * (F_OVER_V + cyc - 1)) if fine_pair else None
    return out


if __name__ == "__main__":
    main()
