#!/usr/bin/env python
"""bench.py — ensemble execution on B200: instances/s, lookups/s, HBM roofline.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload C2|C2U|TSTAR|C1|C3|C4|C5] [--no-extras]

One step = one pass of the whole hot path over one
batch: every instance of the workload launched as ONE persistent ensemble
kernel per app (device-resident args: ens_run_relaunch), plus, for N > 1,
the NCCL all-gather of the per-instance records.  The default workload is
BASELINE.json configs[1] (C2: 64 XSBench-style large instances per GPU, the
paper's 64-instance point); weak scaling: every rank runs 64 instances of a
64*N-line args file sharded by instance id (i mod N).

`e2e` times the same through the public C ABI from HOST buffers each step:
ens_launch (pinned H2D of the args) + ens_collect (D2H of records, tallies,
stdout).  `--impl reference` times the CPU oracle (test infrastructure, the
one other place this script runs it) on the box's host cores.
Timing: W warm-up steps, then K steps bracketed by barrier +
cuda.synchronize, CUDA events on the launching stream, max over ranks.
"""
import argparse
import json
import os
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "instances/sec and lookups/sec per ensemble launch at 1/2/4/8 B200; HBM GB/s vs peak"
FALLBACK_HBM_GBS = 6650.0

# algorithmic bytes.  XS lookup: 16-B bracket + per nuclide
# a 4-B index entry and the 96-B bracketing record pair.
XS_NUM_NUCS = {68: [34, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9], 355: [321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]}


def parse_xs_line(line):
    t = line.split()
    p = {"n_iso": 355, "n_gp": 11303, "L": 17000000, "grid": "unionized", "bins": 10000}
    for i in range(1, len(t) - 1, 2):
        f, v = t[i], t[i + 1]
        if f == "-s":
            p["n_iso"] = 68 if v == "small" else 355
        elif f == "-g":
            p["n_gp"] = int(v)
        elif f == "-l":
            p["L"] = int(v)
        elif f == "-G":
            p["grid"] = v
        elif f == "-h":
            p["bins"] = int(v)
    return p


def xs_init_bytes(p):
    """Per-instance init: 48 n_u grid (+ unionized 8 n_u union + 8 n_u merge + 4 n_u n_iso index,
    or hash 4 n_iso bins) — the bytes the method must write."""
    n_u = p["n_iso"] * p["n_gp"]
    b = 48 * n_u
    if p["grid"] == "unionized":
        b += 8 * n_u + 8 * n_u + 4 * n_u * p["n_iso"]
    elif p["grid"] == "hash":
        b += 4 * p["n_iso"] * p["bins"]
    return b


def xs_lookup_bytes(n_iso, mat_counts):
    nn = XS_NUM_NUCS[n_iso]
    return sum(int(c) * (16 + 100 * nn[m]) for m, c in enumerate(mat_counts))


def algorithmic_bytes(lines, recs, tallies):
    """Exact algorithmic bytes of one launch: per-instance init + per-lookup bytes from the
    per-instance material tallies (XS).  Other apps: SURVEY.md §8(d) per-unit figures."""
    total = 0
    for k, line in enumerate(lines):
        app = line.split()[0]
        if app == "xsbench" and recs[k]["exit_code"] == 0:
            p = parse_xs_line(line)
            total += xs_init_bytes(p) + xs_lookup_bytes(p["n_iso"], tallies[k][5:17])
        elif app == "amgmk" and recs[k]["exit_code"] == 0:
            t = line.split()
            d = {t[i]: t[i + 1] for i in range(1, len(t) - 1, 2)}
            nx, ny, nz = int(d.get("-x", 50)), int(d.get("-y", 50)), int(d.get("-z", 50))
            it = int(d.get("-i", 100))
            n = nx * ny * nz
            nnz = 7 * n - 2 * (nx * ny + ny * nz + nx * nz)
            total += it * (12 * nnz + 4 * (n + 1) + 24 * n) + 12 * nnz + 32 * n
    return total


# RS-3 algorithmic FP64 work, counted from the formulas as written (each +, -, *, /, sqrt, sin,
# cos, atan = 1 op; complex ops expanded textbook-style: c_mul 6, c_div 11, c_add/c_sub 2):
# per nuclide visited: window 2, sigT factors 41, background 3, sigE 1, macro 8 = 55;
# per pole term: doppler |Z| >= 6 (asymptotic) 76, doppler |Z| < 6 (Abrarov, 11 cexp) 766,
# no doppler 43.  Bytes: 64-B pole + 1-B l per term, 32-B window + 32-B K0RS per nuclide.
RS_FLOPS_NUC, RS_FLOPS_FAR, RS_FLOPS_NEAR, RS_FLOPS_NODOPP = 55, 76, 766, 43
RS_BYTES_TERM, RS_BYTES_NUC = 65, 64


def rs_work(lines, recs, tallies):
    """(algorithmic FP64 ops, algorithmic bytes) of the RS instances of one launch, from the
    per-instance work counters (tallies[24..26]: pole terms, Abrarov-branch terms) and material
    tallies (nuclides visited)."""
    flops = byts = 0
    for k, line in enumerate(lines):
        t = line.split()
        if t[0] != "rsbench" or recs[k]["exit_code"] != 0:
            continue
        n_nuc = 355 if ("-s" in t and t[t.index("-s") + 1] == "large") else 68
        nn = XS_NUM_NUCS[n_nuc]
        tal = tallies[k]
        nucs = sum(int(tal[5 + m]) * nn[m] for m in range(12))
        terms = int(tal[24]) | (int(tal[25]) << 32)
        near = int(tal[26])
        if "-d" in t:
            f_terms = RS_FLOPS_NODOPP * terms
        else:
            f_terms = RS_FLOPS_FAR * (terms - near) + RS_FLOPS_NEAR * near
        flops += RS_FLOPS_NUC * nucs + f_terms
        byts += RS_BYTES_NUC * nucs + RS_BYTES_TERM * terms
    return flops, byts


def measured_peak_fp64():
    """FP64 FLOP/s (DFMA = 2) measured now by the DFMA microbenchmark (csrc/tools/fp64_peak.cu)."""
    import ctypes
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_icppw_tiancd23_b200", "libens_tools.so"))
    fl, ms = ctypes.c_double(), ctypes.c_float()
    rc = lib.ens_tool_fp64_peak(None, 5, ctypes.byref(fl), ctypes.byref(ms))
    if rc != 0:
        raise RuntimeError(f"fp64 peak microbenchmark failed: cuda error {rc}")
    return fl.value


def measured_peak_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for l in self.proc.stdout:
            self.lines.append(l.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in self.lines:
            f = [x.strip() for x in l.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        sm.sort()
        med = sm[len(sm) // 2] if sm else None
        return {"sm_mhz": med, "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def workload_lines(name, world):
    from paper_conf_icppw_tiancd23_b200 import workloads as W
    if name == "C2":
        return W.c2(64 * world), "C2: 64 x XSBench-style large (355 nuclides, 11303 gridpoints, hash 10000 bins, " \
                                 "1M lookups) per GPU, distinct seeds; weak scaling by instance id"
    if name == "C2U":
        lines = [l.replace("-G hash -h 10000", "-G unionized") for l in W.c2(24 * world)]
        return lines, "C2u: 24 x XSBench-style large unionized (5.92 GB of tables each; 1M lookups) per GPU"
    if name == "TSTAR":
        return W.tstar(1024 * world), "TSTAR: 1024 x XSBench-style small (68 nuclides, 1000 gridpoints, unionized, " \
                                      "10k lookups) per GPU"
    if name == "C1":
        return W.c1(4 * world), "C1: 4 x XSBench-style small (1000 gridpoints, 10k lookups) per GPU"
    if name == "C3":
        return W.c3(256 * world), "C3: 256 x RSBench-style small, varied args, per GPU"
    if name == "C4":
        return W.c4(1024 * world), "C4: 1024 x AMGmk-style 32^3 Jacobi relax (20 sweeps) per GPU, T=1024"
    if name == "C5":
        return W.c5(4096 * world), "C5: 4096 mixed (XS/XS/RS/AMG) per GPU, sharded by instance id"
    raise SystemExit(f"unknown workload {name}")


THREADS = {"C2": 512, "C2U": 512, "TSTAR": 512, "C1": 256, "C3": 256, "C4": 1024, "C5": 1024}


def time_ours(lines, world, rank, threads, steps, warmup, torch, dist_on, team_ctas=0):
    """Device-resident timing of the ensemble (relaunch) + NCCL all-gather for world > 1."""
    from paper_conf_icppw_tiancd23_b200 import Args, workloads
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    from paper_conf_icppw_tiancd23_b200 import dist as D
    args = Args.parse(workloads.text(lines))
    n_total = len(lines)
    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        ens = Ensemble(args, app="auto", first=rank, stride=world, threads=threads, stream=stream,
                       team_ctas=team_ctas).launch()
    stream.synchronize()
    gather_rows = D.padded_count(n_total, world)
    out_buf = None

    def step():
        ens.relaunch()
        if dist_on:
            with torch.cuda.stream(stream):
                D.all_gather_rows(ens.device_records(), gather_rows)

    for _ in range(warmup):
        step()
    stream.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    if dist_on:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    t_all0 = torch.cuda.Event(enable_timing=True)
    t_all1 = torch.cuda.Event(enable_timing=True)
    t_all0.record(stream)
    for i in range(steps):
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
    t_all1.record(stream)
    torch.cuda.synchronize()
    if dist_on:
        torch.distributed.barrier()
    total_ms = t_all0.elapsed_time(t_all1)
    per_ms = [a.elapsed_time(b) for a, b in ev]
    res = ens.collect()
    info = ens.info()
    return ens, res, info, total_ms, per_ms, out_buf


def time_e2e(lines, world, rank, threads, steps, torch, dist_on):
    """The public C ABI from host buffers: ens_launch (args H2D from pinned host
    memory) + ens_collect (records, tallies and stdout D2H, stdout formatted on
    the host) for every step.  When two workspaces fit in HBM, two steps are in
    flight: step s+1 is launched before step s is collected (ens_collect waits
    for its own run only), so the host-side collect of one step overlaps the
    next step's kernels, as a user streaming ensembles through the API would."""
    from paper_conf_icppw_tiancd23_b200 import Args, workloads, _ens
    args = Args.parse(workloads.text(lines))
    n_local = len(range(rank, len(lines), world))
    cfg = _ens.make_cfg(n_local, first=rank, stride=world, threads=threads)
    ws = _ens.workspace_bytes("auto", args, cfg)
    free, _ = torch.cuda.mem_get_info()
    depth = 2 if 2 * ws + (2 << 30) <= free else 1
    bufs = [torch.empty(ws, dtype=torch.uint8, device="cuda") for _ in range(depth)]
    stream = torch.cuda.current_stream().cuda_stream

    def launch(s):
        b = bufs[s % depth]
        return _ens.Run.launch("auto", args, cfg, b.data_ptr(), ws, stream, keep=b)

    ref = []

    def finish(run):
        out = run.collect()
        i = run.info()
        run.close()
        got = out.records[["instance", "exit_code", "vhash", "bitsum"]]
        if ref and not (got == ref[0]).all():  # every step computes the same, in flight or not
            raise RuntimeError("e2e: a step's records differ from the first step's")
        return out, i

    ref.append(finish(launch(0))[0].records[["instance", "exit_code", "vhash", "bitsum"]])  # warm
    torch.cuda.synchronize()
    if dist_on:
        torch.distributed.barrier()
    t0 = time.perf_counter()
    inflight = []
    for s in range(steps):
        inflight.append(launch(s))
        if len(inflight) == depth:
            out, i = finish(inflight.pop(0))
    while inflight:
        out, i = finish(inflight.pop(0))
    dt = time.perf_counter() - t0
    h2d = int(i.h2d_bytes)
    d2h = int(i.d2h_bytes)
    return dt / steps, h2d, d2h, depth


# host memory per oracle instance caps the sample: a large unionized XS instance holds 5.9 GB
ORACLE_MAX_INSTANCES = {"C2U": 1}


def cpu_oracle_sample(lines, budget_s=20.0, max_instances=None, cap=None):
    """The oracle as it stands on this host: a bounded sample of the workload's instances —
    the first k lines, one per core, k grown x4 while a pass takes under budget_s / 8."""
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import oracle_lib
    oracle_lib.build()
    cores = os.cpu_count() or 1
    k = max(1, min(max_instances or cores, len(lines)))
    cap = cap or len(lines)
    while True:
        t0 = time.perf_counter()
        r = oracle_lib.run_text("".join(l + "\n" for l in lines[:k]), jobs=min(cores, k))
        dt = time.perf_counter() - t0
        if dt >= budget_s / 8 or k >= min(len(lines), cap):
            break
        k = min(len(lines), cap, 4 * k)
    work = int(r.records["work"].sum())
    return {"instances": k, "seconds": dt, "cores": min(cores, k), "work": work}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="C2")
    ap.add_argument("--no-extras", action="store_true", help="skip the TSTAR / solo side measurements")
    ap.add_argument("--threads", type=int, default=0, help="thread limit per team (default: per workload)")
    a = ap.parse_args()
    world, rank, local = dist_env()
    if a.gpus != world and world == 1:
        world_note = f"--gpus {a.gpus} without torchrun: running 1 process"
    else:
        world_note = None
    lines, wl_desc = workload_lines(a.workload, world)
    threads = a.threads or THREADS.get(a.workload, 256)
    n_local = len(range(rank, len(lines), world))
    config = {"workload": wl_desc, "instances_per_gpu": n_local, "instances_total": len(lines),
              "block_threads": threads, "l2": "inputs larger than L2 (per-instance tables >> 126 MB in total)",
              "parallelism": f"instances sharded i mod {world}"}
    if a.impl == "reference":
        if rank != 0:
            return
        cores = os.cpu_count() or 1
        per = []
        for s in range(a.steps):
            r = cpu_oracle_sample(lines, max_instances=min(cores, len(lines), 16, ORACLE_MAX_INSTANCES.get(a.workload, 16)),
                                  cap=ORACLE_MAX_INSTANCES.get(a.workload))
            per.append(r)
        inst = sum(r["instances"] for r in per)
        sec = sum(r["seconds"] for r in per)
        v = inst / sec
        line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "instances/s", "n_gpus": a.gpus,
                "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * sec / a.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": config,
                "cpu_baseline": {"value": v, "unit": "instances/s", "cores": per[0]["cores"], "kind": "oracle",
                                 "sample": f"first {per[0]['instances']} instances of the workload per step, "
                                           f"full size, on {per[0]['cores']} host threads"},
                "e2e": {"value": v, "unit": "instances/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
                "lookups_per_s": sum(r["work"] for r in per) / sec}
        print(json.dumps(line), flush=True)
        return

    import torch
    dist_on = world > 1
    if dist_on:
        torch.cuda.set_device(local)
        torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    sampler = ClockSampler(local)
    sampler_started = False

    ens, res, info, total_ms, per_ms, _ = None, None, None, None, None, None
    # timed region (clocks sampled during it)
    sampler.start()
    sampler_started = True
    ens, res, info, total_ms, per_ms, _ = time_ours(lines, world, rank, threads, a.steps, max(3, a.warmup), torch,
                                                    dist_on)
    clocks = sampler.stop()
    ms = total_ms / a.steps
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if dist_on:
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    ms_max = float(t.item())
    local_lines = lines[rank::world]
    algo = algorithmic_bytes(local_lines, res.records, res.tallies)
    rs_flops, rs_bytes = rs_work(local_lines, res.records, res.tallies)
    algo += rs_bytes
    kern_ms = sum(per_ms) / len(per_ms)
    peak, peak_kind = measured_peak_hbm()
    achieved = algo / (kern_ms * 1e-3) / 1e9
    fp64 = None
    if rs_flops:
        fp64_peak = measured_peak_fp64() / 1e12
        fp64 = {"achieved": rs_flops / (kern_ms * 1e-3) / 1e12, "peak": fp64_peak, "unit": "TFLOP/s",
                "frac": rs_flops / (kern_ms * 1e-3) / 1e12 / fp64_peak, "algorithmic_flops_per_launch": rs_flops,
                "peak_kind": "measured now: DFMA microbenchmark (csrc/tools/fp64_peak.cu), DFMA = 2 FLOP; the "
                             "RS body is built --fmad=false, so its mul/add arithmetic issues 1 FLOP per DP "
                             "instruction and tops out at half of this"}
    lookups_local = int(res.records["work"].sum())
    tt = torch.tensor([lookups_local, algo], dtype=torch.float64, device="cuda")
    if dist_on:
        torch.distributed.all_reduce(tt)
    lookups_total = float(tt[0].item())
    ok = bool((res.records["exit_code"] == 0).all())

    # e2e through the C ABI from host buffers (the device-resident ensemble's
    # workspace is released first: both would not fit for C2U's 145 GB)
    info_kl, info_bt, info_gb, info_tc = (int(info.kernel_launches), max(info.block_threads), max(info.grid_blocks),
                                          max(info.team_ctas))
    ens.close()
    ens = None
    torch.cuda.empty_cache()
    e2e_s, h2d, d2h, e2e_depth = time_e2e(lines, world, rank, threads, max(2, min(a.steps, 5)), torch, dist_on)
    te = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
    if dist_on:
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
    e2e_s = float(te.item())

    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(a.workload)
        except Exception:
            traffic = None

    extras = {}
    if not a.no_extras and world == 1 and a.workload == "C2":
        # the paper's metric T1*N/TN: solo run of line 0 (N=1), same T;
        # T1 on one CTA (the paper's team = one thread block) and on
        # the auto team (a cluster of up to 8 CTAs for a lone instance)
        solo_ens, _, _, solo_ms, _, _ = time_ours(lines[:1], 1, 0, threads, 2, 1, torch, False, team_ctas=1)
        solo_ens.close()
        solo2_ens, _, _, solo2_ms, _, _ = time_ours(lines[:1], 1, 0, threads, 2, 1, torch, False)
        solo2_ens.close()
        extras["speedup_vs_solo"] = {"T1_ms": solo_ms / 2, "TN_ms": ms, "N": len(lines),
                                     "value": (solo_ms / 2) * len(lines) / ms,
                                     "T1_cluster_team_ms": solo2_ms / 2,
                                     "value_vs_cluster_team_T1": (solo2_ms / 2) * len(lines) / ms,
                                     "paper_context": "51x at 64 instances on A100 40GB (P:44-45, P:639-640)"}
        # XSBench's own convention times the lookup phase alone: the same launch with
        # ENS_F_PHASES tracing gives each team's device time in the lookup phases
        # (sample+sort, gathers); every team runs one instance concurrently here
        from paper_conf_icppw_tiancd23_b200 import Args as _Args, workloads as _W
        from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble as _Ens
        pe = _Ens(_Args.parse(_W.text(lines)), app="auto", threads=threads, phases=True).launch()
        torch.cuda.synchronize()
        pe.relaunch()
        torch.cuda.synchronize()
        ph = pe.run.phases_ns()
        pinfo = pe.info()
        teams = max(1, max(pinfo.grid_blocks) // max(1, max(pinfo.team_ctas)))
        lk_ms = (ph[10] + ph[11]) / teams / 1e6
        in_ms = sum(ph[k] for k in range(10)) / teams / 1e6
        pe.close()
        extras["phases_per_team_ms"] = {"init": in_ms, "lookups": lk_ms,
                                        "lookup_phase_rate": lookups_total / (lk_ms * 1e-3),
                                        "note": "XSBench convention (lookup phase only), from ENS_F_PHASES tracing "
                                                "of one warm launch: lookups / mean team lookup-phase time"}
        # north-star target launch: >= 1024 XSBench-style instances per B200 at >= 60% HBM
        tl, _ = workload_lines("TSTAR", 1)
        t_ens, t_res, t_info, t_ms, t_per, _ = time_ours(tl, 1, 0, THREADS["TSTAR"], 5, 3, torch, False)
        t_algo = algorithmic_bytes(tl, t_res.records, t_res.tallies)
        t_k = sum(t_per) / len(t_per)
        extras["tstar"] = {"instances": len(tl), "ms_per_launch": t_k, "instances_per_s": len(tl) / (t_k * 1e-3),
                           "lookups_per_s": float(t_res.records["work"].sum()) / (t_k * 1e-3),
                           "algorithmic_bytes": t_algo, "achieved_gbs": t_algo / (t_k * 1e-3) / 1e9,
                           "frac_of_hbm": t_algo / (t_k * 1e-3) / 1e9 / peak,
                           "parity_exit_ok": bool((t_res.records["exit_code"] == 0).all())}
        t_ens.close()

    if rank == 0:
        out = {"metric": METRIC, "value": len(lines) / (ms_max * 1e-3), "unit": "instances/s", "n_gpus": world,
               "steps": a.steps, "warmup": max(3, a.warmup), "ms_per_step": ms_max, "higher_is_better": True,
               "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": config,
               "lookups_per_s": lookups_total / (ms_max * 1e-3),
               "e2e": {"value": len(lines) / e2e_s, "unit": "instances/s", "h2d_bytes_per_step": h2d,
                       "d2h_bytes_per_step": d2h, "in_flight": e2e_depth},
               "gpu_launches": info_kl * a.steps,
               "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                            "frac": achieved / peak, "traffic": traffic, "peak_kind": peak_kind,
                            "dram_gbs": traffic / (kern_ms * 1e-3) / 1e9 if traffic else None,
                            "dram_frac": traffic / (kern_ms * 1e-3) / 1e9 / peak if traffic else None,
                            "kernel": f"ens_kernel<App,{info_bt}> x {info_gb} CTAs (team of {info_tc} CTAs)",
                            "algorithmic_bytes_per_launch": algo, "kernel_ms": kern_ms},
               "clocks": clocks, "all_exit_ok": ok}
        if fp64 is not None:
            hbm_part = {k: out["roofline"][k] for k in ("bound", "achieved", "peak", "unit", "frac")}
            if all(l.split()[0] == "rsbench" for l in local_lines):
                # RS-only launch: the FP64 pipe is the roofline (reading Q18)
                out["roofline"].update({"bound": "alu", "achieved": fp64["achieved"], "peak": fp64["peak"],
                                        "unit": "TFLOP/s", "frac": fp64["frac"], "peak_kind": fp64["peak_kind"],
                                        "algorithmic_flops_per_launch": rs_flops, "hbm": hbm_part})
            else:
                out["roofline"]["fp64"] = fp64
        if traffic and traffic < 0.5 * algo:
            out["roofline"]["note"] = (
                "algorithmic bytes (SURVEY 8(d): per lookup the XS bracket, index entries and record pairs, or "
                "the RS windows and poles) exceed the DRAM traffic ncu measures: lookups run in (material, "
                "energy)-sorted batches, so neighbouring lanes share entries, pairs and poles through L1/L2; "
                "dram_gbs is the HBM rate actually moved (profiles/ncu_*_r1*.txt)")
        if world_note:
            out["note"] = world_note
        if world == 1:
            cb = cpu_oracle_sample(lines, max_instances=min(os.cpu_count() or 1, 16, len(lines),
                                                             ORACLE_MAX_INSTANCES.get(a.workload, 16)),
                                   cap=ORACLE_MAX_INSTANCES.get(a.workload))
            out["cpu_baseline"] = {"value": cb["instances"] / cb["seconds"], "unit": "instances/s",
                                   "cores": cb["cores"], "kind": "oracle",
                                   "sample": f"first {cb['instances']} instances of the workload (full size) "
                                             f"on {cb['cores']} host threads, {cb['seconds']:.1f} s"}
        out.update(extras)
        print(json.dumps(out), flush=True)
    if ens is not None:
        ens.close()
    if dist_on:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
