"""Turn ncu output into the summaries committed under profiles/.

    python tools/ncu_summary.py launches <ncu --csv log> <out.json> "<command>"
        per-launch device times of `ncu --metrics gpu__time_duration.sum
        --clock-control none --csv ...` (cold-cache, serialised)
    python tools/ncu_summary.py counters <report.ncu-rep> <workload>
        per kernel of the capture: dram__bytes_read.sum + dram__bytes_write.sum and
        smsp__inst_executed.sum into profiles/ncu_counters.json[workload] (read by
        bench.py's roofline: the dram and issue candidates)
    python tools/ncu_summary.py full <report.ncu-rep> <out.txt> [workload]
        key counters of one `ncu --set full` capture + warp-stall samples by
        source line; with a workload name, also writes profiles/traffic.json
        (dram__bytes_read.sum + dram__bytes_write.sum per launch, read by
        bench.py as roofline.traffic)
"""
import collections
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__t_sector_hit_rate.pct",
    "lts__t_sector_hit_rate.pct", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_write.sum",
    "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread",
    "launch__shared_mem_per_block_dynamic", "launch__grid_size", "launch__block_size",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard", "smsp__pcsamp_warps_issue_stalled_wait",
    "smsp__pcsamp_warps_issue_stalled_barrier", "smsp__pcsamp_warps_issue_stalled_selected",
]

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def launches(log, out, command):
    text = open(log).read()
    start = text.find('"ID"')
    rows = list(csv.reader(io.StringIO(text[start:])))
    hdr = rows[0]
    i_id, i_k, i_g, i_b, i_n, i_u, i_v = (hdr.index(k) for k in ("ID", "Kernel Name", "Grid Size", "Block Size",
                                                                   "Metric Name", "Metric Unit", "Metric Value"))
    res = []
    for r in rows[1:]:
        if len(r) <= i_v or r[i_n] != "gpu__time_duration.sum":
            continue
        v = float(r[i_v].replace(",", ""))
        scale = {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "s": 1e9, "second": 1e9,
                 "nsecond": 1}.get(r[i_u], 1)
        res.append({"id": int(r[i_id]), "kernel": r[i_k], "grid": r[i_g], "block": r[i_b], "ns": v * scale})
    total = sum(x["ns"] for x in res) or 1.0
    by = collections.Counter()
    for x in res:
        by[x["kernel"]] += x["ns"]
    json.dump({"command": command, "note": "cold-cache serialised per-launch device times (ncu); compare shares, "
                                           "not absolute times, with the bench line",
               "share_by_kernel": {k: v / total for k, v in by.most_common()}, "launches": res},
              open(out, "w"), indent=1)
    print(f"{len(res)} launches -> {out}")


def summary_of(rep):
    """profiles/<report name>.txt: the committed summary of a capture (the .ncu-rep stays in gpurun_out/)."""
    return os.path.join("profiles", os.path.basename(rep).replace(".ncu-rep", ".txt"))


def _rx(name):
    """ncu --kernel-name regex for a kernel name of the raw page (short demangled form,
    e.g. `void ens_kernel<XsApp, 512>(KParams)`; the source page knows it as
    `ens::ens_kernel<ens::XsApp, (int)512>`): the identifier, then each template argument."""
    base = name.split("(")[0]
    if base.startswith("void "):
        base = base[5:]
    ident, _, targs = base.partition("<")
    rx = ident
    if targs:
        rx += "<" + "".join(".*" + re.escape(t.strip()) for t in targs.rstrip(">").split(",")) + ">"
    return "regex:" + rx


def full(rep, out, workload=None):
    """Every kernel of the capture: key counters, then warp-stall samples by source line."""
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units = rows[0], rows[1]
    lines, dom = [], None
    for vals in rows[2:]:
        d = {hdr[i]: (vals[i], units[i]) for i in range(len(hdr))}
        name = d.get("Kernel Name", ("?",))[0]
        lines += [f"kernel: {name}  grid {d.get('Grid Size', ('?',))[0]} block {d.get('Block Size', ('?',))[0]}",
                  "", "key counters (one launch):"]
        for k in KEYS:
            if k in d:
                lines.append(f"  {k:58s} {d[k][0]:>22s} {d[k][1]}")
        ms = float(d["gpu__time_duration.sum"][0].replace(",", "")) * {"ms": 1.0, "us": 1e-3, "usecond": 1e-3,
                                                                         "msecond": 1.0, "ns": 1e-6,
                                                                         "nsecond": 1e-6}.get(d["gpu__time_duration.sum"][1], 1.0)
        tb = sum(float(d[k][0].replace(",", "")) * UNIT.get(d[k][1], 1)
                 for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
        if dom is None or ms > dom[0]:
            dom = (ms, tb, name)
        src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                              "--kernel-name-base", "demangled", "--kernel-name", _rx(name)],
                             capture_output=True, text=True).stdout
        agg, tot, text, cur, hdr2 = collections.Counter(), 0, {}, None, None
        for r in csv.reader(src.splitlines()):
            if len(r) == 2 and r[0] == "File Path":
                cur = r[1].split("/")[-1]
                continue
            if r and r[0] == "Line No":
                hdr2 = r
                continue
            if hdr2 and len(r) >= 5 and r[0].isdigit():
                try:
                    x = int(r[4] or 0)
                except ValueError:
                    continue
                key = (cur, int(r[0]))
                agg[key] += x
                tot += x
                text[key] = r[1].strip()[:90]
        lines += ["", f"warp-stall samples by source line (top 20 of {tot}):"]
        for key, x in agg.most_common(20):
            lines.append(f"  {100.0 * x / max(tot, 1):5.1f}%  {key[0]}:{key[1]}  {text[key]}")
        lines += ["", ""]
    open(out, "w").write("\n".join(lines))
    print(f"-> {out}")
    if workload and dom:
        tp = os.environ.get("NCU_TRAFFIC", os.path.join(ROOT, "profiles", "traffic.json"))
        t = json.load(open(tp)) if os.path.exists(tp) else {}
        t[workload] = dom[1]
        t[f"_source_{workload}"] = (f"ncu --set full, {os.path.relpath(out, ROOT)}: dram__bytes_read.sum + "
                                    f"dram__bytes_write.sum of one launch of the longest kernel ({dom[2]})")
        t.pop("_source", None)
        json.dump(t, open(tp, "w"), indent=1)
        print(f"traffic[{workload}] = {dom[1]:.4g} B ({dom[2]}) -> {tp}")


APP_OF = {"EchoApp": 1, "XsApp": 2, "RsApp": 3, "AmgApp": 4, "PrApp": 5}


def kernel_key(name):
    """bench.py's key of a kernel: phase1_app<id> for ens_kernel<App,T>, phase2_kind<grid> for
    xs_items_kernel<grid>."""
    if "xs_init_items_kernel" in name:
        return "phase3_app2"
    if "rs_items_kernel" in name:
        return "phase2_kind3"
    m = re.search(r"xs_items_kernel<\(?i?n?t?\)?(\d)>", name)
    if m:
        return f"phase2_kind{m.group(1)}"
    for k, v in APP_OF.items():
        if k in name:
            return f"phase1_app{v}"
    return None


def counters(rep, workload):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,gpu__time_duration.sum,"
                          "l1tex__throughput.avg.pct_of_peak_sustained_active,"
                          "smsp__issue_active.avg.pct_of_peak_sustained_active"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units = rows[0], rows[1]
    out = {}
    for r in rows[2:]:
        d = {hdr[i]: (r[i], units[i]) for i in range(len(hdr))}
        key = kernel_key(d["Kernel Name"][0])
        if not key:
            continue
        tb = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            v, u = d[k]
            tb += float(v.replace(",", "")) * UNIT.get(u, 1)
        ms = float(d["gpu__time_duration.sum"][0].replace(",", ""))
        if d["gpu__time_duration.sum"][1] == "us":
            ms /= 1e3
        out[key] = {"dram_bytes": tb, "inst_executed": float(d["smsp__inst_executed.sum"][0].replace(",", "")),
                    "ncu_ms": ms, "kernel": d["Kernel Name"][0], "source": summary_of(rep)}
        for m, k in (("l1tex__throughput.avg.pct_of_peak_sustained_active", "l1tex_busy"),
                     ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active")):
            if m in d:
                out[key][k] = float(d[m][0].replace(",", "")) / 100.0
    p = os.environ.get("NCU_COUNTERS", os.path.join(ROOT, "profiles", "ncu_counters.json"))
    allc = json.load(open(p)) if os.path.exists(p) else {}
    allc[workload] = {"kernels": out, "note": "one ncu --set full capture of a warm launch (--clock-control none); "
                                              "per-launch counters, cold-cache serialised times"}
    json.dump(allc, open(p, "w"), indent=1)
    print(f"{workload}: {list(out)} -> {p}")


if __name__ == "__main__":
    if sys.argv[1] == "counters":
        counters(sys.argv[2], sys.argv[3])
        sys.exit(0)
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else "")
    else:
        full(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else None)
